#!/bin/bash
# SpMV tuning sweep on one GPU: hot-set size x bins.  One summary line per config.
mkdir -p gpurun_out
out=gpurun_out/tune_spmv.txt
: > $out
for hk in ${HOTK:-"32768" "24576" "16384" "0"}; do
  for bins in ${BINS:-"8,256,4096" "8,128,4096" "8,512,4096" "4,256,4096" "16,256,4096" "32,256,4096"}; do
    r=$(INL_HOT_K=$hk timeout 300 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --bins $bins 2>>gpurun_out/tune_err.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['achieved'], d['roofline']['frac'])")
    echo "hot=$hk bins=$bins $r" | tee -a $out
  done
done
