#!/bin/bash
# One bench line per environment variant: VARIANTS="A=1 B=2;C=3" OPARGS="--op spmv"
mkdir -p gpurun_out
out=gpurun_out/sweep.txt
: > $out
IFS=';' read -ra VS <<< "$VARIANTS"
for v in "${VS[@]}"; do
  r=$(env $v timeout 300 python bench.py --no-e2e --no-cpu-baseline $OPARGS 2>>gpurun_out/sweep_err.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'])")
  echo "[$v] $OPARGS -> $r" | tee -a $out
done
