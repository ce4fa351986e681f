# Experiment record: INL_SSSP_CARVEOUT (a uniform smem carveout for the SSSP loop kernels) was measured
# slower at every setting and removed from frontier.cu; this script no longer changes anything.
mkdir -p gpurun_out
B="python bench.py --no-e2e --no-cpu-baseline --no-context --op sssp --steps 9 --warmup 3"
o=gpurun_out/ab_carveout.txt; : > $o
for v in -1 0 25 50 100 -1 25; do
  if [ "$v" = "-1" ]; then r=$(timeout 300 $B 2>>gpurun_out/ab.err); else r=$(INL_SSSP_CARVEOUT=$v timeout 300 $B 2>>gpurun_out/ab.err); fi
  echo "carveout=$v $(echo "$r" | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])")" >> $o
done
for v in 25 100; do rm -f gpurun_out/tr_$v.txt; INL_SSSP_CARVEOUT=$v INL_SSSP_TRACE=gpurun_out/tr_$v.txt timeout 300 python scripts/sssp_steps.py > /dev/null 2>&1; done
