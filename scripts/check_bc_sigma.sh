# Experiment record: INL_BC_SIGMA_PULL was measured 2x slower and removed from bc.cu.
mkdir -p gpurun_out
o=gpurun_out/check_bc_sigma.txt; : > $o
for sc in 20 22; do for v in 0 1 0 1; do
  r=$(INL_BC_SIGMA_PULL=$v timeout 300 python bench.py --no-e2e --no-cpu-baseline --no-context --op bc --scale $sc --steps 4 --warmup 3 2>>gpurun_out/check_bc.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'])")
  echo "scale $sc sigma_pull=$v -> $r" >> $o
done; done
INL_BC_SIGMA_PULL=1 timeout 900 python -m pytest tests/test_gpu_bc.py -q -x > gpurun_out/pytest_bc_sigma.log 2>&1; echo rc=$? >> gpurun_out/pytest_bc_sigma.log
