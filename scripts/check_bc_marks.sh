mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bc.py -q -x > gpurun_out/pytest_bc_marks.log 2>&1; echo rc=$? >> gpurun_out/pytest_bc_marks.log
o=gpurun_out/check_bc_marks.txt; : > $o
for i in 1 2; do for v in 1; do for sc in 20 22; do
  r=$(INL_BC_MARKS=$v timeout 300 python bench.py --no-e2e --no-cpu-baseline --no-context --op bc --scale $sc --steps 4 --warmup 3 2>>gpurun_out/check_bc_marks.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'])")
  echo "marks=$v scale $sc -> $r" >> $o
done; done; done
