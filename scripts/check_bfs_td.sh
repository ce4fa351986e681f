mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sssp_bfs.py tests/test_gpu_fullsize.py -q -x > gpurun_out/pytest_bfs_td.log 2>&1; echo rc=$? >> gpurun_out/pytest_bfs_td.log
o=gpurun_out/check_bfs_td.txt; : > $o
for i in 1 2; do for v in red atomic; do
  for op in "--scale 26 --steps 8 --warmup 3" "--steps 9 --warmup 3"; do
    r=$(INL_BFS_TD=$v timeout 300 python bench.py --no-e2e --no-cpu-baseline --no-context --op bfs $op 2>>gpurun_out/check_bfs_td.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d.get('ms_per_step_median'), d['roofline']['frac'])")
    echo "td=$v $op -> $r" >> $o
  done
done; done
