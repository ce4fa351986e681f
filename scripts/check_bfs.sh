mkdir -p gpurun_out
B="python bench.py --no-e2e --no-cpu-baseline --no-context"
o=gpurun_out/check_bfs.txt; : > $o
for i in 1 2; do echo "== bfs s23" >> $o; timeout 300 $B --op bfs --steps 9 --warmup 3 >> $o 2>>gpurun_out/check_bfs.err; done
echo "== bfs s26" >> $o; timeout 600 $B --op bfs --scale 26 --steps 8 --warmup 3 >> $o 2>>gpurun_out/check_bfs.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ll_bfs26b.csv python scripts/sssp_steps.py --op bfs --scale 26 --no-warmup > gpurun_out/ll_bfs26b.log 2>&1
timeout 900 python -m pytest tests/test_gpu_sssp_bfs.py tests/test_gpu_fullsize.py tests/test_gpu_bc.py -q -x > gpurun_out/pytest_bfs.log 2>&1; echo rc=$? >> gpurun_out/pytest_bfs.log
