mkdir -p gpurun_out
B="python bench.py --no-e2e --no-cpu-baseline --no-context"
o=gpurun_out/check_sssp.txt; : > $o
for i in 1 2; do echo "== sssp" >> $o; timeout 300 $B --op sssp --steps 9 --warmup 3 >> $o 2>>gpurun_out/check_sssp.err; done
echo "== bfs" >> $o; timeout 300 $B --op bfs --steps 9 --warmup 3 >> $o 2>>gpurun_out/check_sssp.err
rm -f gpurun_out/sssp_trace.txt; INL_SSSP_TRACE=gpurun_out/sssp_trace.txt timeout 300 python scripts/sssp_steps.py > gpurun_out/sssp_trace.log 2>&1
timeout 900 python -m pytest tests/test_gpu_sssp_bfs.py tests/test_gpu_fullsize.py tests/test_gpu_templates.py tests/test_gpu_edge_cases.py -q -x > gpurun_out/pytest_sssp.log 2>&1; echo rc=$? >> gpurun_out/pytest_sssp.log
