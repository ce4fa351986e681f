mkdir -p gpurun_out
B="python bench.py --no-e2e --no-cpu-baseline --no-context"
o=gpurun_out/check_sssp.txt; : > $o
for i in 1 2; do echo "== sssp" >> $o; timeout 300 $B --op sssp --steps 9 --warmup 3 >> $o 2>>gpurun_out/check_sssp.err; done
echo "== sssp dyn" >> $o; INL_SSSP_LOOP=dyn timeout 300 $B --op sssp --steps 9 --warmup 3 >> $o 2>>gpurun_out/check_sssp.err
echo "== sssp dynbits" >> $o; INL_SSSP_LOOP=dyn INL_SSSP_DYN_BITS=1 timeout 300 $B --op sssp --steps 9 --warmup 3 >> $o 2>>gpurun_out/check_sssp.err
rm -f gpurun_out/sssp_trace.txt; INL_SSSP_TRACE=gpurun_out/sssp_trace.txt timeout 300 python scripts/sssp_steps.py > gpurun_out/sssp_trace.log 2>&1
timeout 900 python -m pytest tests/test_gpu_sssp_bfs.py tests/test_gpu_fullsize.py -q -x > gpurun_out/pytest_sssp.log 2>&1; echo rc=$? >> gpurun_out/pytest_sssp.log
