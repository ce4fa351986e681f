# Experiment record: the hub-deferral code (INL_SSSP_HUBS) measured 2.1x slower and was not kept
# (profiles/r02/sssp_hub_deferral_experiment.txt); the INL_SSSP_HUBS switch no longer exists.
mkdir -p gpurun_out
B="python bench.py --no-e2e --no-cpu-baseline --no-context --op sssp --steps 9 --warmup 3"
o=gpurun_out/check_hubs.txt; : > $o
for i in 1 2; do for h in 1 0; do echo "== hubs=$h" >> $o; INL_SSSP_HUBS=$h timeout 300 $B >> $o 2>>gpurun_out/check_hubs.err; done; done
rm -f gpurun_out/sssp_trace.txt; INL_SSSP_TRACE=gpurun_out/sssp_trace.txt timeout 300 python scripts/sssp_steps.py > gpurun_out/sssp_trace.log 2>&1
timeout 900 python -m pytest tests/test_gpu_sssp_bfs.py tests/test_gpu_fullsize.py -q -x > gpurun_out/pytest_sssp.log 2>&1; echo rc=$? >> gpurun_out/pytest_sssp.log
