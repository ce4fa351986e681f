# A/B of programmatic dependent launch (k_build_xhot -> k_gather) + SSSP step trace
mkdir -p gpurun_out
o=gpurun_out/ab_pdl.txt; : > $o
B="python bench.py --no-e2e --no-cpu-baseline --no-context"
for i in 1 2; do
for p in 0 1; do echo "== spmv INL_PDL=$p" >> $o; INL_PDL=$p timeout 300 $B --op spmv >> $o 2>>gpurun_out/ab_pdl.err; done
done
for p in 0 1; do echo "== pagerank INL_PDL=$p" >> $o; INL_PDL=$p timeout 300 $B --op pagerank --steps 3 --warmup 1 >> $o 2>>gpurun_out/ab_pdl.err; done
rm -f gpurun_out/sssp_trace.txt
INL_SSSP_TRACE=gpurun_out/sssp_trace.txt timeout 300 python scripts/sssp_steps.py > gpurun_out/sssp_trace.log 2>&1
timeout 900 python -m pytest tests/test_gpu_spmv.py tests/test_gpu_pagerank.py tests/test_gpu_loopback.py -q -x > gpurun_out/pytest_pdl.log 2>&1; echo rc=$? >> gpurun_out/pytest_pdl.log
