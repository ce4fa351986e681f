mkdir -p gpurun_out
B="python bench.py --no-e2e --no-cpu-baseline --no-context"
o=gpurun_out/check_pr.txt; : > $o
for i in 1 2; do echo "== pagerank" >> $o; timeout 300 $B --op pagerank --steps 3 --warmup 1 >> $o 2>>gpurun_out/check_pr.err; done
timeout 900 python -m pytest tests/test_gpu_pagerank.py tests/test_gpu_loopback.py tests/test_gpu_fullsize.py -q -x -k "pagerank or cfg4" > gpurun_out/pytest_pr.log 2>&1; echo rc=$? >> gpurun_out/pytest_pr.log
