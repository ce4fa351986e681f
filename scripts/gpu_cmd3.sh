mkdir -p gpurun_out
( for n in 4194304 16777216 33554432; do timeout 60 ./scripts/microbench/tma_gather $n; done ) > gpurun_out/tma_gather.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_pagerank.py tests/test_gpu_dist1.py -q -x > gpurun_out/pytest_pr.log 2>&1
( timeout 600 python bench.py --op pagerank --steps 3 --warmup 1 --no-e2e --no-cpu-baseline;
  INL_PR_ORDER=vertex timeout 600 python bench.py --op pagerank --steps 3 --warmup 1 --no-e2e --no-cpu-baseline ) > gpurun_out/pr_order.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather -s 3 -c 1 -o gpurun_out/prof_pr2 -f python bench.py --op pagerank --steps 1 --warmup 1 --iterations 4 --no-e2e --no-cpu-baseline > gpurun_out/ncu_pr2.log 2>&1
