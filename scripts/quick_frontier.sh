#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_sssp_bfs.py tests/test_gpu_dist1.py -x -q > gpurun_out/pytest_frontier.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_frontier.log
: > gpurun_out/bench_frontier.txt
for op in sssp bfs; do timeout 600 python bench.py --op $op --steps 9 --warmup 2 --no-e2e --no-cpu-baseline >> gpurun_out/bench_frontier.txt 2>>gpurun_out/bench_frontier.err; done
if [ -n "$EXTRA" ]; then eval "$EXTRA"; fi
