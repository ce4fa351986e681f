#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_sssp_bfs.py tests/test_gpu_dist1.py -x -q > gpurun_out/pytest_frontier.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_frontier.log
: > gpurun_out/bench_delta.txt
for dl in 0 32 64 128 256 512; do echo "delta=$dl" >> gpurun_out/bench_delta.txt; INL_SSSP_DELTA=$dl timeout 600 python bench.py --op sssp --steps 9 --warmup 2 --no-e2e --no-cpu-baseline >> gpurun_out/bench_delta.txt 2>>gpurun_out/bench_frontier.err; done
