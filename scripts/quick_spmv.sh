#!/bin/bash
# quick SpMV check: gpu tests for spmv, bench default, ncu full of k_gather
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_spmv.py tests/test_gpu_pagerank.py -x -q > gpurun_out/pytest_quick.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_quick.log
timeout 300 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_quick.json 2>gpurun_out/bench_quick.err
if [ -n "$EXTRA" ]; then eval "$EXTRA"; fi
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gather -s 3 -c 1 -o gpurun_out/prof_q -f python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_q.log 2>&1
