#!/bin/bash
# One line per op/config (no cpu baseline, no e2e) -> gpurun_out/bench_all.txt
mkdir -p gpurun_out
out=gpurun_out/bench_all.txt
: > $out
run() { echo "== $*" >> $out; timeout 600 python bench.py --no-e2e --no-cpu-baseline --no-context "$@" >> $out 2>>gpurun_out/bench_all.err; }
run --op spmv
run --op spmv --thread-only
run --op sssp --steps 9 --warmup 3
run --op sssp --steps 9 --warmup 3 --thread-only
run --op bfs --steps 9 --warmup 3
run --op bfs --steps 9 --warmup 3 --thread-only
run --op pagerank --steps 3 --warmup 1
run --op bfs --scale 26 --steps 8 --warmup 3
run --op bc --steps 8 --warmup 3
run --op bc --scale 22 --steps 4 --warmup 3
