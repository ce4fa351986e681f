#!/bin/bash
# Round capture on one GPU: tests, smoke, bench lines of every op, the ncu launch list of
# the default bench command and one `ncu --set full` capture of each op's dominant kernel.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
if [ "${ALL:-1}" = "1" ]; then bash scripts/bench_all.sh; fi
if [ "${NCU:-1}" = "1" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_spmv.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather -s 3 -c 1 -o gpurun_out/prof_spmv -f python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_spmv.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather -s 30 -c 1 -o gpurun_out/prof_pr -f python bench.py --op pagerank --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_pr.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_expand_flat -s 20 -c 1 -o gpurun_out/prof_sssp -f python bench.py --op sssp --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_sssp.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_bfs_bottom_up -s 2 -c 1 -o gpurun_out/prof_bfs -f python bench.py --op bfs --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bfs.log 2>&1
fi
