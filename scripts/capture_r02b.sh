#!/bin/bash
# Round-2 final capture on one GPU: the full -m gpu suite, smoke, the bench lines (default + every
# op + the reference arm), the ncu launch list of the default bench command and `ncu --set full`
# captures of each op's dominant kernels (summaries go to profiles/r02 from here).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt 2>&1
if [ "${TESTS:-1}" = "1" ]; then
timeout 1500 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
fi
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
if [ "${ALL:-1}" = "1" ]; then bash scripts/bench_all.sh; fi
if [ "${NCU:-1}" = "1" ]; then
N="--no-e2e --no-cpu-baseline --no-context"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_spmv.csv python bench.py --steps 5 --warmup 3 $N > gpurun_out/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather -s 3 -c 1 -o gpurun_out/prof_spmv -f python bench.py --steps 2 --warmup 3 $N > gpurun_out/ncu_spmv.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather -s 30 -c 1 -o gpurun_out/prof_pr -f python bench.py --op pagerank --steps 1 --warmup 1 $N > gpurun_out/ncu_pr.log 2>&1
INL_SSSP_LOOP=dyn INL_SSSP_DYN_BITS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_expand_ -s 6 -c 6 -o gpurun_out/prof_sssp -f python scripts/sssp_steps.py --no-warmup > gpurun_out/ncu_sssp.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_bu_thread|k_bu_group" -c 2 -o gpurun_out/prof_bfs -f python scripts/sssp_steps.py --op bfs --scale 26 --no-warmup > gpurun_out/ncu_bfs.log 2>&1
fi
echo capture done
