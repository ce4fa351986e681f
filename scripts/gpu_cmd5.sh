mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_colblock.py -x -q > gpurun_out/pytest_cb.log 2>&1
B="timeout 300 python bench.py --no-e2e --no-cpu-baseline"
( $B --op pagerank --steps 2 --warmup 1 --iterations 3; $B ) > gpurun_out/cb_k.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,smsp__inst_executed.sum,l1tex__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:'k_gather|k_cb' -c 30 --csv --log-file gpurun_out/cb_launches_pr.csv python bench.py --op pagerank --steps 1 --warmup 1 --iterations 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_cb$|k_cb<' -s 2 -c 1 -o gpurun_out/prof_cb_pr -f python bench.py --op pagerank --steps 1 --warmup 1 --iterations 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_cb.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_cb' -s 4 -c 1 -o gpurun_out/prof_cb_spmv -f python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_cb2.log 2>&1
