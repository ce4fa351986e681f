mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_colblock.py tests/test_gpu_pagerank.py -x -q > gpurun_out/pytest_cb.log 2>&1
B="timeout 300 python bench.py --no-e2e --no-cpu-baseline"
( $B --op pagerank --steps 3 --warmup 1 --no-colblock; $B --op pagerank --steps 3 --warmup 1;
  INL_CB_MULT=2 $B --op pagerank --steps 3 --warmup 1; INL_CB_MULT=8 $B --op pagerank --steps 3 --warmup 1 ) > gpurun_out/cb_pr.txt 2>&1
( $B --no-colblock; $B; $B --bins 8,512,16384,4096; $B --bins 8,256,16384,4096 ) > gpurun_out/cb_spmv.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'^k_cb$' -s 4 -c 1 -o gpurun_out/prof_cb_spmv -f python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_cb2.log 2>&1
