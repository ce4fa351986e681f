mkdir -p gpurun_out
( for n in 4194304 33554432; do timeout 60 ./scripts/microbench/tma_gather $n; done ) > gpurun_out/tma_gather.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_colblock.py -x -q > gpurun_out/pytest_cb.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
B="timeout 300 python bench.py --no-e2e --no-cpu-baseline"
( $B --no-colblock; $B; $B --bins 8,512,16384,4096; $B --bins 8,256,16384,4096;
  INL_CB_K=32768 $B --bins 8,256,16384,4096; INL_CB_K=57344 $B --bins 8,256,16384,4096;
  INL_CB_MULT=2 $B --bins 8,256,16384,4096 ) > gpurun_out/cb_spmv.txt 2>&1
( $B --op pagerank --steps 3 --warmup 1 --no-colblock; $B --op pagerank --steps 3 --warmup 1;
  INL_CB_MULT=2 $B --op pagerank --steps 3 --warmup 1 ) > gpurun_out/cb_pr.txt 2>&1
