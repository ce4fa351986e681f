export OPARGS="--op sssp --steps 9 --warmup 3 --no-context"
M4=build/variants/libinl_minb4.so; M5=build/variants/libinl_minb5.so; M6=build/variants/libinl_minb6.so
export VARIANTS="INL_LIB=$M4 INL_SSSP_GRIDS=2,8,8;INL_LIB=$M4 INL_SSSP_GRIDS=2,8,6;INL_LIB=$M4 INL_SSSP_GRIDS=2,6,8;INL_LIB=$M4 INL_SSSP_GRIDS=2,12,8;INL_LIB=$M4 INL_SSSP_GRIDS=2,8,12;INL_LIB=$M5 INL_SSSP_GRIDS=2,8,8;INL_LIB=$M5 INL_SSSP_GRIDS=2,10,10;INL_LIB=$M6 INL_SSSP_GRIDS=2,12,12;INL_LIB=$M4 INL_SSSP_GRIDS=2,8,8 INL_SSSP_DELTA=96;X=0"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_sssp2.txt
export OPARGS="--op bfs --steps 9 --warmup 3 --no-context"
export VARIANTS="X=0;INL_LIB=$M4;INL_LIB=$M5;X=1"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_bfs.txt
export OPARGS="--op bfs --scale 26 --steps 8 --warmup 3 --no-context"
export VARIANTS="X=0;INL_LIB=$M4;INL_LIB=$M5"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_bfs26.txt
