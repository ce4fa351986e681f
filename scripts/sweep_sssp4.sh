export OPARGS="--op sssp --steps 9 --warmup 3 --no-context"
M3=build/variants/libinl_minb3.so; M5=build/variants/libinl_minb5.so
export VARIANTS="X=0;INL_SSSP_GRIDS=2,8,8;INL_SSSP_GRIDS=2,4,8;INL_SSSP_GRIDS=2,6,4;INL_SSSP_GRIDS=2,6,12;INL_LIB=$M3;INL_LIB=$M3 INL_SSSP_GRIDS=2,6,6;INL_LIB=$M5;INL_LIB=$M5 INL_SSSP_GRIDS=2,10,10;INL_SSSP_DELTA=64;INL_SSSP_DELTA=128;INL_SSSP_DELTA=48;X=1"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_sssp4.txt
