export OPARGS="--op sssp --steps 9 --warmup 3 --no-context"
export VARIANTS="X=0;INL_SSSP_GRIDS=2,8,4;INL_SSSP_GRIDS=2,8,8;INL_SSSP_GRIDS=2,16,8;INL_LIB=build/variants/libinl_minb3.so;INL_LIB=build/variants/libinl_minb4.so;INL_LIB=build/variants/libinl_minb4.so INL_SSSP_GRIDS=2,8,8;INL_LIB=build/variants/libinl_minb4.so INL_SSSP_GRIDS=2,16,16;INL_SSSP_DELTA=32;INL_SSSP_DELTA=64;INL_SSSP_DELTA=96;X=1"
bash scripts/sweep_env.sh
