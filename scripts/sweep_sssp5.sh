export OPARGS="--op sssp --steps 9 --warmup 3 --no-context"
export VARIANTS="X=0;INL_LIB=build/variants/libinl_cg.so;INL_LIB=build/variants/libinl_lu.so;X=1;INL_LIB=build/variants/libinl_cg.so;INL_LIB=build/variants/libinl_lu.so"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_sssp5.txt
