export OPARGS="--op sssp --steps 9 --warmup 3 --no-context"
export VARIANTS="X=0;INL_LIB=build/variants/libinl_ept4.so;INL_LIB=build/variants/libinl_ept16.so;X=1;INL_LIB=build/variants/libinl_ept4.so"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_ept_sssp.txt
export OPARGS="--op bfs --scale 26 --steps 8 --warmup 3 --no-context"
export VARIANTS="X=0;INL_LIB=build/variants/libinl_ept4.so;INL_LIB=build/variants/libinl_ept16.so"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_ept_bfs.txt
