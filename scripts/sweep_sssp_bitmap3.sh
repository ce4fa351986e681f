export OPARGS="--op sssp --steps 9 --warmup 3 --no-context"
M4=build/variants/libinl_minb4.so
V=""
for d in 96 128 192 256 384; do for g in 2,8,8 2,6,8; do V="$V;INL_LIB=$M4 INL_SSSP_GRIDS=$g INL_SSSP_DELTA=$d"; done; done
export VARIANTS="${V#;}"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_sssp3.txt
