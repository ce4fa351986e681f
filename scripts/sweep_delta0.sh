# Experiment record: INL_SSSP_DELTA0 (first-bucket width) measured within noise and was removed.
export OPARGS="--op sssp --steps 9 --warmup 3 --no-context"
export VARIANTS="X=0;INL_SSSP_DELTA0=16;INL_SSSP_DELTA0=32;INL_SSSP_DELTA0=48;INL_SSSP_DELTA0=64;X=1;INL_SSSP_DELTA0=32"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_delta0.txt
