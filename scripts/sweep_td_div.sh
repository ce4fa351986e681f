export OPARGS="--op bfs --scale 26 --steps 8 --warmup 3 --no-context"
export VARIANTS="X=0;INL_BFS_TD_DIV=16;INL_BFS_TD_DIV=256;INL_BFS_TD_DIV=1024"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_td_div_s26.txt
export OPARGS="--op bfs --steps 9 --warmup 3 --no-context"
export VARIANTS="X=0;INL_BFS_TD_DIV=16;INL_BFS_TD_DIV=256;INL_BFS_TD_DIV=1024;X=1"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_td_div_s23.txt
