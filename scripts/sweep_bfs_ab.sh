export OPARGS="--op bfs --scale 26 --steps 8 --warmup 3 --no-context"
export VARIANTS="X=0;INL_BFS_AB=7,24;INL_BFS_AB=28,24;INL_BFS_AB=14,12;INL_BFS_AB=14,48;X=1"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_bfs_ab_s26.txt
export OPARGS="--op bfs --steps 9 --warmup 3 --no-context"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_bfs_ab_s23.txt
