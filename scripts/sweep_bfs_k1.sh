export OPARGS="--op bfs --steps 9 --warmup 3 --no-context"
export VARIANTS="INL_BFS_K1=8;INL_BFS_K1=4;INL_BFS_K1=2;INL_BFS_K1=1;INL_BFS_K1=8"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_bfs_k1_s23.txt
export OPARGS="--op bfs --scale 26 --steps 8 --warmup 3 --no-context"
export VARIANTS="INL_BFS_K1=8;INL_BFS_K1=4;INL_BFS_K1=2;INL_BFS_K1=1"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_bfs_k1_s26.txt
