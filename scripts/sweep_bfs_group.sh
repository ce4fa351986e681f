export OPARGS="--op bfs --scale 26 --steps 8 --warmup 3 --no-context"
export VARIANTS="INL_BFS_GROUP=2;INL_BFS_GROUP=1;INL_BFS_GROUP=2;INL_BFS_GROUP=1"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_bfs_group_s26.txt
export OPARGS="--op bfs --steps 9 --warmup 3 --no-context"
export VARIANTS="INL_BFS_GROUP=2;INL_BFS_GROUP=1;INL_BFS_GROUP=2;INL_BFS_GROUP=1"
bash scripts/sweep_env.sh; mv gpurun_out/sweep.txt gpurun_out/sweep_bfs_group_s23.txt
timeout 600 python -m pytest tests/test_gpu_sssp_bfs.py -q -x -k "devloop or scale18" > gpurun_out/pytest_quick.log 2>&1; echo rc=$? >> gpurun_out/pytest_quick.log
