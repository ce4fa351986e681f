mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ll_sssp_graph.csv python scripts/sssp_steps.py > gpurun_out/ll_sssp_graph.log 2>&1; echo rc=$? >> gpurun_out/ll_sssp_graph.log
INL_SSSP_LOOP=dyn timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ll_sssp_dyn.csv python scripts/sssp_steps.py > gpurun_out/ll_sssp_dyn.log 2>&1; echo rc=$? >> gpurun_out/ll_sssp_dyn.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ll_bfs26.csv python scripts/sssp_steps.py --op bfs --scale 26 > gpurun_out/ll_bfs26.log 2>&1; echo rc=$? >> gpurun_out/ll_bfs26.log
