mkdir -p gpurun_out
for i in 0 1 2 3 4 5 6 7; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_expand_grid|k_expand_flat|k_bu_" --csv --log-file gpurun_out/ll_bfs26_s$i.csv python scripts/sssp_steps.py --op bfs --scale 26 --no-warmup --source-index $i > gpurun_out/ll_bfs26_s$i.log 2>&1
done
