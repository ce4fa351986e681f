mkdir -p gpurun_out
o=gpurun_out/sweep_twarp2.txt; : > $o
for op in "sssp --steps 9 --warmup 3" "bfs --scale 26 --steps 8 --warmup 3"; do
for tw in 1024 2048 4096 512 1024; do
  r=$(timeout 300 python bench.py --no-e2e --no-cpu-baseline --no-context --op $op --bins 8,$tw,16384,8192,256 2>>gpurun_out/sweep_twarp2.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'])")
  echo "$op t_warp=$tw -> $r" >> $o
done; done
