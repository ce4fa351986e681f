# A/B of two library builds: ALIB (variant path) vs the in-tree build, alternating, OPARGS
mkdir -p gpurun_out
o=gpurun_out/ab_lib.txt; : > $o
for i in 1 2 3; do
  for L in "$ALIB" ""; do
    r=$(INL_LIB=$L timeout 300 python bench.py --no-e2e --no-cpu-baseline --no-context $OPARGS 2>>gpurun_out/ab_lib.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d.get('ms_per_step_median'))")
    echo "lib=${L:-intree} $r" >> $o
  done
done
