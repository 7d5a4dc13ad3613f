# A/B of planner / kernel variants on one box, interleaved twice: $1 = output dir under gpurun_out,
# $2 = variants file (lines "name bench-args... ENV=value ...")
O=gpurun_out/$1; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
B="python bench.py --steps 4 --warmup 3 --extras 0 --micro 0 --no-cpu-baseline --gfc 0"
for rep in 1 2; do
while read -r name rest; do
  [ -z "$name" ] && continue
  args=""; envs=""
  for w in $rest; do case $w in --*) args="$args $w";; *) envs="$envs $w";; esac; done
  env $envs timeout 600 $B $args > $O/${name}_$rep.json 2> $O/${name}_$rep.err
done < $2
done
