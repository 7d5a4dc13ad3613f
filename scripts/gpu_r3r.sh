# bench line with the configs[1] per-pass binding; sharded plan on one GPU (virtual ranks)
set -x
O=gpurun_out/r3r; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
T0=$(date +%s); timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "bench wall s: $(( $(date +%s) - T0 ))" >> $O/bench_default.err
for g in 2 4 8; do
  timeout 900 python bench.py --workload rqc --n 30 --virtual-ranks $g --steps 3 --micro 0 --extras 0 --no-cpu-baseline --gfc 0 > $O/bench_rqc30_vr$g.json 2> $O/bench_rqc30_vr$g.err
done
