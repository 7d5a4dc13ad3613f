# A/B experiment: env settings in $EXP (space-separated assignments, "-" = defaults)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
for E in ${EXP:-"-"}; do
  [ "$E" = "-" ] && E=""
  if [ -n "$TESTS" ]; then env $E timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/pytest_exp.log 2>&1; echo "[$E] pytest rc=$? $(tail -1 gpurun_out/pytest_exp.log)"; fi
  for w in ${WORKLOADS:-qaoa32 rqc qft28}; do
    env $E timeout 900 python bench.py --workload $w --steps 3 --no-cpu-baseline --micro 0 --gfc 0 2>>gpurun_out/bench_err.log | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); r=d['roofline']
    print('[$E]', d['config']['workload'][:20], 'ms=%.3f'%d['ms_per_step'], 'frac=%.3f'%r['frac'])
"
  done
done
