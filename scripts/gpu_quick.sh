# quick GPU check: parity tests + bench lines of the main workloads (no cpu baseline, no micro)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
if [ "${SKIP_TESTS:-0}" = "0" ]; then
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
fi
for w in ${WORKLOADS:-"qft28" "qaoa32" "rqc --n 30"}; do
  timeout 900 python bench.py --workload $w --steps 3 --no-cpu-baseline --micro 0 2>>gpurun_out/bench_err.log | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); r=d['roofline']
    print(d['config']['workload'][:40], 'ms=%.3f'%d['ms_per_step'], 'frac=%.3f'%r['frac'], 'passes', d['pruning']['passes'], 'e2e=%.3f'%d['e2e']['value'], 'h2d', d['e2e']['h2d_bytes_per_step'])
"
done
