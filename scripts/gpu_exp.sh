mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
QGPU_REMAP=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "jit or fuse or random" > gpurun_out/pytest_gpu_r1.log 2>&1; echo "pytest remap1 rc=$?"; tail -2 gpurun_out/pytest_gpu_r1.log
for R in 0 1; do
for w in "rqc --n 30" qaoa32 qft28; do
  QGPU_REMAP=$R timeout 900 python bench.py --workload $w --steps 3 --no-cpu-baseline --micro 0 2>>gpurun_out/bench_err.log | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); r=d['roofline']
    print('REMAP=$R', d['config']['workload'][:20], 'ms=%.3f'%d['ms_per_step'], 'frac=%.3f'%r['frac'])
"
done; done
