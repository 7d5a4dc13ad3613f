# fused measurement modes: tests, then bench e2e A/B (QGPU_HACC=0 = separate readout for lane/register bits)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_measure.py -x -q > gpurun_out/pytest_measure.log 2>&1; echo "measure rc=$? $(tail -1 gpurun_out/pytest_measure.log)"
for H in 1 0; do
  QGPU_HACC=$H timeout 900 python bench.py --steps 10 --no-cpu-baseline --micro 0 > gpurun_out/bench_hacc$H.json 2>gpurun_out/bench_hacc$H.err
  python -c "import json;d=json.load(open('gpurun_out/bench_hacc$H.json'));print('HACC=$H', d['value'], d['e2e'])"
done
for H in 1 0; do
QGPU_HACC=$H timeout 900 python bench.py --workload qaoa32 --steps 3 --no-cpu-baseline --micro 0 > gpurun_out/bench_qaoa32_hacc$H.json 2>&1
python -c "import json;d=json.load(open('gpurun_out/bench_qaoa32_hacc$H.json'));print('qaoa32 HACC=$H', d['value'], d['e2e'])"
done
if [ -n "$FULL" ]; then timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$? $(tail -1 gpurun_out/pytest_gpu.log)"; fi
