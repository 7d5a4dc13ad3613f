# round-2 re-entry check on HEAD: smoke, full GPU suite, default bench line
set -x
mkdir -p gpurun_out/r3a
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r3a/build.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r3a/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r3a/smoke.log
T0=$(date +%s); timeout 900 python bench.py > gpurun_out/r3a/bench_default.json 2> gpurun_out/r3a/bench_default.err; echo "bench wall s: $(( $(date +%s) - T0 ))" >> gpurun_out/r3a/bench_default.err
timeout 1800 python -m pytest tests -m gpu -q -x --durations=10 > gpurun_out/r3a/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3a/pytest_gpu.log
tail -3 gpurun_out/r3a/pytest_gpu.log; tail -2 gpurun_out/r3a/smoke.log
tail -1 gpurun_out/r3a/bench_default.err
