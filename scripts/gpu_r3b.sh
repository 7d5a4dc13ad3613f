# pass scheduler: default bench line, then the GPU suite
set -x
mkdir -p gpurun_out/r3b
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r3b/build.log 2>&1
timeout 900 python bench.py > gpurun_out/r3b/bench_default.json 2> gpurun_out/r3b/bench_default.err
QGPU_PASS_SCHED=0 timeout 600 python bench.py --steps 5 --micro 0 --no-cpu-baseline > gpurun_out/r3b/bench_nosched.json 2> gpurun_out/r3b/bench_nosched.err
timeout 600 python bench.py --workload rqc --n 30 --steps 5 --micro 0 --no-cpu-baseline > gpurun_out/r3b/bench_rqc30.json 2> gpurun_out/r3b/bench_rqc30.err
timeout 1800 python -m pytest tests -m gpu -q -x --durations=10 > gpurun_out/r3b/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3b/pytest_gpu.log
tail -3 gpurun_out/r3b/pytest_gpu.log
