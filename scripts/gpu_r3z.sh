# final evidence: smoke, default bench line, rqc_30 line, full GPU suite
set -x
O=gpurun_out/r3z; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
T0=$(date +%s); timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "bench wall s: $(( $(date +%s) - T0 ))" >> $O/bench_default.err
timeout 600 python bench.py --workload rqc --n 30 --steps 5 --micro 0 --no-cpu-baseline > $O/bench_rqc30.json 2> $O/bench_rqc30.err
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -n 3 $O/pytest_gpu.log
