# evidence on the final defaults: smoke, default bench line, rqc_30 line, full GPU suite
set -x
O=gpurun_out/r3p; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
T0=$(date +%s); timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "bench wall s: $(( $(date +%s) - T0 ))" >> $O/bench_default.err
timeout 600 python bench.py --workload rqc --n 30 --steps 5 --micro 0 --no-cpu-baseline > $O/bench_rqc30.json 2> $O/bench_rqc30.err
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 15 -c 1 -o $O/qaoa32_last \
  python scripts/profile_step.py --workload qaoa32 > $O/ncu_qaoa.log 2>&1
tail -n 3 $O/pytest_gpu.log
