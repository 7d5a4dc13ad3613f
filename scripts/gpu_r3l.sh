# evidence: smoke, default bench line, reference arm, full GPU suite, ncu launch list of QAOA_32
set -x
O=gpurun_out/r3l; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
T0=$(date +%s); timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo "bench wall s: $(( $(date +%s) - T0 ))" >> $O/bench_default.err
timeout 600 python bench.py --workload rqc --n 30 --steps 5 --micro 0 --no-cpu-baseline > $O/bench_rqc30.json 2> $O/bench_rqc30.err
T0=$(date +%s); timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err; echo "ref wall s: $(( $(date +%s) - T0 ))" >> $O/bench_ref.err
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file $O/launches_rqc30.csv python scripts/profile_step.py --workload rqc --n 30 --stats-out $O/stats_rqc30.json > $O/ncu_rqc.log 2>&1
tail -n 3 $O/pytest_gpu.log
