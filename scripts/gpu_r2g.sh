# round 2 evidence on the current code: default bench line (driver's K/W), reference arm, QAOA_32
# launch list (per-launch DRAM bytes -> roofline.traffic), full GPU test suite, smoke
O=gpurun_out/r2g; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
T0=$(date +%s); timeout 1200 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err; echo "bench rc=$? wall s: $(( $(date +%s) - T0 ))" >> $O/bench.err
T0=$(date +%s); timeout 1200 python bench.py --impl reference --steps 20 --warmup 5 > $O/bench_ref.json 2> $O/bench_ref.err; echo "ref rc=$? wall s: $(( $(date +%s) - T0 ))" >> $O/bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/launches_qaoa32.csv python scripts/profile_step.py --workload qaoa32 > $O/ncu1.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/launches_qft28.csv python scripts/profile_step.py --workload qft28 > $O/ncu2.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
