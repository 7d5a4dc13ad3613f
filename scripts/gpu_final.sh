# round-end evidence: full GPU tests, default bench line (timed), reference arm, QAOA_32 line, ncu launch list + full capture
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
T0=$(date +%s); timeout 900 python bench.py > gpurun_out/bench_qft28.json 2> gpurun_out/bench_qft28.err; echo "bench wall s: $(( $(date +%s) - T0 ))" >> gpurun_out/bench_qft28.err
timeout 900 python bench.py --impl reference --steps 1 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 900 python bench.py --workload qaoa32 --steps 3 --no-cpu-baseline --micro 0 > gpurun_out/bench_qaoa32.json 2> gpurun_out/bench_qaoa32.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_qft28.csv python scripts/profile_step.py --workload qft28 > gpurun_out/ncu1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 7 -c 1 -o gpurun_out/qft28_full python scripts/profile_step.py --workload qft28 > gpurun_out/ncu2.log 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log
tail -1 gpurun_out/bench_qft28.err
