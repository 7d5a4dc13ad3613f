# round 2, first call: GPU tests on the new code, the new default bench line, QAOA_32 launch list,
# lane-bit experiments on the U-heavy workloads
mkdir -p gpurun_out/r2a
O=gpurun_out/r2a
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x --durations=15 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
T0=$(date +%s); timeout 900 python bench.py --steps 5 --warmup 3 > $O/bench.json 2> $O/bench.err; echo "bench rc=$? wall s: $(( $(date +%s) - T0 ))" >> $O/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/launches_qaoa32.csv python scripts/profile_step.py --workload qaoa32 > $O/ncu1.log 2>&1
for L in 3 4; do
  QGPU_LMIN=$L timeout 600 python bench.py --workload qaoa32 --steps 3 --extras 0 --micro 0 --no-cpu-baseline --gfc 0 > $O/qaoa_lmin$L.json 2> $O/qaoa_lmin$L.err
  QGPU_LMIN=$L timeout 600 python bench.py --workload rqc --n 30 --steps 3 --extras 0 --micro 0 --no-cpu-baseline --gfc 0 > $O/rqc_lmin$L.json 2> $O/rqc_lmin$L.err
done
timeout 600 python bench.py --workload rqc --n 30 --steps 3 --extras 0 --micro 0 --no-cpu-baseline --gfc 0 > $O/rqc.json 2> $O/rqc.err
tail -3 $O/pytest_gpu.log; tail -2 $O/bench.err
