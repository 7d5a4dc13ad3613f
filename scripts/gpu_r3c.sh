# pass scheduler evidence: full GPU suite, ncu launch lists (qaoa32, qft28) with the plan fingerprint,
# ncu --set full of the heaviest QAOA_32 pass (the last one: k 31 -> 32)
set -x
O=gpurun_out/r3c
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for w in qaoa32 qft28; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file $O/launches_$w.csv python scripts/profile_step.py --workload $w --stats-out $O/stats_$w.json > $O/ncu_$w.log 2>&1
done
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 15 -c 1 -o $O/qaoa32_last \
  python scripts/profile_step.py --workload qaoa32 > $O/ncu_full.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -3 $O/pytest_gpu.log
