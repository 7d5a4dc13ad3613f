# ncu launch lists on HEAD (qaoa32, qft28, rqc30) with the plan fingerprint
set -x
O=gpurun_out/r4f; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for w in qaoa32 qft28; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file $O/launches_$w.csv python scripts/profile_step.py --workload $w --stats-out $O/stats_$w.json > $O/ncu_$w.log 2>&1
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file $O/launches_rqc30.csv python scripts/profile_step.py --workload rqc --n 30 --stats-out $O/stats_rqc30.json > $O/ncu_rqc.log 2>&1
