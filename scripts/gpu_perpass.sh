# per-pass launch list (time, DRAM bytes, FP64 pipe and issue utilisation) for U-heavy workloads
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum
for w in "qaoa32" "rqc --n 30"; do
  tag=$(echo $w | tr -d ' -')
  timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/pp_$tag.csv python scripts/profile_step.py --workload $w > gpurun_out/pp_$tag.log 2>&1
done
