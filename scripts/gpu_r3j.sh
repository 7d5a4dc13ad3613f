# ncu --set full of the FP64-bound passes on the current kernels (QAOA_32 last pass, rqc_30 heaviest)
set -x
O=gpurun_out/r3j; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 15 -c 1 -o $O/qaoa32_last \
  python scripts/profile_step.py --workload qaoa32 > $O/ncu_qaoa.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_rqc30.csv \
  python scripts/profile_step.py --workload rqc --n 30 > $O/ncu_rqc_l.log 2>&1
