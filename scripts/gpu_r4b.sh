set -x
O=gpurun_out/r4b; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 7 -c 1 -o $O/qft28_last \
  python scripts/profile_step.py --workload qft28 > $O/ncu_qft.log 2>&1
