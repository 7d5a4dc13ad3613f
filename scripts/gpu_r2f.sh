O=gpurun_out/r2f; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build0.log 2>&1
bash scripts/gpu_ab.sh r2f scripts/ab_variants5.txt
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 12 -c 1 -o $O/qaoa32_pass4 python scripts/profile_step.py --workload qaoa32 > $O/ncu_qaoa32.log 2>&1
