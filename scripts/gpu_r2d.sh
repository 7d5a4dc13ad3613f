O=gpurun_out/r2d; mkdir -p $O
bash scripts/gpu_ab.sh r2d scripts/ab_variants3.txt
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 12 -c 1 -o $O/qaoa32_pass4 python scripts/profile_step.py --workload qaoa32 > $O/ncu_qaoa32.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x --durations=15 > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
