set -x
O=gpurun_out/r3m; mkdir -p $O
bash scripts/gpu_ab.sh r3m/ab scripts/ab_variants14.txt
python scripts/meas_profile.py qaoa32 > $O/meas_profile.log 2>&1
