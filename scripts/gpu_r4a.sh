set -x
bash scripts/gpu_ab.sh r4a/ab scripts/ab_variants23.txt
python scripts/write_bw_probe.py > gpurun_out/r4a/write_bw.json 2>&1
