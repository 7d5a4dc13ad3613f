set -x
bash scripts/gpu_ab.sh r3y/ab scripts/ab_variants22.txt
