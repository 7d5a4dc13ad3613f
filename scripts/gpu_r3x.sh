set -x
bash scripts/gpu_ab.sh r3x/ab scripts/ab_variants21.txt
