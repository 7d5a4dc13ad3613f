set -x
bash scripts/gpu_ab.sh r3h/ab scripts/ab_variants11.txt
