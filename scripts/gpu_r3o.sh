set -x
bash scripts/gpu_ab.sh r3o/ab scripts/ab_variants16.txt
