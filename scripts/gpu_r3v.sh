set -x
bash scripts/gpu_ab.sh r3v/ab scripts/ab_variants19.txt
