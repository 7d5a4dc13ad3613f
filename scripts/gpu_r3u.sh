set -x
bash scripts/gpu_ab.sh r3u/ab scripts/ab_variants18.txt
