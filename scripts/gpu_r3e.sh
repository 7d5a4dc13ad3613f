# fused measurement with global reductions; early prefetch gated: measurement parity, then A/B
set -x
O=gpurun_out/r3e; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_measure.py -m gpu -q -x > $O/pytest_a.log 2>&1; echo "rc=$?" >> $O/pytest_a.log
bash scripts/gpu_ab.sh r3e/ab scripts/ab_variants9.txt
tail -n 2 $O/pytest_a.log
