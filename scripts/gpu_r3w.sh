set -x
O=gpurun_out/r3w; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_measure.py -m gpu -q -x > $O/pytest_a.log 2>&1; echo "rc=$?" >> $O/pytest_a.log
bash scripts/gpu_ab.sh r3w/ab scripts/ab_variants20.txt
tail -n 2 $O/pytest_a.log
