# early prefetch + reduce-scatter measurement epilogue: parity first, then interleaved A/B
set -x
O=gpurun_out/r3d; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_measure.py tests/test_gpu_parity.py -m gpu -q -x > $O/pytest_a.log 2>&1; echo "rc=$?" >> $O/pytest_a.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "e2e or qaoa28 or c2_" > $O/pytest_b.log 2>&1; echo "rc=$?" >> $O/pytest_b.log
bash scripts/gpu_ab.sh r3d/ab scripts/ab_variants8.txt
tail -2 $O/pytest_a.log $O/pytest_b.log
