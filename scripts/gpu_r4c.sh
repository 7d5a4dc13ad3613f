set -x
O=gpurun_out/r4c; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_measure.py tests/test_gpu_fullsize.py -m gpu -q -x -k "not c3_qaoa32_vs_oracle" > $O/pytest_a.log 2>&1; echo "rc=$?" >> $O/pytest_a.log
bash scripts/gpu_ab.sh r4c/ab scripts/ab_variants24.txt
tail -n 2 $O/pytest_a.log
