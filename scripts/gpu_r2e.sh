O=gpurun_out/r2e; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build0.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_measure.py tests/test_gpu_zskip.py tests/test_gpu_refined.py tests/test_gpu_sharded.py -q -x > $O/pytest_core.log 2>&1; echo "rc=$?" >> $O/pytest_core.log
bash scripts/gpu_ab.sh r2e scripts/ab_variants4.txt
