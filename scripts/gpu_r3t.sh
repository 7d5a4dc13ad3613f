set -x
O=gpurun_out/r3t; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "pass_schedule" > $O/pytest_a.log 2>&1; echo "rc=$?" >> $O/pytest_a.log
tail -n 2 $O/pytest_a.log
