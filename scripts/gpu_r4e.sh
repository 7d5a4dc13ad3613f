set -x
O=gpurun_out/r4e; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
QGPU_STORE_REMAP=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "families or fuzz or qft_closed" > $O/pytest_a.log 2>&1; echo "rc=$?" >> $O/pytest_a.log
bash scripts/gpu_ab.sh r4e/ab scripts/ab_variants25.txt
tail -n 2 $O/pytest_a.log
