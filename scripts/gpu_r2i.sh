O=gpurun_out/r2i; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
QGPU_DEBUG_HIST=1 timeout 600 python scripts/e2e_breakdown.py qaoa32 > $O/e2e_qaoa32.log 2>&1
timeout 600 python bench.py --steps 10 --warmup 3 --micro 0 --no-cpu-baseline --gfc 0 > $O/bench.json 2> $O/bench.err
timeout 1200 python -m pytest tests/test_gpu_jit_default.py -q -x > $O/pytest_jit_default.log 2>&1; echo "rc=$?" >> $O/pytest_jit_default.log
