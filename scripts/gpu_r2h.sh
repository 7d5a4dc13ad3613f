O=gpurun_out/r2h; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_measure.py tests/test_gpu_fullsize.py -k "measure or e2e or fused" -q -x > $O/pytest_measure.log 2>&1; echo "rc=$?" >> $O/pytest_measure.log
timeout 600 python bench.py --steps 5 --warmup 3 --micro 0 --no-cpu-baseline --gfc 0 > $O/bench.json 2> $O/bench.err
