# round 2 call b: sharded (virtual-rank) tests of the new swap engine, full-size parity at the bench
# configuration (incl. QAOA_32 vs the oracle), ncu full captures of the heaviest fused passes
mkdir -p gpurun_out/r2b
O=gpurun_out/r2b
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_sharded.py -q -x > $O/pytest_sharded.log 2>&1; echo "rc=$?" >> $O/pytest_sharded.log
timeout 1800 python -m pytest tests/test_gpu_fullsize.py -q -x --durations=20 > $O/pytest_fullsize.log 2>&1; echo "rc=$?" >> $O/pytest_fullsize.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 15 -c 2 -o $O/qaoa30_heavy python scripts/profile_step.py --workload qaoa32 --n 30 > $O/ncu_qaoa.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 53 -c 2 -o $O/rqc30_heavy python scripts/profile_step.py --workload rqc --n 30 > $O/ncu_rqc.log 2>&1
tail -3 $O/pytest_sharded.log $O/pytest_fullsize.log
