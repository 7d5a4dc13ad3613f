# round 2 call c: lane-policy auto plans and the two-CTA JIT variant on the U-heavy workloads;
# sharded virtual-rank tests
mkdir -p gpurun_out/r2c
O=gpurun_out/r2c
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_sharded.py -q -x > $O/pytest_sharded.log 2>&1; echo "rc=$?" >> $O/pytest_sharded.log
B="python bench.py --steps 3 --warmup 3 --extras 0 --micro 0 --no-cpu-baseline --gfc 0"
timeout 600 $B --workload qaoa32 > $O/qaoa_auto.json 2> $O/qaoa_auto.err
QGPU_2CTA=1 timeout 600 $B --workload qaoa32 > $O/qaoa_auto_2cta.json 2> $O/qaoa_auto_2cta.err
QGPU_AUTO_LANES=0 QGPU_2CTA=1 timeout 600 $B --workload qaoa32 > $O/qaoa_fixed_2cta.json 2> $O/qaoa_fixed_2cta.err
timeout 600 $B --workload rqc --n 30 > $O/rqc_auto.json 2> $O/rqc_auto.err
QGPU_2CTA=1 timeout 600 $B --workload rqc --n 30 > $O/rqc_auto_2cta.json 2> $O/rqc_auto_2cta.err
QGPU_AUTO_LANES=0 QGPU_2CTA=1 timeout 600 $B --workload rqc --n 30 > $O/rqc_fixed_2cta.json 2> $O/rqc_fixed_2cta.err
QGPU_2CTA=1 timeout 600 $B --workload qft28 > $O/qft_2cta.json 2> $O/qft_2cta.err
timeout 600 $B --workload qft28 > $O/qft.json 2> $O/qft.err
QGPU_2CTA=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "jit or fuzz or famil" > $O/pytest_2cta.log 2>&1; echo "rc=$?" >> $O/pytest_2cta.log
tail -2 $O/pytest_sharded.log $O/pytest_2cta.log
