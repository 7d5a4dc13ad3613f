# HBM access-shape probe + ncu full capture of QFT_28 pass 3 (k 20->26) and refined-rule checks
mkdir -p gpurun_out build
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/bw_probe scripts/bw_probe.cu && ./build/bw_probe > gpurun_out/bw_probe.txt 2>&1
cat gpurun_out/bw_probe.txt
timeout 600 python -m pytest tests/test_gpu_refined.py -x -q 2>&1 | tail -1
timeout 600 python scripts/ablation.py --n 30 --refined --reps 3 --families qft,qaoa > gpurun_out/ablation_refined.log 2>&1; tail -3 gpurun_out/ablation_refined.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 6 -c 1 -o gpurun_out/qft28_pass3 python scripts/profile_step.py --workload qft28 > gpurun_out/ncu3.log 2>&1
tail -2 gpurun_out/ncu3.log
