# QFT_28: bench line, ncu launch list, full captures of passes 3 and 4
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 600 python bench.py --no-cpu-baseline --micro 0 --gfc 0 > gpurun_out/bench_qft28_quick.json 2> gpurun_out/bench_qft28.err
python -c "import json; d=json.load(open('gpurun_out/bench_qft28_quick.json')); print('ms', d['ms_per_step'], 'frac', d['roofline']['frac'], 'e2e', d['e2e']['value'])"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_qft28.csv python scripts/profile_step.py --workload qft28 > gpurun_out/ncu1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:qgpu_tile -s 6 -c 2 -o gpurun_out/qft28_p34 python scripts/profile_step.py --workload qft28 > gpurun_out/ncu2.log 2>&1
tail -1 gpurun_out/ncu2.log
