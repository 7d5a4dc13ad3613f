# host-memory tier (NEXT-2) bench lines: state in pinned host memory, streamed through the GPU.
# WORKLOADS: ';'-separated bench arguments
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
W=${WORKLOADS:-"qft28 --n 30 --host-slice-bits 2;qaoa32 --n 30 --host-slice-bits 2;rqc --n 30 --host-slice-bits 2;qft28 --n 32 --host-slice-bits 3;qaoa32 --n 32 --host-slice-bits 3"}
IFS=';' read -ra WL <<< "$W"
for w in "${WL[@]}"; do
  tag=$(echo $w | tr -d ' -')
  timeout 1200 python bench.py --workload $w --steps 3 --no-cpu-baseline --micro 0 > gpurun_out/bench_host_$tag.json 2>>gpurun_out/bench_err.log
  python -c "
import json,sys
d=json.load(open('gpurun_out/bench_host_$tag.json'))
h=d['host_tier']; r=d['roofline']; l=h['link']
print('$w', 'ms=%.1f'%d['ms_per_step'], 'sweeps', h['sweeps_per_step'], 'loads', h['slice_loads'], 'skips', h['slice_skips'], 'h2d GB %.2f d2h GB %.2f'%(h['h2d_bytes_per_step']/1e9, h['d2h_bytes_per_step']/1e9), 'link %.1f GB/s (h2d pk %.1f d2h pk %.1f) frac %.2f bound %.0f ms sweep %.0f ms'%(l['achieved'], l['h2d_peak'], l['d2h_peak'], l['frac'], l['bound_ms_per_step'], h['sweep_ms_per_step']), 'tile frac %.2f'%r['frac'])
" || tail -5 gpurun_out/bench_err.log
done
