# planner knob sweep on U-heavy circuits (experiment; defaults: MAX_UOPS 24, LOOKAHEAD 192)
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
for W in "qaoa32 --n 30" "rqc --n 30"; do
for E in "QGPU_MAX_UOPS=24" "QGPU_MAX_UOPS=16" "QGPU_MAX_UOPS=32" "QGPU_MAX_UOPS=48" "QGPU_LOOKAHEAD=384" "QGPU_MAX_UOPS=32 QGPU_LOOKAHEAD=384"; do
  env $E timeout 600 python bench.py --workload $W --steps 3 --no-cpu-baseline --micro 0 --gfc 0 2>/dev/null | python -c "import json,sys;d=json.loads(sys.stdin.readline());r=d['roofline'];print('$W', '$E', round(d['value']*1e3,2),'ms', r['launches_per_step'],'passes', round(r['frac'],3))"
done; done
