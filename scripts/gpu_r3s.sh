# compute-sanitizer on the round-2 (second session) paths, NVRTC kernels at the default threshold
set -x
O=gpurun_out/r3s; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
python scripts/sanitize_run.py --meas --jit 1 > $O/plain.log 2>&1; echo "plain rc=$?" >> $O/plain.log
for tool in memcheck racecheck synccheck; do
  QGPU_JIT_MIN_BITS=12 timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_run.py --meas --jit 1 > $O/san_${tool}.log 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|max' $O/san_${tool}.log | tr '\n' ' ')"
done | tee $O/san_summary.log
