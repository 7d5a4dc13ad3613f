# compute-sanitizer on the round's new paths (zero halves, host tier, refined rule)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for jit in 0 2; do
  for tool in memcheck racecheck synccheck; do
    timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_run.py --new --jit $jit > gpurun_out/san_new_${tool}_${jit}.log 2>&1
    echo "new $tool jit=$jit rc=$? $(grep -E 'ERROR SUMMARY|max' gpurun_out/san_new_${tool}_${jit}.log | tr '\n' ' ')"
  done
done | tee gpurun_out/san_summary_new.log
