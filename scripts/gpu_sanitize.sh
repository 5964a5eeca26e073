mkdir -p gpurun_out
for tool in memcheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize.py > gpurun_out/sanitize_$tool.log 2>&1; echo $tool rc=$?
  tail -3 gpurun_out/sanitize_$tool.log
done
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/sanitize.py half > gpurun_out/sanitize_racecheck_half.log 2>&1; echo racecheck-half rc=$?
tail -5 gpurun_out/sanitize_racecheck_half.log
