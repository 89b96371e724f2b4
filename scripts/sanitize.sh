for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_smoke.py > gpurun_out/sanitizer_$tool.log 2>&1
  echo "$tool rc=$?"; tail -2 gpurun_out/sanitizer_$tool.log
done
