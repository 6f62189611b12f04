mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  CME_RES_TIMEOUT_MS=60000 timeout 1800 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 99 python tools/sanitize_case.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; tail -4 gpurun_out/sanitize_$tool.log
done
