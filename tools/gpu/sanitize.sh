# compute-sanitizer over a workload that launches every libspmv kernel
for tool in memcheck racecheck synccheck initcheck; do
  echo "== $tool"
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize_workload.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "exit $?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|sanitize workload done|Error|error" gpurun_out/sanitize_$tool.log | head -8
done
