# compute-sanitizer over every entry point; logs to gpurun_out/sanitize_*.log
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 python tools/sanitize_driver.py 2500 \
    > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool exit $?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|error|hazard" gpurun_out/sanitize_$tool.log | head -5
done
