export PYTHONPATH=$PWD
for tool in memcheck synccheck racecheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_cases.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|MISMATCHES|Error|error" gpurun_out/sanitize_$tool.log | sort | uniq -c | head -8
done
