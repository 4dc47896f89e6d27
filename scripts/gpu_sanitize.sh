for tool in memcheck racecheck synccheck; do
  timeout -s KILL 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python scripts/sanitize.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|========= " gpurun_out/sanitize_$tool.log | tail -3
done
