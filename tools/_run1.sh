for tool in memcheck racecheck initcheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|Program hit' gpurun_out/sanitize_$tool.log | tail -2 | tr '\n' ' ')"
done
bash tools/profile_round.sh r01
