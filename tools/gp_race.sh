export PYTHONPATH=.
timeout 900 python -m pytest tests/ -m gpu -q -x > gpurun_out/gpu_tests.log 2>&1
tail -2 gpurun_out/gpu_tests.log
for p in single two one; do
  echo "=== $p"
  timeout 900 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 4 python tools/sanitize_run.py $p 2>&1 | grep -E "SUMMARY|hazard|^single|^two|^one|in kernel" | sort | uniq -c | head -12
done
