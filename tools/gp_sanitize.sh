export PYTHONPATH=.
for tool in memcheck racecheck synccheck; do
  echo "== $tool"
  timeout 900 compute-sanitizer --tool $tool --print-limit 10 python tools/sanitize_run.py two one split hg single fused ty11 ty12 2>&1 | grep -E "ERROR SUMMARY|RACECHECK SUMMARY|Hazard|Invalid|error|^two|^one|^split|^hg|^single|^fused|^ty1" | head -20
done
