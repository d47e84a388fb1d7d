# round-2 measurement set: full GPU suite, default bench line, ncu launch list of the same
# command, compute-sanitizer on every path
bash tools/gpu_jobs.sh tests
bash tools/gpu_jobs.sh bench --steps 20 --warmup 5
bash tools/gpu_jobs.sh launches
rm -f gpurun_out/sanitize.txt
for tool in memcheck racecheck synccheck; do
  echo "== $tool" >> gpurun_out/sanitize.txt
  timeout 900 compute-sanitizer --tool $tool --print-limit 10 python tools/sanitize_run.py >> gpurun_out/sanitize.txt 2>&1
  echo "rc=$?" >> gpurun_out/sanitize.txt
done
grep -E "==|rc=|SUMMARY" gpurun_out/sanitize.txt | head -20
