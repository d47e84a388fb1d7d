# round-2 measurement set: default bench line, ncu launch list of the same command, one ncu --set
# full capture of each cycle kernel at the headline config, compute-sanitizer on every path
bash tools/gpu_jobs.sh bench --steps 20 --warmup 5
bash tools/gpu_jobs.sh launches
bash tools/gpu_jobs.sh ncu sedov512 "k_zone_stage|k_cycle|k_halo_copy|k_finalize"
for tool in memcheck racecheck synccheck; do
  echo "== $tool" >> gpurun_out/sanitize.txt
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py >> gpurun_out/sanitize.txt 2>&1
  echo "rc=$?" >> gpurun_out/sanitize.txt
done
grep -E "==|rc=|ERROR SUMMARY|hazard" gpurun_out/sanitize.txt | head -20
