export PYTHONPATH=.
timeout 600 python bench.py --no-cpu-baseline --steps 300 > gpurun_out/ab_warp.json 2>/dev/null
HYDRO_LIB=$PWD/build/libhydro_arrall.so timeout 600 python bench.py --no-cpu-baseline --steps 300 > gpurun_out/ab_all.json 2>/dev/null
for f in gpurun_out/ab_warp.json gpurun_out/ab_all.json; do python -c "import json; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), {k:round(v*1e3,1) for k,v in d['kernel_ms'].items()})"; done
echo "=== racecheck per-thread arrive"
HYDRO_LIB=$PWD/build/libhydro_arrall.so timeout 1200 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 4 python tools/sanitize_run.py single 2>&1 | grep -E "SUMMARY|^single" | head
