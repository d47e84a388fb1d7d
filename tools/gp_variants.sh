# Build and bench variants given as arguments (each a quoted set of -D flags); prints stage times.
for V in "$@"; do
  HYDRO_NVCC_FLAGS="$V" python -c "from paper_conf_icppw_pearce18_b200 import _build as b; b.build(force=True)" > /dev/null 2>&1 || { echo "$V build failed"; continue; }
  python bench.py --no-cpu-baseline --steps 100 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernel_ms']; print('$V', round(d['value']/1e9,3), 'zone', round(k['zone_stage_ms']*1e3,1), 'node', round(k['node_stage_ms']*1e3,1))"
done
