# Tile-height sweep of the fused kernel (build variants on the box, bench each).
for TY in 8 10 12 14; do
  HYDRO_NVCC_FLAGS="-DHYDRO_FTY=$TY" python -c "from paper_conf_icppw_pearce18_b200 import _build as b; b.build(force=True)" > /dev/null 2>&1
  echo "TY=$TY $(python bench.py --no-cpu-baseline --steps 100 2>/dev/null | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"]/1e9, d["kernel_ms"]["cycle_kernel_ms"])')"
done
