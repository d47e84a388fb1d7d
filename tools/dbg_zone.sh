# debug: zone kernel with old (-1) and new (0) ring origin
for V in 0 1; do
  HYDRO_NVCC_FLAGS="-DHYDRO_DBG_RING=$V" python -c "from paper_conf_icppw_pearce18_b200 import _build as b; b.build(force=True)" > /dev/null 2>&1
  echo "RING=$V"; PYTHONPATH=. CUDA_LAUNCH_BLOCKING=1 timeout 120 python tools/dbg_step.py 2>&1 | tail -2
done
