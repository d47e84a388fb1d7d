# A/B of the folded finalize (-DHYDRO_FOLD: S9 in the node stage's last CTA, single domain only)
# against the separate k_finalize kernel at 128^3, alternating builds.
for f in "" "-DHYDRO_FOLD" "" "-DHYDRO_FOLD"; do
  HYDRO_NVCC_FLAGS="$f" python -c "from paper_conf_icppw_pearce18_b200 import _build as b; b.build(force=True)"
  python bench.py --no-cpu-baseline --e2e-steps 2 > gpurun_out/fold.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/fold.log').read().strip().splitlines()[-1]);k=d['roofline']['kernels'];print('FOLD=[$f]',round(d['value']/1e9,3),round(d['ms_per_step']*1e3,1),d['gpu_launches'],round(k[1]['ms']*1e3,1))"
done
HYDRO_NVCC_FLAGS="-DHYDRO_FOLD" python -c "from paper_conf_icppw_pearce18_b200 import _build as b; b.build(force=True)"
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py tests/test_gpu_batch.py -x -q 2>&1 | tail -2
