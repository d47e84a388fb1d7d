# A/B of nvcc/ptxas option sets (HYDRO_NVCC_FLAGS) on the default 128^3 bench, alternating builds.
run() {
  HYDRO_NVCC_FLAGS="$1" python -c "from paper_conf_icppw_pearce18_b200 import _build as b; b.build(force=True)" || { echo "build failed: $1"; return; }
  python bench.py --no-cpu-baseline --e2e-steps 2 > gpurun_out/flags.log 2>&1
  python -c "import json,sys;d=json.loads(open('gpurun_out/flags.log').read().strip().splitlines()[-1]);k=d['roofline']['kernels'];print('FLAGS=[$1]',round(d['value']/1e9,3),round(k[0]['ms']*1e3,1),round(k[1]['ms']*1e3,1))"
}
for rep in 1 2; do
  run ""
  run "-Xptxas --allow-expensive-optimizations=true"
  run "--extra-device-vectorization"
  run "-Xptxas -dlcm=cg"
done
