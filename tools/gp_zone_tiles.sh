# Zone-stage tile height x CTAs/SM x deferred EOS (HYDRO_ZONE_BY / HYDRO_ZONE_MINB /
# HYDRO_ZONE_DEFER) at 128^3: fewer warps per SM but room for more registers per thread.
# (HYDRO_ZONE_DEFER was a removed experimental variant; with the current source it is a no-op.)
run() {
  HYDRO_NVCC_FLAGS="$1" python -c "from paper_conf_icppw_pearce18_b200 import _build as b; b.build(force=True)" || { echo "build failed: $1"; return; }
  python bench.py --no-cpu-baseline --e2e-steps 2 --steps 1000 > gpurun_out/zt.log 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/zt.log').read().strip().splitlines()[-1]);k=d['roofline']['kernels'];print('CFG=[$1]',round(d['value']/1e9,3),round(k[0]['ms']*1e3,1),round(k[1]['ms']*1e3,1))" || tail -3 gpurun_out/zt.log
}
run ""
run "-DHYDRO_ZONE_BY=6"
run "-DHYDRO_ZONE_BY=6 -DHYDRO_ZONE_DEFER=1"
run "-DHYDRO_ZONE_BY=12 -DHYDRO_ZONE_MINB=1"
run "-DHYDRO_ZONE_BY=12 -DHYDRO_ZONE_MINB=1 -DHYDRO_ZONE_DEFER=1"
run "-DHYDRO_ZONE_BY=4 -DHYDRO_ZONE_MINB=3 -DHYDRO_ZONE_DEFER=1"
run ""
