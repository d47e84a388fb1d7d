# A/B: zone-stage x_p ring ordered by mbarriers (HYDRO_ZONE_XPBAR=1) vs one __syncthreads/plane.
run() { name=$1; shift; env "$@" timeout 600 python bench.py --no-cpu-baseline --steps 300 > gpurun_out/ab_$name.json 2> gpurun_out/ab_$name.err; }
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -q -x > gpurun_out/gpu_tests.log 2>&1
tail -3 gpurun_out/gpu_tests.log
for i in 1 2; do
run xp1_$i HYDRO_LIB=$PWD/build/libhydro_xp1.so
run xp0_$i HYDRO_LIB=$PWD/build/libhydro_xp0.so
done
for f in gpurun_out/ab_xp*.json; do python -c "import json,sys; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), round(d['ms_per_step']*1e3,1), {k:round(v*1e3,1) for k,v in d['kernel_ms'].items()})"; done
tail -2 gpurun_out/ab_xp1_1.err
