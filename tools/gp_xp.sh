# A/B of zone-stage variants (HYDRO_LIB builds under build/), plus the GPU parity tests.
run() { name=$1; shift; env "$@" timeout 600 python bench.py --no-cpu-baseline --steps 300 > gpurun_out/ab_$name.json 2> gpurun_out/ab_$name.err; }
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py -q -x > gpurun_out/gpu_tests.log 2>&1
tail -3 gpurun_out/gpu_tests.log
rm -f gpurun_out/ab_*.json
for i in 1 2; do
for V in $AB; do run ${V}_$i HYDRO_LIB=$PWD/build/libhydro_$V.so; done
done
for f in gpurun_out/ab_*.json; do python -c "import json,sys; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), round(d['ms_per_step']*1e3,1), {k:round(v*1e3,1) for k,v in d['kernel_ms'].items()})"; done
