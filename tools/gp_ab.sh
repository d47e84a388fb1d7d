# A/B of kernel variants: bench per variant (kernel_ms per stage).
run() { name=$1; shift; env "$@" timeout 600 python bench.py --no-cpu-baseline --steps 300 > gpurun_out/ab_$name.json 2> gpurun_out/ab_$name.err; }
run tma_pers X=1
run tma_chunk HYDRO_KZ_NODE=13
run ldg_chunk HYDRO_KZ_NODE=13 HYDRO_LIB=$PWD/build/libhydro_ldg.so
run ldg_pers HYDRO_LIB=$PWD/build/libhydro_ldg.so
run zchunk HYDRO_KZ_ZONE=15 HYDRO_KZ_NODE=13 HYDRO_LIB=$PWD/build/libhydro_ldg.so
for f in gpurun_out/ab_*.json; do python -c "import json,sys; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), {k:round(v*1e3,1) for k,v in d['kernel_ms'].items()})"; done
