run() { name=$1; shift; env "$@" timeout 600 python bench.py --no-cpu-baseline --steps 300 > gpurun_out/ab_$name.json 2> gpurun_out/ab_$name.err; }
for i in 1 2; do
run zby8_$i X=1
run zby16_$i HYDRO_LIB=$PWD/build/libhydro_zby16.so
run zby4_$i HYDRO_LIB=$PWD/build/libhydro_zby4.so
done
for f in gpurun_out/ab_zby*.json; do python -c "import json,sys; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), round(d['ms_per_step']*1e3,1), {k:round(v*1e3,1) for k,v in d['kernel_ms'].items()})"; done
tail -2 gpurun_out/ab_zby16_1.err
