# Zone-stage schedule sweep: persistent linear split (0) vs chunked with k planes per CTA.
for K in 0 26 32 43 64; do
  HYDRO_KZ_ZONE=$K timeout 600 python bench.py --no-cpu-baseline --steps 300 > gpurun_out/kzz_$K.json 2> gpurun_out/kzz_$K.err
done
for f in gpurun_out/kzz_*.json; do python -c "import json,sys; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), round(d['ms_per_step']*1e3,1), {k:round(v*1e3,1) for k,v in d['kernel_ms'].items()})"; done
