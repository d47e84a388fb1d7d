# A/B: node-stage streams by LPT on domain sizes (HYDRO_NODE_LPT=1) vs index round-robin (0).
timeout 900 python -m pytest tests/test_gpu_halo.py tests/test_gpu_fullsize.py -q -x > gpurun_out/gpu_tests.log 2>&1
tail -2 gpurun_out/gpu_tests.log
rm -f gpurun_out/lpt_*.json
for C in uneven448 sedov512 weak384; do for L in 0 1; do
  HYDRO_NODE_LPT=$L timeout 600 python bench.py --no-cpu-baseline --config $C --steps 30 --warmup 3 > gpurun_out/lpt_${C}_$L.json 2> gpurun_out/lpt_${C}_$L.err
done; done
for f in gpurun_out/lpt_*.json; do python -c "import json; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), round(d['ms_per_step'],3))"; done
