# A/B: intra-GPU halo copy elements per thread per trip (build/libhydro_h{1,4,8}.so).
timeout 900 python -m pytest tests/test_gpu_halo.py -q -x > gpurun_out/gpu_tests.log 2>&1
tail -2 gpurun_out/gpu_tests.log
rm -f gpurun_out/hu_*.json
for C in uneven448 sedov512; do for V in h1 h4 h8; do
  HYDRO_LIB=$PWD/build/libhydro_$V.so timeout 600 python bench.py --no-cpu-baseline --config $C --steps 30 --warmup 3 > gpurun_out/hu_${C}_$V.json 2> gpurun_out/hu_${C}_$V.err
done; done
for f in gpurun_out/hu_*.json; do python -c "import json; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), round(d['ms_per_step'],3), round(d['kernel_ms']['halo_ms'],4))"; done
