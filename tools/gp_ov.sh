# A/B: intra-GPU halo copy per source domain right after its node stage (HYDRO_HALO_OVERLAP=1 on
# the node-stage streams, =2 on a dedicated halo stream) vs one copy after the join (=0).
for C in uneven448 weak384 sedov512; do
  for OV in 0 1 3; do
    HYDRO_HALO_OVERLAP=$OV timeout 600 python bench.py --no-cpu-baseline --config $C --steps 30 --warmup 3 > gpurun_out/ov_${C}_$OV.json 2> gpurun_out/ov_${C}_$OV.err
  done
done
timeout 1200 python -m pytest tests/test_gpu_halo.py -q -x > gpurun_out/gpu_tests.log 2>&1
tail -3 gpurun_out/gpu_tests.log
for f in gpurun_out/ov_*.json; do python -c "import json; d=json.loads(open('$f').read()); print('$f', d['value']/1e9, d['ms_per_step'])"; done
