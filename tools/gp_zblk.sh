# Zone-stage unit order: z-blocks of HYDRO_ZONE_ZBLK planes (0 = column-major), parity + A/B.
HYDRO_ZONE_ZBLK=5 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_halo.py -q -x > gpurun_out/gpu_tests_zb5.log 2>&1
tail -1 gpurun_out/gpu_tests_zb5.log
rm -f gpurun_out/zb_*.json
for Z in 0 16 24 32 43 64; do
  HYDRO_ZONE_ZBLK=$Z timeout 600 python bench.py --no-cpu-baseline --steps 1000 > gpurun_out/zb_$Z.json 2> gpurun_out/zb_$Z.err
done
for Z in 0 32; do
  HYDRO_ZONE_ZBLK=$Z timeout 600 python bench.py --no-cpu-baseline --config uneven448 --steps 30 --warmup 3 > gpurun_out/zb_u448_$Z.json 2> gpurun_out/zb_u448_$Z.err
  HYDRO_ZONE_ZBLK=$Z timeout 600 python bench.py --no-cpu-baseline --config weak384 --steps 30 --warmup 3 > gpurun_out/zb_w384_$Z.json 2> gpurun_out/zb_w384_$Z.err
done
for f in gpurun_out/zb_*.json; do python -c "import json; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), round(d['ms_per_step']*1e3,2), round(d['kernel_ms']['zone_stage_ms']*1e3,1))"; done
