python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_halo.py tests/test_gpu_multirank.py -m gpu -x -q > gpurun_out/halo_tests.log 2>&1
for C in uneven448 weak384 sedov512; do
  for H in fused kernel; do
    timeout 600 python bench.py --no-cpu-baseline --config $C --halo $H --steps 30 --warmup 3 > gpurun_out/halo_${C}_${H}.json 2> gpurun_out/halo_${C}_${H}.err
  done
done
timeout 600 python bench.py --no-cpu-baseline --steps 300 > gpurun_out/halo_sedov128.json 2> gpurun_out/halo_sedov128.err
tail -3 gpurun_out/halo_tests.log
for f in gpurun_out/halo_*.json; do python -c "import json,sys; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), {k: round(v,4) for k,v in d['kernel_ms'].items()})" 2>/dev/null || (echo $f; tail -3 ${f%.json}.err); done
