# Quick GPU iteration: parity tests, bench per path, one ncu capture per cycle kernel.
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
timeout 900 python -m pytest tests/ -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for P in two one; do
  timeout 600 python bench.py --no-cpu-baseline --path $P > gpurun_out/bench_$P.json 2> gpurun_out/bench_$P.err
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_zone_stage|k_cycle" -s 10 -c 2 -o gpurun_out/prof_two python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
cat gpurun_out/smoke.log; tail -15 gpurun_out/gpu_tests.log
for P in two one; do python -c "import json; d=json.loads(open('gpurun_out/bench_$P.json').read()); print('$P', d['value']/1e9, d['kernel_ms'])"; tail -2 gpurun_out/bench_$P.err; done
