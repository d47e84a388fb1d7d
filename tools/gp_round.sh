# Round evidence: smoke, GPU tests, default bench line (with cpu_baseline), reference arm,
# ncu launch list of the bench command, ncu --set full of the two cycle kernels, every BASELINE
# config on the default path, the hourglass (split) path.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,driver_version --format=csv > gpurun_out/gpu.txt
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
timeout 1200 python -m pytest tests/ -m gpu -q > gpurun_out/gpu_tests.log 2>&1
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_zone_stage|k_cycle" -s 10 -c 2 -o gpurun_out/prof_two python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
for C in sedov32 sedov128 weak384 uneven448 sedov512; do
  timeout 900 python bench.py --no-cpu-baseline --config $C --steps 30 --warmup 3 > gpurun_out/cfg_${C}_two.json 2> gpurun_out/cfg_${C}_two.err
done
timeout 900 python bench.py --no-cpu-baseline --path split --steps 100 > gpurun_out/bench_split.json 2> gpurun_out/bench_split.err
timeout 900 python bench.py --no-cpu-baseline --hg 0.03 --steps 100 > gpurun_out/bench_hg.json 2> gpurun_out/bench_hg.err
tail -3 gpurun_out/gpu_tests.log; cat gpurun_out/bench.json gpurun_out/bench_ref.json
