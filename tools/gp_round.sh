# One GPU session: build check, tests, bench, ncu launch list and a full capture of the fused kernel.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
timeout 900 python -m pytest tests/ -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python bench.py --split --no-cpu-baseline > gpurun_out/bench_split.json 2> gpurun_out/bench_split.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_cycle_fused -s 5 -c 2 -o gpurun_out/prof_fused python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/gpu_tests.log
cat gpurun_out/bench.json gpurun_out/bench_split.json
