# Quick GPU iteration: parity tests, bench, one ncu capture of the fused kernel.
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
timeout 900 python -m pytest tests/ -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_cycle_fused -s 5 -c 1 -o gpurun_out/prof_fused python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
cat gpurun_out/smoke.log; tail -15 gpurun_out/gpu_tests.log; cat gpurun_out/bench.json; tail -3 gpurun_out/bench.err
