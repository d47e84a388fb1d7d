# GPU tests + smoke + default bench line.
python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
timeout 1500 python -m pytest tests/ -m gpu -q > gpurun_out/gpu_tests.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err
cat gpurun_out/smoke.log; tail -25 gpurun_out/gpu_tests.log
python -c "import json; d=json.loads(open('gpurun_out/bench_quick.json').read()); print(d['value']/1e9, d['kernel_ms'])"
