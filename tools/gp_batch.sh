# hydro_run_batch: GPU tests, then the default bench line (e2e through run_batch).
timeout 900 python -m pytest tests/test_gpu_batch.py tests/test_gpu_parity.py -q -x > gpurun_out/gpu_tests.log 2>&1
tail -15 gpurun_out/gpu_tests.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
python -c "import json; d=json.loads(open('gpurun_out/bench.json').read()); print(d['value']/1e9, json.dumps(d['e2e']))"
tail -3 gpurun_out/bench.err
