# New GPU tests only (hourglass + rebalance), then the whole GPU suite.
timeout 900 python -m pytest tests/test_gpu_hourglass.py tests/test_gpu_rebalance.py -q -x > gpurun_out/gpu_new.log 2>&1
tail -30 gpurun_out/gpu_new.log
timeout 1200 python -m pytest tests/ -m gpu -q > gpurun_out/gpu_tests.log 2>&1
tail -5 gpurun_out/gpu_tests.log
