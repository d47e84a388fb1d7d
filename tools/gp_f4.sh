# GPU tests, every BASELINE config on both paths, and the paper shape sweeps.
timeout 900 python -m pytest tests/ -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
tail -2 gpurun_out/gpu_tests.log
bash tools/gp_configs.sh
timeout 1500 python tools/shape_sweep.py > gpurun_out/shape_sweep.jsonl 2> gpurun_out/shape_sweep.err
tail -3 gpurun_out/shape_sweep.err; wc -l gpurun_out/shape_sweep.jsonl
