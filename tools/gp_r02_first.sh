set -x
free -g | head -2; nproc
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/r02_gputests.txt
cat gpurun_out/r02_gputests.txt
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err
tail -3 gpurun_out/r02_bench.err; cat gpurun_out/r02_bench.json | head -c 3000
