bash tools/gpu_jobs.sh tests
python tools/shape_sweep.py --figs 17 --steps 5 --max-zones 5e6 2>&1 | grep -v Warn | head -4
HYDRO_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29531 tools/shape_sweep.py --figs 17 --steps 5 --max-zones 3e6 2>&1 | grep -v Warn | grep "{" | head -3
HYDRO_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29532 bench.py --gpus 2 --steps 5 --warmup 3 --e2e-steps 2 --e2e-cycles 5 > gpurun_out/bench_n2.json 2> gpurun_out/bench_n2.err
tail -3 gpurun_out/bench_n2.err | cut -c1-300; head -c 600 gpurun_out/bench_n2.json
