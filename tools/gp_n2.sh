# bench.py --gpus 2 with both ranks on the one B200 (HYDRO_SHARE_GPU=1; numbers meaningless, the
# run checks the N>1 launch path end to end), peer and nccl-free transports.
HYDRO_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --steps 50 --warmup 3 > gpurun_out/n2.json 2> gpurun_out/n2.err
echo rc=$?; cat gpurun_out/n2.json | head -c 600; echo; tail -3 gpurun_out/n2.err
HYDRO_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 bench.py --impl reference --gpus 2 --steps 3 --warmup 1 > gpurun_out/n2_ref.json 2> gpurun_out/n2_ref.err
echo rc=$?; cat gpurun_out/n2_ref.json | head -c 300
