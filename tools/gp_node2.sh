HYDRO_NODE_KERNEL=2 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "two or restart or tangled or t_stop or full_size" 2>&1 | tail -3
for V in 1 2 1 2; do
  echo "NODE=$V $(HYDRO_NODE_KERNEL=$V python bench.py --no-cpu-baseline --steps 100 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernel_ms']; print(round(d['value']/1e9,3), 'zone', round(k['zone_stage_ms']*1e3,1), 'node', round(k['node_stage_ms']*1e3,1))")"
done
HYDRO_NODE_KERNEL=2 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_node2" -s 5 -c 1 -o gpurun_out/prof_node2 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
