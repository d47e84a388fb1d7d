python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
b() { python bench.py --no-cpu-baseline "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernel_ms']; print(round(d['value']/1e9,3), round(d['ms_per_step']*1000,1), 'node', round(k['node_stage_ms']*1000,1))"; }
for C in uneven448 weak384 sedov512; do for N in 1 2 4; do echo "$C streams=$N $(HYDRO_NODE_STREAMS=$N b --config $C --steps 40 --warmup 4)"; done; done
HYDRO_NODE_STREAMS=4 timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_halo.py -m gpu -x -q -k "multi or halo or fused" 2>&1 | tail -1
