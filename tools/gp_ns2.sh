python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
b() { python bench.py --no-cpu-baseline "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernel_ms']; print(round(d['value']/1e9,3), round(d['ms_per_step']*1000,1), 'node', round(k['node_stage_ms']*1000,1))"; }
for K in 0 16 32 48 1000; do echo "uneven448 streams=4 kz=$K $(HYDRO_NODE_STREAMS=4 HYDRO_KZ_NODE=$K b --config uneven448 --steps 40 --warmup 4)"; done
for K in 0 1000; do echo "uneven448 streams=8? kz=$K $(HYDRO_NODE_STREAMS=4 HYDRO_KZ_NODE=$K HYDRO_NODE_TY=12 b --config uneven448 --steps 40 --warmup 4)"; done
