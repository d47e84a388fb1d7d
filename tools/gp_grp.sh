python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
b() { python bench.py --no-cpu-baseline "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernel_ms']; print(round(d['value']/1e9,3), round(d['ms_per_step']*1000,1), 'node', round(k['node_stage_ms']*1000,1))"; }
for C in uneven448 weak384 sedov512; do for G in 0 1; do echo "$C group_node=$G $(HYDRO_GROUP_NODE=$G b --config $C --steps 40 --warmup 4)"; done; done
