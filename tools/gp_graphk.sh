python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
b() { python bench.py --no-cpu-baseline "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,3), round(d['ms_per_step']*1000,1))"; }
for i in 1 2; do for K in 1 2 4 8; do echo "128 K=$K $(HYDRO_GRAPH_CYCLES=$K b --steps 400)"; done; done
for C in weak384 uneven448 sedov512; do for K in 1 4; do echo "$C K=$K $(HYDRO_GRAPH_CYCLES=$K b --config $C --steps 40 --warmup 4)"; done; done
timeout 900 python -m pytest tests/ -m gpu -x -q 2>&1 | tail -2
