python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_halo.py tests/test_gpu_edge.py -m gpu -x -q 2>&1 | tail -1
b() { python bench.py --no-cpu-baseline "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernel_ms']; print(round(d['value']/1e9,3), round(d['ms_per_step']*1000,1), 'zone', round(k['zone_stage_ms']*1000,1))"; }
for i in 1 2; do for E in 0 1; do echo "128 early=$E $(HYDRO_ZONE_EARLY=$E b --steps 400)"; done; done
for C in weak384 uneven448; do for E in 0 1; do echo "$C early=$E $(HYDRO_ZONE_EARLY=$E b --config $C --steps 40 --warmup 4)"; done; done
