python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/ -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; tail -3 gpurun_out/gpu_tests.log
b() { python bench.py --no-cpu-baseline "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,3), round(d['kernel_ms']['node_stage_ms']*1000,1), round(d['kernel_ms']['zone_stage_ms']*1000,1))"; }
echo "128 $(b --steps 300)"
for C in weak384 sedov512 uneven448 sedov32; do echo "$C $(b --config $C --steps 30 --warmup 3)"; done
