python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_halo.py tests/test_gpu_multirank.py -m gpu -x -q > gpurun_out/hc_tests.log 2>&1; tail -2 gpurun_out/hc_tests.log
b() { python bench.py --no-cpu-baseline "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernel_ms']; print(round(d['value']/1e9,3), 'node', round(k['node_stage_ms']*1000,1), 'zone', round(k['zone_stage_ms']*1000,1), 'halo', round(k['halo_ms']*1000,1))"; }
for C in uneven448 weak384 sedov512; do echo "$C $(b --config $C --steps 30 --warmup 3)"; done
