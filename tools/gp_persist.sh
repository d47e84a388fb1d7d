python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_halo.py tests/test_gpu_edge.py -m gpu -x -q > gpurun_out/persist_tests.log 2>&1
tail -3 gpurun_out/persist_tests.log
b() { python bench.py --no-cpu-baseline --steps 300 "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,3), round(d['kernel_ms']['node_stage_ms']*1000,1), round(d['kernel_ms']['zone_stage_ms']*1000,1))"; }
for P in 0 1; do for K in 0 8 11 13 22 43; do echo "persist=$P kz=$K $(HYDRO_NODE_PERSIST=$P HYDRO_KZ_NODE=$K b)"; done; done
for C in weak384 sedov512 uneven448; do for P in 0 1; do echo "$C persist=$P $(HYDRO_NODE_PERSIST=$P b --config $C --steps 30 --warmup 3)"; done; done
