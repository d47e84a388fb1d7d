# A/B: node-stage tile height TY=12 (default) vs TY=11 (build/libhydro_ty11.so)
b() { python bench.py --no-cpu-baseline "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value']/1e9,3), round(d['kernel_ms']['node_stage_ms']*1000,1), round(d['kernel_ms']['zone_stage_ms']*1000,1))"; }
HYDRO_LIB=$PWD/build/libhydro_ty11.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "two" > gpurun_out/ty11_tests.log 2>&1; tail -2 gpurun_out/ty11_tests.log
for i in 1 2; do
echo "128 ty12 $(b --steps 300)"
echo "128 ty11 $(HYDRO_LIB=$PWD/build/libhydro_ty11.so b --steps 300)"
done
for C in weak384 sedov512 uneven448; do
echo "$C ty12 $(b --config $C --steps 30 --warmup 3)"
echo "$C ty11 $(HYDRO_LIB=$PWD/build/libhydro_ty11.so b --config $C --steps 30 --warmup 3)"
done
