b() { python bench.py --no-cpu-baseline "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernel_ms']; print(round(d['value']/1e9,3), 'node', round(k['node_stage_ms']*1000,1), 'zone', round(k['zone_stage_ms']*1000,1))"; }
for i in 1 2; do
for V in base zbal; do echo "128 $V $(HYDRO_LIB=$PWD/build/libhydro_$V.so b --steps 300)"; done
done
for C in weak384 uneven448; do for V in base zbal; do echo "$C $V $(HYDRO_LIB=$PWD/build/libhydro_$V.so b --config $C --steps 30 --warmup 3)"; done; done
HYDRO_LIB=$PWD/build/libhydro_zbal.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "two" 2>&1 | tail -1
