# every BASELINE.json config on one B200 with the round-2 code (bench.py timing)
for c in sedov32 sedov128 sedov512 weak384 uneven448; do
  timeout 900 python bench.py --config $c --second "" --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 3 --e2e-cycles 50 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); r=d['roofline']
print(json.dumps({'config': '$c', 'workload': d['config']['workload'], 'G': round(d['value']/1e9,3), 'ms_per_cycle': round(d['ms_per_step'],4), 'e2e_G': round(d['e2e']['value']/1e9,3), 'dominant': r['kernel'], 'hbm_frac': round(r['frac'],3), 'selfcheck': (d.get('selfcheck') or {}).get('pass'), 'clock': d['clocks']['sm_mhz']}))"
done | tee gpurun_out/r02_all_configs.jsonl
