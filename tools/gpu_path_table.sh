# throughput of every cycle path at the headline config (512^3 in 8 domains), bench.py timing
for a in "--path two" "--path one" "--path split" "--path strict" "--path split --hg 0.03" "--path split --q monotone" "--path strict --q monotone --hg 0.03"; do
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-selfcheck --second "" --e2e-steps 2 --e2e-cycles 5 $a 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read()); c=d['config']
print(json.dumps({'args': '$a', 'G': round(d['value']/1e9,3), 'ms_per_cycle': round(d['ms_per_step'],3), 'path': c['path'], 'hg': c['hg_coef'], 'q': c['q']}))"
done | tee gpurun_out/r02_path_table.jsonl
