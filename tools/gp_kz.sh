# KZ sweep via environment overrides (zone stage, node stage)
for Z in 0 4 8 16 32; do
  echo "KZ_ZONE=$Z $(HYDRO_KZ_ZONE=$Z python bench.py --no-cpu-baseline --steps 100 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernel_ms']; print(round(d['value']/1e9,3), 'zone', round(k['zone_stage_ms']*1e3,1), 'node', round(k['node_stage_ms']*1e3,1))")"
done
for N in 0 6 8 10 16 22 32; do
  echo "KZ_NODE=$N $(HYDRO_KZ_NODE=$N python bench.py --no-cpu-baseline --steps 100 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernel_ms']; print(round(d['value']/1e9,3), 'zone', round(k['zone_stage_ms']*1e3,1), 'node', round(k['node_stage_ms']*1e3,1))")"
done
