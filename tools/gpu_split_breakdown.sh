# per-kernel durations and DRAM bytes of the split path with hourglass + monotone q at 512^3
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_zone_split|k_node_split|k_energy_split|k_strain" -s 32 -c 32 --csv python -c "
import sys; sys.path.insert(0,'.')
import bench
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
kw=bench.workload('sedov512',1)[0]
with Hydro(HydroConfig(path='split', hg_coef=0.03, q='monotone', graph=False, **kw)) as h: h.step(3)
" 2>/dev/null > gpurun_out/split_breakdown.csv
python - <<'PY'
import csv, collections
rows = [r for r in csv.reader(open('gpurun_out/split_breakdown.csv')) if len(r) > 10]
h = rows[0]; ki, mi, vi = h.index('Kernel Name'), h.index('Metric Name'), h.index('Metric Value')
agg = collections.defaultdict(lambda: collections.defaultdict(list))
for r in rows[1:]:
    agg[r[ki].split('(')[0].split('::')[-1]][r[mi]].append(float(r[vi].replace(',', '')))
for k, m in agg.items():
    n = len(m['gpu__time_duration.sum'])
    t = sum(m['gpu__time_duration.sum']) / n / 1e3
    rd = sum(m['dram__bytes_read.sum']) / n / 16.78e6; wr = sum(m['dram__bytes_write.sum']) / n / 16.78e6
    print(f"{k:18s} n={n:2d} {t:8.1f} us/domain  read {rd:6.1f} B/zone  write {wr:6.1f} B/zone")
PY
