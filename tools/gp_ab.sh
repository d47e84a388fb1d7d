# GPU tests, then multi-domain configs grouped vs per-domain launches.
timeout 1200 python -m pytest tests/ -m gpu -q -x > gpurun_out/gpu_tests.log 2>&1
tail -3 gpurun_out/gpu_tests.log
for c in uneven448 weak384 sedov512; do
timeout 600 python bench.py --no-cpu-baseline --steps 100 --config $c > gpurun_out/ab_grp_$c.json 2>gpurun_out/ab_grp_$c.err
HYDRO_NO_GROUP=1 timeout 600 python bench.py --no-cpu-baseline --steps 100 --config $c > gpurun_out/ab_nogrp_$c.json 2>/dev/null
done
for f in gpurun_out/ab_*.json; do python -c "import json,sys; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), round(d['ms_per_step']*1e3,1), {k:round(v*1e3,1) for k,v in d['kernel_ms'].items()})"; done
tail -3 gpurun_out/ab_grp_uneven448.err
