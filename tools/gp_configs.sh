# Bench every BASELINE.json config on one GPU (both cycle paths).
for C in sedov32 sedov128 weak384 uneven448 sedov512; do
  for P in two one; do
    timeout 900 python bench.py --no-cpu-baseline --config $C --path $P --steps 30 --warmup 3 > gpurun_out/cfg_${C}_$P.json 2> gpurun_out/cfg_${C}_$P.err
    echo "$C $P $(python -c "import json; d=json.loads(open('gpurun_out/cfg_${C}_$P.json').read()); print(round(d['value']/1e9,3), d['config']['domains'], round(d['ms_per_step'],3), d['kernel_ms'])" 2>&1 | tail -1)"
  done
done
