# Profile only: ncu full capture of the two cycle kernels of the default path.
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_zone_stage|k_cycle" -s 10 -c 2 -o gpurun_out/prof_two python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/ncu_full.log
