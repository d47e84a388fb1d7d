# ncu of the intra-GPU halo copy (uneven 448^3, 64 domains) and the zone/node kernels of one small domain
timeout 900 ncu --set full --clock-control none -k regex:"k_halo_copy" -s 2 -c 1 -o gpurun_out/prof_halo python bench.py --steps 3 --warmup 3 --no-cpu-baseline --config uneven448 > gpurun_out/ncu_halo.log 2>&1
tail -3 gpurun_out/ncu_halo.log
