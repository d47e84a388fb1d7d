# ncu --set full of one zone-stage and one node-stage launch of a bench workload
CFG=${1:-sedov512}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_zone_stage|k_cycle" -s 4 -c 2 -o gpurun_out/r02_prof_$CFG -f python tools/prof_run.py $CFG 3 > gpurun_out/r02_ncu_$CFG.log 2>&1
tail -3 gpurun_out/r02_ncu_$CFG.log
