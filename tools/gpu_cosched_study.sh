# (study build: git show 5ecd0f5..HEAD~0 history; needs -DHYDRO_NODE_TY_HALF=5 -DHYDRO_RACE_COSCHED, removed after the study)
# co-scheduling study (DESIGN.md §14 lever 1): node stage at half-SM tiles (32x5, 256 threads,
# <= 128 registers, 113 KB) next to the zone stage; HYDRO_RACE_COSCHED runs both kernels of a
# cycle concurrently WITHOUT their dependency (timing only, results wrong)
L=paper_conf_icppw_pearce18_b200/libhydro_cosched.so
for c in sedov512 sedov128; do
  HYDRO_LIB=$L python tools/ab_time.py $c two 20 3
  HYDRO_LIB=$L HYDRO_NODE_TY=5 python tools/ab_time.py $c two 20 3
  HYDRO_LIB=$L HYDRO_NODE_TY=5 HYDRO_RACE_COSCHED=1 python tools/ab_time.py $c two 20 3
  HYDRO_LIB=$L HYDRO_RACE_COSCHED=1 python tools/ab_time.py $c two 20 3
done 2>&1 | grep -v Warn | tee gpurun_out/cosched.txt
