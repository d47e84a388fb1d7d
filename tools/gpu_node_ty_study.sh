# (study build: tools/build_variant.py nty8 -DHYDRO_NODE_TY_EXTRA=8 with the A/B hook of that commit; hook removed after the study)
L=paper_conf_icppw_pearce18_b200
for c in sedov512 sedov128 weak384; do
  python tools/ab_time.py $c two 20 3
  HYDRO_LIB=$L/libhydro_nty8.so HYDRO_NODE_TY=8 python tools/ab_time.py $c two 20 3
  HYDRO_LIB=$L/libhydro_nty10.so HYDRO_NODE_TY=10 python tools/ab_time.py $c two 20 3
done 2>&1 | grep -v Warn | tee gpurun_out/r02_node_ty.txt
