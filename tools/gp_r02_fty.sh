L=paper_conf_icppw_pearce18_b200
for c in sedov128 sedov512; do
  python tools/ab_time.py $c two 20 3
  python tools/ab_time.py $c one 20 3
  for ty in 8 7 6 5; do HYDRO_LIB=$L/libhydro_fty$ty.so python tools/ab_time.py $c one 20 3; done
done 2>&1 | grep -v Warn | tee gpurun_out/r02_fty.txt
