timeout 900 python -m pytest tests/test_gpu_halo.py tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_multirank.py tests/test_gpu_rebalance.py tests/test_gpu_batch.py -m gpu -x -q 2>&1 | tail -4
for c in sedov512 weak384 uneven448; do
  HYDRO_PRING=0 python tools/ab_time.py $c two 20 3
  python tools/ab_time.py $c two 20 3
done 2>&1 | grep -v Warn | tee gpurun_out/r02_pring.txt
