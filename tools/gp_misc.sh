# compute-sanitizer on every cycle path, then the paper shape sweeps.
bash tools/gp_sanitize.sh > gpurun_out/sanitizer.txt 2>&1
cat gpurun_out/sanitizer.txt
timeout 1800 python tools/shape_sweep.py > gpurun_out/shape_sweep.jsonl 2> gpurun_out/shape_sweep.err
tail -3 gpurun_out/shape_sweep.err; wc -l gpurun_out/shape_sweep.jsonl
