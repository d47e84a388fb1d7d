# Round evidence (tools/gp_round.sh) plus the ncu SASS/summary inputs and the shape sweep.
bash tools/gp_round.sh
timeout 1500 python tools/shape_sweep.py > gpurun_out/shape_sweep.jsonl 2> gpurun_out/shape_sweep.err
wc -l gpurun_out/shape_sweep.jsonl
