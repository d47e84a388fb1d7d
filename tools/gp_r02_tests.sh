# round 2: run the given GPU test files (default: all) on the B200, output to gpurun_out/
T=${1:-tests}
timeout 1200 python -m pytest $T -m gpu -x -q 2>&1 | tail -25 > gpurun_out/r02_gputests_sel.txt
cat gpurun_out/r02_gputests_sel.txt
