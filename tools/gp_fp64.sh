nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/fp64_peak.txt
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/fp64_clocks.csv &
P=$!
./tools/fp64_peak >> gpurun_out/fp64_peak.txt 2>&1
kill $P
lscpu | head -20 >> gpurun_out/fp64_peak.txt; nproc >> gpurun_out/fp64_peak.txt; free -g >> gpurun_out/fp64_peak.txt
