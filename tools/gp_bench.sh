# Default bench line (with cpu_baseline) + the one-kernel path line + the launch list of the bench command.
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 python bench.py --no-cpu-baseline --path one > gpurun_out/bench_one.json 2> gpurun_out/bench_one.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
python -c "import json; d=json.loads(open('gpurun_out/bench.json').read()); print(d['value']/1e9, d['clocks'], d['e2e']['value']/1e9)"
python -c "import json; d=json.loads(open('gpurun_out/bench_one.json').read()); print(d['value']/1e9)"
