# GPU-box jobs used during development (run through gpurun from the repo root):
#   bash tools/gpu_jobs.sh tests [pytest targets...]   -m gpu suite -> gpurun_out/gputests.txt
#   bash tools/gpu_jobs.sh bench [bench.py args...]     default bench line -> gpurun_out/bench.json
#   bash tools/gpu_jobs.sh ncu CONFIG [REGEX]           ncu --set full of one launch of each kernel
#   bash tools/gpu_jobs.sh launches                     ncu launch list of the default bench
#   bash tools/gpu_jobs.sh ab CONFIG PATH ENV=VAL ...   A/B timing (tools/ab_time.py) per env setting
set -u
job=${1:-tests}; shift || true
mkdir -p gpurun_out
case "$job" in
  tests)
    timeout 1500 python -m pytest ${@:-tests} -m gpu -q 2>&1 | tail -30 > gpurun_out/gputests.txt
    cat gpurun_out/gputests.txt ;;
  bench)
    timeout 900 python bench.py "$@" > gpurun_out/bench.json 2> gpurun_out/bench.err
    tail -3 gpurun_out/bench.err; head -c 4000 gpurun_out/bench.json ;;
  ncu)
    cfg=${1:-sedov512}; re=${2:-k_zone_stage|k_cycle}
    timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"$re" -s 4 -c 3 \
      -o gpurun_out/prof_$cfg -f python tools/prof_run.py $cfg 3 > gpurun_out/ncu_$cfg.log 2>&1
    tail -2 gpurun_out/ncu_$cfg.log ;;
  launches)
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv \
      --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline \
      --no-selfcheck --second "" > gpurun_out/launches_bench.log 2>&1
    tail -2 gpurun_out/launches_bench.log ;;
  ab)
    cfg=$1; path=$2; shift 2
    for kv in "$@"; do env $kv python tools/ab_time.py $cfg $path 20 3; done 2>&1 \
      | grep -v Warn | tee gpurun_out/ab.txt ;;
esac
