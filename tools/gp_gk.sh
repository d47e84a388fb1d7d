# cycles per captured graph (HYDRO_GRAPH_CYCLES) at 128^3 and 32^3
for K in 1 8 16 32; do
  HYDRO_GRAPH_CYCLES=$K timeout 600 python bench.py --no-cpu-baseline --steps 400 > gpurun_out/gk_128_$K.json 2> gpurun_out/gk_128_$K.err
  HYDRO_GRAPH_CYCLES=$K timeout 600 python bench.py --no-cpu-baseline --config sedov32 --steps 400 > gpurun_out/gk_32_$K.json 2> gpurun_out/gk_32_$K.err
done
for f in gpurun_out/gk_*.json; do python -c "import json; d=json.loads(open('$f').read()); print('$f', round(d['value']/1e9,3), round(d['ms_per_step']*1e3,2))"; done
