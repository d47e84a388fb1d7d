"""A/B timing helper: zone-cycles/s of one bench workload and path (CUDA events, graph-replayed
cycles, as bench.py times them), for the library selected by HYDRO_LIB.

    python tools/ab_time.py CONFIG PATH [STEPS] [REPEATS]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig  # noqa: E402

cfg, path = sys.argv[1], sys.argv[2]
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 20
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 3
kw, _, _, _ = bench.workload(cfg, 1)
n = kw["n"]
zones = n[0] * n[1] * n[2]
with Hydro(HydroConfig(path=path, **kw)) as h:
    s = torch.cuda.current_stream()
    h.step(5, stream=s.cuda_stream)
    vals = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record(s)
        info = h.step(steps, stream=s.cuda_stream)
        b.record(s)
        torch.cuda.synchronize()
        vals.append(zones * steps / (a.elapsed_time(b) * 1e-3))
    kt = h.time_kernels(min(steps, 20))
print(json.dumps({"lib": os.path.basename(os.environ.get("HYDRO_LIB", "default")), "config": cfg,
                  "path": path, "G": [round(v / 1e9, 3) for v in vals], "status": info["status"],
                  "kt": {k: round(v * 1e3, 1) for k, v in kt.items()}}), flush=True)
