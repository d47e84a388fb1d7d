"""Profiling driver (no timing): create a bench.py workload and run a few cycles, so that ncu /
compute-sanitizer see exactly the kernels of that launch configuration.

    python tools/prof_run.py [config] [cycles] [path]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "sedov512"
cyc = int(sys.argv[2]) if len(sys.argv) > 2 else 4
path = sys.argv[3] if len(sys.argv) > 3 else "two"
kw, _, desc, _ = bench.workload(name, 1)
with Hydro(HydroConfig(path=path, **kw)) as h:
    info = h.step(cyc)
print(desc, info)
