"""Wall-clock breakdown of bench.py's e2e step (set_state H2D | 100 cycles | get_fields D2H)."""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig

names = ("x", "y", "z", "u", "v", "w", "e")
with Hydro(HydroConfig(n=(128, 128, 128))) as h:
    h.step(10)
    cur = h.fields(names)
    pinned = {k: torch.from_numpy(v).pin_memory().numpy() for k, v in cur.items()}
    out = {k: torch.empty(v.shape, dtype=torch.float64).pin_memory().numpy() for k, v in cur.items()}
    inf = h.info()
    for rep in range(4):
        t0 = time.perf_counter()
        h.set_state(pinned, pinned["e"], inf["t"], inf["dt"])
        t1 = time.perf_counter()
        h.step(100)
        t2 = time.perf_counter()
        h.fields(names, out=out)
        t3 = time.perf_counter()
        print(f"set_state {1e3 * (t1 - t0):.2f} ms  step(100) {1e3 * (t2 - t1):.2f} ms  "
              f"fields {1e3 * (t3 - t2):.2f} ms  total {1e3 * (t3 - t0):.2f} ms")
