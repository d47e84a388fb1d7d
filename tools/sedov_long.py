"""Run the Sedov workload to t_stop on the GPU with hourglass control and report the shock
radius against the analytic Sedov solution (reading R16), cycles, wall time and throughput.

    python tools/sedov_long.py N [NDOM_Y] [KAPPA] [T_STOP]
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from oracle import sedov as sedov_mod  # noqa: E402  (the analytic solution only)
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig  # noqa: E402
from tests.helpers import sedov_radius, sedov_radius_tolerance  # noqa: E402

n = int(sys.argv[1])
ndy = int(sys.argv[2]) if len(sys.argv) > 2 else 1
kappa = float(sys.argv[3]) if len(sys.argv) > 3 else 0.03
t_stop = float(sys.argv[4]) if len(sys.argv) > 4 else 0.3
cfg = HydroConfig(n=(n, n, n), ndom=(1, ndy, 1), t_stop=t_stop, hg_coef=kappa)
with Hydro(cfg) as h:
    t0 = time.perf_counter()
    info = h.step(100000)
    el = time.perf_counter() - t0
    f = h.fields(("x", "y", "z", "rho", "e"))
R = sedov_radius(f, 1.2 / n)
Re = sedov_mod.shock_radius(t_stop, 8.0 * cfg.sedov_energy, 1.0, 1.4)
print(json.dumps({"n": n, "domains_y": ndy, "kappa": kappa, "t": info["t"], "status": info["status"],
                  "cycles": info["cycle"], "wall_s": el,
                  "zone_cycles_per_s": n ** 3 * info["cycle"] / el,
                  "R_num": R, "R_exact": Re, "rel_err": (R - Re) / Re,
                  "tolerance": sedov_radius_tolerance(1.2 / n, Re)}), flush=True)
