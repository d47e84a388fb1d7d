"""Small runs of every cycle path for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig  # noqa: E402
from paper_conf_icppw_pearce18_b200.inputs import jittered_state  # noqa: E402

n = (40, 30, 20)
cuts = [[0, 17, 40], [0, 12, 30], [0, 20]]
for path in sys.argv[1:] or ["two", "one", "split", "strict", "hg", "mono", "mono_strict",
                             "single", "fused", "ty11", "ty12"]:
    kw = dict(n=n, ndom=(2, 2, 1), cuts=cuts, init="user", user=jittered_state(n, 3), path=path,
              graph=False)
    if path == "hg":  # hourglass control (split kernels)
        kw.update(path="split", hg_coef=0.03)
    if path in ("mono", "mono_strict"):  # monotone q (split / STRICT kernels, owner lookups)
        kw.update(path="split" if path == "mono" else "strict", q="monotone")
    if path == "single":  # one domain: the persistent zone stage without grouping
        kw.update(path="two", ndom=(1, 1, 1), cuts=None)
    if path == "fused":  # ghost slabs stored from the node/energy stage's epilogue
        kw.update(path="two", halo="fused")
    os.environ.pop("HYDRO_NODE_TY", None)
    if path in ("ty11", "ty12"):  # each compiled node-stage tile height
        os.environ["HYDRO_NODE_TY"] = path[2:]
        kw.update(path="two")
    with Hydro(HydroConfig(**kw)) as h:
        r = h.step(3)
        f = h.fields(["e", "rho"])
        print(path, r["status"], float(f["e"].sum()), flush=True)
