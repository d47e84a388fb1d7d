"""Diagnostic: multi-domain (fused / kernel halo) and single-domain runs against the oracle."""
import sys
import numpy as np
sys.path.insert(0, ".")
import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err

F = ("x", "y", "z", "u", "v", "w", "e")
n = (70, 50, 90)
cuts = [[0, 33, 70], [0, 13, 37, 50], [0, 45, 90]]
user = jittered_state(n, 12)
nc = int(sys.argv[1]) if len(sys.argv) > 1 else 8
fo, io = oracle.run(OracleConfig(n=n, init="user", user=user), nc)
for name, kw in (("single", dict()), ("kernel", dict(ndom=(2, 3, 2), cuts=cuts, halo="kernel")),
                 ("fused", dict(ndom=(2, 3, 2), cuts=cuts, halo="fused")),
                 ("single_nograph", dict(graph=False))):
    with Hydro(HydroConfig(n=n, init="user", user=user, **kw)) as h:
        info = h.step(nc)
        f = h.fields()
    errs = {k: rel_err(f[k], fo[k]) for k in F}
    worst = max(errs, key=errs.get)
    d = np.abs(f[worst] - fo[worst])
    idx = np.unravel_index(np.argmax(d), d.shape)
    print(name, info["status"], {k: f"{v:.2e}" for k, v in errs.items()}, "worst at (z,y,x)", idx,
          flush=True)
