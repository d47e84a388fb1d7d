"""GPU parity on Saltzman's skewed-mesh piston (tests/test_oracle_saltzman.py): every path and
variant against the oracle on a strongly distorted mesh with a moving wall -- the fast paths
within the north_star tolerance, STRICT bit for bit."""
import numpy as np
import pytest

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from tests.helpers import rel_err
from tests.test_oracle_saltzman import G, saltzman_state

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")


@pytest.mark.parametrize("path,q,hg", [("two", "scalar", 0.0), ("one", "scalar", 0.0),
                                       ("split", "scalar", 0.03), ("split", "monotone", 0.03),
                                       ("strict", "scalar", 0.0), ("strict", "monotone", 0.0)])
def test_saltzman_against_oracle(path, q, hg):
    n, ext, s = saltzman_state()
    kw = dict(n=n, extent=ext, init="user", user=s, gamma=G, q=q, hg_coef=hg)
    for nc, tol in ((1, 1e-12), (100, 1e-10)):
        fo, io = oracle.run(OracleConfig(**kw), nc)
        with Hydro(HydroConfig(path=path, **kw)) as h:
            ig = h.step(nc)
            fg = h.fields()
        assert ig["status"] == 0 == io["status"]
        for k in FIELDS:
            if path == "strict":
                assert np.array_equal(fg[k].view(np.uint64), fo[k].view(np.uint64)), (nc, k)
            elif k == "w":  # exactly 0 (the mesh is one zone thick in z): round-off only (R15)
                assert float(np.abs(fg[k] - fo[k]).max()) <= tol * float(np.abs(fo["u"]).max())
            else:
                assert rel_err(fg[k], fo[k]) <= tol, (nc, k, rel_err(fg[k], fo[k]))
