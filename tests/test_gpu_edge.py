"""GPU edge cases against the oracle: degenerate meshes (one zone, one-zone-thick meshes and
domains, a domain one zone wide between two others), every cycle path, and the size limit.

The oracle accepts any n >= 1 and any cuts with >= 1 zone per domain; so does the library.  A
1-zone-thick domain has interface nodes on both sides and ghost layers that are the neighbours'
owned zones, which exercises every ghost-slab direction with the smallest possible boxes.
"""
import numpy as np
import pytest

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig, HydroError
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")

CASES = [
    dict(n=(1, 1, 1)),
    dict(n=(2, 1, 1)),
    dict(n=(5, 1, 3)),
    dict(n=(3, 3, 3), ndom=(3, 1, 1)),                       # three 1-zone-thick x-slabs
    dict(n=(7, 5, 4), ndom=(3, 3, 2), cuts=[[0, 3, 4, 7], [0, 1, 4, 5], [0, 1, 4]]),
    dict(n=(33, 9, 2), ndom=(2, 1, 2), cuts=[[0, 32, 33], [0, 9], [0, 1, 2]]),
]


@pytest.mark.parametrize("path", ["two", "one", "split"])
@pytest.mark.parametrize("case", range(len(CASES)))
def test_degenerate_meshes_match_oracle(case, path):
    kw = dict(CASES[case])
    n = kw["n"]
    kw.update(init="user", user=jittered_state(n, 7 + case))
    okw = {k: v for k, v in kw.items() if k in ("n", "ndom", "cuts", "init", "user")}
    fo, io = oracle.run(OracleConfig(**okw), 12)
    with Hydro(HydroConfig(path=path, **kw)) as h:
        ig = h.step(12)
        fg = h.fields()
    assert ig["status"] == io["status"] == 0
    assert ig["dt"] == pytest.approx(io["dt"], rel=1e-11)
    for k in FIELDS:
        assert rel_err(fg[k], fo[k]) <= 1e-11, k


def test_domain_storage_limit_rejected():
    """A domain whose storage would exceed 2^31 nodes is refused before any allocation."""
    with pytest.raises(HydroError) as ei:
        Hydro(HydroConfig(n=(1300, 1300, 1300)))
    assert ei.value.code == -1
