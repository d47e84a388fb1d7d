"""GPU parity of the dt-collapse failure path (reading R23, HYDRO_EDTMIN) against the oracle.

The floor is placed between the zone-dt minima of two cycles of the oracle's own trajectory
(relative gap > 1e-4, far above the 1e-10 parity tolerance), so both sides must halt at the
same cycle with the same state; the Sedov corner-box collapse (the kappa = 0 scheme's failure
mode, DESIGN.md §13 f1) must halt on both sides at the same cycle with the default floor.
"""
import numpy as np
import pytest

import oracle
from oracle import Oracle, OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")


def _oracle_dtmins(n, s, ncyc):
    o = Oracle(OracleConfig(n=n, init="user", user=s, dt_floor=-1.0))
    seq = [o.step(1)["dt_min_zone"] for _ in range(ncyc)]
    o.close()
    return seq


@pytest.mark.parametrize("path,ndom", [("two", (1, 1, 1)), ("one", (1, 1, 1)),
                                       ("split", (1, 1, 1)), ("two", (2, 2, 1))])
def test_edtmin_same_cycle_and_state_as_oracle(path, ndom):
    n = (16, 16, 16)
    s = jittered_state(n, 1)
    seq = _oracle_dtmins(n, s, 12)
    c = 10
    prev = min(seq[:c - 1])
    assert seq[c - 1] < prev * (1 - 1e-4)
    floor = 0.5 * (seq[c - 1] + prev)
    fo, io = oracle.run(OracleConfig(n=n, init="user", user=s, dt_floor=floor), 100)
    assert io["status"] == -7 and io["cycle"] == c and io["bad_zone"] == -1
    with Hydro(HydroConfig(n=n, init="user", user=s, dt_floor=floor, path=path,
                           ndom=ndom)) as h:
        ig = h.step(100)
        fg = h.fields()
        assert ig["status"] == -7 and ig["rc"] == -7
        assert ig["cycle"] == c and ig["bad_zone"] == -1
        assert ig["t"] == pytest.approx(io["t"], rel=1e-12)
        assert ig["dt_min_zone"] == pytest.approx(io["dt_min_zone"], rel=1e-11)
        assert h.step(1)["rc"] == -8  # failed context: ESTATE
    for k in FIELDS:
        assert rel_err(fg[k], fo[k]) <= 1e-11, k


def test_sedov_collapse_halts_at_the_oracle_cycle():
    """kappa = 0 Sedov corner box (zone size of 448^3): the default floor 1e-6 dt^0 is crossed
    at the same cycle on both sides (the oracle: cycle 1295)."""
    n, h = 12, 1.2 / 448
    kw = dict(n=(n, n, n), extent=(h * n,) * 3)
    o = Oracle(OracleConfig(**kw))
    io = o.step(2500)
    o.close()
    assert io["status"] == -7
    with Hydro(HydroConfig(**kw)) as hy:
        ig = hy.step(2500)
    assert ig["status"] == -7 and ig["bad_zone"] == -1
    assert abs(ig["cycle"] - io["cycle"]) <= 1, (ig["cycle"], io["cycle"])
