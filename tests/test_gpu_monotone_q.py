"""GPU parity of the monotone artificial viscosity (reading R24) against the
oracle: the split kernels within the north_star tolerance (1e-12 after one cycle, 1e-10 after
100), the STRICT kernels bit for bit, on jittered inputs, uneven multi-domain cuts (the limiter
reads its neighbours' strain rates from their owner domains, so decomposed == undecomposed
bitwise) and Sedov with hourglass control; a multi-rank context is refused."""
import numpy as np
import pytest

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig, HydroError
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")
OKEYS = ("n", "extent", "init", "user", "ndom", "cuts", "hg_coef", "t_stop", "reflect_mask")


def both(nc, path, **kw):
    fo, io = oracle.run(OracleConfig(q="monotone", **{k: v for k, v in kw.items()
                                                      if k in OKEYS}), nc)
    with Hydro(HydroConfig(q="monotone", path=path, **kw)) as h:
        ig = h.step(nc)
        fg = h.fields()
    return fg, ig, fo, io


@pytest.mark.parametrize("seed", [1, 2])
def test_split_monotone_q_matches_oracle(seed):
    n = (16, 16, 16)
    kw = dict(n=n, init="user", user=jittered_state(n, seed))
    for nc, tol in ((1, 1e-12), (100, 1e-10)):
        fg, ig, fo, io = both(nc, "split", **kw)
        assert ig["status"] == 0 == io["status"]
        for k in FIELDS:
            assert rel_err(fg[k], fo[k]) <= tol, (nc, k)
        assert ig["dt"] == pytest.approx(io["dt"], rel=tol)


def test_strict_monotone_q_bitwise():
    n = (20, 18, 16)
    cuts = [[0, 1, 9, 20], [0, 7, 18], [0, 8, 16]]
    for kw in (dict(n=n, init="user", user=jittered_state(n, 3)),
               dict(n=n, init="user", user=jittered_state(n, 3), ndom=(3, 2, 2), cuts=cuts),
               dict(n=n, init="user", user=jittered_state(n, 4), reflect_mask=0b100110)):
        fg, ig, fo, io = both(40, "strict", **kw)
        for k in FIELDS:
            assert np.array_equal(fg[k].view(np.uint64), fo[k].view(np.uint64)), k
        assert ig["t"] == io["t"] and ig["dt"] == io["dt"]


def test_split_monotone_q_decomposed_bitwise():
    n = (20, 18, 16)
    s = jittered_state(n, 5)
    cuts = [[0, 1, 9, 20], [0, 7, 18], [0, 8, 16]]
    with Hydro(HydroConfig(n=n, init="user", user=s, q="monotone")) as h:
        h.step(30)
        fa = h.fields()
    with Hydro(HydroConfig(n=n, init="user", user=s, q="monotone", ndom=(3, 2, 2),
                           cuts=cuts)) as h:
        h.step(30)
        fb = h.fields()
    for k in FIELDS:
        assert np.array_equal(fa[k], fb[k]), k


def test_sedov_monotone_q_with_hourglass_matches_oracle():
    kw = dict(n=(24, 24, 24), hg_coef=0.03)
    fg, ig, fo, io = both(60, "split", **kw)
    assert ig["status"] == 0
    for k in FIELDS:
        assert rel_err(fg[k], fo[k]) <= 1e-10, k


def test_monotone_q_refuses_multi_rank():
    with pytest.raises(HydroError):
        Hydro(HydroConfig(n=(8, 8, 8), q="monotone", nranks=2, rank=0, transport="peer"))
