"""GPU parity of the viscous hourglass control (reading R17) against the
oracle, through the C ABI.  hg_coef > 0 runs the split kernels (corner-force planes in HBM);
tolerances are north_star's (reading R15): <= 1e-12 after one cycle, <= 1e-10 after 100.
"""
import numpy as np
import pytest

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err, total_energy
from tests.test_oracle_hourglass import _checkerboard

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")


def _pair(nc, ndom=(1, 1, 1), **kw):
    fo, io = oracle.run(OracleConfig(ndom=ndom, **kw), nc)
    with Hydro(HydroConfig(ndom=ndom, **kw)) as h:
        ig = h.step(nc)
        fg = h.fields()
    return fg, ig, fo, io


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_jittered16_hourglass(seed):
    n = (16, 16, 16)
    kw = dict(n=n, init="user", user=jittered_state(n, seed), hg_coef=0.03)
    for nc, tol in ((1, 1e-12), (100, 1e-10)):
        fg, ig, fo, io = _pair(nc, **kw)
        assert ig["status"] == 0
        errs = {k: rel_err(fg[k], fo[k]) for k in FIELDS}
        assert max(errs.values()) <= tol, errs
        assert ig["dt"] == pytest.approx(io["dt"], rel=tol)


def test_hourglass_really_acts_on_the_gpu():
    """The same input with kappa = 0 differs from kappa > 0 well above the tolerance."""
    n = (12, 12, 12)
    s = jittered_state(n, 1)
    with Hydro(HydroConfig(n=n, init="user", user=s, hg_coef=0.03)) as h:
        h.step(20)
        a = h.fields()
    with Hydro(HydroConfig(n=n, init="user", user=s, path="split")) as h:
        h.step(20)
        b = h.fields()
    assert rel_err(a["u"], b["u"]) > 1e-6


@pytest.mark.parametrize("kappa", [0.0, 0.01])
def test_checkerboard_mode(kappa):
    n = (8, 8, 8)
    kw = dict(n=n, extent=(1.0, 1.0, 1.0), init="user", user=_checkerboard(n), hg_coef=kappa)
    fg, ig, fo, io = _pair(40, **kw)
    assert ig["status"] == 0
    ke0 = total_energy(fo)[1]
    # field scales: u, v, w against the pattern amplitude; q (round-off compressions only, the
    # pattern is divergence-free) against p; the rest against their own max (reading R15)
    scale = {k: max(float(np.abs(fo[k]).max()), 1e-300) for k in FIELDS}
    for k in "uvw":
        scale[k] = max(scale[k], 0.01)
    scale["q"] = scale["p"]
    for k in FIELDS:
        assert float(np.abs(fg[k] - fo[k]).max()) <= 1e-10 * scale[k], k
    ke0_init = total_energy(oracle.run(OracleConfig(**kw), 0)[0])[1]
    assert abs(total_energy(fg)[1] - ke0) <= 1e-10 * ke0_init


def test_sedov_multidomain_hourglass():
    n = (24, 20, 16)
    kw = dict(n=n, hg_coef=0.03)
    fg, ig, fo, io = _pair(60, ndom=(2, 2, 1), **kw)
    assert ig["status"] == 0
    errs = {k: rel_err(fg[k], fo[k]) for k in FIELDS}
    assert max(errs.values()) <= 1e-10, errs
