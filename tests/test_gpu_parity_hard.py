"""GPU parity where the kernels take their full-size paths and their rare branches.

* 128^3 (BASELINE.json configs[1]) from a smooth state that moves everywhere from cycle 0, so
  every tile seam, ring column, z-chunk boundary and TMA box edge of the full-size launch sees
  non-trivial values (the at-rest Sedov field leaves > 99 % of them at zero), against the oracle
  element by element.
* Reading R6 (p and c use max(e, 0); e is never clamped) and the subnormal branch of the fast
  square root (csrc/fastmath.cuh fsqrt scales subnormal arguments): zones with negative and
  subnormal energies, on every path, against the oracle.
Tolerance: north_star (R15 norm) -- 1e-12 after one cycle, growing to 1e-10 after 100.
"""
import numpy as np
import pytest

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err, user_state

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")
OKEYS = ("n", "origin", "extent", "init", "user", "ndom", "cuts")


def smooth_state(N, L=1.2):
    """Acoustic-like smooth field (the test_gpu_fullsize.py recipe): velocities from products of
    sines that vanish on the walls in the normal direction, density and energy varying in z / x."""
    s = user_state((N, N, N), extent=(L, L, L))
    x, y, z = s["x"], s["y"], s["z"]
    k = 2.0 * np.pi / L
    s["u"] = 0.05 * np.sin(3 * k * y) * np.cos(2 * k * z) * np.sin(k * x)
    s["v"] = 0.05 * np.sin(2 * k * z) * np.cos(3 * k * x) * np.sin(k * y)
    s["w"] = 0.05 * np.sin(2 * k * x) * np.cos(3 * k * y) * np.sin(k * z)
    zc = (np.arange(N) + 0.5) * (L / N)
    s["rho"] = np.ascontiguousarray(
        1.0 + 0.2 * np.sin(5 * k * zc)[:, None, None] * np.cos(4 * k * zc)[None, :, None]
        * np.ones((1, 1, N)))
    s["e"] = np.ascontiguousarray(1.0 + 0.3 * np.cos(3 * k * zc)[None, None, :] * np.ones((N, N, 1)))
    return s


@pytest.fixture(scope="module")
def oracle128():
    s = smooth_state(128)
    kw = dict(n=(128, 128, 128), init="user", user=s)
    o = oracle.Oracle(OracleConfig(**kw))
    out = {}
    for nc in (1, 8):
        info = o.step(nc - (1 if nc == 8 else 0))
        out[nc] = (o.fields(), info)
    o.close()
    return s, out


@pytest.mark.parametrize("path", ["two", "one"])
def test_full_size_128_moving_state_against_oracle(path, oracle128):
    s, ref = oracle128
    with Hydro(HydroConfig(n=(128, 128, 128), init="user", user=s, path=path)) as h:
        for nc, tol in ((1, 1e-12), (8, 1e-11)):
            ig = h.step(nc - (1 if nc == 8 else 0))
            fg = h.fields()
            fo, io = ref[nc]
            assert ig["status"] == 0 and ig["cycle"] == nc
            errs = {k: rel_err(fg[k], fo[k]) for k in FIELDS}
            bad = {k: v for k, v in errs.items() if not v <= tol}
            assert not bad, (nc, bad)
            assert ig["dt"] == pytest.approx(io["dt"], rel=tol)
            # the state really moves across every tile: compressions somewhere, q > 0
            assert np.count_nonzero(fg["q"]) > 0.2 * fg["q"].size


def _rare_state():
    n = (20, 18, 13)  # ragged: partial tiles in x and y
    s = jittered_state(n, 5)
    e = s["e"].copy()
    e[::3, ::2, ::3] = -0.3          # R6: negative energy, p = c = 0 from max(e, 0)
    e[1::4, 1::3, ::2] = 4.9e-320    # subnormal energy (fsqrt's scaled branch)
    e[2::5, ::4, 1::3] = 2.5e-310    # subnormal, normal after the predictor in some zones
    s["e"] = e
    return n, s


@pytest.mark.parametrize("path", ["two", "one", "split"])
def test_negative_and_subnormal_energy_against_oracle(path):
    n, s = _rare_state()
    kw = dict(n=n, init="user", user=s)
    for nc, tol in ((1, 1e-12), (30, 1e-10)):
        fo, io = oracle.run(OracleConfig(**kw), nc)
        with Hydro(HydroConfig(path=path, **kw)) as h:
            ig = h.step(nc)
            fg = h.fields()
        assert ig["status"] == 0 == io["status"]
        assert (fo["e"] < 0).any() and (fg["e"] < 0).any()  # e is never clamped (R6)
        errs = {k: rel_err(fg[k], fo[k]) for k in FIELDS}
        bad = {k: v for k, v in errs.items() if not v <= tol}
        assert not bad, (nc, bad)
        # zones that still hold a negative energy have p = c = 0 on both sides exactly
        neg = fo["e"] < 0
        assert np.array_equal(fg["p"][neg], np.zeros(neg.sum()))
        assert np.array_equal(fg["c"][neg], np.zeros(neg.sum()))
