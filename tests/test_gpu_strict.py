"""STRICT path (HYDRO_FLAG_STRICT, csrc/strict/kernel_strict.cu) against the oracle: BITWISE.

Both sides evaluate the canonical operation order of SURVEY.md §8c (reading R13) in IEEE fp64
without contraction (reading R12: oracle -O2 -ffp-contract=off, STRICT -fmad=false; '/' and sqrt
correctly rounded on both), so every field, t and dt must be identical bit for bit -- the
north_star tolerance becomes an equality on this path.  The one
exception is the hourglass term (kappa > 0): cbrt is not correctly rounded on either side.
"""
import numpy as np
import pytest

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")
OKEYS = ("n", "origin", "extent", "gamma", "q_lin", "q_quad", "cfl", "c_vol", "dt_growth",
         "dt_max", "dt_init", "t_stop", "dt_first", "t0", "reflect_mask", "init", "rho0", "e0",
         "sedov_energy", "user", "ndom", "cuts", "hg_coef", "dt_floor")


def both(nc, **kw):
    fo, io = oracle.run(OracleConfig(**{k: v for k, v in kw.items() if k in OKEYS}), nc)
    with Hydro(HydroConfig(path="strict", **kw)) as h:
        ig = h.step(nc)
        fg = h.fields()
    return fg, ig, fo, io


def assert_bitwise(fg, ig, fo, io):
    for k in FIELDS:
        a, b = fg[k], fo[k]
        if not np.array_equal(a.view(np.uint64), b.view(np.uint64)):
            bad = np.argwhere(a.view(np.uint64) != b.view(np.uint64))
            raise AssertionError(f"{k}: {len(bad)} entries differ, first {bad[0]}: "
                                 f"{a[tuple(bad[0])]!r} vs {b[tuple(bad[0])]!r}, "
                                 f"rel {rel_err(a, b):.3e}")
    assert ig["t"] == io["t"] and ig["dt"] == io["dt"]
    assert ig["cycle"] == io["cycle"] and ig["dt_min_zone"] == io["dt_min_zone"]
    assert ig["status"] == io["status"]


@pytest.mark.parametrize("seed", [1, 2, 3])
@pytest.mark.parametrize("nc", [1, 100])
def test_strict_jittered16_bitwise(seed, nc):
    n = (16, 16, 16)
    assert_bitwise(*both(nc, n=n, init="user", user=jittered_state(n, seed)))


def test_strict_sedov32_hundred_cycles_bitwise():
    assert_bitwise(*both(100, n=(32, 32, 32)))


def test_strict_decomposed_uneven_bitwise():
    """Uneven cuts incl. 1-zone-thick domains: halo copies are bit copies, so STRICT multi-domain
    equals the (decomposed == undecomposed) oracle bitwise."""
    n = (24, 20, 18)
    cuts = [[0, 5, 13, 24], [0, 1, 20], [0, 9, 10, 18]]
    assert_bitwise(*both(40, n=n, ndom=(3, 2, 3), cuts=cuts, init="user",
                         user=jittered_state(n, 7)))


@pytest.mark.parametrize("phys", [dict(gamma=5.0 / 3.0), dict(q_lin=0.25, q_quad=1.0),
                                  dict(q_lin=0.0, q_quad=0.0),
                                  dict(cfl=0.5, c_vol=0.2, dt_growth=1.05),
                                  dict(dt_max=2e-4, reflect_mask=0b010101)])
def test_strict_physics_parameters_bitwise(phys):
    n = (18, 16, 14)
    assert_bitwise(*both(60, n=n, init="user", user=jittered_state(n, 4), **phys))


def test_strict_t_stop_and_edtmin_bitwise():
    n = (16, 16, 16)
    s = jittered_state(n, 2)
    assert_bitwise(*both(1000, n=n, init="user", user=s, t_stop=0.5))
    fg, ig, fo, io = both(1000, n=n, init="user", user=s, dt_floor=0.0145)
    assert io["status"] == -7
    assert_bitwise(fg, ig, fo, io)


def test_strict_negative_energy_clamp_bitwise():
    """Reading R6 (p and c use max(e, 0); e itself is never clamped): zones with negative and
    subnormal energies on every path of S3."""
    n = (12, 10, 8)
    s = jittered_state(n, 5)
    e = s["e"].copy()
    e[::3, ::2, ::3] = -0.3
    e[1::4, 1::3, ::2] = 4.9e-320  # subnormal
    s["e"] = e
    assert_bitwise(*both(30, n=n, init="user", user=s))


def test_strict_hourglass_close():
    """kappa > 0: cbrt(V) is not correctly rounded, so only (very) close."""
    n = (16, 16, 16)
    fg, ig, fo, io = both(50, n=n, init="user", user=jittered_state(n, 3), hg_coef=0.03)
    for k in FIELDS:
        assert rel_err(fg[k], fo[k]) <= 1e-13, k
