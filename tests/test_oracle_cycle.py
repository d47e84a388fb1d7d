"""Pins for the oracle's full cycle S1-S9 (orc_step) and its domain decomposition.

What pins what:
* forces/update: a uniform gas at rest in a dyadic box stays bitwise at rest; Galilean
  invariance with free boundaries; acoustic standing-wave period 2L/c converging O(h^2);
* energy update: total mass bit-constant, total energy conserved to <=1e-12 (fsum);
* shock capturing: Sod tube vs the exact Riemann solution (tests/riemann.py, Toro);
* Sedov: analytic shock radius (oracle/sedov.py, pinned to literature
  alpha) and axis-permutation symmetry;
* decomposition: decomposed == undecomposed bitwise for uneven cuts.
"""
import math
import os

import numpy as np
import pytest

import oracle
from oracle import Oracle, OracleConfig
from oracle import sedov as sedov_mod
from paper_conf_icppw_pearce18_b200.inputs import jittered_state, splitmix64
from tests.helpers import rel_err, sedov_radius, sedov_radius_tolerance, total_energy, user_state
from tests.riemann import sample, star

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _golden(name):
    rows = []
    for line in open(os.path.join(GOLD, name)):
        line = line.strip()
        if line and not line.startswith("#"):
            rows.append(line.split())
    return rows


# ---------------------------------------------------------------- test-side pins themselves

def test_splitmix64_reference_value():
    (seed, idx, hexval), = _golden("splitmix64.txt")
    assert int(splitmix64(int(seed), int(idx), 1)[0]) == int(hexval, 16)


def test_sedov_alpha_matches_literature():
    for g, a, xi in _golden("sedov_alpha.txt"):
        g, a, xi = float(g), float(a), float(xi)
        assert sedov_mod.alpha(g) == pytest.approx(a, abs=2e-6)
        assert sedov_mod.xi0(g) == pytest.approx(xi, abs=2e-5)


def test_riemann_solver_matches_toro():
    (rl, ul, pl, rr, ur, pr, ps, us), = [[float(v) for v in r] for r in _golden("sod_toro.txt")]
    p, u = star(rl, ul, pl, rr, ur, pr, 1.4)
    assert p == pytest.approx(ps, abs=1e-5)
    assert u == pytest.approx(us, abs=1e-5)


# ---------------------------------------------------------------- oracle cycle pins

def test_uniform_gas_at_rest_stays_bitwise_at_rest():
    n = (8, 8, 8)
    s = user_state(n, extent=(1.0, 1.0, 1.0), rho=1.0, e=1.0)  # h = 2^-3 (dyadic)
    o = Oracle(OracleConfig(n=n, extent=(1.0, 1.0, 1.0), init="user", user=s))
    f0 = o.fields()
    info = o.step(100)
    f = o.fields()
    assert info["status"] == 0 and info["cycle"] == 100
    for k in ("x", "y", "z", "u", "v", "w", "e", "rho", "p"):
        assert np.array_equal(f[k], f0[k]), k


def test_sedov_mass_bit_constant_and_energy_conserved():
    cfg = OracleConfig(n=(24, 24, 24))
    o = Oracle(cfg)
    f0 = o.fields()
    E0 = sum(total_energy(f0))
    assert E0 == pytest.approx(cfg.sedov_energy, rel=1e-15)
    info = o.step(100)
    f = o.fields()
    assert info["status"] == 0
    assert np.array_equal(f["mass"], f0["mass"])
    assert abs(sum(total_energy(f)) - E0) / E0 <= 1e-12
    assert total_energy(f)[1] > 0.1 * E0  # energy really moved into kinetic form


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_jittered_energy_conserved(seed):
    n = (12, 12, 12)
    s = jittered_state(n, seed)
    o = Oracle(OracleConfig(n=n, init="user", user=s))
    E0 = sum(total_energy(o.fields()))
    info = o.step(100)
    assert info["status"] == 0
    E = sum(total_energy(o.fields()))
    assert abs(E - E0) / E0 <= 1e-12


def test_sedov_axis_permutation_symmetry():
    f, info = oracle.run(OracleConfig(n=(20, 20, 20)), 100)
    assert info["status"] == 0
    rho = f["rho"]
    for perm in ((0, 2, 1), (2, 1, 0), (1, 0, 2)):
        assert rel_err(rho.transpose(perm), rho) <= 1e-10
    # velocity components permute with the axes: u(x,y,z) <-> v(y,x,z)
    assert rel_err(f["u"].transpose(0, 2, 1), f["v"]) <= 1e-10


CUTS = [
    [[0, 7, 13, 20], [0, 10, 20], [0, 3, 20]],
    [[0, 1, 19, 20], [0, 2, 4, 20], [0, 20]],
    [[0, 10, 20], [0, 10, 20], [0, 10, 20]],
]


@pytest.mark.parametrize("cuts", CUTS)
def test_sedov_decomposed_equals_undecomposed_bitwise(cuts):
    n = (20, 20, 20)
    ref, ri = oracle.run(OracleConfig(n=n), 40)
    ndom = tuple(len(c) - 1 for c in cuts)
    dec, di = oracle.run(OracleConfig(n=n, ndom=ndom, cuts=cuts), 40)
    assert ri["dt"] == di["dt"] and ri["t"] == di["t"]
    for k in ref:
        assert np.array_equal(ref[k], dec[k]), k


def test_jittered_decomposed_even_split_bitwise():
    n = (13, 11, 9)
    s = jittered_state(n, 2)
    ref, _ = oracle.run(OracleConfig(n=n, init="user", user=s), 30)
    dec, _ = oracle.run(OracleConfig(n=n, init="user", user=s, ndom=(3, 2, 4)), 30)
    for k in ref:
        assert np.array_equal(ref[k], dec[k]), k


def test_galilean_invariance_free_boundaries():
    n = (10, 9, 8)
    s = jittered_state(n, 5)
    U0 = np.array([0.3, -0.2, 0.1])
    s2 = dict(s)
    s2["u"] = s["u"] + U0[0]
    s2["v"] = s["v"] + U0[1]
    s2["w"] = s["w"] + U0[2]
    a, ia = oracle.run(OracleConfig(n=n, init="user", user=s, reflect_mask=0), 30)
    b, ib = oracle.run(OracleConfig(n=n, init="user", user=s2, reflect_mask=0), 30)
    assert ib["t"] == pytest.approx(ia["t"], rel=1e-12)
    t = ia["t"]
    h = 1.2 / 10
    for d, (x, u) in enumerate((("x", "u"), ("y", "v"), ("z", "w"))):
        assert np.abs(b[x] - a[x] - U0[d] * t).max() <= 1e-10 * h
        assert np.abs(b[u] - a[u] - U0[d]).max() <= 1e-10
    assert rel_err(b["e"], a["e"]) <= 1e-10


def _acoustic(N, eps=1e-5, gamma=1.4, frac=1.0):
    n = (N, 1, 1)
    ext = (1.0, 1.0, 1.0)
    s = user_state(n, extent=ext)
    xc = (np.arange(N) + 0.5) / N
    rho = 1.0 + eps * np.cos(np.pi * xc)
    p = rho ** gamma
    s["rho"] = rho.reshape(1, 1, N)
    s["e"] = (p / ((gamma - 1) * rho)).reshape(1, 1, N)
    T = 2.0 / math.sqrt(gamma)  # period 2L/c0, L = 1, c0 = sqrt(gamma p0/rho0)
    cfg = OracleConfig(n=n, extent=ext, init="user", user=s, q_lin=0.0, q_quad=0.0,
                       t_stop=frac * T, c_vol=1.0)
    f, info = oracle.run(cfg, 100000)
    assert info["t"] == pytest.approx(frac * T, rel=1e-14)
    drho = f["rho"].ravel() - 1.0
    amp = 2.0 * np.mean(drho * np.cos(np.pi * xc)) / eps
    return amp, np.abs(drho - eps * np.cos(np.pi * xc)).max() / eps


def test_acoustic_standing_wave_period_second_order():
    a_half, _ = _acoustic(32, frac=0.5)
    assert a_half == pytest.approx(-1.0, abs=0.02)
    a32, e32 = _acoustic(32)
    a64, e64 = _acoustic(64)
    assert a64 == pytest.approx(1.0, abs=1e-4)
    assert e64 < 1e-5
    assert e32 / e64 > 3.5  # at least O(h^2) (eps = 1e-5 keeps nonlinear terms out)


def _sod(N):
    g = 1.4
    n = (N, 1, 1)
    ext = (1.0, 1.0, 1.0)
    s = user_state(n, extent=ext)
    xc = (np.arange(N) + 0.5) / N
    left = xc < 0.5
    rho = np.where(left, 1.0, 0.125)
    p = np.where(left, 1.0, 0.1)
    s["rho"] = rho.reshape(1, 1, N)
    s["e"] = (p / ((g - 1) * rho)).reshape(1, 1, N)
    f, info = oracle.run(OracleConfig(n=n, extent=ext, init="user", user=s, t_stop=0.2), 100000)
    assert info["status"] == 0 and info["t"] == pytest.approx(0.2, rel=1e-14)
    x = f["x"][0, 0]
    xcz = 0.5 * (x[:-1] + x[1:])
    ex = sample(xcz, 0.2, 0.5, (1.0, 0.0, 1.0), (0.125, 0.0, 0.1), g)
    rho_num = f["rho"].ravel()
    L1 = float(np.sum(np.abs(rho_num - ex[0]) * np.diff(x)))
    # shock: last zone whose density exceeds the midpoint of post-shock and right states
    mid = 0.5 * (0.26557 + 0.125)
    shock = xcz[np.nonzero(rho_num > mid)[0].max()]
    return L1, shock, 1.0 / N


def test_sod_shock_tube_against_exact_riemann():
    res = [_sod(N) for N in (100, 200, 400)]
    for (L1a, _, _), (L1b, _, _) in zip(res, res[1:]):
        assert L1b < 0.75 * L1a  # converging (first order at discontinuities)
    for L1, shock, h in res:
        assert abs(shock - 0.8504) <= 2.0 * h  # exact shock position at t = 0.2
    assert res[-1][0] < 0.01


def test_sedov_shock_radius_matches_analytic():
    n = 32
    cfg = OracleConfig(n=(n, n, n), t_stop=0.3)
    f, info = oracle.run(cfg, 100000)
    assert info["status"] == 0 and info["t"] == pytest.approx(0.3, rel=1e-14)
    R = sedov_radius(f, 1.2 / n)
    R_exact = sedov_mod.shock_radius(0.3, 8.0 * cfg.sedov_energy, 1.0, 1.4)
    assert abs(R - R_exact) / R_exact <= sedov_radius_tolerance(1.2 / n, R_exact)


def test_sedov_shock_radius_64_cubed_with_hourglass_control():
    """North_star: the analytic Sedov shock radius on a refined mesh (PAPER.md L637-642 is the
    Sedov workload).  At 64^3 the plain kappa = 0 scheme cannot reach t = 0.3 (a zone next to
    the origin is crushed and dt collapses, halting with EDTMIN: reading R23,
    test_long_sedov_needs_hourglass_control), so this pin runs with the reading-R17 hourglass
    control at kappa = 0.03.  Calibrated once (R16): +0.91 % at 513 cycles, against the
    frozen tolerance 3 % + h/(4R) = 3.76 %."""
    n = 64
    cfg = OracleConfig(n=(n, n, n), t_stop=0.3, hg_coef=0.03)
    f, info = oracle.run(cfg, 100000, names=("x", "y", "z", "rho", "e"))
    assert info["status"] == 0 and info["t"] == pytest.approx(0.3, rel=1e-14)
    R = sedov_radius(f, 1.2 / n)
    R_exact = sedov_mod.shock_radius(0.3, 8.0 * cfg.sedov_energy, 1.0, 1.4)
    assert abs(R - R_exact) / R_exact <= sedov_radius_tolerance(1.2 / n, R_exact)


@pytest.mark.skipif(os.environ.get("HYDRO_SLOW") != "1",
                    reason="~11 min of oracle time; run with HYDRO_SLOW=1 (result in DESIGN.md R16)")
def test_sedov_shock_radius_96_cubed_with_hourglass_control():
    n = 96
    cfg = OracleConfig(n=(n, n, n), t_stop=0.3, hg_coef=0.03)
    f, info = oracle.run(cfg, 100000, names=("x", "y", "z", "rho", "e"))
    assert info["status"] == 0 and info["t"] == pytest.approx(0.3, rel=1e-14)
    R = sedov_radius(f, 1.2 / n)
    R_exact = sedov_mod.shock_radius(0.3, 8.0 * cfg.sedov_energy, 1.0, 1.4)
    assert abs(R - R_exact) / R_exact <= sedov_radius_tolerance(1.2 / n, R_exact)


@pytest.mark.slow
@pytest.mark.skipif(os.environ.get("HYDRO_SLOW") != "1",
                    reason="37 s; the refined-mesh pin is the 64^3 one (HYDRO_SLOW=1 runs it)")
def test_sedov_shock_radius_48_cubed():
    n = 48
    cfg = OracleConfig(n=(n, n, n), t_stop=0.3)
    f, info = oracle.run(cfg, 100000)
    R = sedov_radius(f, 1.2 / n)
    R_exact = sedov_mod.shock_radius(0.3, 8.0 * cfg.sedov_energy, 1.0, 1.4)
    assert abs(R - R_exact) / R_exact <= sedov_radius_tolerance(1.2 / n, R_exact)


def test_dt_rule_growth_and_zone_minimum():
    o = Oracle(OracleConfig(n=(12, 12, 12)))
    prev = o.info()["dt"]
    for _ in range(30):
        info = o.step(1)
        expect = min(min(1.1 * prev, math.inf), info["dt_min_zone"])
        assert info["dt"] == expect
        prev = info["dt"]


def test_tangled_mesh_is_detected():
    n = (6, 6, 6)
    s = user_state(n, e=1.0)
    s["u"][3, 3, 3] = 1e4  # one node shot through its neighbour
    o = Oracle(OracleConfig(n=n, init="user", user=s, dt_first=1e-3))
    info = o.step(5)
    assert info["status"] == -5 and info["cycle"] == 1
    assert 0 <= info["bad_zone"] < 6 ** 3
    assert o.step(1)["status"] == -8


def _floor_between(seq, c):
    """An absolute dt floor that the zone-dt minimum of cycle c (1-based) is the first to cross:
    the midpoint between dtmin(c) and the smallest earlier dtmin (both well separated)."""
    prev = min(seq[:c - 1])
    assert seq[c - 1] < prev * (1 - 1e-4)
    return 0.5 * (seq[c - 1] + prev)


def test_dt_floor_halts_with_edtmin_after_the_crossing_cycle():
    """Reading R23: the first cycle whose min_z dt_z falls below the floor halts the run with
    EDTMIN (-7), bad_zone -1; the state is the one after that cycle (bitwise equal to a run
    without a floor stepped to the same cycle); a later step returns ESTATE (-8)."""
    n = (16, 16, 16)
    s = jittered_state(n, 1)
    o = Oracle(OracleConfig(n=n, init="user", user=s, dt_floor=-1.0))
    seq = [o.step(1)["dt_min_zone"] for _ in range(12)]
    ref = o  # stepped 12 cycles; rebuild to 10 below
    ref.close()
    floor = _floor_between(seq, 10)
    o = Oracle(OracleConfig(n=n, init="user", user=s, dt_floor=floor))
    info = o.step(100)
    assert info["status"] == -7 and info["cycle"] == 10 and info["bad_zone"] == -1
    assert info["dt_min_zone"] == seq[9]
    f = o.fields()
    assert o.step(1)["status"] == -8
    o.close()
    g, ginfo = oracle.run(OracleConfig(n=n, init="user", user=s, dt_floor=-1.0), 10)
    assert ginfo["status"] == 0 and ginfo["t"] == info["t"]
    for k in f:
        assert np.array_equal(f[k], g[k]), k


def test_dt_floor_default_is_relative_to_dt0_and_tstop_clamp_is_not_a_collapse():
    """Default floor 1e-6 dt^0: an ordinary Sedov run to t_stop never trips it, although its
    last dt is clamped to t_stop - t (dtmin, not the clamped dt, is compared)."""
    n = (12, 12, 12)
    o = Oracle(OracleConfig(n=n, t_stop=0.05))
    info = o.step(100000)
    assert info["status"] == 0 and info["t"] == pytest.approx(0.05, rel=1e-14)
    # an absolute floor above every dtmin of the run trips on the first cycle
    o = Oracle(OracleConfig(n=n, dt_floor=1.0))
    info = o.step(5)
    assert info["status"] == -7 and info["cycle"] == 1
