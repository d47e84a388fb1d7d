"""Oracle pins of the monotone artificial viscosity (SURVEY §8f row f1 "q variants", reading R24):
per logical direction d the zone's strain rate eps_d = (du_d . dx_d) / |dx_d|^2 from face-centre
differences, a Christensen / LULESH-type limiter phi_d = max(0, min((r- + r+)/2, 2r-, 2r+, 1)) of
the neighbours' strain-rate ratios, and q = rho sum_d [q_quad dv_d^2 (1 - phi_d^2) +
q_lin c dv_d (1 - phi_d)] with dv_d = L_d max(-eps_d, 0), on compression only.  Pinned by the
limiter's closed form, the strain of affine velocity fields, q = 0 for a linear velocity field
(where the scalar q of R7 is not), the Sod shock tube, decomposition invariance, energy
conservation and the Sedov radius."""
import math

import numpy as np
import pytest

import oracle
from oracle import Oracle, OracleConfig
from oracle import sedov as sedov_mod
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import sedov_radius, sedov_radius_tolerance, total_energy, user_state
from tests.riemann import sample


def test_limiter_closed_forms():
    assert oracle.mono_limiter(1.0, 1.0, 1.0) == 1.0        # smooth: no q
    assert oracle.mono_limiter(0.0, 1.0, 0.0) == 0.0        # isolated compression: full q
    assert oracle.mono_limiter(0.2, 1.0, 5.0) == pytest.approx(0.4)  # 2 r-
    assert oracle.mono_limiter(0.8, 1.0, 0.9) == pytest.approx(0.85)  # (r- + r+)/2
    assert oracle.mono_limiter(-1.0, 1.0, 1.0) == 0.0       # sign change: full q
    assert oracle.mono_limiter(3.0, 0.0, 1.0) == 1.0        # no strain along d
    assert oracle.mono_limiter(-2.0, -1.0, -3.0) == 1.0     # ratios > 1 are capped


def _hex(X0, A, h=(0.3, 0.2, 0.25)):
    X = np.array([[X0[0] + h[0] * (l & 1), X0[1] + h[1] * ((l >> 1) & 1),
                   X0[2] + h[2] * ((l >> 2) & 1)] for l in range(8)])
    return X, X @ np.asarray(A).T


def test_strain_of_affine_fields():
    X, U = _hex((0.1, -0.2, 0.3), np.diag([-0.5, 0.25, 2.0]))
    eps, L = oracle.zone_strain(X, U)
    assert np.allclose(eps, [-0.5, 0.25, 2.0], rtol=1e-14) and np.allclose(L, [0.3, 0.2, 0.25])
    # a rotation rate (antisymmetric gradient) strains nothing; a rigid translation neither
    W = np.array([[0.0, -1.0, 0.5], [1.0, 0.0, -2.0], [-0.5, 2.0, 0.0]])
    eps, _ = oracle.zone_strain(X, X @ W.T + np.array([1.0, 2.0, 3.0]))
    assert np.abs(eps).max() < 1e-14


def test_linear_velocity_field_has_no_monotone_q():
    """Homologous compression u = -0.1 x: every zone has the same strain rates, the limiter is 1
    and the monotone q vanishes in the interior (free boundaries: the missing neighbour counts as
    unstrained, so boundary zones keep their q), while the scalar q of R7 is positive."""
    n = (8, 8, 8)
    s = user_state(n, e=1.0)
    for v, x in (("u", "x"), ("v", "y"), ("w", "z")):
        s[v] = -0.1 * s[x]
    fm, _ = oracle.run(OracleConfig(n=n, init="user", user=s, reflect_mask=0, q="monotone"), 0)
    fs, _ = oracle.run(OracleConfig(n=n, init="user", user=s, reflect_mask=0), 0)
    inner = (slice(1, -1),) * 3
    assert fs["q"][inner].min() > 0.01
    assert fm["q"][inner].max() <= 1e-12 * fs["q"][inner].min()
    assert fm["q"].max() > 0.01  # boundary zones


def _sod(N, q):
    g = 1.4
    n, ext = (N, 1, 1), (1.0, 1.0, 1.0)
    s = user_state(n, extent=ext)
    xc = (np.arange(N) + 0.5) / N
    left = xc < 0.5
    rho = np.where(left, 1.0, 0.125)
    p = np.where(left, 1.0, 0.1)
    s["rho"] = rho.reshape(1, 1, N)
    s["e"] = (p / ((g - 1) * rho)).reshape(1, 1, N)
    f, info = oracle.run(OracleConfig(n=n, extent=ext, init="user", user=s, t_stop=0.2, q=q),
                         100000)
    assert info["status"] == 0 and info["t"] == pytest.approx(0.2, rel=1e-14)
    x = f["x"][0, 0]
    xcz = 0.5 * (x[:-1] + x[1:])
    ex = sample(xcz, 0.2, 0.5, (1.0, 0.0, 1.0), (0.125, 0.0, 0.1), g)
    r = f["rho"].ravel()
    L1 = float(np.sum(np.abs(r - ex[0]) * np.diff(x)))
    shock = xcz[np.nonzero(r > 0.5 * (0.26557 + 0.125))[0].max()]
    return L1, shock, 1.0 / N


def test_sod_with_monotone_q():
    res = [_sod(N, "monotone") for N in (100, 200, 400)]
    for (a, _, _), (b, _, _) in zip(res, res[1:]):
        assert b < 0.75 * a
    for L1, shock, h in res:
        assert abs(shock - 0.8504) <= 2.0 * h
    assert res[-1][0] < 0.01


def test_monotone_q_decomposed_equals_undecomposed_bitwise():
    n = (20, 18, 16)
    s = jittered_state(n, 3)
    cuts = [[0, 1, 9, 20], [0, 7, 18], [0, 8, 16]]
    fa, ia = oracle.run(OracleConfig(n=n, init="user", user=s, q="monotone"), 30)
    fb, ib = oracle.run(OracleConfig(n=n, init="user", user=s, q="monotone", ndom=(3, 2, 2),
                                     cuts=cuts), 30)
    assert ia["dt"] == ib["dt"] and ia["t"] == ib["t"]
    for k in fa:
        assert np.array_equal(fa[k], fb[k]), k
    fs, _ = oracle.run(OracleConfig(n=n, init="user", user=s), 30)
    assert np.abs(fa["e"] - fs["e"]).max() > 1e-6  # the variant really differs from R7


def test_monotone_q_conserves_energy():
    n = (16, 16, 16)
    o = Oracle(OracleConfig(n=n, init="user", user=jittered_state(n, 1), q="monotone"))
    f0 = o.fields()
    E0 = sum(total_energy(f0))
    info = o.step(100)
    f1 = o.fields()
    assert info["status"] == 0
    assert abs(sum(total_energy(f1)) - E0) / E0 <= 1e-12
    assert np.array_equal(f1["mass"], f0["mass"])


def test_sedov_radius_with_monotone_q_and_hourglass_control():
    """Like LULESH, the monotone q runs the Sedov blast with hourglass control on: without it the
    zone-crushing failure of R17 comes sooner (the monotone q damps less; at 32^3 it halts with
    EDTMIN at t = 0.10, R24)."""
    n = 32
    cfg = OracleConfig(n=(n, n, n), t_stop=0.3, q="monotone", hg_coef=0.03)
    f, info = oracle.run(cfg, 100000, names=("x", "y", "z", "rho", "e"))
    assert info["status"] == 0 and info["t"] == pytest.approx(0.3, rel=1e-14)
    R = sedov_radius(f, 1.2 / n)
    R_exact = sedov_mod.shock_radius(0.3, 8.0 * cfg.sedov_energy, 1.0, 1.4)
    assert abs(R - R_exact) / R_exact <= sedov_radius_tolerance(1.2 / n, R_exact)
