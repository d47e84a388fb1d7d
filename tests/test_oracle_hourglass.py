"""Pins for the oracle's viscous hourglass control (reading R17 in
DESIGN.md §3; Flanagan-Belytschko form, oracle/hydro_oracle.cpp ``hourglass``).

What pins what:
* base vectors, sign, |h|^2 = 8 and the kappa rho c V^(2/3) factor: unit-cube closed form for
  every mode and direction (gamma = h there, so f_l = -8 kappa rho c h_l e_d);
* the projection C = H M^-1 (the part a plain h-filter lacks): linear velocity fields and rigid
  rotations give zero force on NON-affine hexes, where the unprojected h.u is far from zero;
* momentum: sum_l f_l = 0 on random hexes with random velocities;
* the V^(2/3) exponent: f(s X) = s^2 f(X) for fixed velocities;
* the cycle: a checkerboard hourglass pattern (divergence-free per zone, so pressure never
  resists it) persists with kappa = 0 and is damped with kappa > 0, total energy conserved to
  round-off in both runs; decomposed == undecomposed bitwise with kappa > 0; a gas at rest stays
  bitwise at rest.
"""
import numpy as np
import pytest

import oracle
from oracle import Oracle, OracleConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import total_energy, user_state

CUBE = np.array([[(l & 1), (l >> 1) & 1, (l >> 2) & 1] for l in range(8)], dtype=float)


def _h(alpha):
    """Reference-cube hourglass base vectors written from their definition: xi = 2a-1 etc."""
    xi = 2 * CUBE[:, 0] - 1
    eta = 2 * CUBE[:, 1] - 1
    zeta = 2 * CUBE[:, 2] - 1
    return [eta * zeta, zeta * xi, xi * eta, xi * eta * zeta][alpha]


def _hex(seed, amp=0.25):
    """A non-affine hex: the unit cube with every corner displaced by up to amp."""
    rng = np.random.default_rng(seed)
    return CUBE + amp * (2 * rng.random((8, 3)) - 1)


@pytest.mark.parametrize("alpha", range(4))
@pytest.mark.parametrize("d", range(3))
def test_unit_cube_pure_mode_closed_form(alpha, d):
    B, V, _ = oracle.zone_geometry(CUBE)
    U = np.zeros((8, 3))
    U[:, d] = _h(alpha)
    kappa, rho, c = 0.07, 1.3, 0.9
    F = oracle.zone_hourglass(CUBE, U, B, V, rho, c, kappa)
    want = np.zeros((8, 3))
    want[:, d] = -8.0 * kappa * rho * c * _h(alpha)
    assert np.allclose(F, want, rtol=0, atol=1e-14)


@pytest.mark.parametrize("seed", range(6))
def test_linear_velocity_field_gives_no_force_on_distorted_hex(seed):
    X = _hex(seed)
    B, V, _ = oracle.zone_geometry(X)
    rng = np.random.default_rng(100 + seed)
    A = rng.standard_normal((3, 3))
    U = X @ A.T + rng.standard_normal(3)
    F = oracle.zone_hourglass(X, U, B, V, 1.0, 1.0, 1.0)
    # the unprojected filter h.u is O(1) here; the projected one must vanish to round-off
    raw = max(abs(float(_h(a) @ U[:, d])) for a in range(4) for d in range(3))
    assert raw > 1e-2
    assert np.abs(F).max() <= 1e-12


def test_rigid_rotation_gives_no_force():
    X = _hex(7)
    B, V, _ = oracle.zone_geometry(X)
    w = np.array([0.3, -1.1, 0.7])
    U = np.cross(w, X)
    F = oracle.zone_hourglass(X, U, B, V, 1.0, 2.0, 0.5)
    assert np.abs(F).max() <= 1e-12


@pytest.mark.parametrize("seed", range(6))
def test_momentum_conserving(seed):
    X = _hex(seed)
    B, V, _ = oracle.zone_geometry(X)
    U = np.random.default_rng(200 + seed).standard_normal((8, 3))
    F = oracle.zone_hourglass(X, U, B, V, 1.0, 1.0, 1.0)
    assert np.abs(F).max() > 0.1
    assert np.abs(F.sum(axis=0)).max() <= 1e-13 * np.abs(F).max() * 8


def test_scaling_with_zone_size():
    X = _hex(3)
    U = np.random.default_rng(5).standard_normal((8, 3))
    B, V, _ = oracle.zone_geometry(X)
    F1 = oracle.zone_hourglass(X, U, B, V, 1.0, 1.0, 1.0)
    s = 1.7
    B2, V2, _ = oracle.zone_geometry(s * X)
    F2 = oracle.zone_hourglass(s * X, U, B2, V2, 1.0, 1.0, 1.0)
    assert np.allclose(F2, s * s * F1, rtol=1e-12, atol=1e-14)


def _checkerboard(n, amp=0.01):
    """Uniform gas (rho = e = 1) with u_x = amp (-1)^(j+k) on the nodes (the h1 = eta*zeta
    pattern in every zone: zero S2 divergence) and u_x = 0 on the x walls (reflecting)."""
    s = user_state(n, extent=(1.0, 1.0, 1.0), rho=1.0, e=1.0)
    nz, ny, nx = s["x"].shape
    k, j, i = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    u = amp * (-1.0) ** (j + k)
    u[:, :, 0] = 0.0
    u[:, :, -1] = 0.0
    s["u"] = u
    return s


@pytest.mark.parametrize("kappa", [0.0, 0.01, 0.03])
def test_checkerboard_hourglass_pattern_damped_and_energy_conserved(kappa):
    n = (8, 8, 8)
    cfg = OracleConfig(n=n, extent=(1.0, 1.0, 1.0), init="user", user=_checkerboard(n),
                       hg_coef=kappa)
    o = Oracle(cfg)
    ie0, ke0 = total_energy(o.fields())
    info = o.step(40)
    assert info["status"] == 0
    ie, ke = total_energy(o.fields())
    assert abs((ie + ke) - (ie0 + ke0)) / (ie0 + ke0) <= 1e-12
    if kappa == 0.0:
        assert ke > 0.5 * ke0    # pressure does not resist the pattern
    else:
        assert ke < 0.05 * ke0   # the viscous hourglass force removes it


def test_uniform_gas_at_rest_stays_at_rest_with_hourglass():
    n = (8, 8, 8)
    s = user_state(n, extent=(1.0, 1.0, 1.0), rho=1.0, e=1.0)
    o = Oracle(OracleConfig(n=n, extent=(1.0, 1.0, 1.0), init="user", user=s, hg_coef=0.03))
    f0 = o.fields()
    assert o.step(50)["status"] == 0
    f = o.fields()
    for k in ("x", "y", "z", "u", "v", "w", "e"):
        assert np.array_equal(f[k], f0[k]), k


def test_hourglass_decomposed_equals_undecomposed_bitwise():
    n = (13, 11, 9)
    s = jittered_state(n, 3)
    ref, _ = oracle.run(OracleConfig(n=n, init="user", user=s, hg_coef=0.03), 30)
    dec, _ = oracle.run(OracleConfig(n=n, init="user", user=s, hg_coef=0.03, ndom=(3, 2, 2)), 30)
    for k in ref:
        assert np.array_equal(ref[k], dec[k]), k


def test_sedov_with_hourglass_conserves_energy():
    cfg = OracleConfig(n=(16, 16, 16), hg_coef=0.03)
    o = Oracle(cfg)
    E0 = sum(total_energy(o.fields()))
    assert o.step(60)["status"] == 0
    E = sum(total_energy(o.fields()))
    assert abs(E - E0) / E0 <= 1e-12


def test_long_sedov_needs_hourglass_control():
    """Characterisation (DESIGN.md §13 f1, reading R23): without hourglass control the SG scheme
    lets a zone next to the blast origin be crushed after ~1000 cycles; dt collapses by many
    orders while every volume stays positive.  With no floor (dt_floor < 0) the run freezes
    silently; with the default floor (1e-6 dt^0) it halts with EDTMIN; with kappa = 0.03 the
    same run keeps a normal dt.  Seen identically on the GPU at 448^3 (tools/sedov_front.py).
    A regression guard on the scheme's behaviour, not a pin of its values."""
    n, h = 12, 1.2 / 448
    dts = {}
    for kappa in (0.0, 0.03):
        o = Oracle(OracleConfig(n=(n, n, n), extent=(h * n,) * 3, hg_coef=kappa, dt_floor=-1.0))
        dt0 = o.step(100)["dt"]
        info = o.step(1200)
        assert info["status"] == 0
        dts[kappa] = info["dt"] / dt0
    assert dts[0.0] < 1e-6      # collapsed, silently
    assert dts[0.03] > 0.1      # healthy
    o = Oracle(OracleConfig(n=(n, n, n), extent=(h * n,) * 3))
    info = o.step(2500)  # the floor is crossed at cycle 1295
    assert info["status"] == -7 and 100 < info["cycle"] < 2500 and info["bad_zone"] == -1
    assert info["dt_min_zone"] < 1e-6 * o_dt0(n, h)


def o_dt0(n, h):
    return Oracle(OracleConfig(n=(n, n, n), extent=(h * n,) * 3)).info()["dt"]
