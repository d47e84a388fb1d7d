"""Pins for the oracle's zone physics S2-S6 (orc_zone_state): readings R5-R8 of DESIGN.md §3.

Closed forms on zones where the geometry is exact (boxes, homologous compression of a cube, for
which sum_l u_l.B_l = dV/dt = -3 kappa V exactly because u is linear and V = 1/3 sum X_l.B_l).
"""
import math

import numpy as np
import pytest

import oracle

CORNERS = np.array([[l & 1, (l >> 1) & 1, (l >> 2) & 1] for l in range(8)], dtype=float)


def cube(h, origin=(0.3, 0.2, 0.1)):
    return np.asarray(origin) + h * CORNERS


@pytest.mark.parametrize("gamma", [1.4, 5.0 / 3.0])
def test_gas_at_rest(gamma):
    h, m, e = 0.25, 0.03, 2.5
    X = cube(h)
    r = oracle.zone_state(X, np.zeros((8, 3)), m, e, 0.01, gamma=gamma)
    V = h ** 3
    rho = m / V
    p = (gamma - 1) * rho * e
    c = math.sqrt(gamma * (gamma - 1) * e)
    assert r["V"] == pytest.approx(V, rel=1e-15)
    assert r["rho"] == pytest.approx(rho, rel=1e-15)
    assert r["ep"] == e  # DV = 0: the predictor leaves e unchanged
    assert r["p"] == pytest.approx(p, rel=1e-15)
    assert r["c"] == pytest.approx(c, rel=1e-15)
    assert r["q"] == 0.0
    assert r["P"] == r["p"]
    assert r["dtz"] == pytest.approx(0.3 * h / c, rel=1e-15)  # S6: cfl*L/c, dt_vol = inf


@pytest.mark.parametrize("hh", [0.0, 1e-3])
@pytest.mark.parametrize("ql,qq", [(0.5, 2.0), (0.25, 1.0), (0.0, 0.0)])
def test_homologous_compression(hh, ql, qq):
    gamma, h, m, e, kappa = 1.4, 0.2, 0.011, 1.7, 0.8
    X = cube(h)
    Xc = X.mean(axis=0)
    U = -kappa * (X - Xc)
    r = oracle.zone_state(X, U, m, e, hh, gamma=gamma, q_lin=ql, q_quad=qq)
    V = h ** 3
    rho = m / V
    DV = -3.0 * kappa * V
    D = DV / V
    pt = (gamma - 1) * rho * e
    ep = e - hh * pt * DV / m
    p = (gamma - 1) * rho * ep
    c = math.sqrt(gamma * (gamma - 1) * ep)
    s = h * (-D)
    qr = s * (qq * s + ql * c)
    q = rho * qr
    assert r["ep"] == pytest.approx(ep, rel=1e-14)
    assert r["p"] == pytest.approx(p, rel=1e-14)
    assert r["c"] == pytest.approx(c, rel=1e-14)
    assert r["q"] == pytest.approx(q, rel=1e-13, abs=0.0)
    assert r["P"] == pytest.approx(p + q, rel=1e-13)
    dtc = 0.3 * h / math.sqrt(c * c + 2 * qr)
    dtv = 0.1 / abs(D)
    assert r["dtz"] == pytest.approx(min(dtc, dtv), rel=1e-13)
    if hh > 0:
        assert r["ep"] > e  # compression heats


def test_expansion_has_no_viscosity():
    X = cube(0.2)
    U = 0.5 * (X - X.mean(axis=0))
    r = oracle.zone_state(X, U, 0.01, 1.0, 1e-3)
    assert r["q"] == 0.0
    assert r["dtz"] == pytest.approx(min(0.3 * 0.2 / r["c"], 0.1 / 1.5), rel=1e-13)


def test_viscosity_continuous_at_zero_divergence():
    X = cube(0.2)
    qs = []
    for kappa in (1e-4, 1e-6, 1e-8):
        U = -kappa * (X - X.mean(axis=0))
        qs.append(oracle.zone_state(X, U, 0.01, 1.0, 0.0)["q"])
    assert qs[0] > qs[1] > qs[2] > 0
    assert qs[2] < 1e-7  # -> 0 linearly in kappa


def test_negative_energy_is_clamped_in_eos_only():
    X = cube(0.2)
    U = -0.3 * (X - X.mean(axis=0))
    r = oracle.zone_state(X, U, 0.01, -0.5, 0.0)
    assert r["p"] == 0.0 and r["c"] == 0.0
    assert r["ep"] == -0.5  # e itself is not clamped (reading R6)
    # sigma = sqrt(2 qr) still gives a finite dt
    assert math.isfinite(r["dtz"]) and r["dtz"] > 0


def test_zero_energy_at_rest_has_infinite_dt():
    r = oracle.zone_state(cube(0.2), np.zeros((8, 3)), 0.01, 0.0, 0.0)
    assert r["P"] == 0.0 and r["dtz"] == math.inf
