"""Pins for the oracle's S2 geometry (orc_zone_geometry): readings R2-R4 of DESIGN.md §3.

Each check compares the oracle with something other than itself: exact values of simple
solids, det(M) for parallelepipeds, a 2-point Gauss-Legendre integral of det J of the trilinear
map, an independent 24-tetrahedron decomposition, and finite-difference gradients of V.
"""
import itertools

import numpy as np
import pytest

import oracle

CORNERS = np.array([[l & 1, (l >> 1) & 1, (l >> 2) & 1] for l in range(8)], dtype=float)


def hex_from_map(f):
    return np.array([f(*c) for c in CORNERS])


def trilinear_volume_gauss(X):
    """Integral of det J over [0,1]^3 (2-point Gauss-Legendre is exact: degree <= 2 per axis)."""
    g = [0.5 - 0.5 / np.sqrt(3.0), 0.5 + 0.5 / np.sqrt(3.0)]
    V = 0.0
    for s, t, r in itertools.product(g, g, g):
        J = np.zeros((3, 3))
        for l, (a, b, c) in enumerate(CORNERS):
            ws = (s if a else 1 - s)
            wt = (t if b else 1 - t)
            wr = (r if c else 1 - r)
            ds = (1 if a else -1) * wt * wr
            dt = ws * (1 if b else -1) * wr
            dr = ws * wt * (1 if c else -1)
            J[:, 0] += ds * X[l]
            J[:, 1] += dt * X[l]
            J[:, 2] += dr * X[l]
        V += 0.125 * np.linalg.det(J)
    return V


FACES = [(0, 2, 6, 4), (1, 3, 7, 5), (0, 1, 5, 4), (2, 3, 7, 6), (0, 1, 3, 2), (4, 5, 7, 6)]


def _oriented_faces():
    """Orient each face cycle outward on the unit cube (test-side construction)."""
    X = CORNERS
    C = X.mean(axis=0)
    out = []
    for f in FACES:
        n = np.cross(X[f[1]] - X[f[0]], X[f[2]] - X[f[0]])
        ctr = X[list(f)].mean(axis=0)
        out.append(f if np.dot(n, ctr - C) > 0 else f[::-1])
    return out


def tet24_volume(X):
    C = X.mean(axis=0)
    V = 0.0
    for f in _oriented_faces():
        F = X[list(f)].mean(axis=0)
        for i in range(4):
            a, b = X[f[i]], X[f[(i + 1) % 4]]
            V += np.linalg.det(np.array([a - C, b - C, F - C])) / 6.0
    return V


def rand_hex(rng, jitter):
    return CORNERS + jitter * (2 * rng.random((8, 3)) - 1)


def test_unit_cube_exact():
    B, V, L = oracle.zone_geometry(CORNERS)
    assert V == 1.0
    assert L == 1.0
    assert np.all(B.sum(axis=0) == 0.0)
    expect = 0.25 * (2 * CORNERS - 1)  # B_l = 0.25*(s(a), s(b), s(c)) for the unit cube
    assert np.array_equal(B, expect)


def test_box_characteristic_length_is_min_side():
    X = CORNERS * np.array([1.0, 2.0, 3.0])
    B, V, L = oracle.zone_geometry(X)
    assert V == 6.0
    assert L == 1.0  # V / max face area = 6/6


def test_parallelepiped_volume_is_det():
    rng = np.random.default_rng(11)
    for _ in range(100):
        M = np.eye(3) + 0.4 * (2 * rng.random((3, 3)) - 1)
        b = 5 * rng.random(3)
        X = hex_from_map(lambda a, bb, c: b + M @ np.array([a, bb, c]))
        _, V, _ = oracle.zone_geometry(X)
        assert V == pytest.approx(np.linalg.det(M), rel=1e-13)


@pytest.mark.parametrize("jitter", [0.05, 0.15, 0.3])
def test_volume_equals_trilinear_integral_and_24_tets(jitter):
    rng = np.random.default_rng(int(jitter * 1000))
    for _ in range(100):
        X = rand_hex(rng, jitter)
        _, V, _ = oracle.zone_geometry(X)
        assert V == pytest.approx(trilinear_volume_gauss(X), rel=1e-13)
        assert V == pytest.approx(tet24_volume(X), rel=1e-13)


def test_corner_vectors_sum_to_zero():
    rng = np.random.default_rng(3)
    for _ in range(100):
        X = rand_hex(rng, 0.3)
        B, _, _ = oracle.zone_geometry(X)
        assert np.abs(B.sum(axis=0)).max() <= 1e-15 * np.abs(B).max() * 8


def _fd_gradient(X, h=1e-6):
    G = np.zeros((8, 3))
    for l in range(8):
        for d in range(3):
            Xp = X.copy()
            Xm = X.copy()
            Xp[l, d] += h
            Xm[l, d] -= h
            G[l, d] = (oracle.zone_geometry(Xp)[1] - oracle.zone_geometry(Xm)[1]) / (2 * h)
    return G


def test_corner_vectors_are_volume_gradient_on_affine_hexes():
    """B_l = dV/dX_l holds exactly for affine (parallelepiped) hexes.  For any other hex,
    including planar-faced ones such as a frustum, the quarter-face-area corner vectors of
    reading R2 differ from the exact gradient (note to R2) -- asserted below so the
    caveat stays documented."""
    rng = np.random.default_rng(5)
    for _ in range(5):
        M = np.eye(3) + 0.3 * (2 * rng.random((3, 3)) - 1)
        X = hex_from_map(lambda a, b, c: M @ np.array([a, b, c]) + 1.0)
        B, _, _ = oracle.zone_geometry(X)
        assert np.abs(B - _fd_gradient(X)).max() < 1e-8
    frustum = hex_from_map(lambda a, b, c: np.array([0.5 + (a - 0.5) * (1 - 0.4 * c),
                                                      0.5 + (b - 0.5) * (1 - 0.4 * c), c]))
    B, _, _ = oracle.zone_geometry(frustum)
    assert np.abs(B - _fd_gradient(frustum)).max() > 1e-3


def test_mirror_flips_sign_and_rigid_motion_invariance():
    rng = np.random.default_rng(9)
    X = rand_hex(rng, 0.2)
    B, V, L = oracle.zone_geometry(X)
    Xm = X * np.array([-1.0, 1.0, 1.0])
    _, Vm, _ = oracle.zone_geometry(Xm)
    assert Vm == pytest.approx(-V, rel=1e-14)
    th = 0.7
    Q = np.array([[np.cos(th), -np.sin(th), 0], [np.sin(th), np.cos(th), 0], [0, 0, 1.0]])
    Xr = X @ Q.T + np.array([3.0, -2.0, 1.0])
    Br, Vr, Lr = oracle.zone_geometry(Xr)
    assert Vr == pytest.approx(V, rel=1e-13)
    assert Lr == pytest.approx(L, rel=1e-13)
    assert np.abs(Br - B @ Q.T).max() < 1e-13
