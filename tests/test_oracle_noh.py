"""Oracle pin: Noh's planar implosion (gamma = 5/3), a strong-shock problem with an exact
solution, for both artificial viscosities (readings R7 and R24).  Cold gas (e = 0) streams at
u = -1 onto a reflecting wall at x = 0; the exact solution is a shock leaving the wall at speed
(gamma-1)/2 |u| = 1/3 with the gas behind it at rest at rho = (gamma+1)/(gamma-1) = 4,
p = 4/3, and the gas ahead untouched (rho = 1).  Pinned: the post-shock plateau (away from the
wall-heating zones next to the wall, a known property of artificial-viscosity schemes), the
shock position within two zones, the undisturbed pre-shock gas, first-order convergence of
the plateau region, and exact total-energy conservation."""
import numpy as np
import pytest

import oracle
from oracle import Oracle, OracleConfig
from tests.helpers import total_energy, user_state

G = 5.0 / 3.0


def noh_state(N):
    n, ext = (N, 1, 1), (1.0, 1.0, 1.0)
    s = user_state(n, extent=ext, e=0.0)
    s["u"][:] = -1.0
    s["u"][:, :, 0] = 0.0  # the wall node
    return n, ext, s


def _run(N, q, t=0.6):
    n, ext, s = noh_state(N)
    f, info = oracle.run(OracleConfig(n=n, extent=ext, init="user", user=s, gamma=G, t_stop=t,
                                      reflect_mask=0b111101, q=q), 100000)
    assert info["status"] == 0 and info["t"] == pytest.approx(t, rel=1e-14)
    x = f["x"][0, 0]
    return f, 0.5 * (x[:-1] + x[1:])


@pytest.mark.parametrize("q", ["scalar", "monotone"])
def test_planar_noh_against_exact_solution(q):
    for N in (100, 200):
        f, xc = _run(N, q)
        h = 1.0 / N
        r, p = f["rho"].ravel(), f["p"].ravel()
        plateau = (xc > 0.05) & (xc < 0.15)
        assert np.abs(r[plateau] - 4.0).max() <= 0.01 * 4.0
        assert np.abs(p[plateau] - 4.0 / 3.0).max() <= 0.01 * 4.0 / 3.0
        shock = xc[np.nonzero(r > 2.5)[0].max()]
        assert abs(shock - 0.2) <= 2.0 * h
        ahead = (xc > 0.3) & (xc < 0.9)
        assert np.abs(r[ahead] - 1.0).max() <= 1e-12  # untouched, uniformly streaming gas
        xn, un = f["x"][0, 0], f["u"][0, 0]
        moving = (xn > 0.3) & (xn < 0.9)
        assert np.abs(un[moving] + 1.0).max() <= 1e-12
        assert 1.5 < r[0] < 4.0  # wall heating: the zone next to the wall is under-dense


def test_noh_energy_conserved():
    n, ext, s = noh_state(64)
    o = Oracle(OracleConfig(n=n, extent=ext, init="user", user=s, gamma=G, reflect_mask=0b111101))
    f0 = o.fields()
    E0 = sum(total_energy(f0))
    o.step(200)
    f1 = o.fields()
    assert abs(sum(total_energy(f1)) - E0) / E0 <= 1e-12
