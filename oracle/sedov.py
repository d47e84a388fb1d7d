"""Sedov-Taylor point-blast similarity solution (TEST INFRASTRUCTURE ONLY).

PAPER.md L637-642 runs "a 3D Sedov blastwave problem [18]" (ref [18] = Sedov 1946, L1212-1214).
The paper gives no formula; this is the textbook self-similar solution used to pin the oracle's
shock radius (reading R16):

    R(t) = xi0 * (E t^2 / rho0)^(1/5),   xi0 = alpha^(-1/5),
    alpha = (16 pi / 25) * int_0^1 (psi phi^2 / 2 + pi_/(gamma-1)) xi^2 dxi,

with u = Rdot*phi(xi), rho = rho0*psi(xi), p = rho0*Rdot^2*pi_(xi), xi = r/R, and the strong-shock
values phi(1) = pi_(1) = 2/(gamma+1), psi(1) = (gamma+1)/(gamma-1).  The three ODEs (mass,
momentum, entropy in spherical symmetry with R ~ t^(2/5)) are

    (phi-xi) psi' + psi (phi' + 2 phi/xi) = 0
    (phi-xi) phi' + pi_'/psi = 3/2 phi
    (phi-xi) pi_' - gamma pi_ (phi-xi) psi'/psi = 3 pi_

integrated inward from xi = 1 with classical RK4 in s = ln(xi).  Nothing here is shared with the
CUDA path (it has no Sedov analytics at all).
"""
from __future__ import annotations

import math


def _rhs(xi, y, g):
    phi, psi, pi_, _ = y
    w = phi - xi
    num = 1.5 * phi - (3.0 * pi_ - 2.0 * g * pi_ * phi / xi) / (w * psi)
    den = w - g * pi_ / (w * psi)
    dphi = num / den
    dpsi = (-2.0 * psi * phi / xi - psi * dphi) / w
    dpi = (3.0 * pi_ - g * pi_ * (2.0 * phi / xi + dphi)) / w
    dI = (0.5 * psi * phi * phi + pi_ / (g - 1.0)) * xi * xi
    # d/ds = xi d/dxi
    return (xi * dphi, xi * dpsi, xi * dpi, xi * dI)


def profile(gamma: float, s_min: float = -12.0, steps: int = 60000):
    """Integrate from xi=1 down to xi=exp(s_min).  Returns (alpha, samples) where samples is a
    list of (xi, phi, psi, pi_) at every step."""
    g = gamma
    y = [2.0 / (g + 1.0), (g + 1.0) / (g - 1.0), 2.0 / (g + 1.0), 0.0]
    h = s_min / steps
    s = 0.0
    out = [(1.0, y[0], y[1], y[2])]
    for _ in range(steps):
        xi0 = math.exp(s)
        k1 = _rhs(xi0, y, g)
        xi1 = math.exp(s + 0.5 * h)
        k2 = _rhs(xi1, [y[i] + 0.5 * h * k1[i] for i in range(4)], g)
        k3 = _rhs(xi1, [y[i] + 0.5 * h * k2[i] for i in range(4)], g)
        xi2 = math.exp(s + h)
        k4 = _rhs(xi2, [y[i] + h * k3[i] for i in range(4)], g)
        y = [y[i] + (h / 6.0) * (k1[i] + 2 * k2[i] + 2 * k3[i] + k4[i]) for i in range(4)]
        s += h
        out.append((math.exp(s), y[0], y[1], y[2]))
    # I accumulated from xi=1 down: int_1^xi -> negate
    integral = -y[3]
    alpha = 16.0 * math.pi / 25.0 * integral
    return alpha, out


def alpha(gamma: float) -> float:
    return profile(gamma)[0]


def xi0(gamma: float) -> float:
    return alpha(gamma) ** -0.2


def shock_radius(t: float, energy: float, rho0: float = 1.0, gamma: float = 1.4) -> float:
    """Full-space shock radius for total blast energy ``energy`` at time ``t``."""
    return xi0(gamma) * (energy * t * t / rho0) ** 0.2


if __name__ == "__main__":
    for g in (1.4, 5.0 / 3.0):
        a = alpha(g)
        print(g, a, a ** -0.2)
