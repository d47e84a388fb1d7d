"""Exact Riemann solver for the 1-D Euler equations, ideal gas (Toro, "Riemann Solvers and
Numerical Methods for Fluid Dynamics", ch. 4).  Test-side pin for the oracle's shock capturing
(Sod tube); shares nothing with oracle/ or the CUDA path."""
import math

import numpy as np


def _f(p, rho, pk, ck, g):
    if p > pk:  # shock
        A = 2.0 / ((g + 1) * rho)
        B = (g - 1) / (g + 1) * pk
        return (p - pk) * math.sqrt(A / (p + B)), math.sqrt(A / (B + p)) * (1 - (p - pk) / (2 * (B + p)))
    r = p / pk  # rarefaction
    return (2 * ck / (g - 1)) * (r ** ((g - 1) / (2 * g)) - 1), (1 / (rho * ck)) * r ** (-(g + 1) / (2 * g))


def star(rl, ul, pl, rr, ur, pr, g):
    cl, cr = math.sqrt(g * pl / rl), math.sqrt(g * pr / rr)
    p = max(1e-8, 0.5 * (pl + pr))
    for _ in range(100):
        fl, dl = _f(p, rl, pl, cl, g)
        fr, dr = _f(p, rr, pr, cr, g)
        dp = (fl + fr + (ur - ul)) / (dl + dr)
        p = max(1e-12, p - dp)
        if abs(dp) < 1e-14 * p:
            break
    fl, _ = _f(p, rl, pl, cl, g)
    fr, _ = _f(p, rr, pr, cr, g)
    return p, 0.5 * (ul + ur) + 0.5 * (fr - fl)


def sample(x, t, x0, left, right, g):
    """Density, velocity, pressure at positions x, time t, interface at x0."""
    rl, ul, pl = left
    rr, ur, pr = right
    cl, cr = math.sqrt(g * pl / rl), math.sqrt(g * pr / rr)
    ps, us = star(rl, ul, pl, rr, ur, pr, g)
    out = np.zeros((3, len(x)))
    for n, xi in enumerate(x):
        S = (xi - x0) / t
        if S <= us:  # left of contact
            if ps > pl:
                rs = rl * ((ps / pl + (g - 1) / (g + 1)) / ((g - 1) / (g + 1) * ps / pl + 1))
                SL = ul - cl * math.sqrt((g + 1) / (2 * g) * ps / pl + (g - 1) / (2 * g))
                w = (rl, ul, pl) if S <= SL else (rs, us, ps)
            else:
                rs = rl * (ps / pl) ** (1 / g)
                cs = cl * (ps / pl) ** ((g - 1) / (2 * g))
                SH, ST = ul - cl, us - cs
                if S <= SH:
                    w = (rl, ul, pl)
                elif S >= ST:
                    w = (rs, us, ps)
                else:
                    u = 2 / (g + 1) * (cl + (g - 1) / 2 * ul + S)
                    c = 2 / (g + 1) * (cl + (g - 1) / 2 * (ul - S))
                    r = rl * (c / cl) ** (2 / (g - 1))
                    w = (r, u, pl * (c / cl) ** (2 * g / (g - 1)))
        else:
            if ps > pr:
                rs = rr * ((ps / pr + (g - 1) / (g + 1)) / ((g - 1) / (g + 1) * ps / pr + 1))
                SR = ur + cr * math.sqrt((g + 1) / (2 * g) * ps / pr + (g - 1) / (2 * g))
                w = (rr, ur, pr) if S >= SR else (rs, us, ps)
            else:
                rs = rr * (ps / pr) ** (1 / g)
                cs = cr * (ps / pr) ** ((g - 1) / (2 * g))
                SH, ST = ur + cr, us + cs
                if S >= SH:
                    w = (rr, ur, pr)
                elif S <= ST:
                    w = (rs, us, ps)
                else:
                    u = 2 / (g + 1) * (-cr + (g - 1) / 2 * ur + S)
                    c = 2 / (g + 1) * (cr - (g - 1) / 2 * (ur - S))
                    r = rr * (c / cr) ** (2 / (g - 1))
                    w = (r, u, pr * (c / cr) ** (2 * g / (g - 1)))
        out[:, n] = w
    return out
