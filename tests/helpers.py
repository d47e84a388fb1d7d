"""Test-side helpers (no method arithmetic beyond diagnostics written from their definitions)."""
import math

import numpy as np

from paper_conf_icppw_pearce18_b200.inputs import lattice


def node_mass(mass):
    """m_p = 1/8 sum of the masses of the (up to 8) zones around each node."""
    nz, ny, nx = mass.shape
    mp = np.zeros((nz + 1, ny + 1, nx + 1))
    for a in (0, 1):
        for b in (0, 1):
            for c in (0, 1):
                mp[c:c + nz, b:b + ny, a:a + nx] += mass
    return 0.125 * mp


def total_energy(f):
    """(internal, kinetic) with exact (fsum) summation."""
    ie = math.fsum((f["mass"] * f["e"]).ravel())
    mp = node_mass(f["mass"])
    ke = math.fsum((0.5 * mp * (f["u"] ** 2 + f["v"] ** 2 + f["w"] ** 2)).ravel())
    return ie, ke


def user_state(n, extent=(1.2, 1.2, 1.2), origin=(0.0, 0.0, 0.0), rho=1.0, e=1.0):
    nx, ny, nz = n
    s = lattice(n, origin, extent)
    for k in ("u", "v", "w"):
        s[k] = np.zeros_like(s["x"])
    s["rho"] = np.full((nz, ny, nx), rho, dtype=float)
    s["e"] = np.full((nz, ny, nx), e, dtype=float)
    return s


def zone_centroids(f):
    nz, ny, nx = f["e"].shape
    out = []
    for nm in ("x", "y", "z"):
        X = f[nm]
        out.append(sum(X[c:c + nz, b:b + ny, a:a + nx] for a in (0, 1) for b in (0, 1)
                       for c in (0, 1)) / 8.0)
    return out


def sedov_radius(f, h):
    """Reading R16: bin zones by centroid radius (bin width h/2); the radius of the bin with the
    largest mean density.  Quantisation error <= h/4."""
    w = 0.5 * h
    xc, yc, zc = zone_centroids(f)
    r = np.sqrt(xc ** 2 + yc ** 2 + zc ** 2)
    bins = (r / w).astype(int).ravel()
    nb = bins.max() + 1
    s = np.bincount(bins, f["rho"].ravel(), nb)
    cnt = np.bincount(bins, None, nb)
    mean = s / np.maximum(cnt, 1)
    return (np.argmax(mean) + 0.5) * w


def sedov_radius_tolerance(h, R):
    """Reading R16 as calibrated on the oracle: 3 % plus the bin quantisation h/(4R)."""
    return 0.03 + 0.25 * h / R


def rel_err(a, b):
    """Reading R15: max|a-b| / max(max|b|, 1e-300)."""
    a = np.asarray(a)
    b = np.asarray(b)
    den = max(float(np.abs(b).max()) if b.size else 0.0, 1e-300)
    return float(np.abs(a - b).max()) / den if b.size else 0.0
