"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

Holds none of the method's arithmetic: only random numbers and the initial lattice.  The
recipe is DESIGN.md §6 (reading R11):

* counter-based splitmix64, double = (r >> 11) * 2**-53, drawn in a fixed order;
* lattice nodes at ``origin + (extent*i)/n`` (reading R1);
* "jittered" state (the parity input of BASELINE.json config 0 / SURVEY §8d L7): interior node
  positions displaced by 0.1*h*(2U-1) per component, wall nodes only tangentially; velocities
  0.05*(2U-1) with zero normal component on walls; rho, e = 1 + 0.5U per zone.
  Draw order: positions (nodes x-fastest, components x,y,z), velocities (same order), rho
  (zones x-fastest), e (zones x-fastest).
"""
from __future__ import annotations

from typing import Dict, Sequence

import numpy as np

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(seed: int, start: int, count: int) -> np.ndarray:
    """Outputs ``start .. start+count-1`` of the splitmix64 stream seeded with ``seed``."""
    with np.errstate(over="ignore"):
        k = np.arange(start + 1, start + count + 1, dtype=np.uint64)
        z = np.uint64(seed) + k * _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def uniform01(seed: int, start: int, count: int) -> np.ndarray:
    """U in [0,1): (r >> 11) * 2**-53."""
    return (splitmix64(seed, start, count) >> np.uint64(11)).astype(np.float64) * 2.0 ** -53


def lattice(n: Sequence[int], origin=(0.0, 0.0, 0.0), extent=(1.2, 1.2, 1.2)) -> Dict[str, np.ndarray]:
    """Node coordinates ``origin + (extent*i)/n`` as (nz+1, ny+1, nx+1) arrays (reading R1)."""
    nx, ny, nz = (int(v) for v in n)
    cx = origin[0] + (extent[0] * np.arange(nx + 1, dtype=np.float64)) / float(nx)
    cy = origin[1] + (extent[1] * np.arange(ny + 1, dtype=np.float64)) / float(ny)
    cz = origin[2] + (extent[2] * np.arange(nz + 1, dtype=np.float64)) / float(nz)
    Z, Y, X = np.meshgrid(cz, cy, cx, indexing="ij")
    return {"x": np.ascontiguousarray(X), "y": np.ascontiguousarray(Y), "z": np.ascontiguousarray(Z)}


def jittered_state(n: Sequence[int], seed: int, origin=(0.0, 0.0, 0.0),
                   extent=(1.2, 1.2, 1.2), jitter=0.1, speed=0.05) -> Dict[str, np.ndarray]:
    """USER-init arrays {x,y,z,u,v,w (nodes), rho,e (zones)} of the jittered parity input."""
    nx, ny, nz = (int(v) for v in n)
    nn = (nx + 1) * (ny + 1) * (nz + 1)
    nzn = nx * ny * nz
    out = lattice(n, origin, extent)
    shape = (nz + 1, ny + 1, nx + 1)
    idx = np.indices(shape)  # (k, j, i)
    gi = [idx[2], idx[1], idx[0]]
    nvec = [nx, ny, nz]
    off = 0
    draws = uniform01(seed, off, 3 * nn).reshape(nn, 3)
    off += 3 * nn
    for a, nm in enumerate(("x", "y", "z")):
        h = extent[a] / nvec[a]
        wall = (gi[a] == 0) | (gi[a] == nvec[a])
        d = (jitter * h) * (2.0 * draws[:, a].reshape(shape) - 1.0)
        out[nm] = out[nm] + np.where(wall, 0.0, d)
    draws = uniform01(seed, off, 3 * nn).reshape(nn, 3)
    off += 3 * nn
    for a, nm in enumerate(("u", "v", "w")):
        wall = (gi[a] == 0) | (gi[a] == nvec[a])
        out[nm] = np.where(wall, 0.0, speed * (2.0 * draws[:, a].reshape(shape) - 1.0))
    zshape = (nz, ny, nx)
    out["rho"] = 1.0 + 0.5 * uniform01(seed, off, nzn).reshape(zshape)
    off += nzn
    out["e"] = 1.0 + 0.5 * uniform01(seed, off, nzn).reshape(zshape)
    return {k: np.ascontiguousarray(v) for k, v in out.items()}


def sedov_grid(n: Sequence[int]) -> Dict[str, object]:
    """The Sedov workload shape of BASELINE.json configs (box [0,1.2]^3, reading R10)."""
    return {"n": tuple(int(v) for v in n), "origin": (0.0, 0.0, 0.0), "extent": (1.2, 1.2, 1.2)}
