"""Oracle: plain single-threaded C++ fp64 reference of the Lagrangian hydro cycle.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  It shares no code with
the CUDA product path (``include/hydro.h``, ``paper_conf_icppw_pearce18_b200/``).

The cycle it computes is SURVEY.md §8c (restated in DESIGN.md §3): the paper (PAPER.md
L637-642, L672) only fixes the workload, a 3-D Sedov blast wave run by a hydro code, on a
block-structured mesh decomposed into domains (L525-572).

Parity status per function: orc_zone_geometry, orc_zone_state, the cycle
(orc_step) and the decomposition are pinned by tests/test_oracle_*.py; nothing is unpinned.
"""
from __future__ import annotations

import ctypes as C
import math
import os
from dataclasses import dataclass, field
from typing import Dict, Optional, Sequence

import numpy as np

from . import _build

NODE_FIELDS = ("x", "y", "z", "u", "v", "w")
ZONE_FIELDS = ("rho", "e", "p", "q", "c", "vol", "mass")
ALL_FIELDS = NODE_FIELDS + ZONE_FIELDS

_lib = None


def lib() -> C.CDLL:
    global _lib
    if _lib is None:
        path = _build.build()
        L = C.CDLL(path)
        L.orc_create.argtypes = [C.POINTER(_Config), C.POINTER(C.c_void_p)]
        L.orc_create.restype = C.c_int
        L.orc_step.argtypes = [C.c_void_p, C.c_int32, C.POINTER(_Info)]
        L.orc_step.restype = C.c_int
        L.orc_get_fields.argtypes = [C.c_void_p, C.c_uint32, C.POINTER(C.POINTER(C.c_double))]
        L.orc_get_fields.restype = C.c_int
        L.orc_info_get.argtypes = [C.c_void_p, C.POINTER(_Info)]
        L.orc_destroy.argtypes = [C.c_void_p]
        L.orc_destroy.restype = None
        L.orc_last_error.restype = C.c_char_p
        L.orc_zone_geometry.argtypes = [C.c_void_p, C.c_void_p, C.POINTER(C.c_double),
                                        C.POINTER(C.c_double)]
        L.orc_zone_geometry.restype = None
        L.orc_zone_state.argtypes = [C.c_void_p, C.c_void_p] + [C.c_double] * 8 + [C.c_void_p]
        L.orc_zone_state.restype = None
        L.orc_zone_hourglass.argtypes = [C.c_void_p] * 3 + [C.c_double] * 4 + [C.c_void_p]
        L.orc_zone_hourglass.restype = None
        L.orc_zone_strain.argtypes = [C.c_void_p] * 4
        L.orc_zone_strain.restype = None
        L.orc_mono_limiter.argtypes = [C.c_double] * 3
        L.orc_mono_limiter.restype = C.c_double
        _lib = L
    return _lib


class _Config(C.Structure):
    _fields_ = [
        ("n", C.c_int64 * 3),
        ("origin", C.c_double * 3),
        ("extent", C.c_double * 3),
        ("ndom", C.c_int32 * 3),
        ("cuts", C.POINTER(C.c_int64) * 3),
        ("gamma", C.c_double), ("q_lin", C.c_double), ("q_quad", C.c_double),
        ("cfl", C.c_double), ("c_vol", C.c_double), ("dt_growth", C.c_double),
        ("dt_max", C.c_double), ("dt_init", C.c_double), ("t_stop", C.c_double),
        ("dt_first", C.c_double), ("t0", C.c_double),
        ("reflect_mask", C.c_uint32),
        ("init_kind", C.c_int32),
        ("rho0", C.c_double), ("e0", C.c_double), ("sedov_energy", C.c_double),
        ("user", C.POINTER(C.c_double) * 8),
        ("hg_coef", C.c_double),
        ("dt_floor", C.c_double),
        ("q_kind", C.c_int32),
    ]


class _Info(C.Structure):
    _fields_ = [("t", C.c_double), ("dt", C.c_double), ("cycle", C.c_int64),
                ("dt_min_zone", C.c_double), ("bad_zone", C.c_int64)]


INIT = {"sedov": 0, "user": 1, "user_mass": 2}


@dataclass
class OracleConfig:
    """Oracle parameters.  Defaults are the readings of DESIGN.md §3 (R7, R8, R9, R10)."""
    n: Sequence[int] = (32, 32, 32)
    origin: Sequence[float] = (0.0, 0.0, 0.0)
    extent: Sequence[float] = (1.2, 1.2, 1.2)
    ndom: Sequence[int] = (1, 1, 1)
    cuts: Optional[Sequence[Sequence[int]]] = None
    gamma: float = 1.4
    q_lin: float = 0.5
    q_quad: float = 2.0
    cfl: float = 0.3
    c_vol: float = 0.1
    dt_growth: float = 1.1
    dt_max: float = math.inf
    dt_init: float = math.inf
    t_stop: float = 0.0
    dt_first: float = 0.0
    t0: float = 0.0
    reflect_mask: int = 0x3F
    init: str = "sedov"
    rho0: float = 1.0
    e0: float = 0.0
    sedov_energy: float = 0.851072 / 8.0   # reading R10: octant share, R(t=1)=1 for gamma=1.4
    user: Optional[Dict[str, np.ndarray]] = None
    hg_coef: float = 0.0                  # reading R17 / SURVEY §8f f1: hourglass kappa, 0 = off
    dt_floor: float = 0.0                 # reading R23: > 0 absolute, 0 = 1e-6 dt^0, < 0 none
    q: str = "scalar"                     # "scalar" (reading R7) | "monotone" (reading R24)


class OracleError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"oracle error {code}: {msg}")
        self.code = code


class Oracle:
    """One oracle run.  ``fields()`` returns global arrays shaped (nz+1,ny+1,nx+1) for nodes and
    (nz,ny,nx) for zones (x fastest in memory)."""

    def __init__(self, cfg: OracleConfig):
        self.cfg = cfg
        L = lib()
        c = _Config()
        self._keep = []
        for a in range(3):
            c.n[a] = int(cfg.n[a])
            c.origin[a] = float(cfg.origin[a])
            c.extent[a] = float(cfg.extent[a])
            c.ndom[a] = int(cfg.ndom[a])
            if cfg.cuts is not None and cfg.cuts[a] is not None:
                arr = np.ascontiguousarray(cfg.cuts[a], dtype=np.int64)
                self._keep.append(arr)
                c.cuts[a] = arr.ctypes.data_as(C.POINTER(C.c_int64))
        for k in ("gamma", "q_lin", "q_quad", "cfl", "c_vol", "dt_growth", "dt_max", "dt_init",
                  "t_stop", "dt_first", "t0", "rho0", "e0", "sedov_energy", "hg_coef",
                  "dt_floor"):
            setattr(c, k, float(getattr(cfg, k)))
        c.reflect_mask = int(cfg.reflect_mask)
        c.init_kind = INIT[cfg.init]
        c.q_kind = {"scalar": 0, "monotone": 1}[cfg.q]
        if cfg.init != "sedov":
            names = ("x", "y", "z", "u", "v", "w", "rho" if cfg.init == "user" else "mass", "e")
            for f, nm in enumerate(names):
                arr = np.ascontiguousarray(cfg.user[nm], dtype=np.float64).ravel()
                self._keep.append(arr)
                c.user[f] = arr.ctypes.data_as(C.POINTER(C.c_double))
        h = C.c_void_p()
        rc = L.orc_create(C.byref(c), C.byref(h))
        if rc != 0:
            raise OracleError(rc, L.orc_last_error().decode())
        self._h = h
        self._keep = []

    def step(self, ncycles: int) -> dict:
        info = _Info()
        rc = lib().orc_step(self._h, int(ncycles), C.byref(info))
        d = self._info_dict(info)
        d["status"] = rc
        return d

    def info(self) -> dict:
        info = _Info()
        lib().orc_info_get(self._h, C.byref(info))
        return self._info_dict(info)

    @staticmethod
    def _info_dict(info: "_Info") -> dict:
        return {"t": info.t, "dt": info.dt, "cycle": info.cycle,
                "dt_min_zone": info.dt_min_zone, "bad_zone": info.bad_zone}

    def fields(self, names: Sequence[str] = ALL_FIELDS) -> Dict[str, np.ndarray]:
        nx, ny, nz = (int(v) for v in self.cfg.n)
        out = {}
        ptrs = (C.POINTER(C.c_double) * 13)()
        mask = 0
        for nm in names:
            f = ALL_FIELDS.index(nm)
            shape = (nz + 1, ny + 1, nx + 1) if f < 6 else (nz, ny, nx)
            arr = np.empty(shape, dtype=np.float64)
            out[nm] = arr
            ptrs[f] = arr.ctypes.data_as(C.POINTER(C.c_double))
            mask |= 1 << f
        rc = lib().orc_get_fields(self._h, mask, ptrs)
        if rc != 0:
            raise OracleError(rc, "get_fields")
        return out

    def close(self):
        if getattr(self, "_h", None):
            lib().orc_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def zone_geometry(X: np.ndarray):
    """S2 geometry of one hex (orc_zone_geometry): X (8,3) -> (B (8,3), V, L)."""
    X = np.ascontiguousarray(X, dtype=np.float64).reshape(8, 3)
    B = np.zeros((8, 3))
    V = C.c_double()
    Lc = C.c_double()
    lib().orc_zone_geometry(X.ctypes.data, B.ctypes.data, C.byref(V), C.byref(Lc))
    return B, V.value, Lc.value


def zone_state(X, U, m, e, hh, gamma=1.4, q_lin=0.5, q_quad=2.0, cfl=0.3, c_vol=0.1) -> dict:
    """S2-S6 for one zone (orc_zone_state)."""
    X = np.ascontiguousarray(X, dtype=np.float64).reshape(8, 3)
    U = np.ascontiguousarray(U, dtype=np.float64).reshape(8, 3)
    out = np.zeros(8)
    lib().orc_zone_state(X.ctypes.data, U.ctypes.data, float(m), float(e), float(hh),
                         float(gamma), float(q_lin), float(q_quad), float(cfl), float(c_vol),
                         out.ctypes.data)
    return dict(zip(("rho", "ep", "p", "c", "q", "P", "dtz", "V"), out.tolist()))


def zone_hourglass(X, U, B, V, rho, c, kappa) -> np.ndarray:
    """f1 / reading R17: Flanagan-Belytschko hourglass corner forces of one zone (8, 3)."""
    X = np.ascontiguousarray(X, dtype=np.float64).reshape(8, 3)
    U = np.ascontiguousarray(U, dtype=np.float64).reshape(8, 3)
    B = np.ascontiguousarray(B, dtype=np.float64).reshape(8, 3)
    F = np.zeros((8, 3))
    lib().orc_zone_hourglass(X.ctypes.data, U.ctypes.data, B.ctypes.data, float(V), float(rho),
                             float(c), float(kappa), F.ctypes.data)
    return F


def zone_strain(X, U):
    """Reading R24: (eps (3,), L (3,)) of one zone (orc_zone_strain)."""
    X = np.ascontiguousarray(X, dtype=np.float64).reshape(8, 3)
    U = np.ascontiguousarray(U, dtype=np.float64).reshape(8, 3)
    eps, L = np.zeros(3), np.zeros(3)
    lib().orc_zone_strain(X.ctypes.data, U.ctypes.data, eps.ctypes.data, L.ctypes.data)
    return eps, L


def mono_limiter(em, e0, ep) -> float:
    """Reading R24: the monotonic limiter phi of one direction (orc_mono_limiter)."""
    return float(lib().orc_mono_limiter(float(em), float(e0), float(ep)))


def run(cfg: OracleConfig, ncycles: int, names: Sequence[str] = ALL_FIELDS):
    """Create, step ``ncycles`` and return (fields, info)."""
    o = Oracle(cfg)
    info = o.step(ncycles)
    f = o.fields(names)
    o.close()
    return f, info
