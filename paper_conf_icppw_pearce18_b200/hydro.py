"""Thin Python binding of include/hydro.h (argument marshalling only).

Every step of the cycle runs in the CUDA kernels of ``libhydro_b200.so``; this module only
fills the C structs, owns host buffers and, for multi-process runs, uses ``torch.distributed``
to broadcast the communicator id and to combine the per-rank parts of ``fields()``.  There is
no CPU fallback: if the library or a CUDA device is missing, ``Hydro(...)`` raises.
"""
from __future__ import annotations

import ctypes as C
import math
import os
from dataclasses import dataclass
from typing import Dict, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# HYDRO_LIB: an alternative build of the same library (A/B measurements of kernel variants)
LIB_PATH = os.environ.get("HYDRO_LIB") or os.path.join(_HERE, "libhydro_b200.so")

NODE_FIELDS = ("x", "y", "z", "u", "v", "w")
ZONE_FIELDS = ("rho", "e", "p", "q", "c", "vol", "mass")
ALL_FIELDS = NODE_FIELDS + ZONE_FIELDS
ABI_VERSION = 4
FLAG_NO_GRAPH = 1 << 0
FLAG_SPLIT = 1 << 1
FLAG_ONE_KERNEL = 1 << 2
FLAG_PEER = 1 << 3
FLAG_HALO_FUSED = 1 << 4
FLAG_STRICT = 1 << 5
FLAG_COMM_SELF = 1 << 6

STATUS = {0: "ok", -1: "EINVAL", -2: "ENOMEM", -3: "ECUDA", -4: "ENCCL", -5: "ETANGLED",
          -6: "ENONFINITE", -7: "EDTMIN", -8: "ESTATE"}


class HydroConfigC(C.Structure):
    _fields_ = [
        ("abi_version", C.c_int32),
        ("n", C.c_int64 * 3),
        ("origin", C.c_double * 3),
        ("extent", C.c_double * 3),
        ("ndom", C.c_int32 * 3),
        ("cuts", C.POINTER(C.c_int64) * 3),
        ("dom_to_rank", C.POINTER(C.c_int32)),
        ("rank_weight", C.POINTER(C.c_double)),
        ("gamma", C.c_double), ("q_lin", C.c_double), ("q_quad", C.c_double),
        ("cfl", C.c_double), ("c_vol", C.c_double),
        ("dt_growth", C.c_double), ("dt_max", C.c_double), ("dt_init", C.c_double),
        ("t_stop", C.c_double), ("dt_first", C.c_double), ("t0", C.c_double),
        ("reflect_mask", C.c_uint32),
        ("init_kind", C.c_int32),
        ("rho0", C.c_double), ("e0", C.c_double), ("sedov_energy", C.c_double),
        ("user", C.POINTER(C.c_double) * 8),
        ("rank", C.c_int32), ("nranks", C.c_int32), ("device", C.c_int32),
        ("comm_id", C.c_void_p),
        ("flags", C.c_uint64),
        ("hg_coef", C.c_double),
        ("dt_floor", C.c_double),
        ("q_kind", C.c_int32),
    ]


class HydroInfoC(C.Structure):
    _fields_ = [("t", C.c_double), ("dt", C.c_double), ("cycle", C.c_int64),
                ("dt_min_zone", C.c_double), ("status", C.c_int32), ("bad_zone", C.c_int64)]


_lib = None


def load_library(path: str = LIB_PATH) -> C.CDLL:
    """Load the CUDA library; raises (loudly) if it has not been built."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError(f"{path} missing: run __graft_entry__.build() (no CPU fallback exists)")
    L = C.CDLL(path)
    L.hydro_config_default.argtypes = [C.POINTER(HydroConfigC)]
    L.hydro_config_default.restype = None
    L.hydro_create.argtypes = [C.POINTER(HydroConfigC), C.POINTER(C.c_void_p)]
    L.hydro_step.argtypes = [C.c_void_p, C.c_int32, C.c_void_p, C.POINTER(HydroInfoC)]
    L.hydro_get_fields.argtypes = [C.c_void_p, C.c_uint32, C.POINTER(C.POINTER(C.c_double))]
    L.hydro_get_box.argtypes = [C.c_void_p, C.POINTER(C.c_int64), C.POINTER(C.c_int64),
                                C.c_uint32, C.POINTER(C.POINTER(C.c_double))]
    L.hydro_set_state.argtypes = [C.c_void_p, C.POINTER(C.POINTER(C.c_double)),
                                  C.POINTER(C.c_double), C.c_double, C.c_double]
    L.hydro_get_info.argtypes = [C.c_void_p, C.POINTER(HydroInfoC)]
    L.hydro_run_batch.argtypes = [C.c_void_p, C.c_int32, C.c_int32,
                                  C.POINTER(C.POINTER(C.c_double)),
                                  C.POINTER(C.POINTER(C.c_double)), C.POINTER(C.c_double),
                                  C.POINTER(C.c_double), C.POINTER(HydroInfoC)]
    L.hydro_destroy.argtypes = [C.c_void_p]
    L.hydro_layout_export.argtypes = [C.POINTER(HydroConfigC), C.POINTER(C.c_int64),
                                      C.POINTER(C.c_size_t)]
    L.hydro_decompose_hierarchical.argtypes = [C.POINTER(C.c_int64), C.c_int32, C.c_int32,
                                               C.POINTER(C.c_int32),
                                               C.POINTER(C.POINTER(C.c_int64)),
                                               C.POINTER(C.c_int32)]
    L.hydro_comm_plan_export.argtypes = [C.POINTER(HydroConfigC), C.POINTER(C.c_int64),
                                         C.POINTER(C.c_size_t)]
    L.hydro_weighted_slabs.argtypes = [C.c_int64, C.c_int32, C.POINTER(C.c_double),
                                       C.POINTER(C.c_int64)]
    L.hydro_rebalance_plan.argtypes = [C.POINTER(HydroConfigC), C.POINTER(C.c_double), C.c_double,
                                       C.c_double, C.POINTER(C.c_int32), C.POINTER(C.c_double),
                                       C.POINTER(C.c_double)]
    L.hydro_domain_bytes.argtypes = [C.c_void_p, C.c_int32, C.POINTER(C.c_size_t)]
    L.hydro_domain_pack.argtypes = [C.c_void_p, C.c_int32, C.c_void_p, C.c_size_t, C.c_void_p]
    L.hydro_domain_unpack.argtypes = [C.c_void_p, C.c_int32, C.c_void_p, C.c_size_t, C.c_void_p]
    L.hydro_set_clock.argtypes = [C.c_void_p, C.c_double, C.c_double, C.c_int64]
    L.hydro_comm_unique_id.argtypes = [C.c_void_p]
    L.hydro_peer_export.argtypes = [C.c_void_p, C.c_void_p, C.POINTER(C.c_size_t)]
    L.hydro_peer_import.argtypes = [C.c_void_p, C.c_void_p, C.c_size_t]
    L.hydro_peer_detach.argtypes = [C.c_void_p]
    L.hydro_time_kernels.argtypes = [C.c_void_p, C.c_int32, C.POINTER(C.c_double)]
    L.hydro_kernels_per_cycle.argtypes = [C.c_void_p]
    L.hydro_strerror.restype = C.c_char_p
    L.hydro_last_error.argtypes = [C.c_void_p]
    L.hydro_last_error.restype = C.c_char_p
    if L.hydro_abi_version() != ABI_VERSION:
        raise RuntimeError("libhydro_b200 ABI version mismatch")
    _lib = L
    return L


@dataclass
class HydroConfig:
    """Mirror of hydro_config (include/hydro.h); defaults = hydro_config_default()."""
    n: Sequence[int] = (32, 32, 32)
    origin: Sequence[float] = (0.0, 0.0, 0.0)
    extent: Sequence[float] = (1.2, 1.2, 1.2)
    ndom: Sequence[int] = (1, 1, 1)
    cuts: Optional[Sequence[Sequence[int]]] = None
    dom_to_rank: Optional[Sequence[int]] = None
    rank_weight: Optional[Sequence[float]] = None
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
    init: str = "sedov"          # "sedov" | "user" | "user_mass"
    rho0: float = 1.0
    e0: float = 0.0
    sedov_energy: float = 0.851072 / 8.0
    user: Optional[Dict[str, np.ndarray]] = None
    rank: int = 0
    nranks: int = 1
    device: int = 0
    path: str = "two"             # "two" (zone + node/energy kernels), "one" (one fused kernel),
                                  # "split" (plain 3-kernel pipeline, HYDRO_FLAG_SPLIT),
                                  # "strict" (the split pipeline in the oracle's canonical
                                  # operation order without FMA: bitwise, HYDRO_FLAG_STRICT)
    graph: bool = True            # CUDA graphs (HYDRO_FLAG_NO_GRAPH when False)
    transport: str = "nccl"       # nranks > 1: "nccl" (NCCL send/recv + allreduce) or "peer"
                                  # (CUDA IPC peer stores + mailbox reduction; ranks may share a GPU)
    halo: str = "kernel"          # default path: "kernel" (separate copy / peer-push kernels after
                                  # the node/energy stage) or "fused" (the stage stores the ghost
                                  # slabs from its own epilogue, HYDRO_FLAG_HALO_FUSED)
    hg_coef: float = 0.0          # viscous hourglass kappa (reading R17); > 0 runs
                                  # the split kernels
    dt_floor: float = 0.0         # dt-collapse floor (reading R23): > 0 absolute, 0 = 1e-6 dt^0,
                                  # < 0 none; below it a run halts with EDTMIN
    q: str = "scalar"             # artificial viscosity: "scalar" (reading R7) or "monotone"
                                  # (reading R24; single rank, split kernels)
    comm_self: bool = False       # nranks == 1: create a one-rank NCCL communicator anyway
                                  # (HYDRO_FLAG_COMM_SELF; exercises the NCCL path on one GPU)


class HydroError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"hydro error {code} ({STATUS.get(code, '?')}): {msg}")
        self.code = code


def _cfg_struct(cfg: HydroConfig, keep: list, comm_id: Optional[bytes] = None) -> HydroConfigC:
    L = load_library()
    c = HydroConfigC()
    L.hydro_config_default(C.byref(c))
    for a in range(3):
        c.n[a] = int(cfg.n[a])
        c.origin[a] = float(cfg.origin[a])
        c.extent[a] = float(cfg.extent[a])
        c.ndom[a] = int(cfg.ndom[a])
        if cfg.cuts is not None and cfg.cuts[a] is not None:
            arr = np.ascontiguousarray(cfg.cuts[a], dtype=np.int64)
            keep.append(arr)
            c.cuts[a] = arr.ctypes.data_as(C.POINTER(C.c_int64))
    if cfg.dom_to_rank is not None:
        arr = np.ascontiguousarray(cfg.dom_to_rank, dtype=np.int32)
        keep.append(arr)
        c.dom_to_rank = arr.ctypes.data_as(C.POINTER(C.c_int32))
    if cfg.rank_weight is not None:
        arr = np.ascontiguousarray(cfg.rank_weight, dtype=np.float64)
        keep.append(arr)
        c.rank_weight = arr.ctypes.data_as(C.POINTER(C.c_double))
    for k in ("gamma", "q_lin", "q_quad", "cfl", "c_vol", "dt_growth", "dt_max", "dt_init",
              "t_stop", "dt_first", "t0", "rho0", "e0", "sedov_energy", "hg_coef", "dt_floor"):
        setattr(c, k, float(getattr(cfg, k)))
    c.reflect_mask = int(cfg.reflect_mask)
    c.init_kind = {"sedov": 0, "user": 1, "user_mass": 2}[cfg.init]
    c.q_kind = {"scalar": 0, "monotone": 1}[cfg.q]
    if cfg.init != "sedov":
        names = ("x", "y", "z", "u", "v", "w", "rho" if cfg.init == "user" else "mass", "e")
        for f, nm in enumerate(names):
            arr = np.ascontiguousarray(cfg.user[nm], dtype=np.float64).ravel()
            keep.append(arr)
            c.user[f] = arr.ctypes.data_as(C.POINTER(C.c_double))
    c.rank, c.nranks, c.device = int(cfg.rank), int(cfg.nranks), int(cfg.device)
    if comm_id is not None:
        buf = C.create_string_buffer(comm_id, 128)
        keep.append(buf)
        c.comm_id = C.cast(buf, C.c_void_p)
    c.flags = ((0 if cfg.graph else FLAG_NO_GRAPH) | (FLAG_SPLIT if cfg.path == "split" else 0)
               | (FLAG_ONE_KERNEL if cfg.path == "one" else 0)
               | (FLAG_STRICT if cfg.path == "strict" else 0)
               | (FLAG_COMM_SELF if cfg.comm_self else 0)
               | (FLAG_PEER if cfg.transport == "peer" else 0)
               | (FLAG_HALO_FUSED if cfg.halo == "fused" else 0))
    return c


def layout_export(cfg: HydroConfig) -> np.ndarray:
    """hydro_layout_export: the integer layout (host-only; no GPU needed)."""
    L = load_library()
    keep: list = []
    c = _cfg_struct(cfg, keep)
    n = C.c_size_t(0)
    L.hydro_layout_export(C.byref(c), None, C.byref(n))
    buf = np.zeros(n.value, dtype=np.int64)
    rc = L.hydro_layout_export(C.byref(c), buf.ctypes.data_as(C.POINTER(C.c_int64)), C.byref(n))
    if rc != 0:
        raise HydroError(rc, L.hydro_last_error(None).decode())
    return buf


def comm_plan_export(cfg: HydroConfig):
    """hydro_comm_plan_export -> (sends, recvs), lists of (pair, peer, count, dst, src, dir)."""
    L = load_library()
    keep: list = []
    c = _cfg_struct(cfg, keep)
    n = C.c_size_t(0)
    L.hydro_comm_plan_export(C.byref(c), None, C.byref(n))
    buf = np.zeros(max(n.value, 2), dtype=np.int64)
    rc = L.hydro_comm_plan_export(C.byref(c), buf.ctypes.data_as(C.POINTER(C.c_int64)),
                                  C.byref(n))
    if rc != 0:
        raise HydroError(rc, "comm_plan_export")
    ns, nr = int(buf[0]), int(buf[1])
    ent = buf[2:].reshape(-1, 6).tolist() if ns + nr else []
    return [tuple(e) for e in ent[:ns]], [tuple(e) for e in ent[ns:ns + nr]]


def decompose_hierarchical(n: Sequence[int], ngpu: int, dpg: int):
    """hydro_decompose_hierarchical -> (ndom, cuts, dom_to_rank)."""
    L = load_library()
    nn = (C.c_int64 * 3)(*[int(v) for v in n])
    nd = (C.c_int32 * 3)()
    cuts = [np.zeros(int(v) + 1, dtype=np.int64) for v in n]
    cptr = (C.POINTER(C.c_int64) * 3)(*[a.ctypes.data_as(C.POINTER(C.c_int64)) for a in cuts])
    d2r = np.zeros(ngpu * dpg, dtype=np.int32)
    rc = L.hydro_decompose_hierarchical(nn, int(ngpu), int(dpg), nd, cptr,
                                        d2r.ctypes.data_as(C.POINTER(C.c_int32)))
    if rc != 0:
        raise HydroError(rc, "decompose_hierarchical")
    ndom = tuple(int(v) for v in nd)
    return ndom, [cuts[a][: ndom[a] + 1].tolist() for a in range(3)], d2r.tolist()


def weighted_slabs(nplanes: int, weights: Sequence[float]):
    L = load_library()
    w = np.ascontiguousarray(weights, dtype=np.float64)
    out = np.zeros(len(w), dtype=np.int64)
    rc = L.hydro_weighted_slabs(int(nplanes), len(w), w.ctypes.data_as(C.POINTER(C.c_double)),
                                out.ctypes.data_as(C.POINTER(C.c_int64)))
    if rc != 0:
        raise HydroError(rc, "weighted_slabs")
    return out.tolist()


def rebalance_plan(cfg: HydroConfig, busy: Sequence[float], beta: float = 0.0,
                   min_gain: float = 0.02):
    """hydro_rebalance_plan (host-only): (new dom_to_rank, rank speeds, (before, after))."""
    L = load_library()
    keep: list = []
    c = _cfg_struct(cfg, keep)
    nd = int(cfg.ndom[0]) * int(cfg.ndom[1]) * int(cfg.ndom[2])
    b = np.ascontiguousarray(busy, dtype=np.float64)
    if b.size != cfg.nranks:
        raise ValueError("busy needs one entry per rank")
    new_map = np.zeros(nd, dtype=np.int32)
    w = np.zeros(cfg.nranks, dtype=np.float64)
    pred = np.zeros(2, dtype=np.float64)
    rc = L.hydro_rebalance_plan(C.byref(c), b.ctypes.data_as(C.POINTER(C.c_double)),
                                float(beta), float(min_gain),
                                new_map.ctypes.data_as(C.POINTER(C.c_int32)),
                                w.ctypes.data_as(C.POINTER(C.c_double)),
                                pred.ctypes.data_as(C.POINTER(C.c_double)))
    if rc != 0:
        raise HydroError(rc, "rebalance_plan")
    return new_map.tolist(), w.tolist(), (float(pred[0]), float(pred[1]))


def dom_to_rank(cfg: HydroConfig):
    """The domain -> rank map cfg resolves to (explicit map or the weighted LPT rule)."""
    lay = layout_export(cfg).tolist()
    return [int(lay[7 + 7 * d + 6]) for d in range(int(lay[1]))]


def _info(i: HydroInfoC) -> dict:
    return {"t": i.t, "dt": i.dt, "cycle": i.cycle, "dt_min_zone": i.dt_min_zone,
            "status": i.status, "bad_zone": i.bad_zone}


class Hydro:
    """One hydro run on this process's GPU (collective over ranks when nranks > 1)."""

    def __init__(self, cfg: HydroConfig, group=None):
        self._L = load_library()
        self._group = group
        self._create(cfg)

    def _create(self, cfg: HydroConfig):
        self.cfg = cfg
        comm_id = None
        if cfg.nranks > 1 and cfg.transport == "nccl":
            comm_id = self._bootstrap_comm_id()
        elif cfg.comm_self:  # one-rank NCCL world (testing the NCCL path on one GPU)
            raw = C.create_string_buffer(128)
            rc = self._L.hydro_comm_unique_id(raw)
            if rc != 0:
                raise HydroError(rc, "hydro_comm_unique_id")
            comm_id = raw.raw
        keep: list = []
        c = _cfg_struct(cfg, keep, comm_id)
        h = C.c_void_p()
        rc = self._L.hydro_create(C.byref(c), C.byref(h))
        if rc != 0:
            raise HydroError(rc, self._L.hydro_last_error(None).decode())
        self._h = h
        if cfg.nranks > 1 and cfg.transport == "peer":
            self._bootstrap_peers()

    def _bootstrap_peers(self):
        """HYDRO_FLAG_PEER: all-gather every rank's IPC handles, then hydro_peer_import."""
        import torch.distributed as dist
        n = C.c_size_t(0)
        self._L.hydro_peer_export(self._h, None, C.byref(n))
        buf = C.create_string_buffer(n.value)
        rc = self._L.hydro_peer_export(self._h, buf, C.byref(n))
        if rc != 0:
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())
        recs = [None] * self.cfg.nranks
        dist.all_gather_object(recs, bytes(buf.raw), group=self._group)
        width = max(len(r) for r in recs)
        allb = b"".join(r.ljust(width, b"\0") for r in recs)
        rc = self._L.hydro_peer_import(self._h, allb, width)
        if rc != 0:
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())

    def _bootstrap_comm_id(self) -> bytes:
        import torch
        import torch.distributed as dist
        buf = bytearray(128)
        if self.cfg.rank == 0:
            raw = C.create_string_buffer(128)
            rc = self._L.hydro_comm_unique_id(raw)
            if rc != 0:
                raise HydroError(rc, "hydro_comm_unique_id")
            buf = bytearray(raw.raw)
        t = torch.tensor(list(buf), dtype=torch.uint8)
        if dist.get_backend(self._group) == "nccl":
            t = t.cuda()
        dist.broadcast(t, 0, group=self._group)
        return bytes(t.cpu().tolist())

    def step(self, ncycles: int, stream: Optional[int] = None) -> dict:
        info = HydroInfoC()
        rc = self._L.hydro_step(self._h, int(ncycles), C.c_void_p(stream) if stream else None,
                                C.byref(info))
        d = _info(info)
        d["rc"] = rc
        if rc in (-3, -4, -1):
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())
        return d

    def time_kernels(self, ncycles: int) -> dict:
        """hydro_time_kernels: per-kernel-class mean device ms (no graphs, CUDA events)."""
        out = (C.c_double * 6)()
        rc = self._L.hydro_time_kernels(self._h, int(ncycles), out)
        if rc in (-3, -4, -1, -8):
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())
        return {"cycle_kernel_ms": out[0], "halo_ms": out[1], "finalize_ms": out[2],
                "cycle_ms": out[3], "zone_stage_ms": out[4], "node_stage_ms": out[5]}

    def kernels_per_cycle(self) -> int:
        return int(self._L.hydro_kernels_per_cycle(self._h))

    def info(self) -> dict:
        info = HydroInfoC()
        self._L.hydro_get_info(self._h, C.byref(info))
        return _info(info)

    def _arrays(self, names, node_shape, zone_shape, alloc=np.zeros, given=None):
        out = {}
        ptrs = (C.POINTER(C.c_double) * 13)()
        mask = 0
        for nm in names:
            f = ALL_FIELDS.index(nm)
            shape = node_shape if f < 6 else zone_shape
            if given is not None and nm in given:
                arr = given[nm]
                if arr.shape != shape or arr.dtype != np.float64 or not arr.flags.c_contiguous:
                    raise ValueError(f"out[{nm!r}] must be a C-contiguous float64 array {shape}")
            else:
                arr = alloc(shape, dtype=np.float64)
            out[nm] = arr
            ptrs[f] = arr.ctypes.data_as(C.POINTER(C.c_double))
            mask |= 1 << f
        return out, ptrs, mask

    def fields(self, names: Sequence[str] = ALL_FIELDS,
               out: Optional[Dict[str, np.ndarray]] = None) -> Dict[str, np.ndarray]:
        """Global fields; ``out`` may supply caller-owned (e.g. pinned) arrays to fill.  With
        nranks > 1 a collective that assembles them on rank 0 (``_combine``)."""
        nx, ny, nz = (int(v) for v in self.cfg.n)
        out, ptrs, mask = self._arrays(names, (nz + 1, ny + 1, nx + 1), (nz, ny, nx), given=out)
        rc = self._L.hydro_get_fields(self._h, mask, ptrs)
        if rc != 0:
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())
        if self.cfg.nranks > 1:
            out = self._combine(out)
        return out

    def box(self, lo: Sequence[int], hi: Sequence[int], names: Sequence[str] = ALL_FIELDS):
        """Fields of the global zone box [lo, hi) (nodes [lo, hi])."""
        ext = [int(hi[a]) - int(lo[a]) for a in range(3)]
        out, ptrs, mask = self._arrays(names, (ext[2] + 1, ext[1] + 1, ext[0] + 1),
                                       (ext[2], ext[1], ext[0]))
        clo = (C.c_int64 * 3)(*[int(v) for v in lo])
        chi = (C.c_int64 * 3)(*[int(v) for v in hi])
        rc = self._L.hydro_get_box(self._h, clo, chi, mask, ptrs)
        if rc != 0:
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())
        if self.cfg.nranks > 1:
            out = self._combine(out)
        return out

    def _combine(self, out):
        """nranks > 1: every global entry is written by exactly one rank (the rest are zero), so a
        sum to rank 0 assembles the global arrays there (collective; rank 0 returns them, the
        other ranks return their own partial arrays).  Rank-local data without any global
        array: pack_domain / hydro_get_box of the owned domains."""
        import torch
        import torch.distributed as dist
        res = {}
        for k, v in out.items():
            t = torch.from_numpy(v)
            if dist.get_backend(self._group) == "nccl":
                t = t.cuda()
            dist.reduce(t, dst=0, group=self._group)
            res[k] = t.cpu().numpy() if self.cfg.rank == 0 else v
        return res

    # ------------------------------------------------------------ domain migration (f2)
    def domain_bytes(self, dom: int) -> int:
        n = C.c_size_t(0)
        rc = self._L.hydro_domain_bytes(self._h, int(dom), C.byref(n))
        if rc != 0:
            raise HydroError(rc, "domain_bytes")
        return int(n.value)

    def pack_domain(self, dom: int, out=None):
        """hydro_domain_pack into ``out`` (a uint8 tensor on the device or in page-locked host
        memory) or a new CUDA uint8 tensor (this rank must own ``dom``)."""
        import torch
        buf = out if out is not None else torch.empty(
            self.domain_bytes(dom), dtype=torch.uint8, device=f"cuda:{self.cfg.device}")
        rc = self._L.hydro_domain_pack(self._h, int(dom), C.c_void_p(buf.data_ptr()), buf.numel(),
                                       None)
        if rc != 0:
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())
        return buf

    def unpack_domain(self, dom: int, buf):
        rc = self._L.hydro_domain_unpack(self._h, int(dom), C.c_void_p(buf.data_ptr()),
                                         buf.numel(), None)
        if rc != 0:
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())

    def _to_device(self, t):
        return t.to(f"cuda:{self.cfg.device}")

    def set_clock(self, t: float, dt: float, cycle: int):
        rc = self._L.hydro_set_clock(self._h, float(t), float(dt), int(cycle))
        if rc != 0:
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())

    def rebalance(self, busy: Optional[Sequence[float]] = None, beta: float = 0.0,
                  min_gain: float = 0.02, measure_cycles: int = 5) -> dict:
        """Measured-weight rebalancing between iterations (PAPER.md L597-603,
        L1077-1081).  Collective.  busy: per-rank device ms per cycle under the current map;
        None = measure it here with hydro_time_kernels over ``measure_cycles`` cycles (real
        cycles: the run advances) and all-gather it.  The plan is hydro_rebalance_plan; domains
        whose owner changes are packed on the old owner, sent with torch.distributed (device
        tensors over NCCL, host copies over gloo) and unpacked into a new context built with the
        new map; the clock carries over, so the run continues exactly."""
        import dataclasses
        import torch
        import torch.distributed as dist
        cfg = self.cfg
        cur = dom_to_rank(cfg)
        if busy is None:
            own = self.time_kernels(measure_cycles)["cycle_kernel_ms"]
            if cfg.nranks > 1:
                allb = [None] * cfg.nranks
                dist.all_gather_object(allb, own, group=self._group)
                busy = allb
            else:
                busy = [own]
        cur_cfg = dataclasses.replace(cfg, dom_to_rank=cur, rank_weight=None)
        new_map, weights, pred = rebalance_plan(cur_cfg, busy, beta, min_gain)
        res = {"map": new_map, "weights": weights, "predicted": pred, "busy": list(busy),
               "moved": sum(int(a != b) for a, b in zip(cur, new_map))}
        if res["moved"] == 0:
            return res
        info = self.info()
        rank = cfg.rank
        bufs = {d: self.pack_domain(d) for d in range(len(cur)) if cur[d] == rank}
        if cfg.nranks > 1:
            host = dist.get_backend(self._group) != "nccl"
            ops, recvd = [], {}
            for d in range(len(cur)):
                a, b = cur[d], new_map[d]
                if a == b:
                    continue
                if a == rank:
                    t = bufs[d].cpu() if host else bufs[d]
                    ops.append(dist.P2POp(dist.isend, t, b, group=self._group))
                if b == rank:
                    n = self.domain_bytes(d)
                    t = torch.empty(n, dtype=torch.uint8,
                                    device="cpu" if host else f"cuda:{cfg.device}")
                    recvd[d] = t
                    ops.append(dist.P2POp(dist.irecv, t, a, group=self._group))
            if ops:
                for r in dist.batch_isend_irecv(ops):
                    r.wait()
            for d, t in recvd.items():
                bufs[d] = self._to_device(t)
        self.close()
        self._create(dataclasses.replace(cfg, dom_to_rank=new_map, rank_weight=None))
        for d in range(len(new_map)):
            if new_map[d] == rank:
                self.unpack_domain(d, bufs[d])
        del bufs
        self.set_clock(info["t"], info["dt"], info["cycle"])
        return res

    def set_state(self, nodes: Dict[str, np.ndarray], e: np.ndarray, t: float, dt: float):
        arrs = [np.ascontiguousarray(nodes[k], dtype=np.float64) for k in NODE_FIELDS]
        ea = np.ascontiguousarray(e, dtype=np.float64)
        ptrs = (C.POINTER(C.c_double) * 6)(*[a.ctypes.data_as(C.POINTER(C.c_double)) for a in arrs])
        rc = self._L.hydro_set_state(self._h, ptrs, ea.ctypes.data_as(C.POINTER(C.c_double)),
                                     float(t), float(dt))
        if rc != 0:
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())

    def run_batch(self, states: Sequence[Dict[str, np.ndarray]], ncycles: int,
                  t0: Sequence[float], dt0: Sequence[float],
                  out: Optional[Sequence[Dict[str, np.ndarray]]] = None):
        """hydro_run_batch: independent runs from the host states ``states[b]`` (x, y, z, u, v,
        w on nodes and e on zones, global arrays), ncycles each, with the host<->device copies
        of neighbouring batches overlapped with the cycles (pin the arrays for the overlap).
        Returns (outputs, infos); ``out`` may supply caller-owned (pinned) result arrays."""
        nb = len(states)
        nx, ny, nz = (int(v) for v in self.cfg.n)
        names = NODE_FIELDS + ("e",)
        ins = [[np.ascontiguousarray(st[k], dtype=np.float64) for k in names] for st in states]
        if out is None:
            out = [{k: np.empty((nz + 1, ny + 1, nx + 1) if k != "e" else (nz, ny, nx))
                    for k in names} for _ in range(nb)]
        P = C.POINTER(C.c_double)
        for b in range(nb):
            for k in names:
                a = out[b][k]
                if a.dtype != np.float64 or not a.flags.c_contiguous:
                    raise ValueError("run_batch: out arrays must be C-contiguous float64")
        pin = (P * (7 * nb))(*[a.ctypes.data_as(P) for row in ins for a in row])
        pout = (P * (7 * nb))(*[out[b][k].ctypes.data_as(P) for b in range(nb) for k in names])
        ct0 = (C.c_double * nb)(*[float(v) for v in t0])
        cdt0 = (C.c_double * nb)(*[float(v) for v in dt0])
        infos = (HydroInfoC * max(nb, 1))()
        rc = self._L.hydro_run_batch(self._h, nb, int(ncycles), pin, pout, ct0, cdt0, infos)
        if rc in (-3, -1):
            raise HydroError(rc, self._L.hydro_last_error(self._h).decode())
        return out, [_info(infos[b]) for b in range(nb)]

    def close(self):
        """Destroy the context (collective).  Peer transport: detach from the other ranks'
        memory, barrier, then free (hydro_peer_detach; freeing memory another process still
        maps is undefined in CUDA)."""
        if getattr(self, "_h", None):
            if self.cfg.nranks > 1 and self.cfg.transport == "peer":
                import torch.distributed as dist
                self._L.hydro_peer_detach(self._h)
                if dist.is_available() and dist.is_initialized():
                    dist.barrier(group=self._group)
            self._L.hydro_destroy(self._h)
            self._h = None

    def __del__(self):
        # garbage collection is not collective: free without the cross-rank barrier
        try:
            if getattr(self, "_h", None):
                self._L.hydro_destroy(self._h)
                self._h = None
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
