"""Multi-rank runs on the GPU: two processes (world size 2) sharing the pool's single B200.

NCCL refuses two ranks on one device, so these use the peer transport (HYDRO_FLAG_PEER): CUDA
IPC maps the neighbour rank's domain allocations and mailbox, the node/energy stage's boundary
layer is stored straight into the neighbour's ghost arrays, and dt / error bits are reduced
through the mailboxes.  Everything above the transport -- the domain->rank assignment, the
inter-rank halo plan, the per-rank domains, the collective get_fields -- is the same code the
NCCL path runs on a multi-GPU node.  Results are compared with the oracle (PAPER.md L548-557:
domains owned by different ranks exchange a halo).
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, kw, ncycles, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
        with Hydro(HydroConfig(rank=rank, nranks=world, device=0, transport="peer", **kw)) as h:
            info = h.step(ncycles)
            f = h.fields()
        q.put((rank, info, f if rank == 0 else None, None))
    except Exception as ex:  # report instead of hanging the other rank
        q.put((rank, None, None, repr(ex)))
    finally:
        dist.destroy_process_group()


def run_two_ranks(kw, ncycles, timeout=240):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, kw, ncycles, q)) for r in range(2)]
    for p in procs:
        p.start()
    try:
        out = [q.get(timeout=timeout) for _ in range(2)]
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    out.sort(key=lambda r: r[0])
    for r in out:
        assert r[3] is None, f"rank {r[0]}: {r[3]}"
    return out[0][1], out[1][1], out[0][2]


def _ocfg(kw):
    keys = ("n", "origin", "extent", "init", "user", "ndom", "cuts")  # halo: GPU-only option
    return OracleConfig(**{k: v for k, v in kw.items() if k in keys})


def test_two_ranks_sedov_slabs_match_oracle():
    kw = dict(n=(32, 32, 32), ndom=(1, 2, 1))  # one y-slab per rank (hierarchical split)
    i0, i1, f = run_two_ranks(kw, 60)
    fo, io = oracle.run(_ocfg(kw), 60)
    assert i0["status"] == 0 and i0["t"] == i1["t"] and i0["dt"] == i1["dt"]
    assert i0["dt"] == pytest.approx(io["dt"], rel=1e-10)
    for k in FIELDS:
        assert rel_err(f[k], fo[k]) <= 1e-10, k


@pytest.mark.parametrize("halo", ["fused", "kernel"])
def test_two_ranks_uneven_mixed_domains_match_oracle(halo):
    """12 uneven domains spread over two ranks so that every domain has both same-rank
    (intra-GPU) and other-rank (peer store) neighbours, incl. edge and corner slabs; the ghost
    slabs go out from the node/energy stage's epilogue (fused) or from the separate copy and
    peer-push kernels."""
    n = (24, 20, 18)
    cuts = [[0, 5, 13, 24], [0, 7, 20], [0, 9, 18]]
    d2r = [(d * 5 + d // 3) % 2 for d in range(12)]
    kw = dict(n=n, ndom=(3, 2, 2), cuts=cuts, dom_to_rank=d2r, init="user",
              user=jittered_state(n, 11), halo=halo)
    i0, i1, f = run_two_ranks(kw, 25)
    fo, io = oracle.run(_ocfg(kw), 25)
    assert i0["status"] == 0 and i0["dt"] == i1["dt"]
    for k in FIELDS:
        assert rel_err(f[k], fo[k]) <= 1e-10, k


def test_tangled_zone_on_one_rank_halts_both_at_the_same_cycle():
    """ADVICE r1 / SURVEY §8b: the error bits are reduced with dt every cycle, so a zone tangled
    in rank 1's domain halts rank 0 too, at the oracle's cycle with the oracle's status (the
    NCCL transport reduces them the same way: one allreduce over [~dt, error words])."""
    from tests.helpers import user_state
    n = (8, 8, 8)
    s = user_state(n, e=1.0)
    s["u"][3, 6, 3] = 1e4  # node (x=3, y=6, z=3): inside the upper y-slab (rank 1)
    kw = dict(n=n, ndom=(1, 2, 1), init="user", user=s, dt_first=1e-3)
    i0, i1, f = run_two_ranks(kw, 5)
    fo, io = oracle.run(OracleConfig(n=n, ndom=(1, 2, 1), init="user", user=s, dt_first=1e-3), 5)
    assert io["status"] == -5 and io["cycle"] == 1
    assert i0["status"] == i1["status"] == -5
    assert i0["cycle"] == i1["cycle"] == io["cycle"]
    assert i1["bad_zone"] == io["bad_zone"]  # the owning rank names the zone
    # both ranks keep the state after the failing cycle (same clock as the oracle); the fields
    # around a zone of negative volume are not comparable within a rounding tolerance (the
    # fast reciprocals and the oracle's division diverge on V <= 0), so only the far side is
    assert i0["t"] == i1["t"] == pytest.approx(io["t"], rel=1e-14)
    for k in ("x", "u", "e"):
        far = (slice(None), slice(0, 2), slice(None))  # y-planes 0-1: rank 0, far from the node
        assert rel_err(f[k][far], fo[k][far]) <= 1e-12, k


def test_dt_floor_halts_both_ranks_at_the_same_cycle():
    n = (16, 16, 16)
    s = jittered_state(n, 1)
    o = oracle.Oracle(OracleConfig(n=n, init="user", user=s, dt_floor=-1.0))
    seq = [o.step(1)["dt_min_zone"] for _ in range(12)]
    o.close()
    floor = 0.5 * (seq[9] + min(seq[:9]))
    kw = dict(n=n, ndom=(1, 2, 1), init="user", user=s, dt_floor=floor)
    i0, i1, f = run_two_ranks(kw, 100)
    assert i0["status"] == i1["status"] == -7
    assert i0["cycle"] == i1["cycle"] == 10
