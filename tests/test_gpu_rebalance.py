"""GPU tests of domain migration and measured rebalancing (PAPER.md
L597-603, L1077-1081: the decomposition "can be adjusted between iterations").

* pack/unpack: the complete state of every domain moved into a fresh context (same cuts), with
  the clock carried over, continues bitwise like the original run;
* two ranks sharing the pool's B200 (peer transport, as in test_gpu_multirank.py): a measured-
  weight plan that moves domains between the ranks mid-run, then the run continues; the result
  equals the same run without migration bitwise and the oracle within north_star's tolerance.
"""
import os

import numpy as np
import pytest
import torch.multiprocessing as mp

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err
from tests.test_gpu_multirank import _free_port

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")


@pytest.mark.parametrize("path", ["two", "split"])
def test_pack_unpack_continues_bitwise(path):
    n = (40, 36, 28)
    kw = dict(n=n, ndom=(2, 2, 1), cuts=[[0, 17, 40], [0, 20, 36], [0, 28]], init="user",
              user=jittered_state(n, 5), path=path)
    with Hydro(HydroConfig(**kw)) as a:
        a.step(15)
        info = a.info()
        bufs = {d: a.pack_domain(d) for d in range(4)}
        with Hydro(HydroConfig(**dict(kw, init="sedov", user=None))) as b:
            for d, t in bufs.items():
                b.unpack_domain(d, t)
            b.set_clock(info["t"], info["dt"], info["cycle"])
            ia = a.step(20)
            ib = b.step(20)
            fa, fb = a.fields(), b.fields()
    assert ia["cycle"] == ib["cycle"] == 35 and ia["t"] == ib["t"] and ia["dt"] == ib["dt"]
    for k in FIELDS:
        assert np.array_equal(fa[k], fb[k]), k


def _worker(rank, world, port, kw, pre, post, busy, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        with Hydro(HydroConfig(rank=rank, nranks=world, device=0, transport="peer", **kw)) as h:
            h.step(pre)
            res = h.rebalance(busy=busy) if busy is not None else None
            info = h.step(post)
            f = h.fields()
        q.put((rank, info, f if rank == 0 else None, res, None))
    except Exception as ex:  # report instead of hanging the other rank
        q.put((rank, None, None, None, repr(ex)))
    finally:
        dist.destroy_process_group()


def _two(kw, pre, post, busy, timeout=300):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, kw, pre, post, busy, q))
             for r in range(2)]
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
        assert r[4] is None, f"rank {r[0]}: {r[4]}"
    return out


def test_two_ranks_measured_rebalance_moves_domains_and_continues_exactly():
    n = (24, 20, 18)
    cuts = [[0, 5, 13, 24], [0, 7, 20], [0, 9, 18]]
    kw = dict(n=n, ndom=(3, 2, 2), cuts=cuts, dom_to_rank=[d % 2 for d in range(12)],
              init="user", user=jittered_state(n, 12))
    # rank 1 "measured" 3x slower than rank 0 per unit of work -> it gives domains away
    out = _two(kw, 10, 15, busy=[1.0, 3.0])
    res = out[0][3]
    assert res["moved"] > 0 and res == out[1][3]
    assert res["predicted"][1] < res["predicted"][0]
    ref = _two(kw, 10, 15, busy=None)  # same cuts, no migration
    f, fr = out[0][2], ref[0][2]
    assert out[0][1]["cycle"] == 25 and out[0][1]["t"] == ref[0][1]["t"]
    for k in FIELDS:
        assert np.array_equal(f[k], fr[k]), k
    fo, io = oracle.run(OracleConfig(n=n, ndom=(3, 2, 2), cuts=cuts, init="user",
                                     user=kw["user"]), 25)
    for k in FIELDS:
        assert rel_err(f[k], fo[k]) <= 1e-10, k
