"""World-size-2 gloo test (CPU) of Hydro.rebalance's migration choreography:
with the device calls stubbed out (pack = a host buffer tagged with the domain id, unpack
records what arrives), every rank must end up holding exactly the domains the plan gives it,
each with the bytes its previous owner packed, and the new context must be built with the new
map and the old clock.  The device side of pack/unpack is covered by tests/test_gpu_rebalance.py.
"""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icppw_pearce18_b200 import HydroConfig, dom_to_rank


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


N = (24, 20, 18)
CUTS = [[0, 5, 13, 24], [0, 7, 20], [0, 9, 18]]


def _cfg(rank, world, d2r):
    return HydroConfig(n=N, ndom=(3, 2, 2), cuts=CUTS, dom_to_rank=d2r, rank=rank,
                       nranks=world)


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icppw_pearce18_b200.hydro import Hydro
        h = Hydro.__new__(Hydro)
        h._group = None
        h.cfg = _cfg(rank, world, [d % 2 for d in range(12)])
        log = {"created": [], "unpacked": {}, "clock": None}

        def size(d):
            return 64 + 8 * d

        h.domain_bytes = size
        h.pack_domain = lambda d: torch.full((size(d),), d + 1, dtype=torch.uint8)
        h.unpack_domain = lambda d, t: log["unpacked"].__setitem__(d, t.clone())
        h.info = lambda: {"t": 0.25, "dt": 1e-3, "cycle": 40}
        h.close = lambda: None
        h._to_device = lambda t: t

        def create(cfg):
            h.cfg = cfg
            log["created"].append(list(cfg.dom_to_rank))

        h._create = create
        h.set_clock = lambda t, dt, c: log.__setitem__("clock", (t, dt, c))
        res = h.rebalance(busy=[1.0, 3.0])
        q.put((rank, res, log["created"], {d: (int(t.numel()), int(t[0]), bool((t == t[0]).all()))
                                           for d, t in log["unpacked"].items()}, log["clock"]))
    finally:
        dist.destroy_process_group()


def test_two_rank_migration_choreography_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = sorted([q.get(timeout=300) for _ in range(2)], key=lambda r: r[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    new_map = out[0][1]["map"]
    assert out[1][1]["map"] == new_map and out[0][1]["moved"] > 0
    cur = dom_to_rank(_cfg(0, 2, [d % 2 for d in range(12)]))
    assert sum(a != b for a, b in zip(cur, new_map)) == out[0][1]["moved"]
    for rank in (0, 1):
        _, res, created, unpacked, clock = out[rank]
        assert created == [new_map]              # one new context, built with the new map
        assert clock == (0.25, 1e-3, 40)        # the run clock carries over
        mine = {d for d in range(12) if new_map[d] == rank}
        assert set(unpacked) == mine              # exactly this rank's domains arrive ...
        for d, (n, tag, uniform) in unpacked.items():
            assert n == 64 + 8 * d and tag == d + 1 and uniform  # ... with their packed bytes
