"""Multi-process (world size 2, gloo, CPU) tests of the N>1 host logic.

The GPU transport (NCCL grouped send/recv of the ghost slabs, allreduce-min of dt) cannot run on
the single-GPU pool; what makes it correct by construction is host logic tested here: every rank
derives the same layout, the send list of rank a to rank b equals the receive list of rank b
from rank a in the same order and with the same sizes (the grouped ncclSend/ncclRecv pairing
rule), the inter-rank slabs cover exactly the halo pairs whose ends live on different ranks, and
the communicator id bootstrap broadcast reaches every rank intact.  PAPER.md L548-557 (halo
exchange between domains owned by different ranks).
"""
import os
import socket

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icppw_pearce18_b200 import HydroConfig, comm_plan_export, layout_export

CUTS = [0, 64, 160, 288, 448]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _cfgs(rank, nranks):
    yield HydroConfig(n=(448,) * 3, ndom=(4, 4, 4), cuts=[CUTS] * 3, nranks=nranks, rank=rank)
    yield HydroConfig(n=(40, 30, 20), ndom=(2, 3, 2), nranks=nranks, rank=rank,
                      dom_to_rank=[(d * 7) % nranks for d in range(12)])
    yield HydroConfig(n=(64, 64, 64), ndom=(1, 4, 1), nranks=nranks, rank=rank,
                      rank_weight=[1.0 + 2.0 * (r % 2) for r in range(nranks)])


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        results = []
        for cfg in _cfgs(rank, world):
            lay = layout_export(cfg).tolist()
            plan = comm_plan_export(cfg)
            everyone = [None] * world
            dist.all_gather_object(everyone, (lay, plan))
            results.append(everyone)
        # communicator-id bootstrap: rank 0's 128 bytes reach every rank unchanged
        from paper_conf_icppw_pearce18_b200.hydro import Hydro
        h = Hydro.__new__(Hydro)
        h.cfg = HydroConfig(rank=rank, nranks=world)
        from paper_conf_icppw_pearce18_b200 import load_library
        h._L = load_library()
        h._group = None
        cid = h._bootstrap_comm_id()
        ids = [None] * world
        dist.all_gather_object(ids, cid)
        q.put((rank, results, ids))
    finally:
        dist.destroy_process_group()


def _check(everyone):
    lays = [e[0] for e in everyone]
    assert all(l == lays[0] for l in lays), "ranks disagree on the layout"
    lay = lays[0]
    nd, nr, npairs = lay[1], lay[2], lay[3]
    dom_rank = [lay[7 + 7 * d + 6] for d in range(nd)]
    base = 7 + 7 * nd
    pairs = [lay[base + 15 * i: base + 15 * (i + 1)] for i in range(npairs)]
    cross = {i for i, p in enumerate(pairs) if dom_rank[p[0]] != dom_rank[p[1]]}
    sent, recvd = set(), set()
    for a in range(nr):
        sends_a, recvs_a = everyone[a][1]
        for e in sends_a:
            assert dom_rank[e[4]] == a and e[1] == dom_rank[e[3]]
            sent.add(e[0])
        for e in recvs_a:
            assert dom_rank[e[3]] == a and e[1] == dom_rank[e[4]]
            recvd.add(e[0])
        for b in range(nr):
            if a == b:
                continue
            a_to_b = [(e[0], e[2]) for e in sends_a if e[1] == b]
            b_from_a = [(e[0], e[2]) for e in everyone[b][1][1] if e[1] == a]
            assert a_to_b == b_from_a, f"send/recv order mismatch {a}->{b}"
    assert sent == cross and recvd == cross
    # message size = 6 node fields over the node slab + e over the zone slab
    for a in range(nr):
        for e in everyone[a][1][0]:
            p = pairs[e[0]]
            nn = (p[6] - p[3]) * (p[7] - p[4]) * (p[8] - p[5])
            nz = (p[12] - p[9]) * (p[13] - p[10]) * (p[14] - p[11])
            assert e[2] == 6 * nn + nz


def test_two_rank_plans_match_under_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    out.sort()
    results = out[0][1]
    for everyone in results:
        _check(everyone)
    ids = out[0][2]
    assert len(ids[0]) == 128 and ids[0] == ids[1]


@pytest.mark.parametrize("nranks", [2, 4, 8])
def test_plans_consistent_single_process(nranks):
    """Same property for more ranks, gathering the plans in one process."""
    for cfgs in zip(*[_cfgs(r, nranks) for r in range(nranks)]):
        everyone = [(layout_export(c).tolist(), comm_plan_export(c)) for c in cfgs]
        _check(everyone)
