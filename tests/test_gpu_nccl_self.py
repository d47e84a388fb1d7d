"""The NCCL transport's device-side plumbing on the pool's single B200: a one-rank NCCL world
(HYDRO_FLAG_COMM_SELF).  Every cycle then moves the ghost slabs between the rank's domains by
the NCCL halo leg (pack kernel, grouped ncclSend/ncclRecv to itself in plan order, unpack
kernel) instead of the copy kernel, and runs the NCCL dt / error allreduce (pack, allreduce over
[~dt, error words], unpack) on its own communicator (ncclCommSplit) and stream, forked after the
zone stage and joined before S9 (two-kernel path) or in line (other paths), all captured in the
CUDA graphs; hydro_step waits while polling ncclCommGetAsyncError.  The slabs are bit copies
and the one-rank reduction is the identity, so every field, t and dt must equal the
communicator-free run bit for bit, including a run that halts with EDTMIN.  (NCCL refuses two
ranks on one GPU; the cross-rank plan matching is covered by the gloo tests and bench.py's
nccl_check at N > 1.)"""
import numpy as np
import pytest

from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")


def _run(nc, **kw):
    with Hydro(HydroConfig(**kw)) as h:
        info = h.step(nc)
        f = h.fields()
        info["kernels"] = h.kernels_per_cycle()
    return f, info


@pytest.mark.parametrize("path", ["two", "one", "split"])
@pytest.mark.parametrize("overlap", ["1", "0"])
def test_one_rank_nccl_equals_no_comm_bitwise(path, overlap, monkeypatch):
    monkeypatch.setenv("HYDRO_DT_OVERLAP", overlap)
    n = (24, 20, 18)
    kw = dict(n=n, ndom=(2, 2, 1), init="user", user=jittered_state(n, 5), path=path)
    fa, ia = _run(30, comm_self=True, **kw)
    fb, ib = _run(30, **kw)
    assert ia["status"] == ib["status"] == 0
    assert ia["t"] == ib["t"] and ia["dt"] == ib["dt"] and ia["cycle"] == ib["cycle"] == 30
    # (under COMM_SELF the copy kernel gets no chunks: stale ghosts would break the equality)
    for k in FIELDS:
        assert np.array_equal(fa[k], fb[k]), k


def test_one_rank_nccl_edtmin_and_graphs():
    n = (16, 16, 16)
    s = jittered_state(n, 1)
    for graph in (True, False):
        fa, ia = _run(100, comm_self=True, graph=graph, n=n, init="user", user=s, dt_floor=0.0146)
        fb, ib = _run(100, graph=graph, n=n, init="user", user=s, dt_floor=0.0146)
        assert ia["status"] == ib["status"] == -7 and ia["cycle"] == ib["cycle"]
        for k in ("x", "u", "e"):
            assert np.array_equal(fa[k], fb[k]), k
