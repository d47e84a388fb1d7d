"""Fused halo (opt-in HydroConfig.halo="fused"): the node/energy stage stores every
neighbour's ghost slab from its own epilogue instead of a separate copy kernel after it.  The ghost layer is what PAPER.md
L548-557 exchanges between neighbouring domains; decomposed runs must equal the undecomposed
run bitwise (SURVEY §8e ghost contract) and the oracle within the north_star tolerance, with
either exchange (HydroConfig.halo = "fused" | "kernel")."""
import numpy as np
import pytest

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")


def run(ncycles, **kw):
    with Hydro(HydroConfig(**kw)) as h:
        info = h.step(ncycles)
        f = h.fields()
    return f, info


def _ocfg(kw):
    keys = ("n", "origin", "extent", "init", "user", "ndom", "cuts", "t_stop")  # no "halo"
    return OracleConfig(**{k: v for k, v in kw.items() if k in keys})


def test_fused_equals_halo_kernels_and_single_domain():
    # 1-zone-thick domains in y and z: a source's interface node is also its send layer
    n = (24, 20, 18)
    cuts = [[0, 5, 13, 24], [0, 1, 20], [0, 9, 10, 18]]
    kw = dict(n=n, ndom=(3, 2, 3), cuts=cuts, init="user", user=jittered_state(n, 7))
    ff, i_f = run(25, halo="fused", **kw)
    fk, i_k = run(25, halo="kernel", **kw)
    fs, _ = run(25, n=n, init="user", user=kw["user"])
    assert i_f["status"] == 0 and i_f["dt"] == i_k["dt"]
    for k in FIELDS:
        assert np.array_equal(ff[k], fk[k]), k
        assert np.array_equal(ff[k], fs[k]), k


def test_fused_halo_many_tiles_and_z_chunks_against_oracle():
    # domains several node-stage tiles (32 x 12) wide, tall enough in z for several z-chunks,
    # so the slabs are split over many CTAs and chunk boundaries
    n = (70, 50, 90)
    cuts = [[0, 33, 70], [0, 13, 37, 50], [0, 45, 90]]
    kw = dict(n=n, ndom=(2, 3, 2), cuts=cuts, init="user", user=jittered_state(n, 12),
              halo="fused")
    fg, ig = run(8, **kw)
    fs, _ = run(8, n=n, init="user", user=kw["user"])
    for k in FIELDS:
        assert np.array_equal(fg[k], fs[k]), k
    fo, io = oracle.run(_ocfg(kw), 8)
    assert ig["dt"] == pytest.approx(io["dt"], rel=1e-11)
    for k in FIELDS:
        assert rel_err(fg[k], fo[k]) <= 1e-11, k


def test_fused_halo_no_op_cycles_after_t_stop():
    # once t_stop is reached the cycles are no-ops that carry the state (and the ghost layer,
    # through the same epilogue stores) to the next parity
    n = (16, 16, 16)
    kw = dict(n=n, ndom=(2, 2, 2), t_stop=0.01, halo="fused")
    fg, ig = run(400, **kw)
    fs, is_ = run(400, n=n, t_stop=0.01)
    assert ig["t"] == pytest.approx(0.01, rel=1e-14) and ig["cycle"] == is_["cycle"]
    for k in FIELDS:
        assert np.array_equal(fg[k], fs[k]), k
    fo, io = oracle.run(_ocfg(kw), 400)
    assert ig["cycle"] == io["cycle"]
    for k in FIELDS:
        assert rel_err(fg[k], fo[k]) <= 1e-10, k


def test_kernels_per_cycle_counts_the_fused_exchange(monkeypatch):
    kw = dict(n=(16, 16, 16), ndom=(1, 2, 1))
    with Hydro(HydroConfig(halo="fused", **kw)) as h:
        kf = h.kernels_per_cycle()
    monkeypatch.setenv("HYDRO_HALO_OVERLAP", "0")
    with Hydro(HydroConfig(halo="kernel", **kw)) as h:
        kk = h.kernels_per_cycle()
    assert kk == kf + 1  # fused: no separate intra-GPU copy kernel
    monkeypatch.setenv("HYDRO_HALO_OVERLAP", "2")
    with Hydro(HydroConfig(halo="kernel", **kw)) as h:
        ko = h.kernels_per_cycle()
    assert ko == kf + 2  # overlapped: one copy per source domain


@pytest.mark.parametrize("mode", ["1", "2", "3"])
def test_overlapped_halo_copy_bitwise(mode, monkeypatch):
    """Per-source-domain halo copies launched right after each domain's node/energy stage
    (HYDRO_HALO_OVERLAP=1: on its node-stage stream; 2: on a dedicated halo stream; 3: one copy
    per node-stage stream after its last domain, the default when each of the 4 streams holds
    at most 2 domains, else 0 = one copy after the join) equal the single copy after the join
    and the undecomposed run bitwise, with more domains than node-stage streams (uneven cuts,
    1-zone-thick domains)."""
    n = (24, 20, 18)
    cuts = [[0, 5, 13, 24], [0, 1, 20], [0, 9, 10, 18]]
    kw = dict(n=n, ndom=(3, 2, 3), cuts=cuts, init="user", user=jittered_state(n, 9),
              halo="kernel")
    monkeypatch.setenv("HYDRO_HALO_OVERLAP", mode)
    fo, io = run(30, **kw)
    monkeypatch.setenv("HYDRO_HALO_OVERLAP", "0")
    fj, ij = run(30, **kw)
    fs, _ = run(30, n=n, init="user", user=kw["user"])
    assert io["status"] == 0 and io["dt"] == ij["dt"]
    for k in FIELDS:
        assert np.array_equal(fo[k], fj[k]), k
        assert np.array_equal(fo[k], fs[k]), k


def test_node_tile_heights_bitwise(monkeypatch):
    """Both compiled node-stage tile heights (kernel_cycle.cu node_tile_ty picks one per domain)
    give the same bits: the tile shape changes which CTA computes a node, not the arithmetic."""
    n = (45, 50, 23)
    kw = dict(n=n, ndom=(1, 2, 1), init="user", user=jittered_state(n, 5))
    monkeypatch.setenv("HYDRO_NODE_TY", "11")
    fa, _ = run(12, **kw)
    monkeypatch.setenv("HYDRO_NODE_TY", "12")
    fb, _ = run(12, **kw)
    for k in FIELDS:
        assert np.array_equal(fa[k], fb[k]), k
    fo, _ = oracle.run(_ocfg(kw), 12)
    for k in FIELDS:
        assert rel_err(fa[k], fo[k]) <= 1e-11, k


@pytest.mark.parametrize("k", ["1", "3"])
def test_multi_cycle_graphs_bitwise(k, monkeypatch):
    """hydro_step replays graphs of HYDRO_GRAPH_CYCLES cycles (default 8) plus one-cycle graphs
    for the rest; an odd count flips the parity inside a replay.  Same bits as the default."""
    n = (20, 18, 16)
    kw = dict(n=n, ndom=(1, 2, 1), init="user", user=jittered_state(n, 8))
    fd, idf = run(29, **kw)
    monkeypatch.setenv("HYDRO_GRAPH_CYCLES", k)
    fk, ik = run(29, **kw)
    assert idf["cycle"] == ik["cycle"] == 29 and idf["t"] == ik["t"]
    for f in FIELDS:
        assert np.array_equal(fd[f], fk[f]), f
