"""Host-side (CPU) tests of the product library: C-ABI exports and the integer layout.

The layout (domain boxes, domain->rank map, halo slabs) is pinned bitwise against an
independent brute-force construction from global indices (SURVEY §8c.7 "Index, layout and halo
maps: brute force, bitwise").  PAPER.md L525-572 (domain decomposition, hierarchical split),
L589-603 and L652-660 (weighted split, whole planes) define the rules; DESIGN.md §5 states them.
"""
import ctypes
import itertools
import os
import re

import numpy as np
import pytest

from paper_conf_icppw_pearce18_b200 import (HydroConfig, decompose_hierarchical, layout_export,
                                            load_library, weighted_slabs)
from paper_conf_icppw_pearce18_b200.hydro import LIB_PATH

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "hydro.h")).read()
    names = sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(hydro_\w+)\s*\(", hdr, re.M)))
    assert len(names) >= 15
    lib = ctypes.CDLL(LIB_PATH)
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing
    assert load_library().hydro_abi_version() == 4


def parse(buf):
    w = list(map(int, buf))
    ver, nd, nranks, npairs = w[:4]
    N = w[4:7]
    pos = 7
    doms = []
    for _ in range(nd):
        doms.append((tuple(w[pos:pos + 3]), tuple(w[pos + 3:pos + 6]), w[pos + 6]))
        pos += 7
    pairs = []
    for _ in range(npairs):
        pairs.append(tuple(w[pos:pos + 15]))
        pos += 15
    assert pos == len(w) and ver == 1
    return N, doms, nranks, pairs


def brute_force_pairs(N, cuts):
    """Ghost slabs from global indices: for every domain, every ghost node/zone that exists is
    tagged with its direction (-1/0/+1 per axis); each direction's set must be one box."""
    nd = [len(c) - 1 for c in cuts]
    doms = []
    for c, b, a in itertools.product(range(nd[2]), range(nd[1]), range(nd[0])):
        lo = (cuts[0][a], cuts[1][b], cuts[2][c])
        n = (cuts[0][a + 1] - lo[0], cuts[1][b + 1] - lo[1], cuts[2][c + 1] - lo[2])
        doms.append(((a, b, c), lo, n))
    index = {d[0]: i for i, d in enumerate(doms)}
    out = []
    for di, (idx, lo, n) in enumerate(doms):
        groups_n, groups_z = {}, {}
        for g in itertools.product(*[range(lo[ax] - 1, lo[ax] + n[ax] + 2) for ax in range(3)]):
            if any(g[ax] < 0 or g[ax] > N[ax] for ax in range(3)):
                continue
            dirv = tuple(-1 if g[ax] < lo[ax] else (1 if g[ax] > lo[ax] + n[ax] else 0)
                         for ax in range(3))
            if dirv != (0, 0, 0):
                groups_n.setdefault(dirv, []).append(g)
        for g in itertools.product(*[range(lo[ax] - 1, lo[ax] + n[ax] + 1) for ax in range(3)]):
            if any(g[ax] < 0 or g[ax] >= N[ax] for ax in range(3)):
                continue
            dirv = tuple(-1 if g[ax] < lo[ax] else (1 if g[ax] >= lo[ax] + n[ax] else 0)
                         for ax in range(3))
            if dirv != (0, 0, 0):
                groups_z.setdefault(dirv, []).append(g)
        for dirv in sorted(set(groups_n) | set(groups_z), key=lambda d: (d[2], d[1], d[0])):
            src_idx = tuple(idx[ax] + dirv[ax] for ax in range(3))
            src = index[src_idx]
            gn = np.array(groups_n[dirv])
            gz = np.array(groups_z[dirv])
            nlo, nhi = gn.min(0), gn.max(0) + 1
            zlo, zhi = gz.min(0), gz.max(0) + 1
            assert len(gn) == np.prod(nhi - nlo) and len(gz) == np.prod(zhi - zlo)  # boxes
            # the slab lies inside the source's owned nodes / zones
            slo, sn = doms[src][1], doms[src][2]
            assert all(slo[ax] <= nlo[ax] and nhi[ax] - 1 <= slo[ax] + sn[ax] for ax in range(3))
            assert all(slo[ax] <= zlo[ax] and zhi[ax] <= slo[ax] + sn[ax] for ax in range(3))
            code = (dirv[0] + 1) + 3 * (dirv[1] + 1) + 9 * (dirv[2] + 1)
            out.append((di, src, code, *nlo.tolist(), *nhi.tolist(), *zlo.tolist(), *zhi.tolist()))
    return doms, out


CASES = [
    ((6, 5, 4), [[0, 6], [0, 5], [0, 4]]),
    ((8, 7, 6), [[0, 3, 8], [0, 7], [0, 2, 6]]),
    ((9, 9, 9), [[0, 1, 5, 9], [0, 4, 9], [0, 3, 6, 9]]),
    ((5, 6, 7), [[0, 1, 2, 3, 4, 5], [0, 6], [0, 7]]),
]


@pytest.mark.parametrize("N,cuts", CASES)
def test_layout_matches_brute_force_bitwise(N, cuts):
    ndom = tuple(len(c) - 1 for c in cuts)
    buf = layout_export(HydroConfig(n=N, ndom=ndom, cuts=cuts))
    NN, doms, nranks, pairs = parse(buf)
    assert tuple(NN) == N and nranks == 1
    bdoms, bpairs = brute_force_pairs(N, cuts)
    assert [(d[1], d[2]) for d in bdoms] == [(d[0], d[1]) for d in doms]
    assert sorted(pairs) == sorted(bpairs)


def test_even_split_default_cuts():
    N = (10, 7, 9)
    buf = layout_export(HydroConfig(n=N, ndom=(3, 2, 4)))
    _, doms, _, _ = parse(buf)
    lo_x = sorted({d[0][0] for d in doms})
    assert lo_x == [(10 * a) // 3 for a in range(3)]


def py_lpt(cost, nranks, w=None):
    w = w or [1.0] * nranks
    order = sorted(range(len(cost)), key=lambda d: (-cost[d], d))
    load = [0.0] * nranks
    own = [0] * len(cost)
    for d in order:
        vals = [(load[g] + cost[d]) / w[g] for g in range(nranks)]
        g = min(range(nranks), key=lambda g: (vals[g], g))
        own[d] = g
        load[g] += cost[d]
    return own


@pytest.mark.parametrize("nranks,weights", [(2, None), (3, None), (4, [1.0, 2.0, 1.0, 0.5]),
                                            (8, None)])
def test_lpt_assignment_matches_independent_python(nranks, weights):
    c = [0, 64, 160, 288, 448]
    cfg = HydroConfig(n=(448,) * 3, ndom=(4, 4, 4), cuts=[c, c, c], nranks=nranks,
                      rank_weight=weights)
    _, doms, _, _ = parse(layout_export(cfg))
    cost = [int(np.prod(d[1])) for d in doms]
    assert [d[2] for d in doms] == py_lpt(cost, nranks, weights)


def test_lpt_graham_bound_exhaustive():
    rng = np.random.default_rng(0)
    for _ in range(30):
        nd = int(rng.integers(2, 7))
        m = int(rng.integers(2, 4))
        cuts = [[0] + sorted(rng.choice(np.arange(1, 20), nd - 1, replace=False).tolist()) + [20],
                [0, 3], [0, 2]]
        cfg = HydroConfig(n=(20, 3, 2), ndom=(nd, 1, 1), cuts=cuts, nranks=m)
        _, doms, _, _ = parse(layout_export(cfg))
        cost = [int(np.prod(d[1])) for d in doms]
        loads = np.zeros(m)
        for d in doms:
            loads[d[2]] += np.prod(d[1])
        opt = min(max(np.bincount(a, weights=cost, minlength=m))
                  for a in itertools.product(range(m), repeat=nd))
        assert loads.max() <= (4.0 / 3.0 - 1.0 / (3 * m)) * opt + 1e-9


def test_uneven448_balance():
    c = [0, 64, 160, 288, 448]
    for G, bound in ((1, 1.0), (2, 1.002), (4, 1.002), (8, 1.015)):
        cfg = HydroConfig(n=(448,) * 3, ndom=(4, 4, 4), cuts=[c, c, c], nranks=G)
        _, doms, _, _ = parse(layout_export(cfg))
        loads = np.zeros(G)
        for d in doms:
            loads[d[2]] += np.prod(d[1])
        assert loads.max() / loads.mean() <= bound


@pytest.mark.parametrize("n,ngpu,dpg", [((512,) * 3, 8, 1), ((512,) * 3, 2, 4), ((384,) * 3, 1, 4),
                                        ((768, 384, 384), 2, 4), ((256, 128, 64), 4, 2),
                                        ((128, 128, 256), 6, 1)])
def test_hierarchical_decomposition(n, ngpu, dpg):
    ndom, cuts, d2r = decompose_hierarchical(n, ngpu, dpg)
    assert ndom[1] % dpg == 0
    gx, gy, gz = ndom[0], ndom[1] // dpg, ndom[2]
    assert gx * gy * gz == ngpu
    # minimal interface area over all factorisations (step 1), x split as little as possible
    best = min(((fx - 1) * n[1] * n[2] + (fy - 1) * n[0] * n[2] + (fz - 1) * n[0] * n[1], fx, fy)
               for fx in range(1, ngpu + 1) for fy in range(1, ngpu + 1) for fz in range(1, ngpu + 1)
               if fx * fy * fz == ngpu)
    area = (gx - 1) * n[1] * n[2] + (gy - 1) * n[0] * n[2] + (gz - 1) * n[0] * n[1]
    assert (area, gx, gy) == best
    # every rank gets dpg domains forming one box, split only along y (step 2)
    for r in range(ngpu):
        mine = [d for d in range(len(d2r)) if d2r[d] == r]
        assert len(mine) == dpg
        coords = [(d % ndom[0], (d // ndom[0]) % ndom[1], d // (ndom[0] * ndom[1])) for d in mine]
        assert len({c[0] for c in coords}) == 1 and len({c[2] for c in coords}) == 1
        ys = sorted(c[1] for c in coords)
        assert ys == list(range(ys[0], ys[0] + dpg))
    for a in range(3):
        assert cuts[a][0] == 0 and cuts[a][-1] == n[a]
        assert all(b > a_ for a_, b in zip(cuts[a], cuts[a][1:]))


def test_weighted_slabs_whole_planes():
    for N, w in ((480, [1, 1, 1, 1] + [0.0125] * 12), (240, [3.0, 1.0]), (100, [1] * 7),
                 (40, [1, 1, 1, 1] + [0.05] * 12)):
        out = weighted_slabs(N, w)
        assert sum(out) == N and min(out) >= 1
        W = sum(w)
        if all(N * x / W >= 1 for x in w):
            assert all(abs(o - N * x / W) < 1 for o, x in zip(out, w))
    assert weighted_slabs(12, [1, 1, 1]) == [4, 4, 4]


def test_invalid_configs_rejected():
    from paper_conf_icppw_pearce18_b200 import HydroError
    with pytest.raises(HydroError):
        layout_export(HydroConfig(n=(8, 8, 8), ndom=(2, 1, 1), cuts=[[0, 8, 8], [0, 8], [0, 8]]))
    with pytest.raises(HydroError):
        layout_export(HydroConfig(n=(8, 8, 8), ndom=(1, 1, 1), nranks=2, dom_to_rank=[5]))
