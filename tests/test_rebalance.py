"""Measured-weight rebalancing ("We started with an
initial guess of work split ... based on FLOPS.  We measured the respective contributions ...
and adjusted the split"; L1077-1081: "static within an iteration, but the decomposition can be
adjusted between iterations").  Host-only planner hydro_rebalance_plan, checked against an
independent Python restatement of its rule (DESIGN.md §3 reading R19 + the f2 speed model) and
against what the rule must achieve.
"""
import itertools

import numpy as np
import pytest

from paper_conf_icppw_pearce18_b200 import HydroConfig, dom_to_rank, layout_export, rebalance_plan

CUTS = [0, 64, 160, 288, 448]  # BASELINE.json config 5 (uneven 448^3, 64 domains)


def _layout(cfg):
    lay = [int(v) for v in layout_export(cfg)]
    nd, nr, npairs = lay[1], lay[2], lay[3]
    doms = [lay[7 + 7 * d: 7 + 7 * (d + 1)] for d in range(nd)]
    base = 7 + 7 * nd
    pairs = [lay[base + 15 * i: base + 15 * (i + 1)] for i in range(npairs)]
    return doms, pairs


def _py_plan(cfg, busy, beta, min_gain):
    """Independent restatement: cost = zones + beta*ghost elements; w_g = load_g/busy_g
    normalised to mean 1; LPT over (-cost, id), argmin (load+c)/w, ties lowest rank."""
    doms, pairs = _layout(cfg)
    nd, G = len(doms), cfg.nranks
    ghost = [0] * nd
    for p in pairs:
        nn = (p[6] - p[3]) * (p[7] - p[4]) * (p[8] - p[5])
        nz = (p[12] - p[9]) * (p[13] - p[10]) * (p[14] - p[11])
        ghost[p[0]] += nn + nz
    cost = [int(round(d[3] * d[4] * d[5] + beta * ghost[i])) for i, d in enumerate(doms)]
    cur = [d[6] for d in doms]
    load = [sum(c for c, r in zip(cost, cur) if r == g) for g in range(G)]
    w = [load[g] / busy[g] if load[g] > 0 else None for g in range(G)]
    known = [v for v in w if v is not None]
    w = [v if v is not None else sum(known) / len(known) for v in w]
    mean = sum(w) / G
    w = [v / mean for v in w]
    order = sorted(range(nd), key=lambda d: (-cost[d], d))
    ld = [0.0] * G
    own = [0] * nd
    for d in order:
        g = min(range(G), key=lambda g: ((ld[g] + cost[d]) / w[g], g))
        own[d] = g
        ld[g] += cost[d]
    before = max(sum(c for c, r in zip(cost, cur) if r == g) / w[g] for g in range(G))
    after = max(ld[g] / w[g] for g in range(G))
    move = after < before * (1 - min_gain)
    return (own if move else cur), w, before, (after if move else before)


def _cfg(G, **kw):
    base = dict(n=(448,) * 3, ndom=(4, 4, 4), cuts=[CUTS] * 3, nranks=G)
    base.update(kw)
    return HydroConfig(**base)


@pytest.mark.parametrize("G", [2, 4, 8])
@pytest.mark.parametrize("beta", [0.0, 1.5])
def test_plan_matches_independent_rule(G, beta):
    rng = np.random.default_rng(G * 10 + int(beta * 2))
    cfg = _cfg(G)
    busy = list(1.0 + 3.0 * rng.random(G))
    new_map, w, (before, after) = rebalance_plan(cfg, busy, beta, 0.02)
    pm, pw, pb, pa = _py_plan(cfg, busy, beta, 0.02)
    assert new_map == pm
    assert np.allclose(w, pw, rtol=1e-14)
    assert before == pytest.approx(pb, rel=1e-14) and after == pytest.approx(pa, rel=1e-14)
    assert sum(w) == pytest.approx(G, rel=1e-14)


def test_equal_speeds_keep_the_map():
    cfg = _cfg(4)
    cur = dom_to_rank(cfg)
    doms, _ = _layout(cfg)
    load = [sum(d[3] * d[4] * d[5] for d in doms if d[6] == g) for g in range(4)]
    # busy proportional to load = identical speeds: nothing to gain, no migration
    new_map, w, (before, after) = rebalance_plan(cfg, load, 0.0, 0.02)
    assert new_map == cur and before == after
    assert np.allclose(w, 1.0, rtol=1e-12)


def test_slow_rank_gets_less_work():
    """Rank 1 measured 3x slower per unit of work: after the plan its modelled time is within
    the LPT bound of the others' and its share drops to about 1/(1+3*(G-1)) of the total."""
    G = 4
    cfg = _cfg(G)
    doms, _ = _layout(cfg)
    cur = dom_to_rank(cfg)
    load = [sum(d[3] * d[4] * d[5] for d, r in zip(doms, cur) if r == g) for g in range(G)]
    busy = [float(l) for l in load]
    busy[1] *= 3.0
    new_map, w, (before, after) = rebalance_plan(cfg, busy, 0.0, 0.02)
    assert w[1] == pytest.approx(w[0] / 3.0, rel=1e-12)
    assert after < 0.75 * before
    tot = sum(d[3] * d[4] * d[5] for d in doms)
    share1 = sum(d[3] * d[4] * d[5] for d, r in zip(doms, new_map) if r == 1) / tot
    assert 0.5 * (1 / 10) <= share1 <= 2.0 * (1 / 10)
    # the modelled makespan obeys Graham's LPT bound against a lower bound of the optimum
    cost = [d[3] * d[4] * d[5] for d in doms]
    lb = max(tot / sum(w), max(cost) / max(w))
    assert after <= (4.0 / 3.0) * lb + max(cost) / min(w)


def test_plan_optimal_on_small_instances_within_graham_bound():
    """<= 8 domains on <= 3 ranks: the LPT makespan is within (4/3 - 1/(3m)) of the exhaustive
    optimum for identical speeds (Graham 1969), and never worse than the current map."""
    for G in (2, 3):
        cfg = HydroConfig(n=(40, 30, 20), ndom=(2, 2, 2), cuts=[[0, 9, 40], [0, 21, 30],
                                                                 [0, 4, 20]], nranks=G,
                          dom_to_rank=[d % G for d in range(8)])
        doms, _ = _layout(cfg)
        cost = [d[3] * d[4] * d[5] for d in doms]
        cur = [d[6] for d in doms]
        load = [sum(c for c, r in zip(cost, cur) if r == g) for g in range(G)]
        new_map, w, (before, after) = rebalance_plan(cfg, [float(l) for l in load], 0.0, 0.0)
        opt = min(max(sum(c for c, r in zip(cost, m) if r == g) for g in range(G))
                  for m in itertools.product(range(G), repeat=8))
        assert after <= (4 / 3 - 1 / (3 * G)) * opt + 1e-9
        assert after <= before


def test_invalid_inputs_rejected():
    cfg = _cfg(2)
    from paper_conf_icppw_pearce18_b200 import HydroError
    with pytest.raises(HydroError):
        rebalance_plan(cfg, [1.0, 0.0])
    with pytest.raises(HydroError):
        rebalance_plan(cfg, [1.0, 1.0], beta=-1.0)
    with pytest.raises(ValueError):
        rebalance_plan(cfg, [1.0])
