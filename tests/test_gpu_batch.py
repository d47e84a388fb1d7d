"""hydro_run_batch (include/hydro.h): independent runs streamed through one context with the
host<->device copies of neighbouring batches overlapped with the cycles.  Every batch must equal,
bitwise, the same run done with the synchronous calls (hydro_set_state + hydro_step +
hydro_get_fields), which the other parity tests pin to the oracle; batch 0 started from the
creation state is also compared with the oracle directly (north_star tolerance)."""
import numpy as np
import pytest

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig, HydroError
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err

pytestmark = pytest.mark.gpu

NAMES = ("x", "y", "z", "u", "v", "w", "e")


def _sync_run(kw, state, t0, dt0, ncycles):
    with Hydro(HydroConfig(**kw)) as h:
        h.set_state(state, state["e"], t0, dt0)
        info = h.step(ncycles)
        f = h.fields(NAMES)
    return f, info


@pytest.mark.parametrize("path", ["two", "one", "split"])
@pytest.mark.parametrize("layout", [dict(), dict(ndom=(2, 2, 1), cuts=[[0, 7, 20], [0, 9, 18], [0, 14]])])
def test_batches_equal_synchronous_runs(layout, path):
    n = (20, 18, 14)
    kw = dict(n=n, init="user", user=jittered_state(n, 3), path=path, **layout)
    states = [jittered_state(n, s) for s in (3, 4, 5, 6, 7)]
    with Hydro(HydroConfig(**kw)) as h:
        i0 = h.info()
        t0 = [0.0] + [0.01 * b for b in range(1, len(states))]
        dt0 = [i0["dt"]] + [2e-4] * (len(states) - 1)
        outs, infos = h.run_batch(states, 12, t0, dt0)
        after = h.fields(NAMES)
    for b, st in enumerate(states):
        ref, ir = _sync_run(kw, st, t0[b], dt0[b], 12)
        assert infos[b]["status"] == 0 and infos[b]["cycle"] == 12
        assert infos[b]["t"] == ir["t"] and infos[b]["dt"] == ir["dt"], b
        for k in NAMES:
            assert np.array_equal(outs[b][k], ref[k]), (b, k)
    for k in NAMES:  # the context continues from the last batch's state
        assert np.array_equal(after[k], outs[-1][k]), k
    # batch 0 is the creation state: the oracle's run of it
    okw = {k: v for k, v in kw.items() if k in ("n", "init", "user", "ndom", "cuts")}
    fo, io = oracle.run(OracleConfig(**okw), 12)
    for k in NAMES:
        assert rel_err(outs[0][k], fo[k]) <= 1e-11, k
    assert infos[0]["dt"] == pytest.approx(io["dt"], rel=1e-11)


def test_batch_edge_cases():
    n = (16, 16, 16)
    with Hydro(HydroConfig(n=n)) as h:
        outs, infos = h.run_batch([], 5, [], [])
        assert outs == [] and infos == []
        st = h.fields(NAMES)
        with pytest.raises(HydroError):
            h.run_batch([st], 5, [0.0], [0.0])  # dt0 must be > 0
        # zero cycles: the output is the input, bit for bit
        outs, infos = h.run_batch([st, st], 0, [0.0, 0.0], [1e-4, 1e-4])
        for b in range(2):
            for k in NAMES:
                assert np.array_equal(outs[b][k], st[k]), k
            assert infos[b]["cycle"] == 0


def test_batch_physics_error_is_per_batch():
    """A tangled batch halts only its own cycles and reports its status; the next batch runs."""
    n = (12, 12, 12)
    good = jittered_state(n, 2)
    bad = {k: v.copy() for k, v in good.items()}
    bad["u"][6, 6, 6] = 1e3  # one node thrown through its neighbours: V <= 0 within a cycle
    kw = dict(n=n, init="user", user=good)
    with Hydro(HydroConfig(**kw)) as h:
        outs, infos = h.run_batch([bad, good], 8, [0.0, 0.0], [1e-3, 1e-4])
    assert infos[0]["status"] == -5 and infos[0]["cycle"] < 8
    assert infos[1]["status"] == 0 and infos[1]["cycle"] == 8
    ref, _ = _sync_run(kw, good, 0.0, 1e-4, 8)
    for k in NAMES:
        assert np.array_equal(outs[1][k], ref[k]), k


def test_batch_t_stop():
    """With t_stop, a batch starting at or past it runs only no-op cycles (state carried), and one
    starting just before it stops at t_stop exactly, as the synchronous calls do."""
    n = (14, 12, 10)
    kw = dict(n=n, init="user", user=jittered_state(n, 6), t_stop=0.01)
    states = [jittered_state(n, s) for s in (6, 7, 8)]
    t0, dt0 = [0.0, 0.0099, 0.01], [1e-4, 5e-4, 1e-4]
    with Hydro(HydroConfig(**kw)) as h:
        outs, infos = h.run_batch(states, 30, t0, dt0)
    for b, st in enumerate(states):
        ref, ir = _sync_run(kw, st, t0[b], dt0[b], 30)
        assert infos[b]["t"] == ir["t"] and infos[b]["cycle"] == ir["cycle"], (b, infos[b], ir)
        for k in NAMES:
            assert np.array_equal(outs[b][k], ref[k]), (b, k)
    assert infos[1]["t"] == pytest.approx(0.01, rel=1e-14)
    for k in NAMES:  # started at t_stop: nothing moves
        assert np.array_equal(outs[2][k], states[2][k]), k
