"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by element.

Tolerance (BASELINE.json north_star): relative max-norm per field <= 1e-12 after one cycle,
<= 1e-10 after 100 cycles (reading R15 defines the norm).  Both sides get the same
seeded inputs (paper_conf_icppw_pearce18_b200.inputs) or generate the same analytic Sedov state.
"""
import math

import numpy as np
import pytest

import oracle
from oracle import OracleConfig
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from paper_conf_icppw_pearce18_b200.inputs import jittered_state
from tests.helpers import rel_err, total_energy, user_state

pytestmark = pytest.mark.gpu

FIELDS = ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass")
PATHS = ["two", "one", "split"]  # zone+node/energy kernels (default), one fused kernel, plain split


def run_gpu(ncycles, **kw):
    with Hydro(HydroConfig(**kw)) as h:
        info = h.step(ncycles)
        f = h.fields()
    return f, info


def compare(fg, fo, tol, fields=FIELDS):
    errs = {k: rel_err(fg[k], fo[k]) for k in fields}
    bad = {k: v for k, v in errs.items() if not v <= tol}
    assert not bad, f"fields over {tol}: {bad}"
    return errs


def ocfg(gk):
    keys = ("n", "origin", "extent", "gamma", "q_lin", "q_quad", "cfl", "c_vol", "dt_growth",
            "dt_max", "dt_init", "t_stop", "dt_first", "t0", "reflect_mask", "init", "rho0", "e0",
            "sedov_energy", "user", "ndom", "cuts")
    return OracleConfig(**{k: v for k, v in gk.items() if k in keys})


@pytest.mark.parametrize("path", PATHS)
def test_sedov32_one_and_hundred_cycles(path):
    kw = dict(n=(32, 32, 32))
    for nc, tol in ((1, 1e-12), (100, 1e-10)):
        fo, io = oracle.run(ocfg(kw), nc)
        fg, ig = run_gpu(nc, path=path, **kw)
        assert ig["status"] == 0 and ig["cycle"] == nc
        compare(fg, fo, tol)
        assert ig["t"] == pytest.approx(io["t"], rel=tol)
        assert ig["dt"] == pytest.approx(io["dt"], rel=tol)


@pytest.mark.parametrize("path", PATHS)
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_jittered16(seed, path):
    n = (16, 16, 16)
    kw = dict(n=n, init="user", user=jittered_state(n, seed))
    for nc, tol in ((1, 1e-12), (100, 1e-10)):
        fo, io = oracle.run(ocfg(kw), nc)
        fg, ig = run_gpu(nc, path=path, **kw)
        assert ig["status"] == 0
        compare(fg, fo, tol)
        assert ig["dt"] == pytest.approx(io["dt"], rel=tol)


@pytest.mark.parametrize("path", PATHS)
def test_ragged_mesh_several_tiles(path):
    n = (77, 37, 21)  # not a multiple of any tile size; x spans several warps
    kw = dict(n=n, init="user", user=jittered_state(n, 4))
    fo, _ = oracle.run(ocfg(kw), 10)
    fg, ig = run_gpu(10, path=path, **kw)
    assert ig["status"] == 0
    compare(fg, fo, 1e-11)


@pytest.mark.parametrize("path", PATHS)
def test_multi_domain_on_one_gpu(path):
    n = (24, 20, 18)
    cuts = [[0, 5, 13, 24], [0, 1, 20], [0, 9, 10, 18]]
    kw = dict(n=n, ndom=(3, 2, 3), cuts=cuts, init="user", user=jittered_state(n, 7))
    fo, _ = oracle.run(ocfg(kw), 25)
    fg, ig = run_gpu(25, path=path, **kw)
    assert ig["status"] == 0
    compare(fg, fo, 1e-10)
    single = dict(kw)
    single.update(ndom=(1, 1, 1), cuts=None)
    fs, _ = run_gpu(25, path=path, **single)
    for k in FIELDS:  # same kernels on the same inputs: bitwise
        assert np.array_equal(fs[k], fg[k]), k


@pytest.mark.parametrize("path", PATHS)
def test_energy_conserved_and_mass_constant(path):
    kw = dict(n=(24, 24, 24))
    with Hydro(HydroConfig(path=path, **kw)) as h:
        f0 = h.fields()
        h.step(100)
        f = h.fields()
    E0 = sum(total_energy(f0))
    assert abs(sum(total_energy(f)) - E0) / E0 <= 1e-12
    assert np.array_equal(f["mass"], f0["mass"])


@pytest.mark.parametrize("path", PATHS)
def test_uniform_rest_bitwise(path):
    n = (8, 8, 8)
    s = user_state(n, extent=(1.0, 1.0, 1.0))
    with Hydro(HydroConfig(n=n, extent=(1.0, 1.0, 1.0), init="user", user=s, path=path)) as h:
        f0 = h.fields()
        h.step(50)
        f = h.fields()
    for k in ("x", "y", "z", "u", "v", "w", "e"):
        assert np.array_equal(f[k], f0[k]), k


def test_t_stop_and_no_op_cycles():
    kw = dict(n=(16, 16, 16), t_stop=0.01)
    fo, io = oracle.run(ocfg(kw), 1000)
    fg, ig = run_gpu(1000, **kw)
    assert ig["t"] == pytest.approx(0.01, rel=1e-14)
    assert ig["cycle"] == io["cycle"]
    compare(fg, fo, 1e-10)


def test_tangled_mesh_reported():
    n = (6, 6, 6)
    s = user_state(n, e=1.0)
    s["u"][3, 3, 3] = 1e4
    with Hydro(HydroConfig(n=n, init="user", user=s, dt_first=1e-3)) as h:
        r = h.step(5)
        assert r["rc"] == -5 and r["cycle"] == 1
        io = oracle.Oracle(ocfg(dict(n=n, init="user", user=s, dt_first=1e-3))).step(5)
        assert r["bad_zone"] == io["bad_zone"]
        assert h.step(1)["rc"] == -8


def test_restart_set_state_bitwise():
    kw = dict(n=(16, 12, 10), init="user", user=jittered_state((16, 12, 10), 9))
    with Hydro(HydroConfig(**kw)) as a:
        a.step(10)
        mid = a.fields()
        ia = a.info()
        a.step(10)
        fa = a.fields()
    with Hydro(HydroConfig(**kw)) as b:
        b.set_state(mid, mid["e"], ia["t"], ia["dt"])
        b.step(10)
        fb = b.fields()
    for k in FIELDS:
        assert np.array_equal(fa[k], fb[k]), k


def test_full_size_128_against_oracle():
    """BASELINE.json config 1 (Sedov 128^3, single domain) in the launch configuration bench.py
    times (fused kernel, CUDA graphs), element by element against the oracle."""
    kw = dict(n=(128, 128, 128))
    fo, io = oracle.run(ocfg(kw), 5)
    fg, ig = run_gpu(5, **kw)
    compare(fg, fo, 1e-12)
    assert ig["dt"] == pytest.approx(io["dt"], rel=1e-12)


@pytest.mark.parametrize("path", ["two", "one"])
def test_full_size_512_eight_domains_corner_window(path):
    """BASELINE.json config 2 (Sedov 512^3 as 8 domains, the layout bench.py --config sedov512
    uses at N=1) against the oracle without ever feeding GPU output to the oracle: while the blast
    has not reached zone 48, the corner window [0,48)^3 of the 512^3 run evolves exactly like a
    48^3 Sedov box with the same zone size (both are at rest beyond the blast; walls reflect), so
    the oracle runs that small box from the analytic initial state.  Far from the blast the mesh
    must stay exactly at rest."""
    from paper_conf_icppw_pearce18_b200 import decompose_hierarchical
    n = (512, 512, 512)
    ndom, cuts, d2r = decompose_hierarchical(n, 1, 8)
    cyc = 40
    with Hydro(HydroConfig(n=n, ndom=ndom, cuts=cuts, dom_to_rank=d2r, path=path)) as h:
        info = h.step(cyc)
        win = h.box((0, 0, 0), (48, 48, 48))
        far = h.box((200, 300, 400), (216, 316, 416), names=("u", "v", "w", "e"))
        mid = h.box((0, 60, 0), (16, 70, 16), names=("u", "e"))  # across the first y interface
    w = 48
    fo, io = oracle.run(OracleConfig(n=(w, w, w), extent=(1.2 * w / 512,) * 3), cyc)
    assert info["status"] == 0 and info["cycle"] == cyc
    assert info["dt"] == pytest.approx(io["dt"], rel=1e-10)
    # the blast is confined well inside the window (fields at its outer layer are still at rest)
    assert np.abs(fo["u"][:, :, -4:]).max() == 0.0 and np.abs(fo["e"][:, :, -4:]).max() == 0.0
    for k in ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass"):
        assert rel_err(win[k], fo[k]) <= 1e-10, k
    for k in ("u", "v", "w", "e"):
        assert np.abs(far[k]).max() == 0.0, k
    assert np.abs(mid["u"]).max() == 0.0 and np.abs(mid["e"]).max() == 0.0


PHYS = [  # readings R5 (gamma 5/3 as a second EOS), R7 (Sedov q coefficients 0.25 / 1.0), R8
    dict(gamma=5.0 / 3.0),
    dict(q_lin=0.25, q_quad=1.0),
    dict(q_lin=0.0, q_quad=0.0),  # no viscosity at all
    dict(cfl=0.5, c_vol=0.2, dt_growth=1.05),
    dict(dt_max=2e-4, reflect_mask=0b010101),  # dt cap; walls only on the low faces
]


@pytest.mark.parametrize("path", PATHS)
@pytest.mark.parametrize("phys", range(len(PHYS)))
def test_physics_parameters(phys, path):
    """The C ABI's physics parameters (hydro_config: gamma, q_lin, q_quad, cfl, c_vol, dt_growth,
    dt_max, reflect_mask) reach every kernel path: jittered 18x16x14 (several tiles, ragged) and
    Sedov 24^3 in 2 x 2 domains, against the oracle with the same parameters."""
    n = (18, 16, 14)
    for kw in (dict(n=n, init="user", user=jittered_state(n, 4), **PHYS[phys]),
               dict(n=(24, 24, 24), ndom=(2, 2, 1), **PHYS[phys])):
        for nc, tol in ((1, 1e-12), (60, 1e-10)):
            fo, io = oracle.run(ocfg(kw), nc)
            fg, ig = run_gpu(nc, path=path, **kw)
            assert ig["status"] == io.get("status", 0) == 0, (ig, io)
            compare(fg, fo, tol)
            assert ig["dt"] == pytest.approx(io["dt"], rel=tol)
            assert ig["t"] == pytest.approx(io["t"], rel=tol)
