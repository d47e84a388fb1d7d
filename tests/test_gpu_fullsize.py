"""Full-size multi-domain check in the launch configuration bench.py times (BASELINE.json
config 5: 448^3 in 64 uneven domains, cuts {0, 64, 160, 288, 448} per axis).

The ghost contract makes a decomposed run equal the
undecomposed one bit for bit: interface nodes are computed by both neighbours from identical
inputs and the exchanged ghost layer carries exact copies.  The Sedov blast never reaches the
first cut at 64 zones with this scheme (without hourglass control a zone next to the origin is
crushed after ~1100 cycles), so the run starts from a smooth, everywhere-moving
state (acoustic waves through every interface from the first cycle) and windows around the cut
lines -- faces, edges, and the corners where eight domains meet -- are compared bitwise with
the single-domain run of the same mesh.  The oracle side of uneven layouts is covered at
smaller sizes (test_gpu_halo.py, test_gpu_parity.py).
"""
import numpy as np
import pytest

from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
from tests.helpers import user_state

pytestmark = pytest.mark.gpu

N = 448
CUTS = [0, 64, 160, 288, 448]
CYCLES = 20
WINDOWS = [((56, 100, 200), (72, 116, 216)),   # x cut at 64
           ((300, 152, 20), (316, 168, 36)),   # y cut at 160
           ((400, 30, 280), (416, 46, 296)),   # z cut at 288
           ((56, 152, 400), (72, 168, 416)),   # x-y edge
           ((56, 56, 56), (72, 72, 72)),       # eight domains meet
           ((152, 280, 56), (168, 296, 72)),
           ((280, 280, 280), (296, 296, 296)),
           ((440, 440, 440), (448, 448, 448))]  # far corner (walls)


def _state(N=N):
    s = user_state((N, N, N), extent=(1.2, 1.2, 1.2))
    L = 1.2
    x, y, z = s["x"], s["y"], s["z"]
    k = 2.0 * np.pi / L
    s["u"] = 0.05 * np.sin(3 * k * y) * np.cos(2 * k * z) * np.sin(k * x)
    s["v"] = 0.05 * np.sin(2 * k * z) * np.cos(3 * k * x) * np.sin(k * y)
    s["w"] = 0.05 * np.sin(2 * k * x) * np.cos(3 * k * y) * np.sin(k * z)
    zc = (np.arange(N) + 0.5) * (L / N)
    s["rho"] = 1.0 + 0.2 * np.sin(5 * k * zc)[:, None, None] * np.cos(4 * k * zc)[None, :, None] \
        * np.ones((1, 1, N))
    s["e"] = 1.0 + 0.3 * np.cos(3 * k * zc)[None, None, :] * np.ones((N, N, 1))
    return s


def _run(s, N=N, windows=WINDOWS, **kw):
    with Hydro(HydroConfig(n=(N, N, N), init="user", user=s, **kw)) as h:
        info = h.step(CYCLES)
        boxes = [h.box(lo, hi) for lo, hi in windows]
    return info, boxes


def test_uneven448_sixty_four_domains_equal_single_domain_bitwise():
    s = _state()
    i_dec, b_dec = _run(s, ndom=(4, 4, 4), cuts=[CUTS, CUTS, CUTS])
    i_one, b_one = _run(s)
    assert i_dec["status"] == 0 and i_dec["cycle"] == CYCLES
    assert i_dec["t"] == i_one["t"] and i_dec["dt"] == i_one["dt"]
    for (lo, hi), bd, bo in zip(WINDOWS, b_dec, b_one):
        for k in bd:
            assert np.array_equal(bd[k], bo[k]), (lo, hi, k)
        assert np.abs(bd["u"]).max() > 0.0 and np.abs(bd["q"]).max() >= 0.0


W384 = [((100, 88, 150), (116, 104, 166)),    # y cut at 96
        ((0, 184, 0), (16, 200, 16)),          # y cut at 192, on the -x/-z walls
        ((368, 280, 368), (384, 296, 384)),    # y cut at 288, on the +x/+z walls
        ((200, 376, 10), (216, 384, 26))]      # +y wall


def test_weak384_four_y_slabs_equal_single_domain_bitwise():
    """BASELINE config 4 at N=1 in bench.py's launch configuration (384^3 as four 384x96x384
    y-slabs on one GPU: grouped zone stage, node stages on four streams, per-stream halo copies
    overlapped with the other streams' node stages) equals the single-domain run bit for bit
    around every cut, from the smooth moving state."""
    n = 384
    s = _state(n)
    i_dec, b_dec = _run(s, N=n, windows=W384, ndom=(1, 4, 1))
    i_one, b_one = _run(s, N=n, windows=W384)
    assert i_dec["status"] == 0 and i_dec["cycle"] == CYCLES
    assert i_dec["t"] == i_one["t"] and i_dec["dt"] == i_one["dt"]
    for (lo, hi), bd, bo in zip(W384, b_dec, b_one):
        for k in bd:
            assert np.array_equal(bd[k], bo[k]), (lo, hi, k)
