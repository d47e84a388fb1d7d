"""The C ABI used from plain C99 (examples/sedov.c, include/hydro.h only): it compiles with
-Wall -Werror against the header on CPU, and on the GPU runs a 32^3 Sedov octant for 100 cycles
conserving total energy to 1e-10 (the program's own check) with the expected mass."""
import os
import re
import subprocess

import pytest

from paper_conf_icppw_pearce18_b200 import _build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_c_example_compiles_against_the_header():
    _build.build()
    exe = _build.build_c_example()
    assert os.access(exe, os.X_OK)


@pytest.mark.gpu
def test_c_example_runs_on_gpu():
    exe = _build.build_c_example()
    r = subprocess.run([exe, "32", "100"], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    m = re.search(r"cycles=(\d+) .* mass=([0-9.eE+-]+) .* rel=([0-9.eE+-]+)", r.stdout)
    assert m and int(m.group(1)) == 100
    assert float(m.group(2)) == pytest.approx(1.2 ** 3, rel=1e-12)  # rho0 = 1 on [0, 1.2]^3
    assert float(m.group(3)) <= 1e-10
