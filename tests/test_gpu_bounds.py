"""Bounds-checked build of libopp (OPP_CHECKED=1: device asserts on every
cell, node, overlay-slot, particle and list index the particle loop, the
continuation, the sort and the hole fill compute) run over the small C1-style
case of tests/sanitize_case.py (TMA pipeline, rings, continuation, periodic
sort with and without the predicted key, fill; all three deposit modes).

compute-sanitizer is closed on the GPU pool (runs under it left GPUs needing
a reset), so this build stands in for its memcheck: an out-of-range index
trips a device assert, the CUDA context reports cudaErrorAssert, the library
call fails and the case exits non-zero (-m gpu)."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "variants", "libopp_checked.so")


@pytest.fixture(scope="module")
def checked_lib():
    env = dict(os.environ, OPP_NVCC_EXTRA="-DOPP_CHECKED=1", OPP_LIB_OUT=LIB)
    os.makedirs(os.path.dirname(LIB), exist_ok=True)
    r = subprocess.run([sys.executable, "-c", "import paper_conf_icpp_lantra0m24_b200.build as b; b.build(force=True)"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    return LIB


@pytest.mark.parametrize("dep,dh,lead", [(1, 1, 0.0), (1, 1, 2.0), (2, 0, 0.0), (0, 2, 0.0), (2, 1, 1.0)])
def test_checked_build_clean(checked_lib, dep, dh, lead):
    env = dict(os.environ, OPP_LIB=checked_lib)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "tests", "sanitize_case.py"), str(dep), str(dh), str(lead)],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "sanitize case ok" in r.stdout, (r.stdout[-2000:], r.stderr[-3000:])


def test_checked_build_trips_on_a_bad_cell(checked_lib):
    """The checks are live: a particle injected with a cell id past the mesh
    makes the step fail (device assert) instead of reading past the lines."""
    code = f"""
import sys; sys.path.insert(0, {ROOT!r})
import numpy as np, gen
from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
mesh = gen.kuhn_duct(4, 4, 6, seed=3)
init = gen.seed_particles(mesh, 1000, 3)
init["cell"][17] = mesh["n_cells"] + 5
sim = MiniFemPic(mesh, np.zeros((mesh["n_cells"], 3)), torch_alloc=False, deposit_mode=1)
try:
    sim.inject(init)
    sim.step(1.0, 0.5, 1.0)
    sim.node_charge_host()
except Exception as e:
    print("failed as expected:", type(e).__name__)
    sys.exit(3)
print("no failure")
"""
    env = dict(os.environ, OPP_LIB=checked_lib)
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode != 0 and "no failure" not in r.stdout, (r.stdout[-2000:], r.stderr[-2000:])
