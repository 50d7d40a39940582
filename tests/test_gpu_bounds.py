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


@pytest.mark.parametrize("checked", [True, False])
def test_bad_input_cell_is_dropped_and_reported(checked_lib, checked):
    """A particle injected with a cell id past the mesh is dropped as a hole
    (no access through it; the checked build's asserts stay quiet) and the
    step that reads statistics reports OPP_ERR_ARG; the other particles are
    stepped normally."""
    code = f"""
import sys; sys.path.insert(0, {ROOT!r})
import numpy as np, gen
from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
mesh = gen.kuhn_duct(4, 4, 6, seed=3)
init = gen.seed_particles(mesh, 1000, 3)
init["cell"][17] = mesh["n_cells"] + 5
sim = MiniFemPic(mesh, np.zeros((mesh["n_cells"], 3)), torch_alloc=False, deposit_mode=1)
sim.inject(init)
try:
    sim.step(1.0, 0.5, 1.0)
    print("no error")
except Exception as e:
    print("reported:", e)
st = sim.step(1.0, 0.5, 1.0)      # the next step runs clean
Q = sim.node_charge_host()
print("after", st["n_after"], "charge", round(float(Q.sum()), 6))
"""
    env = dict(os.environ)
    if checked:
        env["OPP_LIB"] = checked_lib
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, (r.stdout[-2000:], r.stderr[-3000:])
    assert "reported:" in r.stdout and "not a cell of this rank" in r.stdout, r.stdout
    after = [ln for ln in r.stdout.splitlines() if ln.startswith("after")][0].split()
    assert int(after[1]) <= 999 and abs(float(after[3]) - int(after[1])) < 1e-6, r.stdout
