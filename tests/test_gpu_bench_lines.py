"""bench.py's multi-rank lines on one GPU (-m gpu): `--gpus 2 --loopback` runs
two slab ranks as threads joined by the loopback transport; the JSON line
must carry the slab parallelism, the roofline, the e2e number and launches."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _line(*args):
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT,
                         capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [json.loads(x) for x in out.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1, out.stdout
    return lines[0]


def _common(d):
    assert d["value"] > 0 and d["e2e"]["value"] > 0 and d["gpu_launches"] > 0
    assert d["n_gpus"] == 1 and d["config"]["ranks"] == 2
    assert d["config"]["parallelism"].startswith("slab2")
    assert 0 < d["roofline"]["frac"] < 1.5


def test_bench_c3_loopback_two_slabs():
    d = _line("--config", "c3", "--gpus", "2", "--loopback", "--steps", "3", "--warmup", "3",
              "--ppc", "20", "--reps", "1", "--no-cpu")
    _common(d)
    assert d["config"]["mesh_cells"] == 2 * d["config"]["mesh_cells_per_rank"]


def test_bench_c4_loopback_two_slabs():
    d = _line("--config", "c4", "--gpus", "2", "--loopback", "--steps", "3", "--warmup", "3",
              "--n0", "2000000", "--reps", "1", "--no-cpu")
    _common(d)
