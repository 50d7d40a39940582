"""bench.py's reference arm (the CPU oracle timed on host cores) keeps the
JSON-line contract: one line, impl = reference, BASELINE.json's metric and
unit, e2e with zero copy bytes, cpu_baseline describing the run (-m "not gpu")."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("config", ["c4", "c2", "c3", "c2-empty"])
def test_reference_arm_json_line(config):
    extra = ["--empty"] if config.endswith("-empty") else []
    out = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--config", config.split("-")[0],
                          "--steps", "1", "--warmup", "0"] + extra, cwd=ROOT, capture_output=True,
                         text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    base = json.load(open(os.path.join(ROOT, "BASELINE.json")))
    assert d["impl"] == "reference"
    assert d["metric"] == base["metric"]
    assert d["value"] > 0 and d["steps"] == 1 and d["n_gpus"] == 1
    assert d["e2e"]["value"] == d["value"] and d["e2e"]["h2d_bytes_per_step"] == 0
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["value"] == d["value"] and cb["cores"] >= 1 and cb["sample"]


def test_gpus_n_launch_checks():
    """--gpus N outside torchrun starts N ranks itself, and refuses (exit 2,
    one JSON error line) when the box has fewer GPUs; under torchrun
    WORLD_SIZE must equal --gpus."""
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    out = subprocess.run([sys.executable, "bench.py", "--gpus", "2", "--steps", "1"], cwd=ROOT,
                         capture_output=True, text=True, timeout=300, env=env)
    assert out.returncode == 2 and "needs 2 GPUs" in json.loads(out.stdout.strip())["error"]
    env = dict(os.environ, WORLD_SIZE="2", RANK="0")
    out = subprocess.run([sys.executable, "bench.py", "--gpus", "1", "--steps", "1"], cwd=ROOT,
                         capture_output=True, text=True, timeout=300, env=env)
    assert out.returncode == 2 and "WORLD_SIZE=2" in json.loads(out.stdout.strip())["error"]


def _group_worker(rank, world, port, q):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist
    import bench
    try:
        dist.init_process_group("gloo", rank=rank, world_size=world)
        g = bench.Group(world, "dist")
        g.barrier()
        q.put((rank, (g.max("t", 3.0 + rank), g.sum("p", 10 + rank))))
        dist.destroy_process_group()
    except Exception as e:   # noqa: BLE001
        q.put((rank, repr(e)))


def test_group_reductions_gloo_and_loopback():
    """bench.Group: max / sum over ranks under a process group (gloo, world 2,
    as NCCL ranks do it) and over loopback threads (N slabs on one GPU)."""
    import socket
    import threading
    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_group_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = dict(q.get(timeout=180) for _ in range(2))
    for p in ps:
        p.join(timeout=60)
    assert out[0] == out[1] == (4.0, 21), out
    sys.path.insert(0, ROOT)
    import bench
    g = bench.Group(3, "loopback")
    res = [None] * 3

    def w(r):
        g.barrier()
        res[r] = (g.max("a", float(r)), g.sum("b", r + 1), g.max("c", -float(r)))

    th = [threading.Thread(target=w, args=(r,)) for r in range(3)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=30)
    assert res == [(2.0, 6, 0.0)] * 3
