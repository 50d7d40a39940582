"""Bisect: concurrent independent single-rank contexts (tiled) vs oracle."""
import sys, os, threading
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np, torch
from parity_util import c1_case, run_oracle
from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
QM, DT, W = 0.5, 1.0, 1.0
mesh, ef, init, inject, steps = c1_case(drift=0.4, spread=0.1)
om, orc, Qo, ost, rem = run_oracle(mesh, ef, init, inject, steps, QM * DT, DT, W)
so = set(orc["id"].tolist())
def run(kw, nthreads):
    streams = [torch.cuda.Stream() for _ in range(nthreads)]
    out = [None] * nthreads
    def w(r):
        sim = MiniFemPic(mesh, ef, torch_alloc=False, stream=streams[r].cuda_stream, **kw)
        sim.inject(init)
        for s in range(steps):
            sim.inject(inject(s)); sim.step(DT, QM, W)
        out[r] = sim.particles(); sim.close()
    th = [threading.Thread(target=w, args=(r,)) for r in range(nthreads)]
    [t.start() for t in th]; [t.join() for t in th]
    return sum(set(o["id"].tolist()) != so for o in out)
for name, kw, nt in (("tiled x1", {}, 1), ("tiled x2", {}, 2), ("tiled x3", {}, 3), ("direct x3", dict(tma_pipeline=False), 3)):
    f = sum(run(kw, nt) for _ in range(5))
    print(name, "mismatching runs", f, flush=True)
