"""Bisect the flaky multi-rank mismatch: repeat the loopback run under variants."""
import sys, os
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
from parity_util import c1_case, run_oracle
from test_gpu_multirank import _run_ranks, QM, DT, W
mesh, ef, init, inject, steps = c1_case(drift=0.4, spread=0.1)
om, orc, Qo, ost, rem = run_oracle(mesh, ef, init, inject, steps, QM * DT, DT, W)
so = set(orc["id"].tolist())
variants = {
    "default": {},
    "direct": dict(tma_pipeline=False),
    "bigcap": dict(capacity=400_000),
    "direct_bigcap": dict(tma_pipeline=False, capacity=400_000),
}
for name, kw in variants.items():
    fails = 0
    for rep in range(8):
        parts, Qg, stats = _run_ranks(mesh, ef, init, inject, steps, 2, **kw)
        sg = set(parts["id"].tolist())
        if so != sg:
            fails += 1
    print(name, "fails", fails, "/ 8", flush=True)
