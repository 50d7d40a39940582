"""Tiled vs direct fused kernel on the same inputs, step by step."""
import sys, os
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np
from parity_util import c1_case
from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
QM, DT, W = 0.5, 1.0, 1.0
mesh, ef, init, inject, steps = c1_case(drift=0.4, spread=0.1)
sims = {k: MiniFemPic(mesh, ef, torch_alloc=False, tma_pipeline=(k == "tiled")) for k in ("tiled", "direct")}
for k, s in sims.items():
    s.inject(init)
for st in range(steps):
    stats = {}
    raw = {}
    for k, s in sims.items():
        s.inject(inject(st))
        stats[k] = s.step(DT, QM, W, fill=False)
        # storage order view before the fill: holes visible as cell -1
    for k, s in sims.items():
        s.fill_holes()
    P = {k: s.particles() for k, s in sims.items()}
    a, b = P["tiled"], P["direct"]
    sa, sb = set(a["id"].tolist()), set(b["id"].tolist())
    print(st, {k: (v["n_before"], v["n_removed"], v["n_after"], v["total_hops"], v["n_deferred"]) for k, v in stats.items()},
          "only tiled", sorted(sa - sb)[:5], "only direct", sorted(sb - sa)[:5])
    if sa != sb:
        for i in sorted(sa ^ sb)[:4]:
            for nm, p in (("tiled", a), ("direct", b)):
                k = np.searchsorted(p["id"], i)
                if k < len(p["id"]) and p["id"][k] == i:
                    print("   ", nm, "id", i, "cell", p["cell"][k], "pos", p["pos"][k])
        break
    common = np.array(sorted(sa & sb))
    ia, ib = np.searchsorted(a["id"], common), np.searchsorted(b["id"], common)
    dc = np.nonzero(a["cell"][ia] != b["cell"][ib])[0]
    dx = np.nonzero(np.abs(a["pos"][ia] - b["pos"][ib]).max(1) > 0)[0]
    if len(dc) or len(dx):
        print("   cell diffs", len(dc), "pos diffs", len(dx), "ids", common[dc[:4]], common[dx[:4]])
        for q in list(dc[:3]):
            print("    tiled", a["cell"][ia[q]], a["pos"][ia[q]], "direct", b["cell"][ib[q]], b["pos"][ib[q]])
        break
