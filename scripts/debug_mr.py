import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
from parity_util import c1_case, run_oracle, NEAR
from test_gpu_multirank import _run_ranks, QM, DT, W
for R, dep in ((3, 0), (2, 2), (3, 2)):
    mesh, ef, init, inject, steps = c1_case(drift=0.4, spread=0.1)
    om, orc, Qo, ost, rem = run_oracle(mesh, ef, init, inject, steps, QM * DT, DT, W)
    parts, Qg, stats = _run_ranks(mesh, ef, init, inject, steps, R, deposit_mode=dep)
    so, sg = set(orc["id"].tolist()), set(parts["id"].tolist())
    print("R", R, "dep", dep, "final gpu", len(parts["id"]), "oracle", len(orc["id"]), "only-oracle", sorted(so - sg)[:5], "only-gpu", sorted(sg - so)[:5])
    for i in sorted(so ^ sg)[:5]:
        if i in so:
            k = np.searchsorted(orc["id"], i); print("  oracle has", i, orc["cell"][k], orc["pos"][k], orc["margin"][k])
        if i in sg:
            k = np.searchsorted(parts["id"], i); print("  gpu has", i, parts["cell"][k], parts["pos"][k])
        if i in rem: print("  oracle removed margin", rem[i])
    for s in range(steps):
        tot = [sum(st[s][k] for st in stats) for k in ("n_before", "n_removed", "n_after", "total_hops")]
        print(s, "oracle", ost[s]["n_before"], ost[s]["n_removed"], ost[s]["n_after"], ost[s]["total_hops"], "| gpu", tot)
