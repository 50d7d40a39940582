import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
from parity_util import c1_case, run_oracle
from test_gpu_multirank import _run_ranks, QM, DT, W
for tma in (True, False):
    mesh, ef, init, inject, steps = c1_case(drift=0.4, spread=0.1)
    om, orc, Qo, ost, rem = run_oracle(mesh, ef, init, inject, steps, QM * DT, DT, W)
    parts, Qg, stats = _run_ranks(mesh, ef, init, inject, steps, 2, deposit_mode=0, tma_pipeline=tma)
    print("tma", tma, "final gpu", len(parts["id"]), "oracle", len(orc["id"]))
    for s in range(steps):
        print(s, "oracle", ost[s]["n_before"], ost[s]["n_removed"], ost[s]["n_after"], "| gpu", [(st[s]["n_before"], st[s]["n_removed"], st[s]["n_after"], st[s]["n_migrated_out"], st[s]["n_migrated_in"]) for st in stats])
