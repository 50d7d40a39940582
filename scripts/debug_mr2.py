"""Step-by-step comparison of the loopback multi-rank run with the oracle."""
import sys, os, threading
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np
import torch
import gen, oracle
from parity_util import c1_case
from paper_conf_icpp_lantra0m24_b200 import dist
from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
QM, DT, W = 0.5, 1.0, 1.0
R, dep = int(sys.argv[1]), int(sys.argv[2])
mesh, ef, init, inject, steps = c1_case(drift=0.4, spread=0.1)
om = oracle.Mesh.from_gen(mesh); om.set_field(ef)
P = oracle.Particles(); P.append(init["pos"], init["vel"], init["cell"], init["id"])
Q = np.zeros(mesh["n_nodes"])
uid = os.urandom(128); roc = dist.rank_of_cell(mesh, R)
streams = [torch.cuda.Stream() for _ in range(R)]
sims = [None] * R
def mk(r):
    sl = dist.slab(mesh, R, r)
    sims[r] = MiniFemPic(sl, dist.local_field(ef, sl), nranks=R, rank=r, uid=uid, transport=1,
                         torch_alloc=False, stream=streams[r].cuda_stream, deposit_mode=dep)
    sims[r].inject(dist.owned(init, roc, r))
th = [threading.Thread(target=mk, args=(r,)) for r in range(R)]
[t.start() for t in th]; [t.join() for t in th]
for s in range(steps):
    b = inject(s)
    P.append(b["pos"], b["vel"], b["cell"], b["id"])
    ost = oracle.step(om, P, QM * DT, DT, W, Q)
    res = [None] * R
    def st(r):
        sims[r].inject(dist.owned(b, roc, r)); res[r] = sims[r].step(DT, QM, W)
    th = [threading.Thread(target=st, args=(r,)) for r in range(R)]
    [t.start() for t in th]; [t.join() for t in th]
    parts = dist.merge_particles([sims[r].particles() for r in range(R)])
    orc = P.get()
    so, sg = set(orc["id"].tolist()), set(parts["id"].tolist())
    common = np.array(sorted(so & sg))
    io = np.searchsorted(orc["id"], common); ig = np.searchsorted(parts["id"], common)
    badc = common[orc["cell"][io] != parts["cell"][ig]]
    badx = common[np.abs(orc["pos"][io] - parts["pos"][ig]).max(1) > 1e-9]
    print(s, "hops o/g", ost["total_hops"], sum(x["total_hops"] for x in res), "n o/g", len(orc["id"]), len(parts["id"]),
          "only-o", sorted(so - sg)[:4], "only-g", sorted(sg - so)[:4], "badcell", badc[:4], "badpos", badx[:4],
          "mig", [x["n_migrated_out"] for x in res], "rounds?", [x["max_hops"] for x in res])
    for i in list(badc[:2]) + list(badx[:2]):
        k = np.searchsorted(orc["id"], i); q = np.searchsorted(parts["id"], i)
        print("   id", i, "oracle cell", orc["cell"][k], orc["pos"][k], "gpu cell", parts["cell"][q], parts["pos"][q], "owner", roc[orc["cell"][k]], roc[parts["cell"][q]])
    if len(badc) or len(badx) or (so ^ sg):
        break
