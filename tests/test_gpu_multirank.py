"""The multi-rank path (slab partition, migration, node-charge halo) on ONE
GPU: R contexts in one process, one host thread each, joined by the
in-process loopback transport; the merged result must equal the oracle's
single-domain run (-m gpu)."""
import os
import threading

import numpy as np
import pytest

import gen
from parity_util import c1_case, compare, run_oracle

pytestmark = pytest.mark.gpu
QM, DT, W = 0.5, 1.0, 1.0


def _run_ranks(mesh, ef, init, inject, steps, R, **kw):
    import torch
    from paper_conf_icpp_lantra0m24_b200 import dist
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    uid = os.urandom(128)
    roc = dist.rank_of_cell(mesh, R)
    streams = [torch.cuda.Stream() for _ in range(R)]
    out, errs = [None] * R, []

    def worker(r):
        try:
            sl = dist.slab(mesh, R, r)
            sim = MiniFemPic(sl, dist.local_field(ef, sl), nranks=R, rank=r, uid=uid, transport=1,
                             torch_alloc=False, stream=streams[r].cuda_stream, **kw)
            if init is not None:
                sim.inject(dist.owned(init, roc, r))
            stats = []
            for s in range(steps):
                if inject is not None:
                    sim.inject(dist.owned(inject(s), roc, r))
                stats.append(sim.step(DT, QM, W))
            out[r] = (sim.particles(), sl["node_gid"], sim.node_charge_host(), stats)
            sim.close()
        except Exception as e:   # noqa: BLE001
            errs.append((r, e))
            raise

    th = [threading.Thread(target=worker, args=(r,)) for r in range(R)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=300)
    assert not errs, errs
    assert all(o is not None for o in out)
    parts = dist.merge_particles([o[0] for o in out])
    Q = dist.global_node_charge([(o[1], o[2]) for o in out], mesh["n_nodes"])
    return parts, Q, [o[3] for o in out]


@pytest.mark.parametrize("R", [2, 3])
@pytest.mark.parametrize("dep", [0, 2])
def test_loopback_slabs_equal_oracle(R, dep):
    mesh, ef, init, inject, steps = c1_case(drift=0.4, spread=0.1)
    om, orc, Qo, ost, rem = run_oracle(mesh, ef, init, inject, steps, QM * DT, DT, W)
    parts, Qg, stats = _run_ranks(mesh, ef, init, inject, steps, R, deposit_mode=dep)
    compare(om, mesh["c2n"], orc, Qo, rem, parts, Qg, W)
    for s in range(steps):
        assert sum(st[s]["n_after"] for st in stats) == ost[s]["n_after"]
        assert sum(st[s]["n_removed"] for st in stats) == ost[s]["n_removed"]
        assert sum(st[s]["n_migrated_out"] for st in stats) == sum(st[s]["n_migrated_in"] for st in stats)
    assert sum(st[s]["n_migrated_out"] for st in stats for s in range(steps)) > 1000
    # walks are split across ranks but the hop totals are the same walks
    assert sum(st[-1]["total_hops"] for st in stats) == ost[-1]["total_hops"]


def test_loopback_multi_slab_crossing_and_sort():
    """Fast particles cross more than one slab per step (several migration
    rounds); periodic sort on every rank."""
    mesh, ef, init, inject, steps = c1_case(n0=20_000, n_inj=200, steps=4, drift=9.0, spread=0.3)
    om, orc, Qo, ost, rem = run_oracle(mesh, ef, init, inject, steps, QM * DT, DT, W)
    parts, Qg, stats = _run_ranks(mesh, ef, init, inject, steps, 4, sort_every=2, deposit_mode=1)
    compare(om, mesh["c2n"], orc, Qo, rem, parts, Qg, W)
