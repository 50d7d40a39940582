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


@pytest.mark.parametrize("R", [2, 3])
def test_loopback_dh_cell_slots_predicted_sort(R):
    """Slabs with DH seeding (each rank's overlay over its own slab), the
    warp-aggregated deposit into per-cell node slots gathered before the
    halo, and the periodic sort keyed at the predicted cell (sort_lead; the
    recorded keys of migrants fall back to their cell): the merged result
    equals the single-domain oracle (multi-hop walk there: same final cells,
    pin P7; near-face particles excluded as everywhere)."""
    mesh, ef, init, inject, steps = c1_case(drift=0.4, spread=0.1)
    om, orc, Qo, ost, rem = run_oracle(mesh, ef, init, inject, steps, QM * DT, DT, W)
    parts, Qg, stats = _run_ranks(mesh, ef, init, inject, steps, R, deposit_mode=1, direct_hop=1,
                                  overlay_spacing=0.25, sort_every=2, sort_lead=1.5,
                                  sort_axis=(0.0, 0.0, 1.0))
    compare(om, mesh["c2n"], orc, Qo, rem, parts, Qg, W)
    for s in range(steps):
        assert sum(st[s]["n_after"] for st in stats) == ost[s]["n_after"]
        assert sum(st[s]["n_removed"] for st in stats) == ost[s]["n_removed"]
    assert sum(st[s]["n_migrated_out"] for st in stats for s in range(steps)) > 1000


@pytest.mark.parametrize("R", [2, 3])
def test_loopback_field_solve_equals_single_domain(R):
    """Slab-partitioned CG (host-driven, node halo + cross-rank dots) on R
    contexts: the merged potential equals the single-domain direct solve
    within the CG bound, interface copies agree, and each rank's cell field
    is -grad(phi) of its potential."""
    import torch
    from oracle import field as F
    from paper_conf_icpp_lantra0m24_b200 import dist
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    mesh = gen.kuhn_duct(5, 4, 12, jitter=0.15, seed=8)
    rng = np.random.default_rng(3)
    Qg = rng.uniform(0.0, 4.0, mesh["n_nodes"])
    mask, val = gen.duct_bc(mesh, wall=0.03, inlet=0.0)
    rhs_scale, tol = 0.01, 1e-12
    K = F.stiffness(mesh["node_xyz"], mesh["c2n"])
    phi_ref = F.solve(K, F.load_vector(Qg, rhs_scale), mask, val)
    uid = os.urandom(128)
    streams = [torch.cuda.Stream() for _ in range(R)]
    out, errs = [None] * R, []

    def worker(r):
        try:
            sl = dist.slab(mesh, R, r)
            sim = MiniFemPic(sl, np.zeros((sl["n_cells"], 3)), nranks=R, rank=r, uid=uid,
                             transport=1, torch_alloc=False, stream=streams[r].cuda_stream)
            gid = sl["node_gid"]
            sim.field_init(mask[gid], val[gid])
            O.opp_set_dat(sim.ctx, sim.node_charge, np.ascontiguousarray(Qg[gid]), sim.nn)
            st = sim.field_solve(rhs_scale, tol=tol, warm_start=False)
            out[r] = (gid, sim.potential_host(), sim.field_host(), st, sl)
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
    phi = np.full(mesh["n_nodes"], np.nan)
    its = {o[3]["iterations"] for o in out}
    assert len(its) == 1 and all(o[3]["converged"] == 1 for o in out)   # one global CG
    for gid, ph, E, st, sl in out:
        seen = ~np.isnan(phi[gid])
        np.testing.assert_array_equal(phi[gid][seen], ph[seen])     # interface copies agree
        phi[gid] = ph
        Eo = F.efield(sl["node_xyz"], sl["c2n"], ph)
        np.testing.assert_allclose(E, Eo, rtol=0, atol=1e-13 * max(np.abs(Eo).max(), 1e-3))
    assert not np.isnan(phi).any()
    free = mask == 0
    lam_min = np.linalg.eigvalsh(K[free][:, free].toarray())[0]
    b = F.load_vector(Qg, rhs_scale)
    rhs = b[free] - K[free][:, ~free] @ val[~free]
    assert np.linalg.norm(phi - phi_ref) <= 2 * tol * np.linalg.norm(rhs) / lam_min + 1e-14


@pytest.mark.parametrize("R", [2, 3])
def test_loopback_boltzmann_equals_single_domain(R):
    """Boltzmann-electron Newton solve on R slabs (halo-completed K phi and
    lumped mass, electron diagonal on the owning copy, cross-rank norms, the
    slab CG per Newton step): the merged potential equals the single-domain
    Newton oracle, interface copies agree, one global Newton iteration."""
    import torch
    from oracle import boltzmann as B
    from oracle import field as F
    from paper_conf_icpp_lantra0m24_b200 import dist
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    mesh = gen.kuhn_duct(5, 4, 12, jitter=0.15, seed=8)
    Qg = np.random.default_rng(3).uniform(0.0, 2.0, mesh["n_nodes"])
    mask, val = gen.duct_bc(mesh, wall=3.0, inlet=0.0)
    prm = (0.5, 0.8, 0.0, 1.5)                  # rhs_scale, ne_coef, phi0, te
    K = F.stiffness(mesh["node_xyz"], mesh["c2n"])
    M = B.lumped_mass(mesh["node_xyz"], mesh["c2n"])
    phi_o, k_o, hist = B.newton(K, Qg, M, mask, val, *prm, tol=1e-10)
    uid = os.urandom(128)
    streams = [torch.cuda.Stream() for _ in range(R)]
    out, errs = [None] * R, []

    def worker(r):
        try:
            sl = dist.slab(mesh, R, r)
            sim = MiniFemPic(sl, np.zeros((sl["n_cells"], 3)), nranks=R, rank=r, uid=uid,
                             transport=1, torch_alloc=False, stream=streams[r].cuda_stream)
            gid = sl["node_gid"]
            sim.field_init(mask[gid], val[gid])
            O.opp_set_dat(sim.ctx, sim.node_charge, np.ascontiguousarray(Qg[gid]), sim.nn)
            st = sim.field_solve_boltzmann(*prm, newton_tol=1e-10, cg_tol=1e-13)
            out[r] = (gid, sim.potential_host(), st)
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
    steps = {o[2]["newton_steps"] for o in out}
    assert len(steps) == 1 and all(o[2]["converged"] == 1 for o in out)
    assert abs(steps.pop() - k_o) <= 1
    for o in out:
        assert o[2]["ref_norm"] == pytest.approx(hist[0], rel=1e-12)
    phi = np.full(mesh["n_nodes"], np.nan)
    for gid, ph, st in out:
        seen = ~np.isnan(phi[gid])
        np.testing.assert_array_equal(phi[gid][seen], ph[seen])     # interface copies agree
        phi[gid] = ph
    assert not np.isnan(phi).any()
    assert np.abs(phi - phi_o).max() <= 1e-8 * np.abs(phi_o).max()
