"""Full-size parity of the C2 bench launch (-m gpu).

BASELINE.json configs[1] at its full size in the launch configuration bench.py
times (48x48x72 Kuhn duct = 995,328 tets, 50M seeded particles sorted by cell,
250k injected, direct-hop seeding with the h/8 overlay, H_pass 4,
warp-aggregated deposit, TMA pipeline, sort every 10 steps): one step, then

* a 20k-particle sample (seeded and injected ids) against the CPU oracle
  particle by particle -- the step is independent per particle given the
  field: survivor set, final cell bit-exact, position / velocity within
  1e-12 relative (near-face particles excluded and counted, S15); the oracle
  walks multi-hop (the final cell is the containing tet either way, P7);
* properties of the whole population: exact bookkeeping
  (N_after = N_before + injected - removed) and charge conservation
  (sum of node charge = w x particles deposited, Eq. 10 with sum(lambda) = 1).
"""
import numpy as np
import pytest

import gen
import oracle
from parity_util import NEAR

pytestmark = pytest.mark.gpu


def test_c2_full_size_sampled():
    torch = pytest.importorskip("torch")
    import gen.cuda as gc
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    cfg = gen.CONFIGS["c2"]
    nx, ny, nz = cfg["dims"]
    n0, n_inj, seed, dt, w, qm = cfg["n0"], cfg["n_inj"], cfg["seed"], 1.0, 1.0, 1.0
    mesh = gen.kuhn_duct(nx, ny, nz)
    rng = np.random.default_rng(5)
    ef = rng.uniform(-2e-3, 2e-3, (mesh["n_cells"], 3))      # random per-cell c1 E (R2)
    dm = gc.DeviceMesh(mesh)
    ov = 0.125
    sim = MiniFemPic(mesh, ef, capacity=int(n0 * 1.1) + 4 * n_inj,
                     stream=torch.cuda.current_stream().cuda_stream, deposit_mode=1,
                     direct_hop=1, overlay_spacing=ov, hop_budget=4, sort_every=10)
    init = gc.seed_particles(dm, n0, seed)
    sim.inject(init, on_device=True)
    del init
    sim.step(0.0, qm, w, stats=False, fill=True)      # builds the mesh data; dt = 0: no motion
    sim.sort_by_cell()
    before = sim.particles(sort_by_id=False)
    batch = gc.inject_batch(dm, 0, n_inj, seed, id_base=n0)
    bh = {k: batch[k].cpu().numpy() for k in ("pos", "vel", "cell", "id")}
    sim.inject(batch, on_device=True)
    st = sim.step(dt, qm, w, stats=True, fill=True)
    after = sim.particles(sort_by_id=False)
    Q = sim.node_charge_host()
    sim.close()

    # whole population: bookkeeping and charge conservation
    assert st["n_before"] == n0 + n_inj
    assert st["n_after"] == st["n_before"] - st["n_removed"] == after["id"].shape[0]
    assert st["n_removed"] > 0 and st["total_hops"] > 0
    assert abs(Q.sum() - w * st["n_after"]) <= 1e-9 * w * st["n_after"]
    assert np.unique(after["id"]).shape[0] == after["id"].shape[0]

    # the sample: 18k seeded + 2k injected ids, through the oracle one by one
    sid = np.union1d(rng.choice(n0, 18_000, replace=False), n0 + rng.choice(n_inj, 2_000, replace=False))
    m0 = np.isin(before["id"], sid)
    mi = np.isin(bh["id"], sid)
    om = oracle.Mesh.from_gen(mesh)
    om.set_field(ef)
    # the oracle walks multi-hop: the final cell of a particle is the unique
    # tet containing it (near-face particles excluded), so the DH seeding the
    # GPU run uses cannot change it (pin P7: DH final cells = MH final cells);
    # the oracle's brute-force overlay build is too slow for 995k tets
    P = oracle.Particles()
    P.append(before["pos"][m0], before["vel"][m0], before["cell"][m0], before["id"][m0])
    P.append(bh["pos"][mi], bh["vel"][mi], bh["cell"][mi], bh["id"][mi])
    Qs = np.zeros(mesh["n_nodes"])
    ost = oracle.step(om, P, qm * dt, dt, w, Qs, use_dh=0)
    orc = P.get()
    rid, rmg = P.removed()
    excl = set(orc["id"][orc["margin"] < NEAR].tolist()) | {i for i, m in zip(rid.tolist(), rmg.tolist())
                                                              if m < NEAR}
    mg = np.isin(after["id"], sid)
    g_ids = after["id"][mg]
    og, oo = np.argsort(g_ids), np.argsort(orc["id"])
    so, sg = set(orc["id"].tolist()), set(g_ids.tolist())
    assert not ((so ^ sg) - excl), "survivor sets differ"
    common = np.array(sorted((so & sg) - excl), dtype=np.int64)
    io = oo[np.searchsorted(orc["id"][oo], common)]
    ig = og[np.searchsorted(g_ids[og], common)]
    gc_cell = after["cell"][mg][ig]
    assert np.array_equal(orc["cell"][io], gc_cell)
    ex = np.abs(orc["pos"][io] - after["pos"][mg][ig]) / np.maximum(np.abs(orc["pos"][io]), 1.0)
    ev = np.abs(orc["vel"][io] - after["vel"][mg][ig]) / np.maximum(np.abs(orc["vel"][io]), 0.25)
    assert ex.max() <= 1e-12 and ev.max() <= 1e-12
    assert common.size > 19_000 and len(excl) <= 5
    assert ost["n_removed"] >= 0


def test_c4_full_size_sampled():
    """BASELINE.json configs[3] per GPU at full size in bench.py's default
    launch configuration (40x40x72 Kuhn slab = 691,200 tets, 1e9 seeded
    particles generated on the device in 50M chunks, sorted by the duct-axis
    locality key, 3.5M injected per step, DH h/8, H_pass 4, warp-aggregated
    deposit, TMA pipeline, sort every 10 steps keyed at x + 5 dt v): ten
    steps -- the tenth ends with the periodic sort on the predicted key --
    then a 20k-particle sample (seeded ids and ids of the first injected
    batch) against the oracle stepped ten times particle by particle (the
    steps are independent per particle given the fixed random field), with
    exact per-step bookkeeping and charge conservation over the whole
    population.  Particles are selected on the device (the population does
    not fit a host download)."""
    torch = pytest.importorskip("torch")
    if torch.cuda.get_device_properties(0).total_memory < 150e9:
        pytest.skip("needs a 180 GB B200")
    import gen.cuda as gc
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    cfg = gen.CONFIGS["c4"]
    nx, ny, nz = cfg["dims"]
    n0, n_inj, seed, dt, w, qm = cfg["n0"], cfg["n_inj"], cfg["seed"], 1.0, 1.0, 1.0
    steps = 10
    mesh = gen.kuhn_duct(nx, ny, nz)
    rng = np.random.default_rng(7)
    ef = rng.uniform(-2e-3, 2e-3, (mesh["n_cells"], 3)) + np.array([0.0, 0.0, 1e-3])
    dm = gc.DeviceMesh(mesh)
    sim = MiniFemPic(mesh, ef, capacity=int(n0 * 1.04) + 2 * n_inj + 4096,
                     stream=torch.cuda.current_stream().cuda_stream, deposit_mode=1,
                     direct_hop=1, overlay_spacing=0.125, hop_budget=4, sort_every=10,
                     sort_axis=(0.0, 0.0, 1.0), sort_lead=5.0)
    chunk = 50_000_000
    for first in range(0, n0, chunk):
        init = gc.seed_particles(dm, min(chunk, n0 - first), seed, first=first)
        sim.inject(init, on_device=True)
        del init
    sim.step(0.0, qm, w, stats=False, fill=True)      # builds the mesh data; dt = 0: no motion
    sim.sort_by_cell()
    sid = np.union1d(rng.choice(n0, 18_000, replace=False), n0 + rng.choice(n_inj, 2_000, replace=False))
    before = sim.particles_with_ids(sid)
    assert before["id"].shape[0] == 18_000
    b0 = None
    sts = []
    for s in range(steps):
        batch = gc.inject_batch(dm, s, n_inj, seed, id_base=n0)   # ids n0 + s n_inj + k (S21)
        if s == 0:
            b0 = {k: batch[k].cpu().numpy() for k in ("pos", "vel", "cell", "id")}
        sim.inject(batch, on_device=True)
        del batch
        sts.append(sim.step(dt, qm, w, stats=True, fill=True))
    after = sim.particles_with_ids(sid)
    Q = sim.node_charge_host()
    n_final = sim.count()
    sim.close()

    # whole population: bookkeeping per step and charge conservation
    n = n0
    for st in sts:
        assert st["n_before"] == n + n_inj
        n = st["n_before"] - st["n_removed"]
        assert st["n_after"] == n
    assert n_final == n
    assert abs(Q.sum() - w * n) <= 1e-9 * w * n

    # the sample through the oracle, one particle at a time (multi-hop walk:
    # the final cell is the containing tet, pin P7)
    om = oracle.Mesh.from_gen(mesh)
    om.set_field(ef)
    P = oracle.Particles()
    P.append(before["pos"], before["vel"], before["cell"], before["id"])
    mi = np.isin(b0["id"], sid)
    Qs = np.zeros(mesh["n_nodes"])
    excl = set()
    for s in range(steps):
        if s == 0:
            P.append(b0["pos"][mi], b0["vel"][mi], b0["cell"][mi], b0["id"][mi])
        oracle.step(om, P, qm * dt, dt, w, Qs, use_dh=0)
        rid, rmg = P.removed()
        excl |= {i for i, m in zip(rid.tolist(), rmg.tolist()) if m < NEAR}
    orc = P.get()
    excl |= set(orc["id"][orc["margin"] < NEAR].tolist())
    so, sg = set(orc["id"].tolist()), set(after["id"].tolist())
    assert not ((so ^ sg) - excl), "survivor sets differ"
    common = np.array(sorted((so & sg) - excl), dtype=np.int64)
    oo = np.argsort(orc["id"])
    io = oo[np.searchsorted(orc["id"][oo], common)]
    ig = np.searchsorted(after["id"], common)
    assert np.array_equal(orc["cell"][io], after["cell"][ig])
    ex = np.abs(orc["pos"][io] - after["pos"][ig]) / np.maximum(np.abs(orc["pos"][io]), 1.0)
    ev = np.abs(orc["vel"][io] - after["vel"][ig]) / np.maximum(np.abs(orc["vel"][io]), 0.25)
    assert ex.max() <= 1e-12 and ev.max() <= 1e-12
    assert common.size > 15_000 and len(excl) <= 10
