"""CUDA path vs the CPU oracle, element by element (-m gpu).

Config C1 (6x6x30 Kuhn duct, jittered; 100k particles + 1k injected per
step; random per-cell field) in every deposit mode, MH and DH, H_pass in
{1, 8}; plus edge cases (empty set, ragged sizes, everything removed, hop
cap, capacity growth).  All calls go through the C ABI (libopp.so).
"""
import numpy as np
import pytest

import gen
from parity_util import NEAR, c1_case, compare, run_oracle

pytestmark = pytest.mark.gpu

C1, DT, W = 0.5, 1.0, 1.0      # c1 = qm*dt with qm = 0.5, dt = 1


def _gpu_run(mesh, ef, init, inject, steps, qm=C1, dt=DT, w=W, **kw):
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    shuffle_every = kw.pop("shuffle_every", 0)
    sim = MiniFemPic(mesh, ef, **kw)
    if init is not None and init["cell"].shape[0]:
        sim.inject(init)
    stats = []
    for s in range(steps):
        b = inject(s) if inject else None
        if b is not None:
            sim.inject(b)
        stats.append(sim.step(dt, qm, w))
        if shuffle_every and (s + 1) % shuffle_every == 0:
            sim.shuffle(1000 + s)
    out = sim.particles()
    Q = sim.node_charge_host()
    launches = sim.launches()
    sim.close()
    return out, Q, stats, launches


def _check(mesh, ef, init, inject, steps, hcap=1024, dh=False, **kw):
    overlay = None
    if dh:
        box = mesh["box"]
        dx = kw.get("overlay_spacing", 0.5)
        n = [int(np.ceil((box[2 * k + 1] - box[2 * k]) / dx)) for k in range(3)]
        overlay = ([box[0], box[2], box[4]], dx, n)
    om, orc, Qo, ost, rem = run_oracle(mesh, ef, init, inject, steps, C1 * DT, DT, W,
                                       hcap=hcap, use_dh=dh, overlay=overlay)
    gout, Qg, gst, launches = _gpu_run(mesh, ef, init, inject, steps, hop_cap=hcap,
                                        direct_hop=dh, **kw)
    assert launches > 0
    rep = compare(om, mesh["c2n"], orc, Qo, rem, gout, Qg, W)
    # per-step bookkeeping agrees with the oracle exactly
    for so, sg in zip(ost, gst):
        assert sg["n_before"] == so["n_before"]
        assert sg["n_removed"] == so["n_removed"]
        assert sg["n_after"] == so["n_after"]
        assert sg["n_hop_capped"] == so["n_capped"]
    return rep, ost, gst


@pytest.mark.parametrize("dep", [0, 1, 2])
@pytest.mark.parametrize("hpass", [0, 1, 8])
def test_c1_parity_mh(dep, hpass):
    mesh, ef, init, inject, steps = c1_case()
    rep, ost, gst = _check(mesh, ef, init, inject, steps, deposit_mode=dep, hop_budget=hpass)
    assert rep["n_compared"] > 90_000
    # identical arithmetic -> identical walks: hop totals match exactly
    assert [s["total_hops"] for s in gst] == [s["total_hops"] for s in ost]
    assert [s["max_hops"] for s in gst] == [s["max_hops"] for s in ost]
    if hpass <= 1:
        assert sum(s["n_deferred"] for s in gst) > 0


@pytest.mark.parametrize("dep,mode", [(0, 1), (1, 1), (0, 2), (1, 2), (2, 2)])
def test_c1_parity_dh(dep, mode):
    mesh, ef, init, inject, steps = c1_case(drift=0.6, spread=0.3)
    rep, ost, gst = _check(mesh, ef, init, inject, steps, dh=mode, deposit_mode=dep,
                           overlay_spacing=0.5)
    assert [s["total_hops"] for s in gst] == [s["total_hops"] for s in ost]


def test_c1_unjittered_uniform_field():
    mesh, ef, init, inject, steps = c1_case(jitter=0.0, efield="uniform")
    _check(mesh, ef, init, inject, steps)


def test_hop_cap_counts_match():
    mesh, ef, init, inject, steps = c1_case(n0=20_000, n_inj=0, steps=3, drift=1.5, spread=0.5)
    rep, ost, gst = _check(mesh, ef, init, inject, steps, hcap=2, hop_budget=1)
    assert sum(s["n_capped"] for s in ost) > 0


@pytest.mark.parametrize("n0", [0, 1, 31, 33, 257, 4097])
def test_ragged_and_empty(n0):
    mesh, ef, init, inject, steps = c1_case(n0=n0, n_inj=0, steps=3)
    _check(mesh, ef, init, None, steps)


def test_everything_removed():
    mesh = gen.kuhn_duct(3, 3, 4, jitter=0.1, seed=3)
    ef = np.zeros((mesh["n_cells"], 3))
    init = gen.seed_particles(mesh, 5000, 9, drift=5.0, spread=0.0)   # all leave through z = 4
    rep, ost, gst = _check(mesh, ef, init, None, 2)
    assert gst[0]["n_after"] == 0 and gst[0]["n_removed"] == 5000


def test_capacity_growth_through_injection():
    mesh, ef, init, inject, steps = c1_case(n0=3000, n_inj=2500, steps=4)
    _check(mesh, ef, init, inject, steps, capacity=1024)


def test_stale_holes_protocol():
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    mesh, ef, init, inject, steps = c1_case(n0=1000, n_inj=0, steps=1)
    sim = MiniFemPic(mesh, ef)
    sim.inject(init)
    sim.step(DT, C1, W, fill=False)
    with pytest.raises(O.OppError) as e:
        sim.particles()
    assert e.value.code == O.OPP_ERR_STATE
    with pytest.raises(O.OppError):
        sim.step(DT, C1, W)
    sim.fill_holes()
    assert sim.count() == len(sim.particles()["id"])
    sim.close()


def test_invalid_mesh_rejected():
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    mesh = gen.kuhn_duct(2, 2, 2)
    bad = dict(mesh)
    c2n = mesh["c2n"].copy()
    c2n[5, [2, 3]] = c2n[5, [3, 2]]      # inverted tet
    bad["c2n"] = c2n
    sim = MiniFemPic(bad, np.zeros((mesh["n_cells"], 3)))
    with pytest.raises(O.OppError) as e:
        sim.step(DT, C1, W)
    assert e.value.code == O.OPP_ERR_MESH
    sim.close()
    bad2 = dict(mesh)
    c2c = mesh["c2c"].copy()
    c2c[[0, 1]] = c2c[[1, 0]]
    bad2["c2c"] = c2c
    sim = MiniFemPic(bad2, np.zeros((mesh["n_cells"], 3)))
    with pytest.raises(O.OppError) as e:
        sim.step(DT, C1, W)
    assert e.value.code == O.OPP_ERR_MESH
    sim.close()


def test_conservation_and_bookkeeping_gpu_only():
    """Invariants that hold at any size (P5, P6) on a larger run."""
    mesh = gen.kuhn_duct(16, 16, 24, jitter=0.2, seed=5)
    ef = np.tile([0.0, 0.0, 1e-3], (mesh["n_cells"], 1))
    init = gen.seed_particles(mesh, 1_000_000, 5)
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    sim = MiniFemPic(mesh, ef)
    sim.inject(init)
    n = 1_000_000
    for s in range(3):
        b = gen.inject_batch(mesh, s, 5000, 5, id_base=10_000_000)
        sim.inject(b)
        st = sim.step(DT, C1, W)
        assert st["n_before"] == n + 5000
        n = n + 5000 - st["n_removed"]
        assert st["n_after"] == n == sim.count()
        Q = sim.node_charge_host()
        assert abs(Q.sum() - W * n) <= 4 * n * 2 ** -52 * W
        assert st["n_hop_capped"] == 0
    out = sim.particles()
    assert np.unique(out["id"]).size == n
    sim.close()


@pytest.mark.parametrize("dep,sort_every,axis", [(0, 1, 0), (1, 3, 0), (2, 2, 0), (1, 1, 1), (0, 2, 1)])
def test_c1_parity_with_periodic_sort(dep, sort_every, axis):
    """The periodic counting sort by cell (which also compacts) changes the
    storage order only: results keyed by id are identical (plain cell-id key
    and the locality key along the duct axis).  The sort gathers one column
    at a time into the spare of its size (column rotation)."""
    mesh, ef, init, inject, steps = c1_case()
    _check(mesh, ef, init, inject, steps, deposit_mode=dep, sort_every=sort_every,
           sort_axis=(0.0, 0.0, 1.0) if axis else (0.0, 0.0, 0.0))


@pytest.mark.parametrize("dep,sort_every,lead,axis", [(1, 2, 1.0, 1), (0, 3, 1.5, 0), (2, 2, 4.0, 1), (1, 1, 2.0, 0)])
def test_c1_parity_with_predicted_sort_key(dep, sort_every, lead, axis):
    """opp_init_params.sort_lead: the periodic sort keys each particle by the
    overlay tet of its ballistic extrapolation x + lead dt v (recorded by the
    pass before the sort).  Only the storage order changes, so every result
    keyed by id equals the oracle's (DH both sides; the key never reaches the
    walk)."""
    mesh, ef, init, inject, steps = c1_case()
    rep, ost, gst = _check(mesh, ef, init, inject, steps, deposit_mode=dep, dh=1, overlay_spacing=0.25,
                           sort_every=sort_every, sort_lead=lead,
                           sort_axis=(0.0, 0.0, 1.0) if axis else (0.0, 0.0, 0.0))
    assert [s["total_hops"] for s in gst] == [s["total_hops"] for s in ost]


def test_predicted_sort_key_orders_by_extrapolated_cell():
    """After a sort step with sort_lead > 0 the storage order is the order of
    the cells of x + lead dt v (by the overlay), not of the current cells."""
    import oracle
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    mesh, ef, init, inject, steps = c1_case(n0=50_000, n_inj=0, steps=1)
    sim = MiniFemPic(mesh, ef, direct_hop=1, overlay_spacing=0.25, sort_every=2, sort_lead=3.0)
    sim.inject(init)
    for _ in range(2):   # the second step records the key and sorts
        sim.step(DT, C1, W)
    raw = sim.particles(sort_by_id=False)
    box = mesh["box"]
    n = [int(np.ceil((box[2 * k + 1] - box[2 * k]) / 0.25)) for k in range(3)]
    x0 = np.array([box[0], box[2], box[4]])
    omap = oracle.Mesh.from_gen(mesh).build_overlay(x0, 0.25, n)   # [gx + n0 (gy + n1 gz)]
    xp = raw["pos"] + raw["vel"] * (3.0 * DT)
    t = (xp - x0) * (1.0 / 0.25)
    inside = np.all(t >= 0.0, axis=1)
    g = np.floor(np.where(inside[:, None], t, 0.0)).astype(np.int64)
    inside &= np.all(g < np.array(n), axis=1)
    g = np.where(inside[:, None], g, 0)
    key = np.where(inside, omap[g[:, 0] + n[0] * (g[:, 1] + n[1] * g[:, 2])], -1)
    key = np.where(key >= 0, key, raw["cell"])
    assert np.all(np.diff(key) >= 0)
    assert np.any(key != raw["cell"])
    sim.close()


def test_sort_by_cell_orders_and_preserves():
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    mesh, ef, init, inject, steps = c1_case(n0=50_000, n_inj=0, steps=1)
    sim = MiniFemPic(mesh, ef)
    sim.inject(init)
    sim.step(DT, C1, W)                       # builds the mesh data
    before = sim.particles()
    sim.sort_by_cell()
    raw = sim.particles(sort_by_id=False)
    assert np.all(np.diff(raw["cell"]) >= 0)  # sorted by cell
    after = {k: v[np.argsort(raw["id"], kind="stable")] for k, v in raw.items()}
    for k in ("pos", "vel", "cell", "id"):
        np.testing.assert_array_equal(before[k], after[k])
    # sort with holes pending == compaction
    sim.step(DT, C1, W, fill=False)
    st = sim.last_stats()
    sim.sort_by_cell()
    raw = sim.particles(sort_by_id=False)
    assert raw["id"].size == st["n_after"] and np.all(np.diff(raw["cell"]) >= 0)
    with pytest.raises(O.OppError):
        O.opp_sort_by_cell(sim.ctx, sim.cells)   # not a particle set
    sim.close()


@pytest.mark.parametrize("dep", [0, 1])
def test_c1_parity_direct_loads(dep):
    """The non-TMA (direct-load) variant of the fused kernel."""
    mesh, ef, init, inject, steps = c1_case()
    rep, ost, gst = _check(mesh, ef, init, inject, steps, deposit_mode=dep, tma_pipeline=False)
    assert [s["total_hops"] for s in gst] == [s["total_hops"] for s in ost]


@pytest.mark.parametrize("dep,dh,sort_every", [(0, 1, 3), (1, 1, 2), (1, 0, 5), (1, 2, 5)])
def test_every_particle_inside_its_cell_many_steps(dep, dh, sort_every):
    """Consistency at a larger size over many steps with periodic sorts and
    injection: every stored (cell, position) pair satisfies the point-in-tet
    test (up to rounding), charge is conserved and hop counts stay bounded."""
    import oracle
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    mesh = gen.kuhn_duct(16, 16, 24, jitter=0.2, seed=9)
    ef = np.tile([0.0, 0.0, 1e-3], (mesh["n_cells"], 1))
    sim = MiniFemPic(mesh, ef, deposit_mode=dep, direct_hop=dh, overlay_spacing=0.25,
                     sort_every=sort_every, sort_axis=(0.0, 0.0, 1.0))
    sim.inject(gen.seed_particles(mesh, 600_000, 9))
    g, p0, _ = oracle.Mesh.from_gen(mesh).geometry()
    for s in range(12):
        sim.inject(gen.inject_batch(mesh, s, 20_000, 9, id_base=10_000_000))
        st = sim.step(1.0, 1.0, 1.0)
        assert st["max_hops"] <= 12, st
        Q = sim.node_charge_host()
        assert abs(Q.sum() - st["n_after"]) <= 1e-9 * st["n_after"]
    out = sim.particles()
    c = out["cell"]
    d = out["pos"] - p0[c]
    G = g[c].reshape(-1, 3, 3)
    l123 = np.einsum("nij,nj->ni", G, d)
    lam = np.concatenate([1.0 - l123.sum(1, keepdims=True), l123], 1)
    assert lam.min() >= -1e-9 and lam.max() <= 1 + 1e-9
    sim.close()


@pytest.mark.parametrize("dep,shuffle_every", [(1, 1), (0, 2), (2, 1)])
def test_c1_parity_with_periodic_shuffle(dep, shuffle_every):
    """opp_shuffle (the paper's periodic shuffling) between
    steps permutes storage only: compared by id, results equal the oracle's."""
    mesh, ef, init, inject, steps = c1_case()
    rep, ost, gst = _check(mesh, ef, init, inject, steps, deposit_mode=dep,
                           shuffle_every=shuffle_every)
    assert rep["n_compared"] > 90_000


def test_shuffle_permutes_and_preserves():
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    mesh, ef, init, inject, steps = c1_case()
    sim = MiniFemPic(mesh, ef)
    sim.inject(init)
    sim.step(DT, C1, W)
    before = sim.particles()
    sim.shuffle(7)
    raw = sim.particles(sort_by_id=False)
    after = sim.particles()
    for k in before:
        assert np.array_equal(before[k], after[k])
    # storage order is no longer the id order nor cell-sorted
    assert not np.all(np.diff(raw["id"]) > 0)
    assert not np.all(np.diff(raw["cell"]) >= 0)
    sim.close()


@pytest.mark.parametrize("dep,sort_every,cache", [(0, 0, 0), (1, 0, 0), (1, 2, 0), (2, 0, 0), (1, 2, 1),
                                                 (1, 0, 1)])
def test_c5_style_clustered_parity(dep, sort_every, cache):
    """C5's shape at C1 size: 90% of 100k particles in a 2x2x3-hex block
    (72 tets, ~1,250 particles per hot tet): the deposit under heavy
    same-cell contention (plain fp64 atomics, warp-aggregated with and
    without the per-warp node-charge cache, sort + segmented reduction),
    sorted and unsorted storage."""
    mesh = gen.kuhn_duct(6, 6, 30, jitter=0.2, seed=20240816)
    rng = np.random.default_rng(16)
    ef = rng.uniform(-2e-3, 2e-3, (mesh["n_cells"], 3))
    hot = gen.hot_block_cells(mesh, lo=(2, 2, 10), size=(2, 2, 3))
    init = gen.seed_particles(mesh, 100_000, 20240816, cluster=(0.9, hot))
    rep, ost, gst = _check(mesh, ef, init, None, 4, deposit_mode=dep, sort_every=sort_every,
                           deposit_cache=bool(cache))
    assert rep["n_compared"] > 95_000


def exact_geometry_case():
    """Particles whose positions are exact dyadic numbers on an unjittered
    Kuhn duct (h = 1, E = 0): after every step they sit exactly on nodes,
    edges, shared faces (box faces and the Kuhn faces x = y, y = z, x = z of a
    hex), at argmin ties (lambda_i = lambda_j < 0: moves across an edge),
    outside the box beyond faces, edges and corners (removal through them),
    or at rest (v = 0).  Both sides evaluate lambda in the same order, so even
    these decisions (inclusive inside test S1, lowest-index tie S2, removal)
    must agree exactly: compared with NO near-face exclusion."""
    import oracle
    mesh = gen.kuhn_duct(3, 3, 4)
    om = oracle.Mesh.from_gen(mesh)
    ax = [np.arange(-0.25, 3.26, 0.25)] * 2 + [np.arange(-0.25, 4.26, 0.25)]
    T = np.stack(np.meshgrid(*ax, indexing="ij"), -1).reshape(-1, 3)
    V = np.array([(0, 0, 0), (0, 0, 0.25), (0.25, 0.25, 0), (-0.25, 0.25, 0.5), (0.5, -0.25, 0.25),
                  (0.25, 0.25, 0.25), (-0.5, -0.5, -0.25)])
    pos, vel, cell = [], [], []
    for v in V:
        S = T - v
        ok = np.all((S >= 0) & (S <= [3, 3, 4]), axis=1)
        for s in S[ok]:
            c = om.locate_brute(s)
            if c >= 0:
                pos.append(s); vel.append(v); cell.append(c)
    n = len(cell)
    init = {"pos": np.array(pos), "vel": np.array(vel, dtype=np.float64),
            "cell": np.array(cell, np.int32), "id": np.arange(n, dtype=np.int64)}
    ef = np.zeros((mesh["n_cells"], 3))
    return mesh, ef, init


@pytest.mark.parametrize("dh,dep,hpass,cache", [(0, 1, 4, 0), (0, 0, 1, 0), (1, 1, 4, 0), (1, 2, 8, 0),
                                                (2, 1, 4, 0), (0, 1, 0, 0), (1, 1, 4, 1)])
def test_exact_geometry_no_exclusion(dh, dep, hpass, cache):
    mesh, ef, init = exact_geometry_case()
    assert init["cell"].size > 15_000
    overlay = None
    if dh:
        box = mesh["box"]
        n = [int(np.ceil((box[2 * k + 1] - box[2 * k]) / 0.5)) for k in range(3)]
        overlay = ([box[0], box[2], box[4]], 0.5, n)
    steps = 3
    om, orc, Qo, ost, rem = run_oracle(mesh, ef, init, None, steps, C1 * DT, DT, W, use_dh=dh,
                                       overlay=overlay)
    gout, Qg, gst, _ = _gpu_run(mesh, ef, init, None, steps, direct_hop=dh, overlay_spacing=0.5,
                                deposit_mode=dep, hop_budget=hpass, deposit_cache=bool(cache))
    rep = compare(om, mesh["c2n"], orc, Qo, rem, gout, Qg, W, near=None)
    assert rep["n_excluded"] == 0 and rep["n_compared"] > 10_000
    for so, sg in zip(ost, gst):
        assert (sg["n_removed"], sg["n_after"]) == (so["n_removed"], so["n_after"])
    # the cases are really there: particles end on box faces and at rest, and
    # particles leave through the box edges / corners
    assert sum(so["n_removed"] for so in ost) > 1000
    on_face = np.any((gout["pos"] == 0) | (gout["pos"] == 3), axis=1)
    assert on_face.sum() > 500
