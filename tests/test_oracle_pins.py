"""Pins for the CPU oracle (-m "not gpu").

Each test fixes part of oracle/oracle.c against something other than itself:
hand-derived closed forms (tests/golden), the Kuhn closed-form location, brute
force, barycentric identities, the ballistic and uniform-field discrete
leap-frog closed forms, exact conservation and bookkeeping (SURVEY.md §8(c)
pins P1-P7, P10).  A plausible mistake in the oracle -- a dropped term, a sign,
a transposed gradient, a wrong face index in c2c, an off-by-one in the hop
cap -- fails at least one of them.
"""
import itertools
import os

import numpy as np
import pytest

import gen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")
EPS = np.finfo(np.float64).eps


def kuhn_locate(x, nx, ny, nz, h=1.0):
    """Closed-form Kuhn location: hex = floor(x/h),
    tet = index of the permutation sorting the fractional parts descending.
    Returns (cell, f) or (-1, None) outside the box."""
    x = np.asarray(x, dtype=np.float64) / h
    if np.any(x < 0) or x[0] > nx or x[1] > ny or x[2] > nz:
        return -1, None
    ijk = np.minimum(np.floor(x).astype(int), [nx - 1, ny - 1, nz - 1])
    f = x - ijk
    perm = tuple(int(a) for a in np.argsort(-f, kind="stable"))
    t = gen.PERMS.index(perm)
    return 6 * (ijk[0] + nx * (ijk[1] + ny * ijk[2])) + t, f


def _golden():
    rows = np.loadtxt(os.path.join(GOLD, "kuhn_2x2x2.txt"))
    return rows[:, :3], rows[:, 3].astype(int), rows[:, 4:8].astype(int), rows[:, 8:12]


# ---------------------------------------------------------------- P1 barycentrics
def test_golden_kuhn_bary_and_nodes():
    mesh = gen.kuhn_duct(2, 2, 2)
    om = oracle.Mesh.from_gen(mesh)
    X, cells, nodes, lams = _golden()
    for x, c, n, l in zip(X, cells, nodes, lams):
        assert list(mesh["c2n"][c]) == list(n)          # generator pinned too
        np.testing.assert_array_equal(om.bary(c, x), l)  # exact: dyadic inputs
        st, fc, hops, lam, cap = om.walk(0, x)
        assert st == oracle.ORC_DONE and fc == c and cap == 0
        np.testing.assert_array_equal(lam, l)


def test_geometry_volume_positive_and_sums_to_box(c1_mesh_jit):
    om = oracle.Mesh.from_gen(c1_mesh_jit)
    g, p0, v6 = om.geometry()
    assert np.all(v6 > 0)
    assert abs(v6.sum() / 6.0 - 6 * 6 * 30) < 1e-9
    # gradients are dual to the edge vectors: g_i . (p_j - p0) = delta_ij
    xyz, c2n = c1_mesh_jit["node_xyz"], c1_mesh_jit["c2n"]
    E = xyz[c2n[:, 1:]] - xyz[c2n[:, :1]]                # (nc, 3 edges, 3)
    G = g.reshape(-1, 3, 3)
    D = np.einsum("nik,njk->nij", G, E)
    assert np.abs(D - np.eye(3)).max() < 1e-13
    np.testing.assert_array_equal(p0, xyz[c2n[:, 0]])


@pytest.mark.parametrize("zscale", [1.0, 20.0])
def test_bary_identities(zscale):
    """P1: sum = 1 within 4 eps, sum lambda_i p_i = x, lambda(node_j) = delta_ij,
    also far from the origin (node-relative form keeps absolute accuracy)."""
    mesh = gen.kuhn_duct(3, 3, int(30 * zscale), jitter=0.2, seed=11)
    om = oracle.Mesh.from_gen(mesh)
    rng = np.random.default_rng(1)
    xyz, c2n = mesh["node_xyz"], mesh["c2n"]
    worst_sum = worst_rec = worst_delta = 0.0
    for c in rng.integers(0, mesh["n_cells"], 400):
        P = xyz[c2n[c]]
        b = rng.dirichlet(np.ones(4))
        x = b @ P
        lam = om.bary(c, x)
        worst_sum = max(worst_sum, abs(lam.sum() - 1.0))
        worst_rec = max(worst_rec, np.abs(lam @ P - x).max() / max(np.abs(x).max(), 1.0))
        for j in range(4):
            lj = om.bary(c, P[j])
            worst_delta = max(worst_delta, np.abs(lj - np.eye(4)[j]).max())
    assert worst_sum <= 4 * EPS
    assert worst_rec <= 1e-13
    assert worst_delta <= 1e-14


# ---------------------------------------------------------------- P2 walk
def test_walk_equals_brute_force_tiny_jittered():
    mesh = gen.kuhn_duct(2, 2, 4, jitter=0.25, seed=3)
    om = oracle.Mesh.from_gen(mesh)
    rng = np.random.default_rng(2)
    n_checked = 0
    for _ in range(3000):
        start = int(rng.integers(0, mesh["n_cells"]))
        x = rng.uniform([-0.3, -0.3, -0.3], [2.3, 2.3, 4.3])
        st, fc, hops, lam, cap = om.walk(start, x)
        assert cap == 0
        outside = np.any(x < 0) or x[0] > 2 or x[1] > 2 or x[2] > 4
        if st == oracle.ORC_REMOVE:
            assert outside
            continue
        assert not outside
        if np.min(np.abs(lam)) < 1e-10:
            continue
        assert fc == om.locate_brute(x)
        n_checked += 1
    assert n_checked > 1500


def test_walk_equals_kuhn_closed_form_c1(c1_mesh):
    om = oracle.Mesh.from_gen(c1_mesh)
    rng = np.random.default_rng(3)
    for _ in range(4000):
        start = int(rng.integers(0, c1_mesh["n_cells"]))
        x = rng.uniform([-0.5, -0.5, -0.5], [6.5, 6.5, 30.5])
        st, fc, hops, lam, cap = om.walk(start, x)
        kc, f = kuhn_locate(x, 6, 6, 30)
        if kc < 0:
            assert st == oracle.ORC_REMOVE
            continue
        fs = np.sort(f)
        if min(fs[0], 1 - fs[2], fs[1] - fs[0], fs[2] - fs[1]) < 1e-10:
            continue
        assert st == oracle.ORC_DONE and fc == kc


def test_walk_brute_force_c1_jittered(c1_mesh_jit):
    om = oracle.Mesh.from_gen(c1_mesh_jit)
    rng = np.random.default_rng(4)
    for _ in range(300):
        start = int(rng.integers(0, c1_mesh_jit["n_cells"]))
        x = rng.uniform([0, 0, 0], [6, 6, 30])
        st, fc, hops, lam, cap = om.walk(start, x)
        assert st == oracle.ORC_DONE
        if np.min(np.abs(lam)) > 1e-10:
            assert fc == om.locate_brute(x)


def test_walk_hop_cap_semantics(c1_mesh):
    om = oracle.Mesh.from_gen(c1_mesh)
    x = np.array([3.3, 2.2, 20.1])
    st, fc, hops, lam, cap = om.walk(0, x, hcap=1024)
    assert st == oracle.ORC_DONE and cap == 0 and hops > 5
    st2, fc2, hops2, lam2, cap2 = om.walk(0, x, hcap=3)
    assert st2 == oracle.ORC_DONE and cap2 == 1 and hops2 == 3
    # capped cell is the cell reached after 3 hops; lambda is of that cell
    np.testing.assert_array_equal(lam2, om.bary(fc2, x))
    # resuming from (fc2, hops2) reaches the same final cell (H_pass invariance)
    st3, fc3, hops3, lam3, cap3 = om.walk(fc2, x, hcap=1024, hops0=hops2)
    assert (st3, fc3, hops3, cap3) == (st, fc, hops, 0)


def test_c2c_convention(c1_mesh_jit):
    """c2c[c][i] shares exactly the three nodes other than c2n[c][i] (S3)."""
    c2n, c2c = c1_mesh_jit["c2n"], c1_mesh_jit["c2c"]
    for c in range(0, c2n.shape[0], 7):
        for i in range(4):
            nb = c2c[c, i]
            face = set(np.delete(c2n[c], i))
            if nb < 0:
                continue
            assert face <= set(c2n[nb]) and c2n[c, i] not in set(c2n[nb])
    nb_count = (c2c >= 0).sum()
    assert nb_count + 1584 == c2c.size        # 1,584 boundary triangles (Appendix A.1)


# ---------------------------------------------------------------- P3/P4 push
def _run(mesh, parts_in, ef, c1, dt, w, steps, hcap=1024, use_dh=False, inject=None):
    om = oracle.Mesh.from_gen(mesh)
    om.set_field(ef)
    P = oracle.Particles()
    P.append(parts_in["pos"], parts_in["vel"], parts_in["cell"], parts_in["id"])
    Q = np.zeros(mesh["n_nodes"])
    stats = []
    for s in range(steps):
        if inject is not None:
            b = inject(s)
            P.append(b["pos"], b["vel"], b["cell"], b["id"])
        stats.append(oracle.step(om, P, c1, dt, w, Q, hcap=hcap, use_dh=use_dh))
    return om, P, Q, stats


def test_ballistic_zero_field(c1_mesh):
    p = gen.seed_particles(c1_mesh, 2000, seed=5, drift=0.05, spread=0.02)
    ef = np.zeros((c1_mesh["n_cells"], 3))
    n = 7
    om, P, Q, _ = _run(c1_mesh, p, ef, c1=0.7, dt=0.5, w=1.0, steps=n)
    out = P.get()
    idx = np.searchsorted(p["id"], out["id"])
    np.testing.assert_array_equal(out["vel"], p["vel"][idx])        # bit-exact
    exp = p["pos"][idx] + n * p["vel"][idx] * 0.5
    assert np.abs(out["pos"] - exp).max() <= 1e-13 * 30
    # survivors are exactly those whose closed-form trajectory stays in the box
    xe = p["pos"] + n * p["vel"] * 0.5
    inside = np.all((xe >= 0) & (xe <= [6, 6, 30]), axis=1)
    # a particle that left and came back is impossible in straight flight
    assert set(out["id"]) == set(p["id"][inside])


def test_uniform_field_leapfrog_closed_form(c1_mesh_jit):
    p = gen.seed_particles(c1_mesh_jit, 2000, seed=6, drift=0.1, spread=0.01)
    E = np.array([0.002, -0.001, 0.003])
    ef = np.tile(E, (c1_mesh_jit["n_cells"], 1))
    c1, dt, n = 0.5, 1.0, 6
    om, P, Q, _ = _run(c1_mesh_jit, p, ef, c1=c1, dt=dt, w=1.0, steps=n)
    out = P.get()
    idx = np.searchsorted(p["id"], out["id"])
    v0, x0 = p["vel"][idx], p["pos"][idx]
    vn = v0 + n * c1 * E
    xn = x0 + dt * (n * v0 + c1 * E * n * (n + 1) / 2)
    assert np.abs(out["vel"] - vn).max() <= 1e-12 * max(np.abs(vn).max(), 0.1)
    assert np.abs(out["pos"] - xn).max() <= 1e-12 * 30


# ---------------------------------------------------------------- P5 deposit
def test_single_particle_deposit_node_and_centroid(c1_mesh_jit):
    om = oracle.Mesh.from_gen(c1_mesh_jit)
    om.set_field(np.zeros((c1_mesh_jit["n_cells"], 3)))
    xyz, c2n = c1_mesh_jit["node_xyz"], c1_mesh_jit["c2n"]
    c = 1234
    cent = xyz[c2n[c]].mean(axis=0)
    P = oracle.Particles()
    P.append(cent[None], np.zeros((1, 3)), np.array([c], np.int32), np.array([0], np.int64))
    Q = np.zeros(c1_mesh_jit["n_nodes"])
    oracle.step(om, P, 0.0, 1.0, 2.0, Q)
    assert np.count_nonzero(Q) == 4
    np.testing.assert_allclose(Q[c2n[c]], 0.5, rtol=0, atol=8 * EPS)
    # exactly at an interior node: everything lands on that node
    node = c2n[c, 2]
    P2 = oracle.Particles()
    P2.append(xyz[node][None], np.zeros((1, 3)), np.array([c], np.int32), np.array([1], np.int64))
    Q2 = np.zeros_like(Q)
    oracle.step(om, P2, 0.0, 1.0, 3.0, Q2)
    assert abs(Q2[node] - 3.0) <= 1e-14 and abs(Q2.sum() - 3.0) <= 1e-14


def test_charge_conservation_and_bookkeeping(c1_mesh_jit):
    m = c1_mesh_jit
    p = gen.seed_particles(m, 20000, seed=8, drift=0.25, spread=0.05)
    rng = np.random.default_rng(9)
    ef = rng.uniform(-2e-3, 2e-3, (m["n_cells"], 3))
    inj = lambda s: gen.inject_batch(m, s, 500, seed=8, id_base=20000)
    om = oracle.Mesh.from_gen(m)
    om.set_field(ef)
    P = oracle.Particles()
    P.append(p["pos"], p["vel"], p["cell"], p["id"])
    Q = np.zeros(m["n_nodes"])
    ids = set(p["id"].tolist())
    for s in range(6):
        b = inj(s)
        n0 = len(P)
        P.append(b["pos"], b["vel"], b["cell"], b["id"])
        st = oracle.step(om, P, 1.0, 1.0, 0.5, Q)
        # P6: N_{s+1} = N_s + inj - rem ; survivors = (prev U injected) - removed
        assert st["n_before"] == n0 + 500
        assert st["n_after"] == n0 + 500 - st["n_removed"] == len(P)
        rid, _ = P.removed()
        ids = (ids | set(b["id"].tolist())) - set(rid.tolist())
        out = P.get()
        assert set(out["id"].tolist()) == ids and len(ids) == len(out["id"])
        # P5: sum Q = w * N_deposited (= survivors)
        assert abs(Q.sum() - 0.5 * st["n_after"]) <= 4 * st["n_after"] * 2 ** -52 * 0.5
        # removed <=> outside the box (exit margin aside)
        assert np.all((out["pos"] >= 0) & (out["pos"] <= [6, 6, 30]))
        # final cells are point locations
        for k in range(0, len(out["id"]), 997):
            if out["margin"][k] > 1e-10:
                assert out["cell"][k] == om.locate_brute(out["pos"][k])
    assert st["n_capped"] == 0


# ---------------------------------------------------------------- P7 direct hop
def test_overlay_matches_kuhn_closed_form():
    mesh = gen.kuhn_duct(3, 2, 4)
    om = oracle.Mesh.from_gen(mesh)
    n = np.array([6, 4, 8])
    cm = om.build_overlay([0.0, 0.0, 0.0], 0.5, n)
    for gz, gy, gx in itertools.product(range(8), range(4), range(6)):
        ctr = (np.array([gx, gy, gz]) + 0.5) * 0.5
        # all tets of the hex containing ctr (closed form: f_a >= f_b >= f_c)
        ijk = np.floor(ctr).astype(int)
        f = ctr - ijk
        hexi = ijk[0] + 3 * (ijk[1] + 2 * ijk[2])
        cands = [6 * hexi + t for t, (a, b, c) in enumerate(gen.PERMS) if f[a] >= f[b] >= f[c]]
        assert cm[gx + 6 * (gy + 4 * gz)] == min(cands)


def test_direct_hop_equals_multi_hop(c1_mesh_jit):
    m = c1_mesh_jit
    p = gen.seed_particles(m, 5000, seed=12, drift=0.6, spread=0.3)
    ef = np.zeros((m["n_cells"], 3))
    res = {}
    for dh in (0, 1, 2):
        om = oracle.Mesh.from_gen(m)
        om.set_field(ef)
        om.build_overlay([0.0, 0.0, 0.0], 0.5, [12, 12, 60])
        P = oracle.Particles()
        P.append(p["pos"], p["vel"], p["cell"], p["id"])
        Q = np.zeros(m["n_nodes"])
        st = oracle.step(om, P, 1.0, 1.0, 1.0, Q, use_dh=dh)
        res[dh] = (P.get(), Q, st)
    a = res[0][0]
    for dh in (1, 2):
        b = res[dh][0]
        np.testing.assert_array_equal(a["id"], b["id"])
        ok = np.minimum(a["margin"], b["margin"]) > 1e-10
        np.testing.assert_array_equal(a["cell"][ok], b["cell"][ok])
        assert res[dh][2]["total_hops"] < res[0][2]["total_hops"]
        np.testing.assert_allclose(res[0][1], res[dh][1], rtol=1e-12, atol=1e-12)
    # mode 2 consults the overlay only for particles that left their cell, so
    # it never takes more hops than multi-hop alone on any particle that stays
    assert res[2][2]["total_hops"] <= res[0][2]["total_hops"]


def test_direct_hop_mode2_stayers_take_no_hop(c1_mesh_jit):
    """DH mode 2 (reading S19''): a particle still inside its cell after the
    push keeps it with zero hops, even where the overlay would seed another
    tet (centre of the overlay cell in a neighbour)."""
    m = c1_mesh_jit
    g, p0, _ = oracle.Mesh.from_gen(m).geometry()
    # particles at rest at tet centroids: they stay where they are
    cells = np.arange(0, m["n_cells"], 7, dtype=np.int32)
    xyz = m["node_xyz"][m["c2n"][cells]].mean(axis=1)
    ef = np.zeros((m["n_cells"], 3))
    om = oracle.Mesh.from_gen(m)
    om.set_field(ef)
    om.build_overlay([0.0, 0.0, 0.0], 1.0, [3, 2, 15])   # coarse: seeds often wrong
    P = oracle.Particles()
    P.append(xyz, np.zeros_like(xyz), cells, np.arange(cells.size, dtype=np.int64))
    Q = np.zeros(m["n_nodes"])
    st = oracle.step(om, P, 1.0, 1.0, 1.0, Q, use_dh=2)
    assert st["total_hops"] == 0
    np.testing.assert_array_equal(P.get()["cell"], cells)
    P1 = oracle.Particles()
    P1.append(xyz, np.zeros_like(xyz), cells, np.arange(cells.size, dtype=np.int64))
    st1 = oracle.step(om, P1, 1.0, 1.0, 1.0, np.zeros(m["n_nodes"]), use_dh=1)
    assert st1["total_hops"] > 0          # mode 1 re-walks from the (coarse) seed
    np.testing.assert_array_equal(P1.get()["cell"], cells)


# ---------------------------------------------------------------- P10 injection
def test_injection_first_push(c1_mesh):
    m = c1_mesh
    b = gen.inject_batch(m, 0, 300, seed=4, v_inj=0.25)
    assert np.all(b["pos"][:, 2] == 0.0)
    for k in range(0, 300, 17):
        f = m["inlet"][m["inlet"][:, 0] == b["cell"][k]]
        assert f.shape[0] >= 1
    ef = np.zeros((m["n_cells"], 3))
    ef[:, 2] = 1e-3
    om = oracle.Mesh.from_gen(m)
    om.set_field(ef)
    P = oracle.Particles()
    P.append(b["pos"], b["vel"], b["cell"], b["id"])
    Q = np.zeros(m["n_nodes"])
    st = oracle.step(om, P, 1.0, 1.0, 1.0, Q)
    out = P.get()
    assert st["n_removed"] == 0
    vz = 0.25 + 1e-3
    np.testing.assert_array_equal(out["vel"][:, 2], vz)
    np.testing.assert_array_equal(out["pos"][:, 2], vz * 1.0)


def test_walk_tie_takes_lowest_index():
    """S2: on a tie for the most negative lambda the lowest local index wins.
    In tet 0 of hex 0 (path 0 -> e_x -> e_x+e_y -> 111) the closed-form
    coordinates of f = (0.25, 0.5, 0.75) are (1-f_x, f_x-f_y, f_y-f_z, f_z) =
    (0.75, -0.25, -0.25, 0.75): local faces 1 and 2 tie; one capped hop must cross
    face 1."""
    mesh = gen.kuhn_duct(2, 2, 2)
    om = oracle.Mesh.from_gen(mesh)
    x = np.array([0.25, 0.5, 0.75])
    lam = om.bary(0, x)
    assert lam[1] == lam[2] < 0
    st, fc, hops, lam2, cap = om.walk(0, x, hcap=1)
    assert cap == 1 and hops == 1 and fc == mesh["c2c"][0, 1]


def test_seed_generator_chunks_equal_whole():
    """gen.seed_particles(first=...) chunks reproduce the whole population
    (C4's 1e9 particles are generated in chunks on the device)."""
    import gen
    mesh = gen.kuhn_duct(3, 3, 4)
    whole = gen.seed_particles(mesh, 1000, 11, id_base=3)
    a = gen.seed_particles(mesh, 400, 11, id_base=3)
    b = gen.seed_particles(mesh, 600, 11, id_base=3, first=400)
    for k in ("pos", "vel", "cell", "id"):
        np.testing.assert_array_equal(whole[k], np.concatenate([a[k], b[k]]))
