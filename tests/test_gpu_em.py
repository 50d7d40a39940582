"""GPU parity of the CabanaPIC-style EM Move_Deposit (config C3) against the
CPU oracle (oracle/em.c), through the C ABI (opp_em_interpolate,
opp_em_move_deposit).

Bar: interpolator bit-exact; cells bit-exact; offsets and
momenta bit-exact (both sides evaluate the same operations in the same order
without FMA -- checked as <= 1e-12 relative, the north_star bound, and
reported exact); accumulators within 1e-10 of max|acc| (fp64 reduction order:
warp reduce-scatter + atomics vs sequential).  At the full C3 size the
oracle checks a sample of particles one by one (Move_Deposit is independent
per particle given the fields) and the charge-continuity identity is checked
on the whole population.
"""
import numpy as np
import pytest

import gen.em as G
import oracle.em as OE

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _app(nx, ny, nz, e, b, qdt, cdt, kcap=16, dep=1):
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    from paper_conf_icpp_lantra0m24_b200.em_app import CabanaPicEM
    return CabanaPicEM(nx, ny, nz, G.periodic_hex(nx, ny, nz), e, b, qdt, cdt, 1.0, kcap,
                       O.OPP_DEP_ATOMIC_WARPAGG if dep else O.OPP_DEP_ATOMIC)


def _inputs(nx, ny, nz, ppc, seed, shuffle, v0=0.2, vth=0.01):
    p = G.two_stream(nx, ny, nz, ppc, seed, v0=v0, vth=vth)
    if shuffle:
        perm = np.random.default_rng(seed).permutation(p["n"])
        p = {"off": np.ascontiguousarray(p["off"][:, perm]), "u": np.ascontiguousarray(p["u"][:, perm]),
             "w": p["w"][perm].copy(), "cell": p["cell"][perm].copy(), "n": p["n"]}
    return p


def _run_both(nx, ny, nz, ppc, seed, steps, qdt, cdt, kcap=16, dep=1, shuffle=False, v0=0.2,
              vth=0.01, drop=0):
    e, b = G.em_fields(nx, ny, nz, seed, e_amp=0.05, b0=0.4, b_amp=0.05)
    p = _inputs(nx, ny, nz, ppc, seed, shuffle, v0, vth)
    n = p["n"] - drop
    off, u, w, cell = (np.ascontiguousarray(p["off"][:, :n]), np.ascontiguousarray(p["u"][:, :n]),
                       p["w"][:n].copy(), p["cell"][:n].copy())
    interp = OE.interpolate(nx, ny, nz, e, b)
    c2c = G.periodic_hex(nx, ny, nz)
    acc = np.zeros((nx * ny * nz, 12))
    prm = OE.params(qdt, cdt, 1.0, kcap)
    o_off, o_u, o_cell = off.copy(), u.copy(), cell.copy()
    ost = []
    for _ in range(steps):
        ost.append(OE.move_deposit(prm, o_off, o_u, w, o_cell, interp, c2c, acc))
    sim = _app(nx, ny, nz, e, b, qdt, cdt, kcap, dep)
    assert np.array_equal(sim.interp.cpu().numpy(), interp)   # Interpolate: bit-exact
    sim.set_particles(off, u, w, cell)
    gst = [sim.step(want_stats=True) for _ in range(steps)]
    g = sim.state()
    assert sim.launches() >= steps + 1
    sim.close()
    return (o_off, o_u, o_cell, acc, ost), g, gst


def _check(o, g, gst):
    o_off, o_u, o_cell, acc, ost = o
    assert np.array_equal(g["cell"], o_cell)
    np.testing.assert_allclose(g["off"], o_off, rtol=1e-12, atol=1e-15)
    np.testing.assert_allclose(g["u"], o_u, rtol=1e-12, atol=1e-15)
    scale = max(np.abs(acc).max(), 1e-300)
    assert np.abs(g["acc"] - acc).max() <= 1e-10 * scale
    for a, b in zip(ost, gst):
        assert a["n_crossings"] == b["n_crossings"] and a["n_capped"] == b["n_capped"]
        assert a["max_crossings"] == b["max_crossings"]
    return {"exact_off": bool(np.array_equal(g["off"], o_off)), "exact_u": bool(np.array_equal(g["u"], o_u))}


@pytest.mark.parametrize("dep", [0, 1])
@pytest.mark.parametrize("shuffle", [False, True])
def test_em_parity_two_stream(dep, shuffle):
    # 6x5x7 = 210 cells, 40 ppc = 8400 particles minus a ragged tail
    o, g, gst = _run_both(6, 5, 7, 40, 20240814, 4, 0.05, [0.9, 0.8, 1.0], dep=dep,
                          shuffle=shuffle, drop=37)
    rep = _check(o, g, gst)
    assert rep["exact_off"] and rep["exact_u"]
    assert gst[-1]["n_crossings"] > 0


def test_em_parity_fast_multi_crossing():
    # streak up to ~3 offset units: several faces per step, periodic wrap in all axes
    o, g, gst = _run_both(4, 4, 5, 30, 7, 3, 0.1, [3.0, 2.5, 3.5], v0=0.6, vth=0.3)
    _check(o, g, gst)
    assert max(s["max_crossings"] for s in gst) >= 3


def test_em_parity_crossing_cap():
    o, g, gst = _run_both(4, 4, 5, 30, 8, 2, 0.1, [3.0, 2.5, 3.5], kcap=1, v0=0.6, vth=0.3)
    _check(o, g, gst)
    assert gst[0]["n_capped"] > 0


def test_em_empty_and_tiny():
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    e, b = G.em_fields(3, 3, 3, 1)
    sim = _app(3, 3, 3, e, b, 0.05, [1, 1, 1])
    sim.set_particles(np.zeros((3, 0)), np.zeros((3, 0)), np.zeros(0), np.zeros(0, np.int32))
    assert sim.step(want_stats=True)["n_crossings"] == 0
    with pytest.raises(O.OppError):
        O.opp_em_move_deposit(sim.ctx, 10, 5, sim.off, sim.u, sim.w, sim.cell, sim.interp, sim.c2c,
                              27, sim.acc, sim.params)
    sim.close()
    o, g, gst = _run_both(3, 3, 3, 1, 3, 2, 0.05, [1, 1, 1])   # 27 particles: one partial warp
    _check(o, g, gst)


def _node_weights_t(off, cell, w, nx, ny, nz):
    rho = torch.zeros(nx * ny * nz, dtype=torch.float64, device=off.device)
    c = cell.long()
    i, j, k = c % nx, (c // nx) % ny, c // (nx * ny)
    for sx in (0, 1):
        for sy in (0, 1):
            for sz in (0, 1):
                f = ((1 + (2 * sx - 1) * off[0]) * (1 + (2 * sy - 1) * off[1]) *
                     (1 + (2 * sz - 1) * off[2]) / 8)
                nid = (i + sx) % nx + nx * (((j + sy) % ny) + ny * ((k + sz) % nz))
                rho.index_add_(0, nid, w * f)
    return rho


def _divergence_t(acc, nx, ny, nz):
    out = torch.zeros(nx * ny * nz, dtype=torch.float64, device=acc.device)
    c = torch.arange(nx * ny * nz, device=acc.device)
    i, j, k = c % nx, (c // nx) % ny, c // (nx * ny)

    def kidx(sb, sc):
        return (1 if sb > 0 else 0) + (2 if sc > 0 else 0)
    for sx in (-1, 1):
        for sy in (-1, 1):
            for sz in (-1, 1):
                v = 0.5 * (sx * acc[:, kidx(sy, sz)] + sy * acc[:, 4 + kidx(sz, sx)] +
                           sz * acc[:, 8 + kidx(sx, sy)])
                nid = (i + (sx > 0)) % nx + nx * (((j + (sy > 0)) % ny) + ny * ((k + (sz > 0)) % nz))
                out.index_add_(0, nid, v)
    return out


def test_em_full_size_c3_sampled():
    """C3 at full size (40x40x60 cells, 750 ppc = 72M particles), the bench's
    launch: a 20k-particle sample against the oracle particle by particle, and
    charge continuity over the whole population."""
    import gen.cuda as GC
    from paper_conf_icpp_lantra0m24_b200.em_app import CabanaPicEM
    nx, ny, nz, ppc, seed = 40, 40, 60, 750, 20240814
    qdt, cdt = 0.05, [1.0, 1.0, 1.0]
    e, b = G.em_fields(nx, ny, nz, seed, e_amp=1e-2, b0=0.5, b_amp=1e-2)
    sim = CabanaPicEM(nx, ny, nz, G.periodic_hex(nx, ny, nz), e, b, qdt, cdt)
    d = GC.em_two_stream(nx, ny, nz, ppc, seed)
    sim.set_particles(d["off"], d["u"], d["w"], d["cell"])
    n = sim.n
    rng = np.random.default_rng(1)
    idx = np.sort(rng.choice(n, 20000, replace=False))
    ti = torch.from_numpy(idx).to(sim.dev)
    s_off = np.ascontiguousarray(sim.off[:, ti].cpu().numpy())
    s_u = np.ascontiguousarray(sim.u[:, ti].cpu().numpy())
    s_w = sim.w[ti].cpu().numpy()
    s_cell = sim.cell[ti].cpu().numpy()
    rho0 = _node_weights_t(sim.off, sim.cell, sim.w, nx, ny, nz)
    st = sim.step(want_stats=True)
    rho1 = _node_weights_t(sim.off, sim.cell, sim.w, nx, ny, nz)
    div = _divergence_t(sim.acc, nx, ny, nz)
    assert st["n_crossings"] > 0 and st["n_capped"] == 0
    err = (div - (rho1 - rho0)).abs().max().item()
    assert err <= 1e-9, err
    interp = OE.interpolate(nx, ny, nz, e, b)
    acc = np.zeros((nx * ny * nz, 12))
    OE.move_deposit(OE.params(qdt, cdt, 1.0, 16), s_off, s_u, s_w, s_cell, interp,
                    G.periodic_hex(nx, ny, nz), acc)
    assert np.array_equal(sim.cell[ti].cpu().numpy(), s_cell)
    np.testing.assert_allclose(sim.off[:, ti].cpu().numpy(), s_off, rtol=1e-12, atol=1e-15)
    np.testing.assert_allclose(sim.u[:, ti].cpu().numpy(), s_u, rtol=1e-12, atol=1e-15)
    sim.close()


def test_em_sorted_steps_parity():
    """Sort by cell before every step (opp_em_sort_by_cell): the population after
    3 steps equals the oracle's unsorted run as a set of particles (order within
    a cell is unspecified), and the accumulators agree."""
    nx, ny, nz, ppc, seed, qdt, cdt = 5, 4, 6, 30, 12, 0.05, [0.9, 0.8, 1.2]
    e, b = G.em_fields(nx, ny, nz, seed, e_amp=0.05, b0=0.4, b_amp=0.05)
    p = _inputs(nx, ny, nz, ppc, seed, True, v0=0.4, vth=0.05)
    interp = OE.interpolate(nx, ny, nz, e, b)
    c2c = G.periodic_hex(nx, ny, nz)
    acc = np.zeros((nx * ny * nz, 12))
    o_off, o_u, o_cell = p["off"].copy(), p["u"].copy(), p["cell"].copy()
    prm = OE.params(qdt, cdt, 1.0, 16)
    sim = _app(nx, ny, nz, e, b, qdt, cdt)
    sim.set_particles(p["off"], p["u"], p["w"], p["cell"])
    for _ in range(3):
        OE.move_deposit(prm, o_off, o_u, p["w"], o_cell, interp, c2c, acc)
        sim.sort_by_cell()
        assert bool((sim.cell[1:] >= sim.cell[:-1]).all())
        sim.step()
    g = sim.state()
    sim.close()

    def canon(off, u, cell):
        k = np.lexsort((u[2], off[2], off[1], off[0], cell))
        return off[:, k], u[:, k], cell[k]
    a, bb = canon(o_off, o_u, o_cell), canon(g["off"], g["u"], g["cell"])
    assert np.array_equal(a[2], bb[2])
    np.testing.assert_allclose(bb[0], a[0], rtol=1e-12, atol=1e-15)
    np.testing.assert_allclose(bb[1], a[1], rtol=1e-12, atol=1e-15)
    assert np.abs(g["acc"] - acc).max() <= 1e-10 * np.abs(acc).max()


def test_em_face_start_and_rest_edge_cases():
    """Particles starting exactly on a face and moving out (zero-length first
    segment, immediate crossing), on a face moving in, at rest (d = 0), and on
    an edge / corner (two or three faces hit at t = 0: lowest axis first)."""
    nx, ny, nz = 3, 3, 3
    e, b = G.em_fields(nx, ny, nz, 2)
    e[:] = 0.0
    b[:] = 0.0
    cases_off = [(1.0, 0.2, -0.3), (-1.0, 0.5, 0.5), (0.3, 1.0, 0.0), (0.1, 0.1, -1.0),
                 (1.0, 1.0, 0.0), (1.0, 1.0, 1.0), (-1.0, -1.0, -1.0), (0.0, 0.0, 0.0),
                 (1.0, 0.0, 0.0), (0.5, -0.5, 0.25)]
    cases_u = [(0.3, 0.0, 0.0), (-0.2, 0.1, 0.0), (0.0, 0.4, 0.1), (0.0, 0.0, -0.5),
               (0.2, 0.2, 0.0), (0.1, 0.1, 0.1), (-0.3, -0.3, -0.3), (0.0, 0.0, 0.0),
               (-0.3, 0.0, 0.0), (0.0, 0.0, 0.0)]
    n = len(cases_off)
    off = np.ascontiguousarray(np.array(cases_off).T)
    u = np.ascontiguousarray(np.array(cases_u).T)
    w = np.linspace(0.5, 1.5, n)
    cell = np.arange(n, dtype=np.int32) % (nx * ny * nz)
    interp = OE.interpolate(nx, ny, nz, e, b)
    c2c = G.periodic_hex(nx, ny, nz)
    acc = np.zeros((nx * ny * nz, 12))
    prm = OE.params(0.05, [1.0, 1.0, 1.0], 1.0, 16)
    o_off, o_u, o_cell = off.copy(), u.copy(), cell.copy()
    ost = [OE.move_deposit(prm, o_off, o_u, w, o_cell, interp, c2c, acc) for _ in range(2)]
    sim = _app(nx, ny, nz, e, b, 0.05, [1.0, 1.0, 1.0])
    sim.set_particles(off, u, w, cell)
    gst = [sim.step(want_stats=True) for _ in range(2)]
    g = sim.state()
    sim.close()
    _check((o_off, o_u, o_cell, acc, ost), g, gst)
    assert ost[0]["n_crossings"] >= 6


def test_em_field_kernels_bit_exact():
    """AccumulateCurrent / AdvanceB / AdvanceE (C ABI) equal oracle/em_field.py bit for bit."""
    import oracle.em_field as F
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    nx, ny, nz, h, dt = 5, 4, 6, (1.0, 0.8, 1.25), 0.3
    rng = np.random.default_rng(9)
    nc = nx * ny * nz
    e0, b0 = rng.uniform(-1, 1, (3, nc)), rng.uniform(-1, 1, (3, nc))
    acc = rng.uniform(-1, 1, (nc, 12))
    sim = _app(nx, ny, nz, e0, b0, 0.05, [1, 1, 1])
    dev = sim.dev
    ta = torch.from_numpy(acc).to(dev)
    J = torch.empty((3, nc), dtype=torch.float64, device=dev)
    O.opp_em_accumulate_current(sim.ctx, ta, sim.c2c, nc, h, dt, J)
    Jo = F.accumulate_current(acc, nx, ny, nz, h, dt)
    assert np.array_equal(J.cpu().numpy(), Jo)
    O.opp_em_advance_b(sim.ctx, sim.e, sim.b, sim.c2c, nc, h, dt / 2)
    eo, bo = e0.copy(), b0.copy()
    F.advance_b(eo, bo, nx, ny, nz, h, dt / 2)
    assert np.array_equal(sim.b.cpu().numpy(), bo)
    O.opp_em_advance_e(sim.ctx, sim.e, sim.b, J, sim.c2c, nc, h, dt)
    F.advance_e(eo, bo, Jo, nx, ny, nz, h, dt)
    assert np.array_equal(sim.e.cpu().numpy(), eo)
    with pytest.raises(O.OppError):
        O.opp_em_advance_e(sim.ctx, sim.e, sim.b, J, sim.c2c, nc, (1.0, 0.0, 1.0), dt)
    sim.close()


def test_em_full_pic_loop_vs_oracle():
    """Move_Deposit + AccumulateCurrent + AdvanceB/E/B + Interpolate, 4 steps,
    GPU against the oracle loop: fields within 1e-12, particles within
    1e-10 relative (the reduction order of the deposit perturbs the fields at
    the 1e-16 level and the next pushes through them)."""
    import oracle.em_field as F
    nx, ny, nz, ppc, seed = 4, 4, 5, 30, 21
    h, dt, qdt, cdt = (1.0, 1.0, 1.0), 0.5, 0.05, [1.0, 1.0, 1.0]
    e, b = G.em_fields(nx, ny, nz, seed, e_amp=0.05, b0=0.4, b_amp=0.05)
    p = _inputs(nx, ny, nz, ppc, seed, False, v0=0.4, vth=0.05)
    c2c = G.periodic_hex(nx, ny, nz)
    o_off, o_u, o_cell = p["off"].copy(), p["u"].copy(), p["cell"].copy()
    eo, bo = e.copy(), b.copy()
    prm = OE.params(qdt, cdt, 1.0, 16)
    sim = _app(nx, ny, nz, e, b, qdt, cdt)
    sim.set_particles(p["off"], p["u"], p["w"], p["cell"])
    g0 = F.div_e(eo, nx, ny, nz, h) - F.node_charge_density(o_off, o_cell, p["w"], 1.0, nx, ny, nz, h)
    for _ in range(4):
        acc = np.zeros((nx * ny * nz, 12))
        OE.move_deposit(prm, o_off, o_u, p["w"], o_cell, OE.interpolate(nx, ny, nz, eo, bo), c2c, acc)
        J = F.accumulate_current(acc, nx, ny, nz, h, dt)
        F.advance_b(eo, bo, nx, ny, nz, h, dt / 2)
        F.advance_e(eo, bo, J, nx, ny, nz, h, dt)
        F.advance_b(eo, bo, nx, ny, nz, h, dt / 2)
        sim.step()
        sim.field_step(dt, h)
    g = sim.state()
    ge, gb = sim.e.cpu().numpy(), sim.b.cpu().numpy()
    sim.close()
    np.testing.assert_allclose(ge, eo, rtol=0, atol=1e-12)
    np.testing.assert_allclose(gb, bo, rtol=0, atol=1e-12)
    assert np.array_equal(g["cell"], o_cell)
    np.testing.assert_allclose(g["off"], o_off, rtol=1e-10, atol=1e-13)
    np.testing.assert_allclose(g["u"], o_u, rtol=1e-10, atol=1e-13)
    # Gauss's law held on the GPU run too
    g1 = F.div_e(ge, nx, ny, nz, h) - F.node_charge_density(g["off"], g["cell"], p["w"], 1.0, nx, ny, nz, h)
    np.testing.assert_allclose(g1, g0, rtol=0, atol=1e-11)


def test_em_full_size_gauss_law():
    """C3 at full size through one full PIC step (Move_Deposit + field side):
    div E - rho at every node is unchanged (continuity of the Eq. 11 deposit +
    the AccumulateCurrent scale + AdvanceE), and div B stays 0."""
    import gen.cuda as GC
    from paper_conf_icpp_lantra0m24_b200.em_app import CabanaPicEM
    nx, ny, nz, ppc, seed = 40, 40, 60, 750, 20240814
    h, dt = (1.0, 1.0, 1.0), 0.5
    e, b = G.em_fields(nx, ny, nz, seed, e_amp=1e-2, b0=0.5, b_amp=1e-2)
    sim = CabanaPicEM(nx, ny, nz, G.periodic_hex(nx, ny, nz), e, b, 0.05, [1.0, 1.0, 1.0])
    d = GC.em_two_stream(nx, ny, nz, ppc, seed)
    sim.set_particles(d["off"], d["u"], d["w"], d["cell"])
    nc = nx * ny * nz

    def div_e(ev):
        E = ev.view(3, nz, ny, nx)
        return ((E[0] - torch.roll(E[0], 1, 2)) + (E[1] - torch.roll(E[1], 1, 1)) +
                (E[2] - torch.roll(E[2], 1, 0))).reshape(-1)

    def div_b(bv):
        B = bv.view(3, nz, ny, nx)
        return ((torch.roll(B[0], -1, 2) - B[0]) + (torch.roll(B[1], -1, 1) - B[1]) +
                (torch.roll(B[2], -1, 0) - B[2])).reshape(-1)
    rho0 = _node_weights_t(sim.off, sim.cell, sim.w, nx, ny, nz)
    g0 = div_e(sim.e) - rho0
    db0 = div_b(sim.b)
    sim.step()
    sim.field_step(dt, h)
    rho1 = _node_weights_t(sim.off, sim.cell, sim.w, nx, ny, nz)
    g1 = div_e(sim.e) - rho1
    assert (g1 - g0).abs().max().item() <= 1e-9
    assert (div_b(sim.b) - db0).abs().max().item() <= 1e-12
    sim.close()


def test_em_two_stream_growth_rate_gpu():
    """The cold two-stream instability through the product path (Move_Deposit +
    field side kernels, C ABI) grows at the textbook rate omega_b / 2 within
    10% -- the setup of tests/test_oracle_em_twostream.py at 4x the particles."""
    nx, ny, nz, ppc = 1, 1, 16, 4096
    h, dt, qdt = (1.0, 1.0, 1.0), 0.5, 0.05
    k = 2 * np.pi / nz
    v0 = 0.1
    wb = 2 * k * v0 / np.sqrt(3.0)
    qsp = 2 * wb ** 2 / ((2 * qdt / dt) * ppc)
    n = nz * ppc
    half = ppc // 2
    cell = np.repeat(np.arange(nz, dtype=np.int32), ppc)
    j = np.tile(np.arange(ppc), nz)
    offz = -1.0 + (2.0 * (j // 2) + 1.0) / half
    off = np.stack([np.zeros(n), np.zeros(n), offz])
    zpos = cell + (offz + 1.0) / 2.0
    u = np.zeros((3, n))
    u[2] = np.where(j % 2 == 0, 1.0, -1.0) * v0 + 1e-5 * v0 * np.sin(k * zpos)
    from paper_conf_icpp_lantra0m24_b200.em_app import CabanaPicEM
    sim = CabanaPicEM(nx, ny, nz, G.periodic_hex(nx, ny, nz), np.zeros((3, nz)), np.zeros((3, nz)),
                      qdt, [2 * dt / h[0]] * 3, qsp)
    sim.set_particles(off, u, np.ones(n), cell)
    steps, amps = 760, []
    for _ in range(steps):
        sim.step()
        sim.field_step(dt, h)
        amps.append(sim.e[2].clone())
    ez = torch.stack(amps).cpu().numpy()
    sim.close()
    a = np.abs(np.fft.rfft(ez, axis=1)[:, 1])
    t = dt * (np.arange(steps) + 1)
    gamma = np.polyfit(t[450:750], np.log(a[450:750]), 1)[0]
    assert abs(gamma - wb / 2) <= 0.10 * wb / 2, (gamma, wb / 2)
