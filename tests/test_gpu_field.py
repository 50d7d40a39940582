"""CUDA field solve vs the field oracle (oracle/field.py), -m gpu.

The GPU assembles the P1 Poisson matrix, runs the persistent cooperative CG
and writes the cell field; the oracle gives the exact discrete solution
(sparse direct solve), the residual of any candidate and E = -grad(phi_h).
Tolerances follow from the CG stopping rule (F4):
||phi_gpu - phi||_2 <= ||r||_2 / lambda_min(K_FF) with ||r|| <= tol ||b_eff||.
All calls go through the C ABI (libopp.so).
"""
import numpy as np
import pytest

import gen
import oracle
from oracle import field as F
from parity_util import compare

pytestmark = pytest.mark.gpu


def _sim(mesh, ef=None, **kw):
    from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
    if ef is None:
        ef = np.zeros((mesh["n_cells"], 3))
    return MiniFemPic(mesh, ef, **kw)


def _set_charge(sim, Q):
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    O.opp_set_dat(sim.ctx, sim.node_charge, np.ascontiguousarray(Q, np.float64), sim.nn)


@pytest.mark.parametrize("slab", [0, 1])
@pytest.mark.parametrize("precond", [0, 1])
@pytest.mark.parametrize("dims,jit", [((6, 6, 30), 0.2), ((5, 3, 7), 0.1), ((1, 1, 1), 0.0)])
def test_field_solve_matches_direct_solve(dims, jit, precond, slab):
    """slab 1: the multi-rank CG (device-side coefficients, batched
    iterations) on one rank."""
    mesh = gen.kuhn_duct(*dims, jitter=jit, seed=4)
    xyz, c2n = mesh["node_xyz"], mesh["c2n"]
    rng = np.random.default_rng(1)
    Q = rng.uniform(0.0, 5.0, mesh["n_nodes"])
    mask, val = gen.duct_bc(mesh, wall=0.05, inlet=0.0)
    rhs_scale, tol = 0.01, 1e-11
    K = F.stiffness(xyz, c2n)
    b = F.load_vector(Q, rhs_scale)
    phi_ref = F.solve(K, b, mask, val)
    sim = _sim(mesh)
    sim.field_init(mask, val)
    _set_charge(sim, Q)
    st = sim.field_solve(rhs_scale, tol=tol, max_iter=5000, warm_start=False, precond=bool(precond),
                         slab_cg=bool(slab))
    phi = sim.potential_host()
    E = sim.field_host()
    launches = sim.launches()
    sim.close()
    assert launches > 0
    assert st["converged"] == 1 and st["rel_residual"] <= tol
    free = mask == 0
    np.testing.assert_array_equal(phi[~free], val[~free])
    # the true residual of the GPU answer, evaluated by the oracle's K
    assert F.residual(K, b, mask, val, phi) <= 2 * tol
    if 0 < free.sum() <= 3000:
        lam_min = np.linalg.eigvalsh(K[free][:, free].toarray())[0]
        rhs = b[free] - K[free][:, ~free] @ val[~free]
        bound = 2 * tol * np.linalg.norm(rhs) / lam_min + 1e-15
        assert np.linalg.norm(phi - phi_ref) <= bound
    # E of the GPU potential: the oracle's formula on the same phi
    Eo = F.efield(xyz, c2n, phi)
    np.testing.assert_allclose(E, Eo, rtol=0, atol=1e-13 * max(np.abs(Eo).max(), 1e-3))


def test_field_p9_linear_potential():
    """SURVEY.md §8(c) P9 on the device: phi = V z / Z, E = (0, 0, -V/Z)."""
    mesh = gen.kuhn_duct(6, 6, 30, jitter=0.2, seed=3)
    V, Z = 1.5, 30.0
    mask, val = gen.duct_bc(mesh, inlet=0.0, outlet=V)
    sim = _sim(mesh)
    sim.field_init(mask, val)
    st = sim.field_solve(1.0, tol=1e-13, max_iter=10000, warm_start=False)
    phi, E = sim.potential_host(), sim.field_host()
    sim.close()
    assert st["converged"] == 1
    np.testing.assert_allclose(phi, V * mesh["node_xyz"][:, 2] / Z, atol=1e-10)
    np.testing.assert_allclose(E, np.broadcast_to([0, 0, -V / Z], E.shape), atol=1e-10)


def test_field_warm_start_and_zero_rhs():
    mesh = gen.kuhn_duct(4, 4, 8, jitter=0.1, seed=2)
    mask, val = gen.duct_bc(mesh, wall=0.0, inlet=0.0)
    sim = _sim(mesh)
    sim.field_init(mask, val)
    st0 = sim.field_solve(1.0, tol=1e-10, warm_start=False)   # Q = 0, phi_D = 0: b_eff = 0
    assert st0["iterations"] == 0 and st0["converged"] == 1
    assert np.all(sim.potential_host() == 0.0)
    rng = np.random.default_rng(0)
    _set_charge(sim, rng.uniform(0, 1, mesh["n_nodes"]))
    st1 = sim.field_solve(0.1, tol=1e-10, warm_start=False)
    st2 = sim.field_solve(0.1, tol=1e-10, warm_start=True)    # from the solution
    sim.close()
    assert st1["iterations"] > 0 and st2["iterations"] <= 1


def test_field_solve_errors():
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    mesh = gen.kuhn_duct(2, 2, 2)
    sim = _sim(mesh)
    with pytest.raises(O.OppError) as e:
        sim.field_solve(1.0)                    # before opp_field_init
    assert e.value.code == O.OPP_ERR_STATE
    mask, val = gen.duct_bc(mesh, wall=0.0)
    sim.field_init(mask, val)
    prm = O.opp_field_params(1.0, -1.0, 10, 0, 1, 0)
    with pytest.raises(O.OppError) as e:
        O.opp_field_solve(sim.ctx, sim.node_charge, sim.node_potential, sim.cell_ef, prm)
    assert e.value.code == O.OPP_ERR_ARG
    with pytest.raises(O.OppError):             # a cell dat where a node dat belongs
        O.opp_field_solve(sim.ctx, sim.cell_ef, sim.node_potential, sim.cell_ef,
                          O.opp_field_params(1.0, 1e-8, 10, 0, 1, 0))
    sim.close()


def test_pic_loop_with_field_solve_replay():
    """The whole PIC loop (Fig. 1): field solve -> push/move/deposit, C1 mesh,
    injection from empty.  Replay mode: the oracle's
    push consumes the GPU's cell field of each step; the GPU field is checked
    against the oracle's solve of the GPU's own charge every step."""
    mesh = gen.kuhn_duct(6, 6, 30, jitter=0.2, seed=5)
    xyz, c2n = mesh["node_xyz"], mesh["c2n"]
    K = F.stiffness(xyz, c2n)
    mask, val = gen.duct_bc(mesh, wall=0.02, inlet=0.0)
    seed, n_inj, steps, qm, dt, w, rhs_scale, tol = 20240812, 2000, 8, 1.0, 1.0, 1.0, 2e-4, 1e-11
    om = oracle.Mesh.from_gen(mesh)
    P = oracle.Particles()
    Qo = np.zeros(mesh["n_nodes"])
    removed = {}
    sim = _sim(mesh)
    sim.field_init(mask, val)
    for s in range(steps):
        st = sim.field_solve(rhs_scale, tol=tol, warm_start=True)
        assert st["converged"] == 1
        phi, E = sim.potential_host(), sim.field_host()
        Qg = sim.node_charge_host()
        b = F.load_vector(Qg if s else np.zeros_like(Qg), rhs_scale)
        assert F.residual(K, b, mask, val, phi) <= 2 * tol
        np.testing.assert_allclose(E, F.efield(xyz, c2n, phi), rtol=0, atol=1e-14)
        if s:
            assert np.abs(E).max() > 0
        # v_inj not dyadic: cells whose 4 nodes all sit on a wall have E = 0
        # exactly, and 0.25 h/step would land their particles exactly on the
        # z = 1 node plane after 4 steps (a face: excluded by S15)
        batch = gen.inject_batch(mesh, s, n_inj, seed, v_inj=0.2371)
        sim.inject(batch)
        sim.step(dt, qm, w)
        om.set_field(E)                       # replay: the oracle pushes with the GPU's E
        P.append(batch["pos"], batch["vel"], batch["cell"], batch["id"])
        oracle.step(om, P, qm * dt, dt, w, Qo)
        rid, rmg = P.removed()
        for i, m in zip(rid.tolist(), rmg.tolist()):
            removed[i] = m
    gout, Qg = sim.particles(), sim.node_charge_host()
    sim.close()
    rep = compare(om, c2n, P.get(), Qo, removed, gout, Qg, w, v_ref=0.2371)
    assert rep["n_compared"] > 0.9 * n_inj * steps


def test_field_extrapolated_warm_start():
    """warm_start 2 (x0 = 2 phi_{n-1} - phi_{n-2}) changes the start only: every
    solve of a drifting charge sequence still meets the CG bound against the
    direct solve."""
    mesh = gen.kuhn_duct(6, 6, 12, jitter=0.2, seed=6)
    xyz, c2n = mesh["node_xyz"], mesh["c2n"]
    mask, val = gen.duct_bc(mesh, wall=0.05, inlet=0.0)
    K = F.stiffness(xyz, c2n)
    rng = np.random.default_rng(3)
    base, drift = rng.uniform(0, 5, mesh["n_nodes"]), rng.uniform(-1, 1, mesh["n_nodes"])
    sim = _sim(mesh)
    sim.field_init(mask, val)
    its = []
    for n in range(5):
        Q = base + 0.1 * n * drift
        _set_charge(sim, Q)
        st = sim.field_solve(0.01, tol=1e-11, max_iter=5000, warm_start=2)
        phi = sim.potential_host()
        ref = F.solve(K, F.load_vector(Q, 0.01), mask, val)
        assert st["converged"] == 1
        assert F.residual(K, F.load_vector(Q, 0.01), mask, val, phi) <= 2e-11
        assert np.abs(phi - ref).max() <= 1e-8 * np.abs(ref).max()
        its.append(st["iterations"])
    sim.close()
    # a charge drifting linearly is extrapolated exactly: the later solves start
    # at the answer (up to the previous solves' tolerance)
    assert its[-1] < its[0]
