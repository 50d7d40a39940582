"""Pins for the field-solve oracle (oracle/field.py), -m "not gpu".

Each test fixes the oracle against something other than itself: hand-worked
element matrices (tests/golden/ref_tet_stiffness.txt), exact identities of the
P1 Laplacian (symmetry, constants in the null space, the energy of a linear
field = |a|^2 * volume), the FEM patch test (linear Dirichlet data reproduced
exactly -- SURVEY.md §8(c) pin P9), the discrete maximum principle on the
non-obtuse Kuhn mesh (fixes the sign of K and b), scipy's sparse direct
solver within the CG error bound, and the P1 gradient reproducing nodal
differences along every edge.  A dropped volume factor, a flipped sign, a
transposed gradient, a wrong grad(lambda_0), a Dirichlet row left in the
system or a missing lift term each fail one of them.
"""
import os

import numpy as np
import pytest

import gen
from oracle import field as F

GOLD = os.path.join(os.path.dirname(__file__), "golden", "ref_tet_stiffness.txt")


def _golden_tets():
    out, cur = [], None
    for line in open(GOLD):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        if line.startswith("tet"):
            cur = [np.array(line.split()[1:], dtype=float).reshape(4, 3), []]
            out.append(cur)
        else:
            cur[1].append([float(v) for v in line.split()])
    return [(p, np.array(k)) for p, k in out]


def test_golden_element_stiffness():
    for P, K6 in _golden_tets():
        K = F.stiffness(P, np.array([[0, 1, 2, 3]], dtype=np.int32)).toarray()
        np.testing.assert_allclose(6.0 * K, K6, rtol=0, atol=1e-14)


@pytest.fixture(scope="module")
def jmesh():
    return gen.kuhn_duct(3, 4, 5, jitter=0.2, seed=11)


def test_stiffness_symmetric_and_constants_in_nullspace(jmesh):
    K = F.stiffness(jmesh["node_xyz"], jmesh["c2n"])
    scale = abs(K).max()
    assert abs(K - K.T).max() <= 1e-15 * scale
    assert np.abs(K @ np.ones(K.shape[0])).max() <= 1e-13 * scale


def test_energy_of_linear_field(jmesh):
    """u = a.x + c is in the P1 space, so u^T K u = int |grad u|^2 = |a|^2 * volume."""
    xyz = jmesh["node_xyz"]
    K = F.stiffness(xyz, jmesh["c2n"])
    vol = jmesh["nx"] * jmesh["ny"] * jmesh["nz"]
    rng = np.random.default_rng(3)
    for _ in range(3):
        a, c = rng.normal(size=3), rng.normal()
        u = xyz @ a + c
        np.testing.assert_allclose(u @ (K @ u), (a @ a) * vol, rtol=1e-12)


def test_patch_test_linear_dirichlet(jmesh):
    """Dirichlet data a.x + c on every boundary node, no charge: the discrete
    solution is the linear function at every interior node and E = -a."""
    xyz, c2n = jmesh["node_xyz"], jmesh["c2n"]
    K = F.stiffness(xyz, c2n)
    a, c = np.array([0.3, -1.1, 0.7]), 2.5
    u = xyz @ a + c
    mask, val = gen.duct_bc(jmesh, wall=u, inlet=u, outlet=u)
    phi = F.solve(K, np.zeros(len(u)), mask, val)
    np.testing.assert_allclose(phi, u, rtol=0, atol=1e-12 * np.abs(u).max())
    E = F.efield(xyz, c2n, phi)
    np.testing.assert_allclose(E, np.broadcast_to(-a, E.shape), rtol=0, atol=1e-11)


def test_p9_inlet_outlet_linear_potential():
    """Q = 0, phi = 0 at z = 0, phi = V at z = Z, Neumann
    walls => phi = V z / Z exactly in P1, E = (0, 0, -V/Z) in every cell."""
    m = gen.kuhn_duct(4, 3, 6, jitter=0.15, seed=2)
    xyz = m["node_xyz"]
    K = F.stiffness(xyz, m["c2n"])
    V, Z = 2.0, 6.0
    mask, val = gen.duct_bc(m, inlet=0.0, outlet=V)
    phi = F.solve(K, np.zeros(m["n_nodes"]), mask, val)
    np.testing.assert_allclose(phi, V * xyz[:, 2] / Z, rtol=0, atol=1e-12)
    E = F.efield(xyz, m["c2n"], phi)
    np.testing.assert_allclose(E, np.broadcast_to([0.0, 0.0, -V / Z], E.shape), atol=1e-12)
    # the same through CG
    phi2, it, rel = F.cg(K, np.zeros(m["n_nodes"]), mask, val, tol=1e-14)
    np.testing.assert_allclose(phi2, phi, atol=1e-11)


def test_maximum_principle_fixes_signs():
    """Kuhn tets are non-obtuse, so K is an M-matrix: positive charge with
    Dirichlet walls gives phi >= the wall value, strictly above it inside."""
    m = gen.kuhn_duct(4, 4, 6)
    K = F.stiffness(m["node_xyz"], m["c2n"])
    off = K - __import__("scipy.sparse", fromlist=["diags"]).diags(K.diagonal())
    assert off.max() <= 1e-15
    rng = np.random.default_rng(5)
    Q = rng.uniform(0.0, 1.0, m["n_nodes"])
    mask, val = gen.duct_bc(m, wall=0.7, inlet=0.7)
    phi = F.solve(K, F.load_vector(Q, 0.1), mask, val)
    free = mask == 0
    assert np.all(phi[free] > 0.7)
    np.testing.assert_array_equal(phi[~free], 0.7)


def test_cg_equals_direct_solve_within_error_bound(jmesh):
    """CG's ||r|| <= tol ||b|| bounds ||phi_cg - phi||_2 <= ||r||_2 / lambda_min(K_FF)."""
    xyz, c2n = jmesh["node_xyz"], jmesh["c2n"]
    K = F.stiffness(xyz, c2n)
    rng = np.random.default_rng(7)
    Q = rng.uniform(0.0, 3.0, jmesh["n_nodes"])
    mask, val = gen.duct_bc(jmesh, wall=0.05, inlet=0.0)
    b = F.load_vector(Q, 0.02)
    phi = F.solve(K, b, mask, val)
    free = mask == 0
    lam_min = np.linalg.eigvalsh(K[free][:, free].toarray())[0]
    rhs = b[free] - K[free][:, ~free] @ val[~free]
    for tol in (1e-6, 1e-10, 1e-13):
        phi_cg, it, rel = F.cg(K, b, mask, val, tol=tol)
        assert rel <= tol and it > 0
        bound = 1.01 * rel * np.linalg.norm(rhs) / lam_min + 1e-14
        assert np.linalg.norm(phi_cg - phi) <= bound
        assert F.residual(K, b, mask, val, phi_cg) <= 1.01 * tol + 1e-15
        np.testing.assert_array_equal(phi_cg[~free], val[~free])
    # warm start from the answer: zero iterations
    _, it0, _ = F.cg(K, b, mask, val, x0=phi, tol=1e-10)
    assert it0 == 0


def test_efield_reproduces_nodal_differences(jmesh):
    """For any nodal phi, E_c = -grad(phi_h) satisfies E_c . (p_j - p_i) =
    -(phi_j - phi_i) along all 6 edges of every cell (P1 interpolant)."""
    xyz, c2n = jmesh["node_xyz"], jmesh["c2n"]
    rng = np.random.default_rng(9)
    phi = rng.normal(size=jmesh["n_nodes"])
    E = F.efield(xyz, c2n, phi)
    for i in range(4):
        for j in range(i + 1, 4):
            d = xyz[c2n[:, j]] - xyz[c2n[:, i]]
            lhs = np.einsum("ck,ck->c", E, d)
            np.testing.assert_allclose(lhs, -(phi[c2n[:, j]] - phi[c2n[:, i]]), atol=1e-12)
