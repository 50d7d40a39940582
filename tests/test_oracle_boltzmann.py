"""Pins for the Boltzmann-electron Newton oracle (oracle/boltzmann.py), -m "not gpu".

Each test fixes the oracle against something other than itself:
  * ne_coef = 0 reduces it to the (separately pinned) linear Poisson solve;
  * the lumped P1 mass of an unjittered Kuhn duct has closed forms (interior
    node h^3, corner (0,0,0) h^3/4, corner (X,0,0) h^3/12) and sums to the volume;
  * a quasi-neutral load is solved by the constant potential it encodes;
  * the small-amplitude sheath of a duct (Dirichlet A at the inlet, 0 at the
    outlet, uniform ion background) is the textbook Debye-screened profile
    of the 3-point scheme, A sinh((N - k) theta) / sinh(N theta) with
    cosh(theta) = 1 + h^2 / (2 lambda_D^2), lambda_D^2 = te / ne_coef;
  * the large-amplitude sheath follows the nonlinear first integral
    z(psi) = int_psi^A ds / sqrt(2 G(s)), G(s) = ne_coef te (e^{s/te} - 1 - s/te),
    computed by quadrature, with second-order convergence in h;
  * Newton converges quadratically.
A wrong exponent sign, a dropped 1/te in the Jacobian, a consistent instead
of lumped mass, a mass off by a factor, or a Dirichlet row left free fails one.
"""
import numpy as np
import pytest
from scipy import integrate

import gen
from oracle import boltzmann as B
from oracle import field as F


def _sys(nx, ny, nz, jitter=0.0, seed=0):
    m = gen.kuhn_duct(nx, ny, nz, jitter=jitter, seed=seed)
    K = F.stiffness(m["node_xyz"], m["c2n"])
    M = B.lumped_mass(m["node_xyz"], m["c2n"])
    return m, K, M


def test_lumped_mass_closed_forms():
    m, _, M = _sys(3, 4, 5)
    xyz = m["node_xyz"]
    assert np.all(M > 0)
    assert M.sum() == pytest.approx(3 * 4 * 5, rel=1e-14)
    interior = (xyz[:, 0] > 0) & (xyz[:, 0] < 3) & (xyz[:, 1] > 0) & (xyz[:, 1] < 4) \
        & (xyz[:, 2] > 0) & (xyz[:, 2] < 5)
    np.testing.assert_allclose(M[interior], 1.0, rtol=1e-14)
    assert M[0] == pytest.approx(0.25, rel=1e-14)            # (0,0,0): vertex 0 of 6 tets
    assert M[3] == pytest.approx(1.0 / 12.0, rel=1e-14)      # (X,0,0): 2 tets
    mj, _, Mj = _sys(3, 4, 5, jitter=0.2, seed=3)
    assert Mj.sum() == pytest.approx(60.0, rel=1e-13)        # jitter keeps the box


def test_zero_electron_term_is_linear_poisson():
    m, K, M = _sys(4, 3, 6, jitter=0.2, seed=5)
    rng = np.random.default_rng(2)
    Q = rng.uniform(0, 3, m["n_nodes"])
    mask, val = gen.duct_bc(m, wall=0.3, inlet=0.0)
    phi, k, hist = B.newton(K, Q, M, mask, val, 0.02, 0.0, 0.0, 1.0, tol=1e-13)
    ref = F.solve(K, F.load_vector(Q, 0.02), mask, val)
    np.testing.assert_allclose(phi, ref, rtol=0, atol=1e-12 * np.abs(ref).max())
    assert k == 1                                           # a linear problem: one exact step


def test_quasi_neutral_constant_state():
    m, K, M = _sys(4, 4, 8, jitter=0.15, seed=7)
    ne, te, phi0, phic = 3.0, 0.7, 0.2, 1.1
    Q = ne * M * np.exp((phic - phi0) / te) / 0.5          # rhs_scale 0.5
    mask, val = gen.duct_bc(m, wall=phic)
    phi, k, hist = B.newton(K, Q, M, mask, val, 0.5, ne, phi0, te, tol=1e-14, atol=1e-12)
    np.testing.assert_allclose(phi, phic, rtol=0, atol=1e-12)
    assert 2 <= k <= 20


def test_debye_sheath_small_amplitude():
    """Linear regime (A = 1e-6 te): the discrete Debye-screened profile."""
    nz, lam, te = 60, 5.0, 1.0
    m, K, M = _sys(2, 2, nz)
    ne = te / lam ** 2
    A = 1e-6 * te
    mask, val = gen.duct_bc(m, inlet=A, outlet=0.0)
    phi, k, hist = B.newton(K, ne * M, M, mask, val, 1.0, ne, 0.0, te, tol=1e-12, atol=1e-22)
    z = m["node_xyz"][:, 2]
    th = np.arccosh(1.0 + 1.0 / (2.0 * lam ** 2))
    ex = A * np.sinh((nz - z) * th) / np.sinh(nz * th)
    assert np.abs(phi - ex).max() <= 1e-5 * A
    # and the continuum screening length within the O(h^2) scheme error
    cont = A * np.sinh((nz - z) / lam) / np.sinh(nz / lam)
    assert np.abs(phi - cont).max() <= 2e-3 * A


def _sheath_position_error(lam, nz, te=2.0, amp=5.0):
    m, K, M = _sys(1, 1, nz)
    ne = te / lam ** 2
    A = amp * te
    mask, val = gen.duct_bc(m, inlet=A, outlet=0.0)
    phi, k, hist = B.newton(K, ne * M, M, mask, val, 1.0, ne, 0.0, te, tol=1e-12)
    pz = phi.reshape(nz + 1, -1)[:, 0]
    # the profile depends on z only (exactly, on the unjittered Kuhn duct)
    assert np.ptp(phi.reshape(nz + 1, -1), axis=1).max() <= 1e-12 * A
    G = lambda s: ne * te * (np.expm1(s / te) - s / te)
    sel = np.where(pz > 0.02 * A)[0]
    err = [abs(integrate.quad(lambda s: 1.0 / np.sqrt(2.0 * G(s)), pz[i], A, limit=200)[0] - i)
           for i in sel]
    return max(err) / lam, hist


def test_nonlinear_sheath_first_integral_and_quadratic_newton():
    e1, hist = _sheath_position_error(10.0, 120)
    e2, _ = _sheath_position_error(20.0, 240)
    assert e1 <= 0.02                 # node positions within 2% of lambda_D
    assert e1 / e2 >= 3.0             # second order in h / lambda_D
    # quadratic convergence once in the basin: ||F_{k+1}|| <= C ||F_k||^2
    h = np.array(hist)
    tail = [(h[i + 1] / h[i] ** 2) for i in range(len(h) - 1)
            if h[i] < 0.05 * h[0] and h[i + 1] > 1e-12 * h[0]]   # above the rounding floor
    assert tail and max(tail) <= 5.0
    assert h[-1] <= 1e-12 * h[0]


def test_warm_start_reference_is_the_cold_start():
    """Reading B4: the stopping reference is ||F(phi_cold)||, whatever the start:
    a start at the answer takes no step, a perturbed start reaches the same
    answer (to the tolerance)."""
    m, K, M = _sys(4, 4, 8, jitter=0.2, seed=4)
    Q = np.random.default_rng(6).uniform(0, 2, m["n_nodes"])
    mask, val = gen.duct_bc(m, wall=3.0, inlet=0.0)
    args = (K, Q, M, mask, val, 0.5, 0.8, 0.0, 1.5)
    phi, k, hist = B.newton(*args, tol=1e-10)
    assert k >= 3
    _, k0, _ = B.newton(*args, tol=1e-10, phi_start=phi)
    assert k0 == 0
    pert = phi + 0.05 * np.random.default_rng(7).uniform(-1, 1, phi.size)
    phi2, k2, hist2 = B.newton(*args, tol=1e-10, phi_start=pert)
    assert 1 <= k2 <= k
    assert np.abs(phi2 - phi).max() <= 1e-9 * np.abs(phi).max()
