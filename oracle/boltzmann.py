"""Boltzmann-electron field-solve oracle -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.

Plain numpy/scipy (fp64) Newton iteration for the nonlinear Poisson problem
Mini-FEM-PIC actually solves: ions are the
deposited particles, electrons follow the Boltzmann relation, so the field
solve is a Newton loop of ComputeF1Vector (the nonlinear residual),
ComputeJMatrix (its Jacobian) and a linear solve (PETSc KSP in the paper).
Only ``tests/`` and ``bench.py``'s oracle legs may import it; it shares no
code with ``paper_conf_icpp_lantra0m24_b200/csrc``.

Passages followed (PAPER.md line ranges; section / figure / equation):
  field solve is step 1 of the loop ........ 398-412 (§2, Fig. 1; Eq. 1 Gauss' law)
  FE method on unstructured meshes ......... 469-479 (§2)
  ComputeJMatrix / ComputeF1Vector + a
  linear solver (PETSc KSP) ................ 1604-1612 (§4.1.1)
  ComputeElectricField ..................... 1044-1068 (Fig. 6)
The paper names the routines, not their formulas; the readings B1-B4 of
DESIGN.md §11 fix them (normalised units):
  B1  -div(grad phi) = rhs_scale * rho_ion - ne_coef * exp((phi - phi0) / te)
  B2  P1 Galerkin with the electron term on the LUMPED mass (m_n = sum over
      the cells of node n of V_e / 4):
        F_n(phi) = (K phi)_n - rhs_scale * Q_n + ne_coef * m_n * exp((phi_n - phi0) / te)
      on free nodes; Dirichlet nodes hold their values (F_n = 0 there)
  B3  Newton: J = K + diag(ne_coef * m_n / te * exp((phi_n - phi0) / te)),
      J_FF delta_F = -F_F, delta_D = 0, phi <- phi + delta
  B4  start: phi_F = phi0 (or the caller's warm start), phi_D = dval_D;
      stop when ||F_F(phi_k)||_2 <= max(tol * ||F_F(phi_cold)||_2, atol), with
      phi_cold the cold start (phi0 on free nodes, dval_D): a reference that
      does not depend on the warm start (as the linear CG's ||b_eff||);
      or after max_newton steps.
Here each Newton step is solved exactly (sparse direct solve); the product
solves it by Jacobi-preconditioned CG to a tolerance the caller sets.

Pins (tests/test_oracle_boltzmann.py): ne_coef = 0 reduces to the pinned
linear solve; the lumped masses are positive and sum to the duct volume;
a quasi-neutral state (ion load = electron load at a constant potential) is
reproduced exactly from a distant start; the small-amplitude sheath in a duct
matches the Debye-screening closed form
phi - phi0 = A sinh((L - z)/lambda_D) / sinh(L / lambda_D), lambda_D^2 = te / ne_coef;
the large-amplitude 1-D sheath satisfies the nonlinear first integral's
monotone profile bound; Newton converges quadratically.  No function here is
"parity unpinned".
"""
from __future__ import annotations

import numpy as np
import scipy.sparse as sp
import scipy.sparse.linalg as spla

from oracle.field import cell_gradients


def lumped_mass(xyz: np.ndarray, c2n: np.ndarray) -> np.ndarray:
    """Reading B2: m_n = sum over the cells e containing node n of |V_e| / 4."""
    _, V = cell_gradients(xyz, c2n)
    m = np.zeros(xyz.shape[0])
    for i in range(4):
        np.add.at(m, c2n[:, i], np.abs(V) / 4.0)
    return m


def residual_vector(K: sp.csr_matrix, Q: np.ndarray, m: np.ndarray, phi: np.ndarray,
                    dmask: np.ndarray, rhs_scale: float, ne_coef: float, phi0: float,
                    te: float) -> np.ndarray:
    """ComputeF1Vector (reading B2): F = K phi - rhs_scale Q + ne_coef m exp((phi-phi0)/te)
    on free nodes, 0 on Dirichlet nodes."""
    F = K @ phi - rhs_scale * np.asarray(Q, np.float64) + ne_coef * m * np.exp((phi - phi0) / te)
    return np.where(np.asarray(dmask, bool), 0.0, F)


def jacobian(K: sp.csr_matrix, m: np.ndarray, phi: np.ndarray, ne_coef: float, phi0: float,
             te: float) -> sp.csr_matrix:
    """ComputeJMatrix (reading B3): J = K + diag(ne_coef m / te exp((phi-phi0)/te))."""
    return (K + sp.diags(ne_coef * m / te * np.exp((phi - phi0) / te))).tocsr()


def newton(K: sp.csr_matrix, Q: np.ndarray, m: np.ndarray, dmask: np.ndarray, dval: np.ndarray,
           rhs_scale: float, ne_coef: float, phi0: float, te: float, tol: float = 1e-10,
           max_newton: int = 50, phi_start: np.ndarray | None = None, atol: float = 0.0):
    """Newton's method, readings B3-B4, one exact linear solve per step
    (also stops once ||F_F|| <= atol).
    Returns (phi, newton_steps, [||F_F(phi_k)||_2 for k = 0..steps])."""
    D = np.asarray(dmask, bool)
    Fr = ~D
    cold = np.full(K.shape[0], float(phi0))
    cold[D] = np.asarray(dval, np.float64)[D]
    f0 = float(np.linalg.norm(residual_vector(K, Q, m, cold, D, rhs_scale, ne_coef, phi0, te)))
    phi = cold.copy() if phi_start is None else np.array(phi_start, np.float64)
    phi[D] = np.asarray(dval, np.float64)[D]
    F = residual_vector(K, Q, m, phi, D, rhs_scale, ne_coef, phi0, te)
    hist = [float(np.linalg.norm(F))]
    k = 0
    while k < max_newton and hist[-1] > max(tol * f0, atol):
        J = jacobian(K, m, phi, ne_coef, phi0, te)
        delta = np.zeros_like(phi)
        delta[Fr] = spla.spsolve(J[Fr][:, Fr].tocsc(), -F[Fr])
        phi = phi + delta
        F = residual_vector(K, Q, m, phi, D, rhs_scale, ne_coef, phi0, te)
        hist.append(float(np.linalg.norm(F)))
        k += 1
    return phi, k, hist
