"""Field-solve oracle -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.

Plain numpy/scipy (fp64) implementation of the electrostatic field solve that
closes the PIC loop of Mini-FEM-PIC: the P1
finite-element Poisson system on the tetrahedral mesh, its solution, and the
cell-constant electric field the particle push reads.  Only ``tests/`` and
``bench.py``'s oracle legs may import it; it never touches the product
library and shares no code with ``paper_conf_icpp_lantra0m24_b200/csrc``.

Passages followed (PAPER.md line ranges; section / figure / equation):
  field solve is step 1 of the loop ........ 398-412 (§2, Fig. 1; Eq. 1 Gauss' law)
  FE method on unstructured meshes ......... 469-479 (§2: "the finite element (FE)
                                             method is typically used")
  ComputeJMatrix / ComputeF1Vector + linear
  solver, ComputeElectricField ............. 1604-1612 (§4.1.1), 1044-1068 (Fig. 6
                                             compute_electric_field over cells
                                             reading the 4 nodes' potential)
  outer wall at higher potential, inlet .... 1495-1500 (§4: "the outer wall is fixed
                                             at a higher potential")
Readings (F1-F5): linear Poisson  -div(grad phi) = rho/eps
(north_star: "a plain GPU conjugate-gradient on the FEM Poisson system", in
place of the paper's Boltzmann-electron Newton solve, NEXT-4, whose oracle is
oracle/boltzmann.py); the load
vector is the consistent P1 load of the deposited point charges,
b_n = rhs_scale * Q_n with Q_n = w * sum_p lambda_n(x_p) (S7); Dirichlet
nodes take given values, every other boundary is homogeneous Neumann;
E_c = -grad(phi_h) on cell c = -sum_i phi_{c2n[c][i]} grad(lambda_i).

Definitions here are written out plainly (no blocking, no fusion):
  stiffness  K_ij = sum_e V_e grad(lambda_i) . grad(lambda_j)   (P1 Laplacian)
  solve      phi_D = given, K_FF phi_F = b_F - K_FD phi_D        (direct solve)
  cg         Hestenes-Stiefel conjugate gradient on K_FF (textbook, plain)
  efield     E_c = -sum_i phi_i grad(lambda_i)

Pins: tests/test_oracle_field.py (reference-tet element matrix worked by hand
in tests/golden/ref_tet_stiffness.txt, K symmetric with constants in its
null space, energy of a linear field = |a|^2 * volume, FEM patch test
(linear Dirichlet data reproduced exactly), CG = scipy sparse direct solve
within the CG error bound, E of the P1 interpolant reproduces nodal
differences along every edge).  No function here is "parity unpinned".
"""
from __future__ import annotations

import numpy as np
import scipy.sparse as sp
import scipy.sparse.linalg as spla


def cell_gradients(xyz: np.ndarray, c2n: np.ndarray):
    """grad(lambda_i), i = 0..3, and the volume of every tet.

    With M = [p1-p0, p2-p0, p3-p0] (columns), x - p0 = M (l1, l2, l3), so the
    gradients of l1..l3 are the rows of M^-1 and grad(l0) = -(sum of them).
    Returns G (nc, 4, 3) and V (nc,)."""
    P = xyz[c2n]                                   # (nc, 4, 3)
    M = np.stack([P[:, 1] - P[:, 0], P[:, 2] - P[:, 0], P[:, 3] - P[:, 0]], axis=2)
    Minv = np.linalg.inv(M)                        # rows = grad l1, l2, l3
    G = np.empty((c2n.shape[0], 4, 3))
    G[:, 1:, :] = Minv
    G[:, 0, :] = -(Minv[:, 0, :] + Minv[:, 1, :] + Minv[:, 2, :])
    V = np.linalg.det(M) / 6.0
    return G, V


def stiffness(xyz: np.ndarray, c2n: np.ndarray) -> sp.csr_matrix:
    """Global P1 stiffness (ComputeJMatrix, linear case):
    K = sum over cells of V_e * G_e G_e^T scattered to the cell's 4 nodes."""
    G, V = cell_gradients(xyz, c2n)
    Ke = V[:, None, None] * np.einsum("cik,cjk->cij", G, G)     # (nc, 4, 4)
    rows = np.repeat(c2n, 4, axis=1).ravel()
    cols = np.tile(c2n, (1, 4)).ravel()
    nn = xyz.shape[0]
    return sp.coo_matrix((Ke.ravel(), (rows, cols)), shape=(nn, nn)).tocsr()


def load_vector(Q: np.ndarray, rhs_scale: float) -> np.ndarray:
    """ComputeF1Vector analogue (reading F2): b = rhs_scale * Q."""
    return rhs_scale * np.asarray(Q, dtype=np.float64)


def solve(K: sp.csr_matrix, b: np.ndarray, dmask: np.ndarray, dval: np.ndarray) -> np.ndarray:
    """The definition of the discrete potential: phi_D = dval_D and
    K_FF phi_F = b_F - K_FD phi_D (sparse direct solve)."""
    D = np.asarray(dmask, dtype=bool)
    F = ~D
    phi = np.where(D, dval, 0.0).astype(np.float64)
    rhs = b[F] - K[F][:, D] @ phi[D]
    phi[F] = spla.spsolve(K[F][:, F].tocsc(), rhs)
    return phi


def cg(K: sp.csr_matrix, b: np.ndarray, dmask: np.ndarray, dval: np.ndarray,
       x0: np.ndarray | None = None, tol: float = 1e-10, max_iter: int = 100000):
    """Textbook conjugate gradient (Hestenes-Stiefel) on K_FF u = b_F - K_FD phi_D,
    stopping when ||r||_2 <= tol * ||b_F - K_FD phi_D||_2.
    Returns (phi, iterations, ||r||/||rhs||)."""
    D = np.asarray(dmask, dtype=bool)
    F = ~D
    A = K[F][:, F]
    phi = np.where(D, dval, 0.0).astype(np.float64)
    rhs = b[F] - K[F][:, D] @ phi[D]
    x = np.zeros(A.shape[0]) if x0 is None else np.array(x0, dtype=np.float64)[F]
    r = rhs - A @ x
    p = r.copy()
    rr = r @ r
    nb = np.sqrt(rhs @ rhs)
    if nb == 0.0:
        nb = 1.0
    it = 0
    while np.sqrt(rr) > tol * nb and it < max_iter:
        q = A @ p
        alpha = rr / (p @ q)
        x = x + alpha * p
        r = r - alpha * q
        rr_new = r @ r
        p = r + (rr_new / rr) * p
        rr = rr_new
        it += 1
    phi[F] = x
    return phi, it, float(np.sqrt(rr) / nb)


def efield(xyz: np.ndarray, c2n: np.ndarray, phi: np.ndarray) -> np.ndarray:
    """ComputeElectricField (Fig. 6): E_c = -grad(phi_h)
    = -sum_i phi[c2n[c][i]] * grad(lambda_i) on every cell."""
    G, _ = cell_gradients(xyz, c2n)
    return -np.einsum("ci,cik->ck", phi[c2n], G)


def residual(K: sp.csr_matrix, b: np.ndarray, dmask: np.ndarray, dval: np.ndarray,
             phi: np.ndarray) -> float:
    """||b_F - K_F. phi||_2 / ||b_F - K_FD phi_D||_2 of any candidate phi with
    phi_D = dval_D (checked separately): what the CG stopping test bounds."""
    D = np.asarray(dmask, dtype=bool)
    F = ~D
    phid = np.where(D, dval, 0.0)
    rhs = b[F] - K[F][:, D] @ phid[D]
    r = b[F] - K[F] @ phi
    nb = np.linalg.norm(rhs)
    return float(np.linalg.norm(r) / (nb if nb > 0 else 1.0))
