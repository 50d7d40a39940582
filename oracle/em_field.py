"""CPU oracle of the CabanaPIC-style field side -- TEST INFRASTRUCTURE.

AccumulateCurrent, AdvanceB and AdvanceE of the electromagnetic loop
("the accumulator data is processed in the
AccumulateCurrent routine to obtain the current density necessary for field
solving.  Field solving follows a kernel based leap-frog approach, with
AdvanceE and AdvanceB being the key subroutines"), on the periodic hex grid of
config C3 in normalised units (c = 1, eps0 = 1).  Readings (DESIGN.md §10,
E10-E12): Yee staggering matching the interpolator's layout -- E_a on the
cell's edge along a at the (-,-) corner of its transverse offsets, B_a on its
face at offset -1 along a; J_a on the same edges as E_a:

    J_a(edge) = (sum of the 4 adjacent cells' accumulator entries) / (2 dt h_b h_c)

which makes the discrete continuity equation exact for the Whitney deposit
(node charge density rho_n = sum_p Q_p W0_n(x_p) / (h_x h_y h_z)); the
leap-frog B(dt/2) -> E(dt) -> B(dt/2) with
    dB/dt = -curl E,   dE/dt = curl B - J.
Plain numpy with periodic rolls over the (k, j, i) grid; pinned by
tests/test_oracle_em_field.py (div B = 0, Gauss's law preserved with moving
particles, the Yee dispersion relation of a vacuum plane wave).
"""
from __future__ import annotations

import numpy as np


def _g(a, nx, ny, nz):
    """[nc] cell-major (i fastest) -> [nz, ny, nx]."""
    return a.reshape(nz, ny, nx)


def _sh(f, di=0, dj=0, dk=0):
    """f at (i + di, j + dj, k + dk), periodic."""
    return np.roll(f, shift=(-dk, -dj, -di), axis=(0, 1, 2))


def accumulate_current(acc, nx, ny, nz, h, dt):
    """acc[nc][12] (jx[4], jy[4], jz[4] per cell, edge order (-,-), (+,-),
    (-,+), (+,+) over the transverse offsets ((a+1)%3, (a+2)%3)) -> J[3][nc]
    on the E edges."""
    A = np.asarray(acc, dtype=np.float64).reshape(nz, ny, nx, 12)
    J = np.zeros((3, nz, ny, nx))
    hx, hy, hz = h
    # x edges (i+1/2, j, k): corners of cells (i, j-sb, k-sc) for (sb, sc) over (y, z)
    for k_, (sb, sc) in enumerate(((0, 0), (1, 0), (0, 1), (1, 1))):
        J[0] += _sh(A[..., 0 + k_], 0, -sb, -sc)
        J[1] += _sh(A[..., 4 + k_], -sc, 0, -sb)      # y edges: transverse (z, x)
        J[2] += _sh(A[..., 8 + k_], -sb, -sc, 0)      # z edges: transverse (x, y)
    J[0] /= 2.0 * dt * hy * hz
    J[1] /= 2.0 * dt * hz * hx
    J[2] /= 2.0 * dt * hx * hy
    return J.reshape(3, -1)


def curl_e(e, nx, ny, nz, h):
    """curl E on the B faces: (curl E)_x at (i, j+1/2, k+1/2) etc."""
    ex, ey, ez = (_g(e[a], nx, ny, nz) for a in range(3))
    hx, hy, hz = h
    cx = (_sh(ez, 0, 1, 0) - ez) / hy - (_sh(ey, 0, 0, 1) - ey) / hz
    cy = (_sh(ex, 0, 0, 1) - ex) / hz - (_sh(ez, 1, 0, 0) - ez) / hx
    cz = (_sh(ey, 1, 0, 0) - ey) / hx - (_sh(ex, 0, 1, 0) - ex) / hy
    return np.stack([cx, cy, cz]).reshape(3, -1)


def curl_b(b, nx, ny, nz, h):
    """curl B on the E edges: (curl B)_x at (i+1/2, j, k) etc."""
    bx, by, bz = (_g(b[a], nx, ny, nz) for a in range(3))
    hx, hy, hz = h
    cx = (bz - _sh(bz, 0, -1, 0)) / hy - (by - _sh(by, 0, 0, -1)) / hz
    cy = (bx - _sh(bx, 0, 0, -1)) / hz - (bz - _sh(bz, -1, 0, 0)) / hx
    cz = (by - _sh(by, -1, 0, 0)) / hx - (bx - _sh(bx, 0, -1, 0)) / hy
    return np.stack([cx, cy, cz]).reshape(3, -1)


def advance_b(e, b, nx, ny, nz, h, frac_dt):
    """AdvanceB: B -= frac_dt * curl E (in place)."""
    b -= frac_dt * curl_e(e, nx, ny, nz, h)


def advance_e(e, b, J, nx, ny, nz, h, dt):
    """AdvanceE: E += dt * (curl B - J) (in place; c = eps0 = 1)."""
    e += dt * (curl_b(b, nx, ny, nz, h) - J)


def div_b(b, nx, ny, nz, h):
    """divergence of B at cell centres."""
    bx, by, bz = (_g(b[a], nx, ny, nz) for a in range(3))
    hx, hy, hz = h
    return ((_sh(bx, 1, 0, 0) - bx) / hx + (_sh(by, 0, 1, 0) - by) / hy +
            (_sh(bz, 0, 0, 1) - bz) / hz).ravel()


def div_e(e, nx, ny, nz, h):
    """divergence of E at nodes (i, j, k) (node (i, j, k) = corner (-,-,-) of cell (i, j, k))."""
    ex, ey, ez = (_g(e[a], nx, ny, nz) for a in range(3))
    hx, hy, hz = h
    return ((ex - _sh(ex, -1, 0, 0)) / hx + (ey - _sh(ey, 0, -1, 0)) / hy +
            (ez - _sh(ez, 0, 0, -1)) / hz).ravel()


def node_charge_density(off, cell, w, qsp, nx, ny, nz, h):
    """rho at nodes: sum_p Q_p W0_n(x_p) / (h_x h_y h_z), trilinear W0."""
    rho = np.zeros((nz, ny, nx))
    c = np.asarray(cell, dtype=np.int64)
    i, j, k = c % nx, (c // nx) % ny, c // (nx * ny)
    Q = qsp * np.asarray(w)
    for sx in (0, 1):
        for sy in (0, 1):
            for sz in (0, 1):
                f = ((1 + (2 * sx - 1) * off[0]) * (1 + (2 * sy - 1) * off[1]) *
                     (1 + (2 * sz - 1) * off[2]) / 8)
                np.add.at(rho, ((k + sz) % nz, (j + sy) % ny, (i + sx) % nx), Q * f)
    return rho.ravel() / (h[0] * h[1] * h[2])
