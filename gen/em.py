"""Seeded synthetic inputs for the CabanaPIC-style electromagnetic loop (config C3).

INPUTS ONLY (no push, no move, no deposit): the periodic hex mesh declared as
an unstructured mesh through its cell-to-cell map, the two-stream particle
population and the edge / face fields the Interpolate routine turns into
per-cell interpolators.

* ``periodic_hex(nx, ny, nz)`` -- cell id = i + nx (j + ny k); c2c[c][f] for the
  faces f = -x, +x, -y, +y, -z, +z, wrapping periodically.
* ``two_stream(...)`` -- ppc particles per cell in cell-major order (the sorted
  order), offsets uniform in [-1, 1]^3, alternating beams u_z = +-v0 plus a
  per-z-plane sinusoidal perturbation (a host table, ``pert_table``) and a small
  uniform thermal spread; weight w.  Streams 10-15 of gen.u01.
* ``em_fields(...)`` -- random edge E (uniform +-e_amp) and face B (b0 z^ +
  uniform +-b_amp) on the periodic grid, stream 16-17.
The device twin (gen/gen_cuda.cu ``gen_em_two_stream``) is bit-identical.
"""
from __future__ import annotations

import numpy as np

from . import u01

STREAM_EM_OFF = 10      # 10, 11, 12: offsets x, y, z
STREAM_EM_U = 13        # 13, 14, 15: thermal u_x, u_y, u_z
STREAM_EM_E, STREAM_EM_B = 16, 17


def periodic_hex(nx: int, ny: int, nz: int) -> np.ndarray:
    i, j, k = np.meshgrid(np.arange(nx), np.arange(ny), np.arange(nz), indexing="ij")
    i, j, k = (a.transpose(2, 1, 0).ravel() for a in (i, j, k))   # cell-major: i fastest

    def cid(a, b, c):
        return (a % nx) + nx * ((b % ny) + ny * (c % nz))
    c2c = np.stack([cid(i - 1, j, k), cid(i + 1, j, k), cid(i, j - 1, k), cid(i, j + 1, k),
                    cid(i, j, k - 1), cid(i, j, k + 1)], axis=1)
    return np.ascontiguousarray(c2c.astype(np.int32))


def pert_table(nz: int, v0: float, pert: float) -> np.ndarray:
    """u_z perturbation per z-plane: pert * v0 * sin(2 pi (k + 1/2) / nz)."""
    k = np.arange(nz, dtype=np.float64)
    return pert * v0 * np.sin(2.0 * np.pi * (k + 0.5) / nz)


def two_stream(nx: int, ny: int, nz: int, ppc: int, seed: int, v0: float = 0.2,
               pert: float = 0.01, vth: float = 0.01, w: float = 1.0) -> dict:
    n = nx * ny * nz * ppc
    idx = np.arange(n, dtype=np.uint64)
    cell = (np.arange(n, dtype=np.int64) // ppc).astype(np.int32)
    off = np.stack([2.0 * u01(seed, STREAM_EM_OFF + a, idx) - 1.0 for a in range(3)])
    tab = pert_table(nz, v0, pert)
    kz = cell.astype(np.int64) // (nx * ny)
    sgn = np.where(np.arange(n) % 2 == 0, 1.0, -1.0)
    th = [vth * (2.0 * u01(seed, STREAM_EM_U + a, idx) - 1.0) for a in range(3)]
    u = np.stack([th[0], th[1], (sgn * v0 + tab[kz]) + th[2]])
    return {"off": np.ascontiguousarray(off), "u": np.ascontiguousarray(u),
            "w": np.full(n, w), "cell": cell, "n": n}


def em_fields(nx: int, ny: int, nz: int, seed: int, e_amp: float = 1e-2, b0: float = 0.5,
              b_amp: float = 1e-2):
    nc = nx * ny * nz
    idx = np.arange(3 * nc, dtype=np.uint64)
    e = (e_amp * (2.0 * u01(seed, STREAM_EM_E, idx) - 1.0)).reshape(3, nc)
    b = (b_amp * (2.0 * u01(seed, STREAM_EM_B, idx) - 1.0)).reshape(3, nc)
    b[2] += b0
    return np.ascontiguousarray(e), np.ascontiguousarray(b)
