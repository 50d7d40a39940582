"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module produces INPUTS only -- the things an OP-PIC application declares
through ``opp_decl_set/map/dat`` and hands to ``opp_inject`` (PAPER.md:846-960,
Fig. 4; injection PAPER.md:1502-1508).  It contains none of the method's
arithmetic: no barycentric coordinates, no push, no walk, no deposit, no
compaction.  Both ``oracle/`` and the product library derive everything else
(cell gradients, walk lines, overlay maps ...) on their own.

Contents
--------
* ``u01(seed, stream, idx)``  -- counter-based splitmix64 -> 53-bit double in
  [0, 1).  Transcendental-free, so a device implementation (bench's large
  configs, ``paper_conf_icpp_lantra0m24_b200/csrc/opp_gen.cu``) is
  bit-identical.  Streams follow SURVEY.md §8(d): 0 seeding cell, 1 in-tet
  point, 2 velocity, 3 injection face, 4 injection point, 5 mesh jitter.
* ``kuhn_duct`` -- an nx*ny*nz hex duct, every hex split into the 6 Kuhn tets
  (one per axis permutation).  Node numbering is x-fastest, cells are
  z-major (hex-major, then the 6 tets), so a z-slab of hexes is a contiguous
  cell range.  c2n is oriented to positive volume; c2c uses
  the convention "face i is opposite local node i, -1 = domain boundary"
  (the Fig. 4 sentinel PAPER.md:862-864).
* ``seed_particles`` / ``inject_batch`` -- initial population and per-step
  injection arrays (constant count per step, uniform point on a uniformly
  chosen inlet triangle, fixed velocity along the inward normal: S9).
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "u01", "kuhn_duct", "seed_particles", "inject_batch", "CONFIGS",
    "PERMS", "STREAM_CELL", "STREAM_POINT", "STREAM_VEL", "STREAM_FACE",
    "STREAM_INJPT", "STREAM_JITTER",
]

STREAM_CELL, STREAM_POINT, STREAM_VEL, STREAM_FACE, STREAM_INJPT, STREAM_JITTER = range(6)

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_GOLD = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)

# Kuhn permutations in itertools.permutations order.
PERMS = ((0, 1, 2), (0, 2, 1), (1, 0, 2), (1, 2, 0), (2, 0, 1), (2, 1, 0))


def _mix(z: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    z = z.astype(np.uint64, copy=True)
    z ^= z >> np.uint64(30)
    z *= _C1
    z ^= z >> np.uint64(27)
    z *= _C2
    z ^= z >> np.uint64(31)
    return z


def _key(seed: int, stream: int) -> np.uint64:
    s = (int(seed) ^ (int(stream) << 48)) & 0xFFFFFFFFFFFFFFFF
    return _mix(np.array([s], dtype=np.uint64))[0]


def u01(seed: int, stream: int, idx) -> np.ndarray:
    """Counter-based uniform in [0,1): (mix(key + (idx+1)*GOLD) >> 11) * 2^-53."""
    idx = np.asarray(idx, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = _key(seed, stream) + (idx + np.uint64(1)) * _GOLD
    return (_mix(z) >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


# ----------------------------------------------------------------------------
# Mesh
# ----------------------------------------------------------------------------

def kuhn_duct(nx: int, ny: int, nz: int, h: float = 1.0, jitter: float = 0.0,
              seed: int = 0) -> dict:
    """Kuhn-split hex duct [0,nx*h]x[0,ny*h]x[0,nz*h].

    jitter: interior nodes are displaced by U(-jitter, jitter)*h per component
    (boundary nodes stay on the box so the duct stays convex; jitter <= 0.25
    keeps every tet positive).  Multi-GPU slabs are
    contiguous cell ranges cut from one global duct (``slab``).
    """
    nnx, nny, nnz = nx + 1, ny + 1, nz + 1
    i, j, k = np.meshgrid(np.arange(nnx), np.arange(nny), np.arange(nnz), indexing="ij")
    i = i.transpose(2, 1, 0).ravel()
    j = j.transpose(2, 1, 0).ravel()
    k = k.transpose(2, 1, 0).ravel()          # node id = i + nnx*(j + nny*k)
    xyz = np.stack([i * h, j * h, k * h], axis=1).astype(np.float64)
    if jitter > 0.0:
        interior = (i > 0) & (i < nx) & (j > 0) & (j < ny) & (k > 0) & (k < nz)
        gid = (i + nnx * (j + nny * k)).astype(np.uint64)
        for a in range(3):
            u = u01(seed, STREAM_JITTER, gid * np.uint64(3) + np.uint64(a))
            xyz[:, a] += np.where(interior, (2.0 * u - 1.0) * jitter * h, 0.0)

    # cells: hex index = hi + nx*(hj + ny*hk), 6 tets per hex in PERMS order
    hi, hj, hk = np.meshgrid(np.arange(nx), np.arange(ny), np.arange(nz), indexing="ij")
    hi = hi.transpose(2, 1, 0).ravel()
    hj = hj.transpose(2, 1, 0).ravel()
    hk = hk.transpose(2, 1, 0).ravel()
    nhex = hi.size

    def nid(di, dj, dk):
        return (hi + di) + nnx * ((hj + dj) + nny * (hk + dk))

    c2n = np.empty((nhex, 6, 4), dtype=np.int64)
    for t, (a, b, c) in enumerate(PERMS):
        off = [0, 0, 0]
        verts = [nid(0, 0, 0)]
        for ax in (a, b, c):
            off[ax] = 1
            verts.append(nid(*off))
        sign = _perm_sign((a, b, c))
        if sign < 0:                   # swap local nodes 2 and 3 -> positive volume
            verts[2], verts[3] = verts[3], verts[2]
        c2n[:, t, :] = np.stack(verts, axis=1)
    c2n = c2n.reshape(-1, 4)
    c2c = _c2c_from_c2n(c2n, nnx * nny * nnz)
    inlet = _inlet_faces(c2n, c2c, xyz, 0.0)
    return {
        "nx": nx, "ny": ny, "nz": nz, "h": h, "jitter": jitter,
        "node_xyz": np.ascontiguousarray(xyz),
        "c2n": np.ascontiguousarray(c2n.astype(np.int32)),
        "c2c": np.ascontiguousarray(c2c.astype(np.int32)),
        "inlet": inlet,
        "n_cells": c2n.shape[0], "n_nodes": xyz.shape[0],
        "box": (0.0, nx * h, 0.0, ny * h, 0.0, nz * h),
    }


def _perm_sign(p) -> int:
    inv = sum(1 for x in range(3) for y in range(x + 1, 3) if p[x] > p[y])
    return -1 if inv % 2 else 1


def _c2c_from_c2n(c2n: np.ndarray, nn: int) -> np.ndarray:
    """c2c[c][i] = the cell sharing the face opposite local node i, else -1."""
    nc = c2n.shape[0]
    keys = np.empty((nc, 4), dtype=np.int64)
    for i in range(4):
        f = np.sort(np.delete(c2n, i, axis=1), axis=1).astype(np.int64)
        keys[:, i] = (f[:, 0] * nn + f[:, 1]) * nn + f[:, 2]
    flat = keys.ravel()
    order = np.argsort(flat, kind="stable")
    sk = flat[order]
    same = sk[1:] == sk[:-1]
    c2c = np.full(nc * 4, -1, dtype=np.int64)
    a = order[:-1][same]
    b = order[1:][same]
    c2c[a] = b // 4
    c2c[b] = a // 4
    return c2c.reshape(nc, 4)


def _inlet_faces(c2n, c2c, xyz, zin) -> np.ndarray:
    """Boundary triangles on the plane z = zin: rows (cell, n0, n1, n2)."""
    rows = []
    for i in range(4):
        f = np.delete(c2n, i, axis=1)
        on = (c2c[:, i] < 0) & np.all(xyz[f, 2] == zin, axis=1)
        cells = np.nonzero(on)[0]
        rows.append(np.concatenate([cells[:, None], f[cells]], axis=1))
    out = np.concatenate(rows, axis=0)
    out = out[np.argsort(out[:, 0], kind="stable")]
    return np.ascontiguousarray(out.astype(np.int64))


# ----------------------------------------------------------------------------
# Particles
# ----------------------------------------------------------------------------

def seed_particles(mesh: dict, n: int, seed: int, drift: float = 0.25,
                   spread: float = 0.05, id_base: int = 0, cluster=None, first: int = 0) -> dict:
    """n particles: cell uniform over tets (or clustered), point uniform in the
    tet (gaps of 3 sorted uniforms), v = drift*z + U(-spread, spread)^3.

    cluster = (frac, cell_ids): that fraction of particles is drawn uniformly
    from cell_ids instead (config C5).
    first: generate particles [first, first + n) of the population (chunks
    of a large population equal generating it at once).
    """
    idx = np.arange(first, first + n, dtype=np.uint64)
    nc = mesh["n_cells"]
    u = u01(seed, STREAM_CELL, idx * np.uint64(2))
    cell = np.minimum((u * nc).astype(np.int64), nc - 1)
    if cluster is not None:
        frac, hot = cluster
        hot = np.asarray(hot, dtype=np.int64)
        pick = u01(seed, STREAM_CELL, idx * np.uint64(2) + np.uint64(1)) < frac
        hc = hot[np.minimum((u * hot.size).astype(np.int64), hot.size - 1)]
        cell = np.where(pick, hc, cell)
    s = np.stack([u01(seed, STREAM_POINT, idx * np.uint64(3) + np.uint64(a)) for a in range(3)], 1)
    s.sort(axis=1)
    b = np.stack([s[:, 0], s[:, 1] - s[:, 0], s[:, 2] - s[:, 1], 1.0 - s[:, 2]], 1)
    p = mesh["node_xyz"][mesh["c2n"][cell]]               # (n,4,3)
    # explicit left-to-right sum (no BLAS / einsum reordering): the device
    # generator (gen/gen_cuda.cu) reproduces it bit for bit
    pos = b[:, 0:1] * p[:, 0] + b[:, 1:2] * p[:, 1] + b[:, 2:3] * p[:, 2] + b[:, 3:4] * p[:, 3]
    vel = np.stack([(2.0 * u01(seed, STREAM_VEL, idx * np.uint64(3) + np.uint64(a)) - 1.0) * spread
                    for a in range(3)], 1)
    vel[:, 2] += drift
    return {
        "pos": np.ascontiguousarray(pos), "vel": np.ascontiguousarray(vel),
        "cell": np.ascontiguousarray(cell.astype(np.int32)),
        "id": np.arange(id_base + first, id_base + first + n, dtype=np.int64),
    }


def inject_batch(mesh: dict, step: int, n_inj: int, seed: int, v_inj: float = 0.25,
                 id_base: int = 0) -> dict:
    """Step `step`'s injected particles: face uniform over inlet triangles, point
    uniform on it ((a,b) ~ U^2 reflected if a+b>1), v = v_inj * z-hat (inward
    normal of the z = z0 inlet), cell = the face's cell, id = id_base +
    step*n_inj + k."""
    inlet = mesh["inlet"]
    nf = inlet.shape[0]
    g = np.uint64(step) * np.uint64(n_inj) + np.arange(n_inj, dtype=np.uint64)
    f = np.minimum((u01(seed, STREAM_FACE, g) * nf).astype(np.int64), nf - 1)
    a = u01(seed, STREAM_INJPT, g * np.uint64(2))
    b = u01(seed, STREAM_INJPT, g * np.uint64(2) + np.uint64(1))
    flip = (a + b) > 1.0
    a = np.where(flip, 1.0 - a, a)
    b = np.where(flip, 1.0 - b, b)
    xyz = mesh["node_xyz"]
    pa, pb, pc = xyz[inlet[f, 1]], xyz[inlet[f, 2]], xyz[inlet[f, 3]]
    pos = pa + a[:, None] * (pb - pa) + b[:, None] * (pc - pa)
    vel = np.zeros((n_inj, 3))
    vel[:, 2] = v_inj
    return {
        "pos": np.ascontiguousarray(pos), "vel": vel,
        "cell": np.ascontiguousarray(inlet[f, 0].astype(np.int32)),
        "id": (id_base + step * n_inj + np.arange(n_inj)).astype(np.int64),
    }


def duct_bc(mesh: dict, wall=None, inlet=None, outlet=None, node_xyz=None):
    """Dirichlet boundary data for the field solve (an input, like the mesh):
    returns (mask int32[nn], value fp64[nn]).  A None value leaves that
    boundary homogeneous-Neumann.  Side walls are x in {0, X} or y in {0, Y};
    the inlet is z = 0, the outlet z = Z (Mini-FEM-PIC, PAPER.md:1495-1500:
    "the outer wall is fixed at a higher potential"; reading F3:
    a node on both a wall and the inlet/outlet takes the wall value).
    Boundary nodes of a Kuhn duct sit exactly on the box (jitter moves
    interior nodes only), so the tests are exact comparisons."""
    xyz = mesh["node_xyz"] if node_xyz is None else node_xyz
    x0, x1, y0, y1, z0, z1 = mesh["box"]
    nn = xyz.shape[0]
    mask = np.zeros(nn, dtype=np.int32)
    val = np.zeros(nn, dtype=np.float64)
    for v, sel in ((inlet, xyz[:, 2] == z0), (outlet, xyz[:, 2] == z1),
                   (wall, (xyz[:, 0] == x0) | (xyz[:, 0] == x1) | (xyz[:, 1] == y0) | (xyz[:, 1] == y1))):
        if v is None:
            continue
        vv = np.broadcast_to(np.asarray(v, dtype=np.float64), (nn,)) if np.ndim(v) else np.full(nn, float(v))
        mask[sel] = 1
        val[sel] = vv[sel]
    return mask, val


def hot_block_cells(mesh: dict, lo=(18, 18, 30), size=(12, 12, 12)) -> np.ndarray:
    """Cells of the hex block [lo, lo+size) (config C5's clustered region)."""
    nx, ny = mesh["nx"], mesh["ny"]
    ii, jj, kk = np.meshgrid(*[np.arange(l, l + s) for l, s in zip(lo, size)], indexing="ij")
    hexes = (ii + nx * (jj + ny * kk)).ravel()
    return (hexes[:, None] * 6 + np.arange(6)[None, :]).ravel()


# ----------------------------------------------------------------------------
# Configurations (seeds there)
# ----------------------------------------------------------------------------
CONFIGS = {
    # C1: parity config, 6x6x30 hex = 6,480 tets, 100k particles, 1k/step, 10 steps
    "c1": dict(dims=(6, 6, 30), n0=100_000, n_inj=1_000, steps=10, seed=20240812,
               c1E=(0.0, 0.0, 1e-3), dt=1.0, w=1.0),
    # C2: 48x48x72 hex = 995,328 tets, pre-seeded 50M steady state + 250k/step
    "c2": dict(dims=(48, 48, 72), n0=50_000_000, n_inj=250_000, steps=200, seed=20240813,
               c1E=(0.0, 0.0, 1e-3), dt=1.0, w=1.0),
    # C4: weak scaling, per GPU a 40x40x72-hex slab (691,200 tets) holding 1e9
    # particles (~1,447 per cell, the paper's ~70M per 48k cells,
    # PAPER.md:1885-1903); the global duct is 40x40x(72 N); injection on
    # rank 0 balances the outflow at 0.25 h/step over 72 layers (1e9 / 288)
    "c4": dict(dims=(40, 40, 72), n0=1_000_000_000, n_inj=3_500_000, steps=20, seed=20240815,
               c1E=(0.0, 0.0, 1e-3), dt=1.0, w=1.0),
    # C5: C2 mesh, 90% of 50M particles in the 12^3-hex block, no injection
    "c5": dict(dims=(48, 48, 72), n0=50_000_000, n_inj=0, steps=10, seed=20240816,
               c1E=(0.0, 0.0, 1e-3), dt=1.0, w=1.0, cluster=0.9),
}
