"""Pins of the EM Move_Deposit oracle (oracle/em.c) against the mathematics.

Each test fixes something the oracle cannot get right by accident:
Eq. 11 against an independent numerical integration and
the hand-derived closed form; the Whitney-pair charge-continuity identity
(node weights W0 at the end minus the start equal the divergence of the
deposited W1 edge currents -- pins the face-crossing logic, the signs and the
edge order); ballistic motion with periodic wrap (closed form); the Boris
rotation angle 2 atan(|t|) and |u| conservation; the uniform-E momentum
closed form; the interpolator reproducing its edge/face values.
"""
import numpy as np
import pytest

import gen.em as G
import oracle.em as E


def kidx(sb, sc):
    return (1 if sb > 0 else 0) + (2 if sc > 0 else 0)


def test_segment_axis_aligned():
    # along x at fixed (y, z): int N dxi = dx (1 + sb y)(1 + sc z) / 4; no y / z current
    y, z, Q = 0.3, -0.7, 2.5
    acc = E.segment_current([-0.4, y, z], [0.9, y, z], Q)
    for sb in (-1, 1):
        for sc in (-1, 1):
            assert acc[kidx(sb, sc)] == pytest.approx(Q * 1.3 * (1 + sb * y) * (1 + sc * z) / 4, rel=1e-14)
    assert np.all(acc[4:] == 0.0)


def test_segment_vs_riemann_and_closed_form():
    rng = np.random.default_rng(5)
    for _ in range(20):
        p, q = rng.uniform(-1, 1, 3), rng.uniform(-1, 1, 3)
        Q = rng.uniform(0.5, 2)
        acc = E.segment_current(p, q, Q)
        # independent midpoint-rule integration of W1 . dL along the path
        m = 4000
        t = (np.arange(m) + 0.5) / m
        pts = p[None, :] + t[:, None] * (q - p)[None, :]
        d = q - p
        for a in range(3):
            b, c = (a + 1) % 3, (a + 2) % 3
            for sb in (-1, 1):
                for sc in (-1, 1):
                    riem = Q * d[a] * np.mean((1 + sb * pts[:, b]) * (1 + sc * pts[:, c]) / 4)
                    mb, mc = (p[b] + q[b]) / 2, (p[c] + q[c]) / 2
                    closed = Q * d[a] / 4 * ((1 + sb * mb) * (1 + sc * mc) + sb * sc * d[b] * d[c] / 12)
                    got = acc[4 * a + kidx(sb, sc)]
                    assert got == pytest.approx(closed, rel=1e-12, abs=1e-15)
                    assert got == pytest.approx(riem, rel=1e-6, abs=1e-9)


def _setup(nx, ny, nz, n, seed, cdt, qdt, e_amp=0.05, b0=0.3, b_amp=0.05, vmax=0.9):
    rng = np.random.default_rng(seed)
    c2c = G.periodic_hex(nx, ny, nz)
    e, b = G.em_fields(nx, ny, nz, seed, e_amp=e_amp, b0=b0, b_amp=b_amp)
    interp = E.interpolate(nx, ny, nz, e, b)
    off = np.ascontiguousarray(rng.uniform(-1, 1, (3, n)))
    u = np.ascontiguousarray(rng.uniform(-vmax, vmax, (3, n)))
    w = rng.uniform(0.5, 1.5, n)
    cell = rng.integers(0, nx * ny * nz, n).astype(np.int32)
    prm = E.params(qdt, [cdt, cdt * 1.1, cdt * 0.9], 1.0, 16)
    return c2c, interp, off, u, w, cell, prm


def _cell_ijk(cell, nx, ny):
    return cell % nx, (cell // nx) % ny, cell // (nx * ny)


def _node_weights(off, cell, w, nx, ny, nz):
    """sum_p w_p W0_n(x_p) on the periodic node grid (trilinear hat functions)."""
    rho = np.zeros((nz, ny, nx))
    i, j, k = _cell_ijk(cell, nx, ny)
    for sx in (0, 1):
        for sy in (0, 1):
            for sz in (0, 1):
                f = ((1 + (2 * sx - 1) * off[0]) * (1 + (2 * sy - 1) * off[1]) *
                     (1 + (2 * sz - 1) * off[2]) / 8)
                np.add.at(rho, ((k + sz) % nz, (j + sy) % ny, (i + sx) % nx), w * f)
    return rho


def _divergence(acc, nx, ny, nz):
    """node value = 1/2 sum over cells and their corners of s_x jx + s_y jy + s_z jz."""
    out = np.zeros((nz, ny, nx))
    cell = np.arange(nx * ny * nz)
    i, j, k = _cell_ijk(cell, nx, ny)
    for sx in (-1, 1):
        for sy in (-1, 1):
            for sz in (-1, 1):
                v = 0.5 * (sx * acc[:, 0 + kidx(sy, sz)] + sy * acc[:, 4 + kidx(sz, sx)] +
                           sz * acc[:, 8 + kidx(sx, sy)])
                np.add.at(out, ((k + (sz > 0)) % nz, (j + (sy > 0)) % ny, (i + (sx > 0)) % nx), v)
    return out


@pytest.mark.parametrize("cdt", [0.3, 1.7])
def test_charge_continuity(cdt):
    nx, ny, nz = 3, 4, 5
    c2c, interp, off, u, w, cell, prm = _setup(nx, ny, nz, 400, 11, cdt, 0.05)
    acc = np.zeros((nx * ny * nz, 12))
    rho0 = _node_weights(off, cell, w, nx, ny, nz)
    for _ in range(3):
        st = E.move_deposit(prm, off, u, w, cell, interp, c2c, acc)
    rho1 = _node_weights(off, cell, w, nx, ny, nz)
    assert np.all(np.abs(off) <= 1.0)
    if cdt > 1:
        assert st["max_crossings"] >= 2 and st["n_capped"] == 0
    np.testing.assert_allclose(_divergence(acc, nx, ny, nz), rho1 - rho0, rtol=0, atol=1e-12)
    # dropping any one deposited segment breaks it (the pin has teeth)
    acc2 = acc.copy()
    acc2[7, 3] += 1e-6
    assert np.abs(_divergence(acc2, nx, ny, nz) - (rho1 - rho0)).max() > 1e-7


def _global(off, cell, nx, ny):
    i, j, k = _cell_ijk(cell, nx, ny)
    return np.stack([i + (off[0] + 1) / 2, j + (off[1] + 1) / 2, k + (off[2] + 1) / 2])


def test_ballistic_periodic_wrap():
    nx, ny, nz = 4, 3, 5
    c2c, interp, off, u, w, cell, prm = _setup(nx, ny, nz, 300, 3, 1.3, 0.0)
    interp[:] = 0.0
    x0 = _global(off, cell, nx, ny)
    u0 = u.copy()
    rg = 1 / np.sqrt(1 + (u0 ** 2).sum(0))
    cdt = np.array(prm.cdt_2h[:])[:, None]
    acc = np.zeros((nx * ny * nz, 12))
    n = 4
    for _ in range(n):
        E.move_deposit(prm, off, u, w, cell, interp, c2c, acc)
    assert np.array_equal(u, u0)   # no field: momentum untouched
    L = np.array([nx, ny, nz])[:, None]
    want = x0 + n * cdt * u0 * rg / 2        # offset units are 2 per cell
    d = (_global(off, cell, nx, ny) - want + L / 2) % L - L / 2
    assert np.abs(d).max() < 1e-12


def test_boris_uniform_E_closed_form():
    qdt, Ev = 0.05, np.array([0.3, -0.2, 0.1])
    u = np.array([0.1, 0.2, -0.3])
    u0 = u.copy()
    for _ in range(7):
        u = E.boris(np.r_[Ev, 0, 0, 0], qdt, u)
    np.testing.assert_allclose(u, u0 + 7 * 2 * qdt * Ev, rtol=0, atol=1e-15)


def test_boris_rotation_angle():
    rng = np.random.default_rng(2)
    for _ in range(10):
        B = rng.uniform(-1, 1, 3)
        u = rng.uniform(-2, 2, 3)
        qdt = 0.2
        un = E.boris(np.r_[0, 0, 0, B], qdt, u)
        gamma = np.sqrt(1 + u @ u)
        bh = B / np.linalg.norm(B)
        assert np.linalg.norm(un) == pytest.approx(np.linalg.norm(u), rel=1e-14)
        assert un @ bh == pytest.approx(u @ bh, rel=1e-12, abs=1e-14)   # parallel part kept
        up, unp = u - (u @ bh) * bh, un - (un @ bh) * bh
        ang = np.arctan2(np.linalg.norm(np.cross(up, unp)), up @ unp)
        assert ang == pytest.approx(2 * np.arctan(qdt * np.linalg.norm(B) / gamma), rel=1e-10)
        # positive charge: rotation sense is -B (u x B force)
        assert np.cross(up, unp) @ bh < 0


def test_interpolator_reproduces_edges_and_faces():
    nx, ny, nz = 3, 2, 4
    e, b = G.em_fields(nx, ny, nz, 9)
    f = E.interpolate(nx, ny, nz, e, b)
    nc = nx * ny * nz

    def cid(i, j, k):
        return (i % nx) + nx * ((j % ny) + ny * (k % nz))
    for c in range(nc):
        i, j, k = c % nx, (c // nx) % ny, c // (nx * ny)
        for a in range(3):
            q = f[c, 4 * a: 4 * a + 4]
            for s in (-1, 1):
                for t in (-1, 1):
                    val = q[0] + s * q[1] + t * (q[2] + s * q[3])
                    d = [0, 0, 0]
                    d[(a + 1) % 3] = s > 0
                    d[(a + 2) % 3] = t > 0
                    want = e[a, cid(i + d[0], j + d[1], k + d[2])]
                    assert val == pytest.approx(want, rel=1e-14, abs=1e-16)
            for s in (-1, 1):
                d = [0, 0, 0]
                d[a] = s > 0
                assert f[c, 12 + 2 * a] + s * f[c, 13 + 2 * a] == pytest.approx(
                    b[a, cid(i + d[0], j + d[1], k + d[2])], rel=1e-14)


def test_crossing_cap_and_face_landing():
    nx = ny = nz = 4
    c2c = G.periodic_hex(nx, ny, nz)
    interp = np.zeros((nx * ny * nz, 18))
    # lands exactly on the +x face (t == 1): stays in its cell at offset +1
    # (start chosen so that, in IEEE fp64, (1 - p) / d == 1 and p + d == 1)
    u = np.array([[0.75], [0.0], [0.0]])
    d = 1.0 * (0.75 * (1.0 / np.sqrt(1.0 + (0.75 * 0.75 + (0.0 + 0.0)))))
    p0 = next(p for p in (1.0 - d, np.nextafter(1.0 - d, 0), np.nextafter(1.0 - d, 2))
              if (1.0 - p) / d == 1.0 and p + d == 1.0)
    off = np.array([[p0], [0.0], [0.0]])
    prm = E.params(0.0, [1.0, 1, 1], 1.0, 16)
    cell = np.array([5], dtype=np.int32)
    acc = np.zeros((64, 12))
    E.move_deposit(prm, off, u, np.ones(1), cell, interp, c2c, acc)
    assert cell[0] == 5 and off[0, 0] == 1.0
    g = np.sqrt(1 + 0.75 ** 2)
    # a cap of 1 crossing stops a 3-cell streak on the second cell's far face
    off = np.array([[0.0], [0.0], [0.0]])
    prm = E.params(0.0, [6.0 / (0.75 / g), 1, 1], 1.0, 1)
    cell = np.array([5], dtype=np.int32)
    st = E.move_deposit(prm, off, u, np.ones(1), cell, interp, c2c, acc)
    assert st["n_capped"] == 1 and cell[0] == c2c[5, 1] and off[0, 0] == 1.0


def test_two_stream_inputs():
    p = G.two_stream(2, 3, 4, 10, 7, v0=0.2)
    assert p["n"] == 240 and np.all(np.diff(p["cell"]) >= 0)
    assert np.all(np.abs(p["off"]) <= 1)
    uz = p["u"][2]
    assert np.all(uz[0::2] > 0.15) and np.all(uz[1::2] < -0.15)
