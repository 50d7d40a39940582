"""Pins of the EM field-side oracle (oracle/em_field.py): AccumulateCurrent,
AdvanceB, AdvanceE against identities of the discrete
Maxwell system that a wrong sign, index or scale breaks:

* div B = 0 is preserved by AdvanceB for any E (div curl = 0);
* Gauss's law: with particles moved by the Move_Deposit oracle and the
  current from AccumulateCurrent, div E - rho (node charge density from the
  particles' trilinear weights) is unchanged by every step -- this fixes the
  scale 1 / (2 dt h_b h_c), the edge mapping of the 12 accumulator slots and
  the sign of J in AdvanceE;
* a vacuum standing wave E_y = sin(k x) evolves as cos(n theta) with the Yee
  leap-frog phase theta = 2 asin((dt/h) sin(k h / 2)) (closed form).
"""
import numpy as np
import pytest

import gen.em as G
import oracle.em as OE
import oracle.em_field as F


def test_div_b_preserved():
    rng = np.random.default_rng(1)
    nx, ny, nz, h = 4, 5, 6, (1.0, 0.7, 1.3)
    e = rng.uniform(-1, 1, (3, nx * ny * nz))
    b = np.zeros((3, nx * ny * nz))
    F.advance_b(e, b, nx, ny, nz, h, 0.3)
    F.advance_b(rng.uniform(-1, 1, (3, nx * ny * nz)), b, nx, ny, nz, h, 0.2)
    assert np.abs(b).max() > 0.1
    assert np.abs(F.div_b(b, nx, ny, nz, h)).max() < 1e-13


@pytest.mark.parametrize("cdt", [0.4, 1.6])
def test_gauss_law_preserved_with_particles(cdt):
    nx, ny, nz = 4, 3, 5
    h = (1.0, 1.0, 1.0)
    dt = 0.5
    rng = np.random.default_rng(3)
    n = 600
    off = np.ascontiguousarray(rng.uniform(-1, 1, (3, n)))
    u = np.ascontiguousarray(rng.uniform(-0.8, 0.8, (3, n)))
    w = rng.uniform(0.5, 1.5, n)
    cell = rng.integers(0, nx * ny * nz, n).astype(np.int32)
    e, b = G.em_fields(nx, ny, nz, 5, e_amp=0.05, b0=0.3, b_amp=0.05)
    c2c = G.periodic_hex(nx, ny, nz)
    prm = OE.params(0.05, [cdt, cdt, cdt], 1.0, 16)
    g0 = F.div_e(e, nx, ny, nz, h) - F.node_charge_density(off, cell, w, 1.0, nx, ny, nz, h)
    for _ in range(3):
        acc = np.zeros((nx * ny * nz, 12))
        OE.move_deposit(prm, off, u, w, cell, OE.interpolate(nx, ny, nz, e, b), c2c, acc)
        J = F.accumulate_current(acc, nx, ny, nz, h, dt)
        F.advance_b(e, b, nx, ny, nz, h, dt / 2)
        F.advance_e(e, b, J, nx, ny, nz, h, dt)
        F.advance_b(e, b, nx, ny, nz, h, dt / 2)
        g1 = F.div_e(e, nx, ny, nz, h) - F.node_charge_density(off, cell, w, 1.0, nx, ny, nz, h)
        assert np.abs(J).max() > 1e-3
        np.testing.assert_allclose(g1, g0, rtol=0, atol=1e-12)
    # a wrong current scale breaks it
    e2 = e.copy()
    F.advance_e(e2, b * 0, 0.1 * J, nx, ny, nz, h, dt)
    assert np.abs(F.div_e(e2, nx, ny, nz, h) - F.div_e(e, nx, ny, nz, h)).max() > 1e-4


def test_vacuum_standing_wave_yee_phase():
    nx, ny, nz, h, dt = 32, 2, 2, (1.0, 1.0, 1.0), 0.5
    kx = 2 * np.pi * 3 / nx
    i = np.tile(np.arange(nx), ny * nz)
    e = np.zeros((3, nx * ny * nz))
    e[1] = np.sin(kx * i)               # E_y at x = i h
    b = np.zeros_like(e)
    J = np.zeros_like(e)
    n = 40
    for _ in range(n):
        F.advance_b(e, b, nx, ny, nz, h, dt / 2)
        F.advance_e(e, b, J, nx, ny, nz, h, dt)
        F.advance_b(e, b, nx, ny, nz, h, dt / 2)
    theta = 2 * np.arcsin(dt / h[0] * np.sin(kx * h[0] / 2))
    np.testing.assert_allclose(e[1], np.cos(n * theta) * np.sin(kx * i), rtol=0, atol=1e-12)
    assert np.abs(e[0]).max() == 0 and np.abs(e[2]).max() == 0
