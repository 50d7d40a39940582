"""The device generator is bit-identical to the numpy generator (-m gpu)."""
import numpy as np
import pytest

import gen

pytestmark = pytest.mark.gpu


def test_seed_and_inject_bit_identical():
    import gen.cuda as gc
    mesh = gen.kuhn_duct(8, 7, 12, jitter=0.2, seed=4)
    dm = gc.DeviceMesh(mesh)
    for cluster in (None, (0.9, gen.hot_block_cells(mesh, lo=(2, 2, 3), size=(3, 3, 3)))):
        a = gen.seed_particles(mesh, 100_003, 77, cluster=cluster, id_base=5)
        b = gc.seed_particles(dm, 100_003, 77, cluster=cluster, id_base=5)
        for k in ("pos", "vel", "cell", "id"):
            np.testing.assert_array_equal(a[k], b[k].cpu().numpy())
    # chunked generation (C4 seeds 1e9 particles in chunks) = generating at once
    whole = gen.seed_particles(mesh, 50_000, 78, id_base=7)
    for first, n in ((0, 20_000), (20_000, 30_000)):
        b = gc.seed_particles(dm, n, 78, id_base=7, first=first)
        for k in ("pos", "vel", "cell", "id"):
            np.testing.assert_array_equal(whole[k][first:first + n], b[k].cpu().numpy())
    for s in (0, 3):
        a = gen.inject_batch(mesh, s, 5001, 77, id_base=9)
        b = gc.inject_batch(dm, s, 5001, 77, id_base=9)
        for k in ("pos", "vel", "cell", "id"):
            np.testing.assert_array_equal(a[k], b[k].cpu().numpy())


def test_em_two_stream_bit_identical():
    import gen.cuda as gc
    import gen.em as ge
    a = ge.two_stream(5, 4, 6, 37, 91, v0=0.3, vth=0.02)
    b = gc.em_two_stream(5, 4, 6, 37, 91, v0=0.3, vth=0.02)
    for k in ("off", "u", "w", "cell"):
        np.testing.assert_array_equal(a[k], b[k].cpu().numpy())
