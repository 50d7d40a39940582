"""The EM loop over z-slabs (C3 partitioned, PAPER.md:1346-1352 + the
Update_Ghosts of the field side) on ONE GPU: R contexts in one process, one
host thread each, joined by the in-process loopback transport.  The merged
result after several full PIC steps must equal the oracle's single-domain
loop: every particle (by id) in the same cell with the same offset and
velocity, every rank's own layers of E and B within 1e-12 (-m gpu)."""
import os
import threading

import numpy as np
import pytest

import gen.em as G
import oracle.em as OE

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _slabs(nz, R):
    base, rem = divmod(nz, R)
    out, k = [], 0
    for r in range(R):
        n = base + (1 if r < rem else 0)
        out.append((k, k + n))
        k += n
    return out


def _oracle(nx, ny, nz, e, b, p, qdt, cdt, kcap, h, dt, steps):
    import oracle.em_field as F
    off, u, cell = p["off"].copy(), p["u"].copy(), p["cell"].copy()
    eo, bo = e.copy(), b.copy()
    prm = OE.params(qdt, cdt, 1.0, kcap)
    c2c = G.periodic_hex(nx, ny, nz)
    stats = []
    for _ in range(steps):
        acc = np.zeros((nx * ny * nz, 12))
        stats.append(OE.move_deposit(prm, off, u, p["w"], cell, OE.interpolate(nx, ny, nz, eo, bo), c2c, acc))
        J = F.accumulate_current(acc, nx, ny, nz, h, dt)
        F.advance_b(eo, bo, nx, ny, nz, h, dt / 2)
        F.advance_e(eo, bo, J, nx, ny, nz, h, dt)
        F.advance_b(eo, bo, nx, ny, nz, h, dt / 2)
    return off, u, cell, eo, bo, stats


def _ranks(nx, ny, nz, e, b, p, qdt, cdt, kcap, h, dt, steps, R, dep, cap_mul=3):
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    from paper_conf_icpp_lantra0m24_b200.em_app import CabanaPicEM
    uid = os.urandom(128)
    sl = _slabs(nz, R)
    layer = p["cell"] // (nx * ny)
    streams = [torch.cuda.Stream() for _ in range(R)]
    out, errs = [None] * R, []

    def worker(r):
        try:
            k0, k1 = sl[r]
            own = np.nonzero((layer >= k0) & (layer < k1))[0]
            sim = CabanaPicEM(nx, ny, nz, G.periodic_hex(nx, ny, nz), e, b, qdt, cdt, 1.0, kcap,
                              O.OPP_DEP_ATOMIC_WARPAGG if dep else O.OPP_DEP_ATOMIC, nranks=R, rank=r,
                              uid=uid, transport=1, slab=(k0, k1), stream=streams[r].cuda_stream,
                              torch_alloc=False)
            sim.set_particles(np.ascontiguousarray(p["off"][:, own]), np.ascontiguousarray(p["u"][:, own]),
                              p["w"][own].copy(), p["cell"][own].copy(), ids=own.astype(np.int64),
                              capacity=cap_mul * max(len(own), 64))
            st = []
            for _ in range(steps):
                st.append(sim.step(want_stats=True))
                sim.field_step(dt, h)
            g = sim.state()
            g["e"], g["b"] = sim.e.cpu().numpy(), sim.b.cpu().numpy()
            out[r] = (g, st)
            sim.close()
        except Exception as ex:   # noqa: BLE001
            errs.append((r, ex))
            raise

    th = [threading.Thread(target=worker, args=(r,)) for r in range(R)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=300)
    assert not errs, errs
    assert all(o is not None for o in out)
    return sl, out


def _check(nx, ny, nz, p, ora, sl, out, steps):
    off, u, cell, eo, bo, ost = ora
    n = p["n"]
    seen = np.zeros(n, dtype=np.int64)
    lay = nx * ny
    for (k0, k1), (g, _) in zip(sl, out):
        ids = g["id"]
        seen[ids] += 1
        # every particle this rank holds is in its own layers
        assert np.all((g["cell"] // lay >= k0) & (g["cell"] // lay < k1))
        assert np.array_equal(g["cell"], cell[ids])
        np.testing.assert_allclose(g["off"], off[:, ids], rtol=1e-10, atol=1e-13)
        np.testing.assert_allclose(g["u"], u[:, ids], rtol=1e-10, atol=1e-13)
        c = slice(k0 * lay, k1 * lay)
        np.testing.assert_allclose(g["e"][:, c], eo[:, c], rtol=0, atol=1e-12)
        np.testing.assert_allclose(g["b"][:, c], bo[:, c], rtol=0, atol=1e-12)
        assert not np.any(g["acc"][c])            # the field step zeroed this rank's currents
    assert np.all(seen == 1)                      # no particle lost or duplicated
    for s in range(steps):
        assert sum(o[1][s]["n_crossings"] for o in out) == ost[s]["n_crossings"]
        assert sum(o[1][s]["n_capped"] for o in out) == ost[s]["n_capped"]


@pytest.mark.parametrize("R", [2, 3])
@pytest.mark.parametrize("dep", [0, 1])
def test_em_slabs_equal_single_domain(R, dep):
    nx, ny, nz, ppc, seed, steps = 4, 4, 6, 30, 21, 4
    h, dt, qdt, cdt = (1.0, 1.0, 1.0), 0.5, 0.05, [1.0, 1.0, 1.0]
    e, b = G.em_fields(nx, ny, nz, seed, e_amp=0.05, b0=0.4, b_amp=0.05)
    p = G.two_stream(nx, ny, nz, ppc, seed, v0=0.4, vth=0.05)
    ora = _oracle(nx, ny, nz, e, b, p, qdt, cdt, 16, h, dt, steps)
    sl, out = _ranks(nx, ny, nz, e, b, p, qdt, cdt, 16, h, dt, steps, R, dep)
    _check(nx, ny, nz, p, ora, sl, out, steps)


def test_em_slabs_fast_multi_slab_crossing_and_cap():
    """Streaks of ~3 cells through 1-layer slabs (8 ranks): a particle crosses
    several ranks in one step (several migration rounds, the crossing count
    travels with it so the cap kcap = 3 is the single-domain one)."""
    nx, ny, nz, ppc, seed, steps = 3, 3, 8, 20, 7, 3
    h, dt, qdt, cdt = (1.0, 1.0, 1.0), 0.5, 0.1, [3.0, 2.5, 3.5]
    e, b = G.em_fields(nx, ny, nz, seed, e_amp=0.05, b0=0.4, b_amp=0.05)
    p = G.two_stream(nx, ny, nz, ppc, seed, v0=0.6, vth=0.3)
    ora = _oracle(nx, ny, nz, e, b, p, qdt, cdt, 3, h, dt, steps)
    assert max(s["max_crossings"] for s in ora[5]) >= 3 and sum(s["n_capped"] for s in ora[5]) > 0
    sl, out = _ranks(nx, ny, nz, e, b, p, qdt, cdt, 3, h, dt, steps, 8, 1, cap_mul=6)
    _check(nx, ny, nz, p, ora, sl, out, steps)
