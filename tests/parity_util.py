"""Parity harness: run the CPU oracle and the CUDA library on identical
generated inputs and compare them with the north_star tolerances
(SURVEY.md §8(c) S15/S16):

* final cell per particle id: bit-exact, excluding particles whose oracle
  barycentric margin (min_i |lambda_i|, running min over steps) is < 1e-10;
  that count is reported and must stay below 1e-6 of all particles;
* positions / velocities: |dx| <= 1e-12 * max(|x|, h), |dv| <= 1e-12 * max(|v|, v_inj);
* node charge: |dQ_n| <= 1e-10 * max(|Q_n|, w) after each side's excluded
  particles' own deposits are subtracted;
* the surviving id sets are equal (outside the excluded set).

Test infrastructure: imports oracle/ (allowed for tests/ and smoke()).
"""
from __future__ import annotations

import numpy as np

import gen
import oracle

NEAR = 1e-10


def run_oracle(mesh, ef, init, inject, steps, c1, dt, w, hcap=1024, use_dh=False,
               overlay=None):
    om = oracle.Mesh.from_gen(mesh)
    om.set_field(ef)
    if use_dh:
        x0, dx, n = overlay
        om.build_overlay(x0, dx, n)
    P = oracle.Particles()
    if init is not None and init["cell"].shape[0]:
        P.append(init["pos"], init["vel"], init["cell"], init["id"])
    Q = np.zeros(mesh["n_nodes"])
    stats, removed = [], {}
    for s in range(steps):
        b = inject(s) if inject else None
        if b is not None and b["cell"].shape[0]:
            P.append(b["pos"], b["vel"], b["cell"], b["id"])
        st = oracle.step(om, P, c1, dt, w, Q, hcap=hcap, use_dh=use_dh)
        stats.append(st)
        rid, rmg = P.removed()
        for i, m in zip(rid.tolist(), rmg.tolist()):
            removed[i] = m
    out = P.get()
    return om, out, Q, stats, removed


def compare(om, c2n, orc, Q_orc, removed_margin, gpu, Q_gpu, w, h=1.0, v_ref=0.25, near=NEAR):
    """Returns a report dict; raises AssertionError on a parity failure.
    near=None: no near-face exclusion (every particle compared bit-exactly)."""
    excl = set()
    if near is not None:
        excl = set(orc["id"][orc["margin"] < near].tolist())
        excl |= {i for i, m in removed_margin.items() if m < near}
    o_ids, g_ids = orc["id"], gpu["id"]
    so, sg = set(o_ids.tolist()), set(g_ids.tolist())
    assert len(sg) == len(g_ids), "duplicate ids on the GPU side"
    diff = (so ^ sg) - excl
    assert not diff, f"survivor sets differ on {len(diff)} ids, e.g. {sorted(diff)[:5]}"
    common = np.array(sorted((so & sg) - excl), dtype=np.int64)
    io = np.searchsorted(o_ids, common)
    ig = np.searchsorted(g_ids, common)
    assert np.array_equal(o_ids[io], common) and np.array_equal(g_ids[ig], common)
    bad = np.nonzero(orc["cell"][io] != gpu["cell"][ig])[0]
    assert bad.size == 0, f"{bad.size} cell mismatches, ids {common[bad[:5]]}"
    xo, xg = orc["pos"][io], gpu["pos"][ig]
    vo, vg = orc["vel"][io], gpu["vel"][ig]
    ex = np.abs(xo - xg) / np.maximum(np.abs(xo), h)
    ev = np.abs(vo - vg) / np.maximum(np.abs(vo), v_ref)
    assert ex.size == 0 or ex.max() <= 1e-12, f"position error {ex.max()}"
    assert ev.size == 0 or ev.max() <= 1e-12, f"velocity error {ev.max()}"

    def own_deposit(side, ids):
        q = np.zeros_like(Q_orc)
        idx = np.searchsorted(side["id"], ids)
        for k, i in zip(idx, ids):
            if k < side["id"].shape[0] and side["id"][k] == i:
                c = int(side["cell"][k])
                lam = om.bary(c, side["pos"][k])
                np.add.at(q, c2n[c], w * lam)
        return q

    ex_ids = np.array(sorted(excl), dtype=np.int64)
    Qo = Q_orc - own_deposit(orc, ex_ids)
    Qg = Q_gpu - own_deposit(gpu, ex_ids)
    eq = np.abs(Qo - Qg) / np.maximum(np.abs(Qo), w)
    assert eq.max() <= 1e-10, f"node charge error {eq.max()} at node {eq.argmax()}"
    n_all = max(len(so | sg), 1)
    assert len(excl) <= 1e-6 * n_all + 1, f"too many near-face particles: {len(excl)}"
    return {"n_compared": int(common.size), "n_excluded": len(excl),
            "max_pos_rel": float(ex.max()) if ex.size else 0.0,
            "max_vel_rel": float(ev.max()) if ev.size else 0.0,
            "max_charge_rel": float(eq.max())}


def c1_case(jitter=0.2, n0=100_000, n_inj=1_000, steps=10, seed=20240812, efield="random",
            drift=0.25, spread=0.05):
    """Config C1: 6x6x30 Kuhn duct, 100k particles, 1k/step."""
    mesh = gen.kuhn_duct(6, 6, 30, jitter=jitter, seed=seed)
    rng = np.random.default_rng(seed)
    if efield == "random":
        ef = rng.uniform(-2e-3, 2e-3, (mesh["n_cells"], 3))
    else:
        ef = np.tile([0.0, 0.0, 1e-3], (mesh["n_cells"], 1))
    init = gen.seed_particles(mesh, n0, seed, drift=drift, spread=spread)
    inject = (lambda s: gen.inject_batch(mesh, s, n_inj, seed, id_base=n0)) if n_inj else None
    return mesh, ef, init, inject, steps
