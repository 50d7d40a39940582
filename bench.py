#!/usr/bin/env python
"""bench.py -- particle-steps/s of the fused OP-PIC particle loop on B200.

One step = one pass of the whole hot path over the resident
particle population: inject (a1) -> zero node charge (a2) -> gather E + push
(a3, a4) -> multi-hop walk (a6, DH-seeded a5) -> deposit (a7) -> write-back /
holes (a8) -> hole fill (a9) -> (N > 1) migration rounds (a10) and the
node-charge halo (a11).

Default workload = config C4 (BASELINE.json configs[3], the metric's
"at 1/2/4/8 B200" configuration): per GPU a 40x40x72-hex Kuhn slab (691,200
tets) holding 1e9 particles, global duct 40x40x(72 N), contiguous z-slabs,
3.5M particles injected per step on rank 0, fixed uniform E (weak scaling:
per-GPU work fixed).  --config c2 is BASELINE.json's "1xB200" config (the
48x48x72 duct, 50M particles + 250k/step, CG Poisson solve every step timed
apart), c5 the clustered deposit stress, c3 the CabanaPIC-style EM loop.

Launch: `python bench.py --gpus N` starts N ranks itself (torch.distributed.run,
one process per GPU, NCCL) when run outside torchrun; under torchrun
WORLD_SIZE must equal --gpus.  `--gpus N --loopback` runs N slabs as N
contexts on ONE GPU (the in-process transport: a protocol check, not a
scaling number; reports n_gpus 1 and ranks N).

Contract: W untimed warm-up steps, then K timed steps bracketed by a barrier +
cuda synchronize, repeated --reps times (median reported, min shown; each
repetition times exactly K steps); CUDA events on the library's stream; max
over ranks; rank 0 prints ONE JSON line.  --impl reference times the CPU
oracle (oracle/, single thread, pinned core) on a bounded sample of the same
workload.
"""
from __future__ import annotations

import argparse
import contextlib
import hashlib
import json
import os
import socket
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "particle-steps/sec (push+move+deposit) at 1/2/4/8 B200; % of HBM roofline"
UNIT = "particle-steps/s"
DEP_NAMES = {0: "atomic", 1: "atomic_warpagg", 2: "sort_segred"}


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--reps", type=int, default=3,
                    help="timed repetitions of the K steps (median reported, min shown)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="c4", choices=["c4", "c2", "c5", "c1", "c3"])
    ap.add_argument("--loopback", action="store_true",
                    help="with --gpus N: N slabs as N contexts on one GPU (in-process transport)")
    ap.add_argument("--n0", type=int, default=0, help="override the seeded particle count (per rank)")
    ap.add_argument("--empty", action="store_true",
                    help="start from an empty domain (no seeded population): with --config c2 --steps 200 "
                         "the literal Mini-FEM-PIC protocol of PAPER.md:1502-1510 (250k injected/step)")
    ap.add_argument("--deposit", type=int, default=1, choices=[0, 1, 2],
                    help="0 atomic, 1 warp-aggregated atomic (default), 2 sort + segmented reduction")
    ap.add_argument("--deposit-cache", type=int, default=0,
                    help="warp-aggregated deposit through the per-warp node-charge cache (1)")
    ap.add_argument("--mh", action="store_true", help="multi-hop only (no direct-hop seeding)")
    ap.add_argument("--dhmode", type=int, default=1,
                    help="1: overlay seed for every particle; 2: only for particles that left their cell")
    ap.add_argument("--ov", type=float, default=0.125, help="DH overlay spacing (mesh units)")
    ap.add_argument("--hpass", type=int, default=4)
    ap.add_argument("--sort", type=int, default=10, help="sort by cell every K steps (0 = never)")
    ap.add_argument("--sort-lead", type=float, default=-1.0,
                    help="sort key at x + L dt v (opp_init_params.sort_lead); default: --sort / 2 with DH, else 0")
    ap.add_argument("--sort-init", type=int, default=-1,
                    help="sort the seeded population once before the run (default: iff --sort > 0)")
    ap.add_argument("--shuffle", type=int, default=0,
                    help="randomly shuffle the particles every K steps (the paper's GPU policy; use with --sort 0)")
    ap.add_argument("--direct", action="store_true", help="direct loads instead of the TMA pipeline")
    ap.add_argument("--axis", type=int, default=-1,
                    help="sort key along the duct axis z (1) or the cell id (0); default: 1 for c4 "
                         "(the sort moves data almost in place: C4 39.1 vs 43.0 ms/step), 0 otherwise")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=0)
    ap.add_argument("--field", type=int, default=-1,
                    help="solve the field (CG) every step: 1 on, 0 off (fixed uniform E); "
                         "default: on for c2 and c3, off otherwise")
    ap.add_argument("--rhs", type=float, default=2e-7, help="field solve: b = rhs * node charge")
    ap.add_argument("--wall", type=float, default=0.02, help="field solve: side-wall potential")
    ap.add_argument("--cg-tol", type=float, default=1e-10)
    ap.add_argument("--cg-warm", type=int, default=2,
                    help="linear field solve start: 1 = last solution, 2 = extrapolated from the last two")
    ap.add_argument("--field-model", choices=("linear", "boltzmann"), default="linear",
                    help="field solve: linear Poisson CG (north_star) or the Boltzmann-electron "
                         "Newton solve (PAPER.md:1604-1612, DESIGN.md §11)")
    ap.add_argument("--newton-cg-tol", type=float, default=1e-6,
                    help="boltzmann: inner CG tolerance relative to ||F|| per Newton step")
    ap.add_argument("--te", type=float, default=0.01, help="boltzmann: electron temperature (potential units)")
    ap.add_argument("--ne", type=float, default=-1.0,
                    help="boltzmann: electron coefficient (default: the mean ion load per volume)")
    ap.add_argument("--ppc", type=int, default=750, help="c3: particles per cell (750 = 72M, 1500 = 144M)")
    ap.add_argument("--em-sort", type=int, default=0, help="c3: sort particles by cell every K steps (0 = never)")
    args = ap.parse_args(argv)
    args.dh = 0 if args.mh else args.dhmode   # direct-hop seeding is the default
    if args.field < 0:
        args.field = 1 if args.config in ("c2", "c3") else 0
    if args.axis < 0:
        args.axis = 1 if args.config == "c4" else 0
    if args.sort_lead < 0:   # C4 pass 1 33.4 -> 32.2 ms with the key at mid-interval (lead 3 or 5)
        args.sort_lead = args.sort / 2.0 if (args.dh and args.sort > 0 and args.config != "c3") else 0.0
    if args.config in ("c4", "c5") and args.field:
        raise SystemExit("c4 / c5 run with a fixed uniform field (SURVEY.md §8(d))")
    return args


# ---------------------------------------------------------------- helpers
def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:   # noqa: BLE001
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def src_hash() -> str:
    """Hash of the library sources: a stored ncu traffic figure is only
    reported for the kernels it was captured from."""
    h = hashlib.sha256()
    d = os.path.join(ROOT, "paper_conf_icpp_lantra0m24_b200", "csrc")
    for f in sorted(os.listdir(d)):
        if f.endswith((".cu", ".h")):
            with open(os.path.join(d, f), "rb") as fh:
                h.update(f.encode() + fh.read())
    return h.hexdigest()[:16]


def traffic_for(key: str):
    """dram bytes per launch of the dominant kernel from this source tree's
    ncu --set full capture (profiles/ncu_traffic.json, written by
    scripts/ncu_summary.py traffic); null when the capture is of other code."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            e = json.load(f).get(key)
    except Exception:   # noqa: BLE001
        return None, "no capture"
    if not isinstance(e, dict):
        return None, "no capture"
    if e.get("src_hash") != src_hash():
        return None, f"capture {e.get('capture')} is of other kernel sources (stale)"
    return e.get("bytes"), e.get("capture")


def opp_env():
    return {k: v for k, v in os.environ.items() if k.startswith("OPP_")}


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:   # noqa: BLE001
        pass
    return "unknown"


class pinned_core:
    """Pin the calling thread to one host core while the oracle runs."""

    def __enter__(self):
        self.prev = os.sched_getaffinity(0)
        self.core = sorted(self.prev)[0]
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *a):
        os.sched_setaffinity(0, self.prev)


def cpu_meta(core=None) -> dict:
    import oracle
    d = {"cpu": cpu_model(), "threads": 1, **oracle.build_info()}
    if core is not None:
        d["pinned_core"] = core
    return d


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:   # noqa: BLE001
            self.proc = None
        time.sleep(0.15)
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:   # noqa: BLE001
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for k, nm in enumerate(names):
                if len(r) > 4 + k and r[4 + k].lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


# ---------------------------------------------------------------- rank groups
class Group:
    """The ranks this process drives: one (torchrun / N = 1) or all N
    (loopback threads).  Barrier + max / sum reductions over every rank."""

    def __init__(self, world: int, mode: str):
        self.world, self.mode = world, mode      # mode: "single", "dist" (process group), "loopback"
        self._bar = threading.Barrier(world) if mode == "loopback" else None
        self._vals = {}
        self._lock = threading.Lock()

    def barrier(self):
        if self.mode == "dist":
            import torch.distributed as dist
            dist.barrier()
        elif self.mode == "loopback":
            self._bar.wait()

    def _reduce(self, tag, v, op):
        if self.mode == "single":
            return v
        if self.mode == "dist":
            from paper_conf_icpp_lantra0m24_b200 import dist as D
            return D.max_over_ranks(v) if op == "max" else D.sum_over_ranks(v)
        with self._lock:
            self._vals.setdefault(tag, []).append(v)
        self._bar.wait()
        vals = self._vals[tag]
        r = max(vals) if op == "max" else sum(vals)
        self._bar.wait()
        with self._lock:
            self._vals.pop(tag, None)
        return r

    def max(self, tag, v):
        return self._reduce(tag, v, "max")

    def sum(self, tag, v):
        return self._reduce(tag, v, "sum")


# ---------------------------------------------------------------- workload
def workload(args, world=1):
    import gen
    cfg = dict(gen.CONFIGS[args.config])
    if args.n0:
        cfg["n0"] = args.n0
    if args.empty:
        cfg["n0_ref"] = cfg["n0"]   # the oracle sample keeps the steady state's injection ratio
        cfg["n0"] = 0
    nx, ny, nz = cfg["dims"]
    mesh = gen.kuhn_duct(nx, ny, nz * world)
    c1E = np.array(cfg["c1E"])
    qm, dt = 1.0, cfg["dt"]
    ef = np.tile(c1E / (qm * dt), (mesh["n_cells"], 1))
    cluster = None
    if cfg.get("cluster"):
        cluster = (cfg["cluster"], gen.hot_block_cells(mesh))
    field = ("Boltzmann-electron Newton field solve every step" if args.field_model == "boltzmann"
             else "CG Poisson field solve every step") if args.field else "fixed uniform E"
    name = {"c4": f"C4 Mini-FEM-PIC weak scaling: per GPU a 40x40x72-hex Kuhn slab (691,200 tets) "
                  f"with {cfg['n0']:,} particles, global duct 40x40x{72 * world}, "
                  f"{cfg['n_inj']:,} injected/step on rank 0, {field}",
            "c2": ("C2 Mini-FEM-PIC duct 48x48x72 hex (995,328 tets), " +
                   ("starting empty (the literal protocol, PAPER.md:1502-1510)" if args.empty
                    else "pre-seeded steady state") + " + 250k injected/step, " + field),
            "c5": "C5 clustered deposit stress: C2 mesh, 90% of particles in 1.04% of cells",
            "c1": "C1 Mini-FEM-PIC duct 6x6x30 hex (6,480 tets)"}[args.config]
    return cfg, mesh, ef, qm, dt, cluster, name


# ---------------------------------------------------------------- oracle legs
def oracle_sample(mesh, ef, qm, dt, w, cfg, n_sample, steps, cluster, dm=None):
    """Time the CPU oracle (as it stands) on a bounded sample of the workload,
    pinned to one host core.  The sample's inputs come from the seeded
    generator (its device twin when a GPU is present: bit-identical, and fast
    for millions of particles)."""
    import gen
    import oracle
    om = oracle.Mesh.from_gen(mesh)
    om.set_field(ef)
    P = oracle.Particles()
    if dm is not None:
        import gen.cuda as gc
        init = {k: v.cpu().numpy() for k, v in gc.seed_particles(dm, n_sample, cfg["seed"], cluster=cluster).items()
                if k != "_keep"}
    else:
        init = gen.seed_particles(mesh, n_sample, cfg["seed"], cluster=cluster)
    P.append(init["pos"], init["vel"], init["cell"], init["id"])
    Q = np.zeros(mesh["n_nodes"])
    scale = n_sample / max(cfg["n0"], cfg.get("n0_ref", 1))
    n_inj = int(round(cfg["n_inj"] * scale))
    pushed, secs = 0, 0.0
    with pinned_core() as pc:
        for s in range(steps):
            if n_inj:
                b = gen.inject_batch(mesh, s, n_inj, cfg["seed"], id_base=cfg["n0"])
                t0 = time.perf_counter()
                P.append(b["pos"], b["vel"], b["cell"], b["id"])
            else:
                t0 = time.perf_counter()
            st = oracle.step(om, P, qm * dt, dt, w, Q)
            secs += time.perf_counter() - t0
            pushed += st["n_before"]
    return pushed, secs, n_inj, pc.core


def run_reference(args, rank, world):
    if rank != 0:
        return
    cfg, mesh, ef, qm, dt, cluster, name = workload(args)
    w = cfg["w"]
    n_sample = 400_000 if args.config != "c1" else cfg["n0"]
    # warm-up steps are run and discarded, then K timed sample-steps
    if args.warmup > 0:
        oracle_sample(mesh, ef, qm, dt, w, cfg, n_sample, args.warmup, cluster)
    pushed, secs, n_inj, core = oracle_sample(mesh, ef, qm, dt, w, cfg, n_sample, args.steps, cluster)
    v = pushed / secs
    sample = (f"{n_sample:,} particles of the {args.config.upper()} workload "
              f"(+{n_inj:,} injected/step), {args.steps} steps, 1 thread; the GPU arm runs "
              f"{cfg['n0']:,} per rank (different cache behaviour)")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * secs / max(args.steps, 1), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": name, "sample": sample},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": sample, **cpu_meta(core)},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- config C3
C3 = dict(dims=(40, 40, 60), seed=20240814, v0=0.2, pert=0.01, vth=0.01, qdt_2mc=0.05,
          cdt_2h=(1.0, 1.0, 1.0), e_amp=1e-2, b0=0.5, b_amp=1e-2, kcap=16, dt=0.5, h=(1.0, 1.0, 1.0),
          # charge per unit weight: plasma frequency w_p^2 = (q/m) n Q = (2 qdt_2mc / dt) 750 qsp
          # = 0.04, w_p dt = 0.1 (the explicit leap-frog's stable, resolved regime)
          qsp=0.04 / (2 * 0.05 / 0.5 * 750))
C3_NAME = ("C3 CabanaPIC-style two-stream: 40x40x60 periodic hex (96,000 cells) declared through "
           "c2c, {ppc} particles/cell, Boris push + face-crossing move + Eq. 11 current deposit "
           "(Move_Deposit){fields}")


def c3_inputs(args):
    import gen.em as ge
    nx, ny, nz = C3["dims"]
    e, b = ge.em_fields(nx, ny, nz, C3["seed"], e_amp=C3["e_amp"], b0=C3["b0"], b_amp=C3["b_amp"])
    return nx, ny, nz, ge.periodic_hex(nx, ny, nz), e, b


def run_reference_c3(args, rank, world):
    if rank != 0:
        return
    import gen.em as ge
    import oracle.em as OE
    nx, ny, nz, c2c, e, b = c3_inputs(args)
    interp = OE.interpolate(nx, ny, nz, e, b)
    # bounded sample: the first `ppc_s` particles of every cell
    ppc_s = 16
    p = ge.two_stream(nx, ny, nz, ppc_s, C3["seed"], v0=C3["v0"], pert=C3["pert"], vth=C3["vth"])
    prm = OE.params(C3["qdt_2mc"], C3["cdt_2h"], C3["qsp"], C3["kcap"])
    acc = np.zeros((nx * ny * nz, 12))
    off, u, w, cell = p["off"], p["u"], p["w"], p["cell"]
    with pinned_core() as pc:
        for _ in range(max(args.warmup, 0)):
            OE.move_deposit(prm, off, u, w, cell, interp, c2c, acc)
        t0 = time.perf_counter()
        for _ in range(args.steps):
            OE.move_deposit(prm, off, u, w, cell, interp, c2c, acc)
        secs = time.perf_counter() - t0
    v = p["n"] * args.steps / secs
    sample = f"{p['n']:,} particles ({ppc_s}/cell) of the C3 workload, {args.steps} steps, 1 thread"
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * secs / max(args.steps, 1),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": C3_NAME.format(ppc=args.ppc, fields=", fixed fields"),
                                            "sample": sample},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                             **cpu_meta(pc.core)},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def c3_rank_main(args, rank, world, group, uid, transport, stream, res):
    """One rank of C3.  N = 1: the 40x40x60 box.  N > 1: weak scaling along z --
    the periodic box is 40x40x(60 N), rank r owns layers [60 r, 60 (r + 1))
    with its own seeded 750 ppc population (the two-stream perturbation
    repeats per slab); Move_Deposit migrates the particles whose streak leaves
    the slab and the field side exchanges ghost layers (opp_em_*_slab)."""
    import torch
    import gen.cuda as gc
    import gen.em as ge
    from paper_conf_icpp_lantra0m24_b200.em_app import CabanaPicEM
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    dev = torch.cuda.current_device()
    nx, ny, nzl = C3["dims"]
    nz = nzl * world
    e, b = ge.em_fields(nx, ny, nz, C3["seed"], e_amp=C3["e_amp"], b0=C3["b0"], b_amp=C3["b_amp"])
    c2c = ge.periodic_hex(nx, ny, nz)
    nc = nx * ny * nz
    L = nx * ny
    k0, k1 = rank * nzl, (rank + 1) * nzl
    c0, c1 = k0 * L, k1 * L
    slab = (k0, k1) if world > 1 else None
    sim = CabanaPicEM(nx, ny, nz, c2c, e, b, C3["qdt_2mc"], C3["cdt_2h"], C3["qsp"], C3["kcap"],
                      deposit_mode=1 if args.deposit != 0 else 0, device=dev, nranks=world, rank=rank,
                      uid=uid, transport=transport, slab=slab, stream=stream.cuda_stream,
                      torch_alloc=transport == 0)
    d = gc.em_two_stream(nx, ny, nzl, args.ppc, C3["seed"] + rank, v0=C3["v0"], pert=C3["pert"],
                         vth=C3["vth"])
    n0 = d["n"]
    if slab is None:
        sim.set_particles(d["off"], d["u"], d["w"], d["cell"])
    else:
        ids = torch.arange(n0, dtype=torch.int64, device=d["cell"].device) + rank * n0
        sim.set_particles(d["off"], d["u"], d["w"], d["cell"] + c0, ids=ids,
                          capacity=int(n0 * 1.05) + (1 << 16))
        del ids
    del d
    nstep = [0]
    em_field = args.field != 0      # c3 default: the field side runs every step

    def em_step(stats=False):
        if args.em_sort and nstep[0] % args.em_sort == 0:
            sim.sort_by_cell()
        nstep[0] += 1
        st = sim.step(want_stats=stats)
        if em_field:
            sim.field_step(C3["dt"], C3["h"])   # AccumulateCurrent, AdvanceB/E/B, Interpolate
        else:
            sim.zero_acc()
        return st

    for _ in range(args.warmup):
        em_step()
    reps = []
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(dev) if rank == 0 else contextlib.nullcontext() as clk:
        for rep in range(max(args.reps, 1)):
            torch.cuda.synchronize()
            group.barrier()
            torch.cuda.synchronize()
            l0 = sim.launches()
            O.opp_phase_timing(sim.ctx, True)
            O.opp_get_phase_times(sim.ctx)
            n_start = sim.n
            e0.record(stream)
            for _ in range(args.steps):
                em_step()
            e1.record(stream)
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1)
            launches = sim.launches() - l0
            ph = O.opp_get_phase_times(sim.ctx)
            O.opp_phase_timing(sim.ctx, False)
            pushed = n_start * args.steps
            field_ms = ph["field"][0] if em_field else 0.0
            ms = group.max(f"c3ms{rep}", ms)
            field_ms = group.max(f"c3f{rep}", field_ms)
            pushed = group.sum(f"c3p{rep}", pushed)
            launches = group.sum(f"c3l{rep}", launches)
            reps.append(dict(ms=ms, field_ms=field_ms, pushed=pushed, launches=launches, ph=ph,
                             n_local=n_start, value=pushed / ((ms - field_ms) / 1e3)))
    out = {"reps": reps, "st": em_step(stats=True), "n": sim.n, "nc": nc,
           "clocks": clk.summary() if rank == 0 else None}
    if not args.no_e2e:
        # e2e through the public API: the step's fields (this rank's layers) arrive
        # from pinned host memory (H2D), Interpolate + Move_Deposit (+ the field
        # side) run, this rank's accumulator is read back
        ke = args.e2e_steps or min(args.steps, 10)
        eh = torch.from_numpy(np.ascontiguousarray(e[:, c0:c1])).pin_memory()
        bh = torch.from_numpy(np.ascontiguousarray(b[:, c0:c1])).pin_memory()
        acc_h = torch.empty((c1 - c0, 12), dtype=torch.float64).pin_memory()
        # copies on a side stream, overlapped with the previous step's compute:
        # step s's fields are staged H2D while step s-1 runs, the accumulator
        # is snapshotted on the device and read back while step s+1 runs
        cs = torch.cuda.Stream()
        e_st, b_st = torch.empty_like(eh, device=sim.dev), torch.empty_like(bh, device=sim.dev)
        acc_snap = torch.empty((c1 - c0, 12), dtype=torch.float64, device=sim.dev)
        staged, consumed, snapped = torch.cuda.Event(), torch.cuda.Event(), torch.cuda.Event()
        ev, bv = sim.e.view(3, -1)[:, c0:c1], sim.b.view(3, -1)[:, c0:c1]
        torch.cuda.synchronize()
        group.barrier()
        n_e2e = sim.n
        e0.record(stream)
        with torch.cuda.stream(cs):
            cs.wait_event(e0)                       # every copy inside the timed region
            e_st.copy_(eh, non_blocking=True)
            b_st.copy_(bh, non_blocking=True)
            staged.record(cs)
        for s_ in range(ke):
            stream.wait_event(staged)
            ev.copy_(e_st, non_blocking=True)
            bv.copy_(b_st, non_blocking=True)
            consumed.record(stream)
            if s_ + 1 < ke:
                with torch.cuda.stream(cs):
                    cs.wait_event(consumed)
                    e_st.copy_(eh, non_blocking=True)     # the next step's fields
                    b_st.copy_(bh, non_blocking=True)
                    staged.record(cs)
            sim.interpolate()
            em_step()
            if s_ > 0:
                stream.wait_event(snapped)          # the previous read-back left acc_snap
            acc_snap.copy_(sim.acc[c0:c1], non_blocking=True)
            done = torch.cuda.Event()
            done.record(stream)
            with torch.cuda.stream(cs):
                cs.wait_event(done)
                acc_h.copy_(acc_snap, non_blocking=True)
                snapped.record(cs)
        stream.wait_event(snapped)
        e1.record(stream)
        torch.cuda.synchronize()
        out["e2e"] = {"ms": group.max("c3e2e", e0.elapsed_time(e1)), "pushed": group.sum("c3e2ep", n_e2e * ke),
                      "steps": ke, "h2d": int(eh.nbytes + bh.nbytes), "d2h": int(acc_h.nbytes)}
    sim.close()
    res[rank] = out


def run_ours_c3(args, rank, world, mode):
    """C3: one step = Move_Deposit over the whole resident population + the
    field side (timed apart).  mode as run_ours: "single", "dist" (torchrun
    ranks over NCCL), "loopback" (N ranks as threads on one GPU)."""
    import torch
    from paper_conf_icpp_lantra0m24_b200 import dist as D
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    group = Group(world, mode)
    uid, info = None, None
    if mode == "dist":
        uid = D.broadcast_bytes(O.opp_get_nccl_unique_id() if rank == 0 else None)
        info = nccl_info(group, world)
    elif mode == "loopback":
        uid = os.urandom(128)
        info = {"backend": "loopback", "ranks": world, "devices": [0]}
    res = [None] * world
    if mode == "loopback":
        errs = []
        streams = [torch.cuda.Stream() for _ in range(world)]

        def worker(r):
            try:
                with torch.cuda.stream(streams[r]):
                    c3_rank_main(args, r, world, group, uid, 1, streams[r], res)
            except BaseException as ex:   # noqa: BLE001
                errs.append((r, repr(ex)))
                group._bar.abort()
                raise

        th = [threading.Thread(target=worker, args=(r,)) for r in range(world)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        if errs:
            raise SystemExit(f"loopback ranks failed: {errs}")
    else:
        c3_rank_main(args, rank, world, group, uid, 0, torch.cuda.current_stream(), res)
    if rank != 0:
        return
    out = res[0]
    reps = out["reps"]
    em_field = args.field != 0
    order = sorted(range(len(reps)), key=lambda k: reps[k]["value"])
    med = reps[order[len(order) // 2]]
    ms, field_ms, pushed, launches, ph = med["ms"], med["field_ms"], med["pushed"], med["launches"], med["ph"]
    value = med["value"]          # the particle loop; the field side apart (as C2)
    n, nc, st = med["n_local"], out["nc"], out["st"]
    ncl = nc // world             # this rank's cells (the kernel's per-cell traffic)
    peak, peak_src = load_peaks()
    k_ms, k_cnt = ph["em_move_deposit"]
    # algorithmic bytes per launch: particle state in (off, u, w, cell = 60 B) and
    # out (off, u, cell = 52 B); per cell the interpolator (144 B), c2c (24 B)
    # and the accumulator read-modify-write (2 x 96 B)
    bpl = 112.0 * n + (144.0 + 24.0 + 192.0) * ncl
    achieved = bpl / (k_ms / max(k_cnt, 1) / 1e3) / 1e9
    tb, tsrc = traffic_for(f"c3_dep{1 if args.deposit != 0 else 0}")
    fields = (", field side every step (AccumulateCurrent + Yee AdvanceB/E/B + Interpolate, timed apart)"
              if em_field else ", fixed fields")
    workload_name = C3_NAME.format(ppc=args.ppc, fields=fields)
    if world > 1:
        workload_name += (f"; weak scaling: global box 40x40x{60 * world}, one 60-layer z-slab per rank, "
                          "migration + Update_Ghosts")
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": 1 if mode == "loopback" else world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_name, "mesh_cells": nc, "mesh_cells_per_rank": ncl,
                   "particles_per_rank": n, "ppc": args.ppc,
                   "deposit": "atomic_warpagg" if args.deposit != 0 else "atomic",
                   "sort_every": args.em_sort,
                   "l2": "inputs larger than L2 (particle state %.1f GB per rank > 126 MB L2)" % (n * 60 / 1e9),
                   "parallelism": (f"slab{world}" + (" (loopback: all ranks on one GPU)" if mode == "loopback"
                                                     else "")) if world > 1 else "single",
                   "ranks": world},
        "reps": {"values": [r["value"] for r in reps], "median": value,
                 "min": min(r["value"] for r in reps)},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": tb, "traffic_source": tsrc,
                     "kernel": "k_em_move_deposit",
                     "bytes_model": "112 B/particle + 360 B/cell per launch", "peak_source": peak_src},
        "gpu_launches": launches,
        "phases_ms_per_step": {k: v[0] / args.steps for k, v in ph.items() if v[1]},
        "field": ({"ms_per_step": field_ms / args.steps,
                   "note": "value excludes the field side (timed separately, as C2's field solve); "
                           "value_incl_field counts it"} if em_field else None),
        "value_incl_field": pushed / (ms / 1e3),
        "move": {"crossings_per_particle": st["n_crossings"] / max(n, 1),
                 "max_crossings": st["max_crossings"], "capped": st["n_capped"]},
        "clocks": out["clocks"],
        "env": opp_env(),
    }
    if info is not None:
        line["config"]["comm"] = info
    if "e2e" in out:
        e2 = out["e2e"]
        line["e2e"] = {"value": e2["pushed"] / (e2["ms"] / 1e3), "unit": UNIT,
                       "h2d_bytes_per_step": e2["h2d"], "d2h_bytes_per_step": e2["d2h"],
                       "steps": e2["steps"], "note": "edge E and face B of the rank's cells from pinned host "
                       "memory every step, opp_em_interpolate + opp_em_move_deposit (+ field side), the "
                       "rank's accumulator read back; copies on a side stream overlapped with the "
                       "neighbouring steps' compute"}
    if not args.no_cpu and world == 1:
        import gen.em as ge
        import oracle.em as OE
        nx, ny, nz, c2c, e, b = c3_inputs(args)
        interp = OE.interpolate(nx, ny, nz, e, b)
        p = ge.two_stream(nx, ny, nz, 16, C3["seed"], v0=C3["v0"], pert=C3["pert"], vth=C3["vth"])
        acc = np.zeros((nc, 12))
        prm = OE.params(C3["qdt_2mc"], C3["cdt_2h"], C3["qsp"], C3["kcap"])
        with pinned_core() as pc:
            t0 = time.perf_counter()
            for _ in range(2):
                OE.move_deposit(prm, p["off"], p["u"], p["w"], p["cell"], interp, c2c, acc)
            secs = time.perf_counter() - t0
        line["cpu_baseline"] = {"value": 2 * p["n"] / secs, "unit": UNIT, "cores": 1, "kind": "oracle",
                                "sample": f"{p['n']:,} particles (16/cell) of the C3 workload, 2 steps, "
                                          f"1 thread, {secs:.1f} s", **cpu_meta(pc.core)}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- our arm (electrostatic)
class EsRank:
    """One rank of the electrostatic particle loop: its slab (or the whole
    duct), its libopp context, its seeded population and its injection
    batches, all resident on the device before any timed step."""

    def __init__(self, args, cfg, gmesh, gef, world, rank, stream, transport=0, uid=None,
                 cluster=None):
        import torch
        import gen
        import gen.cuda as gc
        from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
        from paper_conf_icpp_lantra0m24_b200 import dist as D
        self.args, self.cfg, self.rank, self.world = args, cfg, rank, world
        self.stream = stream
        w, n0, n_inj, seed = cfg["w"], cfg["n0"], cfg["n_inj"], cfg["seed"]
        base, kw = 0, {}
        mesh, ef = gmesh, gef
        if world > 1:
            mesh = D.slab(gmesh, world, rank)
            ef = D.local_field(gef, mesh)
            base = mesh["cell_base"]
            kw = dict(nranks=world, rank=rank, uid=uid, transport=transport)
            gen_mesh = dict(mesh, inlet=mesh["inlet_local"])
            if cluster is not None:
                cluster = (cluster[0], cluster[1][(cluster[1] >= base) & (cluster[1] < base + mesh["n_cells"])] - base)
        else:
            gen_mesh = mesh
        if args.field:
            ef = np.zeros_like(ef)
        self.mesh, self.base = mesh, base
        dm = gc.DeviceMesh(gen_mesh)
        self.dm = dm
        self.n_inj = n_inj if (world == 1 or mesh["inlet"].shape[0] > 0) else 0
        total = args.warmup + max(args.reps, 1) * args.steps
        self.total = total
        # capacity: the seeded population + a 4% margin for the flow imbalance
        # between ranks + two steps of injection (injection precedes the push)
        cap = int(n0 * 1.04) + 2 * self.n_inj + 4096
        if args.empty:   # the population grows by n_inj per step (no outflow before z = 72 h),
            # through the timed steps and the e2e leg's
            ke = 0 if args.no_e2e else (args.e2e_steps or min(args.steps, 10))
            cap = (total + ke + 2) * self.n_inj + 4096
        self.sim = MiniFemPic(mesh, ef, capacity=cap, stream=stream.cuda_stream, deposit_mode=args.deposit,
                              direct_hop=args.dh, overlay_spacing=args.ov, hop_budget=args.hpass,
                              sort_every=args.sort, tma_pipeline=not args.direct,
                              sort_axis=(0.0, 0.0, 1.0) if args.axis else (0.0, 0.0, 0.0),
                              deposit_cache=bool(args.deposit_cache), sort_lead=args.sort_lead,
                              torch_alloc=transport == 0, device=stream.device.index, **kw)
        sim = self.sim
        if args.field:
            fmask, fval = gen.duct_bc(mesh, wall=args.wall, inlet=0.0)
            sim.field_init(fmask, fval)
        # seed in chunks (C4: 1e9 particles; a chunk is 60 B per particle of
        # temporary device memory), generated on the device, bit-identical to
        # generating the population at once
        chunk = 50_000_000
        with torch.cuda.stream(stream):
            for first in range(0, n0, chunk):
                m = min(chunk, n0 - first)
                init = gc.seed_particles(dm, m, seed + rank, cluster=cluster, id_base=rank * n0, first=first,
                                         stream=stream.cuda_stream)
                if base:
                    init["cell"] += base
                sim.inject(init, on_device=True)
                stream.synchronize()
                del init
            if args.sort_init > 0 or (args.sort_init < 0 and args.sort):
                # the population is born in random cell order; a sorted steady
                # state is what periodic sorting maintains (setup, untimed)
                sim.step(0.0, 1.0, w, stats=False, fill=True)   # builds mesh data; dt = 0: no motion
                sim.sort_by_cell()
            self.batches = [gc.inject_batch(dm, s, self.n_inj, seed, id_base=world * n0,
                                            stream=stream.cuda_stream) if self.n_inj else None
                            for s in range(total)]
        stream.synchronize()
        self.host_batches = None
        self.bz_last = {}

    def field(self):
        a = self.args
        if a.field and a.field_model == "boltzmann":
            self.bz_last.update(self.sim.field_solve_boltzmann(a.rhs, a.ne, 0.0, a.te, newton_tol=a.cg_tol,
                                                               cg_tol=a.newton_cg_tol, warm_start=a.cg_warm))
        elif a.field:
            self.sim.field_solve(a.rhs, tol=a.cg_tol, warm_start=a.cg_warm, stats=False)

    def one_step(self, s, on_device=True):
        sim, a = self.sim, self.args
        self.field()
        b = self.batches[s] if on_device else self.host_batches[s]
        if b is not None:
            sim.inject(b, on_device=on_device)
        sim.step(self.cfg["dt"], 1.0, self.cfg["w"], stats=False, fill=True)
        if a.shuffle and s % a.shuffle == 0:
            sim.shuffle(self.cfg["seed"] + 7919 * s)


def es_rank_main(args, rank, world, group, cfg, gmesh, gef, cluster, uid, transport, res):
    """Everything one rank does: setup, warm-up, the timed repetitions, the
    e2e leg.  Per-rank results go to res[rank] (rank 0's dict carries the
    reduced values)."""
    import torch
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    dev = int(os.environ.get("LOCAL_RANK", 0)) if transport == 0 else 0
    torch.cuda.set_device(dev)
    stream = torch.cuda.Stream(device=dev)
    R = EsRank(args, cfg, gmesh, gef, world, rank, stream, transport=transport, uid=uid, cluster=cluster)
    sim = R.sim
    if args.field and args.field_model == "boltzmann" and args.ne < 0:
        x0, x1, y0, y1, z0, z1 = gmesh["box"]
        args.ne = args.rhs * cfg["w"] * cfg["n0"] * world / ((x1 - x0) * (y1 - y0) * (z1 - z0))
    with torch.cuda.stream(stream):
        for s in range(args.warmup):
            R.one_step(s)
    stream.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    reps = []
    s_next = args.warmup
    with ClockSampler(dev) as clk:
        for rep in range(max(args.reps, 1)):
            st0 = sim.last_stats()
            group.barrier()
            torch.cuda.synchronize()
            l0 = sim.launches()
            sim.phase_timing(True)
            sim.phase_times()  # reset
            with torch.cuda.stream(stream):
                e0.record(stream)
                for s in range(s_next, s_next + args.steps):
                    R.one_step(s)
                e1.record(stream)
            torch.cuda.synchronize()
            group.barrier()
            s_next += args.steps
            ms = e0.elapsed_time(e1)
            launches = sim.launches() - l0
            phases = sim.phase_times()
            sim.phase_timing(False)
            st1 = sim.last_stats()
            pushed = st1["cum_pushed"] - st0["cum_pushed"]
            field_ms = phases["field"][0] if args.field else 0.0
            ms_max = group.max(f"ms{rep}", ms)
            loop_ms_max = group.max(f"lms{rep}", ms - field_ms)
            pushed_sum = group.sum(f"p{rep}", pushed)
            launches_sum = group.sum(f"l{rep}", launches)
            pmd_ms_max = group.max(f"pmd{rep}", phases["push_move_deposit"][0])
            reps.append(dict(ms=ms_max, loop_ms=loop_ms_max, field_ms=field_ms, pushed=pushed_sum,
                             launches=launches_sum, phases=phases, pmd_ms=pmd_ms_max,
                             pushed_local=pushed, value=pushed_sum / (loop_ms_max / 1e3), st=st1))
    out = dict(reps=reps, clocks=clk.summary(), mesh=R.mesh, n_inj=R.n_inj, bz=R.bz_last)
    if args.field == 1 and args.field_model == "linear":
        out["fst"] = sim.field_stats()
    # ---- e2e: same metric through the C ABI with HOST buffers
    if not args.no_e2e:
        ke = args.e2e_steps or min(args.steps, 10)
        lo = args.warmup   # the device batches of these steps were consumed; host copies of them
        R.host_batches = [None] * R.total
        for s in range(lo, lo + ke):
            b = R.batches[s]
            if b is not None:
                R.host_batches[s] = {k: b[k].cpu().pin_memory().numpy() for k in ("pos", "vel", "cell", "id")}
        q_host = torch.empty(R.mesh["n_nodes"], dtype=torch.float64).pin_memory().numpy()
        # rewind is impossible (state advanced); e2e continues the same run
        torch.cuda.synchronize()
        s0 = sim.last_stats()
        group.barrier()
        with torch.cuda.stream(stream):
            e0.record(stream)
            # a user's pipelined loop through the public API: inject the next
            # step's batch (H2D on the library's copy stream) while this step
            # computes, then read this step's node charge back
            if R.host_batches[lo] is not None:
                sim.inject(R.host_batches[lo], on_device=False)
            sim.phase_timing(bool(args.field))
            sim.phase_times()
            for s in range(lo, lo + ke):
                R.field()
                sim.step(cfg["dt"], 1.0, cfg["w"], stats=False, fill=True)
                if s + 1 < lo + ke and R.host_batches[s + 1] is not None:
                    sim.inject(R.host_batches[s + 1], on_device=False)
                O.opp_get_node_charge(sim.ctx, sim.node_charge, q_host)
            e1.record(stream)
        torch.cuda.synchronize()
        ems = e0.elapsed_time(e1)
        if args.field:
            ems -= sim.phase_times()["field"][0]
        sim.phase_timing(False)
        s1 = sim.last_stats()
        out["e2e"] = dict(ms=group.max("e2e_ms", ems), pushed=group.sum("e2e_p", s1["cum_pushed"] - s0["cum_pushed"]),
                          steps=ke, h2d=group.sum("e2e_h2d", R.n_inj * 60),
                          d2h=group.sum("e2e_d2h", R.mesh["n_nodes"] * 8))
    out["dm"] = R.dm
    sim.close()
    res[rank] = out


def nccl_info(group, world):
    """NCCL version, ranks and devices of the job (printed to stderr and
    recorded in the JSON line so a run's rank count can be checked)."""
    import torch
    dev = torch.cuda.current_device()
    p = torch.cuda.get_device_properties(dev)
    me = {"rank": int(os.environ.get("RANK", 0)), "device": dev, "name": p.name,
          "pci_bus_id": f"{p.pci_bus_id:02x}" if hasattr(p, "pci_bus_id") else None,
          "uuid": str(getattr(p, "uuid", ""))}
    if group.mode == "dist":
        import torch.distributed as dist
        allv = [None] * world
        dist.all_gather_object(allv, me)
    else:
        allv = [me]
    info = {"nccl_version": ".".join(map(str, torch.cuda.nccl.version())), "ranks": world,
            "backend": group.mode, "devices": allv}
    return info


def run_ours(args, rank, world, mode):
    """mode: "single" (N = 1), "dist" (this process is one of N torchrun
    ranks, NCCL) or "loopback" (N ranks as threads of this process on one GPU)."""
    import torch
    from paper_conf_icpp_lantra0m24_b200 import dist as D
    from paper_conf_icpp_lantra0m24_b200 import opp as O
    cfg, gmesh, gef, qm, dt, cluster, name = workload(args, world)
    group = Group(world, mode)
    uid = None
    if mode == "dist":
        uid = D.broadcast_bytes(O.opp_get_nccl_unique_id() if rank == 0 else None)
        info = nccl_info(group, world)
        if rank == 0:
            print("[bench] NCCL", json.dumps(info), file=sys.stderr, flush=True)
    elif mode == "loopback":
        uid = os.urandom(128)
        info = {"backend": "loopback", "ranks": world, "devices": [0]}
    else:
        info = None
    res = [None] * world
    if mode == "loopback":
        errs = []

        def worker(r):
            try:
                es_rank_main(args, r, world, group, cfg, gmesh, gef, cluster, uid, 1, res)
            except BaseException as e:   # noqa: BLE001
                errs.append((r, repr(e)))
                group._bar.abort()
                raise

        th = [threading.Thread(target=worker, args=(r,)) for r in range(world)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        if errs:
            raise SystemExit(f"loopback ranks failed: {errs}")
    else:
        es_rank_main(args, rank, world, group, cfg, gmesh, gef, cluster, uid, 0, res)
    if rank != 0:
        return
    out = res[0]
    reps = out["reps"]
    order = sorted(range(len(reps)), key=lambda k: reps[k]["value"])
    med = reps[order[len(order) // 2]]
    value = med["value"]
    mesh = out["mesh"]
    nc, nn = mesh["n_cells"], mesh["n_nodes"]
    n_avg = med["pushed"] / args.steps / world       # per rank
    n_inj = cfg["n_inj"]
    # ---- roofline of the dominant kernel (k_push_move_deposit, pass 1):
    # algorithmic bytes per launch / the pass-1 kernel's mean
    # CUDA-event duration (events recorded by the library on its stream)
    peak, peak_src = load_peaks()
    pmd_ms, pmd_cnt = med["phases"]["push_move_deposit"]
    n_local = med["pushed_local"] / args.steps
    bytes_per_launch = 104.0 * n_local + 160.0 * nc + 16.0 * nn
    achieved = bytes_per_launch / (pmd_ms / max(pmd_cnt, 1) / 1e3) / 1e9
    tb, tsrc = traffic_for(f"{args.config}_dep{args.deposit}_dh{int(args.dh)}")
    # whole-step model bytes (SURVEY.md §8(d) B_ps)
    f_inj = n_inj / max(n_avg * world, 1)
    b_ps = 104.0 + (160.0 * nc + 16.0 * nn) / max(n_avg, 1) + 60.0 * f_inj
    nranks_txt = f"{world} GPU" + ("s" if world > 1 else "")
    line = {
        "metric": METRIC, "value": value, "unit": UNIT,
        "n_gpus": 1 if mode == "loopback" else world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": med["ms"] / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic",
        "config": {"workload": name, "mesh_cells_per_rank": nc, "mesh_nodes_per_rank": nn,
                   "particles_seeded_per_rank": cfg["n0"], "inject_per_step": n_inj,
                   "avg_particles_per_step_per_rank": n_avg,
                   "deposit": DEP_NAMES[args.deposit] + (" + per-warp cache" if args.deposit_cache else ""),
                   "walk": (f"DH{args.dh}(overlay {args.ov} h)+MH" if args.dh else "MH"),
                   "hop_budget_per_pass": args.hpass,
                   "sort_every": args.sort, "shuffle_every": args.shuffle,
                   "pipeline": "direct" if args.direct else "tma",
                   "sort_key": ("axis z" if args.axis else "cell id") +
                               (f" at x + {args.sort_lead:g} dt v" if args.sort_lead > 0 else ""),
                   "l2": ("inputs larger than L2 (particle state %.1f GB per rank > 126 MB L2)" % (n_avg * 60 / 1e9))
                         if not args.empty else
                         ("particle state grows from empty (average %.2f GB per rank; > 126 MB L2 after the first "
                          "~9 steps); the mesh data (walk lines, field, DH overlay) exceeds L2 throughout" % (n_avg * 60 / 1e9)),
                   "parallelism": f"slab{world}" + (" (loopback: all ranks on one GPU)" if mode == "loopback" else ""),
                   "mesh_global": f"{cfg['dims'][0]}x{cfg['dims'][1]}x{cfg['dims'][2] * world} hex",
                   "ranks": world},
        "reps": {"values": [r["value"] for r in reps], "median": value,
                 "min": min(r["value"] for r in reps), "ms_per_step": [r["ms"] / args.steps for r in reps]},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": tb, "traffic_source": tsrc,
                     "kernel": "k_push_move_deposit_tiled (pass 1)",
                     "bytes_model": "104 B/particle + 160 B/cell + 16 B/node per launch",
                     "peak_source": peak_src,
                     "step_frac": b_ps * (value / world) / (peak * 1e9), "step_bytes_per_particle": b_ps},
        "gpu_launches": med["launches"],
        # the fused kernel's own rate (the slowest rank's pass-1 time, all
        # ranks' particles; the continuation, fill, sort and comm excluded)
        "fused_kernel_only": {"value": med["pushed"] / (med["pmd_ms"] / 1e3) if med["pmd_ms"] > 0 else None,
                              "unit": UNIT, "kernel": "k_push_move_deposit_tiled (pass 1)",
                              "ms_per_step": med["pmd_ms"] / args.steps},
        "phases_ms_per_step": {k: v[0] / args.steps for k, v in med["phases"].items() if v[1]},
        "walk": {"hops_per_particle_last_step": med["st"]["total_hops"] / max(med["st"]["n_before"], 1),
                 "max_hops_last_step": med["st"]["max_hops"], "hop_capped": med["st"]["n_hop_capped"],
                 "deferred_last_step": med["st"]["n_deferred"],
                 "migrated_out_last_step_rank0": med["st"]["n_migrated_out"]},
        "clocks": out["clocks"],
        "env": opp_env(),
    }
    if info is not None:
        line["config"]["comm"] = info
    if args.field and args.field_model == "boltzmann":
        line["field"] = {"ms_per_step": med["field_ms"] / args.steps, "model": "boltzmann",
                         "last_solve": out["bz"], "newton_tol": args.cg_tol, "inner_cg_tol": args.newton_cg_tol,
                         "ne_coef": args.ne, "te": args.te, "rhs_scale": args.rhs,
                         "wall_potential": args.wall,
                         "note": "value excludes the field solve (timed separately, SURVEY.md "
                                 "§8(d)); value_incl_field counts it"}
        line["value_incl_field"] = med["pushed"] / (med["ms"] / 1e3)
    elif args.field:
        fst = out["fst"]
        line["field"] = {"ms_per_step": med["field_ms"] / args.steps, "cg_iterations_last": fst["iterations"],
                         "rel_residual_last": fst["rel_residual"], "tol": args.cg_tol,
                         "rhs_scale": args.rhs, "wall_potential": args.wall,
                         "solver": "Jacobi-PCG, one persistent cooperative kernel, warm start " +
                                   ("extrapolated from the last two solutions" if args.cg_warm == 2
                                    else "from the last solution"),
                         "note": "value excludes the field solve (timed separately, SURVEY.md "
                                 "§8(d)); value_incl_field counts it"}
        line["value_incl_field"] = med["pushed"] / (med["ms"] / 1e3)
    if "e2e" in out:
        e = out["e2e"]
        line["e2e"] = {"value": e["pushed"] / (e["ms"] / 1e3), "unit": UNIT,
                       "h2d_bytes_per_step": e["h2d"], "d2h_bytes_per_step": e["d2h"],
                       "steps": e["steps"], "note": "injection arrays from pinned host memory (opp_inject "
                       "on_device=0, H2D overlapped with the previous step on the library's copy "
                       "stream) + node charge read back every step (opp_get_node_charge); the same run "
                       "continued after the timed repetitions (its later steps: a population thinned by "
                       "the side walls, C4 ~0.1% per step), its own sort steps included"}
    # ---- cpu baseline: the oracle on a bounded sample (rank 0, N = 1), one pinned core
    if not args.no_cpu and world == 1:
        n_sample = 4_000_000 if args.config != "c1" else cfg["n0"]
        pushed_c, secs, ninj_c, core = oracle_sample(gmesh, gef, qm, dt, cfg["w"], cfg, n_sample, 3, cluster,
                                                     dm=out["dm"])
        line["cpu_baseline"] = {"value": pushed_c / secs, "unit": UNIT, "cores": 1,
                                "kind": "oracle",
                                "sample": f"{n_sample:,} particles of the same workload "
                                          f"(+{ninj_c:,} injected/step), 3 steps, 1 thread, "
                                          f"{secs:.1f} s", **cpu_meta(core)}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- launch
def free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def main():
    args = parse()
    world_env = os.environ.get("WORLD_SIZE")
    if world_env is None and args.gpus > 1 and not args.loopback and args.impl == "ours":
        # outside torchrun: start the N ranks (one process per GPU) ourselves
        import torch
        ndev = torch.cuda.device_count()
        if ndev < args.gpus:
            print(json.dumps({"error": f"--gpus {args.gpus} needs {args.gpus} GPUs, found {ndev} "
                                       "(--loopback runs the N slabs on one GPU as a protocol check)"}),
                  flush=True)
            sys.exit(2)
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
               f"--nproc-per-node={args.gpus}", "--master-addr", "127.0.0.1",
               "--master-port", str(free_port()), os.path.abspath(__file__)] + sys.argv[1:]
        sys.exit(subprocess.call(cmd))
    world = int(world_env or 1)
    rank = int(os.environ.get("RANK", "0"))
    if world_env is not None and world != args.gpus:
        print(json.dumps({"error": f"WORLD_SIZE={world} but --gpus {args.gpus}"}), flush=True)
        sys.exit(2)
    if world > 1:
        import torch
        import torch.distributed as dist
        if args.impl == "ours":
            torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", 0)))
            dist.init_process_group("nccl")
        else:
            dist.init_process_group("gloo")
    if args.config == "c3" and args.impl == "reference":
        run_reference_c3(args, rank, world)
    elif args.config == "c3":
        if args.loopback and args.gpus > 1:
            run_ours_c3(args, 0, args.gpus, "loopback")
        else:
            run_ours_c3(args, rank, world, "dist" if world > 1 else "single")
    elif args.impl == "reference":
        run_reference(args, rank, world)
    elif args.loopback and args.gpus > 1:
        run_ours(args, 0, args.gpus, "loopback")
    else:
        run_ours(args, rank, world, "dist" if world > 1 else "single")
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
