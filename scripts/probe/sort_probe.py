"""Cost of the sort by cell at C4 against the age of the order (steps of
motion since the last sort): immediate re-sort (identity permutation), then
after 1, 3, 5, 10 steps.  CUDA events around opp_sort_by_cell + the library's
phase times.  Usage: python scripts/probe/sort_probe.py [extra bench args]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
sys.argv = ["bench.py", "--config", "c4", "--sort", "0", "--reps", "1", "--steps", "1", "--warmup", "0",
            "--no-cpu"] + sys.argv[1:]
import bench  # noqa: E402
import torch  # noqa: E402
import gen.cuda as gc  # noqa: E402

SPREAD = float(os.environ.get("PROBE_SPREAD", "0.05"))   # transverse velocity spread of the seeded particles
_seed = gc.seed_particles


def _seed_spread(*a, **k):
    k["spread"] = SPREAD
    return _seed(*a, **k)


gc.seed_particles = _seed_spread

args = bench.parse()
args.sort_init = 0
cfg, gmesh, gef, qm, dt, cluster, name = bench.workload(args, 1)
torch.cuda.set_device(0)
stream = torch.cuda.Stream()
args.steps, args.reps = 40, 1
R = bench.EsRank(args, cfg, gmesh, gef, 1, 0, stream, cluster=cluster)
if os.environ.get("PROBE_L2FETCH"):
    # cudaLimitMaxL2FetchGranularity = 0x05 (bytes: 0..128)
    import ctypes
    rt = ctypes.CDLL("libcudart.so")
    v = ctypes.c_size_t()
    rt.cudaDeviceGetLimit(ctypes.byref(v), 5)
    print("L2 fetch granularity was", v.value, flush=True)
    rc = rt.cudaDeviceSetLimit(5, ctypes.c_size_t(int(os.environ["PROBE_L2FETCH"])))
    rt.cudaDeviceGetLimit(ctypes.byref(v), 5)
    print("set rc", rc, "now", v.value, flush=True)
sim = R.sim
out = {}
with torch.cuda.stream(stream):
    sim.step(0.0, 1.0, cfg["w"], stats=False, fill=True)
    sim.sort_by_cell()
    stream.synchronize()
    s = 0
    for age in [int(x) for x in os.environ.get("PROBE_AGES", "0,0,1,3,5,10").split(",")]:
        for _ in range(age):
            R.one_step(s)
            s += 1
        stream.synchronize()
        sim.phase_timing(True)
        sim.phase_times()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        sim.sort_by_cell()
        e1.record(stream)
        stream.synchronize()
        ph = sim.phase_times()
        sim.phase_timing(False)
        out.setdefault(str(age), []).append({"ms": e0.elapsed_time(e1),
                                             **{k: v[0] for k, v in ph.items() if v[1]}})
        print(age, out[str(age)][-1], flush=True)
print(json.dumps(out))

if os.environ.get("PROBE_REUSE"):
    # reuse distance of the sort's gather: for every 128-B line of a source
    # column (16 particles of 8 B), the spread of the destinations that read it
    from paper_conf_icpp_lantra0m24_b200 import opp as O

    class _Arr:
        def __init__(self, ptr, n, typestr):
            self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False),
                                             "version": 3}

    def col(h, n, typestr):
        return torch.as_tensor(_Arr(O.opp_get_dat_device_ptr(sim.ctx, h)[0], n, typestr), device="cuda").clone()

    with torch.cuda.stream(stream):
        for age in [int(x) for x in os.environ["PROBE_REUSE"].split(",")]:
            for _ in range(age):
                R.one_step(s)
                s += 1
            stream.synchronize()
            n = sim.count()
            before = col(sim.pid, n, "<i8")
            sim.sort_by_cell()
            stream.synchronize()
            n2 = sim.count()
            after = col(sim.pid, n2, "<i8")
            lo = int(min(before.min().item(), after.min().item()))
            inv = torch.full((int(max(before.max().item(), after.max().item())) - lo + 1,), -1,
                             dtype=torch.int64, device="cuda")
            inv[before - lo] = torch.arange(n, device="cuda")
            src = inv[after - lo]
            del inv, before, after
            d = torch.arange(n2, device="cuda", dtype=torch.int64)
            moved = (src != d).double().mean().item()
            far = ((src - d).abs() > 1_000_000).double().mean().item()
            line = src.div_(16, rounding_mode="floor")
            nl = int(line.max().item()) + 1
            mn = torch.full((nl,), 1 << 62, dtype=torch.int64, device="cuda").scatter_reduce(0, line, d, "amin")
            mx = torch.full((nl,), -1, dtype=torch.int64, device="cuda").scatter_reduce(0, line, d, "amax")
            ok = mx >= 0
            spread = (mx - mn)[ok].double()
            q = torch.quantile(spread[torch.randint(0, spread.numel(), (1 << 22,), device="cuda")],
                               torch.tensor([0.5, 0.75, 0.9, 0.99], dtype=torch.float64, device="cuda"))
            print("reuse age", age, "line spread quantiles (dst particles) 50/75/90/99%:",
                  [int(x) for x in q.tolist()], "frac moved", round(moved, 3), "frac |src-dst|>1M", round(far, 4),
                  flush=True)
            del src, line, d, mn, mx, spread
