"""A small C1-style run for compute-sanitizer (tests/test_gpu_sanitize.py):
the TMA-pipelined pass 1 (stages, mbarriers, per-warp rings and hop queues),
the continuation, hole fill, a periodic sort and the warp-aggregated and SR
deposits, on a jittered Kuhn duct.  No torch: the library allocates with
cudaMalloc on the default stream.  Exits 0 when the run matches the oracle's
particle count."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import gen  # noqa: E402
from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic  # noqa: E402


def main(dep: int, dh: int, lead: float = 0.0):
    mesh = gen.kuhn_duct(4, 4, 12, jitter=0.2, seed=3)
    ef = np.random.default_rng(3).uniform(-2e-3, 2e-3, (mesh["n_cells"], 3))
    init = gen.seed_particles(mesh, 20_000, 3, drift=0.4, spread=0.1)
    sim = MiniFemPic(mesh, ef, torch_alloc=False, deposit_mode=dep, direct_hop=dh, overlay_spacing=0.25,
                     sort_every=2, hop_budget=2, sort_lead=lead if dh else 0.0)
    sim.inject(init)
    for s in range(3):
        sim.inject(gen.inject_batch(mesh, s, 300, 3, id_base=20_000))
        st = sim.step(1.0, 0.5, 1.0)
    n = sim.count()
    sim.close()
    assert n == st["n_after"] and n > 10_000, (n, st)
    print("sanitize case ok", n)


if __name__ == "__main__":
    main(int(sys.argv[1]) if len(sys.argv) > 1 else 1, int(sys.argv[2]) if len(sys.argv) > 2 else 1,
         float(sys.argv[3]) if len(sys.argv) > 3 else 0.0)
