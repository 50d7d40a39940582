"""Host-side multi-rank plumbing under torch.distributed gloo, world size 2,
on CPU (-m "not gpu"): slab partition, ownership of particles, the halo node
sets, the unique-id broadcast and the max/sum-over-ranks reductions bench.py
uses for N > 1.  (The device side of migration and halo is covered on one GPU
by tests/test_gpu_multirank.py through the loopback transport.)"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist
    import gen
    from paper_conf_icpp_lantra0m24_b200 import dist as D
    try:
        dist.init_process_group("gloo", rank=rank, world_size=world)
        mesh = gen.kuhn_duct(4, 3, 9, jitter=0.2, seed=2)
        sl = D.slab(mesh, world, rank)
        res = {}
        # 1. slabs tile the global cell range, in rank order
        rng = [None] * world
        dist.all_gather_object(rng, (sl["cell_base"], sl["cell_base"] + sl["n_cells"]))
        res["ranges"] = rng
        # 2. halo: the nodes both ranks hold are exactly the interface plane
        gids = [None] * world
        dist.all_gather_object(gids, sl["node_gid"].tolist())
        res["shared"] = sorted(set(gids[0]) & set(gids[1]))
        # 3. every particle is owned by exactly one rank
        p = gen.seed_particles(mesh, 5000, 3)
        mine = D.owned(p, sl["rank_of_cell"], rank)
        res["owned_total"] = D.sum_over_ranks(mine["cell"].shape[0])
        res["owned_ok"] = bool(np.all((mine["cell"] >= sl["cell_base"]) &
                                      (mine["cell"] < sl["cell_base"] + sl["n_cells"])))
        # 4. unique-id broadcast (the 128-byte NCCL id travels this way)
        uid = os.urandom(128) if rank == 0 else None
        got = D.broadcast_bytes(uid)
        allu = [None] * world
        dist.all_gather_object(allu, got)
        res["uid_same"] = len(got) == 128 and all(u == allu[0] for u in allu)
        # 5. timing reduction: max over ranks
        res["max"] = D.max_over_ranks(10.0 + rank)
        # 6. local c2n refers to local nodes with the right coordinates
        res["coords_ok"] = bool(np.array_equal(sl["node_xyz"][sl["c2n"]],
                                               mesh["node_xyz"][mesh["c2n"][sl["cell_base"]:sl["cell_base"] + sl["n_cells"]]]))
        q.put((rank, res))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:   # noqa: BLE001
        q.put((rank, {"error": repr(e)}))


def test_gloo_two_ranks_plumbing():
    import gen
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = dict(q.get(timeout=180) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    for r in range(world):
        assert "error" not in out[r], out[r]
    mesh = gen.kuhn_duct(4, 3, 9, jitter=0.2, seed=2)
    r0 = out[0]
    assert r0["ranges"][0][0] == 0 and r0["ranges"][0][1] == r0["ranges"][1][0]
    assert r0["ranges"][1][1] == mesh["n_cells"]
    # interface plane: z = k1 of rank 0 (layers 0..3 | 4..8): (4+1)*(3+1) nodes
    k = 9 // 2
    plane = [i + 5 * (j + 4 * k) for j in range(4) for i in range(5)]
    assert r0["shared"] == sorted(plane)
    assert r0["owned_total"] == 5000 and all(out[r]["owned_ok"] for r in range(world))
    assert all(out[r]["uid_same"] for r in range(world))
    assert all(out[r]["max"] == 11.0 for r in range(world))
    assert all(out[r]["coords_ok"] for r in range(world))
