"""Host-side plumbing of the multi-GPU path (no compute).

The mesh is partitioned into contiguous z-slabs of hex layers -- the paper's
custom partition "along the principal direction of motion of particles"
 -- one slab per rank.  Because cells are numbered
z-major, a slab is one contiguous global cell range, so the owner of any cell
is a closed form and the library needs no rank map (what the paper's
direct-hop global move keeps an MPI-RMA rank-map for).

This module only cuts inputs and moves host metadata: slab extraction,
particle ownership, the unique-id broadcast, result gathering and the
max-over-ranks timing reduction.  Everything on the particle path runs in
libopp's kernels; the exchange between ranks is NCCL inside libopp.
"""
from __future__ import annotations

import numpy as np


def layer_bounds(nz: int, nranks: int):
    """Hex-layer range [k0, k1) of every rank (as even as possible)."""
    return [((r * nz) // nranks, ((r + 1) * nz) // nranks) for r in range(nranks)]


def rank_of_cell(mesh: dict, nranks: int) -> np.ndarray:
    """rank_of_cell[g] for every global cell (the opp_set_partition input)."""
    cpl = 6 * mesh["nx"] * mesh["ny"]
    out = np.empty(mesh["n_cells"], dtype=np.int32)
    for r, (k0, k1) in enumerate(layer_bounds(mesh["nz"], nranks)):
        out[k0 * cpl:k1 * cpl] = r
    return out


def slab(mesh: dict, nranks: int, rank: int, rank_of_cell_: np.ndarray | None = None) -> dict:
    """Rank `rank`'s slab of a global gen.kuhn_duct mesh.

    Local cells are the global range [cell_base, cell_base + n_cells) in
    order; c2c keeps GLOBAL cell ids (neighbours on other ranks included);
    c2n is renumbered to the slab's own nodes, whose global ids are in
    node_gid (interface-plane nodes appear on both neighbouring ranks).
    rank_of_cell_: any partition into contiguous cell ranges (default: whole
    hex layers, rank_of_cell); ranges that cut layers make some nodes shared
    by more than two ranks."""
    cpl = 6 * mesh["nx"] * mesh["ny"]
    if rank_of_cell_ is None:
        k0, k1 = layer_bounds(mesh["nz"], nranks)[rank]
        lo, hi = k0 * cpl, k1 * cpl
        roc = rank_of_cell(mesh, nranks)
    else:
        roc = np.ascontiguousarray(rank_of_cell_, dtype=np.int32)
        mine = np.nonzero(roc == rank)[0]
        lo, hi = int(mine[0]), int(mine[-1]) + 1
        k0, k1 = lo // cpl, -(-hi // cpl)
    c2n_g = mesh["c2n"][lo:hi]
    gid = np.unique(c2n_g)
    c2n_l = np.searchsorted(gid, c2n_g).astype(np.int32)
    inl = mesh["inlet"]
    inl = inl[(inl[:, 0] >= lo) & (inl[:, 0] < hi)]
    inl_local = inl.copy()
    inl_local[:, 0] -= lo
    inl_local[:, 1:] = np.searchsorted(gid, inl[:, 1:])
    return {
        "nx": mesh["nx"], "ny": mesh["ny"], "nz": k1 - k0, "h": mesh["h"],
        "node_xyz": np.ascontiguousarray(mesh["node_xyz"][gid]),
        "c2n": np.ascontiguousarray(c2n_l),
        "c2c": np.ascontiguousarray(mesh["c2c"][lo:hi]),
        "n_cells": hi - lo, "n_nodes": int(gid.size),
        "node_gid": gid.astype(np.int64), "cell_base": lo,
        "n_cells_global": mesh["n_cells"], "rank_of_cell": roc,
        "inlet": inl, "inlet_local": np.ascontiguousarray(inl_local), "box": mesh["box"],
        "rank": rank, "nranks": nranks,
        "layers": (k0, k1),
    }


def owned(batch: dict, rank_of_cell_: np.ndarray, rank: int) -> dict:
    """The particles of `batch` whose (global) cell this rank owns."""
    m = rank_of_cell_[batch["cell"]] == rank
    return {k: (v[m] if isinstance(v, np.ndarray) else v) for k, v in batch.items()}


def local_field(ef_global: np.ndarray, sl: dict) -> np.ndarray:
    lo = sl["cell_base"]
    return np.ascontiguousarray(ef_global[lo:lo + sl["n_cells"]])


def global_node_charge(parts, n_nodes_global: int):
    """Assemble global node charge from per-rank (node_gid, Q) pairs; the
    interface copies must agree (the halo makes them bit-identical)."""
    Q = np.full(n_nodes_global, np.nan)
    for gid, q in parts:
        prev = Q[gid]
        seen = ~np.isnan(prev)
        if np.any(prev[seen] != q[seen]):
            raise AssertionError("interface node charge differs between ranks")
        Q[gid] = q
    Q[np.isnan(Q)] = 0.0
    return Q


def merge_particles(parts) -> dict:
    out = {k: np.concatenate([p[k] for p in parts]) for k in parts[0]}
    o = np.argsort(out["id"], kind="stable")
    return {k: v[o] for k, v in out.items()}


# ------------------------------------------------------------ torch.distributed
def broadcast_bytes(data: bytes | None, src: int = 0) -> bytes:
    """Broadcast a small byte string (the 128-byte NCCL unique id) from src
    over the default process group (gloo or nccl)."""
    import torch.distributed as dist
    obj = [data]
    dist.broadcast_object_list(obj, src=src)
    return obj[0]


def max_over_ranks(value: float) -> float:
    """Max of a per-rank scalar (device timings are reported as the max)."""
    import torch
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([float(value)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(value: int) -> int:
    import torch
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([int(value)], dtype=torch.int64, device=dev)
    dist.all_reduce(t)
    return int(t.item())
