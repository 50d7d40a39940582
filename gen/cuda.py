"""Device twin of the seeded generators (gen/gen_cuda.cu -> gen/libgen_cuda.so).

Input generation only; bit-identical to gen.seed_particles / gen.inject_batch
(tests/test_gen_cuda.py).  Returns torch CUDA tensors (AoS pos/vel).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen_cuda.cu")
_LIB = os.path.join(_HERE, "libgen_cuda.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a",
                               "-O3", "-lineinfo", "-Xcompiler", "-fPIC", "-shared", "-cudart", "static",
                               _SRC, "-o", _LIB])
    return _LIB


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P, L, U, D = C.c_void_p, C.c_longlong, C.c_ulonglong, C.c_double
        _lib.gen_seed_particles.argtypes = [P, P, L, L, L, U, D, D, L, P, L, D, P, P, P, P, P]
        _lib.gen_inject_batch.argtypes = [P, P, L, L, L, U, D, L, P, P, P, P, P]
        I = C.c_int
        _lib.gen_em_two_stream.argtypes = [I, I, I, I, U, D, D, D, P, P, P, P, P, P]
    return _lib


class DeviceMesh:
    """The generator's view of a gen.kuhn_duct mesh on the device."""

    def __init__(self, mesh: dict, device="cuda"):
        import torch
        self.xyz = torch.from_numpy(mesh["node_xyz"]).to(device)
        self.c2n = torch.from_numpy(mesh["c2n"]).to(device)
        self.inlet = torch.from_numpy(mesh["inlet"]).to(device)
        self.nc = int(mesh["n_cells"])
        self.nf = int(mesh["inlet"].shape[0])
        self.device = device


def _out(n, device):
    import torch
    return {"pos": torch.empty((n, 3), dtype=torch.float64, device=device),
            "vel": torch.empty((n, 3), dtype=torch.float64, device=device),
            "cell": torch.empty(n, dtype=torch.int32, device=device),
            "id": torch.empty(n, dtype=torch.int64, device=device)}


def seed_particles(dm: DeviceMesh, n: int, seed: int, drift=0.25, spread=0.05, id_base=0,
                   cluster=None, stream=None, first=0):
    """Particles [first, first + n) of the seeded population (chunks of a
    large population are bit-identical to generating it at once)."""
    import torch
    o = _out(n, dm.device)
    hot_t, nhot, frac = None, 0, 0.0
    if cluster is not None:
        frac, hot = cluster
        hot_t = torch.from_numpy(np.asarray(hot, dtype=np.int64)).to(dm.device)
        nhot = hot_t.numel()
    s = stream if stream is not None else torch.cuda.current_stream().cuda_stream
    rc = lib().gen_seed_particles(dm.xyz.data_ptr(), dm.c2n.data_ptr(), dm.nc, first, n, seed, drift, spread,
                                  id_base, hot_t.data_ptr() if hot_t is not None else None, nhot,
                                  float(frac), o["pos"].data_ptr(), o["vel"].data_ptr(),
                                  o["cell"].data_ptr(), o["id"].data_ptr(), s)
    if rc:
        raise RuntimeError(f"gen_seed_particles: cuda error {rc}")
    o["_keep"] = hot_t
    return o


def inject_batch(dm: DeviceMesh, step: int, n_inj: int, seed: int, v_inj=0.25, id_base=0,
                 stream=None):
    import torch
    o = _out(n_inj, dm.device)
    s = stream if stream is not None else torch.cuda.current_stream().cuda_stream
    rc = lib().gen_inject_batch(dm.xyz.data_ptr(), dm.inlet.data_ptr(), dm.nf, step, n_inj, seed,
                                v_inj, id_base, o["pos"].data_ptr(), o["vel"].data_ptr(),
                                o["cell"].data_ptr(), o["id"].data_ptr(), s)
    if rc:
        raise RuntimeError(f"gen_inject_batch: cuda error {rc}")
    return o


def em_two_stream(nx: int, ny: int, nz: int, ppc: int, seed: int, v0: float = 0.2,
                  pert: float = 0.01, vth: float = 0.01, w: float = 1.0, device="cuda",
                  stream=None) -> dict:
    """Device twin of gen.em.two_stream (SoA torch tensors off[3][n], u[3][n], w, cell)."""
    import torch
    from .em import pert_table
    n = nx * ny * nz * ppc
    tab = torch.from_numpy(pert_table(nz, v0, pert)).to(device)
    o = {"off": torch.empty((3, n), dtype=torch.float64, device=device),
         "u": torch.empty((3, n), dtype=torch.float64, device=device),
         "w": torch.empty(n, dtype=torch.float64, device=device),
         "cell": torch.empty(n, dtype=torch.int32, device=device), "n": n}
    s = stream if stream is not None else torch.cuda.current_stream().cuda_stream
    rc = lib().gen_em_two_stream(nx, ny, nz, ppc, seed, v0, vth, w, tab.data_ptr(),
                                 o["off"].data_ptr(), o["u"].data_ptr(), o["w"].data_ptr(),
                                 o["cell"].data_ptr(), s)
    if rc:
        raise RuntimeError(f"gen_em_two_stream: cuda error {rc}")
    o["_keep"] = tab
    return o
