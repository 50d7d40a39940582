"""CabanaPIC-style electromagnetic application (config C3) on the libopp C ABI.

The periodic hex grid is declared as an unstructured mesh by its cell-to-cell
map; per step the application runs the
library's Move_Deposit on device-resident SoA particle
columns.  This module only marshals arguments: Interpolate and Move_Deposit
run in libopp's CUDA kernels (csrc/opp_em.cu); PyTorch holds the device
memory and the stream.  ``field_step`` runs the field side (AccumulateCurrent,
AdvanceB / AdvanceE leap-frog, Interpolate) in the library's kernels too.
"""
from __future__ import annotations

import numpy as np

from . import opp as O
from .app import _torch_allocator


class CabanaPicEM:
    """One rank of the EM loop.  nranks > 1 (or slab given): this rank owns the
    z-layers slab = (k0, k1) of the global grid (opp_em_set_partition); e, b
    are the GLOBAL fields; particles are this rank's (cells in its layers),
    kept in columns of capacity `capacity` with an id each; step() and
    field_step() run the slab forms (migration, Update_Ghosts)."""

    def __init__(self, nx: int, ny: int, nz: int, c2c: np.ndarray, e: np.ndarray, b: np.ndarray,
                 qdt_2mc: float, cdt_2h, qsp: float = 1.0, kcap: int = 16,
                 deposit_mode: int = O.OPP_DEP_ATOMIC_WARPAGG, device: int = 0, nranks: int = 1,
                 rank: int = 0, uid: bytes | None = None, transport: int = 0, slab=None,
                 stream=None, torch_alloc: bool = True):
        import ctypes as C
        import torch
        self.torch = torch
        self.dev = torch.device("cuda", device)
        p = O.opp_init_params_default()
        p.device = device
        p.cuda_stream = stream if stream is not None else torch.cuda.current_stream(self.dev).cuda_stream
        self._cb = None
        if torch_alloc:
            self._cb = _torch_allocator()
            p.alloc, p.free = self._cb
        p.nranks, p.rank, p.transport = int(nranks), int(rank), int(transport)
        self._uid = None
        if nranks > 1:
            self._uid = C.create_string_buffer(bytes(uid), 128)
            p.nccl_unique_id = C.cast(self._uid, C.c_void_p)
        self.ctx = O.opp_init(p)
        self.slab = slab if slab is not None else ((0, nz) if nranks > 1 else None)
        if self.slab is not None:
            O.opp_em_set_partition(self.ctx, nx, ny, nz, self.slab[0], self.slab[1])
        self.nx, self.ny, self.nz = nx, ny, nz
        self.nc = nx * ny * nz
        self.c2c = torch.from_numpy(np.ascontiguousarray(c2c, np.int32)).to(self.dev)
        self.e = torch.from_numpy(np.ascontiguousarray(e, np.float64)).to(self.dev)
        self.b = torch.from_numpy(np.ascontiguousarray(b, np.float64)).to(self.dev)
        self.interp = torch.empty((self.nc, 18), dtype=torch.float64, device=self.dev)
        self.acc = torch.zeros((self.nc, 12), dtype=torch.float64, device=self.dev)
        self.params = O.opp_em_params_make(qdt_2mc, cdt_2h, qsp, kcap, deposit_mode)
        self.interpolate()
        self.n = 0

    def interpolate(self) -> None:
        O.opp_em_interpolate(self.ctx, self.nx, self.ny, self.nz, self.e, self.b, self.interp)

    def set_particles(self, off, u, w, cell, ids=None, capacity: int = 0) -> None:
        """Host arrays off[3][n], u[3][n], w[n], cell[n] or device tensors of those shapes
        (slabs: columns of `capacity` >= n rows, ids carried along)."""
        t = self.torch

        def dev(a, dt):
            if isinstance(a, t.Tensor):
                return a.to(self.dev, dt).contiguous()
            return t.from_numpy(np.ascontiguousarray(a)).to(self.dev, dt)
        n = int(np.asarray(cell).shape[0]) if not isinstance(cell, t.Tensor) else int(cell.shape[0])
        self.n = n
        if self.slab is None:
            self.off, self.u = dev(off, t.float64), dev(u, t.float64)
            self.w, self.cell = dev(w, t.float64), dev(cell, t.int32)
            self.cap = n
            return
        cap = max(int(capacity), n, 1)
        self.cap = cap
        self.off = t.zeros((3, cap), dtype=t.float64, device=self.dev)
        self.u = t.zeros((3, cap), dtype=t.float64, device=self.dev)
        self.w = t.zeros(cap, dtype=t.float64, device=self.dev)
        self.cell = t.full((cap,), -1, dtype=t.int32, device=self.dev)
        self.pid = t.zeros(cap, dtype=t.int64, device=self.dev)
        self.off[:, :n] = dev(off, t.float64)
        self.u[:, :n] = dev(u, t.float64)
        self.w[:n] = dev(w, t.float64)
        self.cell[:n] = dev(cell, t.int32)
        self.pid[:n] = dev(ids if ids is not None else np.arange(n), t.int64)

    def step(self, want_stats: bool = False):
        if self.slab is not None:
            self.n, st = O.opp_em_move_deposit_slab(self.ctx, self.n, self.cap, self.off, self.u, self.w,
                                                    self.cell, self.pid, self.interp, self.c2c, self.nc,
                                                    self.acc, self.params, want_stats)
        else:
            st = O.opp_em_move_deposit(self.ctx, self.n, self.n, self.off, self.u, self.w, self.cell,
                                       self.interp, self.c2c, self.nc, self.acc, self.params, want_stats)
        return st.as_dict() if st is not None else None

    def sort_by_cell(self) -> None:
        """Group the particles by cell (opp_em_sort_by_cell into spare columns, then swap)."""
        if self.slab is not None:
            raise NotImplementedError("sort_by_cell: single domain only (the sort does not carry ids)")
        t = self.torch
        if getattr(self, "_alt", None) is None or self._alt[3].shape[0] != self.n:
            self._alt = (t.empty_like(self.off), t.empty_like(self.u), t.empty_like(self.w),
                         t.empty_like(self.cell))
        ao, au, aw, ac = self._alt
        O.opp_em_sort_by_cell(self.ctx, self.n, self.n, self.off, self.u, self.w, self.cell, self.nc,
                              ao, au, aw, ac)
        self._alt = (self.off, self.u, self.w, self.cell)
        self.off, self.u, self.w, self.cell = ao, au, aw, ac

    def field_step(self, dt: float, h=(1.0, 1.0, 1.0)) -> None:
        """AccumulateCurrent -> AdvanceB(dt/2) -> AdvanceE(dt) -> AdvanceB(dt/2) ->
        Interpolate, then the accumulator is cleared for the next Move_Deposit."""
        c = self.ctx
        if getattr(self, "J", None) is None:
            self.J = self.torch.empty_like(self.e)
        if self.slab is not None:
            O.opp_em_field_step_slab(c, self.e, self.b, self.J, self.acc, self.interp, self.c2c, self.nc,
                                     h, dt)
            return
        O.opp_em_accumulate_current(c, self.acc, self.c2c, self.nc, h, dt, self.J)
        O.opp_em_advance_b(c, self.e, self.b, self.c2c, self.nc, h, dt / 2)
        O.opp_em_advance_e(c, self.e, self.b, self.J, self.c2c, self.nc, h, dt)
        O.opp_em_advance_b(c, self.e, self.b, self.c2c, self.nc, h, dt / 2)
        self.interpolate()
        self.acc.zero_()

    def zero_acc(self) -> None:
        self.acc.zero_()

    def state(self) -> dict:
        self.torch.cuda.synchronize(self.dev)
        if self.slab is not None:
            n = self.n
            return {"off": self.off[:, :n].cpu().numpy(), "u": self.u[:, :n].cpu().numpy(),
                    "cell": self.cell[:n].cpu().numpy(), "id": self.pid[:n].cpu().numpy(),
                    "acc": self.acc.cpu().numpy()}
        return {"off": self.off.cpu().numpy(), "u": self.u.cpu().numpy(),
                "cell": self.cell.cpu().numpy(), "acc": self.acc.cpu().numpy()}

    def launches(self) -> int:
        return O.opp_kernel_launch_count(self.ctx)

    def close(self) -> None:
        if self.ctx:
            O.opp_finalize(self.ctx)
            self.ctx = None
