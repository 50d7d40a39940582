"""CPU oracle -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.

ctypes wrapper over ``oracle/liboracle.so`` (plain C, ``oracle.c``).  Only
``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product library never links, loads or calls it, and it never calls the
product library.

Parity status: every exported function is pinned by ``tests/test_oracle_pins.py``
against the paper and the mathematics (brute-force point location, the Kuhn
closed-form location, the ballistic and uniform-field leap-frog closed forms,
barycentric identities, exact charge conservation, bookkeeping); see
DESIGN.md §4.  No function here is "parity unpinned".
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

ORC_DONE, ORC_REMOVE = 0, 2


CC = "gcc"
CFLAGS = ["-O2", "-ffp-contract=off", "-std=c99", "-Wall"]


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc, -O2 -ffp-contract=off: no FMA, S11)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call([CC, *CFLAGS, "-shared", "-fPIC", _SRC, "-o", _LIB, "-lm"])
    return _LIB


def build_info() -> dict:
    """Compiler and flags of the oracle build (reported with cpu_baseline)."""
    try:
        ver = subprocess.run([CC, "--version"], capture_output=True, text=True).stdout.split("\n")[0]
    except Exception:   # noqa: BLE001
        ver = CC
    return {"compiler": ver, "flags": " ".join(CFLAGS)}


class _Params(C.Structure):
    _fields_ = [("c1", C.c_double), ("dt", C.c_double), ("w", C.c_double),
                ("hcap", C.c_int32), ("use_dh", C.c_int32), ("zero_charge", C.c_int32),
                ("pad", C.c_int32)]


class _Stats(C.Structure):
    _fields_ = [("n_before", C.c_int64), ("n_injected", C.c_int64), ("n_removed", C.c_int64),
                ("n_after", C.c_int64), ("total_hops", C.c_int64), ("n_capped", C.c_int64),
                ("max_hops", C.c_int32), ("pad", C.c_int32)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P, i32, i64, d = C.c_void_p, C.c_int32, C.c_int64, C.c_double
        sig = {
            "orc_mesh_new": (P, [i64, P, i64, P, P]),
            "orc_mesh_free": (None, [P]),
            "orc_mesh_geometry": (None, [P, P, P, P]),
            "orc_mesh_set_field": (None, [P, P]),
            "orc_bary": (None, [P, i32, P, P]),
            "orc_locate_brute": (i32, [P, P, d]),
            "orc_walk": (C.c_int, [P, i32, P, i32, i32, P, P, P, P]),
            "orc_overlay_build": (C.c_int, [P, P, d, P]),
            "orc_overlay_get": (None, [P, P]),
            "orc_parts_new": (P, []),
            "orc_parts_free": (None, [P]),
            "orc_parts_count": (i64, [P]),
            "orc_parts_removed": (i64, [P, P, P]),
            "orc_parts_append": (C.c_int, [P, i64, P, P, P, P]),
            "orc_parts_get": (None, [P, P, P, P, P, P]),
            "orc_step": (C.c_int, [P, P, P, P, P]),
        }
        for name, (res, args) in sig.items():
            f = getattr(_lib, name)
            f.restype = res
            f.argtypes = args
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


class Mesh:
    """Oracle-side mesh: copies node_xyz, c2n, c2c; derives its own geometry."""

    def __init__(self, node_xyz, c2n, c2c):
        self._xyz = np.ascontiguousarray(node_xyz, dtype=np.float64)
        self._c2n = np.ascontiguousarray(c2n, dtype=np.int32)
        self._c2c = np.ascontiguousarray(c2c, dtype=np.int32)
        self.nn, self.nc = self._xyz.shape[0], self._c2n.shape[0]
        self.h = lib().orc_mesh_new(self.nn, _p(self._xyz), self.nc, _p(self._c2n), _p(self._c2c))
        if not self.h:
            raise MemoryError("orc_mesh_new")
        self.overlay = None

    @classmethod
    def from_gen(cls, mesh: dict) -> "Mesh":
        return cls(mesh["node_xyz"], mesh["c2n"], mesh["c2c"])

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.orc_mesh_free(self.h)
            self.h = None

    def geometry(self):
        g = np.empty((self.nc, 9))
        p0 = np.empty((self.nc, 3))
        v6 = np.empty(self.nc)
        lib().orc_mesh_geometry(self.h, _p(g), _p(p0), _p(v6))
        return g, p0, v6

    def set_field(self, ef):
        ef = np.ascontiguousarray(ef, dtype=np.float64).reshape(self.nc, 3)
        lib().orc_mesh_set_field(self.h, _p(ef))

    def bary(self, cell: int, x) -> np.ndarray:
        x = np.ascontiguousarray(x, dtype=np.float64)
        lam = np.empty(4)
        lib().orc_bary(self.h, int(cell), _p(x), _p(lam))
        return lam

    def locate_brute(self, x, tol: float = 0.0) -> int:
        x = np.ascontiguousarray(x, dtype=np.float64)
        return int(lib().orc_locate_brute(self.h, _p(x), float(tol)))

    def walk(self, cell: int, x, hcap: int = 1024, hops0: int = 0):
        x = np.ascontiguousarray(x, dtype=np.float64)
        oc, oh, cap = C.c_int32(), C.c_int32(), C.c_int32()
        lam = np.empty(4)
        st = lib().orc_walk(self.h, int(cell), _p(x), int(hops0), int(hcap), C.byref(oc),
                            C.byref(oh), _p(lam), C.byref(cap))
        return st, oc.value, oh.value, lam, cap.value

    def build_overlay(self, x0, dx: float, n):
        x0 = np.ascontiguousarray(x0, dtype=np.float64)
        n = np.ascontiguousarray(n, dtype=np.int32)
        if lib().orc_overlay_build(self.h, _p(x0), float(dx), _p(n)):
            raise MemoryError("orc_overlay_build")
        out = np.empty(int(np.prod(n)), dtype=np.int32)
        lib().orc_overlay_get(self.h, _p(out))
        self.overlay = (x0.copy(), float(dx), tuple(int(v) for v in n))
        return out


class Particles:
    def __init__(self):
        self.h = lib().orc_parts_new()

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.orc_parts_free(self.h)
            self.h = None

    def __len__(self):
        return int(lib().orc_parts_count(self.h))

    def append(self, pos, vel, cell, ids):
        pos = np.ascontiguousarray(pos, dtype=np.float64)
        vel = np.ascontiguousarray(vel, dtype=np.float64)
        cell = np.ascontiguousarray(cell, dtype=np.int32)
        ids = np.ascontiguousarray(ids, dtype=np.int64)
        n = cell.shape[0]
        if lib().orc_parts_append(self.h, n, _p(pos), _p(vel), _p(cell), _p(ids)):
            raise MemoryError("orc_parts_append")

    def get(self) -> dict:
        n = len(self)
        out = {"pos": np.empty((n, 3)), "vel": np.empty((n, 3)),
               "cell": np.empty(n, np.int32), "id": np.empty(n, np.int64),
               "margin": np.empty(n)}
        lib().orc_parts_get(self.h, _p(out["pos"]), _p(out["vel"]), _p(out["cell"]),
                            _p(out["id"]), _p(out["margin"]))
        return out

    def removed(self):
        n = int(lib().orc_parts_removed(self.h, None, None))
        ids, mg = np.empty(n, np.int64), np.empty(n)
        lib().orc_parts_removed(self.h, _p(ids), _p(mg))
        return ids, mg


def step(mesh: Mesh, parts: Particles, c1: float, dt: float, w: float, Q: np.ndarray,
         hcap: int = 1024, use_dh: int = 0, zero_charge: bool = True) -> dict:
    """One oracle time step on an already-injected population (orc_step).
    use_dh: 0 multi-hop only, 1 overlay seed for every particle, 2 overlay
    seed only for particles no longer inside their cell (reading S19'')."""
    assert Q.dtype == np.float64 and Q.flags.c_contiguous and Q.shape[0] == mesh.nn
    if use_dh and mesh.overlay is None:
        raise ValueError("build_overlay first")
    prm = _Params(float(c1), float(dt), float(w), int(hcap), int(use_dh),
                  int(bool(zero_charge)), 0)
    st = _Stats()
    lib().orc_step(mesh.h, parts.h, C.byref(prm), _p(Q), C.byref(st))
    return {k: getattr(st, k) for k, _ in _Stats._fields_ if k != "pad"}
