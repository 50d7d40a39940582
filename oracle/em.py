"""CPU oracle of the CabanaPIC-style EM Move_Deposit -- TEST INFRASTRUCTURE.

ctypes wrapper over ``oracle/liboracle_em.so`` (plain C, ``em.c``).  Same
rules as the package: only tests/, smoke() and bench.py's cpu_baseline /
--impl reference legs may import it.  Every function is pinned by
tests/test_oracle_em.py.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "em.c")
_LIB = os.path.join(_HERE, "liboracle_em.so")
NI, NA = 18, 12


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-std=c99", "-Wall",
                               "-shared", "-fPIC", _SRC, "-o", _LIB, "-lm"])
    return _LIB


class Params(C.Structure):
    _fields_ = [("qdt_2mc", C.c_double), ("cdt_2h", C.c_double * 3), ("qsp", C.c_double),
                ("kcap", C.c_int32), ("pad", C.c_int32)]


class Stats(C.Structure):
    _fields_ = [("n_crossings", C.c_int64), ("n_capped", C.c_int64),
                ("max_crossings", C.c_int32), ("pad", C.c_int32)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P = C.c_void_p
        _lib.em_move_deposit.argtypes = [C.c_int64, P, P, P, P, P, P, P, P, P]
        _lib.em_move_deposit.restype = None
        _lib.em_boris.argtypes = [P, C.c_double, P]
        _lib.em_segment_current.argtypes = [P, P, C.c_double, P]
        _lib.em_interpolate.argtypes = [C.c_int, C.c_int, C.c_int, P, P, P]
    return _lib


def _p(a):
    return a.ctypes.data_as(C.c_void_p)


def params(qdt_2mc: float, cdt_2h, qsp: float, kcap: int = 16) -> Params:
    return Params(qdt_2mc, (C.c_double * 3)(*cdt_2h), qsp, kcap, 0)


def move_deposit(prm: Params, off, u, w, cell, interp, c2c, acc) -> dict:
    """One step in place: off[3][n], u[3][n] float64, w[n], cell[n] int32,
    interp[nc][18], c2c[nc][6] int32, acc[nc][12] (added to)."""
    n = int(cell.shape[0])
    for a, dt in ((off, np.float64), (u, np.float64), (w, np.float64), (cell, np.int32),
                  (interp, np.float64), (c2c, np.int32), (acc, np.float64)):
        assert a.dtype == dt and a.flags.c_contiguous
    st = Stats()
    lib().em_move_deposit(n, _p(off), _p(u), _p(w), _p(cell), _p(interp), _p(c2c), _p(acc),
                          C.byref(prm), C.byref(st))
    return {"n_crossings": st.n_crossings, "n_capped": st.n_capped, "max_crossings": st.max_crossings}


def boris(fields6, qdt_2mc: float, u) -> np.ndarray:
    f = np.ascontiguousarray(fields6, dtype=np.float64)
    uu = np.array(u, dtype=np.float64)
    lib().em_boris(_p(f), qdt_2mc, _p(uu))
    return uu


def segment_current(p, q, Q: float) -> np.ndarray:
    acc = np.zeros(NA)
    pp, qq = np.array(p, dtype=np.float64), np.array(q, dtype=np.float64)
    lib().em_segment_current(_p(pp), _p(qq), Q, _p(acc))
    return acc


def interpolate(nx: int, ny: int, nz: int, e, b) -> np.ndarray:
    nc = nx * ny * nz
    out = np.zeros((nc, NI))
    e = np.ascontiguousarray(e, dtype=np.float64)
    b = np.ascontiguousarray(b, dtype=np.float64)
    lib().em_interpolate(nx, ny, nz, _p(e), _p(b), _p(out))
    return out
