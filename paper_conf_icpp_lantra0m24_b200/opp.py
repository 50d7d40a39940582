"""Thin ctypes binding of libopp.so (include/opp.h) -- argument marshalling only.

Every entry point of the C ABI is exposed under the same name; a negative
return code raises OppError carrying opp_last_error().  There is no fallback:
if libopp.so is missing or cannot be loaded, importing this module raises.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# OPP_LIB: an alternative build of the same library (measurement A/B runs;
# bench.py records every OPP_* variable in its JSON line)
LIB_PATH = os.environ.get("OPP_LIB") or os.path.join(_HERE, "libopp.so")

OPP_OK, OPP_ERR_ARG, OPP_ERR_STATE, OPP_ERR_NOMEM, OPP_ERR_CAPACITY = 0, -1, -2, -3, -4
OPP_ERR_CUDA, OPP_ERR_NCCL, OPP_ERR_MESH = -5, -6, -7
OPP_REAL, OPP_INT, OPP_INT64 = 0, 1, 2
OPP_MOVE_DONE, OPP_NEED_MOVE, OPP_NEED_REMOVE, OPP_NEED_MIGRATE = 0, 1, 2, 3
OPP_DEP_ATOMIC, OPP_DEP_ATOMIC_WARPAGG, OPP_DEP_SORT_SEGRED, OPP_DEP_AUTO = 0, 1, 2, 3

ALLOC_FN = C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)
FREE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_size_t, C.c_void_p, C.c_void_p)

# Every symbol include/opp.h declares (checked by tests/test_abi.py).
EXPORTS = (
    "opp_init_params_default", "opp_init", "opp_finalize", "opp_get_nccl_unique_id",
    "opp_decl_set", "opp_decl_particle_set", "opp_decl_map", "opp_decl_dat",
    "opp_set_partition", "opp_inject", "opp_push_move_deposit", "opp_fill_holes",
    "opp_get_node_charge", "opp_get_dat", "opp_set_dat", "opp_get_particle_count",
    "opp_get_dat_device_ptr", "opp_kernel_launch_count", "opp_sync", "opp_last_error",
    "opp_phase_timing", "opp_get_phase_times", "opp_get_step_stats", "opp_sort_by_cell",
    "opp_field_init", "opp_field_solve", "opp_get_field_stats", "opp_field_solve_boltzmann",
    "opp_em_interpolate", "opp_em_move_deposit", "opp_em_get_stats", "opp_em_sort_by_cell",
    "opp_shuffle", "opp_em_accumulate_current", "opp_em_advance_b", "opp_em_advance_e",
    "opp_em_set_partition", "opp_em_move_deposit_slab", "opp_em_field_step_slab",
)
PHASES = ("inject", "begin", "push_move_deposit", "continue", "segred", "fill", "migrate", "halo",
          "sort_count", "sort_move", "field", "em_move_deposit")
# note: "fill" includes the periodic sort-by-cell when opp_init_params.sort_every > 0


class OppError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"opp error {code}: {msg}")
        self.code = code


class opp_init_params(C.Structure):
    _fields_ = [("device", C.c_int), ("cuda_stream", C.c_void_p), ("rank", C.c_int),
                ("nranks", C.c_int), ("nccl_unique_id", C.c_void_p), ("alloc", ALLOC_FN),
                ("free", FREE_FN), ("alloc_user", C.c_void_p), ("deposit_mode", C.c_int),
                ("direct_hop", C.c_int), ("overlay_spacing", C.c_double),
                ("hop_budget_per_pass", C.c_int), ("hop_cap", C.c_int),
                ("allow_growth", C.c_int), ("sort_every", C.c_int),
                ("tma_pipeline", C.c_int), ("transport", C.c_int),
                ("sort_axis", C.c_double * 3), ("deposit_cache", C.c_int),
                ("sort_lead", C.c_double)]


class opp_step_params(C.Structure):
    _fields_ = [("dt", C.c_double), ("qm", C.c_double), ("weight", C.c_double),
                ("zero_charge", C.c_int), ("fill_inline", C.c_int)]


class opp_step_stats(C.Structure):
    _fields_ = [("n_before", C.c_int64), ("n_injected", C.c_int64), ("n_removed", C.c_int64),
                ("n_after", C.c_int64), ("n_migrated_out", C.c_int64),
                ("n_migrated_in", C.c_int64), ("total_hops", C.c_int64),
                ("n_hop_capped", C.c_int64), ("n_deferred", C.c_int64),
                ("max_hops", C.c_int32), ("migrate_rounds", C.c_int32),
                ("cum_pushed", C.c_int64), ("cum_steps", C.c_int64)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class opp_field_params(C.Structure):
    _fields_ = [("rhs_scale", C.c_double), ("tol", C.c_double), ("max_iter", C.c_int),
                ("warm_start", C.c_int), ("precond", C.c_int), ("slab_cg", C.c_int)]


class opp_boltzmann_params(C.Structure):
    _fields_ = [("rhs_scale", C.c_double), ("ne_coef", C.c_double), ("phi0", C.c_double),
                ("te", C.c_double), ("newton_tol", C.c_double), ("newton_atol", C.c_double),
                ("cg_tol", C.c_double), ("max_newton", C.c_int), ("cg_max_iter", C.c_int),
                ("warm_start", C.c_int), ("precond", C.c_int)]


class opp_boltzmann_stats(C.Structure):
    _fields_ = [("newton_steps", C.c_int32), ("converged", C.c_int32),
                ("cg_iterations", C.c_int64), ("res_norm", C.c_double),
                ("res0_norm", C.c_double), ("ref_norm", C.c_double)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class opp_field_stats(C.Structure):
    _fields_ = [("iterations", C.c_int32), ("converged", C.c_int32),
                ("rel_residual", C.c_double), ("rhs_norm", C.c_double)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class opp_em_params(C.Structure):
    _fields_ = [("qdt_2mc", C.c_double), ("cdt_2h", C.c_double * 3), ("qsp", C.c_double),
                ("kcap", C.c_int), ("deposit_mode", C.c_int)]


class opp_em_stats(C.Structure):
    _fields_ = [("n_crossings", C.c_int64), ("n_capped", C.c_int64),
                ("max_crossings", C.c_int32), ("pad", C.c_int32)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_ if k != "pad"}


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() "
                          "(python -m paper_conf_icpp_lantra0m24_b200.build)")
    lib = C.CDLL(LIB_PATH)
    P, I, I64, I32 = C.c_void_p, C.c_int, C.c_int64, C.c_int32
    sig = {
        "opp_init_params_default": (None, [C.POINTER(opp_init_params)]),
        "opp_init": (I, [C.POINTER(opp_init_params), C.POINTER(P)]),
        "opp_finalize": (I, [P]),
        "opp_get_nccl_unique_id": (I, [P]),
        "opp_decl_set": (I, [P, I64, C.c_char_p, C.POINTER(I32)]),
        "opp_decl_particle_set": (I, [P, C.c_char_p, I32, I64, I64, C.POINTER(I32)]),
        "opp_decl_map": (I, [P, I32, I32, I, P, C.c_char_p, C.POINTER(I32)]),
        "opp_decl_dat": (I, [P, I32, I, I, P, C.c_char_p, C.POINTER(I32)]),
        "opp_set_partition": (I, [P, I32, I64, P, I32, P]),
        "opp_inject": (I, [P, I32, I64, I, P, P, I]),
        "opp_push_move_deposit": (I, [P, I32, I32, I32, I32, I32, I32, I32, I32, I32,
                                      C.POINTER(opp_step_params), C.POINTER(opp_step_stats)]),
        "opp_fill_holes": (I, [P, I32, C.POINTER(I64)]),
        "opp_get_step_stats": (I, [P, I32, C.POINTER(opp_step_stats)]),
        "opp_sort_by_cell": (I, [P, I32]),
        "opp_shuffle": (I, [P, I32, C.c_uint64]),
        "opp_get_node_charge": (I, [P, I32, P, I64]),
        "opp_get_dat": (I, [P, I32, P, I64]),
        "opp_set_dat": (I, [P, I32, P, I64, I]),
        "opp_get_particle_count": (I, [P, I32, C.POINTER(I64)]),
        "opp_get_dat_device_ptr": (I, [P, I32, C.POINTER(P), C.POINTER(I64)]),
        "opp_kernel_launch_count": (I64, [P]),
        "opp_sync": (I, [P]),
        "opp_phase_timing": (I, [P, I]),
        "opp_get_phase_times": (I, [P, P, P]),
        "opp_last_error": (C.c_char_p, []),
        "opp_field_init": (I, [P, I32, I32, P, P]),
        "opp_field_solve": (I, [P, I32, I32, I32, C.POINTER(opp_field_params),
                                C.POINTER(opp_field_stats)]),
        "opp_get_field_stats": (I, [P, C.POINTER(opp_field_stats)]),
        "opp_field_solve_boltzmann": (I, [P, I32, I32, I32, C.POINTER(opp_boltzmann_params),
                                          C.POINTER(opp_boltzmann_stats)]),
        "opp_em_interpolate": (I, [P, I, I, I, P, P, P]),
        "opp_em_move_deposit": (I, [P, I64, I64, P, P, P, P, P, P, I64, P,
                                    C.POINTER(opp_em_params), C.POINTER(opp_em_stats)]),
        "opp_em_get_stats": (I, [P, C.POINTER(opp_em_stats)]),
        "opp_em_sort_by_cell": (I, [P, I64, I64, P, P, P, P, I64, P, P, P, P]),
        "opp_em_accumulate_current": (I, [P, P, P, I64, P, C.c_double, P]),
        "opp_em_advance_b": (I, [P, P, P, P, I64, P, C.c_double]),
        "opp_em_advance_e": (I, [P, P, P, P, P, I64, P, C.c_double]),
        "opp_em_set_partition": (I, [P, I, I, I, I, I]),
        "opp_em_move_deposit_slab": (I, [P, C.POINTER(C.c_int64), I64, P, P, P, P, P, P, P, I64, P,
                                         C.POINTER(opp_em_params), C.POINTER(opp_em_stats)]),
        "opp_em_field_step_slab": (I, [P, P, P, P, P, P, P, I64, P, C.c_double]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    return lib


lib = _load()


def _ck(rc: int) -> int:
    if rc < 0:
        raise OppError(rc, lib.opp_last_error().decode(errors="replace"))
    return rc


def _name(s) -> bytes:
    return (s or "").encode()


def _ptr(a):
    """Pointer of a numpy array / torch tensor / int / None."""
    if a is None:
        return None
    if isinstance(a, int):
        return a
    if hasattr(a, "data_ptr"):
        return a.data_ptr()
    return a.ctypes.data


# ----------------------------------------------------------------- ABI mirror
def opp_init_params_default() -> opp_init_params:
    p = opp_init_params()
    lib.opp_init_params_default(C.byref(p))
    return p


def opp_init(params: opp_init_params) -> int:
    out = C.c_void_p()
    _ck(lib.opp_init(C.byref(params), C.byref(out)))
    return out.value


def opp_finalize(ctx) -> None:
    _ck(lib.opp_finalize(ctx))


def opp_get_nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _ck(lib.opp_get_nccl_unique_id(buf))
    return buf.raw


def opp_decl_set(ctx, size: int, name: str) -> int:
    out = C.c_int32()
    _ck(lib.opp_decl_set(ctx, int(size), _name(name), C.byref(out)))
    return out.value


def opp_decl_particle_set(ctx, name: str, cells: int, n_init: int = 0, capacity: int = 0) -> int:
    out = C.c_int32()
    _ck(lib.opp_decl_particle_set(ctx, _name(name), cells, int(n_init), int(capacity), C.byref(out)))
    return out.value


def opp_decl_map(ctx, frm: int, to: int, dim: int, host, name: str) -> int:
    out = C.c_int32()
    _ck(lib.opp_decl_map(ctx, frm, to, dim, _ptr(host), _name(name), C.byref(out)))
    return out.value


def opp_decl_dat(ctx, set_: int, dim: int, typ: int, host, name: str) -> int:
    out = C.c_int32()
    _ck(lib.opp_decl_dat(ctx, set_, dim, typ, _ptr(host), _name(name), C.byref(out)))
    return out.value


def opp_set_partition(ctx, cells: int, rank_of_cell, nodes: int, node_gid) -> None:
    _ck(lib.opp_set_partition(ctx, cells, int(rank_of_cell.shape[0]), _ptr(rank_of_cell), nodes,
                              _ptr(node_gid)))


def opp_inject(ctx, parts: int, n: int, cols, data, on_device: bool) -> None:
    k = len(cols)
    ca = (C.c_int32 * k)(*cols)
    da = (C.c_void_p * k)(*[_ptr(d) for d in data])
    _ck(lib.opp_inject(ctx, parts, int(n), k, ca, da, int(bool(on_device))))


def opp_push_move_deposit(ctx, parts, pos, vel, p2c, c2c, c2n, node_pos, cell_ef, node_charge,
                          params: opp_step_params, want_stats: bool = True):
    st = opp_step_stats() if want_stats else None
    _ck(lib.opp_push_move_deposit(ctx, parts, pos, vel, p2c, c2c, c2n, node_pos, cell_ef,
                                  node_charge, C.byref(params), C.byref(st) if st else None))
    return st


def opp_get_step_stats(ctx, parts: int) -> opp_step_stats:
    st = opp_step_stats()
    _ck(lib.opp_get_step_stats(ctx, parts, C.byref(st)))
    return st


def opp_fill_holes(ctx, parts: int, want_count: bool = True):
    if not want_count:
        _ck(lib.opp_fill_holes(ctx, parts, None))
        return None
    n = C.c_int64()
    _ck(lib.opp_fill_holes(ctx, parts, C.byref(n)))
    return n.value


def opp_sort_by_cell(ctx, parts: int) -> None:
    _ck(lib.opp_sort_by_cell(ctx, parts))


def opp_shuffle(ctx, parts: int, seed: int) -> None:
    _ck(lib.opp_shuffle(ctx, parts, int(seed) & 0xFFFFFFFFFFFFFFFF))


def opp_get_node_charge(ctx, dat: int, out) -> None:
    _ck(lib.opp_get_node_charge(ctx, dat, _ptr(out), int(out.shape[0])))


def opp_get_dat(ctx, dat: int, out, n: int) -> None:
    _ck(lib.opp_get_dat(ctx, dat, _ptr(out), int(n)))


def opp_set_dat(ctx, dat: int, src, n: int, on_device: bool = False) -> None:
    _ck(lib.opp_set_dat(ctx, dat, _ptr(src), int(n), int(bool(on_device))))


def opp_get_particle_count(ctx, parts: int) -> int:
    n = C.c_int64()
    _ck(lib.opp_get_particle_count(ctx, parts, C.byref(n)))
    return n.value


def opp_get_dat_device_ptr(ctx, dat: int):
    p, s = C.c_void_p(), C.c_int64()
    _ck(lib.opp_get_dat_device_ptr(ctx, dat, C.byref(p), C.byref(s)))
    return p.value, s.value


def opp_kernel_launch_count(ctx) -> int:
    return int(lib.opp_kernel_launch_count(ctx))


def opp_sync(ctx) -> None:
    _ck(lib.opp_sync(ctx))


def opp_last_error() -> str:
    return lib.opp_last_error().decode(errors="replace")


def opp_phase_timing(ctx, enable: bool) -> None:
    _ck(lib.opp_phase_timing(ctx, int(bool(enable))))


def opp_get_phase_times(ctx) -> dict:
    ms = (C.c_double * len(PHASES))()
    cnt = (C.c_int64 * len(PHASES))()
    _ck(lib.opp_get_phase_times(ctx, ms, cnt))
    return {PHASES[k]: (ms[k], cnt[k]) for k in range(len(PHASES))}


def opp_field_init(ctx, c2n: int, node_pos: int, dirichlet_mask, dirichlet_value) -> None:
    import numpy as np
    m = np.ascontiguousarray(dirichlet_mask, dtype=np.int32)
    v = np.ascontiguousarray(dirichlet_value, dtype=np.float64)
    _ck(lib.opp_field_init(ctx, c2n, node_pos, _ptr(m), _ptr(v)))


def opp_field_solve(ctx, node_charge: int, node_potential: int, cell_ef: int,
                    params: opp_field_params, want_stats: bool = True):
    st = opp_field_stats() if want_stats else None
    _ck(lib.opp_field_solve(ctx, node_charge, node_potential, cell_ef, C.byref(params),
                            C.byref(st) if st else None))
    return st


def opp_field_solve_boltzmann(ctx, node_charge: int, node_potential: int, cell_ef: int,
                              params: opp_boltzmann_params) -> opp_boltzmann_stats:
    st = opp_boltzmann_stats()
    _ck(lib.opp_field_solve_boltzmann(ctx, node_charge, node_potential, cell_ef,
                                      C.byref(params), C.byref(st)))
    return st


def opp_get_field_stats(ctx) -> opp_field_stats:
    st = opp_field_stats()
    _ck(lib.opp_get_field_stats(ctx, C.byref(st)))
    return st


def opp_em_params_make(qdt_2mc: float, cdt_2h, qsp: float, kcap: int = 16,
                       deposit_mode: int = OPP_DEP_ATOMIC_WARPAGG) -> opp_em_params:
    return opp_em_params(qdt_2mc, (C.c_double * 3)(*cdt_2h), qsp, kcap, deposit_mode)


def opp_em_interpolate(ctx, nx: int, ny: int, nz: int, e, b, interp) -> None:
    """Device tensors: e[3][nc], b[3][nc] -> interp[nc][18]."""
    _ck(lib.opp_em_interpolate(ctx, nx, ny, nz, _ptr(e), _ptr(b), _ptr(interp)))


def opp_em_move_deposit(ctx, n: int, stride: int, off, u, w, cell, interp, c2c, n_cells: int, acc,
                        params: opp_em_params, want_stats: bool = True):
    """Device tensors (SoA columns of row stride `stride`); returns stats or None."""
    st = opp_em_stats() if want_stats else None
    _ck(lib.opp_em_move_deposit(ctx, int(n), int(stride), _ptr(off), _ptr(u), _ptr(w), _ptr(cell),
                                _ptr(interp), _ptr(c2c), int(n_cells), _ptr(acc), C.byref(params),
                                C.byref(st) if st else None))
    return st


def opp_em_get_stats(ctx) -> opp_em_stats:
    st = opp_em_stats()
    _ck(lib.opp_em_get_stats(ctx, C.byref(st)))
    return st


def opp_em_sort_by_cell(ctx, n: int, stride: int, off, u, w, cell, n_cells: int, off_out, u_out,
                        w_out, cell_out) -> None:
    _ck(lib.opp_em_sort_by_cell(ctx, int(n), int(stride), _ptr(off), _ptr(u), _ptr(w), _ptr(cell),
                                int(n_cells), _ptr(off_out), _ptr(u_out), _ptr(w_out),
                                _ptr(cell_out)))


def _h3(h):
    return (C.c_double * 3)(*[float(x) for x in h])


def opp_em_accumulate_current(ctx, acc, c2c, n_cells: int, h, dt: float, J) -> None:
    _ck(lib.opp_em_accumulate_current(ctx, _ptr(acc), _ptr(c2c), int(n_cells), _h3(h), float(dt), _ptr(J)))


def opp_em_advance_b(ctx, e, b, c2c, n_cells: int, h, frac_dt: float) -> None:
    _ck(lib.opp_em_advance_b(ctx, _ptr(e), _ptr(b), _ptr(c2c), int(n_cells), _h3(h), float(frac_dt)))


def opp_em_advance_e(ctx, e, b, J, c2c, n_cells: int, h, dt: float) -> None:
    _ck(lib.opp_em_advance_e(ctx, _ptr(e), _ptr(b), _ptr(J), _ptr(c2c), int(n_cells), _h3(h), float(dt)))


def opp_em_set_partition(ctx, nx: int, ny: int, nz: int, k0: int, k1: int) -> None:
    _ck(lib.opp_em_set_partition(ctx, int(nx), int(ny), int(nz), int(k0), int(k1)))


def opp_em_move_deposit_slab(ctx, n: int, cap: int, off, u, w, cell, pid, interp, c2c, n_cells: int, acc,
                             params: opp_em_params, want_stats: bool = True):
    """Device tensors (SoA columns of row stride `cap`); returns (new n, stats or None)."""
    st = opp_em_stats() if want_stats else None
    nn = C.c_int64(int(n))
    _ck(lib.opp_em_move_deposit_slab(ctx, C.byref(nn), int(cap), _ptr(off), _ptr(u), _ptr(w), _ptr(cell),
                                     _ptr(pid) if pid is not None else None, _ptr(interp), _ptr(c2c),
                                     int(n_cells), _ptr(acc), C.byref(params), C.byref(st) if st else None))
    return nn.value, st


def opp_em_field_step_slab(ctx, e, b, J, acc, interp, c2c, n_cells: int, h, dt: float) -> None:
    _ck(lib.opp_em_field_step_slab(ctx, _ptr(e), _ptr(b), _ptr(J), _ptr(acc), _ptr(interp), _ptr(c2c),
                                   int(n_cells), _h3(h), float(dt)))
