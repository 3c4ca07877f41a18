"""Thin ctypes binding of libptas_b200.so (include/ptas.h).

Argument marshalling only: every step of the hot path runs in the library's
CUDA kernels or its C++ host driver.  The library must be built in-tree
(``python -m paper_conf_ipps_ligsg18_b200.build`` or ``__graft_entry__.build()``);
there is no fallback of any kind — a missing library raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PTAS_LIB") or os.path.join(_HERE, "libptas_b200.so")

PTAS_OK, PTAS_EINVAL, PTAS_ETOOBIG, PTAS_ENOMEM, PTAS_ECUDA, PTAS_ENCCL, PTAS_EINTERNAL = 0, -1, -2, -3, -4, -5, -6
MODE_SINGLE, MODE_LEVEL_SHARDED, MODE_MULTI_PROBE = 0, 1, 2

i32p = ctypes.POINTER(ctypes.c_int32)
i64p = ctypes.POINTER(ctypes.c_int64)
vp = ctypes.c_void_p


class PtasOptions(ctypes.Structure):
    _fields_ = [("probes_per_round", ctypes.c_int32), ("mode", ctypes.c_int32), ("device", ctypes.c_int32),
                ("comm", vp), ("table_budget_bytes", ctypes.c_int64), ("memoize", ctypes.c_int32),
                ("virtual_shards", ctypes.c_int32), ("layout", ctypes.c_int32), ("stream", vp),
                ("speculate", ctypes.c_int32), ("window", ctypes.c_int32), ("slab_pipeline", ctypes.c_int32),
                ("shard_min_rows", ctypes.c_int64)]


class PtasStats(ctypes.Structure):
    _fields_ = [("probes", ctypes.c_int32), ("rounds", ctypes.c_int32), ("unique_dps", ctypes.c_int32),
                ("K_at_Tstar", ctypes.c_int32), ("T_star", ctypes.c_int64), ("sigma_max", ctypes.c_int64),
                ("opt_at_Tstar", ctypes.c_int64), ("relaxations", ctypes.c_double),
                ("dp_seconds", ctypes.c_double), ("fill_seconds", ctypes.c_double),
                ("total_seconds", ctypes.c_double), ("alg_bytes", ctypes.c_double), ("states", ctypes.c_int64),
                ("kernel_launches", ctypes.c_int32), ("fill_launches", ctypes.c_int32),
                ("h2d_bytes", ctypes.c_int64), ("d2h_bytes", ctypes.c_int64), ("relax_executed", ctypes.c_double),
                ("exec_bytes", ctypes.c_double), ("spec_dps", ctypes.c_int32), ("spec_wasted", ctypes.c_int32),
                ("fill_wall_seconds", ctypes.c_double), ("window_dps", ctypes.c_int32), ("pad_", ctypes.c_int32),
                ("dev_bytes_max", ctypes.c_int64)]

    def to_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class PtasProbe(ctypes.Structure):
    _fields_ = [("T", ctypes.c_int64), ("round", ctypes.c_int32), ("feasible", ctypes.c_int32),
                ("K", ctypes.c_int32), ("opt", ctypes.c_int32), ("sigma", ctypes.c_int64),
                ("memo_hit", ctypes.c_int32), ("rank", ctypes.c_int32)]


EXPORTS = [
    "ptas_default_options", "ptas_solve", "ptas_solve_ex", "ptas_solve_device", "dp_table_shape", "dp_fill",
    "dp_fill_device", "ptas_get_unique_id", "ptas_comm_init", "ptas_comm_destroy", "ptas_strerror", "ptas_k",
    "ptas_bounds", "ptas_classify", "ptas_probe_targets", "ptas_interval_update", "ptas_shard_range",
    "dp_configs", "dp_row_index", "hmbp_solve", "ptas_table_order", "ptas_level_shard", "dp_fill_opt", "dp_fill_alg4",
    "ptas_slab_plan",
]

_lib = None


class PtasError(RuntimeError):
    def __init__(self, fn, rc):
        super().__init__(f"{fn} failed: {rc} ({strerror(rc)})")
        self.rc = rc


def lib():
    """Load the in-tree library (raises if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built: run `python -m paper_conf_ipps_ligsg18_b200.build` "
                          "(no CPU fallback exists)")
    L = ctypes.CDLL(LIB_PATH)
    L.ptas_default_options.argtypes = [ctypes.POINTER(PtasOptions)]
    L.ptas_default_options.restype = None
    L.ptas_solve.argtypes = [i64p, ctypes.c_int32, ctypes.c_int32, ctypes.c_double, ctypes.POINTER(PtasOptions),
                             i64p, i32p, ctypes.POINTER(PtasStats)]
    L.ptas_solve_ex.argtypes = L.ptas_solve.argtypes + [ctypes.POINTER(PtasProbe), ctypes.c_int32, i32p]
    L.ptas_solve_device.argtypes = [vp, ctypes.c_int32, ctypes.c_int32, ctypes.c_double,
                                    ctypes.POINTER(PtasOptions), i64p, vp, ctypes.POINTER(PtasStats)]
    L.dp_table_shape.argtypes = [i32p, ctypes.c_int32, i64p, i32p]
    L.dp_fill.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int64, vp, ctypes.c_int64, i32p,
                          ctypes.POINTER(PtasStats)]
    L.dp_fill_device.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int64, vp, ctypes.c_int64, vp, i32p]
    L.ptas_get_unique_id.argtypes = [vp]
    L.ptas_comm_init.argtypes = [ctypes.POINTER(vp), ctypes.c_int32, ctypes.c_int32, vp, ctypes.c_int32]
    L.ptas_comm_destroy.argtypes = [vp]
    L.ptas_strerror.argtypes = [ctypes.c_int]
    L.ptas_strerror.restype = ctypes.c_char_p
    L.ptas_k.argtypes = [ctypes.c_double]
    L.ptas_bounds.argtypes = [i64p, ctypes.c_int32, ctypes.c_int32, i64p, i64p]
    L.ptas_classify.argtypes = [i64p, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, i64p, i32p, i64p, i32p, i32p]
    L.ptas_probe_targets.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int32, i64p, i32p]
    L.ptas_interval_update.argtypes = [i64p, i64p, i64p, i32p, ctypes.c_int32]
    L.ptas_shard_range.argtypes = [ctypes.c_int64, ctypes.c_int32, ctypes.c_int32, i64p, i64p]
    L.ptas_level_shard.argtypes = [ctypes.c_int64, ctypes.c_int32, ctypes.c_int32, ctypes.c_int64, i64p, i64p, i64p]
    L.ptas_slab_plan.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32, i64p, i64p, i64p, i64p,
                                 i64p]
    L.dp_configs.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int64, i32p, ctypes.c_int64, i64p]
    L.dp_fill_opt.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int64, ctypes.c_int64, ctypes.c_int32, i32p,
                              ctypes.POINTER(PtasStats)]
    L.dp_fill_alg4.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, vp, ctypes.c_int64, i32p,
                               i32p, ctypes.POINTER(PtasStats)]
    L.hmbp_solve.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int64, i32p, i32p, ctypes.c_int32,
                             ctypes.POINTER(PtasStats)]
    L.ptas_table_order.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int32, i32p, i32p]
    L.dp_row_index.argtypes = [i32p, ctypes.c_int32, i64p, ctypes.c_int64, i64p, ctypes.c_int64]
    _lib = L
    return L


def strerror(rc: int) -> str:
    return lib().ptas_strerror(int(rc)).decode()


def _chk(fn, rc):
    if rc != PTAS_OK:
        raise PtasError(fn, rc)


def _a(x, dt):
    return np.ascontiguousarray(x, dtype=dt)


def _ptr(a, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))
