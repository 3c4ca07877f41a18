"""ORACLE — plain CPU implementation of the PTAS hot path (test infrastructure).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  It wraps
``oracle/ptas_oracle.c`` (plain sequential C, compiled with gcc) through
ctypes and shares no code with the product library.

Functions (each cites its PAPER.md passage in ptas_oracle.c):
  k_of(eps)
  bounds(p, m)                    Alg 1 l.2-3
  classify(p, T, k)               Alg 1 l.6-8
  configs(N, r, T)                PAPER.md:68, Alg 2 l.17
  dp(N, r, T)                     Eq. 1; Alg 2
  ptas(p, m, eps, P)              Alg 1 / Alg 3
  dp_omp(N, r, T)                 Alg 2 level-parallel comparator, OpenMP
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ptas_oracle.c")
_LIB = os.path.join(_HERE, "libptas_oracle.so")
_lock = threading.Lock()
_lib = None


class OracleProbe(ctypes.Structure):
    _fields_ = [("T", ctypes.c_int64), ("round", ctypes.c_int32),
                ("feasible", ctypes.c_int32), ("K", ctypes.c_int32),
                ("opt", ctypes.c_int32), ("sigma", ctypes.c_int64)]


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain -O2, no OpenMP, no vectorisation hints)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            i32p = ctypes.POINTER(ctypes.c_int32)
            i64p = ctypes.POINTER(ctypes.c_int64)
            lib.oracle_k.restype = ctypes.c_int32
            lib.oracle_k.argtypes = [ctypes.c_double]
            lib.oracle_bounds.argtypes = [i64p, ctypes.c_int32, ctypes.c_int32, i64p, i64p]
            lib.oracle_classify.argtypes = [i64p, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32,
                                            i64p, i32p, i64p, i32p, i32p]
            lib.oracle_configs.restype = ctypes.c_int64
            lib.oracle_configs.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int64, i32p, ctypes.c_int64]
            lib.oracle_sigma.restype = ctypes.c_int64
            lib.oracle_sigma.argtypes = [i32p, ctypes.c_int32]
            lib.oracle_dp.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int64, i32p, ctypes.c_int64,
                                      i32p, ctypes.POINTER(ctypes.c_double)]
            lib.oracle_ptas.argtypes = [i64p, ctypes.c_int32, ctypes.c_int32, ctypes.c_double, ctypes.c_int32,
                                        i64p, i64p, i32p, ctypes.POINTER(OracleProbe), ctypes.c_int32, i32p]
            lib.oracle_hmbp.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int64, i32p, i32p, ctypes.c_int32]
            _lib = lib
    return _lib


def _p(a, ct):
    return a.ctypes.data_as(ctypes.POINTER(ct))


def k_of(eps: float) -> int:
    return int(_load().oracle_k(float(eps)))


def bounds(p, m: int) -> tuple[int, int]:
    p = np.ascontiguousarray(p, dtype=np.int64)
    lb, ub = ctypes.c_int64(), ctypes.c_int64()
    rc = _load().oracle_bounds(_p(p, ctypes.c_int64), len(p), int(m), ctypes.byref(lb), ctypes.byref(ub))
    if rc:
        raise ValueError(f"oracle_bounds rc={rc}")
    return lb.value, ub.value


def classify(p, T: int, k: int):
    """Returns (u, r[K], N[K], cls[n])."""
    p = np.ascontiguousarray(p, dtype=np.int64)
    n = len(p)
    r = np.zeros(max(n, 1), np.int64)
    N = np.zeros(max(n, 1), np.int32)
    cls = np.zeros(max(n, 1), np.int32)
    u, K = ctypes.c_int64(), ctypes.c_int32()
    _load().oracle_classify(_p(p, ctypes.c_int64), n, int(T), int(k), ctypes.byref(u), ctypes.byref(K),
                            _p(r, ctypes.c_int64), _p(N, ctypes.c_int32), _p(cls, ctypes.c_int32))
    K = K.value
    return u.value, r[:K].copy(), N[:K].copy(), cls[:n].copy()


def sigma(N) -> int:
    N = np.ascontiguousarray(N, dtype=np.int32)
    return int(_load().oracle_sigma(_p(N, ctypes.c_int32), len(N)))


def configs(N, r, T: int) -> np.ndarray:
    """C(T) in lexicographic order, shape (|C|, K) int32."""
    N = np.ascontiguousarray(N, dtype=np.int32)
    r = np.ascontiguousarray(r, dtype=np.int64)
    K = len(N)
    lib = _load()
    cnt = lib.oracle_configs(_p(N, ctypes.c_int32), _p(r, ctypes.c_int64), K, int(T), None, 0)
    out = np.zeros((max(cnt, 1), max(K, 1)), np.int32)
    lib.oracle_configs(_p(N, ctypes.c_int32), _p(r, ctypes.c_int64), K, int(T), _p(out, ctypes.c_int32), cnt)
    return out[:cnt, :K].copy()


def dp(N, r, T: int):
    """Whole OPT table (row-major over the given class order, int32) and the
    number of relaxations performed.  Returns (table[N_0+1, ..., N_{K-1}+1], relax)."""
    N = np.ascontiguousarray(N, dtype=np.int32)
    r = np.ascontiguousarray(r, dtype=np.int64)
    K = len(N)
    sg = sigma(N)
    if sg < 0:
        raise OverflowError("sigma overflows int64")
    tab = np.zeros(sg, np.int32)
    opt = ctypes.c_int32()
    relax = ctypes.c_double()
    rc = _load().oracle_dp(_p(N, ctypes.c_int32), _p(r, ctypes.c_int64), K, int(T), _p(tab, ctypes.c_int32),
                           sg, ctypes.byref(opt), ctypes.byref(relax))
    if rc:
        raise ValueError(f"oracle_dp rc={rc}")
    shape = tuple(int(x) + 1 for x in N) if K else ()
    return tab.reshape(shape) if K else tab.reshape(()), relax.value


def ptas(p, m: int, eps: float, P: int = 1, log_cap: int = 4096):
    """Full PTAS.  Returns dict(T_star, makespan, assignment, probes=[(T, round, feasible, K, opt, sigma)])."""
    p = np.ascontiguousarray(p, dtype=np.int64)
    n = len(p)
    ts, ms = ctypes.c_int64(), ctypes.c_int64()
    asg = np.zeros(n, np.int32)
    log = (OracleProbe * log_cap)()
    nlog = ctypes.c_int32()
    rc = _load().oracle_ptas(_p(p, ctypes.c_int64), n, int(m), float(eps), int(P), ctypes.byref(ts),
                             ctypes.byref(ms), _p(asg, ctypes.c_int32), log, log_cap, ctypes.byref(nlog))
    if rc:
        raise ValueError(f"oracle_ptas rc={rc}")
    probes = [(log[i].T, log[i].round, log[i].feasible, log[i].K, log[i].opt, log[i].sigma)
              for i in range(min(nlog.value, log_cap))]
    return {"T_star": ts.value, "makespan": ms.value, "assignment": asg, "probes": probes}


def hmbp(N, r, T: int):
    """High-multiplicity bin packing (Eq. 1 with capacity T): (bins, packing[bins, K])
    with the traceback of reading R11 (oracle_hmbp)."""
    N = np.ascontiguousarray(N, dtype=np.int32)
    r = np.ascontiguousarray(r, dtype=np.int64)
    K = len(N)
    mx = max(int(N.sum()), 1)
    pk = np.zeros((mx, max(K, 1)), np.int32)
    bins = ctypes.c_int32()
    rc = _load().oracle_hmbp(_p(N, ctypes.c_int32), _p(r, ctypes.c_int64), K, int(T), ctypes.byref(bins),
                             _p(pk, ctypes.c_int32), mx)
    if rc:
        raise ValueError(f"oracle_hmbp rc={rc}")
    return bins.value, pk[:bins.value, :K].copy()


# ---------------------------------------------------------------------------
# The paper's CPU comparator shape (Alg 2, OpenMP level-parallel)
# in its own file, ptas_oracle_omp.c, for bench.py's all-core cpu_baseline.
_SRC_OMP = os.path.join(_HERE, "ptas_oracle_omp.c")
_LIB_OMP = os.path.join(_HERE, "libptas_oracle_omp.so")
_lib_omp = None


def build_omp(force: bool = False) -> str:
    """Compile the Alg-2 comparator with gcc -O2 -fopenmp."""
    if force or not os.path.exists(_LIB_OMP) or os.path.getmtime(_LIB_OMP) < os.path.getmtime(_SRC_OMP):
        tmp = _LIB_OMP + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fopenmp", "-shared", "-fPIC", "-o", tmp, _SRC_OMP])
        os.replace(tmp, _LIB_OMP)
    return _LIB_OMP


def _load_omp():
    global _lib_omp
    with _lock:
        if _lib_omp is None:
            lib = ctypes.CDLL(build_omp())
            i32p = ctypes.POINTER(ctypes.c_int32)
            i64p = ctypes.POINTER(ctypes.c_int64)
            lib.oracle_omp_threads.restype = ctypes.c_int
            lib.oracle_dp_omp.argtypes = [i32p, i64p, ctypes.c_int32, ctypes.c_int64, i32p, ctypes.c_int64,
                                          i32p, ctypes.POINTER(ctypes.c_double)]
            _lib_omp = lib
    return _lib_omp


def omp_threads() -> int:
    return int(_load_omp().oracle_omp_threads())


def dp_omp(N, r, T: int):
    """Same contract as dp(): (table, relax), computed by Alg 2's level-parallel
    loop on all OpenMP threads."""
    N = np.ascontiguousarray(N, dtype=np.int32)
    r = np.ascontiguousarray(r, dtype=np.int64)
    K = len(N)
    sg = sigma(N)
    if sg < 0:
        raise OverflowError("sigma overflows int64")
    tab = np.zeros(sg, np.int32)
    opt = ctypes.c_int32()
    relax = ctypes.c_double()
    rc = _load_omp().oracle_dp_omp(_p(N, ctypes.c_int32), _p(r, ctypes.c_int64), K, int(T),
                                   _p(tab, ctypes.c_int32), sg, ctypes.byref(opt), ctypes.byref(relax))
    if rc:
        raise ValueError(f"oracle_dp_omp rc={rc}")
    shape = tuple(int(x) + 1 for x in N) if K else ()
    return tab.reshape(shape) if K else tab.reshape(()), relax.value
