"""CPU ORACLE for the LightTraffic walk-update path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and --impl reference) may
import this module. The product package never does. The C source (oracle.c) follows SURVEY.md §8(c)
and PAPER.md:45/:287/:297 line by line; see oracle.h for the definition and DESIGN.md for the
readings of the paper it implements. Every oracle function is pinned by tests/test_oracle_pins.py.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

DEEPWALK = 0
PPR = 1
PAGERANK = 2
EMPTY = 0xFFFFFFFF
DEFAULT_LMAX = 127  # DESIGN.md reading R6

_u64p = ctypes.POINTER(ctypes.c_uint64)
_u32p = ctypes.POINTER(ctypes.c_uint32)


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make oracle`")
        lib = ctypes.CDLL(path)
        lib.oracle_philox4x32_10.argtypes = [_u32p, _u32p, _u32p]
        lib.oracle_ppr_threshold.argtypes = [ctypes.c_double]
        lib.oracle_ppr_threshold.restype = ctypes.c_uint32
        lib.oracle_lemire.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, _u32p]
        lib.oracle_lemire.restype = ctypes.c_uint32
        lib.oracle_lemire_accept.argtypes = [ctypes.c_uint32, ctypes.c_uint32, _u32p]
        lib.oracle_lemire_accept.restype = ctypes.c_int
        lib.oracle_walks.argtypes = [ctypes.c_uint32, _u64p, _u32p, ctypes.c_uint64, _u64p, _u32p, ctypes.c_int,
                                     ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint64, _u32p,
                                     ctypes.c_uint32, _u32p, _u64p, ctypes.c_int]
        lib.oracle_walks.restype = ctypes.c_uint64
        lib.oracle_lemire_exhaustive.argtypes = [ctypes.c_uint32, _u64p, _u64p, ctypes.c_int]
        lib.oracle_visit_counts.argtypes = [ctypes.c_uint64, _u32p, ctypes.c_uint32, _u32p, _u64p]
        _LIB = lib
    return _LIB


def _p(a, t):
    return a.ctypes.data_as(t) if a is not None else None


def philox4x32_10(ctr, key):
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    _lib().oracle_philox4x32_10(_p(c, _u32p), _p(k, _u32p), _p(out, _u32p))
    return [int(x) for x in out]


def ppr_threshold(alpha: float) -> int:
    return int(_lib().oracle_ppr_threshold(alpha))


def lemire(seed: int, w: int, t: int, d: int):
    used = ctypes.c_uint32()
    idx = _lib().oracle_lemire(seed, w, t, d, ctypes.byref(used))
    return int(idx), int(used.value)


def lemire_accept(x: int, d: int):
    idx = ctypes.c_uint32()
    ok = _lib().oracle_lemire_accept(x, d, ctypes.byref(idx))
    return bool(ok), int(idx.value)


def lemire_exhaustive(d: int, threads: int = 0):
    hist = np.zeros(d, dtype=np.uint64)
    rej = ctypes.c_uint64()
    _lib().oracle_lemire_exhaustive(d, _p(hist, _u64p), ctypes.byref(rej), threads)
    return hist, int(rej.value)


def stride_for(app: int, length: int = 0, lmax: int = DEFAULT_LMAX) -> int:
    return (lmax + 1) if app == PPR else (length + 1)


def visit_counts(paths, lengths, n):
    """Visit frequency per vertex from path rows."""
    paths = np.ascontiguousarray(paths, dtype=np.uint32)
    lengths = np.ascontiguousarray(lengths, dtype=np.uint32)
    counts = np.zeros(n, dtype=np.uint64)
    _lib().oracle_visit_counts(len(lengths), _p(paths, _u32p), paths.shape[1] if paths.ndim == 2 else 1,
                               _p(lengths, _u32p), _p(counts, _u64p))
    return counts


def walks(row_ptr, col, starts, app=DEEPWALK, length=80, alpha=0.15, lmax=DEFAULT_LMAX, seed=1,
          ids=None, threads=0):
    """Run the oracle for walks `ids` (default 0..len(starts)-1) from `starts`. alpha is the PPR
    termination probability or the PageRank restart probability.
    Returns (paths u32[count, stride], lengths u32[count], steps, truncated)."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.uint64)
    col = np.ascontiguousarray(col, dtype=np.uint32)
    starts = np.ascontiguousarray(starts, dtype=np.uint32)
    count = len(starts)
    if ids is not None:
        ids = np.ascontiguousarray(ids, dtype=np.uint64)
        assert len(ids) == count
    n = len(row_ptr) - 1
    T = ppr_threshold(alpha) if app in (PPR, PAGERANK) else 0
    stride = stride_for(app, length, lmax)
    paths = np.empty((count, stride), dtype=np.uint32)
    lengths = np.empty(count, dtype=np.uint32)
    trunc = ctypes.c_uint64()
    col_arg = col if len(col) else np.zeros(1, dtype=np.uint32)
    steps = _lib().oracle_walks(n, _p(row_ptr, _u64p), _p(col_arg, _u32p), count, _p(ids, _u64p),
                                _p(starts, _u32p), app, length, T, lmax, seed, _p(paths, _u32p), stride,
                                _p(lengths, _u32p), ctypes.byref(trunc), threads)
    return paths, lengths, int(steps), int(trunc.value)
