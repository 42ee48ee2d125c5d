"""Seeded synthetic inputs shared by the CUDA path and the CPU oracle (INPUT GENERATION ONLY).

This module holds none of the random-walk method's arithmetic: its randomness is a splitmix64
counter hash (not the walk RNG), and it only builds graphs and start vectors. Recipe: ltgen.h and
DESIGN.md "Input recipe"; preprocessing follows PAPER.md:273 (§IV-A Workload).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


class _CGraph(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_uint32),
        ("m", ctypes.c_uint64),
        ("row_ptr", ctypes.POINTER(ctypes.c_uint64)),
        ("col", ctypes.POINTER(ctypes.c_uint32)),
        ("max_deg", ctypes.c_uint32),
        ("argmax_deg", ctypes.c_uint32),
    ]


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libltgen.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make -C {os.path.dirname(_HERE)} inputs`")
        lib = ctypes.CDLL(path)
        lib.ltgen_rmat_cpu.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int,
                                       ctypes.c_int, ctypes.POINTER(_CGraph)]
        lib.ltgen_rmat_cpu.restype = ctypes.c_int
        lib.ltgen_free.argtypes = [ctypes.POINTER(_CGraph)]
        lib.ltgen_tuple.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, ctypes.c_uint64,
                                    ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32)]
        lib.ltgen_rmat_gpu.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int,
                                       ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint64),
                                       ctypes.POINTER(ctypes.c_void_p), ctypes.POINTER(ctypes.c_void_p),
                                       ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32)]
        lib.ltgen_rmat_gpu.restype = ctypes.c_int
        lib.ltgen_gpu_free.argtypes = [ctypes.c_void_p]
        lib.ltgen_rmat_gpu_count.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int,
                                             ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)]
        lib.ltgen_rmat_gpu_into.argtypes = [ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_int,
                                            ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                                            ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint64),
                                            ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32),
                                            ctypes.POINTER(ctypes.c_uint32)]
        lib.ltgen_gpu_last_error.restype = ctypes.c_char_p
        lib.ltgen_gpu_memcpy.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64]
        lib.ltgen_gpu_memcpy.restype = ctypes.c_int
        _LIB = lib
    return _LIB


@dataclass
class Graph:
    """CSR graph: row_ptr u64[n+1], col u32[m] (numpy on host, or torch tensors on device)."""
    n: int
    m: int
    row_ptr: object
    col: object
    max_deg: int
    argmax_deg: int


# BASELINE.json "configs" as generator parameters. E = R-MAT tuples.
CONFIGS = {
    1: dict(name="rmat-s12", scale=12, tuples=65_536, permute=False, app="deepwalk", length=10,
            walks="4096", partitions=4),
    2: dict(name="lj-rmat-s22", scale=22, tuples=69_000_000, permute=False, app="deepwalk", length=80,
            walks="V", partitions=None),
    3: dict(name="tw-rmat-s26-ppr", scale=26, tuples=1_500_000_000, permute=False, app="ppr", alpha=0.15,
            walks="V", partitions=None),
    4: dict(name="fs-rmat-s26", scale=26, tuples=1_800_000_000, permute=False, app="deepwalk", length=80,
            walks="V", partitions=None),
    5: dict(name="uk-kron-s28", scale=28, tuples=5_500_000_000, permute=True, app="deepwalk", length=80,
            walks="V", partitions=None),
}


def rmat_cpu(scale: int, tuples: int, seed: int = 1, permute: bool = False, threads: int = 0) -> Graph:
    lib = _lib()
    g = _CGraph()
    rc = lib.ltgen_rmat_cpu(scale, tuples, seed, int(permute), threads, ctypes.byref(g))
    if rc != 0:
        raise RuntimeError(f"ltgen_rmat_cpu failed rc={rc}")
    try:
        row_ptr = np.ctypeslib.as_array(g.row_ptr, shape=(g.n + 1,)).copy()
        col = np.ctypeslib.as_array(g.col, shape=(max(g.m, 1),))[: g.m].copy()
    finally:
        lib.ltgen_free(ctypes.byref(g))
    return Graph(int(g.n), int(g.m), row_ptr, col, int(g.max_deg), int(g.argmax_deg))


def rmat_gpu_ranged(scale: int, tuples: int, seed: int = 1, permute: bool = False, device: int = 0,
                    max_pass_keys: int | None = None) -> Graph:
    """Same graph as rmat_cpu, generated on the GPU one source-vertex range at a time (for graphs whose
    key arrays exceed device memory, e.g. BASELINE configs[4]); row_ptr/col are torch CUDA tensors
    (col is a view of an allocation sized for every key before deduplication)."""
    import torch

    lib = _lib()
    torch.cuda.set_device(device)
    total, mx = ctypes.c_uint64(), ctypes.c_uint64()
    if lib.ltgen_rmat_gpu_count(scale, tuples, seed, int(permute), ctypes.byref(total), ctypes.byref(mx)) != 0:
        raise RuntimeError("ltgen_rmat_gpu_count failed: " + lib.ltgen_gpu_last_error().decode())
    row_ptr = torch.empty((1 << scale) + 1, dtype=torch.int64, device="cuda")
    col = torch.empty(max(total.value, 1), dtype=torch.int32, device="cuda")
    if max_pass_keys is None:  # pass buffers: 2 x 8 B keys + 1 B flag + sort scratch per key
        free, _ = torch.cuda.mem_get_info()
        max_pass_keys = max(int(mx.value), int(0.6 * free / 20))
    n, m, md, am, passes = (ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_uint32(), ctypes.c_uint32(),
                            ctypes.c_uint32())
    rc = lib.ltgen_rmat_gpu_into(scale, tuples, seed, int(permute), int(max_pass_keys), row_ptr.data_ptr(),
                                 col.data_ptr(), total.value, ctypes.byref(n), ctypes.byref(m), ctypes.byref(md),
                                 ctypes.byref(am), ctypes.byref(passes))
    if rc != 0:
        raise RuntimeError("ltgen_rmat_gpu_into failed: " + lib.ltgen_gpu_last_error().decode())
    g = Graph(int(n.value), int(m.value), row_ptr[: n.value + 1], col[: m.value], int(md.value), int(am.value))
    g.passes = int(passes.value)
    return g


def rmat_gpu(scale: int, tuples: int, seed: int = 1, permute: bool = False, device: int = 0) -> Graph:
    """Same graph as rmat_cpu, generated on the GPU; row_ptr/col are torch CUDA tensors. Falls back to
    the ranged build when the one-shot key arrays (about 40 B per tuple) do not fit."""
    import torch

    lib = _lib()
    torch.cuda.set_device(device)
    free, _ = torch.cuda.mem_get_info(device)
    if 44 * tuples > 0.8 * free:
        return rmat_gpu_ranged(scale, tuples, seed, permute, device)
    n = ctypes.c_uint32()
    m = ctypes.c_uint64()
    drp = ctypes.c_void_p()
    dcol = ctypes.c_void_p()
    mx = ctypes.c_uint32()
    am = ctypes.c_uint32()
    torch.cuda.synchronize()
    rc = lib.ltgen_rmat_gpu(scale, tuples, seed, int(permute), ctypes.byref(n), ctypes.byref(m),
                            ctypes.byref(drp), ctypes.byref(dcol), ctypes.byref(mx), ctypes.byref(am))
    if rc != 0:
        raise RuntimeError("ltgen_rmat_gpu failed: " + lib.ltgen_gpu_last_error().decode())
    try:
        row_ptr = torch.empty(n.value + 1, dtype=torch.int64, device="cuda")
        col = torch.empty(max(m.value, 1), dtype=torch.int32, device="cuda")[: m.value]
        if lib.ltgen_gpu_memcpy(row_ptr.data_ptr(), drp.value, 8 * (n.value + 1)) != 0 or \
                lib.ltgen_gpu_memcpy(col.data_ptr(), dcol.value, 4 * m.value) != 0:
            raise RuntimeError("ltgen_gpu_memcpy failed: " + lib.ltgen_gpu_last_error().decode())
    finally:
        lib.ltgen_gpu_free(drp)
        lib.ltgen_gpu_free(dcol)
    return Graph(int(n.value), int(m.value), row_ptr, col, int(mx.value), int(am.value))


def tuple_at(scale: int, seed: int, permute: bool, e: int) -> tuple[int, int]:
    u = ctypes.c_uint32()
    v = ctypes.c_uint32()
    _lib().ltgen_tuple(scale, seed, int(permute), e, ctypes.byref(u), ctypes.byref(v))
    return int(u.value), int(v.value)


def deepwalk_starts(num_walks: int, n: int, first_walk_id: int = 0) -> np.ndarray:
    """Walk w starts at vertex w mod n (SURVEY.md §8(c) reading #7 of PAPER.md:287)."""
    w = np.arange(first_walk_id, first_walk_id + num_walks, dtype=np.uint64)
    return (w % np.uint64(n)).astype(np.uint32)


def ppr_starts(num_walks: int, source: int) -> np.ndarray:
    """All PPR walks start at the max-degree source (ties -> smallest ID)."""
    return np.full(num_walks, source, dtype=np.uint32)


def small_graph(edges, n: int | None = None) -> Graph:
    """Build a CSR from an explicit undirected edge list (tiny hand-made test graphs).
    Symmetrizes, drops self loops/duplicates and sorts adjacency; keeps vertex IDs as given."""
    adj: dict[int, set] = {}
    nn = 0
    for u, v in edges:
        nn = max(nn, u + 1, v + 1)
        if u == v:
            continue
        adj.setdefault(u, set()).add(v)
        adj.setdefault(v, set()).add(u)
    if n is None:
        n = nn
    row_ptr = np.zeros(n + 1, dtype=np.uint64)
    cols = []
    for u in range(n):
        nb = sorted(adj.get(u, ()))
        cols.extend(nb)
        row_ptr[u + 1] = row_ptr[u] + len(nb)
    col = np.asarray(cols, dtype=np.uint32)
    deg = np.diff(row_ptr.astype(np.int64))
    am = int(np.argmax(deg)) if n else 0
    return Graph(n, int(row_ptr[-1]), row_ptr, col, int(deg.max()) if n else 0, am)
