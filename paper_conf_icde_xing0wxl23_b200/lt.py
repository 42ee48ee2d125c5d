"""Thin ctypes binding of liblt.so (include/lt.h). Argument marshalling only: every step of the
walk-update path runs in the CUDA kernels behind the C ABI. There is no CPU fallback: if liblt.so
is missing or fails to load, importing this module raises.

Arrays may be numpy arrays / CPU torch tensors (host pointers; pinned tensors give fast copies)
or CUDA torch tensors (device pointers, borrowed). uint64/uint32 data may be passed as int64/int32
torch tensors (same bits).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("LT_LIBRARY") or os.path.join(_HERE, "liblt.so")  # override: experiments only

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build the CUDA extension first (`make lt` or "
                      f"__graft_entry__.build()); there is no CPU fallback")
_lib = ctypes.CDLL(LIB_PATH)

LT_OK, LT_ERR_INVALID, LT_ERR_STATE, LT_ERR_OOM, LT_ERR_CUDA, LT_ERR_NCCL = range(6)
DEEPWALK, PPR, PAGERANK = 0, 1, 2
POLICY_SELECTIVE, POLICY_ROUND_ROBIN, POLICY_SELECTIVE_ONLY, POLICY_PREEMPTIVE_ONLY = 0, 1, 2, 3
INSERT_WARP_AGGREGATED, INSERT_DIRECT = 0, 1
LAYOUT_AUTO, LAYOUT_CSR, LAYOUT_ADJ, LAYOUT_ADJ12 = 0, 1, 2, 3
EMPTY = 0xFFFFFFFF

EXPORTED = [
    "lt_config_default", "lt_create", "lt_destroy", "lt_last_error", "lt_partition_bounds", "lt_graph_load",
    "lt_graph_load_device", "lt_get_bounds", "lt_walks_init", "lt_walks_init_ex", "lt_run", "lt_path_stride",
    "lt_get_paths", "lt_get_paths_rows", "lt_get_paths_device", "lt_get_stats", "lt_get_pool_state",
    "lt_pending", "lt_exchange_pack", "lt_exchange_insert", "lt_run_to_host", "lt_walks_init_pagerank",
    "lt_get_visit_counts", "lt_get_visit_counts_device", "lt_get_paths_compact", "lt_run_to_host_compact",
    "lt_exchange_buffers", "lt_exchange_attach", "lt_exchange_sent", "lt_exchange_take", "lt_ipc_handle",
    "lt_ipc_open", "lt_superstep_p2p", "lt_paths_buffers", "lt_paths_attach", "lt_philox_device", "lt_compress_columns",
]


class Config(ctypes.Structure):
    _fields_ = [
        ("device", ctypes.c_int),
        ("stream", ctypes.c_void_p),
        ("chunk_walks", ctypes.c_uint32),
        ("ppr_max_len", ctypes.c_uint32),
        ("policy", ctypes.c_uint32),
        ("insert_mode", ctypes.c_uint32),
        ("timing", ctypes.c_uint32),
        ("block_threads", ctypes.c_uint32),
        ("blocks_per_sm", ctypes.c_uint32),
        ("l2_fetch_bytes", ctypes.c_uint32),
        ("gather_mode", ctypes.c_uint32),
        ("ilp", ctypes.c_uint32),
        ("layout", ctypes.c_uint32),
        ("path_mode", ctypes.c_uint32),
        ("zero_copy", ctypes.c_uint32),
        ("zc_alpha_bytes", ctypes.c_uint32),
        ("ooc_prefetch", ctypes.c_uint32),
        ("graph_pool_bytes", ctypes.c_uint64),
        ("rank", ctypes.c_uint32),
        ("world", ctypes.c_uint32),
        ("refill", ctypes.c_uint32),
        ("visit_counts", ctypes.c_uint32),
        ("continue_resident", ctypes.c_uint32),
        ("walk_spill", ctypes.c_uint32),
        ("walk_pool_walks", ctypes.c_uint64),
        ("direct_start", ctypes.c_uint32),
        ("l2_persist", ctypes.c_uint32),
        ("arena", ctypes.c_void_p),
        ("arena_bytes", ctypes.c_uint64),
        ("ooc_compress", ctypes.c_uint32),
    ]


class Stats(ctypes.Structure):
    _fields_ = [(name, ctypes.c_uint64) for name in (
        "num_walks", "steps", "visits", "truncated", "sweeps", "update_launches", "kernel_launches",
        "chunks_total", "chunks_free_min", "h2d_bytes", "d2h_bytes")] + [
        ("update_ms", ctypes.c_double), ("run_ms", ctypes.c_double), ("init_ms", ctypes.c_double),
        ("graph_prep_ms", ctypes.c_double), ("layout", ctypes.c_uint32), ("out_of_core", ctypes.c_uint32)] + [
        (name, ctypes.c_uint64) for name in (
            "iterations", "explicit_copies", "pool_hits", "zero_copy_launches", "preemptive_launches",
            "graph_h2d_bytes", "pool_blocks", "pool_block_bytes", "admissions", "peak_live", "direct_start", "graph_device_bytes", "l2_persist_bytes", "prefetches",
            "spilled_chunks", "reloaded_chunks", "spill_d2h_bytes", "spill_h2d_bytes", "host_chunks_peak",
            "spill_prefetched_chunks")] + [
        ("load_ms", ctypes.c_double), ("spill_xfer_ms", ctypes.c_double), ("host_syncs", ctypes.c_uint64),
        ("arena_bytes_used", ctypes.c_uint64), ("hub_deg", ctypes.c_uint64), ("visit_recounts", ctypes.c_uint64),
        ("graph_h2d_raw_bytes", ctypes.c_uint64), ("ooc_compressed_bytes", ctypes.c_uint64),
        ("visit_hot_slots", ctypes.c_uint64)]


class PoolState(ctypes.Structure):
    _fields_ = [("free_chunks", ctypes.c_int64), ("ring_chunks", ctypes.c_uint64), ("host_chunks", ctypes.c_uint64),
                ("total_chunks", ctypes.c_uint64), ("pending", ctypes.c_uint64), ("finished", ctypes.c_uint64),
                ("device_err", ctypes.c_uint32), ("reserved", ctypes.c_uint32)]


_vp = ctypes.c_void_p
_u32, _u64 = ctypes.c_uint32, ctypes.c_uint64
_lib.lt_config_default.argtypes = [ctypes.POINTER(Config)]
_lib.lt_create.argtypes = [ctypes.POINTER(Config), ctypes.POINTER(_vp)]
_lib.lt_destroy.argtypes = [_vp]
_lib.lt_destroy.restype = None
_lib.lt_last_error.restype = ctypes.c_char_p
_lib.lt_partition_bounds.argtypes = [_u32, _vp, _u32, _vp]
_lib.lt_graph_load.argtypes = [_vp, _u32, _u64, _vp, _vp, _u32]
_lib.lt_graph_load_device.argtypes = [_vp, _u32, _u64, _vp, _vp, _u32]
_lib.lt_get_bounds.argtypes = [_vp, _vp, ctypes.POINTER(_u32)]
_lib.lt_walks_init.argtypes = [_vp, _u64, _vp, ctypes.c_int, ctypes.c_double, _u64]
_lib.lt_walks_init_ex.argtypes = [_vp, _u64, _vp, ctypes.c_int, _u64, ctypes.c_int, ctypes.c_double, _u64]
_lib.lt_walks_init_pagerank.argtypes = [_vp, _u64, _vp, ctypes.c_int, _u64, _u32, ctypes.c_double, _u64]
_lib.lt_get_visit_counts.argtypes = [_vp, _vp]
_lib.lt_get_visit_counts_device.argtypes = [_vp, _vp]
_lib.lt_run.argtypes = [_vp]
_lib.lt_path_stride.argtypes = [_vp, ctypes.POINTER(_u32)]
_lib.lt_get_paths.argtypes = [_vp, _vp, _vp]
_lib.lt_get_paths_rows.argtypes = [_vp, _vp, _u64, _vp, _vp]
_lib.lt_get_paths_device.argtypes = [_vp, _vp, _vp]
_lib.lt_get_stats.argtypes = [_vp, ctypes.POINTER(Stats)]
_lib.lt_get_pool_state.argtypes = [_vp, ctypes.POINTER(PoolState)]
_lib.lt_pending.argtypes = [_vp, ctypes.POINTER(_u64), _vp]
_lib.lt_exchange_pack.argtypes = [_vp, _vp, _u64, _vp]
_lib.lt_exchange_insert.argtypes = [_vp, _vp, _u64]
_lib.lt_exchange_buffers.argtypes = [_vp, _u64, _vp, _vp]
_lib.lt_exchange_attach.argtypes = [_vp, _vp, _vp]
_lib.lt_exchange_sent.argtypes = [_vp, ctypes.POINTER(_u64)]
_lib.lt_exchange_take.argtypes = [_vp, ctypes.POINTER(_u64)]
_lib.lt_ipc_handle.argtypes = [_vp, _vp]
_lib.lt_ipc_open.argtypes = [_vp, _vp, ctypes.POINTER(_vp)]
_lib.lt_superstep_p2p.argtypes = [_vp, _vp]
_lib.lt_paths_buffers.argtypes = [_vp, ctypes.POINTER(_vp), ctypes.POINTER(_vp), ctypes.POINTER(_u64)]
_lib.lt_paths_attach.argtypes = [_vp, _vp, _vp, _u64]
_lib.lt_philox_device.argtypes = [ctypes.c_int, _u64, _vp, _vp, _vp]
_lib.lt_compress_columns.argtypes = [_vp, _u64, _vp, _vp, ctypes.POINTER(_u64)]


def compress_columns(col):
    """lt_compress_columns (host): (hdr u32[nblk + 1, 2], payload u32[words]) of a u32 column slice."""
    col = np.ascontiguousarray(col, dtype=np.uint32)
    words = _u64()
    _check(_lib.lt_compress_columns(col.ctypes.data, len(col), None, None, ctypes.byref(words)))
    hdr = np.zeros(((len(col) + 31) // 32 + 1, 2), dtype=np.uint32)
    pay = np.zeros(max(1, words.value), dtype=np.uint32)
    _check(_lib.lt_compress_columns(col.ctypes.data, len(col), hdr.ctypes.data, pay.ctypes.data, ctypes.byref(words)))
    return hdr, pay[:words.value]


def philox_device(ctr, key, device: int = 0) -> np.ndarray:
    """The update kernels' Philox4x32-10 on the device (lt_philox_device): ctr u32[n, 4], key u32[n, 2]."""
    ctr = np.ascontiguousarray(ctr, dtype=np.uint32).reshape(-1, 4)
    key = np.ascontiguousarray(key, dtype=np.uint32).reshape(-1, 2)
    assert len(ctr) == len(key)
    out = np.zeros_like(ctr)
    _check(_lib.lt_philox_device(device, len(ctr), ctr.ctypes.data, key.ctypes.data, out.ctypes.data))
    return out
_lib.lt_run_to_host.argtypes = [_vp, _u64, _vp, _u64, ctypes.c_int, ctypes.c_double, _u64, _vp, _vp, _u32]
_lib.lt_run_to_host_compact.argtypes = [_vp, _u64, _vp, _u64, ctypes.c_int, ctypes.c_double, _u64, _vp, _vp, _u64, _u32]
_lib.lt_get_paths_compact.argtypes = [_vp, _vp, _vp, _u64, ctypes.POINTER(_u64)]


def ipc_handle(dptr: int) -> bytes:
    """CUDA IPC handle (64 bytes) of the device allocation at dptr (an allocation base)."""
    buf = ctypes.create_string_buffer(64)
    _check(_lib.lt_ipc_handle(_vp(dptr), buf))
    return buf.raw


class LTError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"lt status {status}: {msg}")
        self.status = status


def _check(status):
    if status != LT_OK:
        raise LTError(status, _lib.lt_last_error().decode(errors="replace"))


def _is_torch(x):
    return type(x).__module__.startswith("torch")


def _ptr(x, np_dtype):
    """(pointer, on_device, keepalive) for a numpy array or torch tensor of the given bit width."""
    if x is None:
        return None, False, None
    if _is_torch(x):
        if not x.is_contiguous():
            raise ValueError("tensor must be contiguous")
        if x.element_size() != np.dtype(np_dtype).itemsize:
            raise ValueError(f"tensor element size must be {np.dtype(np_dtype).itemsize}")
        return x.data_ptr(), bool(x.is_cuda), x
    a = np.ascontiguousarray(x)
    if a.dtype != np_dtype:
        if a.dtype.itemsize == np.dtype(np_dtype).itemsize and a.dtype.kind in "iu":
            a = a.view(np_dtype)
        else:
            a = a.astype(np_dtype)
    return a.ctypes.data, False, a


def partition_bounds(row_ptr, num_partitions: int) -> np.ndarray:
    """Host-only range partitioner (lt_partition_bounds)."""
    p, dev, keep = _ptr(row_ptr, np.uint64)
    assert not dev, "partition_bounds takes host row_ptr"
    n = len(keep) - 1
    out = np.zeros(num_partitions + 1, dtype=np.uint32)
    _check(_lib.lt_partition_bounds(n, p, num_partitions, out.ctypes.data))
    return out


class Engine:
    """One lt_ctx on one GPU."""

    def __init__(self, device: int = 0, chunk_walks: int = 8192, ppr_max_len: int = 127,
                 policy: int = POLICY_SELECTIVE, insert_mode: int = INSERT_WARP_AGGREGATED,
                 timing: bool = False, stream=None, blocks_per_sm: int = 0, l2_fetch_bytes: int = 0,
                 gather_mode: int = 3, ilp: int = 0, layout: int = LAYOUT_AUTO,
                 path_mode: int = 0, graph_pool_bytes: int = 0, zero_copy: bool = False,
                 zc_alpha_bytes: int = 0, rank: int = 0, world: int = 1, refill: int = 0,
                 visit_counts: bool = False, continue_resident: bool = False, walk_pool_walks: int = 0,
                 direct_start: bool = True, l2_persist: int = 0, ooc_prefetch: bool = False,
                 walk_spill: bool = False, arena=None, ooc_compress: bool = True):
        cfg = Config()
        _check(_lib.lt_config_default(ctypes.byref(cfg)))
        cfg.device = device
        cfg.stream = stream
        cfg.chunk_walks = chunk_walks
        cfg.ppr_max_len = ppr_max_len
        cfg.policy = policy
        cfg.insert_mode = insert_mode
        cfg.timing = int(bool(timing))
        cfg.blocks_per_sm = blocks_per_sm
        cfg.l2_fetch_bytes = l2_fetch_bytes
        cfg.gather_mode = gather_mode
        cfg.ilp = ilp
        cfg.layout = layout
        cfg.path_mode = path_mode
        cfg.graph_pool_bytes = graph_pool_bytes
        cfg.zero_copy = int(bool(zero_copy))
        cfg.zc_alpha_bytes = zc_alpha_bytes
        cfg.rank = rank
        cfg.world = world
        cfg.refill = refill
        cfg.continue_resident = int(bool(continue_resident))
        cfg.walk_pool_walks = int(walk_pool_walks)
        cfg.walk_spill = int(bool(walk_spill))
        if arena is not None:  # caller-owned device memory (a CUDA tensor) for every pool
            if not (_is_torch(arena) and arena.is_cuda and arena.is_contiguous()):
                raise ValueError("arena must be a contiguous CUDA tensor")
            cfg.arena = arena.data_ptr()
            cfg.arena_bytes = arena.numel() * arena.element_size()
        self._arena_keep = arena
        cfg.direct_start = 0 if direct_start else 1  # 0 auto (on where it applies), 1 off
        cfg.l2_persist = int(l2_persist)
        cfg.ooc_compress = 0 if ooc_compress else 1  # 0 auto (compressed partition copies), 1 off
        cfg.ooc_prefetch = int(bool(ooc_prefetch))
        cfg.visit_counts = int(visit_counts)  # False/0 off, True/1 on (auto counter width), 2 u64 counters
        self._lmax = ppr_max_len
        self.rank, self.world, self.device = rank, world, device
        h = _vp()
        _check(_lib.lt_create(ctypes.byref(cfg), ctypes.byref(h)))
        self._h = h
        self._graph_keep = None
        self.num_walks = 0

    def close(self):
        if getattr(self, "_h", None):
            _lib.lt_destroy(self._h)
            self._h = None
        self._graph_keep = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def graph_load(self, row_ptr, col, num_partitions: int):
        prp, dev_r, krp = _ptr(row_ptr, np.uint64)
        pcol, dev_c, kcol = _ptr(col, np.uint32)
        if dev_r != dev_c:
            raise ValueError("row_ptr and col must both be host or both be device")
        n = (len(krp) if not _is_torch(krp) else krp.numel()) - 1
        m = len(kcol) if not _is_torch(kcol) else kcol.numel()
        if dev_r:
            _check(_lib.lt_graph_load_device(self._h, n, m, prp, pcol, num_partitions))
            # borrowed device memory stays alive; col only while the steps read it (CSR layout)
            self._graph_keep = (krp, kcol) if self.stats()["layout"] == LAYOUT_CSR else (krp,)
        else:
            _check(_lib.lt_graph_load(self._h, n, m, prp, pcol, num_partitions))
            self._graph_keep = None
        self.n, self.m = n, m

    def bounds(self) -> np.ndarray:
        P = _u32()
        _check(_lib.lt_get_bounds(self._h, None, ctypes.byref(P)))
        out = np.zeros(P.value + 1, dtype=np.uint32)
        _check(_lib.lt_get_bounds(self._h, out.ctypes.data, ctypes.byref(P)))
        return out

    def walks_init(self, starts, app: int = DEEPWALK, param: float = 80, seed: int = 1, first_walk_id: int = 0):
        p, dev, keep = _ptr(starts, np.uint32)
        W = keep.numel() if _is_torch(keep) else len(keep)
        _check(_lib.lt_walks_init_ex(self._h, W, p, int(dev), first_walk_id, app, float(param), seed))
        self._starts_keep = keep
        self.num_walks = W

    def walks_init_pagerank(self, starts, length: int, restart_p: float, seed: int = 1, first_walk_id: int = 0):
        """PageRank / random walk with restart (lt_walks_init_pagerank)."""
        p, dev, keep = _ptr(starts, np.uint32)
        W = keep.numel() if _is_torch(keep) else len(keep)
        _check(_lib.lt_walks_init_pagerank(self._h, W, p, int(dev), first_walk_id, int(length), float(restart_p), seed))
        self._starts_keep = keep
        self.num_walks = W

    def visit_counts(self, out=None):
        """Per-vertex visit frequency u64[n] (lt_get_visit_counts; needs visit_counts=True). `out` may be a
        host array or a CUDA int64 tensor (device copy)."""
        if out is None:
            out = np.zeros(self.n, dtype=np.uint64)
        p, dev, keep = _ptr(out, np.uint64)
        _check((_lib.lt_get_visit_counts_device if dev else _lib.lt_get_visit_counts)(self._h, p))
        return out

    def run(self):
        _check(_lib.lt_run(self._h))

    def run_to_host(self, starts, app: int = DEEPWALK, param: float = 80, seed: int = 1, first_walk_id: int = 0,
                    paths=None, lengths=None, chunks: int = 0):
        """Walk and copy every path to host buffers with the copy-out overlapped (lt_run_to_host).
        starts/paths/lengths are host arrays (pinned torch tensors for overlapped copies)."""
        ps, dev, keep = _ptr(starts, np.uint32)
        if dev:
            raise ValueError("run_to_host takes host starts")
        W = keep.numel() if _is_torch(keep) else len(keep)
        S = (int(param) + 1) if app == DEEPWALK else self._lmax + 1
        if paths is None:
            paths = np.empty((W, S), dtype=np.uint32)
        if lengths is None:
            lengths = np.empty(W, dtype=np.uint32)
        pp, dp, kp = _ptr(paths, np.uint32)
        pl, dl, kl = _ptr(lengths, np.uint32)
        if dp or dl:
            raise ValueError("run_to_host writes host buffers")
        _check(_lib.lt_run_to_host(self._h, W, ps, first_walk_id, app, float(param), seed, pp, pl, chunks))
        return paths, lengths

    def run_to_host_compact(self, starts, app: int = DEEPWALK, param: float = 80, seed: int = 1,
                            first_walk_id: int = 0, offsets=None, vertices=None, chunks: int = 0):
        """lt_run_to_host with the ragged output: (offsets u64[W+1], vertices u32[offsets[W]]).
        Preallocated host buffers (pinned torch tensors for overlapped copies) may be passed; vertices
        needs room for W * stride entries in the worst case."""
        ps, dev, keep = _ptr(starts, np.uint32)
        if dev:
            raise ValueError("run_to_host_compact takes host starts")
        W = keep.numel() if _is_torch(keep) else len(keep)
        S = (int(param) + 1) if app == DEEPWALK else self._lmax + 1
        if offsets is None:
            offsets = np.empty(W + 1, dtype=np.uint64)
        if vertices is None:
            vertices = np.empty(max(W * S, 1), dtype=np.uint32)
        po, do, ko = _ptr(offsets, np.uint64)
        pv, dv, kv = _ptr(vertices, np.uint32)
        if do or dv:
            raise ValueError("run_to_host_compact writes host buffers")
        cap = kv.numel() if _is_torch(kv) else len(kv)
        _check(_lib.lt_run_to_host_compact(self._h, W, ps, first_walk_id, app, float(param), seed, po, pv, cap, chunks))
        total = int(offsets[W])
        return offsets, vertices[:total]

    def get_paths_compact(self):
        """Ragged copy-out (lt_get_paths_compact): (offsets u64[W+1], vertices u32[offsets[W]])."""
        W, S = self.num_walks, self.stride()
        offsets = np.empty(W + 1, dtype=np.uint64)
        vertices = np.empty(max(W * S, 1), dtype=np.uint32)
        total = _u64()
        _check(_lib.lt_get_paths_compact(self._h, offsets.ctypes.data, vertices.ctypes.data, len(vertices),
                                         ctypes.byref(total)))
        return offsets, vertices[: total.value]

    def stride(self) -> int:
        s = _u32()
        _check(_lib.lt_path_stride(self._h, ctypes.byref(s)))
        return s.value

    def get_paths(self, paths=None, lengths=None):
        """Copy paths/lengths to host. Pass preallocated (e.g. pinned torch) buffers to reuse them;
        pass paths=False to skip the path matrix."""
        W, S = self.num_walks, self.stride()
        if paths is None:
            paths = np.empty((W, S), dtype=np.uint32)
        if lengths is None:
            lengths = np.empty(W, dtype=np.uint32)
        pp, dp, kp = _ptr(paths, np.uint32) if paths is not False else (None, False, None)
        pl, dl, kl = _ptr(lengths, np.uint32)
        if dp or dl:
            raise ValueError("get_paths copies to host; use get_paths_device for device buffers")
        _check(_lib.lt_get_paths(self._h, pp, pl))
        return (paths if paths is not False else None), lengths

    def get_paths_rows(self, rows):
        rows = np.ascontiguousarray(rows, dtype=np.uint64)
        S = self.stride()
        out = np.empty((len(rows), S), dtype=np.uint32)
        ln = np.empty(len(rows), dtype=np.uint32)
        _check(_lib.lt_get_paths_rows(self._h, rows.ctypes.data, len(rows), out.ctypes.data, ln.ctypes.data))
        return out, ln

    def get_paths_device(self, d_paths, d_lengths):
        pp, dp, _ = _ptr(d_paths, np.uint32)
        pl, dl, _ = _ptr(d_lengths, np.uint32)
        if (d_paths is not None and not dp) or (d_lengths is not None and not dl):
            raise ValueError("get_paths_device needs CUDA tensors")
        _check(_lib.lt_get_paths_device(self._h, pp, pl))

    # ---- range ownership across ranks (include/lt.h "Range ownership"; driven by dist.py)
    def pending(self):
        """(walks in owned buckets, [walks in the send bucket of each rank])"""
        loc = _u64()
        out = np.zeros(self.world, dtype=np.uint64)
        _check(_lib.lt_pending(self._h, ctypes.byref(loc), out.ctypes.data))
        return int(loc.value), [int(x) for x in out]

    def exchange_pack(self, d_send):
        """Move every send bucket into the CUDA int32 tensor d_send [capacity, 4] (16-B records grouped
        by destination rank); returns the per-rank record counts."""
        pp, dev, keep = _ptr(d_send, np.uint32)
        if d_send is not None and not dev:
            raise ValueError("exchange_pack needs a CUDA tensor")
        cap = keep.numel() // 4 if keep is not None else 0
        counts = np.zeros(self.world, dtype=np.uint64)
        _check(_lib.lt_exchange_pack(self._h, pp, cap, counts.ctypes.data))
        return [int(x) for x in counts]

    def exchange_insert(self, d_recv, count: int):
        pp, dev, _ = _ptr(d_recv, np.uint32)
        if d_recv is not None and count and not dev:
            raise ValueError("exchange_insert needs a CUDA tensor")
        _check(_lib.lt_exchange_insert(self._h, pp, count))
        self._recv_keep = d_recv  # read asynchronously by the insert kernel (stream-ordered)

    # ---- peer exchange (lt_exchange_buffers / attach / sent / take; dist.run_supersteps_p2p)
    def exchange_buffers(self, capacity: int):
        """This rank's receive buffers and cursors (device addresses) for parity 0 and 1."""
        recv = (_vp * 2)()
        cur = (_vp * 2)()
        _check(_lib.lt_exchange_buffers(self._h, int(capacity), recv, cur))
        self._xcap = int(capacity)
        return [int(x) for x in recv], [int(x) for x in cur]

    def exchange_attach(self, recv, cursor):
        """recv / cursor: 2 * world device addresses, [e * world + q] = rank q's buffer of parity e."""
        r = (_vp * len(recv))(*recv)
        c = (_vp * len(cursor))(*cursor)
        _check(_lib.lt_exchange_attach(self._h, r, c))

    def exchange_sent(self) -> int:
        x = _u64()
        _check(_lib.lt_exchange_sent(self._h, ctypes.byref(x)))
        return int(x.value)

    def exchange_take(self) -> int:
        x = _u64()
        _check(_lib.lt_exchange_take(self._h, ctypes.byref(x)))
        return int(x.value)

    def superstep_p2p(self, d_sent):
        """One fused superstep (lt_superstep_p2p); d_sent: CUDA int64 tensor [1] receiving the number of
        records this rank sent. No host synchronisation."""
        pp, dev, _ = _ptr(d_sent, np.uint64)
        if not dev:
            raise ValueError("superstep_p2p needs a CUDA tensor")
        _check(_lib.lt_superstep_p2p(self._h, pp))

    def paths_buffers(self):
        """Home rank: (path matrix, length array, capacity in u32 entries) device addresses (lt_paths_buffers)."""
        p, l, c = _vp(), _vp(), _u64()
        _check(_lib.lt_paths_buffers(self._h, ctypes.byref(p), ctypes.byref(l), ctypes.byref(c)))
        return int(p.value), int(l.value), int(c.value)

    def paths_attach(self, d_paths, d_lengths, capacity: int):
        """Write this rank's path entries and lengths into the home rank's buffers (lt_paths_attach);
        (None, None, 0) writes locally again."""
        _check(_lib.lt_paths_attach(self._h, _vp(d_paths) if d_paths else None, _vp(d_lengths) if d_lengths else None,
                                    int(capacity)))

    def home_paths(self):
        """Home rank after the epoch: (paths [W, stride], lengths [W]) CUDA int32 tensors (all ranks' entries)."""
        return self.partial_paths()

    def export_buffers(self):
        """CUDA IPC handles of this rank's receive buffers (parity 0, 1) and of its cursor pair."""
        recv, cur = self.exchange_buffers(self._xcap)
        return ipc_handle(recv[0]), ipc_handle(recv[1]), ipc_handle(cur[0])

    def import_buffers(self, handles):
        """Open another rank's export_buffers() handles: ([recv0, recv1], [cursor0, cursor1])."""
        r0, r1, c0 = (self.ipc_open(h) for h in handles)
        return [r0, r1], [c0, c0 + 256]  # cursor[1] = cursor[0] + 256 bytes (one allocation, lt.h)

    def ipc_open(self, handle: bytes) -> int:
        """Open another process's CUDA IPC handle (64 bytes) on this engine's device."""
        buf = ctypes.create_string_buffer(bytes(handle), 64)
        out = _vp()
        _check(_lib.lt_ipc_open(self._h, buf, ctypes.byref(out)))
        return int(out.value)

    def partial_paths(self):
        """This rank's share of paths (CUDA int32 tensors [W, stride], [W]) for the cross-rank merge."""
        import torch
        W, S = self.num_walks, self.stride()
        paths = torch.empty((W, S), dtype=torch.int32, device=f"cuda:{self.device}")
        lengths = torch.empty(W, dtype=torch.int32, device=f"cuda:{self.device}")
        if W:
            self.get_paths_device(paths, lengths)
        return paths, lengths

    def pool_state(self) -> dict:
        s = PoolState()
        _check(_lib.lt_get_pool_state(self._h, ctypes.byref(s)))
        return {name: getattr(s, name) for name, _ in PoolState._fields_}

    def stats(self) -> dict:
        s = Stats()
        _check(_lib.lt_get_stats(self._h, ctypes.byref(s)))
        return {name: getattr(s, name) for name, _ in Stats._fields_}
