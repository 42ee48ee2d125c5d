"""Test-only CPU stand-in for one rank of the range-ownership mode (include/lt.h "Range ownership").

It implements the Engine methods dist.run_supersteps / dist.merge_paths call (run, pending,
exchange_pack, exchange_insert, partial_paths) with per-visit stepping built on the ORACLE's
primitives (Philox and Lemire from oracle/), so the multi-process protocol (ownership ranges,
send buckets, count + payload all-to-all, termination, min/max merge) can run on CPU under gloo.
It is not the product: the product's kernels are exercised by tests/test_gpu_ownership.py.

The peer exchange (dist.attach_peers / run_supersteps_p2p) is emulated with POSIX shared memory:
rank q's receive buffer of parity e is one segment per sender (no cross-process atomics needed on
CPU), "device addresses" are (segment name, ...) tuples, export/import pass the names.
"""
from multiprocessing import shared_memory

import numpy as np

import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT

EMPTY = 0xFFFFFFFF


class CpuOwnerEngine:
    def __init__(self, g, P, rank, world):
        self.g, self.P, self.rank, self.world = g, P, rank, world
        self.bounds = LT.partition_bounds(g.row_ptr, P)
        self.own_lo = P * rank // world
        self.own_hi = P * (rank + 1) // world
        self.owner = np.zeros(P, dtype=np.int64)
        for r in range(world):
            self.owner[P * r // world: P * (r + 1) // world] = r

    # ---- peer exchange emulation (shared memory): segment layout per rank: [2 parities][world
    # senders] x (cursor u64 + capacity records of 4 u32)
    def exchange_buffers(self, capacity):
        self.xcap = int(capacity)
        self._seg_bytes = 8 + 16 * self.xcap
        name = f"ltp2p_{id(self) & 0xFFFFFF:x}_{self.rank}_{np.random.randint(1 << 30)}"
        self._own_shm = shared_memory.SharedMemory(name=name, create=True, size=2 * self.world * self._seg_bytes)
        self._own_shm.buf[:] = bytes(len(self._own_shm.buf))
        self._shms = {}
        return [(name, 0), (name, 1)], [(name, 0), (name, 1)]

    def export_buffers(self):
        return self._own_shm.name

    def import_buffers(self, name):
        return [(name, 0), (name, 1)], [(name, 0), (name, 1)]

    def exchange_attach(self, recv, cursor):
        self.peers = [recv[q][0] for q in range(self.world)]  # segment name of rank q
        for nm in self.peers:
            if nm != self._own_shm.name and nm not in self._shms:
                self._shms[nm] = shared_memory.SharedMemory(name=nm)
        self.epoch, self.sent = 0, 0

    def _seg(self, name, epoch, sender):
        shm = self._own_shm if name == self._own_shm.name else self._shms[name]
        off = (epoch * self.world + sender) * self._seg_bytes
        cur = np.ndarray((1,), dtype=np.uint64, buffer=shm.buf, offset=off)
        recs = np.ndarray((self.xcap, 4), dtype=np.uint32, buffer=shm.buf, offset=off + 8)
        return cur, recs

    def _send(self, q, rec):
        cur, recs = self._seg(self.peers[q], self.epoch, self.rank)
        i = int(cur[0])
        assert i < self.xcap, "peer receive buffer overflow"
        recs[i] = (rec[0], rec[1], rec[2], 0)
        cur[0] = i + 1
        self.sent += 1

    def exchange_sent(self):
        return self.sent

    def exchange_take(self):
        got = 0
        for sender in range(self.world):
            cur, recs = self._seg(self._own_shm.name, self.epoch, sender)
            for w, v, t, _ in recs[: int(cur[0])]:
                self.buckets[self._bucket(self._part(int(v)))].append((int(w), int(v), int(t)))
            got += int(cur[0])
            cur[0] = 0
        self.sent = 0
        self.epoch ^= 1
        return got

    def superstep_p2p(self, sent):
        """Fused superstep (lt_superstep_p2p): arrivals of the previous parity into the owned bucket,
        then the owned partition stepped once; `sent` (a tensor [1]) receives the records sent."""
        assert self.own_hi - self.own_lo == 1
        prev = self.epoch ^ 1
        for sender in range(self.world):
            cur, recs = self._seg(self._own_shm.name, prev, sender)
            for w, v, t, _ in recs[: int(cur[0])]:
                self.buckets[self._bucket(self._part(int(v)))].append((int(w), int(v), int(t)))
            cur[0] = 0
        self.sent = 0
        k = self.own_lo
        lo, hi = int(self.bounds[k]), int(self.bounds[k + 1])
        recs, self.buckets[k] = self.buckets[k], []
        for rec in recs:
            out = self._visit(rec, lo, hi)
            if out is not None:
                self._send(self._bucket(self._part(out[1])) - self.P, out)
        sent.fill_(self.sent)
        self.epoch ^= 1

    def close_exchange(self):
        for shm in self._shms.values():
            shm.close()
        self._own_shm.close()
        self._own_shm.unlink()

    def _part(self, v):
        return int(np.searchsorted(self.bounds, v, side="right") - 1)

    def _bucket(self, q):
        return q if self.own_lo <= q < self.own_hi else self.P + int(self.owner[q])

    def walks_init(self, starts, app, param, seed, lmax=127):
        self.app, self.param, self.seed, self.lmax = app, param, seed, lmax
        self.T = O.ppr_threshold(param) if app == LT.PPR else 0
        self.stride = int(param) + 1 if app == LT.DEEPWALK else lmax + 1
        self._init(starts)

    def walks_init_pagerank(self, starts, length, restart_p, seed):
        self.app, self.param, self.seed, self.lmax = LT.PAGERANK, length, seed, 127
        self.T = O.ppr_threshold(restart_p)
        self.stride = int(length) + 1
        self._init(starts)

    def _init(self, starts):
        W = len(starts)
        self.n = self.g.n
        self.counts = np.zeros(self.g.n, dtype=np.uint64)
        self.num_walks = W
        self.paths = np.full((W, self.stride), EMPTY, dtype=np.uint32)
        self.lengths = np.zeros(W, dtype=np.uint32)
        self.buckets = {b: [] for b in range(self.P + self.world)}
        for w in range(W):
            q = self._part(int(starts[w]))
            if self.own_lo <= q < self.own_hi:
                self.paths[w, 0] = starts[w]
                self.counts[int(starts[w])] += 1
                self.buckets[q].append((w, int(starts[w]), 0))

    def _visit(self, rec, lo, hi):
        w, v, t = rec
        rp, col = self.g.row_ptr, self.g.col
        while True:
            if self.app in (LT.DEEPWALK, LT.PAGERANK) and t == int(self.param):
                break
            if self.app == LT.PPR and t == self.lmax:
                break
            if self.app == LT.PPR:
                x0 = O.philox4x32_10([t, 0, w & 0xFFFFFFFF, w >> 32], [self.seed & 0xFFFFFFFF, self.seed >> 32])[0]
                if x0 < self.T:
                    break
            restart = False
            if self.app == LT.PAGERANK:
                x0 = O.philox4x32_10([t, 0, w & 0xFFFFFFFF, w >> 32], [self.seed & 0xFFFFFFFF, self.seed >> 32])[0]
                restart = x0 < self.T
            d = int(rp[v + 1] - rp[v])
            if restart:
                v, _ = O.lemire(self.seed, w, t, self.g.n)
            else:
                if d == 0:
                    break
                idx, _ = O.lemire(self.seed, w, t, d)
                v = int(col[int(rp[v]) + idx])
            t += 1
            self.paths[w, t] = v
            self.counts[v] += 1
            if not (lo <= v < hi):
                return (w, v, t)
        self.lengths[w] = t + 1
        return None

    def run(self):
        while True:
            ks = [k for k in range(self.own_lo, self.own_hi) if self.buckets[k]]
            if not ks:
                return
            for k in ks:
                lo, hi = int(self.bounds[k]), int(self.bounds[k + 1])
                recs, self.buckets[k] = self.buckets[k], []
                for rec in recs:
                    out = self._visit(rec, lo, hi)
                    if out is not None:
                        b = self._bucket(self._part(out[1]))
                        if b >= self.P and getattr(self, "peers", None):  # peer exchange: into rank q's buffer
                            self._send(b - self.P, out)
                        else:
                            self.buckets[b].append(out)

    def pending(self):
        loc = sum(len(self.buckets[k]) for k in range(self.own_lo, self.own_hi))
        return loc, [len(self.buckets[self.P + r]) if self.world > 1 else 0 for r in range(self.world)]

    def exchange_pack(self, buf):
        counts, off = [], 0
        for r in range(self.world):
            recs = self.buckets[self.P + r]
            self.buckets[self.P + r] = []
            for i, (w, v, t) in enumerate(recs):
                buf[off + i, 0] = w
                buf[off + i, 1] = int(np.uint32(v).view(np.int32))
                buf[off + i, 2] = t
                buf[off + i, 3] = 0
            counts.append(len(recs))
            off += len(recs)
        return counts

    def exchange_insert(self, recv, count):
        arr = recv[:count].numpy().view(np.uint32)
        for w, v, t, _ in arr:
            self.buckets[self._bucket(self._part(int(v)))].append((int(w), int(v), int(t)))

    def visit_counts(self, out):
        import torch
        out.copy_(torch.from_numpy(self.counts.view(np.int64)))
        return out

    def partial_paths(self):
        import torch
        return (torch.from_numpy(self.paths.view(np.int32).copy()),
                torch.from_numpy(self.lengths.view(np.int32).copy()))
