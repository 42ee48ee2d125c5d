"""Multi-GPU range-ownership mode (the north star's 8-GPU mode, not in
the paper): the superstep exchange around the C ABI.

Rank r owns a contiguous range of partitions (lt_config.rank/world). Each superstep:
  1. lt_run            advance every walk in the owned buckets until it ends or leaves the range
                       (walks for rank q collect in send bucket q);
  2. lt_exchange_pack  move the send buckets into one device buffer, grouped by destination (the
                       counts come from lt_run's last count read: no extra device round trip);
  3. all-gather        of every rank's per-destination counts (R x R): each rank reads what it will
                       receive and the global number of crossing walks (the termination test) from
                       the same matrix, in ONE small collective;
  4. all-to-all        of the 16-B walk records (NCCL over NVLink via torch.distributed; gloo on CPU
                       in the tests), stream-ordered after the pack;
  5. lt_exchange_insert the received walks into the owned buckets (warp-aggregated insertion),
                       stream-ordered, no host synchronisation;
until no walk crossed ranks in a superstep (every live walk is then in some owned bucket, and lt_run
ended them all). Host round trips per superstep: lt_run's count reads and the count all-gather.
Paths are merged once at the end: element-wise unsigned min of the path rows (unwritten entries are
0xFFFFFFFF) and max of the lengths.

The exchange is the only data-path collective; this module only sequences ABI calls and
collectives (plumbing), every walk step runs in the CUDA kernels behind the ABI.
"""
from __future__ import annotations

import threading

SIGN = -0x80000000  # int32 with only the sign bit: x ^ SIGN maps unsigned order onto signed order


class TorchComm:
    """Collectives over a torch.distributed process group (NCCL for CUDA tensors, gloo for CPU)."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)

    def alltoall_counts(self, counts, device):
        import torch
        t = torch.tensor(counts, dtype=torch.int64, device=device)
        out = torch.empty_like(t)
        self.dist.all_to_all_single(out, t, group=self.group)
        return [int(x) for x in out.tolist()]

    def allgather_counts(self, counts, device):
        """Every rank's count vector: returns the R x R matrix M (M[r][q] = records r sends to q)."""
        import torch
        t = torch.tensor(counts, dtype=torch.int64, device=device)
        parts = [torch.empty_like(t) for _ in range(self.world)]
        self.dist.all_gather(parts, t, group=self.group)
        m = torch.stack(parts).tolist()
        return [[int(x) for x in row] for row in m]

    def alltoallv(self, send, send_counts, recv_counts):
        """send: int32 [sum(send_counts), 4]; returns int32 [sum(recv_counts), 4]."""
        import torch
        recv = torch.empty((sum(recv_counts), 4), dtype=torch.int32, device=send.device)
        self.dist.all_to_all_single(recv.view(-1), send[: sum(send_counts)].reshape(-1).contiguous(),
                                    output_split_sizes=[4 * c for c in recv_counts],
                                    input_split_sizes=[4 * c for c in send_counts], group=self.group)
        return recv

    def allreduce_sum(self, x: int, device) -> int:
        import torch
        t = torch.tensor([x], dtype=torch.int64, device=device)
        self.dist.all_reduce(t, group=self.group)
        return int(t.item())

    def allreduce_(self, t, op: str):
        ops = {"min": self.dist.ReduceOp.MIN, "max": self.dist.ReduceOp.MAX, "sum": self.dist.ReduceOp.SUM}
        self.dist.all_reduce(t, op=ops[op], group=self.group)

    def allreduce_dev_(self, t):
        """In-place sum of a device tensor over ranks (NCCL: enqueued, no host synchronisation)."""
        self.dist.all_reduce(t, group=self.group)

    def allgather_obj(self, obj):
        out = [None] * self.world
        self.dist.all_gather_object(out, obj, group=self.group)
        return out

    same_process = False


class ThreadComm:
    """In-process collectives between `world` threads (each driving one Engine), used to exercise
    the ownership mode with several engines on one GPU. Create one shared ThreadComm.Hub and a
    ThreadComm(hub, rank) per thread."""

    class Hub:
        def __init__(self, world):
            self.world = world
            self.barrier = threading.Barrier(world)
            self.slots = [None] * world

    def __init__(self, hub, rank):
        self.hub, self.rank, self.world = hub, rank, hub.world

    def _gather(self, x):
        self.hub.barrier.wait()
        self.hub.slots[self.rank] = x
        self.hub.barrier.wait()
        allv = list(self.hub.slots)
        self.hub.barrier.wait()
        return allv

    def alltoall_counts(self, counts, device):
        allc = self._gather(list(counts))
        return [allc[r][self.rank] for r in range(self.world)]

    def allgather_counts(self, counts, device):
        return [list(c) for c in self._gather(list(counts))]

    def alltoallv(self, send, send_counts, recv_counts):
        import torch
        offs = [0]
        for c in send_counts:
            offs.append(offs[-1] + c)
        # the copies out of the other ranks' send buffers must be complete before the last barrier:
        # once past it a sender may start its next superstep and pack into the same buffer; and the
        # sender's pack (on the engine's stream) must be complete before anyone reads its buffer
        if send.is_cuda:
            torch.cuda.synchronize(send.device)
        self.hub.barrier.wait()
        self.hub.slots[self.rank] = (send, offs)
        self.hub.barrier.wait()
        allv = list(self.hub.slots)
        parts = [allv[r][0][allv[r][1][self.rank]: allv[r][1][self.rank + 1]].to(send.device, copy=True)
                 for r in range(self.world)]
        out = torch.cat(parts) if parts else send[:0].clone()
        if out.is_cuda:
            torch.cuda.current_stream(out.device).synchronize()
        self.hub.barrier.wait()
        return out

    def allreduce_sum(self, x: int, device) -> int:
        return sum(self._gather(int(x)))

    def allgather_obj(self, obj):
        return self._gather(obj)

    def allreduce_dev_(self, t):
        t.fill_(sum(self._gather(int(t.item()))))

    same_process = True

    def allreduce_(self, t, op: str):
        allv = self._gather(t.clone())
        acc = allv[0].to(t.device)
        for o in allv[1:]:
            o = o.to(t.device)
            acc = acc.minimum(o) if op == "min" else acc.maximum(o) if op == "max" else acc + o
        t.copy_(acc)


def send_buffer(engine, device, cache: dict):
    """A device buffer large enough for every walk this rank holds in its send buckets."""
    import torch
    _, out = engine.pending()
    need = max(sum(out), 1)
    buf = cache.get("send")
    if buf is None or buf.shape[0] < need:
        buf = torch.empty((max(need, 2 * (0 if buf is None else buf.shape[0])), 4), dtype=torch.int32, device=device)
        cache["send"] = buf
    return buf


def run_supersteps(engine, comm, device, max_supersteps: int = 1 << 20) -> dict:
    """Drive lt_run + exchange until no walk is alive on any rank. Returns counters."""
    cache: dict = {}
    supersteps, moved = 0, 0
    while True:
        engine.run()
        buf = send_buffer(engine, device, cache)
        counts = engine.exchange_pack(buf)
        mat = comm.allgather_counts(counts, device)  # mat[r][q]: records rank r sends to rank q
        crossed = sum(sum(row) for row in mat)
        supersteps += 1
        moved += sum(counts)
        if crossed == 0:
            return {"supersteps": supersteps, "records_sent": moved}
        recv_counts = [mat[r][comm.rank] for r in range(comm.world)]
        recv = comm.alltoallv(buf, counts, recv_counts)
        engine.exchange_insert(recv, sum(recv_counts))
        if supersteps >= max_supersteps:
            raise RuntimeError("ownership supersteps did not converge")


def attach_peers(engine, comm, capacity: int):
    """Peer exchange setup (lt_exchange_buffers / lt_exchange_attach): every rank allocates its two
    receive buffers of `capacity` records, the ranks share them — raw device addresses between
    threads of one process, CUDA IPC handles between processes (lt_ipc_handle / lt_ipc_open) — and
    each rank installs the table of every rank's buffers."""
    recv, cur = engine.exchange_buffers(capacity)
    R, me = comm.world, comm.rank
    if comm.same_process:
        allv = comm.allgather_obj((recv, cur))
    else:  # CUDA IPC handles (Engine.export_buffers / import_buffers)
        hs = comm.allgather_obj(engine.export_buffers())
        allv = [(recv, cur) if q == me else engine.import_buffers(hs[q]) for q in range(R)]
    table_r = [allv[q][0][e] for e in range(2) for q in range(R)]
    table_c = [allv[q][1][e] for e in range(2) for q in range(R)]
    engine.exchange_attach(table_r, table_c)


def run_supersteps_p2p(engine, comm, device, max_supersteps: int = 1 << 20) -> dict:
    """Superstep loop of the peer exchange: the update kernels already appended every walk that
    crossed ranks into its owner's receive buffer (peer memory, overlapped with the steps), so a
    superstep is lt_run, ONE small collective (the sum of records sent, which is also the barrier
    after which every receive buffer of this parity is complete) and lt_exchange_take."""
    supersteps, moved = 0, 0
    while True:
        engine.run()
        sent = engine.exchange_sent()
        total = comm.allreduce_sum(sent, device)
        supersteps += 1
        moved += sent
        if total == 0:
            return {"supersteps": supersteps, "records_sent": moved}
        engine.exchange_take()
        if supersteps >= max_supersteps:
            raise RuntimeError("ownership supersteps did not converge")


def run_supersteps_p2p_fused(engine, comm, device, max_supersteps: int = 1 << 20, sync_every: int = 4) -> dict:
    """The peer-exchange superstep loop without per-superstep host decisions (one owned partition per
    rank): lt_superstep_p2p (insert arrivals, step every owned walk, count what was sent — all
    stream-ordered) and a device all-reduce of the sent count. The host reads that sum only every
    `sync_every` supersteps: a superstep after the last walk ended is empty and cheap (nothing to
    insert, an update launch over an empty bucket), so running up to sync_every - 1 of them costs less
    than a host round trip per superstep. A zero sum ends the loop; a final lt_run (no walk left)
    finalises statistics and visit counts."""
    import torch
    sent = torch.zeros(1, dtype=torch.int64, device=device)
    moved = torch.zeros(1, dtype=torch.int64, device=device)  # this rank's records sent, summed on the device
    supersteps = 0
    while True:
        engine.superstep_p2p(sent)
        moved += sent
        comm.allreduce_dev_(sent)  # NCCL: asynchronous; threads: a host gather
        supersteps += 1
        if supersteps % sync_every == 0 or comm.same_process:
            if int(sent.item()) == 0:
                engine.run()
                return {"supersteps": supersteps, "records_sent": int(moved.item())}
        if supersteps >= max_supersteps:
            raise RuntimeError("ownership supersteps did not converge")


def attach_paths(engine, comm, home: int = 0):
    """Paths on the home rank (lt_paths_buffers / lt_paths_attach): every rank writes its path entries and
    lengths straight into the home rank's matrix over peer memory, so no merge is needed (SURVEY.md §8(b):
    the merged result lands on rank 0). Call once, after every rank's walks_init of the first epoch
    (path_mode 0) and before its superstep loop: it synchronises the device and barriers so that no rank
    writes into the home matrix before the home's walks_init (which pre-fills it that once) has run; later
    epochs stay attached and need no call (include/lt.h). Calling it again is harmless. Handles are
    exchanged once and cached on the engine."""
    import torch
    me = comm.rank
    key = getattr(engine, "_home_key", None)
    if me == home:
        p, l, cap = engine.paths_buffers()
        mine = (p, l, cap) if comm.same_process else (lt_ipc(p), lt_ipc(l), cap, p, l)
    else:
        mine = None
    allv = comm.allgather_obj(mine)
    hv = allv[home]
    if me != home:
        if comm.same_process:
            p, l, cap = hv
        else:
            if key != (hv[3], hv[4]):  # open the home's IPC handles once per allocation
                engine._home_ptrs = (engine.ipc_open(hv[0]), engine.ipc_open(hv[1]))
                engine._home_key = (hv[3], hv[4])
            p, l = engine._home_ptrs
            cap = hv[2]
        engine.paths_attach(p, l, cap)
    torch.cuda.synchronize()
    comm.allgather_obj(None)  # barrier: the home's pre-fill is complete before anyone writes into it


def lt_ipc(dptr: int) -> bytes:
    from .lt import ipc_handle
    return ipc_handle(dptr)


def merge_paths(engine, comm):
    """Cross-rank merge of the partial path matrices: unsigned min of entries, max of lengths.
    Returns CUDA/CPU int32 tensors (paths [W, stride], lengths [W]) identical on every rank."""
    paths, lengths = engine.partial_paths()
    paths ^= SIGN
    comm.allreduce_(paths, "min")
    paths ^= SIGN
    comm.allreduce_(lengths, "max")
    return paths, lengths


def merge_visit_counts(engine, comm, device):
    """Global per-vertex visit frequency: each rank counted the starts it kept and the
    steps it took, so the global count is the sum over ranks. Returns an int64 tensor [n] (u64 bits)."""
    import torch
    counts = torch.empty(engine.n, dtype=torch.int64, device=device)
    engine.visit_counts(counts)
    comm.allreduce_(counts, "sum")
    return counts
