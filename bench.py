#!/usr/bin/env python3
"""Benchmark of the B200-native LightTraffic walk-update path (one JSON line on rank 0).

A "step" is one pass of the whole hot path over one batch of synthetic input: lt_walks_init (walk
records + path[w][0] + insertion into the start partitions' buckets, §8(a) a2/a5) followed by
lt_run (partition scheduler + walk-update/insertion kernels until every walk has terminated,
a3-a7). Workload (default): BASELINE.json configs[3], the Friendster-shaped R-MAT graph at scale 26
(1.8B tuples) with |V| DeepWalk walks of length 80 on one B200, HBM-resident.

  value     walk steps/s with inputs (graph, starts) resident in HBM, device-timed with CUDA events
            on the stream the library launches on, max over ranks.
  e2e       the same metric through the C ABI with HOST buffers: pinned starts copied H2D inside
            lt_walks_init, and every path and length copied D2H by lt_get_paths, per step.
  roofline  the update kernel (the dominant kernel): algorithmic bytes per launch / its CUDA-event
            timed average launch duration, against MEASURED_PEAKS.json hbm_gbs. Algorithmic bytes are
            SURVEY.md §8(d)'s per-unit figures at 32-B sector granularity with no cache reuse (DESIGN.md
            "Roofline"): 104 B per step (row_ptr pair 40 + col 32 + path entry 32) plus 16 B per
            record read (every visit) and 16 B per record write (every partition change).
            `gather` adds the measured random-access view: DRAM-missing gathers per second against
            the ceiling tools/gather_bench measured on this pool (profiles/gather_ceiling.json).
  cpu_baseline  the CPU oracle (oracle/, as it stands) on this box's host cores over a bounded
            sample of the same workload's walks (rank 0, N=1 only).

Multi-GPU (N>1, one process per GPU; `--gpus N` without torchrun re-launches itself under
torch.distributed.run): the north star's range-ownership mode by default — |V| walks in total over N
ranks, rank r owning a contiguous edge-balanced vertex range, walks crossing ranks appended by the
update kernels straight into the owner's receive buffer over peer memory, one small all-reduce per
superstep (strong scaling). The line adds a per-superstep breakdown and a `replicas_upper_bound` leg
(every rank the whole graph and |V|/N of the walks, no exchange: the communication-free bound).
`--mode replicas` makes the replicas run the headline instead (weak scaling: |V| walks per rank).
At N=1 the line adds `projection_8gpu`: the ownership mode's 8-GPU time predicted from one-GPU
measurements (the P=8 partitioned kernel's update time / 8 plus a per-superstep cost), stated with
its assumptions.
`--impl reference` times the oracle (the reference arm of this tier) on the host cores instead.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import lt_inputs  # noqa: E402

METRIC = "walk steps/sec (device-timed, max over ranks) at 1/2/4/8 B200; HBM GB/s vs peak"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="lt", choices=["lt", "reference"])
    ap.add_argument("--config", type=int, default=4, help="BASELINE.json configs[i-1]")
    ap.add_argument("--scale", type=int, default=None, help="override the config's R-MAT scale")
    ap.add_argument("--tuples", type=int, default=None)
    ap.add_argument("--partitions", type=int, default=None, help="P; default per DESIGN.md")
    ap.add_argument("--chunk-walks", type=int, default=8192)
    ap.add_argument("--policy", type=int, default=0)
    ap.add_argument("--insert-mode", type=int, default=0)
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--e2e-chunks", type=int, default=16, help="lt_run_to_host walk ranges (copy-out overlap)")
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="oracle sample budget")
    ap.add_argument("--layout", type=int, default=0, help="0 auto, 1 CSR, 2 ADJ, 3 ADJ12 (lt_layout)")
    ap.add_argument("--release-col", type=int, default=1,
                    help="1: once an augmented layout is built, keep a host copy of the CSR for the oracle legs "
                         "and free the device col (the steps never read it): room for the path matrix")
    ap.add_argument("--ilp", type=int, default=0)
    ap.add_argument("--gather-mode", type=int, default=3, help="lt_config.gather_mode: 3 L2 hints (default), 0 none")
    ap.add_argument("--l2-persist", type=int, default=0, help="lt_config.l2_persist: 1 = L2 set-aside for evict_last lines")
    ap.add_argument("--path-mode", type=int, default=0)
    ap.add_argument("--refill", type=int, default=0)
    ap.add_argument("--direct-start", type=int, default=1,
                    help="1: with P == 1 the update kernel takes new walks straight from starts (no records)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--sweep", default="", help="comma list of P values to time (extra key)")
    ap.add_argument("--graph-pool-gb", type=float, default=0.0,
                    help="> 0: out-of-core mode, CSR in pinned host memory, device graph pool of this size")
    ap.add_argument("--zero-copy", type=int, default=1, help="out-of-core: adaptive zero copy (PAPER.md:265)")
    ap.add_argument("--ooc-prefetch", type=int, default=1, help="out-of-core: load the next partition during a compute")
    ap.add_argument("--ooc-compress", type=int, default=1, help="out-of-core: partitions travel as compressed column blocks")
    ap.add_argument("--continue-resident", type=int, default=1,
                    help="out-of-core: walks keep stepping into partitions resident in the graph pool (f4)")
    ap.add_argument("--app", default="config", choices=["config", "deepwalk", "ppr", "pagerank"],
                    help="override the config's application; pagerank = random walk with restart "
                         "(PAPER.md:287, SURVEY.md 8(f) f2) of the config's length, with visit counting")
    ap.add_argument("--restart-p", type=float, default=0.15, help="PageRank restart probability")
    ap.add_argument("--visit-counts", type=int, default=-1, help="fused visit counting: -1 auto (on for pagerank)")
    ap.add_argument("--exchange", default="p2p", choices=["nccl", "p2p"],
                    help="--mode own: walks crossing ranks are appended by the update kernels straight into "
                         "the owner's receive buffer over peer memory (p2p, default: CUDA IPC, one small "
                         "all-reduce per superstep), or go through lt_exchange_pack + an NCCL all-to-all "
                         "(nccl, the baseline)")
    ap.add_argument("--mode", default=None, choices=["replicas", "own"],
                    help="N>1: own (default: range ownership, |V| walks in total, the crossing walks exchanged "
                         "every superstep, strong scaling) or replicas (each rank its own |V| walks, no "
                         "collective, weak scaling)")
    ap.add_argument("--project-gpus", type=int, default=8,
                    help="N=1, DeepWalk: predict the ownership mode's time at this many GPUs from one-GPU "
                         "measurements (0: off)")
    ap.add_argument("--no-replicas-bound", action="store_true", help="N>1 own mode: skip the replicas leg")
    return ap.parse_args()


def free_port():
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


def launch_ranks(args):
    """`--gpus N` (N > 1) outside torchrun: run this script under torch.distributed.run with one
    process per GPU (the driver's own launch line) and pass its output through."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


DEFAULT_P = {1: 4, 2: 1, 3: 1, 4: 1, 5: 1}


def workload(args):
    c = dict(lt_inputs.CONFIGS[args.config])
    if args.scale is not None:
        c["scale"] = args.scale
    if args.tuples is not None:
        c["tuples"] = args.tuples
    c["partitions"] = args.partitions if args.partitions is not None else (c.get("partitions") or DEFAULT_P[args.config])
    if args.app != "config" and args.app != c["app"]:
        c["name"] = f"{args.app} on {c['name']}"
        c["app"] = args.app
        c.setdefault("length", 80)
        c.setdefault("alpha", 0.15)
    if c["app"] == "pagerank":
        c["restart_p"] = args.restart_p
    return c


def app_param(c):
    import paper_conf_icde_xing0wxl23_b200 as LT
    if c["app"] == "deepwalk":
        return LT.DEEPWALK, float(c["length"])
    if c["app"] == "pagerank":
        return LT.PAGERANK, float(c["length"])
    return LT.PPR, float(c["alpha"])


def init_walks(eng, c, starts, seed, first):
    """lt_walks_init_ex, or lt_walks_init_pagerank for the random walk with restart."""
    import paper_conf_icde_xing0wxl23_b200 as LT
    app, param = app_param(c)
    if app == LT.PAGERANK:
        eng.walks_init_pagerank(starts, int(param), c["restart_p"], seed, first)
    else:
        eng.walks_init(starts, app, param, seed, first)


def starts_for(c, g, W, first):
    if c["app"] in ("deepwalk", "pagerank"):
        return lt_inputs.deepwalk_starts(W, g.n, first_walk_id=first)
    return lt_inputs.ppr_starts(W, g.argmax_deg)


def num_walks(c, g):
    return 4096 if c["walks"] == "4096" else g.n


# ------------------------------------------------------------------------------ clocks sampling
class Clocks:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(device), f"--query-gpu={self.FIELDS}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.p.terminate()
        self.p.wait()
        self.f.flush()
        rows = [r.split(",") for r in open(self.f.name).read().strip().splitlines() if r.strip()]
        os.unlink(self.f.name)
        sm = [float(r[1]) for r in rows if len(r) >= 9 and r[1].strip().replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if len(r) >= 9 and r[2].strip().replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            if len(r) < 9:
                continue
            for nm, val in zip(names, r[5:9]):
                if "Active" in val and "Not" not in val:
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------ CPU oracle legs
def oracle_sample(c, g_host, W, first, seconds, threads=None, runs=1):
    """Time the oracle (as it stands) on a bounded sample of the workload's walks — `runs` repetitions of
    the same spread sample (every k-th walk), median and spread reported — with one OpenMP thread per
    host core this process may use (explicitly: torchrun exports OMP_NUM_THREADS=1, which would otherwise
    leave the oracle on one core). The clock brackets the oracle's walk loop only (oracle_walks through
    ctypes, output buffers preallocated by the binding)."""
    if threads is None:
        threads = cores()
    import oracle as O
    app = {"deepwalk": O.DEEPWALK, "ppr": O.PPR, "pagerank": O.PAGERANK}[c["app"]]
    alpha = float(c["restart_p"]) if c["app"] == "pagerank" else float(c.get("alpha", 0.15))
    kw = dict(app=app, length=int(c.get("length", 0)), alpha=alpha, seed=c["seed"], threads=threads)
    all_starts = starts_for(c, g_host, W, first)
    # calibrate on a small spread sample, then size the sample for ~`seconds` / runs of work per run
    n0 = min(W, 200_000)
    ids0 = np.linspace(0, W - 1, num=n0).astype(np.uint64)
    t0 = time.perf_counter()
    O.walks(g_host.row_ptr, g_host.col, all_starts[ids0.astype(np.int64)], ids=ids0 + np.uint64(first), **kw)
    dt = max(time.perf_counter() - t0, 1e-4)
    ns = int(min(W, max(n0, n0 * seconds / runs / dt)))
    rows = np.linspace(0, W - 1, num=ns).astype(np.uint64)
    st = all_starts[rows.astype(np.int64)]
    vals, secs = [], []
    for _ in range(runs):
        t0 = time.perf_counter()
        paths, lengths, steps, _ = O.walks(g_host.row_ptr, g_host.col, st, ids=rows + np.uint64(first), **kw)
        secs.append(time.perf_counter() - t0)
        vals.append(steps / secs[-1])
    return dict(value=statistics.median(vals), values=vals, steps=steps, seconds=statistics.median(secs), walks=ns,
                rows=rows, paths=paths, lengths=lengths)


def host_graph(g):
    if isinstance(g.row_ptr, np.ndarray):
        return g
    return lt_inputs.Graph(g.n, g.m, g.row_ptr.cpu().numpy().view(np.uint64), g.col.cpu().numpy().view(np.uint32),
                           g.max_deg, g.argmax_deg)


def make_graph(c, device):
    import torch
    if c["scale"] <= 16:
        g = lt_inputs.rmat_cpu(c["scale"], c["tuples"], seed=c.get("graph_seed", 1), permute=c["permute"])
        return lt_inputs.Graph(g.n, g.m, torch.from_numpy(g.row_ptr.view(np.int64)).cuda(device),
                               torch.from_numpy(g.col.view(np.int32)).cuda(device), g.max_deg, g.argmax_deg)
    return lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=c.get("graph_seed", 1), permute=c["permute"],
                              device=device)


def cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count()


def cpu_model():
    """The host CPU's model name (the oracle baseline states its cores and CPU)."""
    try:
        with open("/proc/cpuinfo") as fh:
            for line in fh:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cfg_json(c, g, W, extra):
    d = {"workload": f"{c['name']} (BASELINE.json configs[{c['idx'] - 1}])", "scale": c["scale"],
         "rmat_tuples": c["tuples"], "kronecker": bool(c["permute"]), "vertices": g.n, "csr_entries": g.m,
         "walks_per_gpu": W, "app": c["app"]}
    if c["app"] in ("deepwalk", "pagerank"):
        d["length"] = c["length"]
    if c["app"] == "pagerank":
        d["restart_p"] = c["restart_p"]
    if c["app"] == "ppr":
        d["alpha"] = c["alpha"]
    d.update(extra)
    return d


# ------------------------------------------------------------------------------ reference arm
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    c = workload(args)
    c["idx"] = args.config
    c["seed"] = args.seed
    g = lt_inputs.rmat_cpu(c["scale"], c["tuples"], seed=1, permute=c["permute"]) if c["scale"] <= 22 else None
    if g is None:
        import torch
        torch.cuda.set_device(0)
        g = host_graph(make_graph(c, 0))
    W = num_walks(c, g)
    per = max(1.0, 120.0 / max(1, args.steps + args.warmup))  # whole run within a few minutes
    for _ in range(args.warmup):
        oracle_sample(c, g, W, 0, min(per, 3.0))
    vals, steps_all, secs = [], 0, 0.0
    ns = None
    for _ in range(args.steps):
        r = oracle_sample(c, g, W, 0, per)
        vals.append(r["value"])
        steps_all += r["steps"]
        secs += r["seconds"]
        ns = r["walks"]
    value = steps_all / secs
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "steps/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * secs / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic", "config": cfg_json(c, g, W, {"partitions": None}),
            "cpu_baseline": {"value": value, "unit": "steps/s", "cores": cores(), "cpu_model": cpu_model(), "kind": "oracle",
                             "sample": f"walks 0..{ns - 1} of the workload per step (oracle/ C + OpenMP, {cores()} threads)"},
            "e2e": {"value": value, "unit": "steps/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------------------ CUDA arm
def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return launch_ranks(args)
    if int(os.environ.get("WORLD_SIZE", "1")) != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={os.environ.get('WORLD_SIZE')} processes were "
              f"launched; run one process per GPU", file=sys.stderr)
        return 2
    if args.impl == "reference":
        return run_reference(args)
    import torch
    import torch.distributed as dist

    import paper_conf_icde_xing0wxl23_b200 as LT

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # LT_BENCH_SHARE_DEVICE=1 (tests of the multi-rank launch on a 1-GPU box only): every rank on
    # cuda:0 with gloo for the barrier / max-over-ranks reductions. Never used for reported numbers.
    share = os.environ.get("LT_BENCH_SHARE_DEVICE") == "1" and world > 1
    if share:
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    c = workload(args)
    c["idx"] = args.config
    c["seed"] = args.seed
    P = c["partitions"]
    t0 = time.time()
    g = make_graph(c, local)
    gen_s = time.time() - t0
    W = num_walks(c, g)
    mode = args.mode or ("own" if world > 1 else "replicas")
    own = mode == "own" and world > 1
    if own and args.partitions is None:
        P = c["partitions"] = world  # one contiguous partition per rank: fewest crossings
    first = 0 if own else rank * W
    app, param = app_param(c)
    starts_h = starts_for(c, g, W, first)
    starts_d = torch.from_numpy(starts_h.view(np.int32)).cuda(local)

    ooc = args.graph_pool_gb > 0
    vis = args.visit_counts == 1 or (args.visit_counts == -1 and c["app"] == "pagerank")
    eng = LT.Engine(visit_counts=vis, device=local, chunk_walks=args.chunk_walks, policy=args.policy,
                    insert_mode=args.insert_mode, gather_mode=args.gather_mode,
                    timing=True, layout=args.layout, ilp=args.ilp, path_mode=args.path_mode,
                    graph_pool_bytes=int(args.graph_pool_gb * 2 ** 30), zero_copy=bool(args.zero_copy),
                    rank=rank if own else 0, world=world if own else 1, refill=args.refill,
                    continue_resident=bool(args.continue_resident), direct_start=bool(args.direct_start),
                    l2_persist=args.l2_persist, ooc_prefetch=bool(args.ooc_prefetch),
                    ooc_compress=bool(args.ooc_compress))
    torch.cuda.empty_cache()  # generator scratch back to the device before the library reserves its graph
    t0 = time.time()
    eng.graph_load(g.row_ptr, g.col, P)
    load_s = time.time() - t0
    g_host = None
    want_projection = world == 1 and args.project_gpus > 1 and c["app"] == "deepwalk" and not ooc and P == 1

    def release_col():
        """Once an augmented layout is built the steps never read col: keep a host copy for the oracle legs
        and free the device one (room for the e2e buffers)."""
        nonlocal g, g_host
        if args.release_col and not ooc and eng.stats()["layout"] != LT.LAYOUT_CSR and \
                not isinstance(g.col, np.ndarray) and g.col is not None and not args.sweep and not own:
            if rank == 0 and world == 1 and not args.no_cpu_baseline:
                g_host = host_graph(g)
            g = lt_inputs.Graph(g.n, g.m, g.row_ptr, None, g.max_deg, g.argmax_deg)
            torch.cuda.empty_cache()

    if not want_projection:
        release_col()

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
            torch.cuda.synchronize()

    comm = None
    p2p = own and args.exchange == "p2p"
    if own:
        from paper_conf_icde_xing0wxl23_b200 import dist as ltdist
        comm = ltdist.TorchComm()
    superstep_counters = {}
    attached = []

    def one_step():
        init_walks(eng, c, starts_d, args.seed, first)
        if p2p:
            if not attached:  # receive buffers for every walk, shared once through CUDA IPC; every rank
                ltdist.attach_peers(eng, comm, W)  # writes its path entries into rank 0's matrix (no merge)
                if args.path_mode == 0:
                    ltdist.attach_paths(eng, comm)
                attached.append(True)
            # one owned partition per rank, HBM-resident: the fused superstep (one host round trip each)
            fused = P == world and not ooc
            run = ltdist.run_supersteps_p2p_fused if fused else ltdist.run_supersteps_p2p
            superstep_counters.update(run(eng, comm, f"cuda:{local}"), fused=fused)
        elif own:
            superstep_counters.update(ltdist.run_supersteps(eng, comm, f"cuda:{local}"))
        else:
            eng.run()
        return eng.stats()

    for _ in range(args.warmup):
        one_step()
    # ---- timed region: K steps, device-timed on the library's stream (the legacy default stream)
    clocks = Clocks(local)
    barrier()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record()
    stats = []
    for _ in range(args.steps):
        stats.append(one_step())
    ev1.record()
    barrier()
    ck = clocks.stop()
    ms = ev0.elapsed_time(ev1)
    t = torch.tensor([ms], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    steps_local = sum(s["steps"] for s in stats)
    tot = torch.tensor([steps_local], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(tot)
    value = float(tot.item()) / (ms_max / 1000.0)

    # ---- roofline of the update kernel (algorithmic bytes / CUDA-event launch time)
    upd_ms = sum(s["update_ms"] for s in stats)
    upd_launches = sum(s["update_launches"] for s in stats)
    visits = sum(s["visits"] for s in stats)
    steps_k = steps_local
    finished = sum(s["num_walks"] for s in stats) if not own else len(stats) * W // world
    moves = max(0, visits - finished)  # a walk's final visit ends in termination, every other in a move
    # + one 32-B sector read-modify-write per path entry for the fused visit counts (when on)
    alg_bytes = steps_k * (104 + (32 if vis else 0)) + visits * 16 + moves * 16
    peaks_path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    peak, peak_src = 6650.0, "fallback (B200_PROFILING.md)"
    if os.path.exists(peaks_path):
        peak, peak_src = float(json.load(open(peaks_path))["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs"
    achieved = (alg_bytes / upd_launches) / (upd_ms / upd_launches / 1000.0) / 1e9 if upd_ms > 0 else None
    # DRAM traffic of the update kernel: not measurable inside a timed run (ncu replays the kernel), so it
    # is the static figure of the last `ncu --set full` capture of this configuration, marked as such
    traffic = None
    traffic_source = None
    sector_eff = None
    prof = os.path.join(ROOT, "profiles", "update_kernel_traffic.json")
    if os.path.exists(prof):
        key = f"cfg{args.config}-P{P}-layout{args.layout}-{c['app']}"
        pj = next((e for e in json.load(open(prof))["entries"] if e.get("config_key") == key), {})
        if pj and not own and not ooc:
            traffic = pj.get("dram_bytes_per_launch")
            traffic_source = (f"static: ncu --set full capture {pj.get('source', 'profiles/update_kernel_traffic.json')} "
                              f"of this configuration ({pj.get('captured', 'see file')}), not measured in this run")
            sector_eff = {"ld_bytes_per_sector": pj.get("sector_efficiency_ld_bytes"),
                          "st_bytes_per_sector": pj.get("sector_efficiency_st_bytes"),
                          "source": "static: ncu, profiles/update_kernel_traffic.json"}
    layout = stats[-1]["layout"]
    # DRAM-missing random gathers issued by the update kernel: one per step (ADJ: adj entry;
    # CSR: col entry) + the row_ptr line per step (CSR) or per visit (ADJ)
    aug = layout in (LT.LAYOUT_ADJ, LT.LAYOUT_ADJ12)
    gathers = steps_k * (1 if aug else 2) + (visits if aug else 0)
    gather = None
    gc_path = os.path.join(ROOT, "profiles", "gather_ceiling.json")
    if upd_ms > 0:
        gather = {"gathers_per_s": gathers / (upd_ms / 1000.0), "per_step": gathers / max(1, steps_k)}
        if os.path.exists(gc_path):
            gc = json.load(open(gc_path))
            gather["microbench_per_s"] = gc["microbench_gathers_per_s"]
            gather["vs_microbench"] = gather["gathers_per_s"] / gc["microbench_gathers_per_s"]
            gather["microbench_source"] = ("profiles/gather_ceiling.json (tools/gather_bench at the workload's "
                                           "footprint; a reference rate, not a proven ceiling: it can be exceeded)")
    frac = (achieved / peak) if achieved else None
    if frac is not None and frac > 1.0:  # algorithmic bytes above the copy peak: the timing is broken
        print(f"bench.py: roofline frac {frac:.3f} > 1 (update_ms {upd_ms}, {upd_launches} launches): refusing "
              f"to report it", file=sys.stderr)
        achieved, frac = None, None
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": frac, "traffic": traffic, "traffic_source": traffic_source,
            "kernel": "k_update", "launches": upd_launches, "avg_launch_ms": upd_ms / max(1, upd_launches),
            "alg_bytes_per_step": alg_bytes / max(1, steps_k), "peak_source": peak_src,
            "update_share_of_step": upd_ms / ms, "gather": gather, "sector_efficiency": sector_eff}

    # ---- ownership mode at R GPUs predicted from one-GPU measurements (N=1, DeepWalk, HBM-resident)
    projection = None
    if want_projection:
        R = args.project_gpus
        eng.graph_load(g.row_ptr, g.col, R)  # same engine, R partitions: the R ranks' partitions on one GPU
        sts2 = []
        for i in range(3):
            init_walks(eng, c, starts_d, args.seed, first)
            eng.run()
            if i:
                sts2.append(eng.stats())
        upd = sum(s["update_ms"] for s in sts2) / len(sts2)
        run_ms = sum(s["run_ms"] for s in sts2) / len(sts2)
        sweeps = sts2[-1]["sweeps"]
        launches = sts2[-1]["update_launches"]
        gap = (run_ms - upd) / max(1, launches)  # host + launch time per update launch on one GPU
        allreduce_ms = 0.020  # ASSUMED: one 8-byte NCCL all-reduce over NVSwitch per superstep
        t_r = upd / R + sweeps * (2 * gap + allreduce_ms)
        projection = {
            "gpus": R, "projected_ms_per_step": t_r, "projected_speedup": (ms_max / args.steps) / t_r,
            "projected_steps_per_s": steps_local / args.steps / (t_r / 1e3),
            "inputs": {"update_ms_all_partitions_1gpu": upd, "supersteps": sweeps, "update_launches_1gpu": launches,
                       "gap_ms_per_launch_1gpu": gap, "allreduce_ms_assumed": allreduce_ms,
                       "kernel": "refill auto at P = R", "visits_per_step": sts2[-1]["visits"] / max(1, sts2[-1]["steps"])},
            "model": ("ownership, one partition per rank: every superstep each rank runs one update launch over its "
                      "partition's bucket (the P = R run's update time split evenly over R ranks: edge-balanced "
                      "ranges, stationary load proportional to degree) plus an insert launch and one 8-byte "
                      "all-reduce; supersteps = the P = R run's sweeps. Not a measurement: no multi-GPU box.")}
        eng.graph_load(g.row_ptr, g.col, P)  # back to the headline configuration for the legs below
        release_col()

    # ---- extra partition-count sweep (context; the headline uses P above)
    sweep = {}
    for ps in ([int(x) for x in args.sweep.split(",") if x.strip()] if not own else []):
        with LT.Engine(device=local, chunk_walks=args.chunk_walks, timing=True, layout=args.layout,
                       refill=args.refill) as e2:
            e2.graph_load(g.row_ptr, g.col, ps)
            for _ in range(2):
                init_walks(e2, c, starts_d, args.seed, first)
                e2.run()
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            sts = []
            for _ in range(3):
                init_walks(e2, c, starts_d, args.seed, first)
                e2.run()
                sts.append(e2.stats())
            b.record()
            torch.cuda.synchronize()
            sweep[str(ps)] = {"steps_per_s": sum(s["steps"] for s in sts) / (a.elapsed_time(b) / 1000),
                              "visits_per_step": sum(s["visits"] for s in sts) / max(1, sum(s["steps"] for s in sts)),
                              "sweeps": sts[-1]["sweeps"], "update_launches": sts[-1]["update_launches"]}

    # ---- e2e through the C ABI with host buffers (pinned), H2D + D2H inside the timed region
    # ---- out-of-core: host-link traffic of the timed steps against the measured pinned H2D bandwidth
    host_link = None
    if ooc:
        gb = sum(s["graph_h2d_bytes"] for s in stats)
        hb = torch.empty(1 << 30, dtype=torch.uint8, pin_memory=True)
        db = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
        for _ in range(2):
            db.copy_(hb, non_blocking=True)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(5):
            db.copy_(hb, non_blocking=True)
        b.record()
        torch.cuda.synchronize()
        h2d_peak = 5 * (1 << 30) / (a.elapsed_time(b) / 1000) / 1e9
        del hb, db
        last = stats[-1]
        host_link = {"achieved_gbs": gb / (ms / 1000) / 1e9, "peak_gbs": h2d_peak,
                     "peak_source": "pinned 1 GiB H2D copy, measured in this run",
                     "frac": gb / (ms / 1000) / 1e9 / h2d_peak, "graph_h2d_bytes_per_step": gb / len(stats),
                     "pool_blocks": last["pool_blocks"], "pool_block_bytes": last["pool_block_bytes"],
                     "iterations": last["iterations"], "explicit_copies": last["explicit_copies"],
                     "pool_hits": last["pool_hits"], "zero_copy_launches": last["zero_copy_launches"],
                     "preemptive_launches": last["preemptive_launches"], "prefetches": last["prefetches"],
                     "hit_rate": last["pool_hits"] / max(1, last["iterations"]),
                     "continue_resident": bool(args.continue_resident),
                     "visits_per_step": last["visits"] / max(1, last["steps"]),
                     # compressed partition transfers: raw CSR bytes delivered per byte over the link
                     "ooc_compress": bool(args.ooc_compress),
                     "graph_h2d_raw_bytes_per_step": sum(s["graph_h2d_raw_bytes"] for s in stats) / len(stats),
                     "compression_ratio": (sum(s["graph_h2d_raw_bytes"] for s in stats) / gb) if gb else None,
                     "ooc_compressed_host_bytes": last["ooc_compressed_bytes"]}

    e2e = None
    if not args.no_e2e and args.e2e_steps > 0 and not own and vis:
        # the visit-frequency workload's result is the count vector: per step, pinned starts H2D
        # (lt_walks_init_pagerank / _ex from host memory), the walk, and the u64[n] counts D2H
        h_starts = torch.from_numpy(starts_h.view(np.int32)).pin_memory()
        h_counts = torch.empty(g.n, dtype=torch.int64, pin_memory=True)
        init_walks(eng, c, h_starts, args.seed, first)  # untimed warm-up (first-touch of the buffers)
        eng.run()
        eng.visit_counts(h_counts)
        barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        e_steps = 0
        for _ in range(args.e2e_steps):
            init_walks(eng, c, h_starts, args.seed, first)
            eng.run()
            eng.visit_counts(h_counts)
            e_steps += eng.stats()["steps"]
        b.record()
        barrier()
        e2e = {"value": e_steps / (a.elapsed_time(b) / 1000), "unit": "steps/s", "h2d_bytes_per_step": W * 4,
               "d2h_bytes_per_step": g.n * 8, "pinned": True, "steps": args.e2e_steps,
               "api": "lt_walks_init* (host starts) + lt_run + lt_get_visit_counts (host)"}
    elif not args.no_e2e and args.e2e_steps > 0 and not own and c["app"] == "ppr":
        # PPR rows are mostly padding (E[length] = 1/alpha of L_max + 1 slots): the ragged layout
        # (offsets + packed vertices, lt_run_to_host_compact) is the result copied out
        h_starts = torch.from_numpy(starts_h.view(np.int32)).pin_memory()
        h_off = torch.empty(W + 1, dtype=torch.int64, pin_memory=True)
        h_vert = torch.empty(W * 128, dtype=torch.int32, pin_memory=True)
        eng.run_to_host_compact(h_starts, app, param, args.seed, first, offsets=h_off, vertices=h_vert,
                                chunks=args.e2e_chunks)  # untimed warm-up (scratch reservation, first touch)
        barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        e_steps = 0
        for _ in range(args.e2e_steps):
            eng.run_to_host_compact(h_starts, app, param, args.seed, first, offsets=h_off, vertices=h_vert,
                                    chunks=args.e2e_chunks)
            e_steps += eng.stats()["steps"]
        b.record()
        barrier()
        tot = int(h_off[W].item())
        e2e = {"value": e_steps / (a.elapsed_time(b) / 1000), "unit": "steps/s", "h2d_bytes_per_step": W * 4,
               "d2h_bytes_per_step": (W + 1) * 8 + tot * 4, "pinned": True, "steps": args.e2e_steps,
               "api": f"lt_run_to_host_compact (offsets + packed vertices), {args.e2e_chunks} overlapped ranges"}
        del h_vert
    elif not args.no_e2e and args.e2e_steps > 0 and not own:
        S = int(c["length"]) + 1 if c["app"] == "deepwalk" else 128
        try:
            h_paths = torch.empty((W, S), dtype=torch.int32, pin_memory=True)
            h_len = torch.empty(W, dtype=torch.int32, pin_memory=True)
            h_starts = torch.from_numpy(starts_h.view(np.int32)).pin_memory()
            pinned = True
        except Exception:
            h_paths = np.empty((W, S), dtype=np.uint32)
            h_len = np.empty(W, dtype=np.uint32)
            h_starts = starts_h
            pinned = False
        eng.run_to_host(h_starts, app, param, args.seed, first, paths=h_paths, lengths=h_len,
                        chunks=args.e2e_chunks)  # untimed warm-up (double buffers, first touch)
        barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        e_steps = 0
        for _ in range(args.e2e_steps):
            # lt_run_to_host: H2D of the starts, walks, and the D2H of every path and length, with the
            # copy-out of walk range c overlapped with the walking of range c+1
            eng.run_to_host(h_starts, app, param, args.seed, first, paths=h_paths, lengths=h_len,
                            chunks=args.e2e_chunks)
            e_steps += eng.stats()["steps"]
        b.record()
        barrier()
        ems = a.elapsed_time(b)
        et = torch.tensor([ems], dtype=torch.float64, device="cuda")
        es = torch.tensor([e_steps], dtype=torch.float64, device="cuda")
        if world > 1:
            dist.all_reduce(et, op=dist.ReduceOp.MAX)
            dist.all_reduce(es)
        # the link the e2e copy-out rides on: pinned 1 GiB D2H, measured now
        hb = torch.empty(1 << 30, dtype=torch.uint8, pin_memory=True)
        db = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
        hb.copy_(db, non_blocking=True)
        a2, b2 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a2.record()
        for _ in range(4):
            hb.copy_(db, non_blocking=True)
        b2.record()
        torch.cuda.synchronize()
        d2h_gbs = 4 * (1 << 30) / (a2.elapsed_time(b2) / 1000) / 1e9
        del hb, db
        e2e = {"value": float(es.item()) / (float(et.item()) / 1000), "unit": "steps/s",
               "d2h_link_gbs": d2h_gbs,
               "d2h_bound_steps_per_s": float(es.item()) / args.e2e_steps / ((W * S * 4 + W * 4) / (d2h_gbs * 1e9)),
               "h2d_bytes_per_step": W * 4, "d2h_bytes_per_step": W * S * 4 + W * 4, "pinned": pinned,
               "steps": args.e2e_steps, "api": f"lt_run_to_host, {args.e2e_chunks} overlapped ranges"}
        del h_paths, h_len

    # ---- CPU oracle baseline on a bounded sample (rank 0, N=1) + sampled parity of that sample
    cpu = None
    parity = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        init_walks(eng, c, starts_d, args.seed, first)
        eng.run()
        gh = g_host if g_host is not None else host_graph(g)
        r = oracle_sample(c, gh, W, first, args.cpu_seconds, runs=5)
        cpu = {"value": r["value"], "unit": "steps/s", "cores": cores(), "cpu_model": cpu_model(), "kind": "oracle",
               "runs": 5, "stat": "median", "spread": [min(r["values"]), max(r["values"])],
               "sample": f"{r['walks']} walks spread evenly over the workload's {W} ({r['steps']} steps, "
                         f"median {r['seconds']:.2f} s per run; oracle/ C + OpenMP, {cores()} threads)"}
        r1 = oracle_sample(c, gh, W, first, min(3.0, args.cpu_seconds / 4), threads=1)  # per-core context
        cpu["single_thread"] = {"value": r1["value"], "cores": 1, "sample": f"{r1['walks']} walks spread evenly"}
        # sampled parity: every walk of the timed sample (the oracle's paths) against the GPU's rows
        gp, gl = eng.get_paths_rows(r["rows"])
        mism = int(np.sum(np.any(gp != r["paths"], axis=1) | (gl != r["lengths"])))
        parity = {"sampled_walks": int(len(r["rows"])), "mismatched_walks": mism, "vs": "oracle (bit-exact)"}
        if vis:  # the counts are a global sum: check their total and one sampled property exactly
            import oracle as O
            cnt = eng.visit_counts().astype(np.int64)
            parity["visit_counts_total"] = int(cnt.sum())
            parity["visit_counts_total_ok"] = bool(cnt.sum() == eng.stats()["steps"] + W)
            parity["visit_counts_of_sample_le_gpu"] = bool(np.all(
                O.visit_counts(r["paths"], r["lengths"], g.n).astype(np.int64) <= cnt))

    # ---- N>1 ownership: the communication-free bound (every rank the whole graph and 1/N of the walks)
    replicas_bound = None
    breakdown = None
    if own:
        upd = torch.tensor([sum(s["update_ms"] for s in stats) / len(stats)], dtype=torch.float64, device="cuda")
        dist.all_reduce(upd, op=dist.ReduceOp.MAX)
        breakdown = {"supersteps": superstep_counters.get("supersteps"),
                     "records_sent_rank0": superstep_counters.get("records_sent"),
                     "update_ms_per_step_max_rank": float(upd.item()),
                     "exchange_sync_ms_per_step": ms_max / args.steps - float(upd.item()),
                     "exchange": args.exchange, "fused": superstep_counters.get("fused")}
    if own and not args.no_replicas_bound:
        eng.close()
        torch.cuda.empty_cache()
        a0, a1 = rank * W // world, (rank + 1) * W // world
        with LT.Engine(device=local, timing=True, layout=args.layout, chunk_walks=args.chunk_walks,
                       visit_counts=vis) as er:
            er.graph_load(g.row_ptr, g.col, 1)
            st_r = torch.from_numpy(starts_h[a0:a1].view(np.int32)).cuda(local)

            def one_r():
                init_walks(er, c, st_r, args.seed, a0)
                er.run()
                return er.stats()["steps"]

            one_r()
            barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            rs = sum(one_r() for _ in range(args.steps))
            e1.record()
            barrier()
            rt = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device="cuda")
            rsum = torch.tensor([rs], dtype=torch.float64, device="cuda")
            dist.all_reduce(rt, op=dist.ReduceOp.MAX)
            dist.all_reduce(rsum)
            replicas_bound = {"value": float(rsum.item()) / (float(rt.item()) / 1e3), "unit": "steps/s",
                              "ms_per_step": float(rt.item()) / args.steps, "walks_per_rank": a1 - a0,
                              "what": "upper bound of the ownership mode: every rank holds the whole graph and "
                                      "walks 1/N of the workload's walks, no exchange"}

    last = stats[-1]
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "steps/s", "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
                "scaling": "strong" if own else "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
                "config": cfg_json(c, g, W, {"partitions": P, "chunk_walks": args.chunk_walks,
                                             "policy": "selective" if args.policy == 0 else "round_robin",
                                             "insert_mode": "warp_aggregated" if args.insert_mode == 0 else "direct",
                                             "parallelism": (f"own{world}" if own else f"replicas{world}") if world > 1 else "single",
                                             "mode": "out_of_core" if ooc else "hbm_resident",
                                             "graph_pool_gb": args.graph_pool_gb if ooc else None,
                                             "l2": "inputs larger than L2 (CSR >> 126 MB); no flush",
                                             "layout": {LT.LAYOUT_ADJ: "adj", LT.LAYOUT_ADJ12: "adj12"}.get(layout, "csr"),
                                             "graph_gen_s": round(gen_s, 2), "graph_load_s": round(load_s, 2),
                                             "graph_prep_ms": stats[-1]["graph_prep_ms"]}),
                "clocks": ck, "gpu_launches": int(sum(s["kernel_launches"] for s in stats)),
                "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "parity_sample": parity,
                "per_step": {"steps": last["steps"], "visits": last["visits"], "sweeps": last["sweeps"],
                             "update_launches": last["update_launches"], "run_ms": last["run_ms"],
                             "init_ms": last["init_ms"], "update_ms": last["update_ms"],
                             "direct_start": bool(last["direct_start"]),
                             "chunks_total": last["chunks_total"], "chunks_free_min": last["chunks_free_min"]}}
        if share:
            line["config"]["shared_device_test"] = "all ranks on cuda:0 over gloo: launch test, not a measurement"
        if host_link:
            line["host_link"] = host_link
        if own:
            line["ownership"] = dict(superstep_counters, exchange=args.exchange)
            line["superstep_breakdown"] = breakdown
            if replicas_bound:
                line["replicas_upper_bound"] = replicas_bound
        if projection:
            line["projection_8gpu" if projection["gpus"] == 8 else f"projection_{projection['gpus']}gpu"] = projection
        if sweep:
            line["partition_sweep"] = sweep
        print(json.dumps(line), flush=True)
    eng.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
