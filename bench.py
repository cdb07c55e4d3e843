#!/usr/bin/env python
"""bench.py — batched HB+-tree lookups on B200 (one JSON line on rank 0).

Default workload = BASELINE.json configs[3] (c4), the north_star's sharded
config and the largest one that fits one B200: an implicit tree of 2^31
stratified uint64 keys (fanout 16, 36 GiB of tree) and 2^28 uniform hit
queries in total.  At N = 1 the whole tree sits on one GPU; at N > 1 it is
key-range sharded over the N ranks (2^31/N keys and 2^28/N queries per rank,
every query routed to its owner shard and its result returned),
so the total work is fixed: "scaling": "strong".  A "step" is one search of the
whole batch (every hot-path row: routing, bucketing, the bucket-local directory /
node search through every level, the leaf search, the result write and, at
N > 1, the exchange both ways).  Inputs are seeded synthetic (gen/, SURVEY
§8(d)) generated on the device; queries + results per step exceed the 126 MB
L2, so no L2 flush is done between steps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c1|c2|c3|c4|c5]
  python bench.py --impl reference ...   # the CPU oracle arm (rank 0 only)

--gpus N without a torchrun environment re-launches itself under
torch.distributed.run with N local ranks (127.0.0.1).  When there are more ranks
than visible GPUs (a dry run of the multi-rank path on one GPU) the ranks share
the devices round-robin, the process group is gloo and the sharded tree uses the
host-callback communicator with the fused peer-memory exchange.
c1/c2/c3 at N > 1 run one replica per rank, each searching its own batch (weak
scaling); c5 ("query-batch split at 8 GPUs") splits its 2^26-query batch over the
replicas (strong scaling); no collective on the data path.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
from tools import roofline  # noqa: E402

NVLINK_GBS = 770.0  # measured peer copy per direction (B200_PROFILING.md), for c4's a2a term


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=400)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="hbt", choices=["hbt", "reference"])
    ap.add_argument("--config", default="c4", choices=["c1", "c2", "c3", "c4", "c5"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--smem-mode", type=int, default=None, help="implicit directory: 2 = staged (default), 3 = in place")
    ap.add_argument("--l2-levels", type=int, default=None, help="L2 budget for index+sector levels (bytes)")
    ap.add_argument("--exchange", type=int, default=None, help="c4: 0 = fused peer-memory exchange, 1 = NCCL")
    ap.add_argument("--bucket", type=int, default=None, help="query bucketing: 0 = off, 1 = on, 2 = auto (default)")
    ap.add_argument("--bucket-slice", type=int, default=None, help="tree bytes per query bucket")
    ap.add_argument("--bucket-items", type=int, default=None, help="bucket-local shared-memory directory: 0 | 1")
    ap.add_argument("--leaf256", type=int, default=None, help="leaf / key lines by 256-bit lane loads: 0 | 1")
    ap.add_argument("--full-levels", type=int, default=None, help="implicit: bit mask of levels read whole")
    ap.add_argument("--origin-rank0", action="store_true",
                    help="replicated configs: all queries start on rank 0 (NCCL scatter / gather in the step)")
    ap.add_argument("--leaf-host", action="store_true",
                    help="implicit trees: L-segment in pinned host memory (the paper's split, SURVEY f4)")
    ap.add_argument("--graph", default="auto", choices=["0", "1", "auto"],
                    help="replay the step from a CUDA graph (auto: batches <= 2^20 queries, launch-bound)")
    ap.add_argument("--param", action="append", default=[], metavar="NAME=VALUE",
                    help="any hbt_set_param knob (repeatable), e.g. ctas_per_sm=1")
    ap.add_argument("--queries", default=None, choices=["normal", "gamma", "zipf_clustered", "uniform_values"],
                    help="replace the config's queries by the paper's skewed VALUE distributions (P:346-352)")
    ap.add_argument("--update-frac", type=float, default=0.0,
                    help="after timing, apply a bulk update of this fraction of n (half fresh UPSERTs, half "
                         "DELETEs; c3 does 1%% by default) and time search again")
    ap.add_argument("--range-k", type=int, default=0,
                    help="time range scans returning k keys per query (PAPER.md:392) instead of point lookups")
    a = ap.parse_args()
    if a.origin_rank0 and a.config == "c4":
        ap.error("--origin-rank0 is for replicated trees; c4 routes queries by key range")
    return a


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def maybe_spawn(args):
    """--gpus N outside torchrun: re-launch this script under torch.distributed.run
    with N local ranks (rendezvous on 127.0.0.1) and return its exit code."""
    if args.gpus <= 1 or "WORLD_SIZE" in os.environ or args.impl == "reference":
        return None
    import socket
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


class Dist:
    """The process group of a run: NCCL with one rank per GPU; gloo (CPU tensors)
    when more ranks than visible GPUs share the devices (multi-rank dry run)."""

    def __init__(self, rank, world, local):
        import torch
        import torch.distributed as dist
        self.rank, self.world = rank, world
        ndev = max(torch.cuda.device_count(), 1)
        self.device = local % ndev
        self.shared_gpus = world > ndev
        self.backend = None
        torch.cuda.set_device(self.device)
        if world > 1:
            self.backend = "gloo" if self.shared_gpus else "nccl"
            if self.backend == "nccl":
                dist.init_process_group("nccl", device_id=torch.device("cuda", self.device))
            else:
                dist.init_process_group("gloo")

    def barrier(self):
        import torch.distributed as dist
        if self.world > 1:
            dist.barrier()

    def max(self, x: float) -> float:
        """max over ranks (device tensor under NCCL, CPU tensor under gloo)."""
        import torch
        import torch.distributed as dist
        if self.world == 1:
            return float(x)
        t = torch.tensor([x], dtype=torch.float64, device="cuda" if self.backend == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def close(self):
        import torch.distributed as dist
        if self.world > 1:
            dist.destroy_process_group()


def probe_a2a_gbs(d: "Dist", nbytes=256 << 20):
    """In-run NVLink probe (SURVEY §8(d) BW_NVL): NCCL all_to_all_single of `nbytes`
    per rank, best of 3; returns the bytes each GPU sends to its peers per second
    ((N-1)/N of the buffer) in GB/s, or None (one rank, or ranks sharing a GPU)."""
    import torch
    import torch.distributed as dist
    if d.world == 1 or d.backend != "nccl":
        return None
    a = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    b = torch.empty_like(a)
    best = 0.0
    for _ in range(4):
        d.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        dist.all_to_all_single(b, a)
        e1.record()
        torch.cuda.synchronize()
        t = d.max(e0.elapsed_time(e1) * 1e-3)
        best = max(best, nbytes * (d.world - 1) / d.world / t / 1e9)
    del a, b
    return best


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d.get("hbm_gbs", 6650.0), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.gpu = gpu_index
        self.proc = None
        self.path = f"/tmp/hbt_clocks_{os.getpid()}.csv"

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
            time.sleep(0.3)
        except Exception:
            self.proc = None

    def stop(self):
        if not self.proc:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        rows = []
        for line in open(self.path):
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 9:
                rows.append(parts)
        if not rows:
            return None
        sm = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def measure_h2d_gbs():
    """Pinned host -> device copy bandwidth (1 GiB, best of 3, CUDA events)."""
    import torch
    h = torch.empty(1 << 30, dtype=torch.uint8).pin_memory()
    d = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
    best = 0.0
    for _ in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        d.copy_(h, non_blocking=True)
        b.record()
        torch.cuda.synchronize()
        best = max(best, (1 << 30) / (a.elapsed_time(b) * 1e-3) / 1e9)
    del h, d
    return best


def probe_line_rate(nbytes=8 << 30):
    """G random 64 B lines/s from a DRAM-resident buffer (tools/probe.cu probe_gather64)."""
    try:
        import ctypes as C
        L = C.CDLL(os.path.join(ROOT, "tools", "libhbtprobe.so"))
        L.probe_gather64.restype = C.c_double
        L.probe_gather64.argtypes = [C.c_uint64, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int]
        v = L.probe_gather64(nbytes, 0, 2, 1024, 1, 3)
        return v if v > 0 else None
    except OSError:
        return None


def probe_l2_gbs(chunk, nbytes=32 << 20):
    """All-SM random reads of `chunk`-byte aligned chunks over an `nbytes` buffer
    (32 MB: L2-resident; 1 GB: every read misses, i.e. the random-DRAM rate)."""
    import ctypes as C
    try:
        L = C.CDLL(os.path.join(ROOT, "tools", "libhbtprobe.so"))
        L.probe_random_read_gbs.restype = C.c_double
        L.probe_random_read_gbs.argtypes = [C.c_uint64, C.c_int, C.c_int]
        v = L.probe_random_read_gbs(nbytes, chunk, 3)
        return v if v > 0 else None
    except OSError:
        return None


# --------------------------------------------------------------------------- workloads


class Work:
    """One rank's share of a configuration, ready to time."""

    def __init__(self, **kw):
        self.__dict__.update(kw)


def make_work(cfg_name, d, args):
    import torch

    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    from gen.device import GenLib

    rank, world = d.rank, d.world
    g = GenLib()
    c = gen.CONFIGS[cfg_name]
    n, m, w, F = c["n"], c["m"], c["width"], c["fanout"]
    sk = gen.stream_seed(c["cfg"], gen.STREAM_K)
    sv = gen.stream_seed(c["cfg"], gen.STREAM_V)
    sq = gen.stream_seed(c["cfg"], gen.STREAM_Q)
    sdt = torch.int32 if w == 4 else torch.int64
    extra = {}
    hit_rate = 1.0
    if cfg_name == "c4":
        lo, hi = hbt.shard_plan(n, world, rank)
        keys = g.stratified_keys(hi - lo, sk, start=lo)
        vals = g.mix_stream(hi - lo, w, sv, start=lo)
        m_local = m // world
        q = g.stratified_queries(m_local, n, sq, sk, start=rank * m_local)
        if world == 1:
            comm = hbt.Comm.single()  # no NCCL at one rank
        elif d.backend == "nccl":
            comm = hbt.Comm.from_torch()
        else:  # ranks sharing a GPU: NCCL refuses them; host all-gathers over gloo + IPC windows
            comm = hbt.Comm.from_torch_host()
        tree = hbt.ShardedTree(comm, keys, vals, fanout=F)
        if d.backend == "gloo":
            tree.set_param("exchange", 0)
        qdesc = f"uniform hits over all {n} keys, {m_local} per rank, routed to their owner shard"
        extra["comm"] = comm
        m = m_local
    else:
        keys = g.mix_stream(n, w, sk)
        vals = g.mix_stream(n, w, sv)
        if c["queries"] == "uniform":
            q = g.uniform_queries(m, n, w, sq, sk, start=rank * m)
            qdesc = "uniform hits with replacement"
        elif c["queries"] == "uniform_ins":
            bk, bv, bo, n_ins = gen.update_batch(cfg_name, n)
            q = g.uniform_queries(m, n + n_ins, w, sq, sk, start=rank * m)
            hit_rate = n / (n + n_ins)
            qdesc = f"uniform over key indices [0, n + {n_ins}) (misses = not-yet-inserted keys)"
            extra["batch"] = (torch.from_numpy(bk.view(np.int64)).cuda(), torch.from_numpy(bv.view(np.int64)).cuda(),
                              torch.from_numpy(bo).cuda())
        elif c["queries"] == "shuffle":
            hk = gen.keys(n, w, sk)
            q = torch.from_numpy(gen.workload_queries(cfg_name, hk).view(np.int32 if w == 4 else np.int64)).cuda()
            qdesc = "Knuth shuffle of the keys (PAPER.md:298)"
        elif c["queries"] == "zipf":
            # c5 = BASELINE configs[4], "query-batch split at 8 GPUs": the 2^26-query batch is
            # split over the ranks (2^23 each at 8; strong scaling), every rank holding a replica
            m = m // world
            hk = gen.keys(n, w, sk)
            r = gen.zipf_ranks(m, n, c["theta"], sq, start=rank * m)
            q = torch.from_numpy(hk[r - 1].view(np.int64)).cuda()
            qdesc = f"Zipf({c['theta']}) over key ranks, scrambled through the key order"
        else:
            raise SystemExit(cfg_name)
        tree = hbt.Tree(keys, vals, fanout=F, layout=c["layout"])
    if args.update_frac and "batch" not in extra and cfg_name != "c4":
        bk, bv, bo, _ = gen.update_batch(cfg_name, n, int(args.update_frac * n))
        dt = np.int32 if w == 4 else np.int64
        extra["batch"] = (torch.from_numpy(bk.view(dt)).cuda(), torch.from_numpy(bv.view(dt)).cuda(),
                          torch.from_numpy(bo).cuda())
    if args.queries:  # the paper's skew experiment: values on [0, 1] mapped to [0, MAX] (mostly misses)
        kind = {"normal": "normal", "gamma": "gamma", "zipf_clustered": "zipf", "uniform_values": "uniform"}[args.queries]
        hv = gen.skew_values(kind, m, w, sq ^ 0x5EED, start=rank * m)
        q = torch.from_numpy(hv.view(np.int32 if w == 4 else np.int64)).cuda()
        hit_rate = 0.0
        qdesc = f"{args.queries} query values on [0, 1] mapped to [0, MAX] (PAPER.md:346-352)"
    del keys, vals
    if args.smem_mode is not None:
        tree.set_param("smem_mode", args.smem_mode)
    if args.l2_levels is not None and c["layout"] == "implicit":
        tree.set_param("l2_levels_bytes", args.l2_levels)
    if args.exchange is not None:
        tree.set_param("exchange", args.exchange)
    if args.bucket is not None:
        tree.set_param("bucket", args.bucket)
    if args.bucket_slice is not None:
        tree.set_param("bucket_slice", args.bucket_slice)
    if args.bucket_items is not None:
        tree.set_param("bucket_items", args.bucket_items)
    if args.leaf256 is not None:
        tree.set_param("leaf256", args.leaf256)
    if args.full_levels is not None:
        tree.set_param("full_levels", args.full_levels)
    if args.leaf_host:
        tree.set_leaf_placement("host")  # f4: L-segment in pinned host memory
        qdesc += "; L-segment in pinned host memory, leaf lines read by zero-copy loads over the host link"
    params = {}
    for kv in args.param:
        name, val = kv.split("=", 1)
        params[name] = int(val, 0)
    # the host pipeline of the e2e number: c4's 2^28-query batch in 4 Mi-query chunks, each
    # chunk's search bucketed, copies both ways overlapping the searches (D2H-bound:
    # 1.99 -> 3.27 G q/s against H2D + search + D2H in sequence, profiles/r02_c4_e2e_sweep.jsonl)
    params.setdefault("host_chunk_log2", 22 if cfg_name == "c4" else 20)
    params.setdefault("host_bufs", 2)
    for name, val in params.items():
        tree.set_param(name, val)
    out_pos = torch.empty(m, dtype=torch.int64, device="cuda")
    out_val = torch.empty(m, dtype=sdt, device="cuda")
    hi = None
    if args.range_k:
        hi = torch.full_like(q, -1)  # MAX: every range returns k keys unless the tree ends
        qdesc += f"; range scans of {args.range_k} keys from each query key"
    origin = None
    if args.origin_rank0:
        # the batch of every rank starts on rank 0 (gathered there once, untimed); each
        # step scatters it, searches and gathers the results back to rank 0
        import torch.distributed as dist
        if world > 1:
            full = torch.empty(world * m, dtype=q.dtype, device="cuda") if rank == 0 else None
            dist.gather(q, list(full.chunk(world)) if rank == 0 else None, dst=0)
        else:
            full = q.clone()
        origin = {"full": full, "recv": torch.empty_like(q),
                  "gpos": torch.empty(world * m, dtype=torch.int64, device="cuda") if rank == 0 else None,
                  "gval": torch.empty(world * m, dtype=sdt, device="cuda") if rank == 0 else None}
        qdesc += "; the queries of all ranks originate on rank 0 (scatter + gather inside each step)"
    return Work(c=c, name=cfg_name, tree=tree, q=q, m=m, w=w, hit_rate=hit_rate, qdesc=qdesc, extra=extra,
                host_chunk_log2=params["host_chunk_log2"], host_bufs=params["host_bufs"],
                out_pos=out_pos, out_val=out_val, info=tree.info(), range_k=args.range_k, hi=hi,
                origin=origin, rank=rank, world=world, dist=d)


def step(work):
    """One step: the whole batch through the hot path."""
    o = getattr(work, "origin", None)
    if o is not None:  # queries originate on rank 0: scatter, search, gather
        import torch.distributed as dist
        if work.world > 1:
            dist.scatter(o["recv"], list(o["full"].chunk(work.world)) if work.rank == 0 else None, src=0)
            work.tree.search(o["recv"], work.out_pos, work.out_val)
            dist.gather(work.out_pos, list(o["gpos"].chunk(work.world)) if work.rank == 0 else None, dst=0)
            dist.gather(work.out_val, list(o["gval"].chunk(work.world)) if work.rank == 0 else None, dst=0)
        else:
            o["recv"].copy_(o["full"])
            work.tree.search(o["recv"], work.out_pos, work.out_val)
            o["gpos"].copy_(work.out_pos)
            o["gval"].copy_(work.out_val)
        return
    if work.range_k:
        work.tree.range(work.q, work.hi, work.range_k)
    else:
        work.tree.search(work.q, work.out_pos, work.out_val)


def warm_update_path(work):
    """Run one small bulk update on a scratch tree of the same form and width so the
    timed update does not pay first-launch module loading."""
    import torch

    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    dt = torch.int32 if work.w == 4 else torch.int64
    k = torch.arange(1, 200001, dtype=dt, device="cuda") * 7
    t = hbt.Tree(k, k, fanout=work.c["fanout"], layout=work.c["layout"])
    bk = torch.arange(0, 20000, dtype=dt, device="cuda") * 13
    ops = (torch.arange(20000, device="cuda") % 2).to(torch.uint8)
    t.update(bk, bk, ops)
    torch.cuda.synchronize()
    t.close()


def capture_step(work):
    """The step captured once in a CUDA graph (small batches are host-launch bound:
    the Python binding + ctypes + launch cost ~10 us, the c1 kernel ~5 us)."""
    import torch
    gs = torch.cuda.Stream()
    gs.wait_stream(torch.cuda.current_stream())
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.stream(gs):
        step(work)
        torch.cuda.synchronize()
        with torch.cuda.graph(graph, stream=gs):
            step(work)
    torch.cuda.synchronize()
    return graph


def step_fits_l2(work):
    """True when the tree plus one step's queries and results fit in the L2 (c1)."""
    import torch
    info = work.info
    data = info["inner_bytes"] + info["leaf_bytes"] + work.m * (2 * work.w + 8)
    return data < torch.cuda.get_device_properties(torch.cuda.current_device()).L2_cache_size


def time_search_flushed(work, steps, graph=None):
    """Small working sets (the tree and the batch fit in the L2): flush the L2 between
    timed steps by writing a 2x-L2 buffer, and sum per-step CUDA-event intervals (the
    flush itself is outside every interval).  Max over ranks."""
    import torch
    d = work.dist
    stream = torch.cuda.current_stream()
    l2 = torch.cuda.get_device_properties(torch.cuda.current_device()).L2_cache_size
    flush = torch.empty(2 * l2 // 4, dtype=torch.int32, device="cuda")
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    d.barrier()
    torch.cuda.synchronize()
    for a, b in evs:
        flush.fill_(1)
        a.record(stream)
        if graph is not None:
            graph.replay()
        else:
            step(work)
        b.record(stream)
    torch.cuda.synchronize()
    d.barrier()
    return d.max(sum(a.elapsed_time(b) for a, b in evs)) / steps


def time_search(work, steps, graph=None):
    """K launches of the step, CUDA events on the launching stream, max over ranks."""
    import torch
    if step_fits_l2(work):
        return time_search_flushed(work, steps, graph)
    d = work.dist
    stream = torch.cuda.current_stream()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    d.barrier()
    torch.cuda.synchronize()
    ev0.record(stream)
    if graph is not None:
        for _ in range(steps):
            graph.replay()
    else:
        for _ in range(steps):
            step(work)
    ev1.record(stream)
    torch.cuda.synchronize()
    d.barrier()
    return d.max(ev0.elapsed_time(ev1)) / steps


def time_e2e(work, steps):
    """Same metric through the public API with pinned HOST buffers (H2D + D2H inside)."""
    import torch
    d = work.dist
    m, w = work.m, work.w
    hq = work.q.cpu().pin_memory()
    hp = torch.empty(m, dtype=torch.int64).pin_memory()
    hv = torch.empty(m, dtype=work.q.dtype).pin_memory()
    # a multi-rank sharded search is a collective over every rank's whole batch; one
    # shard (N = 1) is an ordinary tree for the host pipeline (global pos = local rank)
    sharded = work.name == "c4" and d.world > 1

    # sharded (N > 1): the batch in chunks, every chunk one collective hbt_search_sharded on
    # the current stream; chunk c+1's H2D (copy stream) and chunk c-1's D2H (copy stream)
    # overlap chunk c's search, as hbt_search_host does for one tree
    nchunk = max(1, min(8, m >> 22)) if sharded else 1
    bounds = [m * c // nchunk for c in range(nchunk + 1)]
    if sharded:
        dqs = torch.empty_like(work.q)
        dps = torch.empty(m, dtype=torch.int64, device="cuda")
        dvs = torch.empty(m, dtype=work.q.dtype, device="cuda")
        s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()

    def one():
        if sharded:
            main = torch.cuda.current_stream()
            ev_in = [torch.cuda.Event() for _ in range(nchunk)]
            ev_srch = [torch.cuda.Event() for _ in range(nchunk)]
            with torch.cuda.stream(s_in):
                for c in range(nchunk):
                    a, b = bounds[c], bounds[c + 1]
                    dqs[a:b].copy_(hq[a:b], non_blocking=True)
                    ev_in[c].record(s_in)
            for c in range(nchunk):
                a, b = bounds[c], bounds[c + 1]
                main.wait_event(ev_in[c])
                work.tree.search(dqs[a:b], dps[a:b], dvs[a:b])
                ev_srch[c].record(main)
                with torch.cuda.stream(s_out):
                    s_out.wait_event(ev_srch[c])
                    hp[a:b].copy_(dps[a:b], non_blocking=True)
                    hv[a:b].copy_(dvs[a:b], non_blocking=True)
            torch.cuda.synchronize()
        else:
            work.tree.search_host(hq, hp, hv)

    one()
    d.barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(steps):
        one()
    el = d.max(time.perf_counter() - t0)
    qps = d.world * m * steps / el
    check = None
    if sharded:  # the chunked collective searches return what one whole-batch search returns
        p_all, v_all = work.tree.search(work.q)
        torch.cuda.synchronize()
        same = torch.equal(p_all.cpu(), hp) and torch.equal(v_all.cpu(), hv)
        check = "equal to one whole-batch search" if same else "MISMATCH against one whole-batch search"
        if not same:
            print(f"[rank {d.rank}] e2e: chunked sharded search differs from the whole-batch search", file=sys.stderr)
    # the host link alone: the step's H2D and D2H bytes copied concurrently on two streams
    # (no search) -- the ceiling the end-to-end number runs against
    link = None
    try:
        dq = torch.empty_like(work.q)
        sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
        best = 1e30
        for _ in range(3):
            torch.cuda.synchronize()
            t1 = time.perf_counter()
            with torch.cuda.stream(sa):
                dq.copy_(hq, non_blocking=True)
            with torch.cuda.stream(sb):
                hp.copy_(work.out_pos, non_blocking=True)
                hv.copy_(work.out_val, non_blocking=True)
            torch.cuda.synchronize()
            best = min(best, time.perf_counter() - t1)
        del dq
        best = d.max(best)
        link = {"value": round(d.world * m / best / 1e6, 2), "unit": "M queries/s",
                "frac": round(qps / (d.world * m / best), 4),
                "what": "the step's H2D (queries) and D2H (pos|found, values) bytes copied concurrently on two "
                        "streams, no search: the host-link ceiling of e2e"}
    except RuntimeError:
        link = None
    api = (f"H2D + hbt_search_sharded + D2H (pinned host buffers; {nchunk} chunks, copies overlapping the "
           "collective searches)" if sharded else
           "hbt_search_host (pinned host buffers; chunks of 2^%d queries: H2D, search, D2H pipelined over %d "
           "streams)" % (work.host_chunk_log2, work.host_bufs))
    out = {"value": round(qps / 1e6, 2), "unit": "M queries/s", "h2d_bytes_per_step": m * w,
           "d2h_bytes_per_step": m * (8 + w), "api": api, "link_ceiling": link}
    if check:
        out["check"] = check
    return out


def run_hbt(args):
    import torch
    import torch.distributed as dist

    rank, world, local = dist_env()
    d = Dist(rank, world, local)
    work = make_work(args.config, d, args)
    c, m, w, info = work.c, work.m, work.w, work.info
    torch.cuda.synchronize()
    node_b = ((c["fanout"] * w + 31) // 32) * 32
    l2_probe = probe_l2_gbs(32 if node_b > 32 else node_b) if rank == 0 else None
    # the probe at every access granularity of the tree (reported beside the roofline)
    l2_probe_by_chunk = {str(b): round(probe_l2_gbs(b) or 0.0, 1) for b in (32, 64, 128)} if rank == 0 else None
    # random 64 B reads over 1 GB (8x the L2): the rate DRAM sustains for the leaf-line access
    # pattern (row activations, not bytes, bind it) -- context beside the HBM copy peak
    dram_rand64 = probe_l2_gbs(64, 1 << 30) if rank == 0 else None
    # random 64 B LINE reads (lane pairs, 256-bit loads) from an 8 GB buffer: the rate the HBM
    # serves the leaf-line access of the bucketed item search (tools/probe.cu probe_gather64;
    # saturates with 512 lines in flight per SM, profiles/r02s_gather64_probe.jsonl)
    line_rate = probe_line_rate() if rank == 0 else None
    # NVLink (SURVEY 8(d) BW_NVL) for the sharded config's a2a term, measured in this run
    a2a_gbs = probe_a2a_gbs(d) if args.config == "c4" else None

    use_graph = args.graph == "1" or (args.graph == "auto" and m <= (1 << 20) and args.config != "c4"
                                      and not args.origin_rank0)
    graph = capture_step(work) if use_graph else None
    for _ in range(max(args.warmup, 3)):
        if graph is not None:
            graph.replay()
        else:
            step(work)
    torch.cuda.synchronize()
    sampler = ClockSampler(d.device)
    sampler.start()
    ms_step = time_search(work, args.steps, graph)
    clocks = sampler.stop()
    qps = world * m / (ms_step * 1e-3)
    launches_per_step = 4 if args.config == "c4" else (2 if args.range_k else 1)

    after = None
    if "batch" in work.extra:  # c3: the 1 % bulk update, timed once, then search again
        bk, bv, bo = work.extra["batch"]
        warm_update_path(work)  # first-use costs (lazy kernel loading, pool growth) are not the update
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        work.tree.update(bk, bv, bo)
        torch.cuda.synchronize()
        upd_s = time.perf_counter() - t0
        for _ in range(3):
            work.tree.search(work.q, work.out_pos, work.out_val)
        ms_after = time_search(work, args.steps)
        after = {"update_ops": int(bk.numel()), "update_ms": round(upd_s * 1e3, 3),
                 "update_ops_per_s": round(bk.numel() / upd_s, 1),
                 "search_after_update": {"value": round(world * m / (ms_after * 1e-3) / 1e6, 2),
                                         "unit": "M queries/s", "ms_per_step": round(ms_after, 4)},
                 "n_distinct_after": work.tree.info()["n_distinct"]}

    e2e = time_e2e(work, args.e2e_steps) if not args.range_k else None

    # ---- roofline of the step's dominant kernel.  Unbucketed: the step IS one search
    # launch.  Bucketed (regular trees beyond the L2, csrc/bucketed.cu): the step is
    # count / scan / scatter / search / gather; the library's phase events (CUDA events
    # on the launching stream) give the tree-search kernel's own duration.
    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    phases = None
    if hasattr(work.tree, "last_phases") and not args.range_k:
        try:
            work.tree.set_param("phase_timing", 1)
            acc = {}
            reps = 5
            for _ in range(reps):
                step(work)
                for k_, v_ in work.tree.last_phases().items():
                    acc[k_] = acc.get(k_, 0.0) + v_
            work.tree.set_param("phase_timing", 0)
            phases = {k_: (round(v_ / reps, 4) if k_ != "launches" else int(v_ / reps)) for k_, v_ in acc.items()}
        except hbt.HBTError:
            phases = None
    l2_size = torch.cuda.get_device_properties(d.device).L2_cache_size
    gran_extra = 0
    if phases:
        mdl = roofline.model_bucketed(info, m)
        t_kernel = phases["search"] * 1e-3
        kernel = ("regular_search_items_kernel" if c["layout"] == "regular" else "implicit_search_items_kernel")
        # c4: the sharded step's own kernels (count / publish / barrier / return) + the pipeline
        # c4 at N > 1, fused exchange: f_count, f_publish, f_put and three device barriers
        # around the owner's bucketed search (whose gather stores into the requesters' windows)
        launches_per_step = phases["launches"] + (6 if args.config == "c4" and world > 1 else 0)
        model_desc = "bucketed search: query + 16 B record + distinct tree lines per pass (tools/roofline.py)"
    else:
        mdl = roofline.model(info, l2_size, work.hit_rate)
        t_kernel = ms_step * 1e-3
        kernel = ("regular_search_v2" if c["layout"] == "regular" else "implicit_search_kernel")
        model_desc = "ideal static L2 cache of %d B (SURVEY §8d)%s" % (
            l2_size, "; Zipf modelled as uniform (upper bound on bytes)" if args.config == "c5" else "")
    if args.range_k:  # + the further leaf lines walked and the k pairs written (+ count)
        P = 64 // (2 * w)
        extra_b = ((args.range_k - 1 + P - 1) // P) * 64 + args.range_k * 2 * w + 4
        mdl["hbm_bytes_per_query"] += extra_b
        mdl["l2_bytes_per_query"] += extra_b
        gran_extra = extra_b
        kernel = "range_scan_kernel"
    peak, peak_src = measured_peaks()
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp) and not (args.config == "c4" and world > 1):  # measured on one GPU
        traffic = json.load(open(tp)).get(args.config)
    traffic_bytes = traffic.get("dram_bytes_per_launch") if isinstance(traffic, dict) and not args.range_k else None
    if traffic_bytes and traffic.get("kernel") and not args.range_k:
        # the dominant kernel's name as ncu reported it in the traffic capture
        kernel = traffic["kernel"].split("::")[-1].split("<")[0]
    hbm_ach = mdl["hbm_bytes_per_query"] * m / t_kernel / 1e9
    roof_hbm = {"bound": "hbm", "achieved": round(hbm_ach, 1), "peak": peak, "unit": "GB/s",
                "frac": round(hbm_ach / peak, 4), "traffic": traffic_bytes,
                "traffic_source": traffic.get("source") if isinstance(traffic, dict) else None,
                # measured DRAM bytes of one launch (ncu, steady state) over this run's launch time
                "traffic_gbs": round(traffic_bytes / t_kernel / 1e9, 1) if traffic_bytes else None,
                "traffic_frac": round(traffic_bytes / t_kernel / 1e9 / peak, 4) if traffic_bytes else None,
                "bytes_per_query_model": round(mdl["hbm_bytes_per_query"], 2), "peak_source": peak_src,
                # SURVEY 8(d) reporting: measured B/q from ncu and the fraction of the 8 TB/s spec HBM roof
                "traffic_bytes_per_query": round(traffic_bytes / m, 2) if traffic_bytes else None,
                "frac_of_8tbs_spec": round(hbm_ach / 8000.0, 4),
                "random_64b_read_probe_gbs": round(dram_rand64, 1) if dram_rand64 else None,
                "frac_of_random_64b_probe": round(hbm_ach / dram_rand64, 4) if dram_rand64 else None,
                # every query reads >= 1 random leaf line: queries/s of the kernel against the
                # random-line rate of the HBM measured in this run (the access-rate roof)
                "random_line_probe_glines_per_s": round(line_rate, 2) if line_rate else None,
                "frac_of_random_line_rate": round(m / t_kernel / 1e9 / line_rate, 4) if line_rate else None,
                "model": model_desc}
    if args.config == "c4" and world > 1:
        a2a_b = (world - 1) / world * (w + 8 + w)
        bw_nvl = a2a_gbs or NVLINK_GBS
        t_roof = mdl["hbm_bytes_per_query"] / (peak * 1e9) + a2a_b / (bw_nvl * 1e9)
        roof_hbm["a2a_bytes_per_query"] = round(a2a_b, 2)
        roof_hbm["nvlink_gbs"] = round(bw_nvl, 1)
        roof_hbm["nvlink_source"] = ("measured in this run (NCCL all_to_all_single)" if a2a_gbs else
                                     "B200_PROFILING.md peer copy 770 GB/s per direction (fallback)")
        roof_hbm["frac_with_nvlink"] = round((m / t_kernel) * t_roof, 4)
    roof_l2 = None
    if l2_probe:
        # the model's L2 bytes by access granularity, each class at the probe of its own
        # granularity: roof time = sum(bytes_c / BW_c); peak = bytes / roof time
        gran = roofline.l2_granularity(info, work.hit_rate, bucketed=bool(phases),
                                       level=info["height"] if phases else None)
        gran[64] += gran_extra
        probes = {32: l2_probe_by_chunk.get("32") or l2_probe, 64: l2_probe_by_chunk.get("64") or l2_probe}
        t_q = sum(b / (probes[g] * 1e9) for g, b in gran.items())
        l2_peak = mdl["l2_bytes_per_query"] / t_q / 1e9
        l2_ach = mdl["l2_bytes_per_query"] * m / t_kernel / 1e9
        roof_l2 = {"bound": "l2", "achieved": round(l2_ach, 1), "peak": round(l2_peak, 1), "unit": "GB/s",
                   "frac": round(l2_ach / l2_peak, 4), "bytes_per_query_model": round(mdl["l2_bytes_per_query"], 2),
                   "bytes_per_query_by_access": {str(g): round(b, 2) for g, b in gran.items()},
                   "peak_source": "measured in this run: all-SM random reads of a 32 MB L2-resident buffer at 32 B "
                                  "and 64 B granularity (tools/probe.cu; SURVEY §8d BW_L2), weighted by the model's "
                                  "bytes at each granularity",
                   "probe_gbs_by_access_bytes": l2_probe_by_chunk,
                   "frac_vs_32b_probe": round(l2_ach / l2_probe, 4)}
    # roof time = max(B_HBM / BW_HBM, B_L2 / BW_L2); the binding term is the
    # kernel's roofline, its frac = roof time / measured kernel time.
    roof = dict(roof_l2 if roof_l2 and roof_l2["frac"] > roof_hbm["frac"] else roof_hbm)
    roof["traffic"] = traffic_bytes
    roof["kernel"] = kernel
    roof["kernel_ms"] = round(t_kernel * 1e3, 4)
    roof["frac_hbm"] = roof_hbm["frac"]
    roof["frac_l2"] = roof_l2["frac"] if roof_l2 else None
    if args.leaf_host:
        # zero-copy: the leaf line crosses the host link once per query; streamed (the
        # library's auto rule, 160 B x m > L-segment): the whole L-segment once per step
        h2d = measure_h2d_gbs()
        ls = dict(kv.split("=", 1) for kv in args.param).get("leaf_stream", "2")
        streamed = c["layout"] == "implicit" and (ls == "1" or (ls == "2" and m * 160 > info["leaf_bytes"]
                                                                and info["leaf_bytes"] > (8 << 20)))
        link_b = info["leaf_bytes"] if streamed else 64 * m
        link_ach = link_b / t_kernel / 1e9
        roof["link"] = {"bound": "host link (%s)" % ("L-segment slices streamed into HBM per bucket"
                                                     if streamed else "zero-copy leaf reads"),
                        "bytes_per_query": round(link_b / m, 2),
                        "achieved": round(link_ach, 1), "unit": "GB/s", "peak": round(h2d, 1),
                        "peak_source": "measured in this run: pinned H2D cudaMemcpy of 1 GiB",
                        "frac": round(link_ach / h2d, 4)}
        if streamed:  # partition (count, run starts, scatter) + one search per bucket + gather
            slice_b = int(dict(kv.split("=", 1) for kv in args.param).get("stream_slice", "0"), 0) or (8 << 20)
            nb = min(1024, -(-info["leaf_bytes"] // slice_b), info["leaf_lines"])
            launches_per_step = 5 + nb
    if m <= (1 << 20) and not args.range_k:
        roof["note"] = ("latency-bound batch: %d queries are one wave of the GPU, so the step is the launch "
                        "plus one query's chain of dependent memory round trips; no byte roofline binds" % m)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(args.config)

    d.barrier()
    if rank == 0:
        line = {
            "metric": "lookups/sec (M queries/s)",
            "value": round(qps / 1e6, 2),
            "unit": "M queries/s",
            "n_gpus": world,
            "steps": args.steps,
            "warmup": max(args.warmup, 3),
            "ms_per_step": round(ms_step, 4),
            "higher_is_better": True,
            "scaling": "strong" if args.config in ("c4", "c5") else "weak",
            "vs_baseline": None,
            "dtype": "u64" if w == 8 else "u32",
            "data": "synthetic (seeded counter-based generators, gen/)",
            "config": bench_config(args, world),
            "e2e": e2e,
            "gpu_launches": args.steps * launches_per_step,
            "gpu_launches_per_step": launches_per_step,
            "roofline": roof,
            "roofline_hbm": roof_hbm,
            "roofline_l2": roof_l2,
            "phases_ms": phases,
            "clocks": clocks,
            "cpu_baseline": cpu,
            "launch": "CUDA graph replay of the captured step" if graph is not None else "direct",
            "tree": {k: info[k] for k in ("height", "smem_levels", "level_nodes", "leaf_lines", "chain_len",
                                          "inner_bytes", "leaf_bytes", "n_distinct")},
            "ranks_share_gpus": d.shared_gpus,
            "process_group": d.backend,
            "context": "paper: up to 240 M queries/s (HB+ implicit, GTX 780 + Xeon E5-2665, PAPER.md:9,57)",
        }
        if args.config == "c4":
            line["nvlink"] = {"a2a_gbs_measured": round(a2a_gbs, 1) if a2a_gbs else None,
                              "a2a_bytes_per_query": round((world - 1) / world * (w + 8 + w), 2),
                              "probe": ("NCCL all_to_all_single of 256 MiB per rank in this run, bytes leaving "
                                        "each GPU per second" if a2a_gbs else
                                        "not measured (one rank, or ranks sharing a GPU)")}
        if after:
            line["update"] = after
        print(json.dumps(line), flush=True)
    d.close()


def bench_config(args, world):
    """The workload description shared by both arms (this one and --impl reference),
    from the configuration alone (BASELINE.json configs[], gen.CONFIGS)."""
    c = gen.CONFIGS[args.config]
    w = c["width"]
    m_total = c["m"] if args.config in ("c4", "c5") else c["m"] * world
    qk = {"uniform": "uniform hits with replacement", "stratified": "uniform hits over all keys",
          "uniform_ins": "uniform over key indices [0, n + n_ins) (misses = not-yet-inserted keys)",
          "shuffle": "Knuth shuffle of the keys (PAPER.md:298)",
          "zipf": f"Zipf({c.get('theta')}) over key ranks, scrambled through the key order"}[c["queries"]]
    if args.queries:
        qk = f"{args.queries} query values on [0, 1] mapped to [0, MAX] (PAPER.md:346-352)"
    keys = "stratified (i << 33 | mix64 low bits), sorted" if args.config == "c4" else "mix64 / fmix32 stream"
    if args.config == "c4":
        par = f"key-range sharded x{world}" if world > 1 else "single GPU, whole tree (one shard)"
    else:
        par = f"replicated x{world}" if world > 1 else "single"
    fits_l2 = args.config == "c1"
    return {"workload": f"{args.config}: {c['layout']} tree, n={c['n']} keys (u{8 * w}, {keys}), fanout "
                        f"{c['fanout']}, m={m_total} queries in total ({qk})"
                        + (f"; range scans of {args.range_k} keys" if args.range_k else ""),
            "n_keys": c["n"], "queries_total": m_total, "queries_per_rank": m_total // world if world else m_total,
            "fanout": c["fanout"], "layout": c["layout"], "key_bits": 8 * w, "parallelism": par,
            "exchange": (("fused peer-memory (CUDA IPC windows)" if not args.exchange else "NCCL send/recv")
                         if args.config == "c4" and world > 1 else None),
            "l2_policy": ("L2 flushed between timed steps (2x-L2 buffer write outside the per-step CUDA-event "
                          "intervals; the tree and the batch fit in the L2)" if fits_l2 else
                          "inputs larger than L2 (queries + results per step exceed the 126 MB L2)")}


def _oracle_workload(cfg_name, m):
    """Host copy of the config's keys/values and an m-query sample (same generators)."""
    c = gen.CONFIGS[cfg_name]
    k, v = gen.workload_keys_values(cfg_name)
    if cfg_name == "c3":
        _, _, _, n_ins = gen.update_batch(cfg_name, len(k))
        return c, k, v, gen.workload_queries(cfg_name, k, m, n_ins=n_ins)
    if cfg_name == "c1":
        return c, k, v, gen.workload_queries(cfg_name, k)
    return c, k, v, gen.workload_queries(cfg_name, k, m)


C4_SLICE = 1 << 26  # keys of the contiguous c4 slice the oracle builds (2^26 of 2^31)


def c4_oracle_sample(m):
    """c4 for the oracle, bounded: the contiguous slice of the first 2^26 stratified keys
    (a complete subtree of the 2^31-key tree: global rank = slice rank), and m queries
    of the same recipe restricted to it (q = K_u, u uniform over the slice)."""
    c = gen.CONFIGS["c4"]
    sk = gen.stream_seed(c["cfg"], gen.STREAM_K)
    sv = gen.stream_seed(c["cfg"], gen.STREAM_V)
    sq = gen.stream_seed(c["cfg"], gen.STREAM_Q)
    k = gen.stratified_keys(C4_SLICE, sk)
    v = gen.values(C4_SLICE, 8, sv)
    q = k[gen.uniform_indices(m, C4_SLICE, sq).astype(np.int64)]
    return c, k, v, q


def c4_closed_form_qps(chunk=1 << 24):
    """SURVEY §8(c).4 pin timed as a CPU program: the stratified closed form over ALL
    2^28 c4 queries (i = q >> 33, r = i + (q > K_i), found iff q == K_i), numpy on
    the host, in chunks.  Query generation is outside the timed part."""
    c = gen.CONFIGS["c4"]
    sk = gen.stream_seed(c["cfg"], gen.STREAM_K)
    sv = gen.stream_seed(c["cfg"], gen.STREAM_V)
    sq = gen.stream_seed(c["cfg"], gen.STREAM_Q)
    n, m = c["n"], c["m"]
    el = 0.0
    for s in range(0, m, chunk):
        u = gen.uniform_indices(min(chunk, m - s), n, sq, start=s)
        q = (u << np.uint64(33)) | (gen.mix64(u ^ np.uint64(sk)) & np.uint64((1 << 33) - 1))
        t0 = time.perf_counter()
        i = q >> np.uint64(33)
        ki = (i << np.uint64(33)) | (gen.mix64(i ^ np.uint64(sk)) & np.uint64((1 << 33) - 1))
        r = i + (q > ki).astype(np.uint64)
        found = q == ki
        val = np.where(found, gen.mix64(i ^ np.uint64(sv)), np.uint64(0))
        pf = np.where(r < np.uint64(n), r, np.uint64(0x7FFFFFFFFFFFFFFF)) | (found.astype(np.uint64) << np.uint64(63))
        el += time.perf_counter() - t0
        del pf, val
    return m / el, el


def cpu_baseline(cfg_name, target_s=8.0):
    """The oracle as it stands, on this host's cores, over a bounded sample."""
    import oracle
    if cfg_name == "c4":
        c, k, v, q = c4_oracle_sample(1 << 20)
    else:
        c, k, v, q = _oracle_workload(cfg_name, 1 << 20)
    t0 = time.perf_counter()
    tree = (oracle.ITree if c["layout"] == "implicit" else oracle.RTree).from_pairs(k, v, c["fanout"], c["width"])
    build_s = time.perf_counter() - t0
    cores = oracle.default_threads()
    tree.search(q[: 1 << 16], nthreads=cores)
    t0 = time.perf_counter()
    reps = 0
    while True:
        tree.search(q, nthreads=cores)
        reps += 1
        el = time.perf_counter() - t0
        if el > target_s or reps >= 50:
            break
    qps = reps * len(q) / el
    # SURVEY 8(d) oracle timings beside it: one thread, and std::lower_bound over the
    # sorted array with all threads (bounded samples)
    q1 = q[: 1 << 18]
    t0 = time.perf_counter()
    tree.search(q1, nthreads=1)
    qps1 = len(q1) / (time.perf_counter() - t0)
    Kd, Vd = oracle.dedupe(k, v)
    oracle.lower_bound(Kd, Vd, q[: 1 << 16], nthreads=cores)
    t0 = time.perf_counter()
    oracle.lower_bound(Kd, Vd, q, nthreads=cores)
    qps_lb = len(q) / (time.perf_counter() - t0)
    del tree
    cpu_model = ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                cpu_model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    sample = (f"{reps} x {len(q)} queries of the same workload, oracle tree search "
              f"(scalar node scan, OpenMP static chunks), {el:.1f} s; oracle build {build_s:.1f} s")
    out = {"value": round(qps / 1e6, 3), "unit": "M queries/s", "cores": cores, "kind": "oracle",
           "sample": sample, "one_thread": round(qps1 / 1e6, 3), "lower_bound_all_threads": round(qps_lb / 1e6, 3),
           "build_s": round(build_s, 2), "cpu_model": cpu_model, "nproc": os.cpu_count()}
    if cfg_name == "c4":
        out["sample"] = (f"c4 slice: the oracle tree built on the first {C4_SLICE} stratified keys (a complete "
                         f"subtree of the 2^31-key tree), {reps} x {len(q)} uniform hit queries over that slice; "
                         + sample)
        cf_qps, cf_s = c4_closed_form_qps()
        out["closed_form_all_queries"] = {
            "value": round(cf_qps / 1e6, 3), "unit": "M queries/s", "seconds": round(cf_s, 2), "cores": 1,
            "what": "SURVEY 8(c).4 stratified closed form (i = q >> 33, r = i + (q > K_i)) over all 2^28 queries, "
                    "numpy, one thread: not a tree search, only valid for this key generator"}
    return out


def run_reference(args):
    """--impl reference: the CPU oracle on this host, same config/metric/unit.  c4: the
    oracle tree of the contiguous 2^26-key slice (built once, untimed), each step a
    2^20-query sample of the c4 recipe restricted to that slice."""
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import oracle
    if args.config == "c4":
        c, k, v, q = c4_oracle_sample(1 << 20)
        what = (f"oracle tree of the first {C4_SLICE} c4 keys (contiguous slice), {len(q)} uniform hit "
                f"queries over that slice per step")
    else:
        c, k, v, q = _oracle_workload(args.config, 1 << 20)
        what = f"{len(q)} queries of {args.config} per step"
    tree = (oracle.ITree if c["layout"] == "implicit" else oracle.RTree).from_pairs(k, v, c["fanout"], c["width"])
    cores = oracle.default_threads()
    for _ in range(max(args.warmup, 1)):
        tree.search(q, nthreads=cores)
    steps = max(1, min(args.steps, 200))
    t0 = time.perf_counter()
    for _ in range(steps):
        tree.search(q, nthreads=cores)
    el = time.perf_counter() - t0
    qps = steps * len(q) / el
    val = round(qps / 1e6, 3)
    line = {
        "impl": "reference", "metric": "lookups/sec (M queries/s)", "value": val, "unit": "M queries/s",
        "n_gpus": world, "steps": steps, "warmup": args.warmup, "ms_per_step": round(el / steps * 1e3, 3),
        "higher_is_better": True, "scaling": "strong" if args.config in ("c4", "c5") else "weak", "vs_baseline": None,
        "dtype": "u64" if c["width"] == 8 else "u32", "data": "synthetic (seeded counter-based generators, gen/)",
        "config": bench_config(args, world),
        "cpu_baseline": {"value": val, "unit": "M queries/s", "cores": cores, "kind": "oracle",
                         "sample": f"{what}, {steps} steps, OpenMP static chunks on {cores} threads"},
        "e2e": {"value": val, "unit": "M queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    rc = maybe_spawn(args)
    if rc is not None:
        sys.exit(rc)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_hbt(args)


if __name__ == "__main__":
    main()
