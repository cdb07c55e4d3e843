#!/usr/bin/env python
"""bench.py — batched HB+-tree lookups on B200 (one JSON line on rank 0).

Workload (BASELINE.json configs[1], the metric's 1-GPU configuration): implicit
tree, 2^23 uint64 keys, fanout 16, 2^24 uniform hit queries per GPU.  A "step"
is one hbt_search over the whole batch (all hot-path rows: node search through
every level, leaf search, result write).  Inputs are seeded synthetic
(gen/); queries (128 MiB) + results (256 MiB) per step exceed the
126 MB L2, so no explicit flush is done between steps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2|c1|c5|c3]
  python bench.py --impl reference ...   # the CPU oracle arm (rank 0 only)

Multi-GPU (torchrun): every rank holds a replica and searches its own 2^24
queries (weak scaling, no collective on the data path).
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


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=400)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="hbt", choices=["hbt", "reference"])
    ap.add_argument("--config", default="c2", choices=["c1", "c2", "c3", "c5"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--smem", type=int, default=0, help="override smem budget (bytes)")
    ap.add_argument("--qpl", type=int, default=0, help="queries per lane per warp round (1|2)")
    ap.add_argument("--threads", type=int, default=0, help="threads per CTA (256|512)")
    ap.add_argument("--smem-mode", type=int, default=None, help="2 = directory (default), 0 = staged levels, 1 = hi/lo")
    ap.add_argument("--carveout", type=int, default=-1, help="smem carve-out percent (-1 default)")
    return ap.parse_args()


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


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


def probe_l2_gbs(chunk):
    import ctypes as C
    try:
        L = C.CDLL(os.path.join(ROOT, "tools", "libhbtprobe.so"))
        L.probe_random_read_gbs.restype = C.c_double
        L.probe_random_read_gbs.argtypes = [C.c_uint64, C.c_int, C.c_int]
        v = L.probe_random_read_gbs(32 << 20, chunk, 3)
        return v if v > 0 else None
    except OSError:
        return None


def make_workload(cfg_name, rank, dev_gen):
    """Device keys/values and this rank's queries, plus host copies needed later."""
    import torch
    c = gen.CONFIGS[cfg_name]
    n, m, w = c["n"], c["m"], c["width"]
    sk = gen.stream_seed(c["cfg"], gen.STREAM_K)
    sv = gen.stream_seed(c["cfg"], gen.STREAM_V)
    sq = gen.stream_seed(c["cfg"], gen.STREAM_Q)
    keys = dev_gen.mix_stream(n, w, sk)
    vals = dev_gen.mix_stream(n, w, sv)
    hit_rate = 1.0
    if c["queries"] in ("uniform",):
        q = dev_gen.uniform_queries(m, n, w, sq, sk, start=rank * m)
        qdesc = "uniform hits with replacement"
    elif c["queries"] == "shuffle":
        hk = gen.keys(n, w, sk)
        q = torch.from_numpy(gen.workload_queries(cfg_name, hk).view(np.int32 if w == 4 else np.int64)).cuda()
        qdesc = "Knuth shuffle of the keys (PAPER.md:298)"
    elif c["queries"] == "zipf":
        hk = gen.keys(n, w, sk)
        r = gen.zipf_ranks(m, n, c["theta"], sq, start=rank * m)
        q = torch.from_numpy(hk[r - 1].view(np.int64)).cuda()
        qdesc = f"Zipf({c['theta']}) over key ranks, scrambled"
    else:
        raise SystemExit(f"config {cfg_name} not wired into bench.py yet")
    return keys, vals, q, hit_rate, qdesc


def run_hbt(args):
    import torch
    import torch.distributed as dist

    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    from gen.device import GenLib

    rank, world, local = dist_env()
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    c = gen.CONFIGS[args.config]
    w = c["width"]
    g = GenLib()
    keys, vals, q, hit_rate, qdesc = make_workload(args.config, rank, g)
    m = q.numel()
    tree = hbt.Tree(keys, vals, fanout=c["fanout"], layout=c["layout"])
    tree.set_search_config(smem_bytes=args.smem, threads_per_cta=args.threads, queries_per_lane=args.qpl,
                           smem_mode=args.smem_mode, carveout=args.carveout)
    info = tree.info()
    del keys, vals
    out_pos = torch.empty(m, dtype=torch.int64, device="cuda")
    out_val = torch.empty(m, dtype=q.dtype, device="cuda")
    torch.cuda.synchronize()

    l2_probe = probe_l2_gbs(min(128, ((c["fanout"] * w + 31) // 32) * 32)) if rank == 0 else None

    for _ in range(max(args.warmup, 3)):
        tree.search(q, out_pos, out_val)
    torch.cuda.synchronize()

    sampler = ClockSampler(local)
    sampler.start()
    stream = torch.cuda.current_stream()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    ev0.record(stream)
    for _ in range(args.steps):
        tree.search(q, out_pos, out_val)
    ev1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    ms = ev0.elapsed_time(ev1)
    t = torch.tensor([ms], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    ms_step = ms_max / args.steps
    qps = world * m / (ms_step * 1e-3)

    # ---- end to end through the public API with pinned HOST buffers
    hq = q.cpu().pin_memory()
    hp = torch.empty(m, dtype=torch.int64).pin_memory()
    hv = torch.empty(m, dtype=q.dtype).pin_memory()
    tree.search_host(hq, hp, hv)  # warm the pipeline buffers
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(args.e2e_steps):
        tree.search_host(hq, hp, hv)
    e2e_s = time.perf_counter() - t0
    te = torch.tensor([e2e_s], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_qps = world * m * args.e2e_steps / float(te.item())
    chunks = -(-m // (1 << 22))

    # ---- roofline of the (only) kernel of the step
    l2_size = torch.cuda.get_device_properties(local).L2_cache_size
    mdl = roofline.model(info, l2_size, hit_rate)
    peak, peak_src = measured_peaks()
    achieved = mdl["hbm_bytes_per_query"] * m / (ms_step * 1e-3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        traffic = json.load(open(tp)).get(args.config)
    roof = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 4), "traffic": traffic,
            "bytes_per_query_model": round(mdl["hbm_bytes_per_query"], 2), "peak_source": peak_src,
            "model": "ideal static L2 cache of %d B (SURVEY §8d)" % l2_size}
    l2_roof = None
    if l2_probe:
        l2_ach = mdl["l2_bytes_per_query"] * m / (ms_step * 1e-3) / 1e9
        l2_roof = {"bound": "l2", "achieved": round(l2_ach, 1), "peak": round(l2_probe, 1), "unit": "GB/s",
                   "frac": round(l2_ach / l2_probe, 4), "bytes_per_query_model": mdl["l2_bytes_per_query"],
                   "peak_source": "in-run random-read probe, 32 MB buffer (tools/probe.cu)"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(args.config)

    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    if rank != 0:
        return
    line = {
        "metric": "lookups/sec (M queries/s)",
        "value": round(qps / 1e6, 2),
        "unit": "M queries/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": max(args.warmup, 3),
        "ms_per_step": round(ms_step, 4),
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "u64" if w == 8 else "u32",
        "data": "synthetic (seeded counter-based generators, gen/)",
        "config": {"workload": f"{args.config}: {c['layout']} tree, n={c['n']} keys (u{8 * w}), fanout {c['fanout']}, "
                               f"m={m} queries/GPU ({qdesc})",
                   "n_keys": c["n"], "queries_per_gpu": m, "fanout": c["fanout"], "layout": c["layout"],
                   "key_bits": 8 * w, "parallelism": f"replicated x{world}" if world > 1 else "single",
                   "l2_policy": "inputs larger than L2 (queries+results %d MiB/step > L2)" % (m * (2 * w + 8) >> 20),
                   "tree": {"height": info["height"], "smem_levels": info["smem_levels"],
                            "level_nodes": info["level_nodes"], "leaf_lines": info["leaf_lines"],
                            "inner_bytes": info["inner_bytes"], "leaf_bytes": info["leaf_bytes"]}},
        "e2e": {"value": round(e2e_qps / 1e6, 2), "unit": "M queries/s", "h2d_bytes_per_step": m * w,
                "d2h_bytes_per_step": m * (8 + w), "api": "hbt_search_host (pinned host buffers, 4 Mi-query buckets "
                "double-buffered over 2 streams)", "gpu_launches_per_step": chunks},
        "gpu_launches": args.steps,
        "roofline": roof,
        "roofline_l2": l2_roof,
        "clocks": clocks,
        "cpu_baseline": cpu,
        "context": "paper: up to 240 M queries/s (HB+ implicit, GTX 780 + Xeon E5-2665, PAPER.md:9,57)",
    }
    print(json.dumps(line), flush=True)


def cpu_baseline(cfg_name, target_s=8.0):
    """The oracle as it stands, on this host's cores, over a bounded sample."""
    import oracle
    c = gen.CONFIGS[cfg_name]
    n, w = c["n"], c["width"]
    k, v = gen.workload_keys_values(cfg_name)
    t0 = time.perf_counter()
    if c["layout"] == "implicit":
        tree = oracle.ITree.from_pairs(k, v, c["fanout"], w)
    else:
        tree = oracle.RTree.from_pairs(k, v, c["fanout"], w)
    build_s = time.perf_counter() - t0
    cores = oracle.default_threads()
    m = 1 << 20
    q = gen.workload_queries(cfg_name, k, m) if cfg_name != "c1" else gen.workload_queries(cfg_name, k)
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
    return {"value": round(qps / 1e6, 3), "unit": "M queries/s", "cores": cores, "kind": "oracle",
            "sample": f"{reps} x {len(q)} queries of the same workload, oracle tree search "
                      f"(scalar node scan, OpenMP static chunks), {el:.1f} s; oracle build {build_s:.1f} s"}


def run_reference(args):
    """--impl reference: the CPU oracle on this host, same config/metric/unit."""
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import oracle
    c = gen.CONFIGS[args.config]
    w = c["width"]
    k, v = gen.workload_keys_values(args.config)
    tree = (oracle.ITree if c["layout"] == "implicit" else oracle.RTree).from_pairs(k, v, c["fanout"], w)
    cores = oracle.default_threads()
    m = 1 << 20
    q = gen.workload_queries(args.config, k, m)
    for _ in range(args.warmup):
        tree.search(q, nthreads=cores)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        tree.search(q, nthreads=cores)
    el = time.perf_counter() - t0
    qps = args.steps * len(q) / el
    val = round(qps / 1e6, 3)
    line = {
        "impl": "reference", "metric": "lookups/sec (M queries/s)", "value": val, "unit": "M queries/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(el / args.steps * 1e3, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64" if w == 8 else "u32",
        "data": "synthetic", "config": {"workload": f"{args.config} (oracle, {len(q)}-query sample per step)"},
        "cpu_baseline": {"value": val, "unit": "M queries/s", "cores": cores, "kind": "oracle",
                         "sample": f"{len(q)} queries of {args.config} per step"},
        "e2e": {"value": val, "unit": "M queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_hbt(args)


if __name__ == "__main__":
    main()
