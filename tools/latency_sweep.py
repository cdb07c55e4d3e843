"""Batch-size sweep: per-batch latency and throughput of hbt_search (the paper's
bucket-size experiment, and latency figure).

For each batch size m the same tree (c2: implicit, 2^23 u64 keys, F = 16) is
searched with m uniform hit queries; every launch is timed with CUDA events on
its stream (median of 50 after 10 warm-ups), and the same with the batch
captured in a CUDA graph (launch overhead removed).  Prints one JSON object.
"""
import json
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
import paper_conf_sigmod_shahvaranij16_b200 as hbt  # noqa: E402
from gen.device import GenLib  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
    c = gen.CONFIGS[cfg]
    g = GenLib()
    sk, sv, sq = (gen.stream_seed(c["cfg"], s) for s in (gen.STREAM_K, gen.STREAM_V, gen.STREAM_Q))
    n, w = c["n"], c["width"]
    tree = hbt.Tree(g.mix_stream(n, w, sk), g.mix_stream(n, w, sv), fanout=c["fanout"], layout=c["layout"])
    out = {"config": cfg, "n_keys": n, "rows": []}
    s = torch.cuda.current_stream()
    for m in [1 << 10, 1 << 12, 1 << 14, 1 << 16, 1 << 18, 1 << 20, 1 << 22, 1 << 24]:
        q = g.uniform_queries(m, n, w, sq, sk)
        pos = torch.empty(m, dtype=torch.int64, device="cuda")
        val = torch.empty(m, dtype=q.dtype, device="cuda")
        for _ in range(10):
            tree.search(q, pos, val)
        times = []
        for _ in range(50):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            tree.search(q, pos, val)
            b.record(s)
            torch.cuda.synchronize()
            times.append(a.elapsed_time(b))
        # the same batch as a CUDA graph (launch overhead removed)
        gs = torch.cuda.Stream()
        gs.wait_stream(s)
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.stream(gs):
            tree.search(q, pos, val, stream=gs)
            torch.cuda.synchronize()
            with torch.cuda.graph(graph, stream=gs):
                tree.search(q, pos, val, stream=gs)
        torch.cuda.synchronize()
        gt = []
        for _ in range(50):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            graph.replay()
            b.record(s)
            torch.cuda.synchronize()
            gt.append(a.elapsed_time(b))
        med, gmed = statistics.median(times), statistics.median(gt)
        out["rows"].append({"m": m, "latency_ms": round(med, 4), "mqps": round(m / med / 1e3, 1),
                            "graph_latency_ms": round(gmed, 4), "graph_mqps": round(m / gmed / 1e3, 1)})
    print(json.dumps(out))


if __name__ == "__main__":
    main()
