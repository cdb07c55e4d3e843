"""Bucketed vs unbucketed search by batch size on the c3 tree (regular, 2^27 u64 keys,
F = 32): where does the partition start to pay?  CUDA events, median of 20."""
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
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c3"
    c = gen.CONFIGS[cfg]
    g = GenLib()
    sk, sv, sq = (gen.stream_seed(c["cfg"], s) for s in (gen.STREAM_K, gen.STREAM_V, gen.STREAM_Q))
    n, w = c["n"], c["width"]
    tree = hbt.Tree(g.mix_stream(n, w, sk), g.mix_stream(n, w, sv), fanout=c["fanout"], layout=c["layout"])
    out = {"config": cfg, "rows": []}
    s = torch.cuda.current_stream()
    for m in [1 << 18, 1 << 19, 1 << 20, 1 << 21, 1 << 22, 1 << 23]:
        q = g.uniform_queries(m, n, w, sq, sk)
        pos = torch.empty(m, dtype=torch.int64, device="cuda")
        val = torch.empty(m, dtype=q.dtype, device="cuda")
        row = {"m": m}
        for b in (0, 1):
            tree.set_param("bucket", b)
            for _ in range(5):
                tree.search(q, pos, val)
            ts = []
            for _ in range(20):
                a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                tree.search(q, pos, val)
                e.record(s)
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(e))
            med = statistics.median(ts)
            row["bucketed" if b else "plain"] = {"ms": round(med, 4), "mqps": round(m / med / 1e3, 1)}
        out["rows"].append(row)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
