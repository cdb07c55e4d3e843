"""End-to-end (pinned host buffers) throughput of c4 on one GPU through hbt_search_host
for several pipeline shapes (chunk size, streams).  One JSON line per shape."""
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_sigmod_shahvaranij16_b200 as hbt  # noqa: E402
from gen.device import GenLib  # noqa: E402

c = gen.CONFIGS["c4"]
g = GenLib()
sk, sv, sq = (gen.stream_seed(c["cfg"], s) for s in (gen.STREAM_K, gen.STREAM_V, gen.STREAM_Q))
n, m = c["n"], c["m"]
comm = hbt.Comm.single()
tree = hbt.ShardedTree(comm, g.stratified_keys(n, sk), g.mix_stream(n, 8, sv), fanout=16)
torch.cuda.empty_cache()
hq = g.stratified_queries(m, n, sq, sk).cpu().pin_memory()
hp = torch.empty(m, dtype=torch.int64).pin_memory()
hv = torch.empty(m, dtype=torch.int64).pin_memory()
for lg, bufs in [(20, 2), (22, 2), (22, 3), (24, 2), (24, 3), (24, 4), (25, 3), (26, 2)]:
    tree.set_param("host_chunk_log2", lg)
    tree.set_param("host_bufs", bufs)
    tree.search_host(hq, hp, hv)
    t0 = time.perf_counter()
    for _ in range(2):
        tree.search_host(hq, hp, hv)
    el = (time.perf_counter() - t0) / 2
    print(json.dumps({"chunk_log2": lg, "bufs": bufs, "ms": round(el * 1e3, 2), "gqps": round(m / el / 1e9, 3)}),
          flush=True)
