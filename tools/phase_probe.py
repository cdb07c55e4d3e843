import json, os, sys, torch
sys.path.insert(0, ".")
import gen
import paper_conf_sigmod_shahvaranij16_b200 as hbt
from gen.device import GenLib
c = gen.CONFIGS["c3"]; g = GenLib()
sk, sv, sq = (gen.stream_seed(c["cfg"], s) for s in (gen.STREAM_K, gen.STREAM_V, gen.STREAM_Q))
n, w = c["n"], c["width"]
tree = hbt.Tree(g.mix_stream(n, w, sk), g.mix_stream(n, w, sv), fanout=c["fanout"], layout=c["layout"])
tree.set_param("bucket", 1); tree.set_param("phase_timing", 1)
for m in [1 << 18, 1 << 20, 1 << 22]:
    q = g.uniform_queries(m, n, w, sq, sk)
    for _ in range(5): tree.search(q)
    torch.cuda.synchronize()
    print(m, tree.last_phases())
