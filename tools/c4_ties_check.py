"""c4 recipe at reduced size with a last-inner-level item directory (bucket_slice chosen so
the compressed directory ties): every output vs the stratified closed form.
  python tools/debug_gang.py LOG2_N LOG2_M BUCKET_SLICE_BYTES"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import gen  # noqa: E402
import paper_conf_sigmod_shahvaranij16_b200 as hbt  # noqa: E402
from gen.device import GenLib  # noqa: E402
from test_gpu_c4_full import closed_form  # noqa: E402

n, m = 1 << int(sys.argv[1]), 1 << int(sys.argv[2])
slice_bytes = int(sys.argv[3])
c = gen.CONFIGS["c4"]
sk, sv, sq = (gen.stream_seed(c["cfg"], s) for s in (gen.STREAM_K, gen.STREAM_V, gen.STREAM_Q))
g = GenLib()
keys = g.stratified_keys(n, sk)
vals = g.mix_stream(n, 8, sv)
q = g.stratified_queries(m, n, sq, sk)
t = hbt.Tree(keys, vals, fanout=16)
t.set_param("bucket", 1)
t.set_param("bucket_slice", slice_bytes)
epf, ev = closed_form(q.cpu().numpy().view(np.uint64), n, sk, sv)
print(t.info() if hasattr(t, "info") else "")
for gangs in (0,):
    pf, v = t.search(q)
    torch.cuda.synchronize()
    pf = pf.cpu().numpy().view(np.uint64)
    bad = np.nonzero(pf != epf)[0]
    print("gangs", gangs, "mismatches", len(bad), flush=True)
    if len(bad):
        qq = q.cpu().numpy().view(np.uint64)[bad[:8]]
        print("  idx", bad[:8], "\n  q>>33", qq >> np.uint64(33), "\n  got", pf[bad[:8]] & np.uint64((1 << 63) - 1),
              "found", pf[bad[:8]] >> np.uint64(63), "\n  exp", epf[bad[:8]] & np.uint64((1 << 63) - 1))
        vv = v.cpu().numpy().view(np.uint64)
        print("  q", qq, "\n  got v", vv[bad[:8]], "exp v", ev[bad[:8]])
        r = (epf[bad[:8]] & np.uint64((1 << 63) - 1))
        print("  line", r // np.uint64(4), "slot", r % np.uint64(4), "node(H-1)", r // np.uint64(64), "slot in node", (r // np.uint64(4)) % np.uint64(16))
        d = (pf[bad] & np.uint64((1 << 63) - 1)).astype(np.int64) - (epf[bad] & np.uint64((1 << 63) - 1)).astype(np.int64)
        print("  diff hist", np.unique(d, return_counts=True))

