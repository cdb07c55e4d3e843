"""Minimal repro of the streamed host-L-segment search (debug aid)."""
import sys
import numpy as np
import torch
sys.path.insert(0, "tests")
sys.path.insert(0, ".")
import paper_conf_sigmod_shahvaranij16_b200 as hbt
import oracle
from gpu_util import gpu_build, gpu_search
from test_oracle_implicit import gen_keys, query_set

width, F, n = 8, 16, int(sys.argv[1]) if len(sys.argv) > 1 else 5000
rng = np.random.default_rng(3)
k, v = gen_keys(n, width, rng)
o = oracle.ITree.from_pairs(k, v, F, width)
t = gpu_build(hbt, k, v, F, width)
t.set_leaf_placement("host")
t.set_param("leaf_stream", 1)
t.set_param("stream_slice", int(sys.argv[2]) if len(sys.argv) > 2 else 4096)
q = query_set(k, width, rng, 20000)
pf, val = gpu_search(t, q, width)
epf, ev = o.search(q)
print("match", np.array_equal(pf, epf), np.array_equal(val, ev))
