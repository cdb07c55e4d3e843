"""Small scenarios for compute-sanitizer (memcheck / racecheck / synccheck runs,
tools/sanitize.sh): every kernel family of libhbt.so on a tiny input, each result
checked against the oracle so a run that passes also computed the right thing.

  compute-sanitizer --tool memcheck python tools/sanitize_scenarios.py [names...]
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import gen  # noqa: E402
import oracle  # noqa: E402  (test tool: checks the results)
import paper_conf_sigmod_shahvaranij16_b200 as hbt  # noqa: E402
from gpu_util import from_dev, to_dev  # noqa: E402


def check(t, o, q, width):
    pf, v = t.search(to_dev(q, width))
    torch.cuda.synchronize()
    epf, ev = o.search(q)
    assert np.array_equal(pf.cpu().numpy().view(np.uint64), epf), "pos|found"
    assert np.array_equal(from_dev(v, width), ev), "value"


def sc_implicit_c1():
    """c1 recipe (u32, F = 8): small-batch (in-place directory) and staged-directory searches."""
    k, v = gen.workload_keys_values("c1")
    q = gen.workload_queries("c1", k)
    o = oracle.ITree.from_pairs(k, v, 8, 4)
    t = hbt.Tree(to_dev(k, 4), to_dev(v, 4), fanout=8)
    check(t, o, q, 4)
    t.set_param("small_batch", 0)  # staged directory (mode 2)
    check(t, o, q, 4)


def sc_implicit_u64_levels():
    """u64, F = 16, index + sector levels and whole-node levels, leaf 256-bit loads."""
    k, v = gen.workload_keys_values("c2", 1 << 17)
    q = gen.workload_queries("c2", k, 1 << 17)
    o = oracle.ITree.from_pairs(k, v, 16, 8)
    t = hbt.Tree(to_dev(k, 8), to_dev(v, 8), fanout=16)
    t.set_param("small_batch", 0)
    t.set_param("l2_levels_bytes", 4096)
    check(t, o, q, 8)


def sc_bucketed_both_forms():
    """Bucketed search with the item directory (count, run starts, scatter, item search, gather),
    8 B-key directory and compressed per-bucket directory (bulk copies + mbarrier)."""
    for layout, F, cfg in (("implicit", 16, "c2"), ("regular", 32, "c3")):
        k, v = gen.workload_keys_values(cfg, 1 << 16)
        q = gen.workload_queries(cfg, k, 1 << 17)
        o = (oracle.ITree if layout == "implicit" else oracle.RTree).from_pairs(k, v, F, 8)
        t = hbt.Tree(to_dev(k, 8), to_dev(v, 8), fanout=F, layout=layout)
        t.set_param("bucket", 1)
        t.set_param("bucket_slice", 4096)
        for cdir in (0, 2):
            t.set_param("item_cdir", cdir)
            check(t, o, q, 8)


def sc_regular_update_splits():
    """Regular F = 4 tree, batches that split big leaves, remove leaves and empty the tree."""
    rng = np.random.default_rng(3)
    k = rng.integers(0, 2**64 - 1, 3000, dtype=np.uint64, endpoint=True)
    v = rng.integers(0, 2**64 - 1, 3000, dtype=np.uint64, endpoint=True)
    o = oracle.RTree.from_pairs(k, v, 4, 8)
    t = hbt.Tree(to_dev(k, 8), to_dev(v, 8), fanout=4, layout="regular")
    for b in range(3):
        bk = np.concatenate([rng.integers(0, 2**64 - 1, 2000, dtype=np.uint64, endpoint=True), k[b::3]])
        bv = rng.integers(0, 2**64 - 1, len(bk), dtype=np.uint64, endpoint=True)
        bo = np.concatenate([np.zeros(2000, np.uint8), np.ones(len(k[b::3]), np.uint8)])
        o.update(bk, bv, bo)
        t.update(to_dev(bk, 8), to_dev(bv, 8), torch.from_numpy(bo).cuda())
        check(t, o, np.concatenate([bk[:500], k[:500]]), 8)


def sc_range():
    rng = np.random.default_rng(4)
    k = rng.integers(0, 2**32 - 1, 5000, dtype=np.uint64, endpoint=True)
    for layout in ("implicit", "regular"):
        o = (oracle.ITree if layout == "implicit" else oracle.RTree).from_pairs(k, k, 8, 4)
        t = hbt.Tree(to_dev(k, 4), to_dev(k, 4), fanout=8, layout=layout)
        lo = k[:300]
        hi = np.full(300, 2**32 - 1, np.uint64)
        ok, ov, oc = t.range(to_dev(lo, 4), to_dev(hi, 4), 40)
        torch.cuda.synchronize()
        ek, ev, ec = o.range(lo, hi, 40)
        assert np.array_equal(oc.cpu().numpy().astype(np.uint32), ec)


def sc_virtual_shards():
    """Key-range shard group on one device: fused exchange (f_count / f_publish / f_put /
    remote gather / f_return) and the NCCL-free copy path."""
    n = 40000
    allk = gen.stratified_keys(n, 7)
    allv = gen.values(n, 8, 9)
    full = oracle.ITree.from_pairs(allk, allv, 16, 8)
    for exchange, bucket in ((0, 1), (0, 0), (1, 0)):
        trees = []
        for g in range(3):
            lo, hi = g * n // 3, (g + 1) * n // 3
            t = hbt.Tree(to_dev(allk[lo:hi], 8), to_dev(allv[lo:hi], 8), fanout=16)
            t.set_param("exchange", exchange)
            t.set_param("bucket", bucket)
            t.set_param("bucket_slice", 4096)
            trees.append(t)
        grp = hbt.LocalShardGroup(trees)
        rng = np.random.default_rng(exchange)
        qs = [allk[rng.integers(0, n, 3000 + 1000 * g)] for g in range(3)]
        outs = grp.search([to_dev(q, 8) for q in qs])
        torch.cuda.synchronize()
        for q, (pf, v) in zip(qs, outs):
            epf, ev = full.search(q)
            assert np.array_equal(pf.cpu().numpy().view(np.uint64), epf)


def sc_versioned():
    rng = np.random.default_rng(5)
    k = rng.integers(0, 2**64 - 1, 4000, dtype=np.uint64, endpoint=True)
    for layout, F in (("implicit", 16), ("regular", 4)):
        T = oracle.ITree if layout == "implicit" else oracle.RTree
        o = T.from_pairs(k, k, F, 8)
        vt = hbt.VersionedTree(hbt.Tree(to_dev(k, 8), to_dev(k, 8), fanout=F, layout=layout))
        bk = rng.integers(0, 2**64 - 1, 1500, dtype=np.uint64, endpoint=True)
        bo = np.zeros(1500, np.uint8)
        r = o.update(bk, bk, bo)
        o = r if layout == "implicit" else o
        vt.update(to_dev(bk, 8), to_dev(bk, 8), torch.from_numpy(bo).cuda())
        pf, v, ver = vt.search(to_dev(bk, 8))
        torch.cuda.synchronize()
        assert ver == 1 and np.array_equal(pf.cpu().numpy().view(np.uint64), o.search(bk)[0])
        vt.close()


SCENARIOS = {f.__name__[3:]: f for f in [sc_implicit_c1, sc_implicit_u64_levels, sc_bucketed_both_forms,
                                         sc_regular_update_splits, sc_range, sc_virtual_shards, sc_versioned]}

if __name__ == "__main__":
    torch.cuda.set_device(0)
    names = sys.argv[1:] or list(SCENARIOS)
    for name in names:
        SCENARIOS[name]()
        print("scenario", name, "ok", flush=True)
