"""GPU parity of the BUCKETED search (csrc/bucketed.cu): queries partitioned by
key range before the tree walk and gathered back to query order.  Every output
must equal the oracle's bit for bit, for both tree forms, every bucket count
from 2 to the 1024 cap, empty / tiny trees, misses, 0 and MAX, and after
updates (the splitters are re-derived from the updated tree)."""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_util import GenLib, from_dev, gpu_build, gpu_search, to_dev
from test_oracle_implicit import gen_keys, kmax, query_set

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def hbt():
    import paper_conf_sigmod_shahvaranij16_b200 as m
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return m


def _oracle(layout, k, v, F, width):
    return (oracle.ITree if layout == "implicit" else oracle.RTree).from_pairs(k, v, F, width)


# (bucket_items, bucket_cap, leaf256, item_cdir): plain search, 8 B smem directory, global
# fallback, 128-bit lane loads (directory form auto), compressed per-bucket directory forced
ITEM_MODES = [(0, 0, 1, 1), (1, 0, 1, 0), (1, 7, 1, 1), (1, 0, 0, 1), (1, 0, 1, 2)]


@pytest.mark.parametrize("layout", ["implicit", "regular"])
@pytest.mark.parametrize("width,F", [(4, 8), (8, 16), (8, 32), (4, 32)])
@pytest.mark.parametrize("items,cap,leaf256,dir32", ITEM_MODES)
def test_bucketed_edge_suite(hbt, layout, width, F, items, cap, leaf256, dir32):
    P = 64 // (2 * width)
    rng = np.random.default_rng(900 + 10 * F + width)
    for n in sorted({0, 1, 2, P + 1, F * P + 1, 5 * F * P + 3, 30011}):
        k, v = gen_keys(n, width, rng, dup=(n % 2 == 1), with_max=(n % 3 == 0))
        o = _oracle(layout, k, v, F, width)
        t = gpu_build(hbt, k, v, F, width, layout=layout)
        q = query_set(k, width, rng, 5000)
        q = np.concatenate([q, np.array([0, kmax(width)] * 50, dtype=np.uint64)])
        epf, ev = o.search(q)
        t.set_param("bucket", 1)
        t.set_param("bucket_items", items)
        t.set_param("bucket_cap", cap)
        t.set_param("leaf256", leaf256)
        t.set_param("item_cdir", dir32)
        for slice_bytes, cnode in ((1, 1), (4096, 1), (1 << 16, 1), (4096, 2), (1 << 16, 2)):
            # 1 B: one bucket per unit up to the 1024 cap; cnode 2: compact last-inner-level
            # nodes forced wherever the directory sits on the last inner level
            t.set_param("bucket_slice", slice_bytes)
            t.set_param("item_cnode", cnode)
            pf, val = gpu_search(t, q, width)
            assert np.array_equal(pf, epf), (layout, n, F, width, slice_bytes, cnode, items, cap,
                                             np.nonzero(pf != epf)[0][:5])
            assert np.array_equal(val, ev), (layout, n, F, width, slice_bytes, cnode, items, cap)
        t.close()


@pytest.mark.parametrize("layout,F", [("implicit", 16), ("regular", 32)])
@pytest.mark.parametrize("items,cap,leaf256,dir32", ITEM_MODES)
def test_bucketed_scaled_workload(hbt, layout, F, items, cap, leaf256, dir32):
    """c2 / c3 recipes at reduced size, several bucket counts, every output vs the oracle."""
    cfg = "c2" if layout == "implicit" else "c3"
    n, m = 1 << 19, 1 << 20
    k, v = gen.workload_keys_values(cfg, n)
    q = gen.workload_queries(cfg, k, m) if cfg == "c2" else gen.workload_queries(cfg, k, m, n_ins=n // 100)
    o = _oracle(layout, k, v, F, 8)
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    t = gpu_build(hbt, k, v, F, 8, layout=layout)
    t.set_param("bucket", 1)
    t.set_param("bucket_items", items)
    t.set_param("bucket_cap", cap)
    t.set_param("leaf256", leaf256)
    t.set_param("item_cdir", dir32)
    for slice_bytes in (1 << 16, 1 << 20, 1 << 22):
        t.set_param("bucket_slice", slice_bytes)
        for one_round in (0, 1):  # default and single-round work items
            t.set_param("item_rounds", 1 if one_round else 0)
            for hint, qpf in ((0, 0), (1, 1), (3, 3)):  # L2 hints / query-prefetch distance
                if layout == "implicit":
                    t.set_param("item_l2_hint", hint)
                t.set_param("item_qpf", qpf)
                pf, val = gpu_search(t, q, 8)
                assert np.array_equal(pf, epf) and np.array_equal(val, ev), (layout, slice_bytes, one_round, hint,
                                                                             qpf)
    t.set_param("item_qpf", 1)
    t.set_param("bucket", 0)
    for hint in (0, 1, 2, 3, 4):  # plain search with the same hints (4 = auto)
        t.set_param("l2_hint", hint)
        pf, val = gpu_search(t, q, 8)
        assert np.array_equal(pf, epf) and np.array_equal(val, ev), hint
    t.close()


@pytest.mark.parametrize("layout", ["implicit", "regular"])
@pytest.mark.parametrize("items,cap,leaf256,dir32", ITEM_MODES)
def test_bucketed_after_update(hbt, layout, items, cap, leaf256, dir32):
    """The splitters follow the tree: search, update (keys move between buckets,
    regular leaves split / empty), search again."""
    width, F = 8, 8
    rng = np.random.default_rng(4242)
    n = 20000
    k, v = gen_keys(n, width, rng, dup=True)
    o = _oracle(layout, k, v, F, width)
    t = gpu_build(hbt, k, v, F, width, layout=layout)
    t.set_param("bucket", 1)
    t.set_param("bucket_items", items)
    t.set_param("bucket_cap", cap)
    t.set_param("leaf256", leaf256)
    t.set_param("item_cdir", dir32)
    t.set_param("bucket_slice", 2048)
    q = query_set(k, width, rng, 4000)
    pf, val = gpu_search(t, q, width)
    epf, ev = o.search(q)
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)
    for trial in range(3):
        mu = 6000
        src = np.concatenate([k[rng.integers(0, len(k), mu // 2)],
                              rng.integers(0, kmax(width), mu - mu // 2, dtype=np.uint64)]).astype(np.uint64)
        bv = rng.integers(0, kmax(width), mu, dtype=np.uint64)
        bo = rng.integers(0, 2, mu).astype(np.uint8)
        o = o.update(src, bv, bo) or o  # ITree.update returns the rebuilt tree
        t.update(to_dev(src, width), to_dev(bv, width), torch.from_numpy(bo).cuda())
        q = query_set(np.concatenate([k, src]), width, rng, 4000)
        pf, val = gpu_search(t, q, width)
        epf, ev = o.search(q)
        assert np.array_equal(pf, epf) and np.array_equal(val, ev), (layout, trial)
    t.close()


@pytest.mark.parametrize("layout,F", [("implicit", 16), ("regular", 32), ("regular", 4)])
@pytest.mark.parametrize("nsmall,slice_bytes", [(20000, 1 << 20), (20000, 4096), (20000, 1), (400000, 1 << 30)])
def test_compressed_directory_ties(hbt, layout, F, nsmall, slice_bytes):
    """Compressed per-bucket directory (item_cdir; implicit: unit maxima, regular: leaf
    lines of the chain leaves) where 32-bit truncation ties: dense
    small keys share a bucket with keys near 2^63, so the bucket's shift is ~31 and
    every small maximum truncates to the same value.  Ties are resolved by the walk
    (256-bit whole-node / leaf reads at the directory level) or against the exact
    maxima (16 B reads, index + sector levels).  The 400 K-key tree in one bucket puts
    the directory on the last inner level (whole nodes with l2_levels_bytes = 4096);
    the others on the leaf lines.  Also u32 keys (shift 0)."""
    rng = np.random.default_rng(31)
    small = np.arange(0, 3 * nsmall, 3, dtype=np.uint64)
    big = (np.uint64(1) << np.uint64(63)) + rng.integers(0, 1 << 40, 300, dtype=np.uint64)
    for width, k in ((8, np.concatenate([small, big])), (4, small)):
        v = rng.integers(0, kmax(width), len(k), dtype=np.uint64, endpoint=True)
        o = _oracle(layout, k, v, F, width)
        t = gpu_build(hbt, k, v, F, width, layout=layout)
        q = np.concatenate([query_set(k, width, rng, 6000), k[::7], k[::11] + np.uint64(1), k[::13] - np.uint64(1)])
        q = np.concatenate([q, np.array([0, kmax(width)], dtype=np.uint64)]) & np.uint64(kmax(width))
        epf, ev = o.search(q)
        t.set_param("bucket", 1)
        t.set_param("item_cdir", 2)
        t.set_param("bucket_slice", slice_bytes)
        for rounds, leaf256, full256, l2b, cnode in ((0, 1, 1, 0, 1), (0, 1, 1, 4096, 1), (1, 1, 1, 4096, 1),
                                                     (0, 0, 1, 0, 1), (0, 1, 0, 4096, 1), (1, 0, 0, 0, 1),
                                                     (0, 1, 1, 0, 2), (1, 1, 1, 4096, 2)):
            t.set_param("item_rounds", rounds)
            t.set_param("leaf256", leaf256)
            t.set_param("full256", full256)
            t.set_param("l2_levels_bytes", l2b)
            t.set_param("item_cnode", cnode)  # 2: compact last-level nodes forced (their own ties)
            pf, val = gpu_search(t, q, width)
            cfg = (layout, F, width, slice_bytes, rounds, leaf256, full256, l2b, cnode)
            assert np.array_equal(pf, epf), (cfg, np.nonzero(pf != epf)[0][:5])
            assert np.array_equal(val, ev), cfg
        t.close()


@pytest.mark.parametrize("chunk_log2,bufs", [(22, 2), (20, 2), (20, 3), (14, 4)])
def test_bucketed_host_pipeline(hbt, chunk_log2, bufs):
    """hbt_search_host runs the bucketed path per pipeline chunk, for several chunk
    sizes and numbers of (stream, buffer) pairs, with a ragged last chunk."""
    n, m = 1 << 16, (1 << 22) + 12345
    k, v = gen.workload_keys_values("c2", n)
    q = gen.workload_queries("c2", k, m)
    o = _oracle("implicit", k, v, 16, 8)
    t = gpu_build(hbt, k, v, 16, 8)
    t.set_param("bucket", 1)
    t.set_param("bucket_slice", 1 << 14)
    t.set_param("host_chunk_log2", chunk_log2)
    t.set_param("host_bufs", bufs)
    pf = np.empty(m, np.uint64)
    val = np.empty(m, np.uint64)
    t.search_host(q.copy(), pf, val)
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)
    t.close()


def _full_c3_tree(hbt):
    c = gen.CONFIGS["c3"]
    n, m, w = c["n"], c["m"], 8
    g = GenLib()
    sk = gen.stream_seed(c["cfg"], gen.STREAM_K)
    sv = gen.stream_seed(c["cfg"], gen.STREAM_V)
    sq = gen.stream_seed(c["cfg"], gen.STREAM_Q)
    _, _, _, n_ins = gen.update_batch("c3", n)
    t = hbt.Tree(g.mix_stream(n, w, sk), g.mix_stream(n, w, sv), fanout=c["fanout"], layout="regular")
    dq = g.uniform_queries(m, n + n_ins, w, sq, sk)
    return c, n, m, n_ins, sk, sv, sq, t, dq


def test_c3_full_size_bench_launch(hbt):
    """configs[2] at full size (2^27 u64 keys, F = 32, 2^26 queries) through the bench's
    launch path: auto bucketing with the item directory (asserted via the phase timer),
    before and after the 1 % bulk update.  EVERY output (pos|found and value of all 2^26
    queries) equals the oracle's regular tree, built from the same keys and updated with
    the same batch; found / value are also checked against the generator's closed form
    (found iff the query index is a built key, value = V_u)."""
    c, n, m, n_ins, sk, sv, sq, t, dq = _full_c3_tree(hbt)
    t.set_param("phase_timing", 1)
    pf, val = t.search(dq)
    torch.cuda.synchronize()
    assert t.last_phases()["launches"] == 6  # count, run-start scan, run starts, scatter, search, gather
    pf = pf.cpu().numpy().view(np.uint64)
    val = from_dev(val, 8)
    u = gen.uniform_indices(m, n + n_ins, sq).astype(np.int64)
    hit = u < n
    v = gen.values(n, 8, sv)
    assert np.array_equal((pf >> np.uint64(63)).astype(bool), hit)
    assert np.array_equal(val[hit], v[u[hit]]) and not val[~hit].any()
    k = gen.keys(n, 8, sk)
    o = oracle.RTree.from_pairs(k, v, c["fanout"], 8)
    del k
    q = from_dev(dq, 8)
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    bad = np.nonzero(pf != epf)[0]
    assert bad.size == 0, (bad.size, bad[:5])
    assert np.array_equal(val, ev)
    # the bench's 1 % update, then search again (splitters and item directory re-derived)
    bk, bv, bo, _ = gen.update_batch("c3", n)
    o.update(bk, bv, bo)
    t.update(to_dev(bk, 8), to_dev(bv, 8), torch.from_numpy(bo).cuda())
    pf, val = t.search(dq)
    torch.cuda.synchronize()
    pf = pf.cpu().numpy().view(np.uint64)
    val = from_dev(val, 8)
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    bad = np.nonzero(pf != epf)[0]
    assert bad.size == 0, (bad.size, bad[:5])
    assert np.array_equal(val, ev)
    t.close()


@pytest.mark.parametrize("slice_bytes", [1 << 30, 12 << 20, 5 << 20])
def test_compact_last_level_nodes(hbt, slice_bytes):
    """Compact last-inner-level nodes (item_cnode; bucketed implicit u64 search, F = 16)
    on a tree whose compressed directory sits on the last inner level (1, 2 or 3 buckets
    of a 2^20-key tree: more leaf lines per bucket than the 16-bit directory holds):
    random keys with duplicates and MAX as a key, hits, misses, 0, MAX and neighbours of
    keys, compact nodes off / auto / forced against the oracle."""
    rng = np.random.default_rng(4242)
    n = 1 << 20
    k, v = gen_keys(n, 8, rng, dup=True, with_max=True)
    o = _oracle("implicit", k, v, 16, 8)
    t = gpu_build(hbt, k, v, 16, 8, layout="implicit")
    q = query_set(k, 8, rng, 1 << 18)
    q = np.concatenate([q, k[::5], k[::7] + np.uint64(1), k[::9] - np.uint64(1),
                        np.array([0, kmax(8)], dtype=np.uint64)])
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    t.set_param("bucket", 1)
    t.set_param("bucket_slice", slice_bytes)
    t.set_param("l2_levels_bytes", 4096)  # the last inner level read as whole nodes: compact form in auto mode
    for cnode in (0, 1, 2):
        t.set_param("item_cnode", cnode)
        pf, val = gpu_search(t, q, 8)
        assert np.array_equal(pf, epf), (slice_bytes, cnode, np.nonzero(pf != epf)[0][:5])
        assert np.array_equal(val, ev), (slice_bytes, cnode)
    t.close()
