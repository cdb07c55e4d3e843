"""GPU parity of the IMPLICIT tree against the oracle (bit-exact pos|found and
value; bitwise build arrays).  Calls go through the C ABI (libhbt.so)."""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_util import (END, GenLib, expected_implicit_bytes, from_dev, gpu_build, gpu_search, np_dtype,
                      to_dev)
from test_oracle_implicit import gen_keys, query_set

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def hbt():
    import paper_conf_sigmod_shahvaranij16_b200 as m
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return m


def sizes(F, P):
    return sorted({0, 1, 2, P - 1, P, P + 1, F * P - 1, F * P, F * P + 1, F * F * P - 1, F * F * P + 1,
                   F * F * F * P + 3, 5000})


@pytest.mark.parametrize("width", [4, 8])
@pytest.mark.parametrize("F", [4, 8, 16, 32])
def test_edge_suite_parity(hbt, width, F):
    P = 64 // (2 * width)
    rng = np.random.default_rng(100 * F + width)
    for n in sizes(F, P):
        k, v = gen_keys(n, width, rng, dup=(n % 2 == 1), with_max=(n % 3 == 0))
        o = oracle.ITree.from_pairs(k, v, F, width)
        t = gpu_build(hbt, k, v, F, width)
        info = t.info()
        a = o.arrays()
        assert info["n_distinct"] == a["n"] and info["height"] == a["H"]
        assert info["level_nodes"] == a["nodes"]
        inner, leaf = expected_implicit_bytes(o, width)
        assert t.export(hbt.SEG_INNER).tobytes() == inner, (n, F, width)
        assert t.export(hbt.SEG_LEAF).tobytes() == leaf, (n, F, width)
        assert t.export(hbt.SEG_INNER_IDX).tobytes() == expected_index_bytes(o, width), (n, F, width)
        q = query_set(k, width, rng, 3000)
        epf, ev = o.search(q)
        # top-level modes x per-level read modes (l2b = 1: every level read whole, by
        # 256-bit (f256) or 16 B lane loads)
        for mode, l2b, f256 in ((2, 0, 1), (2, 1, 1), (2, 1, 0), (2, 4096, 1), (3, 0, 1), (3, 1, 0)):
            t.set_search_config(smem_mode=mode)
            t.set_param("l2_levels_bytes", l2b)
            t.set_param("full256", f256)
            pf, val = gpu_search(t, q, width)
            assert np.array_equal(pf, epf), (mode, n, F, width, np.nonzero(pf != epf)[0][:5])
            assert np.array_equal(val, ev), (mode, n, F, width)
        t.close()


def expected_index_bytes(o, width):
    """Per-node index sector derived from the oracle's nodes: entry t = the max
    key of the node's t-th 32 B sector (PAPER.md:134's I_s applied to implicit
    nodes), MAX-padded to max(16, NSEC*S) bytes; empty when F*S <= 32."""
    a = o.arrays()
    F = a["F"]
    node_bytes = F * width
    if node_bytes <= 32 or a["H"] == 0:
        return b""
    kps = 32 // width
    nsec = node_bytes // 32
    ent = max(16, nsec * width) // width
    inner = a["inner"]
    idx = np.full((inner.shape[0], ent), (1 << (8 * width)) - 1, dtype=np.uint64)
    idx[:, :nsec] = inner[:, kps - 1::kps][:, :nsec]
    return idx.astype(np_dtype(width)).tobytes()


@pytest.mark.parametrize("width,F", [(8, 16), (4, 8), (8, 32), (4, 32)])
@pytest.mark.parametrize("ctas,mode", [(0, 2), (1, 2), (0, 3), (2, 3)])
@pytest.mark.parametrize("leaf256", [1, 0])
def test_launch_shape_variants(hbt, width, F, ctas, mode, leaf256):
    """Results must not depend on the resident CTAs per SM, where the level-T
    directory is read from (shared memory or in place) or how the leaf line is loaded."""
    rng = np.random.default_rng(ctas + F + mode)
    k, v = gen_keys(300000, width, rng)
    o = oracle.ITree.from_pairs(k, v, F, width)
    t = gpu_build(hbt, k, v, F, width)
    t.set_search_config(ctas_per_sm=ctas, smem_mode=mode)
    t.set_param("leaf256", leaf256)
    t.set_param("small_batch", 0)  # mode 2 stays mode 2 at this batch size (mode 3 is asked for explicitly)
    q = query_set(k[:5000], width, rng, 20011)
    pf, val = gpu_search(t, q, width)
    epf, ev = o.search(q)
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)


def test_c1_full(hbt):
    """BASELINE configs[0]: implicit, 2^16 u32 keys, F = 8, 2^16 Knuth-shuffled queries
    (PAPER.md:298), plus the c1 suite: 50 % hits, 25 % random u32, 25 % edges."""
    c = gen.CONFIGS["c1"]
    k, v = gen.workload_keys_values("c1")
    q = gen.workload_queries("c1", k)
    o = oracle.ITree.from_pairs(k, v, c["fanout"], c["width"])
    t = gpu_build(hbt, k, v, c["fanout"], c["width"])
    pf, val = gpu_search(t, q, c["width"])
    epf, ev = o.search(q)
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)
    assert (pf >> np.uint64(63)).all()  # every query hits
    rng = np.random.default_rng(1)
    mx = 2**32 - 1
    kk = k.astype(np.uint64)
    edges = np.concatenate([[0, mx, kk.min(), kk.max()], kk[:4000] + 1, kk[4000:8000] - 1]).astype(np.uint64)
    edges = np.clip(edges, 0, mx).astype(np.uint64)
    suite = np.concatenate([kk[rng.integers(0, len(kk), 32768)],
                            rng.integers(0, mx, 16384, dtype=np.uint64, endpoint=True), edges[:16384]])
    pf, val = gpu_search(t, suite, 4)
    epf, ev = o.search(suite)
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)


def test_c2_scaled_full_compare(hbt):
    """configs[1] recipe at 1/32 scale: every output compared with the oracle."""
    n, m = 1 << 18, 1 << 19
    k, v = gen.workload_keys_values("c2", n)
    q = gen.workload_queries("c2", k, m)
    o = oracle.ITree.from_pairs(k, v, 16, 8)
    t = gpu_build(hbt, k, v, 16, 8)
    pf, val = gpu_search(t, q, 8)
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)


def test_c2_full_size_bench_launch(hbt):
    """configs[1] at full size (2^23 u64 keys, F = 16, 2^24 uniform hit queries)
    through the same generator/launch path bench.py times: sampled outputs vs the
    oracle, and for ALL outputs the properties that hold at any size
    (found, value = V_u of the generator, pos = rank of K_u)."""
    c = gen.CONFIGS["c2"]
    n, m, w = c["n"], c["m"], 8
    g = GenLib()
    sk = gen.stream_seed(2, gen.STREAM_K)
    sv = gen.stream_seed(2, gen.STREAM_V)
    sq = gen.stream_seed(2, gen.STREAM_Q)
    dk = g.mix_stream(n, w, sk)
    dv = g.mix_stream(n, w, sv)
    dq = g.uniform_queries(m, n, w, sq, sk)
    t = hbt.Tree(dk, dv, fanout=16, layout="implicit")
    pf, val = t.search(dq)
    torch.cuda.synchronize()
    pf = pf.cpu().numpy().view(np.uint64)
    val = from_dev(val, w)
    # all outputs: properties
    k = gen.keys(n, w, sk)
    v = gen.values(n, w, sv)
    u = gen.uniform_indices(m, n, sq).astype(np.int64)
    order = np.argsort(k, kind="stable")
    rank = np.empty(n, np.int64)
    rank[order] = np.arange(n)
    assert (pf >> np.uint64(63)).all()
    assert np.array_equal(val, v[u])
    assert np.array_equal((pf & np.uint64(END)).astype(np.int64), rank[u])
    # sample: the oracle tree, one by one
    o = oracle.ITree.from_pairs(k, v, 16, 8)
    idx = np.random.default_rng(0).integers(0, m, 1 << 18)
    q = from_dev(dq, w)[idx]
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    assert np.array_equal(pf[idx], epf) and np.array_equal(val[idx], ev)


@pytest.mark.parametrize("width", [4, 8])
def test_implicit_update_parity(hbt, width):
    rng = np.random.default_rng(width)
    for n in [0, 10, 4000]:
        k, v = gen_keys(n, width, rng, dup=True)
        o = oracle.ITree.from_pairs(k, v, 8, width)
        t = gpu_build(hbt, k, v, 8, width)
        for _ in range(3):
            nops = 1500
            mx = (1 << (8 * width)) - 1
            live = k if len(k) else np.zeros(1, np.uint64)
            ok = np.where(rng.random(nops) < 0.5, live[rng.integers(0, len(live), nops)],
                          rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)).astype(np.uint64)
            ov = rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)
            op = (rng.random(nops) < 0.4).astype(np.uint8)
            o = o.update(ok, ov, op)
            t.update(to_dev(ok, width), to_dev(ov, width), torch.from_numpy(op).cuda())
            inner, leaf = expected_implicit_bytes(o, width)
            assert t.export(hbt.SEG_INNER).tobytes() == inner
            assert t.export(hbt.SEG_LEAF).tobytes() == leaf
            q = query_set(ok[:500], width, rng, 2000)
            pf, val = gpu_search(t, q, width)
            epf, ev = o.search(q)
            assert np.array_equal(pf, epf) and np.array_equal(val, ev)


@pytest.mark.parametrize("pinned", [True, False])
def test_search_host_pipeline(hbt, pinned):
    """hbt_search_host: host buffers, chunked H2D / search / D2H over two streams."""
    width, F = 8, 16
    rng = np.random.default_rng(3)
    k, v = gen_keys(100000, width, rng)
    o = oracle.ITree.from_pairs(k, v, F, width)
    t = gpu_build(hbt, k, v, F, width)
    m = (1 << 22) + 12345  # more than one 4 Mi bucket, ragged tail
    q = k[rng.integers(0, len(k), m)].astype(np.uint64)
    q[::7] = rng.integers(0, 2**64 - 1, len(q[::7]), dtype=np.uint64, endpoint=True)
    if pinned:
        hq = torch.from_numpy(q.view(np.int64)).pin_memory()
        hp = torch.empty(m, dtype=torch.int64).pin_memory()
        hv = torch.empty(m, dtype=torch.int64).pin_memory()
    else:
        hq = q.copy()
        hp = np.empty(m, np.uint64)
        hv = np.empty(m, np.uint64)
    t.search_host(hq, hp, hv)
    pf = hp.numpy().view(np.uint64) if pinned else hp
    val = hv.numpy().view(np.uint64) if pinned else hv
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)


def test_device_generators_match_numpy():
    g = GenLib()
    for w in (4, 8):
        s = gen.stream_seed(2, gen.STREAM_K)
        assert np.array_equal(from_dev(g.mix_stream(100000, w, s, start=7), w),
                              gen.keys(100000, w, s, start=7).astype(np.uint64))
        sq = gen.stream_seed(2, gen.STREAM_Q)
        keys = gen.keys(5000, w, s)
        assert np.array_equal(from_dev(g.uniform_queries(50000, 5000, w, sq, s, start=3), w),
                              gen.uniform_hit_queries(keys, 50000, sq, start=3).astype(np.uint64))
    s = gen.stream_seed(4, gen.STREAM_K)
    assert np.array_equal(from_dev(g.stratified_keys(1000, s, start=5), 8), gen.stratified_keys(1000, s, start=5))


@pytest.mark.parametrize("width", [4, 8])
def test_presorted_input_fast_path(hbt, width):
    """Strictly increasing input skips the sort (c4's stratified keys); a sorted
    input with a duplicate must still take the sort + dedupe path."""
    rng = np.random.default_rng(width)
    k, v = gen_keys(50000, width, rng)
    Kd, Vd = oracle.dedupe(k, v)
    o = oracle.ITree(Kd, Vd, 16, width)
    t = gpu_build(hbt, Kd, Vd, 16, width)
    inner, leaf = expected_implicit_bytes(o, width)
    assert t.export(hbt.SEG_INNER).tobytes() == inner and t.export(hbt.SEG_LEAF).tobytes() == leaf
    q = query_set(Kd[:3000], width, rng, 3000)
    pf, val = gpu_search(t, q, width)
    epf, ev = o.search(q)
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)
    kd2 = np.insert(Kd, 100, Kd[100])  # sorted, not distinct: last occurrence wins
    vd2 = np.insert(Vd, 101, np.uint64(7))
    o2 = oracle.ITree.from_pairs(kd2, vd2, 16, width)
    t2 = gpu_build(hbt, kd2, vd2, 16, width)
    assert t2.export(hbt.SEG_LEAF).tobytes() == expected_implicit_bytes(o2, width)[1]


@pytest.mark.parametrize("kind", ["normal", "gamma", "zipf", "uniform"])
def test_skewed_query_values(hbt, kind):
    """The paper's skew experiment: query values from Normal / Gamma /
    clustered Zipf on [0, 1] mapped to [0, MAX] — mostly misses, concentrated in
    a part of the key space; both tree forms vs the oracle."""
    import gen as g
    rng = np.random.default_rng(1)
    k, v = gen_keys(200000, 8, rng)
    q = g.skew_values(kind, 50000, 8, 99).astype(np.uint64)
    for layout in ("implicit", "regular"):
        T = oracle.ITree if layout == "implicit" else oracle.RTree
        o = T.from_pairs(k, v, 16, 8)
        t = gpu_build(hbt, k, v, 16, 8, layout=layout)
        pf, val = gpu_search(t, q, 8)
        epf, ev = o.search(q)
        assert np.array_equal(pf, epf) and np.array_equal(val, ev)


def test_c5_full_size_bench_launch(hbt):
    """configs[4] at full size on one GPU (2^27 u64 keys, F = 16, 2^26 Zipf(0.99)
    queries scrambled through the key order) through the bench's launch path.
    ALL outputs: found, value = V_{r-1}, pos = rank of K_{r-1}; a 2^18 sample vs the oracle."""
    c = gen.CONFIGS["c5"]
    n, m, w = c["n"], c["m"], 8
    g = GenLib()
    sk = gen.stream_seed(c["cfg"], gen.STREAM_K)
    sv = gen.stream_seed(c["cfg"], gen.STREAM_V)
    sq = gen.stream_seed(c["cfg"], gen.STREAM_Q)
    t = hbt.Tree(g.mix_stream(n, w, sk), g.mix_stream(n, w, sv), fanout=16, layout="implicit")
    k = gen.keys(n, w, sk)
    r = gen.zipf_ranks(m, n, c["theta"], sq)
    q = k[r - 1]
    pf, val = t.search(torch.from_numpy(q.view(np.int64)).cuda())
    torch.cuda.synchronize()
    pf = pf.cpu().numpy().view(np.uint64)
    val = from_dev(val, w)
    v = gen.values(n, w, sv)
    rank = np.empty(n, np.int64)
    rank[np.argsort(k, kind="stable")] = np.arange(n)
    assert (pf >> np.uint64(63)).all()
    assert np.array_equal(val, v[r - 1])
    assert np.array_equal((pf & np.uint64(END)).astype(np.int64), rank[r - 1])
    o = oracle.ITree.from_pairs(k, v, 16, w)
    idx = np.random.default_rng(7).integers(0, m, 1 << 18)
    epf, ev = o.search(q[idx], nthreads=oracle.default_threads())
    assert np.array_equal(pf[idx], epf) and np.array_equal(val[idx], ev)
    t.close()


def test_search_in_cuda_graph(hbt):
    """hbt_search is capturable: a graph captured once and replayed over new query
    values in the same buffer gives the oracle's results (bench.py replays
    launch-bound steps this way)."""
    width, F = 4, 8
    rng = np.random.default_rng(7)
    k, v = gen_keys(65536, width, rng)
    o = oracle.ITree.from_pairs(k, v, F, width)
    t = gpu_build(hbt, k, v, F, width)
    q0 = query_set(k, width, rng, 65536)
    dq = to_dev(q0, width)
    pos = torch.empty(dq.numel(), dtype=torch.int64, device="cuda")
    val = torch.empty(dq.numel(), dtype=dq.dtype, device="cuda")
    gs = torch.cuda.Stream()
    gs.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(gs):
        t.search(dq, pos, val, stream=gs)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=gs):
            t.search(dq, pos, val, stream=gs)
    torch.cuda.synchronize()
    for rep in range(3):
        q = query_set(k, width, rng, 65536)
        dq.copy_(to_dev(q, width))
        g.replay()
        torch.cuda.synchronize()
        epf, ev = o.search(q)
        assert np.array_equal(pos.cpu().numpy().view(np.uint64), epf), rep
        assert np.array_equal(val.cpu().numpy().view(np_dtype(width)).astype(np.uint64), ev), rep
    t.close()
