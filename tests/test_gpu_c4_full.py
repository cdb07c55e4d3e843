"""configs[3] (c4) at FULL size on one B200, in the launch configuration bench.py
times: the 2^31-key stratified implicit tree (fanout 16, 36 GiB) held as ONE shard
(ShardedTree over a one-rank communicator, the bucketed owner search), 2^28 uniform
hit queries.

Pins, none of which comes from the CUDA path:
* ALL 2^28 outputs against the stratified closed form: keys K_i = (i << 33) | low_i
  are sorted with one key per 2^33-wide stratum, so for any q with i = q >> 33,
  lower_bound = i + (q > K_i) (n when i >= n), found iff q == K_i, value V_i.
  For the hit queries q = K_u this is pos = u, found, value V_u.
* 2^22 misses / edge queries (q + 1, random u64, 0, MAX) against the same closed form.
* A 2^18 sample against the ORACLE tree built on a contiguous 2^26-key slice of the
  same tree (a complete key range: global rank = slice start + oracle rank).
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_util import GenLib, from_dev, to_dev

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

END = np.uint64(0x7FFFFFFFFFFFFFFF)
FOUND = np.uint64(1 << 63)
LOW = np.uint64((1 << 33) - 1)


def closed_form(q, n, sk, sv):
    """lower bound / found / value of q over the stratified keys K_0..K_{n-1}."""
    q = np.asarray(q, dtype=np.uint64)
    i = q >> np.uint64(33)
    inr = i < np.uint64(n)
    ic = np.where(inr, i, np.uint64(0))
    ki = (ic << np.uint64(33)) | (gen.mix64(ic ^ np.uint64(sk)) & LOW)
    r = np.where(inr, ic + (q > ki).astype(np.uint64), np.uint64(n))
    found = inr & (q == ki)
    pf = np.where(r < np.uint64(n), r, END) | np.where(found, FOUND, np.uint64(0))
    val = np.where(found, gen.mix64(ic ^ np.uint64(sv)), np.uint64(0))
    return pf, val


@pytest.fixture(scope="module")
def c4():
    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    c = gen.CONFIGS["c4"]
    n, m = c["n"], c["m"]
    sk = gen.stream_seed(c["cfg"], gen.STREAM_K)
    sv = gen.stream_seed(c["cfg"], gen.STREAM_V)
    sq = gen.stream_seed(c["cfg"], gen.STREAM_Q)
    g = GenLib()
    keys = g.stratified_keys(n, sk)
    vals = g.mix_stream(n, 8, sv)
    comm = hbt.Comm.single()  # as bench.py at N = 1 (no NCCL)
    tree = hbt.ShardedTree(comm, keys, vals, fanout=c["fanout"])
    del keys, vals
    torch.cuda.empty_cache()
    yield dict(hbt=hbt, tree=tree, comm=comm, n=n, m=m, sk=sk, sv=sv, sq=sq, g=g)
    tree.close()
    comm.close()


def test_c4_all_outputs_closed_form(c4):
    n, m, sk, sv, sq = c4["n"], c4["m"], c4["sk"], c4["sv"], c4["sq"]
    dq = c4["g"].stratified_queries(m, n, sq, sk)
    t = c4["tree"]
    t.set_param("phase_timing", 1)
    pf, val = t.search(dq)
    torch.cuda.synchronize()
    assert t.last_phases()["launches"] == 6  # the bucketed owner search ran
    t.set_param("phase_timing", 0)
    del dq
    chunk = 1 << 24
    for s in range(0, m, chunk):
        u = gen.uniform_indices(chunk, n, sq, start=s)
        got_pf = pf[s:s + chunk].cpu().numpy().view(np.uint64)
        got_v = from_dev(val[s:s + chunk], 8)
        # hits: pos = u, found, value = V_u
        exp_pf = u | FOUND
        bad = np.nonzero(got_pf != exp_pf)[0]
        assert bad.size == 0, (s, bad.size, bad[:4], got_pf[bad[:4]], exp_pf[bad[:4]])
        assert np.array_equal(got_v, gen.mix64(u ^ np.uint64(sv)))


def test_c4_misses_and_edges_closed_form(c4):
    n, sk, sv, sq = c4["n"], c4["sk"], c4["sv"], c4["sq"]
    rng = np.random.default_rng(44)
    mq = 1 << 22
    u = gen.uniform_indices(mq, n, sq ^ 0x77)
    hit = (u << np.uint64(33)) | (gen.mix64(u ^ np.uint64(sk)) & LOW)
    q = np.concatenate([hit[: mq // 4] + np.uint64(1), hit[mq // 4: mq // 2] - np.uint64(1),
                        rng.integers(0, 2**64 - 1, mq // 2, dtype=np.uint64, endpoint=True),
                        np.array([0, 1, 2**64 - 1, 2**64 - 2, (n - 1) << 33, ((n - 1) << 33) | ((1 << 33) - 1),
                                  (n // 2) << 33], np.uint64)])
    t = c4["tree"]
    pf, val = t.search(to_dev(q, 8))
    torch.cuda.synchronize()
    epf, ev = closed_form(q, n, sk, sv)
    got = pf.cpu().numpy().view(np.uint64)
    bad = np.nonzero(got != epf)[0]
    assert bad.size == 0, (bad.size, q[bad[:4]], got[bad[:4]], epf[bad[:4]])
    assert np.array_equal(from_dev(val, 8), ev)


def test_c4_sample_vs_oracle_slice(c4):
    """2^18 of the bench batch's outputs whose query falls in a contiguous 2^26-key slice,
    against the oracle tree of that slice (global pos = slice start + oracle pos)."""
    n, m, sk, sv, sq = c4["n"], c4["m"], c4["sk"], c4["sv"], c4["sq"]
    s0, ns = (1 << 30) + 12345, 1 << 26
    k = gen.stratified_keys(ns, sk, start=s0)
    v = gen.values(ns, 8, sv, start=s0)
    o = oracle.ITree.from_pairs(k, v, 16, 8)
    u = gen.uniform_indices(m, n, sq)
    sel = np.nonzero((u >= np.uint64(s0)) & (u < np.uint64(s0 + ns)))[0][: 1 << 18]
    assert sel.size == 1 << 18
    q = k[(u[sel] - np.uint64(s0)).astype(np.int64)]
    # the same queries inside the bench batch: search the whole batch, read the sample
    dq = c4["g"].stratified_queries(m, n, sq, sk)
    pf, val = c4["tree"].search(dq)
    torch.cuda.synchronize()
    idx = torch.from_numpy(sel.astype(np.int64)).cuda()
    got_pf = pf[idx].cpu().numpy().view(np.uint64)
    got_v = from_dev(val[idx], 8)
    assert np.array_equal(from_dev(dq[idx], 8), q)
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    assert not (epf == END).any()
    exp = (epf & ~FOUND) + np.uint64(s0) | (epf & FOUND)
    assert np.array_equal(got_pf, exp)
    assert np.array_equal(got_v, ev)


@pytest.mark.parametrize("slice_bytes", [20_000_000, 0])
def test_c4_recipe_last_inner_level_directory_ties(slice_bytes):
    """The c4 recipe at 2^26 keys / 2^24 queries with ~63 buckets (bucket_slice 20 MB):
    the compressed item directory sits on the LAST INNER level, and hits on the first
    key of a node whose predecessor's max lies within 2^26 below tie in the directory
    (regression: the walk must move on to the next lines).  Every output vs the
    stratified closed form; the default slice as a control."""
    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    c = gen.CONFIGS["c4"]
    n, m = 1 << 26, 1 << 24
    sk = gen.stream_seed(c["cfg"], gen.STREAM_K)
    sv = gen.stream_seed(c["cfg"], gen.STREAM_V)
    sq = gen.stream_seed(c["cfg"], gen.STREAM_Q)
    g = GenLib()
    t = hbt.Tree(g.stratified_keys(n, sk), g.mix_stream(n, 8, sv), fanout=16)
    t.set_param("bucket", 1)
    t.set_param("bucket_slice", slice_bytes)
    dq = g.stratified_queries(m, n, sq, sk)
    # hits, plus misses just above each hit (lower bound = next key)
    q = torch.cat([dq, dq + 1])
    qh = q.cpu().numpy().view(np.uint64)
    epf, ev = closed_form(qh, n, sk, sv)
    for cnode in (1, 0):  # compact last-inner-level nodes (default, on at this size) and the full nodes
        t.set_param("item_cnode", cnode)
        pf, val = t.search(q)
        torch.cuda.synchronize()
        got = pf.cpu().numpy().view(np.uint64)
        bad = np.nonzero(got != epf)[0]
        assert bad.size == 0, (cnode, bad.size, qh[bad[:4]], got[bad[:4]], epf[bad[:4]])
        assert np.array_equal(from_dev(val, 8), ev)
    t.close()
