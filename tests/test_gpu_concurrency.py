"""Concurrency on one tree (GPU):

* versioned trees (hbt_versioned_*; the paper's concurrent
  search / update queries, App. B.3): a search thread on one
  stream and an update thread on another; every search must equal the ORACLE of the
  version it reports (the oracle applies the same batches in order);
* bucketed searches on two streams right after the bucket splitters were invalidated
  (the shared splitters must be fully prepared before any stream reads them);
* hbt_search_host with PINNED buffers (its chunks run on several streams);
* range scans on two streams at once (per-call lower-bound scratch);
* bulk updates of key-range shards are refused (their routing tables would go stale).
"""
import threading

import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_util import from_dev, gpu_build, to_dev
from test_oracle_implicit import gen_keys, kmax, query_set

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def hbt():
    import paper_conf_sigmod_shahvaranij16_b200 as m
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return m


def _batches(rng, k, width, nb, size):
    mx = kmax(width)
    out = []
    for b in range(nb):
        ins = rng.integers(0, mx, size // 2, dtype=np.uint64, endpoint=True)
        dele = k[rng.integers(0, len(k), size - size // 2)]
        bk = np.concatenate([ins, dele])
        bv = rng.integers(0, mx, len(bk), dtype=np.uint64, endpoint=True)
        bo = np.concatenate([np.zeros(len(ins), np.uint8), np.ones(len(dele), np.uint8)])
        p = rng.permutation(len(bk))
        out.append((bk[p], bv[p], bo[p]))
    return out


@pytest.mark.parametrize("layout,width,F", [("implicit", 8, 16), ("regular", 8, 4), ("regular", 4, 8),
                                            ("implicit", 4, 8)])
def test_versioned_search_during_updates(hbt, layout, width, F):
    rng = np.random.default_rng(77 + F + width)
    n = 60000
    k, v = gen_keys(n, width, rng, dup=True)
    batches = _batches(rng, k, width, 6, 6000 if layout == "regular" else 20000)
    q = np.concatenate([query_set(k[:2000], width, rng, 20000), batches[2][0][:3000]])
    # expected outputs of every version (the oracle applies the batches in order)
    T = oracle.ITree if layout == "implicit" else oracle.RTree
    o = T.from_pairs(k, v, F, width)
    expect = [o.search(q)]
    for bk, bv, bo in batches:
        r = o.update(bk, bv, bo)  # ITree.update returns the rebuilt tree, RTree updates in place
        o = r if layout == "implicit" else o
        expect.append(o.search(q))
    vt = hbt.VersionedTree(gpu_build(hbt, k, v, F, width, layout=layout))
    dq = to_dev(q, width)
    s_search, s_update = torch.cuda.Stream(), torch.cuda.Stream()
    seen = []
    stop = threading.Event()
    errors = []

    def searcher():
        try:
            with torch.cuda.stream(s_search):
                while not stop.is_set() or len(seen) < 3:
                    pf, val, ver = vt.search(dq, stream=s_search)
                    s_search.synchronize()
                    seen.append((ver, pf.cpu().numpy().view(np.uint64), from_dev(val, width)))
        except Exception as e:  # pragma: no cover - reported below
            errors.append(e)

    th = threading.Thread(target=searcher)
    th.start()
    try:
        with torch.cuda.stream(s_update):
            for i, (bk, bv, bo) in enumerate(batches):
                ver = vt.update(to_dev(bk, width), to_dev(bv, width), torch.from_numpy(bo).cuda(), stream=s_update)
                assert ver == i + 1
    finally:
        stop.set()
        th.join()
    assert not errors, errors
    assert vt.version == len(batches)
    versions = {s[0] for s in seen}
    assert len(seen) >= 3
    for ver, pf, val in seen:
        epf, ev = expect[ver]
        assert np.array_equal(pf, epf), (layout, ver, np.nonzero(pf != epf)[0][:5])
        assert np.array_equal(val, ev), (layout, ver)
    # the final version, searched after the last update
    pf, val, ver = vt.search(dq)
    torch.cuda.synchronize()
    assert ver == len(batches)
    assert np.array_equal(pf.cpu().numpy().view(np.uint64), expect[-1][0])
    assert np.array_equal(from_dev(val, width), expect[-1][1])
    vt.close()
    print("versions seen by the searcher:", sorted(versions))


@pytest.mark.parametrize("layout,F", [("implicit", 16), ("regular", 32)])
def test_bucketed_two_streams_after_invalidation(hbt, layout, F):
    n, m = 1 << 18, 1 << 20
    cfg = "c2" if layout == "implicit" else "c3"
    k, v = gen.workload_keys_values(cfg, n)
    q1 = gen.workload_queries(cfg, k, m)
    q2 = gen.workload_queries(cfg, k, m, start=m)
    o = (oracle.ITree if layout == "implicit" else oracle.RTree).from_pairs(k, v, F, 8)
    e1, e2 = o.search(q1, nthreads=oracle.default_threads()), o.search(q2, nthreads=oracle.default_threads())
    t = gpu_build(hbt, k, v, F, 8, layout=layout)
    t.set_param("bucket", 1)
    d1, d2 = to_dev(q1, 8), to_dev(q2, 8)
    sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
    for slice_bytes in (1 << 16, 1 << 20, 4096, 1 << 18):
        t.set_param("bucket_slice", slice_bytes)  # splitters re-derived by the next search
        pa, va = t.search(d1, stream=sa)
        pb, vb = t.search(d2, stream=sb)
        torch.cuda.synchronize()
        assert np.array_equal(pa.cpu().numpy().view(np.uint64), e1[0])
        assert np.array_equal(from_dev(va, 8), e1[1])
        assert np.array_equal(pb.cpu().numpy().view(np.uint64), e2[0])
        assert np.array_equal(from_dev(vb, 8), e2[1])
    t.close()


@pytest.mark.parametrize("layout,F", [("implicit", 16), ("regular", 32)])
def test_search_host_pinned_bucketed(hbt, layout, F):
    n, m = 1 << 17, (1 << 16) + 777
    cfg = "c2" if layout == "implicit" else "c3"
    k, v = gen.workload_keys_values(cfg, n)
    q = gen.workload_queries(cfg, k, m)
    o = (oracle.ITree if layout == "implicit" else oracle.RTree).from_pairs(k, v, F, 8)
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    t = gpu_build(hbt, k, v, F, 8, layout=layout)
    t.set_param("bucket", 1)
    t.set_param("host_chunk_log2", 12)  # 17 chunks over the (stream, buffer) pairs
    hq = torch.from_numpy(q.view(np.int64).copy()).pin_memory()
    for bufs, slice_bytes in ((2, 1 << 14), (4, 1 << 12), (3, 1 << 16)):
        t.set_param("host_bufs", bufs)
        t.set_param("bucket_slice", slice_bytes)
        hp = torch.empty(m, dtype=torch.int64).pin_memory()
        hv = torch.empty(m, dtype=torch.int64).pin_memory()
        t.search_host(hq, hp, hv)
        assert np.array_equal(hp.numpy().view(np.uint64), epf)
        assert np.array_equal(hv.numpy().view(np.uint64), ev)
    t.close()


@pytest.mark.parametrize("layout", ["implicit", "regular"])
def test_range_two_streams(hbt, layout):
    rng = np.random.default_rng(5)
    k, v = gen_keys(50000, 8, rng)
    o = (oracle.ITree if layout == "implicit" else oracle.RTree).from_pairs(k, v, 16, 8)
    t = gpu_build(hbt, k, v, 16, 8, layout=layout)
    Kd, _ = oracle.dedupe(k, v)
    lo1 = Kd[rng.integers(0, len(Kd), 4000)]
    lo2 = Kd[rng.integers(0, len(Kd), 4000)] + np.uint64(1)
    hi = np.full(4000, kmax(8), np.uint64)
    # a larger scan first, so the old per-tree scratch would have had room for both
    t.range(to_dev(Kd[:20000], 8), to_dev(np.full(20000, kmax(8), np.uint64), 8), 4)
    sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
    for _ in range(5):
        a = t.range(to_dev(lo1, 8), to_dev(hi, 8), 7, stream=sa)
        b = t.range(to_dev(lo2, 8), to_dev(hi, 8), 7, stream=sb)
        torch.cuda.synchronize()
        for (ok, ov, oc), lo in ((a, lo1), (b, lo2)):
            ek, ev, ec = o.range(lo, hi, 7)
            assert np.array_equal(oc.cpu().numpy().astype(np.uint32), ec)
            assert np.array_equal(from_dev(ok.reshape(-1), 8).reshape(ek.shape), ek)
            assert np.array_equal(from_dev(ov.reshape(-1), 8).reshape(ev.shape), ev)
    t.close()


def test_sharded_update_refused(hbt):
    k = gen.stratified_keys(5000, 3)
    trees = [gpu_build(hbt, k[:2500], k[:2500], 16, 8), gpu_build(hbt, k[2500:], k[2500:], 16, 8)]
    g = hbt.LocalShardGroup(trees)
    bk = to_dev(k[:10] + np.uint64(1), 8)
    with pytest.raises(hbt.HBTError) as e:
        trees[0].update(bk, bk, torch.zeros(10, dtype=torch.uint8, device="cuda"))
    assert e.value.code == hbt.EUNSUPPORTED
    comm = hbt.Comm.single()
    st = hbt.ShardedTree(comm, to_dev(k, 8), to_dev(k, 8), fanout=16)
    with pytest.raises(hbt.HBTError):
        st.update(bk, bk, torch.zeros(10, dtype=torch.uint8, device="cuda"))
    st.close()
    del g
