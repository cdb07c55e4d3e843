"""GPU parity with the L-segment in pinned HOST memory (hbt_set_leaf_placement, the
paper's I-segment-on-GPU / L-segment-in-host split; SURVEY 8(f)
f4): every search mode, the bucketed search, range scans and rebuilding updates must
give the oracle's results with the leaf lines read by zero-copy loads, and the
placement must survive an update and move back to HBM."""
import numpy as np
import pytest
import torch

import oracle
from gpu_util import from_dev, gpu_build, gpu_search, to_dev
from test_gpu_implicit import expected_implicit_bytes
from test_gpu_range import check as range_check, ranges
from test_oracle_implicit import gen_keys, query_set

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def hbt():
    import paper_conf_sigmod_shahvaranij16_b200 as m
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return m


@pytest.mark.parametrize("width,F", [(8, 16), (4, 8), (8, 32), (4, 4)])
def test_host_leaves_search_modes(hbt, width, F):
    rng = np.random.default_rng(31 * F + width)
    P = 64 // (2 * width)
    for n in [0, 1, P + 1, F * P + 1, 5000, 300000]:
        k, v = gen_keys(n, width, rng, dup=(n % 2 == 1), with_max=(n % 3 == 0))
        o = oracle.ITree.from_pairs(k, v, F, width)
        t = gpu_build(hbt, k, v, F, width)
        t.set_leaf_placement("host")
        assert t.leaf_placement == "host"
        inner, leaf = expected_implicit_bytes(o, width)
        assert t.export(hbt.SEG_LEAF).tobytes() == leaf  # the copy is bitwise the build
        q = query_set(k, width, rng, 20000)
        epf, ev = o.search(q)
        for mode, l2b in ((2, 0), (2, 1), (3, 0), (3, 1)):
            t.set_search_config(smem_mode=mode)
            t.set_param("l2_levels_bytes", l2b)
            t.set_param("small_batch", 0)
            pf, val = gpu_search(t, q, width)
            assert np.array_equal(pf, epf), (n, mode, l2b)
            assert np.array_equal(val, ev), (n, mode, l2b)
        t.set_search_config(smem_mode=2)
        # streamed slices: many small buckets, the 1024-bucket cap, and auto
        for ls, slice_ in ((1, 4096), (1, 64), (1, 0), (2, 0)):
            t.set_param("leaf_stream", ls)
            t.set_param("stream_slice", slice_)
            pf, val = gpu_search(t, q, width)
            assert np.array_equal(pf, epf) and np.array_equal(val, ev), (n, ls, slice_)
        t.set_param("leaf_stream", 0)
        t.set_param("bucket", 1)  # bucketed search (splitters and item directory read the host leaves)
        pf, val = gpu_search(t, q, width)
        assert np.array_equal(pf, epf) and np.array_equal(val, ev), n
        t.set_param("bucket", 2)
        t.set_leaf_placement("device")
        assert t.leaf_placement == "device"
        assert t.export(hbt.SEG_LEAF).tobytes() == leaf
        pf, val = gpu_search(t, q, width)
        assert np.array_equal(pf, epf) and np.array_equal(val, ev), n
        t.close()


@pytest.mark.parametrize("width", [4, 8])
def test_host_leaves_update_and_range(hbt, width):
    rng = np.random.default_rng(5 + width)
    F = 8
    k, v = gen_keys(20000, width, rng, dup=True)
    o = oracle.ITree.from_pairs(k, v, F, width)
    t = gpu_build(hbt, k, v, F, width)
    t.set_leaf_placement("host")
    mx = (1 << (8 * width)) - 1
    for _ in range(3):
        nops = 3000
        ok = np.where(rng.random(nops) < 0.5, k[rng.integers(0, len(k), nops)],
                      rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)).astype(np.uint64)
        ov = rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)
        op = (rng.random(nops) < 0.4).astype(np.uint8)
        o = o.update(ok, ov, op)
        t.update(to_dev(ok, width), to_dev(ov, width), torch.from_numpy(op).cuda())
        assert t.leaf_placement == "host"  # the rebuild keeps the placement
        inner, leaf = expected_implicit_bytes(o, width)
        assert t.export(hbt.SEG_INNER).tobytes() == inner
        assert t.export(hbt.SEG_LEAF).tobytes() == leaf
        q = query_set(ok[:500], width, rng, 4000)
        epf, ev = o.search(q)
        for ls in (0, 1):
            t.set_param("leaf_stream", ls)
            t.set_param("stream_slice", 2048)
            pf, val = gpu_search(t, q, width)
            assert np.array_equal(pf, epf) and np.array_equal(val, ev), ls
    Kd, _ = oracle.dedupe(k, v)
    lo, hi = ranges(Kd, width, rng, 500)
    for kk in (1, 9, 40):
        range_check(t, o, lo, hi, kk, width)
    t.close()


@pytest.mark.parametrize("width,F", [(8, 32), (4, 8)])
def test_host_leaves_regular(hbt, width, F):
    """Regular tree with its big-leaf pool in host memory: searches (both kernels and
    the bucketed item search), updates that split leaves and grow the pool (which
    stays in host memory), range scans, and the way back to HBM."""
    rng = np.random.default_rng(11 * F + width)
    k, v = gen_keys(30000, width, rng, dup=True)
    o = oracle.RTree.from_pairs(k, v, F, width)
    t = gpu_build(hbt, k, v, F, width, layout="regular")
    t.set_leaf_placement("host")
    assert t.leaf_placement == "host"
    mx = (1 << (8 * width)) - 1
    for rep in range(3):
        q = query_set(k, width, rng, 20000)
        epf, ev = o.search(q)
        for mode, bucket in ((2, 0), (3, 0), (2, 1)):
            t.set_search_config(smem_mode=mode)
            t.set_param("bucket", bucket)
            pf, val = gpu_search(t, q, width)
            assert np.array_equal(pf, epf) and np.array_equal(val, ev), (rep, mode, bucket)
        t.set_param("bucket", 2)
        nops = 20000  # mostly inserts of fresh keys: big leaves split, the pool grows
        ok = rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)
        ok[:3000] = k[rng.integers(0, len(k), 3000)]
        ov = rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)
        op = (rng.random(nops) < 0.1).astype(np.uint8)
        o.update(ok, ov, op)  # the oracle's regular tree updates in place
        t.update(to_dev(ok, width), to_dev(ov, width), torch.from_numpy(op).cuda())
        assert t.leaf_placement == "host"
        k = np.concatenate([k, ok])
    q = query_set(k, width, rng, 20000)
    epf, ev = o.search(q)
    pf, val = gpu_search(t, q, width)
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)
    Kd, _ = oracle.dedupe(k, np.zeros(len(k), np.uint64))
    lo, hi = ranges(Kd, width, rng, 300)
    for kk in (1, 20):
        range_check(t, o, lo, hi, kk, width)
    t.set_leaf_placement("device")
    pf, val = gpu_search(t, q, width)
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)
    t.close()


def test_host_leaves_streamed_through_host_pipeline(hbt):
    """hbt_search_host (host buffers, chunked over two streams) on a tree whose
    L-segment streams from host memory: the streamed search runs inside the host
    pipeline's chunks (its own lock; a shared one deadlocked)."""
    width, F = 8, 16
    rng = np.random.default_rng(77)
    k, v = gen_keys(300000, width, rng)
    o = oracle.ITree.from_pairs(k, v, F, width)
    t = gpu_build(hbt, k, v, F, width)
    t.set_leaf_placement("host")
    t.set_param("stream_slice", 65536)  # many buckets; auto mode streams this batch
    q = query_set(k, width, rng, 1 << 20)
    hp = np.empty(len(q), np.uint64)
    hv = np.empty(len(q), np.uint64)
    t.search_host(np.ascontiguousarray(q), hp, hv)
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    assert np.array_equal(hp, epf) and np.array_equal(hv, ev)
    t.close()
