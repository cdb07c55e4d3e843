"""GPU parity of the REGULAR tree against the oracle: bit-exact pos|found and
value, bitwise build arrays (big leaves, counts, last-level nodes, upper pool,
chain), before and after GPU bulk updates (splits, removals, the empty tree)."""
import os

import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_util import END, GenLib, from_dev, gpu_build, gpu_search, np_dtype, to_dev
from test_oracle_implicit import gen_keys, kmax, query_set

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def hbt():
    import paper_conf_sigmod_shahvaranij16_b200 as m
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return m


def check_arrays(hbt, t, o, width):
    a = o.arrays()
    dt = np_dtype(width)
    F, P, NI, pool = a["F"], a["P"], a["NI"], a["pool"]
    nip = 32 // width
    mx = kmax(width)
    info = t.info()
    assert info["leaf_lines"] == pool and info["chain_len"] == len(a["chain"]) and info["n_distinct"] == a["n"]
    leaf = t.export(hbt.SEG_LEAF).view(dt).reshape(pool, F, 2 * P)
    ek = a["lkeys"].reshape(pool, F, P).astype(dt)
    ev = a["lvals"].reshape(pool, F, P).astype(dt)
    assert np.array_equal(leaf[:, :, :P], ek) and np.array_equal(leaf[:, :, P:], ev)
    assert np.array_equal(t.export(hbt.SEG_COUNT).view(np.uint32), a["lcount"])
    assert np.array_equal(t.export(hbt.SEG_LAST_KEYS).view(dt).reshape(pool, F), a["lsep"].astype(dt))
    lidx = t.export(hbt.SEG_LAST_IDX).view(dt).reshape(pool, nip)
    assert np.array_equal(lidx[:, :NI], a["lidx"].astype(dt)) and (lidx[:, NI:] == mx).all()
    assert np.array_equal(t.export(hbt.SEG_CHAIN).view(np.uint32), a["chain"].astype(np.uint32))
    tot = a["uoff"][-1]
    assert info["level_nodes"] == a["unodes"]
    if tot:
        assert np.array_equal(t.export(hbt.SEG_UPPER_KEYS).view(dt).reshape(tot, F), a["ukeys"].astype(dt))
        uidx = t.export(hbt.SEG_UPPER_IDX).view(dt).reshape(tot, nip)
        assert np.array_equal(uidx[:, :NI], a["uidx"].astype(dt)) and (uidx[:, NI:] == mx).all()
        assert np.array_equal(t.export(hbt.SEG_UPPER_REFS).view(np.uint32).reshape(tot, F), a["urefs"])


@pytest.mark.parametrize("width", [4, 8])
@pytest.mark.parametrize("F", [4, 8, 16, 32])
def test_regular_edge_suite_parity(hbt, width, F):
    P = 64 // (2 * width)
    rng = np.random.default_rng(300 * F + width)
    for n in sorted({0, 1, 2, P, F * P - 1, F * P, F * P + 1, 3 * F * P, F * F * P + 7, 20000}):
        k, v = gen_keys(n, width, rng, dup=(n % 2 == 1), with_max=(n % 3 == 0))
        o = oracle.RTree.from_pairs(k, v, F, width)
        t = gpu_build(hbt, k, v, F, width, layout="regular")
        check_arrays(hbt, t, o, width)
        q = query_set(k, width, rng, 3000)
        epf, ev = o.search(q)
        for ctas in (0, 1):  # launch shapes
            t.set_search_config(ctas_per_sm=ctas)
            pf, val = gpu_search(t, q, width)
            assert np.array_equal(pf, epf), (ctas, n, F, width, np.nonzero(pf != epf)[0][:5])
            assert np.array_equal(val, ev), (ctas, n, F, width)
        t.close()


@pytest.mark.parametrize("width,F", [(8, 4), (4, 8), (8, 32), (4, 32)])
def test_regular_update_parity(hbt, width, F):
    """Random UPSERT/DELETE batches: merges, even splits into appended pool
    indices, removal of emptied leaves, and finally the empty tree."""
    rng = np.random.default_rng(17 * F + width)
    mx = kmax(width)
    for trial in range(4):
        n = int(rng.integers(0, 3000))
        k, v = gen_keys(n, width, rng, dup=True)
        o = oracle.RTree.from_pairs(k, v, F, width)
        t = gpu_build(hbt, k, v, F, width, layout="regular")
        live = set(np.asarray(k, np.uint64).tolist())
        for batch in range(5):
            nops = int(rng.integers(1, 2500))
            pool = np.array(sorted(live) or [0], np.uint64)
            ok = np.where(rng.random(nops) < 0.5, pool[rng.integers(0, len(pool), nops)],
                          rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)).astype(np.uint64)
            ov = rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)
            p_del = [0.1, 0.5, 0.9, 0.3, 1.0][batch]
            op = (rng.random(nops) < p_del).astype(np.uint8)
            if batch == 4:
                ok = np.array(sorted(live) or [1], np.uint64)
                ov = np.zeros(len(ok), np.uint64)
                op = np.ones(len(ok), np.uint8)
            o.update(ok, ov, op)
            t.update(to_dev(ok, width), to_dev(ov, width), torch.from_numpy(op).cuda())
            for a_, o_ in zip(ok.tolist(), op.tolist()):
                if o_ == 0:
                    live.add(a_)
                else:
                    live.discard(a_)
            check_arrays(hbt, t, o, width)
            q = query_set(ok[:300], width, rng, 3000)
            epf, ev = o.search(q)
            pf, val = gpu_search(t, q, width)
            assert np.array_equal(pf, epf), (trial, batch)
            assert np.array_equal(val, ev), (trial, batch)
        assert t.info()["n_distinct"] == 0


def test_regular_one_leaf_absorbs_huge_batch(hbt):
    """An empty tree receiving many inserts: one leaf splits into many."""
    width, F = 8, 8
    o = oracle.RTree.from_pairs(np.zeros(0, np.uint64), np.zeros(0, np.uint64), F, width)
    t = gpu_build(hbt, np.zeros(0, np.uint64), np.zeros(0, np.uint64), F, width, layout="regular")
    rng = np.random.default_rng(5)
    ok = rng.integers(0, 2**64 - 1, 5000, dtype=np.uint64, endpoint=True)
    ov = rng.integers(0, 2**64 - 1, 5000, dtype=np.uint64, endpoint=True)
    op = np.zeros(5000, np.uint8)
    o.update(ok, ov, op)
    t.update(to_dev(ok, width), to_dev(ov, width), torch.from_numpy(op).cuda())
    check_arrays(hbt, t, o, width)
    q = query_set(ok[:500], width, rng, 2000)
    pf, val = gpu_search(t, q, width)
    epf, ev = o.search(q)
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)


def test_c3_scaled(hbt):
    """configs[2] recipe at 1/128 scale: regular u64, F = 32, uniform queries over
    [0, n + n_ins) before and after a 1 % bulk update; every output vs the oracle."""
    n = 1 << 20
    m = 1 << 19
    k, v = gen.workload_keys_values("c3", n)
    bk, bv, bo, n_ins = gen.update_batch("c3", n)
    q = gen.workload_queries("c3", k, m, n_ins=n_ins)
    o = oracle.RTree.from_pairs(k, v, 32, 8)
    t = gpu_build(hbt, k, v, 32, 8, layout="regular")
    pf, val = gpu_search(t, q, 8)
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)
    o.update(bk, bv, bo)
    t.update(to_dev(bk, 8), to_dev(bv, 8), torch.from_numpy(bo).cuda())
    check_arrays(hbt, t, o, 8)
    pf, val = gpu_search(t, q, 8)
    epf, ev = o.search(q, nthreads=oracle.default_threads())
    assert np.array_equal(pf, epf) and np.array_equal(val, ev)
