"""Randomised GPU parity: many small trees, each with a random form, key width,
fanout, size (duplicates, MAX as a real key, empty), query mix (hits, misses, 0,
MAX, neighbours of keys) and a random combination of the search knobs (top-level
mode, per-level read widths, CTA size, bucketing with its slice / item directory /
capacity, L-segment placement and streaming), every output compared with the
oracle.  Complements the targeted suites: a knob interaction no suite lists still
has to give the oracle's bits.  Seeded, so a failure reproduces."""
import os

import numpy as np
import pytest
import torch

import oracle
from gpu_util import gpu_build, gpu_search
from test_oracle_implicit import gen_keys, kmax, query_set

pytestmark = pytest.mark.gpu

# HBT_FUZZ_CASES / HBT_FUZZ_SEED widen the sweep for long runs (the defaults are the suite's)
CASES = int(os.environ.get("HBT_FUZZ_CASES", "600"))
SEED0 = int(os.environ.get("HBT_FUZZ_SEED", "7000"))


@pytest.fixture(scope="module")
def hbt():
    import paper_conf_sigmod_shahvaranij16_b200 as m
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return m


def _queries(k, width, rng, m):
    q = query_set(k, width, rng, m)
    if len(k):
        kk = k[rng.integers(0, len(k), min(m, 64))].astype(object)
        mx = kmax(width)
        nb = np.array([min(mx, int(x) + 1) for x in kk] + [max(0, int(x) - 1) for x in kk], dtype=np.uint64)
        q = np.concatenate([q, nb, np.array([0, kmax(width)], dtype=np.uint64)])
    return q


@pytest.mark.parametrize("case", range(CASES))
def test_random_knob_parity(hbt, case):
    rng = np.random.default_rng(SEED0 + case)
    layout = "regular" if rng.random() < 0.4 else "implicit"
    width = int(rng.choice([4, 8]))
    F = int(rng.choice([4, 8, 16, 32]))
    n = int(rng.choice([0, 1, 2, 3, 7, 17, 64, 65, 500, 4097, 20000, 70000]))
    k, v = gen_keys(n, width, rng, dup=bool(rng.random() < 0.5), with_max=bool(rng.random() < 0.3))
    o = (oracle.ITree if layout == "implicit" else oracle.RTree).from_pairs(k, v, F, width)
    t = gpu_build(hbt, k, v, F, width, layout=layout)
    knobs = {}
    if layout == "implicit":
        knobs["smem_mode"] = int(rng.choice([2, 3]))
        knobs["l2_levels_bytes"] = int(rng.choice([0, 1, 4096]))
        knobs["full256"] = int(rng.integers(0, 2))
        knobs["small_batch"] = int(rng.choice([0, 1 << 16]))
        knobs["ctas_per_sm"] = int(rng.choice([0, 1, 2]))
    knobs["leaf256"] = int(rng.integers(0, 2))
    knobs["bucket"] = int(rng.choice([0, 1, 2]))
    if knobs["bucket"]:
        knobs["bucket_slice"] = int(rng.choice([1, 4096, 1 << 16, 1 << 20]))
        knobs["bucket_items"] = int(rng.integers(0, 2))
        knobs["bucket_cap"] = int(rng.choice([0, 0, 7]))
    host = bool(rng.random() < 0.25)
    if host:
        t.set_leaf_placement("host")
        if layout == "implicit":
            knobs["leaf_stream"] = int(rng.choice([0, 1, 2]))
            knobs["stream_slice"] = int(rng.choice([64, 4096, 0]))
    # L2 eviction-priority hints (own generator: the cases above keep their draws)
    hrng = np.random.default_rng(SEED0 + case + 777)
    knobs["l2_hint"] = int(hrng.integers(0, 5))
    knobs["item_l2_hint"] = int(hrng.integers(0, 4))
    knobs["item_rounds"] = int(hrng.choice([0, 1, 3, 16]))
    knobs["item_qpf"] = int(hrng.choice([0, 1, 2]))
    knobs["item_cnode"] = int(hrng.choice([0, 1, 2]))
    for name, val in knobs.items():
        t.set_param(name, val)
    q = _queries(k, width, rng, int(rng.choice([1, 31, 1000, 40000])))
    epf, ev = o.search(q)
    pf, val = gpu_search(t, q, width)
    assert np.array_equal(pf, epf), (layout, width, F, n, host, knobs, np.nonzero(pf != epf)[0][:5])
    assert np.array_equal(val, ev), (layout, width, F, n, host, knobs)
    t.close()


@pytest.mark.parametrize("case", range(150))
def test_random_update_sequences(hbt, case):
    """Random UPSERT / DELETE batches (splits, removals, emptying the tree, MAX keys)
    on both forms, searched after every batch with random knobs."""
    import torch as _t
    from gpu_util import to_dev
    rng = np.random.default_rng(9100 + case)
    layout = "regular" if rng.random() < 0.6 else "implicit"
    width = int(rng.choice([4, 8]))
    F = int(rng.choice([4, 8, 16, 32]))
    n = int(rng.choice([0, 1, 9, 300, 5000, 30000]))
    k, v = gen_keys(n, width, rng, dup=bool(rng.random() < 0.5), with_max=bool(rng.random() < 0.3))
    o = (oracle.ITree if layout == "implicit" else oracle.RTree).from_pairs(k, v, F, width)
    t = gpu_build(hbt, k, v, F, width, layout=layout)
    if rng.random() < 0.2:
        t.set_leaf_placement("host")
    mx = kmax(width)
    live = k.copy()
    for b in range(3):
        nops = int(rng.choice([1, 50, 2000, 12000]))
        pool = live if len(live) else np.zeros(1, np.uint64)
        ok = np.where(rng.random(nops) < 0.5, pool[rng.integers(0, len(pool), nops)],
                      rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)).astype(np.uint64)
        if rng.random() < 0.2:
            ok[: nops // 3] = mx
        ov = rng.integers(0, mx, nops, dtype=np.uint64, endpoint=True)
        pdel = float(rng.choice([0.0, 0.3, 0.9, 1.0]))
        op = (rng.random(nops) < pdel).astype(np.uint8)
        r = o.update(ok, ov, op)
        if layout == "implicit":
            o = r
        t.update(to_dev(ok, width), to_dev(ov, width), _t.from_numpy(op).cuda())
        live = np.concatenate([live, ok])
        t.set_param("bucket", int(rng.choice([0, 1, 2])))
        t.set_param("bucket_slice", int(rng.choice([1, 4096, 1 << 20])))
        q = _queries(live, width, rng, int(rng.choice([100, 5000])))
        epf, ev = o.search(q)
        pf, val = gpu_search(t, q, width)
        assert np.array_equal(pf, epf), (layout, width, F, n, b, np.nonzero(pf != epf)[0][:5])
        assert np.array_equal(val, ev), (layout, width, F, n, b)
    t.close()
