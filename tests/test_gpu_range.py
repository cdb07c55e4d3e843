"""GPU parity of hbt_range (range scans, PAPER.md:89 / P:392) against the
oracle's range scan, for both tree forms, k across warp-chunk boundaries, and
for the regular tree after updates that split and remove big leaves."""
import numpy as np
import pytest
import torch

import oracle
from gpu_util import from_dev, gpu_build, to_dev
from test_oracle_implicit import gen_keys, kmax, query_set

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def hbt():
    import paper_conf_sigmod_shahvaranij16_b200 as m
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    return m


def ranges(Kd, width, rng, n):
    mx = kmax(width)
    lo = query_set(Kd[:300], width, rng, n)
    span = rng.integers(0, max(1, mx // 300), len(lo), dtype=np.uint64)
    hi = np.minimum(lo.astype(object) + span.astype(object), mx).astype(np.uint64)
    hi[::17] = mx
    return lo, hi


def check(t, o, lo, hi, k, width):
    ok, ov, oc = t.range(to_dev(lo, width), to_dev(hi, width), k)
    torch.cuda.synchronize()
    ek, ev, ec = o.range(lo, hi, k)
    assert np.array_equal(oc.cpu().numpy().astype(np.uint32), ec)
    assert np.array_equal(from_dev(ok.reshape(-1), width).reshape(ek.shape), ek)
    assert np.array_equal(from_dev(ov.reshape(-1), width).reshape(ev.shape), ev)


@pytest.mark.parametrize("layout", ["implicit", "regular"])
@pytest.mark.parametrize("width,F", [(8, 16), (4, 8), (8, 32), (4, 32)])
def test_range_parity(hbt, layout, width, F):
    rng = np.random.default_rng(F + width + (layout == "regular"))
    for n in [0, 1, 7, 5000]:
        k, v = gen_keys(n, width, rng, dup=True)
        T = oracle.ITree if layout == "implicit" else oracle.RTree
        o = T.from_pairs(k, v, F, width)
        t = gpu_build(hbt, k, v, F, width, layout=layout)
        Kd, _ = oracle.dedupe(k, v)
        lo, hi = ranges(Kd if len(Kd) else np.zeros(1, np.uint64), width, rng, 500)
        for kk in (1, 5, 32, 33, 100):
            check(t, o, lo, hi, kk, width)


@pytest.mark.parametrize("width", [4, 8])
def test_range_regular_after_updates(hbt, width):
    rng = np.random.default_rng(9 + width)
    mx = kmax(width)
    k, v = gen_keys(4000, width, rng)
    o = oracle.RTree.from_pairs(k, v, 4, width)
    t = gpu_build(hbt, k, v, 4, width, layout="regular")
    for _ in range(3):
        ins = rng.integers(0, mx, 3000, dtype=np.uint64, endpoint=True)
        dels = k[rng.integers(0, len(k), 1500)]
        ok = np.concatenate([ins, dels])
        ov = rng.integers(0, mx, len(ok), dtype=np.uint64, endpoint=True)
        op = np.concatenate([np.zeros(len(ins), np.uint8), np.ones(len(dels), np.uint8)])
        o.update(ok, ov, op)
        t.update(to_dev(ok, width), to_dev(ov, width), torch.from_numpy(op).cuda())
        lo, hi = ranges(np.sort(ins), width, rng, 800)
        for kk in (3, 32, 70):
            check(t, o, lo, hi, kk, width)
