"""Generator module checks (CPU): bijectivity/distinctness, mulhi64 against
Python big integers, Knuth shuffle is a permutation, Zipf sampler against its
pmf, stratified keys sorted and distinct, update batch shape."""
import numpy as np

import gen


def test_mix64_reference_values():
    # splitmix64 finalizer from its published constants, computed with Python ints
    def ref(x):
        z = (x + 0x9E3779B97F4A7C15) & (2**64 - 1)
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & (2**64 - 1)
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & (2**64 - 1)
        return z ^ (z >> 31)
    xs = [0, 1, 2, 12345, 2**63, 2**64 - 1]
    assert gen.mix64(np.array(xs, np.uint64)).tolist() == [ref(x) for x in xs]


def test_fmix32_bijective_on_prefix():
    x = np.arange(1 << 22, dtype=np.uint32)
    assert len(np.unique(gen.fmix32(x))) == len(x)


def test_keys_distinct():
    for w in (4, 8):
        k = gen.keys(1 << 20, w, gen.stream_seed(1, gen.STREAM_K))
        assert len(np.unique(k)) == len(k)


def test_mulhi64_matches_python():
    rng = np.random.default_rng(0)
    a = rng.integers(0, 2**64 - 1, 1000, dtype=np.uint64, endpoint=True)
    b = rng.integers(0, 2**64 - 1, 1000, dtype=np.uint64, endpoint=True)
    got = gen.mulhi64(a, b).tolist()
    assert got == [(int(x) * int(y)) >> 64 for x, y in zip(a.tolist(), b.tolist())]


def test_uniform_indices_in_range():
    u = gen.uniform_indices(1 << 16, 1000, 5)
    assert u.max() < 1000
    cnt = np.bincount(u.astype(np.int64), minlength=1000)
    assert cnt.min() > 20 and cnt.max() < 120


def test_knuth_shuffle_is_permutation():
    k = gen.keys(1 << 12, 4, 3)
    s = gen.knuth_shuffle(k, 9)
    assert sorted(s.tolist()) == sorted(k.tolist()) and not np.array_equal(s, k)


def test_zipf_matches_pmf():
    n, theta, m = 1000, 0.99, 400000
    r = gen.zipf_ranks(m, n, theta, 17)
    assert r.min() >= 1 and r.max() <= n
    pmf = np.arange(1, n + 1, dtype=np.float64) ** -theta
    pmf /= pmf.sum()
    cnt = np.bincount(r, minlength=n + 1)[1:]
    # top ranks within 3 sigma of the pmf
    for k in range(10):
        e = m * pmf[k]
        assert abs(cnt[k] - e) < 4 * np.sqrt(e), (k, cnt[k], e)
    # deterministic given the seed
    assert np.array_equal(r[:1000], gen.zipf_ranks(1000, n, theta, 17))


def test_stratified_sorted_distinct():
    k = gen.stratified_keys(1 << 16, 11)
    assert np.all(k[1:] > k[:-1])
    k2 = gen.stratified_keys(100, 11, start=1 << 16)
    assert k2[0] > k[-1]


def test_update_batch_shape():
    n = 1 << 14
    bk, bv, bo, n_ins = gen.update_batch("c3", n, n_ops=200)
    assert len(bk) == 200 and (bo == 0).sum() == n_ins == 100
    base = set(gen.keys(n, 8, gen.stream_seed(3, gen.STREAM_K)).tolist())
    ins = bk[bo == 0].tolist()
    dels = bk[bo == 1].tolist()
    assert not (set(ins) & base) and set(dels) <= base and len(set(dels)) == len(dels)


def test_skew_values_moments():
    """The paper's skewed query distributions before the [0, MAX] mapping."""
    m = 200000
    mx = float(2**64 - 1)
    x = gen.skew_values("normal", m, 8, 5).astype(np.float64) / mx
    assert abs(x.mean() - 0.5) < 0.01 and abs(x.std() - 0.304) < 0.01  # sigma 0.354 clipped to [0, 1]: 0.304
    g = gen.skew_values("gamma", m, 8, 6).astype(np.float64) / mx
    assert abs(g.mean() - 9.0 / 30.0) < 0.01                          # E[Gamma(3,3)] = 9
    z = gen.skew_values("zipf", m, 8, 7, n_ranks=1 << 20).astype(np.float64) / mx
    assert (z == 0).mean() > 0.55                                     # rank 1 has p = 1/zeta(2) = 0.61
    u = gen.skew_values("uniform", m, 4, 8)
    assert u.dtype == np.uint32 and abs(u.astype(np.float64).mean() / (2**32 - 1) - 0.5) < 0.01
    assert np.array_equal(gen.skew_values("normal", 100, 8, 5), gen.skew_values("normal", 100, 8, 5))
