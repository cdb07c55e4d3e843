"""Seeded synthetic workload generators shared by the oracle side (tests, bench
cpu_baseline) and the CUDA side (bench, parity tests).

This module holds NO arithmetic of the method (no sorting, no tree, no search):
only counter-based random streams, so that every rank, the oracle and the GPU
path can regenerate identical inputs.  The recipes follow the paper's workload
(§6.1 "keys and values are randomly generated according to a
uniform distribution on [0 - MAX] ... randomly permuted the pairs using the Knuth
shuffle") and SURVEY.md §8(d) "Generators":

* mix64   = splitmix64 finalizer (bijection on 2^64)
* fmix32  = murmur3 finalizer   (bijection on 2^32)
* keys    K_i = mixS(i ^ seed_k)            -> distinct by construction
* values  V_i = mixS(i ^ seed_v)
* uniform hit queries q_j = K[mulhi64(mix64(j ^ seed_q), n)]   (Lemire)
* Knuth/Fisher-Yates shuffle driven by mix64(j ^ seed_q)
* Zipf(theta) ranks by rejection-inversion (Hormann & Derflinger), scrambled
  through the key order: q = K[rank-1]
* stratified keys K_i = (i << 33) | (mix64(i ^ seed_k) & (2^33-1)) (c4)

The device-side twin of the integer streams is gen/gen.cu (libhbtgen.so); the
GPU test suite checks both produce identical arrays.
"""
from __future__ import annotations

import numpy as np

M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
BASE_SEED = 20160626
STREAM_K, STREAM_V, STREAM_Q, STREAM_OP = 1, 2, 3, 4


def _u64(x):
    return np.asarray(x, dtype=np.uint64)


def mix64(x):
    """splitmix64 finalizer: z += golden; z = (z^(z>>30))*C1; z = (z^(z>>27))*C2; z ^= z>>31."""
    with np.errstate(over="ignore"):
        z = _u64(x) + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def fmix32(x):
    """murmur3 fmix32 on uint32 arrays (bijection on 2^32)."""
    with np.errstate(over="ignore"):
        h = np.asarray(x, dtype=np.uint32)
        h = h ^ (h >> np.uint32(16))
        h = h * np.uint32(0x85EBCA6B)
        h = h ^ (h >> np.uint32(13))
        h = h * np.uint32(0xC2B2AE35)
        h = h ^ (h >> np.uint32(16))
    return h


def stream_seed(cfg: int, stream: int) -> int:
    """Per-config, per-stream 64-bit seed: mix64((20160626 + 1000*cfg) * 8 + stream)."""
    return int(mix64(np.uint64((BASE_SEED + 1000 * cfg) * 8 + stream)))


def mulhi64(a, b):
    """High 64 bits of the 128-bit product a*b (element-wise, uint64)."""
    a = _u64(a)
    b = _u64(b)
    m32 = np.uint64(0xFFFFFFFF)
    s32 = np.uint64(32)
    with np.errstate(over="ignore"):
        a_lo, a_hi = a & m32, a >> s32
        b_lo, b_hi = b & m32, b >> s32
        ll = a_lo * b_lo
        lh = a_lo * b_hi
        hl = a_hi * b_lo
        hh = a_hi * b_hi
        mid = (ll >> s32) + (lh & m32) + (hl & m32)
        return hh + (lh >> s32) + (hl >> s32) + (mid >> s32)


def dtype_of(width: int):
    if width == 4:
        return np.uint32
    if width == 8:
        return np.uint64
    raise ValueError("width must be 4 or 8")


def mix_stream(idx, seed: int, width: int):
    """K_i = mixS(i ^ seed): mix64 for width 8, fmix32 on the low 32 bits for width 4."""
    idx = _u64(idx)
    if width == 8:
        return mix64(idx ^ np.uint64(seed))
    x = (idx ^ np.uint64(seed)).astype(np.uint32)
    return fmix32(x)


def keys(n: int, width: int, seed: int, start: int = 0):
    """Distinct uniform-looking keys K_start..K_{start+n-1}."""
    return mix_stream(np.arange(start, start + n, dtype=np.uint64), seed, width)


def values(n: int, width: int, seed: int, start: int = 0):
    return mix_stream(np.arange(start, start + n, dtype=np.uint64), seed, width)


def uniform_indices(m: int, n: int, seed: int, start: int = 0):
    """u_j = mulhi64(mix64(j ^ seed), n): uniform over [0, n) with replacement."""
    j = np.arange(start, start + m, dtype=np.uint64)
    return mulhi64(mix64(j ^ np.uint64(seed)), np.uint64(n))


def uniform_hit_queries(key_arr, m: int, seed: int, start: int = 0):
    return key_arr[uniform_indices(m, len(key_arr), seed, start).astype(np.int64)]


def knuth_shuffle(arr, seed: int):
    """Fisher-Yates (Knuth) shuffle; swap index mulhi64(mix64(j^seed), j+1)."""
    a = np.array(arr, copy=True)
    n = len(a)
    if n < 2:
        return a
    js = np.arange(n - 1, 0, -1, dtype=np.uint64)
    rs = mulhi64(mix64(js ^ np.uint64(seed)), js + np.uint64(1)).astype(np.int64)
    for j, r in zip(js.astype(np.int64).tolist(), rs.tolist()):
        a[j], a[r] = a[r], a[j]
    return a


def unit_doubles(counter, seed: int):
    """Uniform doubles in [0,1) from a counter: (mix64(mix64(counter ^ seed)) >> 11) * 2^-53."""
    z = mix64(mix64(_u64(counter) ^ np.uint64(seed)))
    return (z >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


def zipf_ranks(m: int, n: int, theta: float, seed: int, start: int = 0):
    """Zipf(theta) ranks in [1, n] by rejection-inversion sampling
    (Hormann & Derflinger 1996), vectorised; sample j, attempt a draws the
    uniform unit_doubles(j + a * 2^40, seed).  Exact for the Zipf pmf
    p(k) ~ k^-theta on 1..n."""
    e = float(theta)

    def h(x):
        return np.exp(-e * np.log(x))

    def helper1(x):
        x = np.asarray(x, dtype=np.float64)
        out = np.ones_like(x)
        nz = np.abs(x) > 1e-8
        out[nz] = np.log1p(x[nz]) / x[nz]
        out[~nz] = 1.0 - x[~nz] * (0.5 - x[~nz] * (1.0 / 3.0 - 0.25 * x[~nz]))
        return out

    def helper2(x):
        x = np.asarray(x, dtype=np.float64)
        out = np.ones_like(x)
        nz = np.abs(x) > 1e-8
        out[nz] = np.expm1(x[nz]) / x[nz]
        out[~nz] = 1.0 + x[~nz] * 0.5 * (1.0 + x[~nz] * (1.0 / 3.0) * (1.0 + 0.25 * x[~nz]))
        return out

    def h_integral(x):
        lx = np.log(np.asarray(x, dtype=np.float64))
        return helper2((1.0 - e) * lx) * lx

    def h_integral_inv(x):
        t = np.asarray(x, dtype=np.float64) * (1.0 - e)
        t = np.maximum(t, -1.0)
        return np.exp(helper1(t) * x)

    hx1 = float(h_integral(np.array([1.5]))[0]) - 1.0
    hn = float(h_integral(np.array([n + 0.5]))[0])
    s = 2.0 - float(h_integral_inv(np.array([float(h_integral(np.array([2.5]))[0]) - float(h(2.0))]))[0])

    out = np.zeros(m, dtype=np.int64)
    pending = np.arange(m, dtype=np.int64)
    attempt = 0
    while pending.size:
        ctr = (pending + start).astype(np.uint64) + np.uint64(attempt) * np.uint64(1 << 40)
        u = hn + unit_doubles(ctr, seed) * (hx1 - hn)
        x = h_integral_inv(u)
        k = np.floor(x + 0.5).astype(np.int64)
        k = np.clip(k, 1, n)
        kf = k.astype(np.float64)
        ok = ((kf - x) <= s) | (u >= h_integral(kf + 0.5) - h(kf))
        out[pending[ok]] = k[ok]
        pending = pending[~ok]
        attempt += 1
    return out


def skew_values(kind: str, m: int, width: int, seed: int, n_ranks: int = 1 << 20, start: int = 0):
    """Query VALUES drawn from the paper's skewed distributions on [0, 1] and
    mapped linearly to [0, MAX] (reading R15/R20 in DESIGN.md):
      normal  N(mu = 0.5, sigma^2 = 0.125) (Box-Muller), clipped to [0, 1]
      gamma   Gamma(k = 3, theta = 3) = -3 ln(u1 u2 u3), divided by 30, clipped to [0, 1]
      zipf    Zipf(alpha = 2) rank r in [1, n_ranks] -> (r - 1) / n_ranks  (clustered at 0)
      uniform u
    Counter-based: sample j draws unit_doubles(3j + t, seed) for t = 0, 1, 2."""
    j = np.arange(start, start + m, dtype=np.uint64) * np.uint64(3)
    u1 = unit_doubles(j, seed)
    u2 = unit_doubles(j + np.uint64(1), seed)
    u3 = unit_doubles(j + np.uint64(2), seed)
    if kind == "normal":
        x = 0.5 + np.sqrt(0.125) * np.sqrt(-2.0 * np.log1p(-u1)) * np.cos(2.0 * np.pi * u2)
    elif kind == "gamma":
        x = -3.0 * (np.log1p(-u1) + np.log1p(-u2) + np.log1p(-u3)) / 30.0
    elif kind == "zipf":
        x = (zipf_ranks(m, n_ranks, 2.0, seed, start) - 1).astype(np.float64) / n_ranks
    elif kind == "uniform":
        x = u1
    else:
        raise ValueError(kind)
    x = np.clip(x, 0.0, 1.0)
    mx = float((1 << (8 * width)) - 1)
    # x * MAX in float64, then exact integer conversion (values >= 2^63 via the high half)
    v = x * mx
    with np.errstate(over="ignore", invalid="ignore"):
        out = np.where(v >= 2.0 ** 63, (np.minimum(v, 2.0 ** 64 - 4096.0) - 2.0 ** 63).astype(np.uint64)
                       + np.uint64(1 << 63), np.minimum(v, 2.0 ** 63 - 1).astype(np.uint64))
    out = np.where(x >= 1.0, np.uint64((1 << (8 * width)) - 1), out)  # x = 1 maps to MAX exactly
    return out.astype(dtype_of(width))


def stratified_keys(n: int, seed: int, start: int = 0):
    """c4: K_i = (i << 33) | (mix64(i ^ seed) & (2^33-1)); sorted and distinct for i < 2^31."""
    i = np.arange(start, start + n, dtype=np.uint64)
    return (i << np.uint64(33)) | (mix64(i ^ np.uint64(seed)) & np.uint64((1 << 33) - 1))


def affine_perm(t, nbits: int):
    """A bijection on [0, 2^nbits): (t * 0x9E3779B1 + 0x7F4A7C15) mod 2^nbits (odd multiplier)."""
    mask = np.uint64((1 << nbits) - 1)
    with np.errstate(over="ignore"):
        return (_u64(t) * np.uint64(0x9E3779B1) + np.uint64(0x7F4A7C15)) & mask


# ----------------------------------------------------------------------------
# Workload recipes per BASELINE.json config (SURVEY §8(d) "Per-config inputs")
# ----------------------------------------------------------------------------

CONFIGS = {
    # name: (cfg id, layout, width, fanout, log2 n, log2 m, query kind)
    "c1": dict(cfg=1, layout="implicit", width=4, fanout=8, n=1 << 16, m=1 << 16, queries="shuffle"),
    "c2": dict(cfg=2, layout="implicit", width=8, fanout=16, n=1 << 23, m=1 << 24, queries="uniform"),
    "c3": dict(cfg=3, layout="regular", width=8, fanout=32, n=1 << 27, m=1 << 26, queries="uniform_ins",
               update_frac=0.01),
    "c4": dict(cfg=4, layout="implicit", width=8, fanout=16, n=1 << 31, m=1 << 28, queries="stratified"),
    "c5": dict(cfg=5, layout="implicit", width=8, fanout=16, n=1 << 27, m=1 << 26, queries="zipf", theta=0.99),
}


def workload_keys_values(name: str, n: int | None = None):
    c = CONFIGS[name]
    n = c["n"] if n is None else n
    w = c["width"]
    if name == "c4":
        k = stratified_keys(n, stream_seed(c["cfg"], STREAM_K))
    else:
        k = keys(n, w, stream_seed(c["cfg"], STREAM_K))
    v = values(n, w, stream_seed(c["cfg"], STREAM_V))
    return k, v


def workload_queries(name: str, key_arr, m: int | None = None, start: int = 0, n_ins: int = 0):
    """Queries for a config; key_arr are the generated (unsorted) keys K_0..K_{n-1}."""
    c = CONFIGS[name]
    m = c["m"] if m is None else m
    sq = stream_seed(c["cfg"], STREAM_Q)
    kind = c["queries"]
    if kind == "shuffle":
        return knuth_shuffle(key_arr, sq)[:m]
    if kind in ("uniform", "stratified"):
        return uniform_hit_queries(key_arr, m, sq, start)
    if kind == "uniform_ins":
        # index space [0, n + n_ins): u >= n are fresh keys (misses before the update)
        n = len(key_arr)
        u = uniform_indices(m, n + n_ins, sq, start).astype(np.int64)
        out = np.empty(m, dtype=key_arr.dtype)
        hit = u < n
        out[hit] = key_arr[u[hit]]
        if (~hit).any():
            out[~hit] = mix_stream(u[~hit].astype(np.uint64), stream_seed(c["cfg"], STREAM_K), c["width"])
        return out
    if kind == "zipf":
        r = zipf_ranks(m, len(key_arr), c["theta"], sq, start)
        return key_arr[r - 1]
    raise ValueError(kind)


def update_batch(name: str, n: int, n_ops: int | None = None):
    """c3 bulk update: half UPSERTs of fresh keys K_n.., half DELETEs
    of K_{pi(t)}, shuffled by mix64 order.  Returns (keys, values, ops u8: 0=UPSERT 1=DELETE)."""
    c = CONFIGS[name]
    w = c["width"]
    if n_ops is None:
        n_ops = int(c.get("update_frac", 0.01) * n)
    n_ins = (n_ops + 1) // 2
    n_del = n_ops - n_ins
    sk = stream_seed(c["cfg"], STREAM_K)
    sv = stream_seed(c["cfg"], STREAM_V)
    sop = stream_seed(c["cfg"], STREAM_OP)
    ins_k = keys(n_ins, w, sk, start=n)
    ins_v = values(n_ins, w, sv ^ 0x5555, start=n)
    nbits = max(1, int(np.ceil(np.log2(max(n, 2)))))
    t = np.arange(n_del, dtype=np.uint64)
    idx = affine_perm(t, nbits)
    # restrict to [0, n): walk the permutation cycle (cycle-walking keeps it a bijection)
    while True:
        bad = idx >= np.uint64(n)
        if not bad.any():
            break
        idx[bad] = affine_perm(idx[bad], nbits)
    del_k = mix_stream(idx, sk, w)
    del_v = np.zeros(n_del, dtype=dtype_of(w))
    bk = np.concatenate([ins_k, del_k])
    bv = np.concatenate([ins_v, del_v])
    bo = np.concatenate([np.zeros(n_ins, np.uint8), np.ones(n_del, np.uint8)])
    order = np.argsort(mix64(np.arange(n_ops, dtype=np.uint64) ^ np.uint64(sop)), kind="stable")
    return bk[order], bv[order], bo[order], n_ins
