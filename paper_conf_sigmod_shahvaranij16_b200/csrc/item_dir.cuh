// item_dir.cuh — the per-item prefix table of the bucket-local directory
// (ItemDir, bucketed.cu).  After a work item has staged the sorted maxima
// s_M[0, cnt) of its unit range, one table of 2^kPrefixBits + 1 lower bounds
// over evenly spaced keys of [s_M[0], s_M[cnt-1]] narrows every query's lower
// bound to a short slice, so a query costs one table read plus a few probes
// instead of log2(cnt) bank-conflicted probes (ncu, profiles/r01_items_*: the
// LSU pipe was 86-88 % busy, 60-70 % of it shared-memory bank conflicts).
#pragma once

#include <stdint.h>

namespace hbt {

constexpr uint32_t kPrefixBits = 10;

// Warp rounds per work item of the bucketed item searches: 16 (staging the item's
// directory is amortised over 16 K queries), fewer when the batch would leave SMs
// idle (a 2^18-query c3 batch ran its 16 items on 16 SMs: 0.18 ms of search).
inline uint32_t item_rounds(uint64_t m, uint32_t sms, uint32_t threads, uint32_t cap = 16) {
  const uint64_t per_sm = (m + uint64_t(sms) * threads - 1) / (uint64_t(sms) * threads);
  return uint32_t(per_sm < 1 ? 1 : (per_sm > cap ? cap : per_sm));
}

// One thread asks the TMA unit to pull a contiguous byte range into the L2
// (cp.async.bulk.prefetch.L2, sm_90+): the bucket count pass prefetches its next
// chunk's queries this way (c3 count 0.167 -> 0.158 ms).  Only whole 16 B units inside
// the range are requested, in pieces of <= 64 KB.
__device__ __forceinline__ void prefetch_l2_range(const void* p, uint64_t bytes) {
  const uint64_t a = reinterpret_cast<uint64_t>(p);
  const uint64_t a0 = (a + 15) & ~uint64_t(15);
  const uint64_t a1 = (a + bytes) & ~uint64_t(15);
  for (uint64_t x = a0; x < a1; x += 65536) {
    const uint32_t n = uint32_t(a1 - x < 65536 ? a1 - x : 65536);
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(x), "r"(n) : "memory");
  }
}

template <typename K>
__device__ __forceinline__ uint32_t lb_range(const K* s, uint32_t lo, uint32_t hi, K q) {
  uint32_t len = hi - lo;
  while (len > 0) {
    const uint32_t half = len >> 1;
    if (s[lo + half] < q) { lo += half + 1; len -= half + 1; } else { len = half; }
  }
  return lo;
}

template <typename K>
struct PrefixTab {
  K lo, span;
  uint32_t sh;
};

// Builds s_T[p] = #{s_M < lo + p * 2^sh} for p in [0, 2^PB] (cnt past the range; PB <= 12);
// (span >> sh) < 2^PB.  Caller synchronises before use.
template <typename K>
__device__ __forceinline__ PrefixTab<K> build_prefix(const K* s_M, uint32_t cnt, uint32_t* s_T, uint32_t threads,
                                                     uint32_t PB = kPrefixBits) {
  PrefixTab<K> pt;
  pt.lo = s_M[0];
  pt.span = K(s_M[cnt - 1] - pt.lo);
  const uint32_t bits = pt.span ? uint32_t(8 * sizeof(K)) - uint32_t(sizeof(K) == 8 ? __clzll((long long)pt.span)
                                                                                    : __clz(int(pt.span)))
                                : 0u;
  pt.sh = bits > PB ? bits - PB : 0u;
  const K pmax = K(pt.span >> pt.sh);
  for (uint32_t p = threadIdx.x; p <= (1u << PB); p += threads)
    s_T[p] = K(p) > pmax ? cnt : lb_range(s_M, 0, cnt, K(pt.lo + (K(p) << pt.sh)));
  return pt;
}

// lower_bound(s_M[0, cnt), q) through the table.
template <typename K>
__device__ __forceinline__ uint32_t prefix_lower_bound(const K* s_M, uint32_t cnt, const uint32_t* s_T,
                                                       const PrefixTab<K>& pt, K q) {
  if (q <= pt.lo) return 0;
  const K d = K(q - pt.lo);
  if (d > pt.span) return cnt;
  const uint32_t p = uint32_t(d >> pt.sh);
  return lb_range(s_M, s_T[p], s_T[p + 1], q);
}

// lower_bound over bucket b's compressed maxima (ItemDir::bd): the prefix table T names
// the slice of entries whose 32-bit offsets M' share the query's top bits, E holds the
// next 16 bits.  Truncation is order-preserving, so the result is exact except where
// the query's truncated value TIES with an entry's (then the answer is that unit or a
// later one).  A RUN of ties (or fixable = false) is settled against the exact maxima
// gM; a single tie is left to the caller's walk (the answer is the returned unit or the
// next one).
template <typename K>
__device__ __forceinline__ uint32_t lower_bound16(const uint16_t* E, const uint16_t* T, uint32_t cnt, K q, K lo,
                                                  uint32_t sh, uint32_t top, uint32_t ssh, uint32_t esh,
                                                  const K* __restrict__ gM, bool fixable) {
  if (q <= lo) return 0;
  const K dq = K(q - lo) >> sh;
  if (dq > K(top)) return cnt;
  const uint32_t q32 = uint32_t(dq);
  const uint32_t p = q32 >> ssh;
  uint32_t a = T[p];
  const uint32_t b = T[p + 1];
  const uint16_t q16 = uint16_t(q32 >> esh);
  uint32_t len = b - a;
  while (len > 0) {
    const uint32_t half = len >> 1;
    if (E[a + half] < q16) { a += half + 1; len -= half + 1; } else { len = half; }
  }
  if ((sh | esh) && a < b && E[a] == q16) {
    if (fixable && (a + 1 >= b || E[a + 1] != q16)) return a;
    while (a < b && E[a] == q16 && __ldg(gM + a) < q) ++a;
  }
  return a;
}

}  // namespace hbt
