// implicit_search.cu — hbt_search for the IMPLICIT tree (the hot path).
//
// Node search = "the minimum i such that q <= sep[i]" = #{t : sep[t] < q}
// (PAPER.md:190 read with the comments of Snippets 1/2, P:520 / P:566; reading
// R1), then descend to child node*F + i (Snippet 3's
// (nodeIndex+result)<<3).  Two phases per warp round of 32 queries:
//
//  1. The top of the I-segment in the fastest memory, in its B200
//     form: the root-first descent through levels 0..T-1 always reaches the FIRST
//     level-T node whose subtree max is >= q, i.e. lower_bound(M_T, q) over the
//     level-T maxima; M_T and a prefix directory are staged in shared memory once
//     per persistent CTA and ONE lane per query does one directory probe plus a
//     short binary search.
//  2. L2/HBM levels: a GROUP of G = 2 (4 for 256-byte nodes) lanes per query.
//     A node wider than one 32 B sector is read through its index sector
//     (entry t = max key of sector t, the paper's index line of P:134 applied
//     to implicit nodes): t = popc(ballot(idx < q)), then ONLY key sector t is
//     read: i = t*KPS + popc(ballot(key < q)).  So a level moves 64 B instead of
//     F*S bytes, with 16 B vector loads, no divergence and no barriers (Snippet
//     3 needs two __syncthreads per level).  Levels beyond the L2
//     budget are read whole in one round trip (256-bit lane loads).  Each group
//     keeps QPG queries in flight level-synchronously (the GPU form of the
//     software pipelining of Alg. 2).
//  Leaf: the 64 B line [P keys | P values] is read by the group in one round
//  trip; s = popc(ballot(key < q)); r = line*P + s; found = r < n' && key[s] == q.
// Queries and results stream with evict-first (.cs) accesses so they do not
// displace the tree from L2.
#include <algorithm>

#include "block_util.cuh"
#include "hbt_internal.cuh"
#include "item_dir.cuh"

namespace hbt {
namespace {

constexpr uint64_t kEnd = HBT_POS_END;
constexpr uint64_t kFound = HBT_FOUND_BIT;

template <typename K>
__device__ __forceinline__ K key_max() { return K(~K(0)); }

template <typename K>
union V16 {
  uint4 u;
  K k[16 / sizeof(K)];
};

template <typename K>
__device__ __forceinline__ void ld16(V16<K>& v, const uint8_t* p) {
  v.u = __ldg(reinterpret_cast<const uint4*>(p));
}

// 32 B held by one lane (a whole sector), loaded with one 256-bit load (sm_100).
template <typename K>
union L256 {
  unsigned long long u[4];
  K k[32 / sizeof(K)];
};

template <typename K>
__device__ __forceinline__ void ld32(L256<K>& v, const uint8_t* p) {
  asm volatile("ld.global.nc.v4.u64 {%0, %1, %2, %3}, [%4];"
               : "=l"(v.u[0]), "=l"(v.u[1]), "=l"(v.u[2]), "=l"(v.u[3])
               : "l"(p));
}

// The same with an L2 eviction-priority policy (createpolicy): leaf lines that are
// read once per batch go evict-first so they do not push the inner levels out.
template <typename K>
__device__ __forceinline__ void ld32_pol(L256<K>& v, const uint8_t* p, uint64_t pol) {
  asm volatile("ld.global.nc.L2::cache_hint.v4.u64 {%0, %1, %2, %3}, [%4], %5;"
               : "=l"(v.u[0]), "=l"(v.u[1]), "=l"(v.u[2]), "=l"(v.u[3])
               : "l"(p), "l"(pol));
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}

template <typename K>
__device__ __forceinline__ void fill_max32(L256<K>& v) {
#pragma unroll
  for (int e = 0; e < 4; ++e) v.u[e] = ~0ull;
}

template <typename K>
__device__ __forceinline__ void fill_max(V16<K>& v) {
#pragma unroll
  for (int e = 0; e < int(16 / sizeof(K)); ++e) v.k[e] = key_max<K>();
}

__device__ __forceinline__ uint32_t ldcs(const uint32_t* p) { return __ldcs(p); }
__device__ __forceinline__ uint64_t ldcs(const uint64_t* p) {
  return __ldcs(reinterpret_cast<const unsigned long long*>(p));
}
__device__ __forceinline__ void stcs(uint32_t* p, uint32_t v) { __stcs(p, v); }
__device__ __forceinline__ void stcs(uint64_t* p, uint64_t v) {
  __stcs(reinterpret_cast<unsigned long long*>(p), (unsigned long long)v);
}

template <typename K, int F>
struct Cfg {
  static constexpr int S = int(sizeof(K));
  static constexpr int NODE_BYTES = F * S;
  static constexpr int KPS = 32 / S;                                      // keys per 32 B sector
  static constexpr int NSEC = NODE_BYTES >= 32 ? NODE_BYTES / 32 : 1;     // sectors per node
  static constexpr bool HAS_IDX = NSEC > 1;
  static constexpr int IDXB = HAS_IDX ? (NSEC * S > 16 ? NSEC * S : 16) : 0;  // index bytes per node
  static constexpr int IL = IDXB / 16;                                    // lanes loading the index
  static constexpr int SECB = NODE_BYTES < 32 ? NODE_BYTES : 32;          // bytes read after the index
  static constexpr int SL_ = SECB / 16;                                   // lanes loading them
  static constexpr int G = IL > 2 ? IL : 2;                               // lanes per query group
  static constexpr int NG = 32 / G;                                       // groups per warp
  static constexpr int P = 64 / (2 * S);                                  // pairs per leaf line
};

template <typename K, int N>
__device__ __forceinline__ K pick(const K (&k)[N], uint32_t slot) {
  K r = k[0];
#pragma unroll
  for (int t = 1; t < N; ++t) r = (slot == uint32_t(t)) ? k[t] : r;
  return r;
}

template <typename K>
__device__ __forceinline__ uint32_t count_less16(const V16<K>& v, K q, unsigned gmask) {
  uint32_t c = 0;
#pragma unroll
  for (int e = 0; e < int(16 / sizeof(K)); ++e) c += __popc(__ballot_sync(0xffffffffu, v.k[e] < q) & gmask);
  return c;
}

// Phase 2 of a warp round: levels [d0, H) by lane groups, the leaf line, and the
// results of the round (slot j of group g = round query j*NG + g, stored at
// base + j*NG + g).
// FIX (compressed item directory, implicit_search_cdir_kernel): the directory may
// place a query ONE unit early (a tie of truncated maxima; runs of ties are settled
// before the walk).  Every real separator of that unit u is < q and its last key slot
// is MAX (reading R3), so the walk takes the last child at every level and ends
// on the LAST leaf line of u's subtree with s = P, which cannot happen on the right
// unit.  The lower bound then lies in the following lines (u + 1's first lines, in
// key order): the slot reads line + 1, ... until s < P, at most up to line fix_last
// (the bucket's last real line).  For hits on ties (c4) that is one extra line.
template <typename K, int F, int QPG, bool REC = false, bool FIX = false>
__device__ __forceinline__ void descend_and_store(const uint8_t* __restrict__ inner,
                                                  const uint8_t* __restrict__ inner_idx,
                                                  const uint8_t* __restrict__ leaf, const LevelTable& lt,
                                                  uint32_t d0, K (&q)[QPG], uint32_t (&node)[QPG], int g, int k,
                                                  unsigned gmask, uint64_t base, uint64_t m, uint64_t n,
                                                  uint64_t pos_base, uint64_t* __restrict__ out_pf,
                                                  K* __restrict__ out_v, uint32_t fix_last = 0) {
  using C = Cfg<K, F>;
  const uint32_t H = lt.H;
  for (uint32_t d = d0; d < H; ++d) {
    const uint8_t* lvl = inner + lt.offset[d] * C::NODE_BYTES;
    if constexpr (C::HAS_IDX) {
      if ((lt.full_mask >> d) & 1u) {
        // Level beyond the L2-resident budget: a miss costs a whole DRAM line
        // anyway, so read the full node in ONE round trip (each of the G lanes
        // loads NODE_BYTES/G contiguous bytes) instead of index + sector.
        if constexpr (C::NODE_BYTES / C::G >= 32) {
          if (lt.full256) {
            // 256-bit lane loads: half the load instructions (and L1TEX wavefronts,
            // the pipe that binds the item search, profiles/r01_c4_items_*) of 16 B loads
            constexpr int NC32 = C::NODE_BYTES / C::G / 32;
            L256<K> fw[QPG][NC32];
            const uint64_t pol = policy_evict_last();
            auto load = [&](int j) {
#pragma unroll
              for (int h = 0; h < NC32; ++h) {
                const uint8_t* p = lvl + uint64_t(node[j]) * C::NODE_BYTES + (k * NC32 + h) * 32;
                if (lt.l2_hint & 2u) ld32_pol(fw[j][h], p, pol);
                else ld32(fw[j][h], p);
              }
            };
            auto count = [&](int j) {
              uint32_t c = 0;
#pragma unroll
              for (int h = 0; h < NC32; ++h)
#pragma unroll
                for (int e = 0; e < 32 / C::S; ++e) c += (fw[j][h].k[e] < q[j]) ? 1u : 0u;
#pragma unroll
              for (int x = 1; x < C::G; x <<= 1) c += __shfl_xor_sync(0xffffffffu, c, x);
              return c;
            };
#pragma unroll
            for (int j = 0; j < QPG; ++j) load(j);
            uint32_t c[QPG];
#pragma unroll
            for (int j = 0; j < QPG; ++j) c[j] = count(j);
#pragma unroll
            for (int j = 0; j < QPG; ++j) node[j] = node[j] * F + c[j];
            continue;
          }
        }
        constexpr int NCH = C::NODE_BYTES / C::G / 16;
        V16<K> fv[QPG][NCH];
#pragma unroll
        for (int j = 0; j < QPG; ++j)
#pragma unroll
          for (int h = 0; h < NCH; ++h)
            ld16(fv[j][h], lvl + uint64_t(node[j]) * C::NODE_BYTES + (k * NCH + h) * 16);
#pragma unroll
        for (int j = 0; j < QPG; ++j) {
          uint32_t c = 0;
#pragma unroll
          for (int h = 0; h < NCH; ++h)
#pragma unroll
            for (int e = 0; e < 16 / C::S; ++e) c += (fv[j][h].k[e] < q[j]) ? 1u : 0u;
#pragma unroll
          for (int x = 1; x < C::G; x <<= 1) c += __shfl_xor_sync(0xffffffffu, c, x);
          node[j] = node[j] * F + c;
        }
        continue;
      }
    }
    uint32_t sec[QPG];
    if constexpr (C::HAS_IDX) {
      const uint8_t* lidx = inner_idx + lt.offset[d] * C::IDXB;
      V16<K> iv[QPG];
#pragma unroll
      for (int j = 0; j < QPG; ++j) {
        if (k < C::IL) ld16(iv[j], lidx + uint64_t(node[j]) * C::IDXB + k * 16);
        else fill_max(iv[j]);
      }
#pragma unroll
      for (int j = 0; j < QPG; ++j) sec[j] = count_less16(iv[j], q[j], gmask);
    } else {
#pragma unroll
      for (int j = 0; j < QPG; ++j) sec[j] = 0;
    }
    V16<K> kv[QPG];
#pragma unroll
    for (int j = 0; j < QPG; ++j) {
      if (k < C::SL_) ld16(kv[j], lvl + uint64_t(node[j]) * C::NODE_BYTES + sec[j] * 32 + k * 16);
      else fill_max(kv[j]);
    }
#pragma unroll
    for (int j = 0; j < QPG; ++j) node[j] = node[j] * F + sec[j] * C::KPS + count_less16(kv[j], q[j], gmask);
  }
  uint64_t my_pf[QPG / C::G];
  K my_v[QPG / C::G];
  if (lt.leaf256) {
    // ---- leaf line [P keys | P values] in ONE 64 B request per group: lane 0 loads
    //      the key sector, lane 1 the value sector with 256-bit loads (sm_100).
    //      s = #{keys < q} on lane 0, broadcast; key / value picked by lanes 0 / 1.
    L256<K> lw[QPG];
    const uint64_t pol = policy_evict_first();
    auto load = [&](int j) {
      if (k < 2) {
        const uint8_t* p = leaf + uint64_t(node[j]) * 64 + k * 32;
        if (lt.l2_hint & 1u) ld32_pol(lw[j], p, pol);
        else ld32(lw[j], p);
      } else {
        fill_max32(lw[j]);
      }
    };
    auto count = [&](int j) {
      uint32_t c = 0;
#pragma unroll
      for (int e = 0; e < C::P; ++e) c += (lw[j].k[e] < q[j]) ? 1u : 0u;
      return __shfl_sync(0xffffffffu, c, g * C::G);
    };
#pragma unroll
    for (int j = 0; j < QPG; ++j) load(j);
    uint32_t sl[QPG];
#pragma unroll
    for (int j = 0; j < QPG; ++j) sl[j] = count(j);
    if constexpr (FIX) {
      {
        uint32_t adv = 0;
#pragma unroll
        for (int j = 0; j < QPG; ++j) adv |= (sl[j] == uint32_t(C::P) && node[j] < fix_last) ? 1u << j : 0u;
        while (__any_sync(0xffffffffu, adv != 0)) {
#pragma unroll
          for (int j = 0; j < QPG; ++j)
            if ((adv >> j) & 1u) {
              ++node[j];
              load(j);
            }
          uint32_t nadv = 0;
#pragma unroll
          for (int j = 0; j < QPG; ++j) {
            const uint32_t cc = count(j);
            if ((adv >> j) & 1u) {
              sl[j] = cc;
              nadv |= (cc == uint32_t(C::P) && node[j] < fix_last) ? 1u << j : 0u;
            }
          }
          adv = nadv;
        }
      }
    }
#pragma unroll
    for (int j = 0; j < QPG; ++j) {
      const uint32_t s = sl[j];
      const uint32_t sc = s < uint32_t(C::P) ? s : uint32_t(C::P - 1);
      const K x = pick(lw[j].k, sc);
      const K key_s = __shfl_sync(0xffffffffu, x, g * C::G);
      const K val_s = __shfl_sync(0xffffffffu, x, g * C::G + 1);
      const uint64_t r = uint64_t(node[j]) * C::P + s;
      const bool found = (s < uint32_t(C::P)) && (r < n) && (key_s == q[j]);
      if (j % C::G == k) {
        my_pf[j / C::G] = (r < n ? r + pos_base : kEnd) | (found ? kFound : 0ull);
        my_v[j / C::G] = found ? val_s : K(0);
      }
    }
  } else {
  // ---- leaf line [P keys | P values]: lanes 0 and 1 of the group each load one
  //      16 B half of the key sector and of the value sector, so every load
  //      instruction touches exactly one 32 B sector per group.
  constexpr int E16 = 16 / C::S;
  V16<K> lkey[QPG], lval[QPG];
#pragma unroll
  for (int j = 0; j < QPG; ++j) {
    if (k < 2) {
      const uint8_t* p = leaf + uint64_t(node[j]) * 64 + k * 16;
      ld16(lkey[j], p);
      ld16(lval[j], p + 32);
    } else {
      fill_max(lkey[j]);
      fill_max(lval[j]);
    }
  }
#pragma unroll
  for (int j = 0; j < QPG; ++j) {
    const uint32_t s = count_less16(lkey[j], q[j], gmask);  // lanes >= 2 hold MAX
    const uint32_t sc = s < uint32_t(C::P) ? s : uint32_t(C::P - 1);
    const int src = g * C::G + int(sc / E16);
    const K key_s = __shfl_sync(0xffffffffu, pick(lkey[j].k, sc % E16), src);
    const K val_s = __shfl_sync(0xffffffffu, pick(lval[j].k, sc % E16), src);
    const uint64_t r = uint64_t(node[j]) * C::P + s;
    const bool found = (s < uint32_t(C::P)) && (r < n) && (key_s == q[j]);
    if (j % C::G == k) {
      my_pf[j / C::G] = (r < n ? r + pos_base : kEnd) | (found ? kFound : 0ull);
      my_v[j / C::G] = found ? val_s : K(0);
    }
  }
  }
  // lane (g, k) stores slots j = k + G*t: round queries (k + G*t)*NG + g
#pragma unroll
  for (int t = 0; t < QPG / C::G; ++t) {
    const uint64_t i = base + uint64_t(k + C::G * t) * C::NG + g;
    if (i < m) {
      if constexpr (REC) {
        // 16 B record {pos|found, value} (bucketed search: the gather reads records)
        __stcs(reinterpret_cast<ulonglong2*>(out_pf) + i, make_ulonglong2(my_pf[t], (unsigned long long)my_v[t]));
      } else {
        stcs(out_pf + i, my_pf[t]);
        stcs(out_v + i, my_v[t]);
      }
    }
  }
}

// The plain (unbucketed) search: one persistent pass over the batch, one query per
// lane in phase 1 (the level-T directory), lane groups in phase 2 (descend_and_store).
// MODE 2: the directory [M_T | prefix table] is staged in shared memory once per CTA;
// MODE 3 (small batches): it is read in place from L2 (staging ~70 KB per CTA would
// dominate a launch that serves only a few warp rounds).
template <typename K, int F, int THREADS, int MODE>
__global__ void __launch_bounds__(THREADS, 1)
implicit_search_kernel(const uint8_t* __restrict__ inner, const uint8_t* __restrict__ inner_idx,
                       const uint8_t* __restrict__ leaf, const uint32_t* __restrict__ dirbuf,
                       const K* __restrict__ queries, uint64_t m, uint64_t* __restrict__ out_pf,
                       K* __restrict__ out_v, const LevelTable lt, uint64_t n, uint64_t pos_base) {
  static_assert(MODE == 2 || MODE == 3, "directory staged (2) or read in place (3)");
  using C = Cfg<K, F>;
  constexpr int ROUND = 32;              // queries per warp round
  constexpr int QPG = ROUND / C::NG;     // queries per group in phase 2
  static_assert(QPG % C::G == 0, "every group lane stores QPG/G results");
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t* s_words = reinterpret_cast<uint32_t*>(smem);
  if constexpr (MODE == 2) {
    // directory: [M_T (dcount keys) | 2^dbits x (u16 lo, u16 hi)]
    const uint32_t words = (lt.dcount * uint32_t(sizeof(K)) + (4u << lt.dbits)) / 4;
    for (uint32_t i = threadIdx.x; i < words; i += THREADS) s_words[i] = __ldg(dirbuf + i);
  }
  __syncthreads();
  const K* d_M = MODE == 3 ? reinterpret_cast<const K*>(dirbuf) : reinterpret_cast<const K*>(smem);
  const uint32_t* d_dir = MODE == 3 ? reinterpret_cast<const uint32_t*>(reinterpret_cast<const uint8_t*>(dirbuf) +
                                                                         lt.dcount * sizeof(K))
                                    : reinterpret_cast<const uint32_t*>(smem + lt.dcount * sizeof(K));

  const int lane = threadIdx.x & 31;
  const int g = lane / C::G, k = lane % C::G;
  const unsigned gmask = ((1u << C::G) - 1u) << (g * C::G);
  const uint64_t warp = (uint64_t(blockIdx.x) * THREADS + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * THREADS) >> 5;
  const uint64_t rounds = (m + ROUND - 1) / ROUND;

  // The query stream is pipelined across rounds: the next round's queries are
  // loaded while this round walks the tree (their HBM latency was the largest single
  // stall, profiles/r01_c2_v11_*).  Lanes past the batch end repeat the batch's last
  // query (results discarded) so they walk to a leaf line the batch itself uses: a
  // streamed host L-segment stages only the bucket's slice.
  K nextq;
  {
    const uint64_t i = warp * ROUND + lane;
    nextq = warp < rounds ? ldcs(queries + (i < m ? i : m - 1)) : key_max<K>();
  }
  for (uint64_t rd = warp; rd < rounds; rd += nwarps) {
    const uint64_t base = rd * ROUND;
    // ---- phase 1: one lane per query; coalesced query loads
    const K myq = nextq;
    {
      const uint64_t i = (rd + nwarps) * ROUND + lane;
      nextq = rd + nwarps < rounds ? ldcs(queries + (i < m ? i : m - 1)) : key_max<K>();
    }
    // level-T node = lower_bound(M_T, q), narrowed by the prefix directory
    uint32_t mynode;
    {
      const uint32_t e = d_dir[uint32_t(myq >> (8 * sizeof(K) - lt.dbits))];
      uint32_t lo = e & 0xFFFFu, hi = e >> 16;
      while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (d_M[mid] < myq) lo = mid + 1; else hi = mid;
      }
      mynode = lo;
    }
    // ---- phase 2: lane groups; slot j of group g is round query j*NG + g,
    //      owned in phase 1 by lane (j*NG)%32 + g
    K q[QPG];
    uint32_t node[QPG];
#pragma unroll
    for (int j = 0; j < QPG; ++j) {
      const int src = (j * C::NG) % 32 + g;
      q[j] = __shfl_sync(0xffffffffu, myq, src);
      node[j] = __shfl_sync(0xffffffffu, mynode, src);
    }
    descend_and_store<K, F, QPG>(inner, inner_idx, leaf, lt, lt.SL, q, node, g, k, gmask, base, m, n, pos_base,
                                 out_pf, out_v);
  }
}

// Bucketed search with a bucket-local directory (bucketed.cu, ItemDir).  One
// persistent CTA works through items of rounds * THREADS consecutive bucketed
// queries.  Per item: the item's first and last queries give its bucket range
// [b0, b1] (binary search over the staged bucket starts), hence a contiguous range
// of level-`level` nodes [u0, u1] that contains every query's node at that level:
// all nodes before u0 end at or below splitter b0-1 < q and q <= splitter b1 <= max
// of node u1.  The maxima of [u0, u1] are staged in shared memory; a query's node is
// u0 + lower_bound(maxima, q) (clamped to u1, which only binds past the last key),
// exactly the node the root-first descent reaches (every level picks the first
// child whose subtree max is >= q, R1/R3).  The rest of the walk is
// descend_and_store from that level.
//
// Measured and dropped (profiles/r02_c4_*): a strided item schedule in which all
// CTAs move through the bucketed order together cut c4's DRAM reads 40.1 -> 29.2 GB
// per launch (the leaf slices stay L2-resident while their bucket's queries arrive)
// but ran slower (9.9 -> 10.5 ms): this kernel is bound by latency and the LSU pipe,
// not by DRAM, and the wider per-item directory cost more than the saved bytes.

// Cooperative copy of cnt keys into shared memory, four loads in flight per thread.
template <typename K>
__device__ __forceinline__ void stage_keys(K* dst, const K* __restrict__ src, uint32_t cnt, uint32_t threads) {
  for (uint32_t i = threadIdx.x; i < cnt; i += 4 * threads) {
    K x[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) x[u] = i + u * threads < cnt ? __ldg(src + i + u * threads) : K(0);
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (i + u * threads < cnt) dst[i + u * threads] = x[u];
  }
}

template <typename K, int F, int THREADS>
__global__ void __launch_bounds__(THREADS)
implicit_search_items_kernel(const uint8_t* __restrict__ inner, const uint8_t* __restrict__ inner_idx,
                             const uint8_t* __restrict__ leaf, const ItemDir d, const K* __restrict__ queries,
                             uint64_t m, uint64_t* __restrict__ out_pf, K* __restrict__ out_v, const LevelTable lt,
                             uint64_t n) {
  using C = Cfg<K, F>;
  constexpr int QPG = 32 / C::NG;
  const uint64_t W = uint64_t(THREADS) * d.rounds;
  extern __shared__ __align__(16) uint8_t smem[];
  uint64_t* s_bstart = reinterpret_cast<uint64_t*>(smem);
  K* s_M = reinterpret_cast<K*>(s_bstart + d.B + 1);
  uint32_t* s_T = reinterpret_cast<uint32_t*>(s_M + d.cap);
  __shared__ uint64_t s_range[2];
  const K* gM = static_cast<const K*>(d.M);
  for (uint32_t i = threadIdx.x; i <= d.B; i += THREADS) s_bstart[i] = d.bstart[i];
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int g = lane / C::G, k = lane % C::G;
  const unsigned gmask = ((1u << C::G) - 1u) << (g * C::G);
  const uint64_t items = (m + W - 1) / W;
  for (uint64_t it = blockIdx.x; it < items; it += gridDim.x) {
    const uint64_t p0 = it * W, p1 = (p0 + W < m ? p0 + W : m) - 1;
    if (threadIdx.x < 2) {
      const uint64_t p = threadIdx.x ? p1 : p0;
      uint32_t lo = 0, hi = d.B;  // largest b with bstart[b] <= p
      while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (s_bstart[mid] <= p) lo = mid; else hi = mid;
      }
      const uint64_t lu = threadIdx.x ? ((uint64_t(lo) + 1) * d.U) / d.B - 1 : (uint64_t(lo) * d.U) / d.B;
      s_range[threadIdx.x] = lu / d.span;
    }
    __syncthreads();
    const uint64_t u0 = s_range[0], u1 = s_range[1];
    const uint32_t cnt = uint32_t(u1 - u0 + 1);
    const bool in_smem = cnt <= d.cap;
    if (in_smem) stage_keys(s_M, gM + u0, cnt, THREADS);
    __syncthreads();
    PrefixTab<K> pt{};
    if (in_smem) pt = build_prefix(s_M, cnt, s_T, THREADS);
    __syncthreads();
    const K* M = in_smem ? s_M : gM + u0;
    // the next round's queries are loaded while this round walks the tree
    K nextq;
    {
      const uint64_t i = p0 + uint64_t(wid) * 32 + lane;
      nextq = i <= p1 ? ldcs(queries + i) : key_max<K>();
    }
#pragma unroll 1
    for (int r = 0; r < int(d.rounds); ++r) {
      const uint64_t base = p0 + (uint64_t(r) * (THREADS / 32) + wid) * 32;
      if (base > p1) break;
      const K myq = nextq;
      {
        const uint64_t i = base + (THREADS / 32) * 32 + lane;
        nextq = (r + 1 < int(d.rounds) && i <= p1) ? ldcs(queries + i) : key_max<K>();
      }
      const uint32_t lo = in_smem ? prefix_lower_bound(s_M, cnt, s_T, pt, myq) : lb_range(M, 0, cnt, myq);
      const uint32_t mynode = uint32_t(u0) + (lo < cnt ? lo : cnt - 1);
      K q[QPG];
      uint32_t node[QPG];
#pragma unroll
      for (int j = 0; j < QPG; ++j) {
        const int src = (j * C::NG) % 32 + g;
        q[j] = __shfl_sync(0xffffffffu, myq, src);
        node[j] = __shfl_sync(0xffffffffu, mynode, src);
      }
      descend_and_store<K, F, QPG, true>(inner, inner_idx, leaf, lt, d.level, q, node, g, k, gmask, base, p1 + 1, n,
                                         d.pos_base, out_pf, out_v);
    }
    __syncthreads();
  }
}

// The same with the COMPRESSED per-bucket directory (ItemDir::bd, 16-bit entries under a
// 2^12-slice prefix table), used when it reaches a deeper level than 8 B keys would (c4:
// the last inner level instead of the one above it, one dependent node read less per
// query; c5: the leaf lines themselves).  Work items are cut inside one bucket each
// (bucket b's queries split into ceil(cnt_b / W) near-equal items), so an item stages
// exactly its bucket's directory: one elected thread moves the entries and the prefix
// table into shared memory with bulk copies (cp.async.bulk, completion on an mbarrier).
// Ties of truncated values: lower_bound16 (item_dir.cuh) and descend_and_store FIX.
// Items are handed off on two mbarriers instead of CTA barriers: every warp arrives on
// `empty` right after its LAST directory lookup of an item; thread 0 waits for all of
// them, publishes the next item (its range and bucket record, double-buffered by item
// parity) and starts its directory copy, which completes `full`.  A warp starts the next
// item as soon as `full` completes -- it does not wait for the other warps' last walks
// (leaf reads) of the previous item (c4 item search -1..-5 %, c5 -3 %,
// profiles/r02s_item_pipe_ab.jsonl).  With ItemDir::cnode (u64, F = 16, the directory on the
// last inner level) a lane reads its unit's 32 B compact node (bk_cnode, bucketed.cu)
// instead of the 128 B node and goes straight to the leaf line (c4 item search -15 %).
template <typename K, int F, int THREADS>
__global__ void __launch_bounds__(THREADS)
implicit_search_cdir_kernel(const uint8_t* __restrict__ inner, const uint8_t* __restrict__ inner_idx,
                            const uint8_t* __restrict__ leaf, const ItemDir d, const K* __restrict__ queries,
                            uint64_t m, uint64_t* __restrict__ out_pf, K* __restrict__ out_v, const LevelTable lt,
                            uint64_t n) {
  using C = Cfg<K, F>;
  constexpr int QPG = 32 / C::NG;
  constexpr int NW = THREADS / 32;
  const uint64_t W = uint64_t(THREADS) * d.rounds;
  const uint32_t B = d.B;
  extern __shared__ __align__(16) uint8_t smem[];
  uint16_t* s_E = reinterpret_cast<uint16_t*>(smem);
  uint16_t* s_T = s_E + d.cap;
  uint64_t* s_bs = reinterpret_cast<uint64_t*>(s_T + kT16);
  uint32_t* s_is = reinterpret_cast<uint32_t*>(s_bs + B + 1);
  __shared__ uint64_t full_bar, empty_bar;
  __shared__ uint32_t s_tmp[32];
  __shared__ uint64_t s_p[2][2];
  __shared__ BucketDir s_bd[2];
  const K* gM = static_cast<const K*>(d.M);
  for (uint32_t i = threadIdx.x; i <= B; i += THREADS) s_bs[i] = d.bstart[i];
  __syncthreads();
  for (uint32_t b = threadIdx.x; b < B; b += THREADS) s_is[b] = uint32_t((s_bs[b + 1] - s_bs[b] + W - 1) / W);
  __syncthreads();
  const uint32_t last = s_is[B - 1];
  block_exclusive_scan<THREADS>(s_is, s_is, B, s_tmp);
  if (threadIdx.x == 0) {
    s_is[B] = s_is[B - 1] + last;
    mbar_init(&full_bar, 1);
    mbar_init(&empty_bar, NW);
    fence_mbar_init();
  }
  __syncthreads();
  const uint32_t items = s_is[B];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int g = lane / C::G, k = lane % C::G;
  const unsigned gmask = ((1u << C::G) - 1u) << (g * C::G);
  auto bucket_of_item = [&](uint32_t it) {
    uint32_t lo = 0, hi = B;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (s_is[mid] <= it) lo = mid; else hi = mid;
    }
    return lo;
  };
  // thread 0: the item `it` of bucket lo into metadata slot x, and its directory copy
  // (the expect_tx arrive releases the metadata writes to the phase's waiters)
  auto issue = [&](uint32_t it, int x) {
    const uint32_t lo = bucket_of_item(it);
    const BucketDir bd = d.bd[lo];
    const uint64_t nb = s_is[lo + 1] - s_is[lo], j = it - s_is[lo];
    const uint64_t c0 = s_bs[lo], cnt = s_bs[lo + 1] - c0;
    s_p[x][0] = c0 + (cnt * j) / nb;
    s_p[x][1] = c0 + (cnt * (j + 1)) / nb - 1;
    s_bd[x] = bd;
    fence_proxy_async_smem();
    const uint32_t eb = ((bd.cnt + 7u) & ~7u) * 2u;
    mbar_expect_tx(&full_bar, eb + kT16 * 2u);
    bulk_g2s(s_E, d.E16 + bd.off16, eb, &full_bar);
    bulk_g2s(s_T, d.T16 + uint64_t(lo) * kT16, kT16 * 2u, &full_bar);
  };
  if (threadIdx.x == 0 && blockIdx.x < items) issue(blockIdx.x, 0);
  uint32_t kk = 0;
  for (uint32_t it = blockIdx.x; it < items; it += gridDim.x, ++kk) {
    const int x = int(kk & 1u);
    mbar_wait(&full_bar, kk & 1u);
    const uint64_t p0 = s_p[x][0], p1 = s_p[x][1];
    const uint64_t u0 = s_bd[x].u0;
    const uint32_t cnt = s_bd[x].cnt;
    const uint64_t wb0 = p0 + uint64_t(wid) * 32;
    const int nr = wb0 > p1 ? 0 : int(min(uint64_t(d.rounds), (p1 - wb0) / (NW * 32) + 1));
    // past this warp's last directory lookup: release the directory buffer; thread 0 waits
    // for every warp, then publishes the next item
    auto done_with_dir = [&]() {
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty_bar);
      if (threadIdx.x == 0) {
        mbar_wait(&empty_bar, kk & 1u);
        if (it + gridDim.x < items) issue(it + gridDim.x, x ^ 1);
      }
    };
    if (nr == 0) done_with_dir();
    K nextq;
    {
      const uint64_t i = wb0 + lane;
      nextq = i <= p1 ? ldcs(queries + i) : key_max<K>();
    }
#pragma unroll 1
    for (int r = 0; r < nr; ++r) {
      const uint64_t base = wb0 + uint64_t(r) * (NW * 32);
      const K myq = nextq;
      {
        const uint64_t i = base + NW * 32 + lane;
        nextq = (r + 1 < nr && i <= p1) ? ldcs(queries + i) : key_max<K>();
        if (d.qpf && r + 1 + int(d.qpf) < nr && i + d.qpf * (NW * 32) <= p1)
          asm volatile("prefetch.global.L2 [%0];" ::"l"(queries + i + d.qpf * (NW * 32)));
      }
      const uint32_t a = lower_bound16(s_E, s_T, cnt, myq, K(s_bd[x].lo), s_bd[x].sh, s_bd[x].top, s_bd[x].ssh,
                                       s_bd[x].esh, gM + u0, d.fix);
      uint32_t mynode = uint32_t(u0) + (a < cnt ? a : cnt - 1);
      uint32_t lvl0 = d.level;
      if constexpr (sizeof(K) == 8 && F == 16) {
        if (d.cnode) {
          // the directory unit's compact node (32 B, one 256-bit load per lane): child =
          // 0 if M'(q) <= b0, else 1 + #{slots 1..14 with entry < (M'(q) - b0) >> nsh}
          const uint64_t lo = s_bd[x].lo;
          const uint32_t sh = s_bd[x].sh, nsh = s_bd[x].nsh;
          L256<K> cn;
          ld32(cn, d.cnode + uint64_t(mynode) * 32);
          const uint64_t dq = myq <= lo ? 0ull : (uint64_t(myq) - lo) >> sh;
          const uint32_t qp = dq > 0xFFFFFFFFull ? 0xFFFFFFFFu : uint32_t(dq);
          const uint32_t b0 = uint32_t(cn.u[0]);
          uint32_t c = 0;
          if (qp > b0) {
            const uint32_t t16 = min((qp - b0) >> nsh, 0xFFFFu);
            const uint32_t qq = t16 * 0x10001u;
            // u16 slots 1..14: two per 32-bit word, words 1..7 (word 0 is b0)
            const uint32_t cmp = __popc(__vcmpltu2(uint32_t(cn.u[0] >> 32), qq)) +
                                 __popc(__vcmpltu2(uint32_t(cn.u[1]), qq)) +
                                 __popc(__vcmpltu2(uint32_t(cn.u[1] >> 32), qq)) +
                                 __popc(__vcmpltu2(uint32_t(cn.u[2]), qq)) +
                                 __popc(__vcmpltu2(uint32_t(cn.u[2] >> 32), qq)) +
                                 __popc(__vcmpltu2(uint32_t(cn.u[3]), qq)) +
                                 __popc(__vcmpltu2(uint32_t(cn.u[3] >> 32), qq));
            c = 1 + cmp / 16;
          }
          mynode = mynode * 16 + c;
          lvl0 = d.level + 1;
        }
      }
      if (r == nr - 1) done_with_dir();
      K q[QPG];
      uint32_t node[QPG];
#pragma unroll
      for (int j = 0; j < QPG; ++j) {
        const int src = (j * C::NG) % 32 + g;
        q[j] = __shfl_sync(0xffffffffu, myq, src);
        node[j] = __shfl_sync(0xffffffffu, mynode, src);
      }
      descend_and_store<K, F, QPG, true, true>(inner, inner_idx, leaf, lt, lvl0, q, node, g, k, gmask, base,
                                               p1 + 1, n, d.pos_base, out_pf, out_v,
                                               d.fix ? uint32_t(min((u0 + cnt) * d.span, d.U) - 1) : 0u);
    }
  }
}

template <typename K, int F>
struct Launch {
  using C = Cfg<K, F>;

  // Levels below the shared-memory top are read as index sector + one key sector while
  // their cumulative bytes fit the L2 budget, as whole nodes beyond it.
  static uint32_t full_mask(const hbt_tree* t, uint32_t first) {
    uint32_t mask = 0;
    uint64_t cum = 0;
    const uint64_t budget = t->cfg.l2_levels_bytes ? t->cfg.l2_levels_bytes : (32ull << 20);
    for (uint32_t d = first; d < t->H; ++d) {
      cum += t->nodes[d] * uint64_t(C::NODE_BYTES + C::IDXB);
      if (C::HAS_IDX && cum > budget && d < 32) mask |= 1u << d;
    }
    if (t->cfg.full_levels) mask = C::HAS_IDX ? uint32_t(t->cfg.full_levels) : 0u;  // explicit override
    return mask;
  }

  template <int THREADS, int MODE>
  static int run_t(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t base,
                   cudaStream_t s, const void* leafp) {
    auto kern = implicit_search_kernel<K, F, THREADS, MODE>;
    LevelTable lt{};
    for (uint32_t d = 0; d <= t->H; ++d) lt.offset[d] = t->offset[d];
    lt.H = t->H;
    lt.leaf256 = t->cfg.leaf256;
    lt.full256 = t->cfg.full256;
    lt.l2_hint = t->cfg.l2_hint;
    if (lt.l2_hint == 4) {
      // auto: while the I-segment fits in a quarter of the L2, the leaf lines (read
      // about once per batch) go evict-first so they cannot push the inner levels out
      // (c2 0.426 -> 0.415 ms); a larger I-segment leaves the L2 to whatever the query
      // distribution repeats (c5 Zipf: 2.84 -> 3.00 ms with the hint)
      static int l2 = 0;
      if (!l2) HBT_CUDA_TRY(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, t->device));
      lt.l2_hint = (t->inner_bytes + t->inner_idx_bytes) * 4 <= uint64_t(l2) ? 1u : 0u;
    }
    lt.SL = t->dir_T;
    lt.dcount = t->dir_count;
    lt.dbits = t->dir_bits;
    lt.full_mask = full_mask(t, lt.SL);
    const size_t smem = MODE == 2 ? t->dir_bytes : 0;
    static bool attr_set = false;  // per instantiation
    if (!attr_set) {
      HBT_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
      attr_set = true;
    }
    // occupancy of this instantiation for this smem size (cached: the query costs
    // microseconds, which dominate small batches)
    static size_t occ_smem = ~size_t(0);
    static int occ_cached = 0;
    if (occ_smem != smem) {
      HBT_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_cached, kern, THREADS, smem));
      occ_smem = smem;
    }
    int occ = occ_cached;
    if (t->cfg.ctas_per_sm && int(t->cfg.ctas_per_sm) < occ) occ = int(t->cfg.ctas_per_sm);
    if (occ < 1) occ = 1;
    const uint64_t rounds = (m + 31) / 32;
    uint64_t grid = uint64_t(t->num_sms) * occ;
    const uint64_t need = (rounds + THREADS / 32 - 1) / (THREADS / 32);
    if (need < grid) grid = need ? need : 1;
    kern<<<unsigned(grid), THREADS, smem, s>>>((const uint8_t*)t->d_inner, (const uint8_t*)t->d_inner_idx,
                                              (const uint8_t*)leafp, (const uint32_t*)t->d_dir, (const K*)q, m, pf,
                                              (K*)v, lt, t->n, base);
    HBT_CUDA_TRY(cudaGetLastError());
    return HBT_OK;
  }

  static int run_items(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, const ItemDir& d,
                       cudaStream_t s) {
    constexpr int TH = C::NODE_BYTES > 128 ? 512 : 1024;
    auto kern = implicit_search_items_kernel<K, F, TH>;
    LevelTable lt{};
    for (uint32_t x = 0; x <= t->H; ++x) lt.offset[x] = t->offset[x];
    lt.H = t->H;
    lt.SL = d.level;
    lt.leaf256 = t->cfg.leaf256;
    lt.full256 = t->cfg.full256;
    lt.l2_hint = t->cfg.item_l2_hint;
    lt.full_mask = full_mask(t, d.level);
    static bool attr_set = false;
    if (!attr_set) {
      HBT_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
      attr_set = true;
    }
    ItemDir dd = d;
    dd.rounds = item_rounds(m, t->num_sms, TH, t->cfg.item_rounds ? t->cfg.item_rounds : 16);
    uint64_t grid = t->num_sms;
    const uint64_t items = (m + uint64_t(TH) * dd.rounds - 1) / (uint64_t(TH) * dd.rounds);
    if (items < grid) grid = items ? items : 1;
    const size_t smem = (d.B + 1) * 8 + size_t(dd.cap) * C::S + ((1u << kPrefixBits) + 1) * 4;
    kern<<<unsigned(grid), TH, smem, s>>>((const uint8_t*)t->d_inner, (const uint8_t*)t->d_inner_idx,
                                          (const uint8_t*)t->d_leaf, dd, (const K*)q, m, pf, (K*)v, lt, t->n);
    HBT_CUDA_TRY(cudaGetLastError());
    return HBT_OK;
  }

  static int run_cdir(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, const ItemDir& d,
                         cudaStream_t s) {
    constexpr int TH = C::NODE_BYTES > 128 ? 512 : 1024;
    auto kern = implicit_search_cdir_kernel<K, F, TH>;
    LevelTable lt{};
    for (uint32_t x = 0; x <= t->H; ++x) lt.offset[x] = t->offset[x];
    lt.H = t->H;
    lt.SL = d.level;
    lt.leaf256 = t->cfg.leaf256;
    lt.full256 = t->cfg.full256;
    lt.l2_hint = t->cfg.item_l2_hint;
    lt.full_mask = full_mask(t, d.level);
    static bool attr_set = false;
    if (!attr_set) {
      HBT_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024));
      attr_set = true;
    }
    ItemDir dd = d;
    // Warp rounds per work item: 16, or 8 when the leaf lines the in-flight items reach
    // (one item per SM, each anywhere in its bucket's leaf range) exceed twice the L2:
    // smaller items keep the concurrently searched buckets -- and the DRAM rows their leaf
    // reads open -- closer together.  c4: 148 items x 16 K queries reach ~300 MB of leaf
    // lines, 8 rounds: item search 8.9 -> 8.1-8.3 ms (4 rounds: 8.9, the per-item directory
    // copy is exposed); c5 (74 MB) keeps 16.  Random-line probe over a sliding window:
    // 36 G lines/s over 512 MB, 44 over 128 MB, 59 over 32 MB (profiles/r02s_*).
    uint32_t rcap = t->cfg.item_rounds;
    if (!rcap) {
      static int l2 = 0;
      if (!l2) HBT_CUDA_TRY(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, t->device));
      const double reach = double(t->num_sms) * TH * 16 / double(m) * double(t->leaf_bytes);
      rcap = reach > 2.0 * l2 ? 8 : 16;
    }
    dd.rounds = item_rounds(m, t->num_sms, TH, rcap);
    // the walk resolves directory ties (it detects them on the 256-bit leaf read)
    dd.fix = lt.leaf256 != 0;
    dd.qpf = t->cfg.item_qpf;
    const size_t smem = (size_t(d.cap) + kT16) * 2 + (size_t(d.B) + 1) * 12;
    kern<<<t->num_sms, TH, smem, s>>>((const uint8_t*)t->d_inner, (const uint8_t*)t->d_inner_idx,
                                     (const uint8_t*)t->d_leaf, dd, (const K*)q, m, pf, (K*)v, lt, t->n);
    HBT_CUDA_TRY(cudaGetLastError());
    return HBT_OK;
  }

  static int run(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t b, cudaStream_t s,
                 const void* lp) {
    // small batches read the directory in place with 256-thread CTAs, so a one-wave
    // batch spreads over every SM (c1: 10.1 -> 8.3 us per batch)
    if (t->cfg.mode == 3 || (t->cfg.mode == 2 && m <= t->cfg.small_batch)) return run_t<256, 3>(t, q, m, pf, v, b, s, lp);
    // 256-byte nodes (u64, F = 32) need more registers than a 1024-thread CTA allows
    if constexpr (C::NODE_BYTES > 128) return run_t<512, 2>(t, q, m, pf, v, b, s, lp);
    else return run_t<1024, 2>(t, q, m, pf, v, b, s, lp);
  }
};

template <typename K>
int dispatch_f(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t b, cudaStream_t s,
               const void* lp) {
  switch (t->F) {
    case 4: return Launch<K, 4>::run(t, q, m, pf, v, b, s, lp);
    case 8: return Launch<K, 8>::run(t, q, m, pf, v, b, s, lp);
    case 16: return Launch<K, 16>::run(t, q, m, pf, v, b, s, lp);
    case 32: return Launch<K, 32>::run(t, q, m, pf, v, b, s, lp);
  }
  set_error("unsupported fanout %u", t->F);
  return HBT_EINVAL;
}

}  // namespace

uint32_t implicit_idx_stride(uint32_t F, uint32_t S) {
  const uint32_t node = F * S;
  if (node <= 32) return 0;
  const uint32_t b = (node / 32) * S;
  return b > 16 ? b : 16;
}

int implicit_search_base(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t base,
                         cudaStream_t s) {
  return implicit_search_leaf(t, q, m, pf, v, base, t->d_leaf, s);
}

int implicit_search_leaf(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t base,
                         const void* lp, cudaStream_t s) {
  if (m == 0) return HBT_OK;
  return t->width == 4 ? dispatch_f<uint32_t>(t, q, m, pf, v, base, s, lp)
                       : dispatch_f<uint64_t>(t, q, m, pf, v, base, s, lp);
}

int implicit_search_items(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, const ItemDir& d,
                          cudaStream_t s) {
  if (m == 0) return HBT_OK;
  auto go = [&](auto tag) -> int {
    using K = decltype(tag);
    if (d.bd) {
      switch (t->F) {
        case 4: return Launch<K, 4>::run_cdir(t, q, m, pf, v, d, s);
        case 8: return Launch<K, 8>::run_cdir(t, q, m, pf, v, d, s);
        case 16: return Launch<K, 16>::run_cdir(t, q, m, pf, v, d, s);
        case 32: return Launch<K, 32>::run_cdir(t, q, m, pf, v, d, s);
      }
    }
    switch (t->F) {
      case 4: return Launch<K, 4>::run_items(t, q, m, pf, v, d, s);
      case 8: return Launch<K, 8>::run_items(t, q, m, pf, v, d, s);
      case 16: return Launch<K, 16>::run_items(t, q, m, pf, v, d, s);
      case 32: return Launch<K, 32>::run_items(t, q, m, pf, v, d, s);
    }
    set_error("unsupported fanout %u", t->F);
    return HBT_EINVAL;
  };
  return t->width == 4 ? go(uint32_t{}) : go(uint64_t{});
}

int implicit_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s) {
  return implicit_search_base(t, q, m, pf, v, 0, s);
}

}  // namespace hbt
