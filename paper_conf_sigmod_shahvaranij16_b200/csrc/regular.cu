// regular.cu — the REGULAR (pointer) tree: build, search, batch update.
//
// Node formats (generalised to fanout F):
//   upper inner node u (pool index, bottom-up, left to right):
//       idx[u]  : NIP = 32/S index entries (one 32 B sector); entry t = the max key
//                 of key line t ("I_s = K_8s"), entries >= NI are MAX
//       keys[u] : F separator keys = max key of child i for i < cnt-1, else MAX
//       refs[u] : F uint32 child references (pool indices)
//   last-level inner node v and big leaf v share the pool index v:
//       lidx[v], lkeys[v] : as above over the F lines of big leaf v
//       leaf[v]           : F lines of 64 B = [P keys | P values], dense-packed
//       count[v]          : entries in big leaf v (node fragmentation)
//   chain : live big leaves in key order.
// Search = three dependent accesses per upper level (index sector -> one 64 B
// key line -> one reference), two at the last level, one leaf line;
// the leaf's MAX padding needs no size except when the slot holds MAX.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_select.cuh>

#include <algorithm>

#include "block_util.cuh"
#include "hbt_internal.cuh"
#include "item_dir.cuh"

namespace hbt {
namespace {

constexpr uint64_t kEnd = HBT_POS_END;
constexpr uint64_t kFound = HBT_FOUND_BIT;
constexpr uint32_t kNoRef = 0xFFFFFFFFu;

template <typename K>
__host__ __device__ constexpr K key_max() { return K(~K(0)); }

inline unsigned grid_for(uint64_t n) {
  uint64_t g = (n + 255) / 256;
  if (g > 148 * 64) g = 148 * 64;
  return unsigned(g ? g : 1);
}

#define GRID_STRIDE(i, n) \
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < (n); i += uint64_t(gridDim.x) * blockDim.x)

template <typename K>
struct Geo {
  static constexpr uint32_t S = sizeof(K);
  static constexpr uint32_t P = 64 / (2 * S);
  static constexpr uint32_t KPL = 64 / S;  // keys per 64 B key line
  static constexpr uint32_t NIP = 32 / S;  // index entries per 32 B sector
};

// ---------------------------------------------------------------- build kernels

template <typename K>
__global__ void pack_big_leaves(const K* __restrict__ kd, const K* __restrict__ vd, uint64_t nd, uint64_t nb,
                                uint32_t F, K* __restrict__ leaf, uint32_t* __restrict__ count) {
  constexpr uint32_t P = Geo<K>::P;
  const uint64_t B = uint64_t(F) * P;
  GRID_STRIDE(x, nb * B) {
    const uint64_t v = x / B, e = x % B;
    const uint64_t lo = v * nd / nb, hi = (v + 1) * nd / nb;  // nd < 2^32: no overflow
    K* line = leaf + (v * F + e / P) * (2 * P);
    const bool real = e < hi - lo;
    line[e % P] = real ? kd[lo + e] : key_max<K>();
    line[P + e % P] = real ? vd[lo + e] : K(0);
    if (e == 0) count[v] = uint32_t(hi - lo);
  }
}

// Last-level inner node v from big leaf v: sep[j] = max of line j for j < lines-1.
template <typename K>
__global__ void derive_last_level(const K* __restrict__ leaf, const uint32_t* __restrict__ count, uint64_t pool,
                                  uint32_t F, const uint8_t* __restrict__ dirty, K* __restrict__ lkeys,
                                  K* __restrict__ lidx) {
  constexpr uint32_t P = Geo<K>::P, KPL = Geo<K>::KPL, NIP = Geo<K>::NIP;
  const uint32_t NI = F > KPL ? F / KPL : 1;
  GRID_STRIDE(v, pool) {
    if (dirty && !dirty[v]) continue;
    const uint32_t c = count[v];
    const uint32_t lines = c == 0 ? 1 : (c + P - 1) / P;
    K* sep = lkeys + v * F;
    for (uint32_t j = 0; j < F; ++j)
      sep[j] = (j + 1 < lines) ? leaf[(v * F + j) * (2 * P) + (P - 1)] : key_max<K>();
    for (uint32_t t = 0; t < NIP; ++t) {
      uint32_t slot = t * KPL + KPL - 1;
      if (slot > F - 1) slot = F - 1;
      lidx[v * NIP + t] = t < NI ? sep[slot] : key_max<K>();
    }
  }
}

__global__ void iota_chain(uint32_t* chain, uint64_t n) {
  GRID_STRIDE(i, n) chain[i] = uint32_t(i);
}

template <typename K>
__global__ void chain_leaf_max(const K* __restrict__ leaf, const uint32_t* __restrict__ count,
                               const uint32_t* __restrict__ chain, uint64_t nchain, uint32_t F, K* __restrict__ mx) {
  constexpr uint32_t P = Geo<K>::P;
  GRID_STRIDE(i, nchain) {
    const uint64_t v = chain[i];
    const uint32_t c = count[v];
    mx[i] = c ? leaf[(v * F + (c - 1) / P) * (2 * P) + (c - 1) % P] : key_max<K>();
  }
}

// One upper level: node j groups children [jF, jF+cnt) of the level below.
template <typename K>
__global__ void build_upper_level(const uint32_t* __restrict__ child_ids, uint64_t child_base, const K* __restrict__ child_max,
                                  uint64_t cnt_below, uint64_t nodes, uint64_t node_base, uint32_t F,
                                  K* __restrict__ ukeys, K* __restrict__ uidx, uint32_t* __restrict__ urefs,
                                  K* __restrict__ out_max) {
  constexpr uint32_t KPL = Geo<K>::KPL, NIP = Geo<K>::NIP;
  const uint32_t NI = F > KPL ? F / KPL : 1;
  GRID_STRIDE(j, nodes) {
    const uint64_t first = j * F;
    const uint64_t cnt = (cnt_below - first < F) ? cnt_below - first : F;
    const uint64_t id = node_base + j;
    K* keys = ukeys + id * F;
    uint32_t* refs = urefs + id * F;
    for (uint32_t i = 0; i < F; ++i) {
      keys[i] = (i + 1 < cnt) ? child_max[first + i] : key_max<K>();
      refs[i] = (i < cnt) ? (child_ids ? child_ids[first + i] : uint32_t(child_base + first + i)) : kNoRef;
    }
    for (uint32_t t = 0; t < NIP; ++t) {
      uint32_t slot = t * KPL + KPL - 1;
      if (slot > F - 1) slot = F - 1;
      uidx[id * NIP + t] = t < NI ? keys[slot] : key_max<K>();
    }
    out_max[j] = child_max[first + cnt - 1];
  }
}

// Directory over root-first level T (search mode 2; same argument as the
// implicit tree's, implicit_build.cu): the descent through levels 0..T-1
// reaches the FIRST level-T node whose max key is >= q (the last node
// otherwise), so node_T(q) = lower_bound(M_T, q) with M_T[j] = max key below
// level-T node j and M_T[last] = MAX.  Level-T nodes sit in key order at pool
// indices uoff + j (upper levels are regrouped in chain order), and node j
// covers chain leaves [j*span, (j+1)*span) with span = F^(U-T).
template <typename K>
__global__ void reg_dir_max(const K* __restrict__ leaf, const uint32_t* __restrict__ count,
                            const uint32_t* __restrict__ chain, uint64_t nchain, uint32_t F, uint64_t nodes,
                            uint64_t span, K* __restrict__ M) {
  constexpr uint32_t P = Geo<K>::P;
  GRID_STRIDE(j, nodes) {
    if (j + 1 == nodes) {
      M[j] = key_max<K>();
    } else {
      uint64_t e = (j + 1) * span;
      if (e > nchain) e = nchain;
      const uint64_t v = chain[e - 1];
      const uint32_t c = count[v];
      M[j] = c ? leaf[(v * F + (c - 1) / P) * (2 * P) + (c - 1) % P] : key_max<K>();
    }
  }
}

template <typename K>
__device__ __forceinline__ uint32_t lower_bound_u(const K* M, uint32_t n, K q) {
  uint32_t lo = 0, hi = n - 1;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (M[mid] < q) lo = mid + 1; else hi = mid;
  }
  return lo;
}

template <typename K>
__global__ void reg_dir_table(const K* __restrict__ M, uint32_t n, uint32_t bits, uint32_t* __restrict__ dir) {
  const uint32_t shift = 8 * sizeof(K) - bits;
  GRID_STRIDE(p, (1ull << bits)) {
    const K first = K(K(p) << shift);
    const K last = K(first | K((K(1) << shift) - 1));
    dir[p] = lower_bound_u(M, n, first) | (lower_bound_u(M, n, last) << 16);
  }
}

// ---------------------------------------------------------------- search kernel

struct RView {
  const uint8_t* leaf;
  const uint32_t* count;
  const uint8_t* lkeys;
  const uint8_t* lidx;
  const uint8_t* ukeys;
  const uint8_t* uidx;
  const uint32_t* urefs;
  uint64_t uoff[HBT_MAX_LEVELS + 1];
  uint32_t U;
  uint32_t leaf256;     // item search: key line and leaf line by 256-bit lane loads
};

template <typename K, int N>
__device__ __forceinline__ K pick(const K (&k)[N], uint32_t slot) {
  K r = k[0];
#pragma unroll
  for (int t = 1; t < N; ++t) r = (slot == uint32_t(t)) ? k[t] : r;
  return r;
}

template <typename K>
union V16 {
  uint4 u;
  K k[16 / sizeof(K)];
};

// 32 B held by one lane, loaded with one 256-bit load (sm_100)
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

template <typename K>
__device__ __forceinline__ void fill_max32(L256<K>& v) {
#pragma unroll
  for (int e = 0; e < 4; ++e) v.u[e] = ~0ull;
}

template <typename K>
__device__ __forceinline__ V16<K> ld16g(const uint8_t* p) {
  V16<K> v;
  v.u = __ldg(reinterpret_cast<const uint4*>(p));
  return v;
}

__device__ __forceinline__ uint32_t ldcs(const uint32_t* p) { return __ldcs(p); }
__device__ __forceinline__ uint64_t ldcs(const uint64_t* p) { return __ldcs(reinterpret_cast<const unsigned long long*>(p)); }
__device__ __forceinline__ void stcs(uint32_t* p, uint32_t v) { __stcs(p, v); }
__device__ __forceinline__ void stcs(uint64_t* p, uint64_t v) { __stcs(reinterpret_cast<unsigned long long*>(p), (unsigned long long)v); }


// Search v2 (mode 2, default).  Phase 1: ONE lane per query finds its node at
// root-first level T through the directory + a lower bound over M_T (shared
// memory).  Phase 2: groups of G = 2 lanes per query, 2*QPL queries in flight
// per group: per upper level index sector -> ONE 64 B key line -> one
// reference; last level index -> key line -> line j of big leaf v;
// leaf key sector + value sector.  Every load instruction touches one 32 B
// sector per group; no barriers, no divergence except the MAX slow path.
struct RDir {
  uint32_t T, count, bits;
  uint64_t T_base;  // pool index of level T's first node (T < U), unused when T == U
};

template <typename K, int F, int QPL, int THREADS>
__global__ void __launch_bounds__(THREADS)
regular_search_v2(const RView rv, const RDir rd, const uint32_t* __restrict__ dirbuf,
                  const uint32_t* __restrict__ chain, const K* __restrict__ queries, uint64_t m,
                  uint64_t* __restrict__ out_pf, K* __restrict__ out_v) {
  constexpr int G = 2, NG = 16, ROUND = 32 * QPL, QPG = ROUND / NG;
  constexpr uint32_t S = sizeof(K), P = Geo<K>::P, KPL = Geo<K>::KPL;
  constexpr uint32_t E16 = 16 / S;
  constexpr uint32_t NI = uint32_t(F) > KPL ? uint32_t(F) / KPL : 1;
  constexpr uint32_t LINE = uint32_t(F) * S < 64 ? uint32_t(F) * S : 64;  // bytes of one key line
  constexpr int LCH = int(LINE / 16);                                      // 16 B chunks in it (1..4)
  extern __shared__ __align__(16) uint8_t smem[];
  {
    const uint32_t words = (rd.count * S + (4u << rd.bits)) / 4;
    uint32_t* w = reinterpret_cast<uint32_t*>(smem);
    for (uint32_t i = threadIdx.x; i < words; i += THREADS) w[i] = __ldg(dirbuf + i);
  }
  __syncthreads();
  const K* s_M = reinterpret_cast<const K*>(smem);
  const uint32_t* s_dir = reinterpret_cast<const uint32_t*>(smem + rd.count * S);

  const int lane = threadIdx.x & 31;
  const int g = lane / G, k = lane % G;
  const unsigned gmask = 3u << (g * G);
  const uint64_t warp = (uint64_t(blockIdx.x) * THREADS + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * THREADS) >> 5;
  const uint64_t rounds = (m + ROUND - 1) / ROUND;
  const uint32_t U = rv.U;

  for (uint64_t r0 = warp; r0 < rounds; r0 += nwarps) {
    const uint64_t base = r0 * ROUND;
    K myq[QPL];
    uint32_t myj[QPL];
#pragma unroll
    for (int u = 0; u < QPL; ++u) {
      const uint64_t i = base + uint64_t(u) * 32 + lane;
      myq[u] = i < m ? ldcs(queries + i) : key_max<K>();
      const uint32_t e = s_dir[uint32_t(myq[u] >> (8 * S - rd.bits))];
      uint32_t lo = e & 0xFFFFu, hi = e >> 16;
      while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (s_M[mid] < myq[u]) lo = mid + 1; else hi = mid;
      }
      myj[u] = lo;
    }
    K q[QPG];
    uint32_t cur[QPG];
#pragma unroll
    for (int j = 0; j < QPG; ++j) {
      const int src = (j * NG) % 32 + g;
      q[j] = __shfl_sync(0xffffffffu, myq[(j * NG) / 32], src);
      const uint32_t pj = __shfl_sync(0xffffffffu, myj[(j * NG) / 32], src);
      cur[j] = rd.T < U ? uint32_t(rd.T_base + pj) : __ldg(chain + pj);
    }
    // ---- upper levels T .. U-1 (root-first), then the last level
    for (uint32_t d = rd.T; d <= U; ++d) {
      const bool last = d == U;
      const uint8_t* idxb = last ? rv.lidx : rv.uidx;
      const uint8_t* keyb = last ? rv.lkeys : rv.ukeys;
      uint32_t t[QPG];
      if constexpr (NI > 1) {
        V16<K> iv[QPG];
#pragma unroll
        for (int j = 0; j < QPG; ++j) iv[j] = ld16g<K>(idxb + uint64_t(cur[j]) * 32 + k * 16);
#pragma unroll
        for (int j = 0; j < QPG; ++j) {
          uint32_t c = 0;
#pragma unroll
          for (uint32_t e = 0; e < E16; ++e) c += __popc(__ballot_sync(0xffffffffu, iv[j].k[e] < q[j]) & gmask);
          t[j] = c;
        }
      } else {
#pragma unroll
        for (int j = 0; j < QPG; ++j) t[j] = 0;
      }
      // one key line: lane k holds 16 B chunks k and k + 2
      V16<K> kv[QPG][2];
#pragma unroll
      for (int j = 0; j < QPG; ++j)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int ch = k + 2 * h;
          if (ch < LCH) kv[j][h] = ld16g<K>(keyb + (uint64_t(cur[j]) * F + t[j] * KPL) * S + ch * 16);
          else {
#pragma unroll
            for (uint32_t e = 0; e < E16; ++e) kv[j][h].k[e] = key_max<K>();
          }
        }
      uint32_t slot[QPG];
#pragma unroll
      for (int j = 0; j < QPG; ++j) {
        uint32_t c = 0;
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
          for (uint32_t e = 0; e < E16; ++e) c += __popc(__ballot_sync(0xffffffffu, kv[j][h].k[e] < q[j]) & gmask);
        slot[j] = t[j] * KPL + c;
      }
      if (last) {
#pragma unroll
        for (int j = 0; j < QPG; ++j) t[j] = slot[j];  // line j of big leaf cur
        // ---- leaf line (cur*F + line): key sector + value sector, 16 B per lane each
        V16<K> lk[QPG], lvv[QPG];
#pragma unroll
        for (int j = 0; j < QPG; ++j) {
          const uint8_t* p = rv.leaf + (uint64_t(cur[j]) * F + t[j]) * 64 + k * 16;
          lk[j] = ld16g<K>(p);
          lvv[j] = ld16g<K>(p + 32);
        }
        uint64_t my_pf[QPG / G];
        K my_v[QPG / G];
#pragma unroll
        for (int j = 0; j < QPG; ++j) {
          uint32_t s = 0;
#pragma unroll
          for (uint32_t e = 0; e < E16; ++e) s += __popc(__ballot_sync(0xffffffffu, lk[j].k[e] < q[j]) & gmask);
          const uint32_t sc = s < P ? s : P - 1;
          const int src = g * G + int(sc / E16);
          const K key_s = __shfl_sync(0xffffffffu, pick(lk[j].k, sc % E16), src);
          const K val_s = __shfl_sync(0xffffffffu, pick(lvv[j].k, sc % E16), src);
          bool end = (s == P);
          if (!end && key_s == key_max<K>()) {
            // MAX slot: padding unless it is a counted entry ("must read the node size")
            const int64_t in_line = int64_t(__ldg(rv.count + cur[j])) - int64_t(t[j]) * P;
            const int64_t lim = in_line < int64_t(P) ? in_line : int64_t(P);
            end = int64_t(s) >= lim;
          }
          const bool found = !end && key_s == q[j];
          if (j % G == k) {
            my_pf[j / G] = end ? kEnd : (((uint64_t(cur[j]) * F + t[j]) * P + s) | (found ? kFound : 0ull));
            my_v[j / G] = found ? val_s : K(0);
          }
        }
#pragma unroll
        for (int tt = 0; tt < QPG / G; ++tt) {
          const uint64_t i = base + uint64_t(k + G * tt) * NG + g;
          if (i < m) {
            stcs(out_pf + i, my_pf[tt]);
            stcs(out_v + i, my_v[tt]);
          }
        }
      } else {
#pragma unroll
        for (int j = 0; j < QPG; ++j) cur[j] = __ldg(rv.urefs + uint64_t(cur[j]) * F + slot[j]);
      }
    }
  }
}


// Bucketed search with a bucket-local directory (bucketed.cu, ItemDir): per item
// of kItemRounds * THREADS consecutive bucketed queries, the true maxima of the
// key lines of the chain leaves [c0, c1] its buckets cover (and their chain
// ids) are staged in shared memory.  A query's (chain leaf c, key line t) =
// lower_bound over them: the root-first descent reaches the first big leaf whose
// max is >= q (every upper separator is its child's max, the last one MAX, R11)
// and in it the first key line whose index entry is >= q, and an index entry
// equals the key line's true max except on the leaf's last used line (MAX),
// where both rules stop anyway.  Then: key line t of last-level node v (one
// 64 B access) -> slot j -> leaf line (v*F + j): two dependent accesses instead
// of three per level.
constexpr int kItemRounds = 16;

// Cooperative copy of cnt elements into shared memory, four loads in flight per thread.
template <typename T>
__device__ __forceinline__ void stage4(T* dst, const T* __restrict__ src, uint32_t cnt, uint32_t threads) {
  for (uint32_t i = threadIdx.x; i < cnt; i += 4 * threads) {
    T x[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) x[u] = i + u * threads < cnt ? __ldg(src + i + u * threads) : T(0);
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (i + u * threads < cnt) dst[i + u * threads] = x[u];
  }
}

template <typename K, int F, int THREADS>
__global__ void __launch_bounds__(THREADS)
regular_search_items_kernel(const RView rv, const ItemDir d, const K* __restrict__ queries, uint64_t m,
                            uint64_t* __restrict__ out_pf, K* __restrict__ out_v) {
  constexpr int G = 2, NG = 16, QPG = 32 / NG;
  constexpr uint32_t S = sizeof(K), P = Geo<K>::P, KPL = Geo<K>::KPL;
  constexpr uint32_t E16 = 16 / S;
  constexpr uint32_t LINE = uint32_t(F) * S < 64 ? uint32_t(F) * S : 64;
  constexpr int LCH = int(LINE / 16);
  const uint64_t W = uint64_t(THREADS) * d.rounds;
  extern __shared__ __align__(16) uint8_t smem[];
  uint64_t* s_bstart = reinterpret_cast<uint64_t*>(smem);
  K* s_M = reinterpret_cast<K*>(s_bstart + d.B + 1);
  uint32_t* s_chain = reinterpret_cast<uint32_t*>(s_M + d.cap);
  uint32_t* s_T = s_chain + d.cap;
  __shared__ uint64_t s_range[2];
  const K* gM = static_cast<const K*>(d.M);
  const uint32_t NI = uint32_t(d.span);
  for (uint32_t i = threadIdx.x; i <= d.B; i += THREADS) s_bstart[i] = d.bstart[i];
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int g = lane / G, k = lane % G;
  const unsigned gmask = 3u << (g * G);
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
      s_range[threadIdx.x] = threadIdx.x ? ((uint64_t(lo) + 1) * d.U) / d.B - 1 : (uint64_t(lo) * d.U) / d.B;
    }
    __syncthreads();
    const uint64_t c0 = s_range[0], c1 = s_range[1];
    const uint32_t cnt = uint32_t((c1 - c0 + 1) * NI);
    const bool in_smem = cnt <= d.cap;
    if (in_smem) {
      stage4(s_M, gM + c0 * NI, cnt, THREADS);
      stage4(s_chain, d.chain + c0, uint32_t(c1 - c0 + 1), THREADS);
    }
    __syncthreads();
    PrefixTab<K> pt{};
    if (in_smem) pt = build_prefix(s_M, cnt, s_T, THREADS);
    __syncthreads();
    const K* M = in_smem ? s_M : gM + c0 * NI;
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
      const uint32_t e = lo < cnt ? lo : cnt - 1;
      const uint32_t myv = in_smem ? s_chain[e / NI] : __ldg(d.chain + c0 + e / NI);
      const uint32_t myt = e % NI;
      K q[QPG];
      uint32_t cur[QPG], t[QPG];
#pragma unroll
      for (int j = 0; j < QPG; ++j) {
        const int src = (j * NG) % 32 + g;
        q[j] = __shfl_sync(0xffffffffu, myq, src);
        cur[j] = __shfl_sync(0xffffffffu, myv, src);
        t[j] = __shfl_sync(0xffffffffu, myt, src);
      }
      uint64_t my_pf = 0;
      K my_v = 0;
      if (LINE >= 32 && rv.leaf256) {
        // 256-bit lane loads: the key line and the leaf line each in ONE 64 B request
        // per group (lane k holds bytes [32k, 32k+32) of the line)
        L256<K> kw[QPG];
#pragma unroll
        for (int j = 0; j < QPG; ++j) {
          if (uint32_t(k) * 32 < LINE) {
            ld32(kw[j], rv.lkeys + (uint64_t(cur[j]) * F + t[j] * KPL) * S + k * 32);
          } else {
            fill_max32(kw[j]);
          }
        }
        uint32_t line[QPG];
#pragma unroll
        for (int j = 0; j < QPG; ++j) {
          uint32_t c = 0;
#pragma unroll
          for (uint32_t x = 0; x < 32 / S; ++x) c += kw[j].k[x] < q[j] ? 1u : 0u;
          c += __shfl_xor_sync(0xffffffffu, c, 1);
          line[j] = t[j] * KPL + c;
        }
        L256<K> lw[QPG];
#pragma unroll
        for (int j = 0; j < QPG; ++j) ld32(lw[j], rv.leaf + (uint64_t(cur[j]) * F + line[j]) * 64 + k * 32);
#pragma unroll
        for (int j = 0; j < QPG; ++j) {
          uint32_t c = 0;
#pragma unroll
          for (uint32_t x = 0; x < P; ++x) c += lw[j].k[x] < q[j] ? 1u : 0u;
          const uint32_t sl = __shfl_sync(0xffffffffu, c, g * G);  // lane 0 holds the keys
          const uint32_t sc = sl < P ? sl : P - 1;
          const K xk = pick(lw[j].k, sc);
          const K key_s = __shfl_sync(0xffffffffu, xk, g * G);
          const K val_s = __shfl_sync(0xffffffffu, xk, g * G + 1);
          bool end = (sl == P);
          if (!end && key_s == key_max<K>()) {
            // MAX slot: padding unless it is a counted entry ("must read the node size")
            const int64_t in_line = int64_t(__ldg(rv.count + cur[j])) - int64_t(line[j]) * P;
            const int64_t lim = in_line < int64_t(P) ? in_line : int64_t(P);
            end = int64_t(sl) >= lim;
          }
          const bool found = !end && key_s == q[j];
          if (j == k) {
            my_pf = end ? kEnd : (((uint64_t(cur[j]) * F + line[j]) * P + sl) | (found ? kFound : 0ull));
            my_v = found ? val_s : K(0);
          }
        }
      } else {
      // key line t of last-level node cur: lane k holds 16 B chunks k and k + 2
      V16<K> kv[QPG][2];
#pragma unroll
      for (int j = 0; j < QPG; ++j)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int ch = k + 2 * h;
          if (ch < LCH) kv[j][h] = ld16g<K>(rv.lkeys + (uint64_t(cur[j]) * F + t[j] * KPL) * S + ch * 16);
          else {
#pragma unroll
            for (uint32_t x = 0; x < E16; ++x) kv[j][h].k[x] = key_max<K>();
          }
        }
      uint32_t line[QPG];
#pragma unroll
      for (int j = 0; j < QPG; ++j) {
        uint32_t c = 0;
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
          for (uint32_t x = 0; x < E16; ++x) c += __popc(__ballot_sync(0xffffffffu, kv[j][h].k[x] < q[j]) & gmask);
        line[j] = t[j] * KPL + c;
      }
      // leaf line (cur*F + line): key sector + value sector, 16 B per lane each
      V16<K> lk[QPG], lvv[QPG];
#pragma unroll
      for (int j = 0; j < QPG; ++j) {
        const uint8_t* p = rv.leaf + (uint64_t(cur[j]) * F + line[j]) * 64 + k * 16;
        lk[j] = ld16g<K>(p);
        lvv[j] = ld16g<K>(p + 32);
      }
#pragma unroll
      for (int j = 0; j < QPG; ++j) {
        uint32_t sl = 0;
#pragma unroll
        for (uint32_t x = 0; x < E16; ++x) sl += __popc(__ballot_sync(0xffffffffu, lk[j].k[x] < q[j]) & gmask);
        const uint32_t sc = sl < P ? sl : P - 1;
        const int src = g * G + int(sc / E16);
        const K key_s = __shfl_sync(0xffffffffu, pick(lk[j].k, sc % E16), src);
        const K val_s = __shfl_sync(0xffffffffu, pick(lvv[j].k, sc % E16), src);
        bool end = (sl == P);
        if (!end && key_s == key_max<K>()) {
          // MAX slot: padding unless it is a counted entry ("must read the node size")
          const int64_t in_line = int64_t(__ldg(rv.count + cur[j])) - int64_t(line[j]) * P;
          const int64_t lim = in_line < int64_t(P) ? in_line : int64_t(P);
          end = int64_t(sl) >= lim;
        }
        const bool found = !end && key_s == q[j];
        if (j == k) {
          my_pf = end ? kEnd : (((uint64_t(cur[j]) * F + line[j]) * P + sl) | (found ? kFound : 0ull));
          my_v = found ? val_s : K(0);
        }
      }
      }
      const uint64_t o = base + uint64_t(k) * NG + g;
      if (o <= p1)  // 16 B record {pos|found, value}: the bucket gather reads records
        __stcs(reinterpret_cast<ulonglong2*>(out_pf) + o, make_ulonglong2(my_pf, (unsigned long long)my_v));
    }
    __syncthreads();
  }
}

// Item search on the COMPRESSED per-bucket LEAF-LINE directory (ItemDir::bd; units =
// the F lines of each chain leaf, M = the line's true max, lines past the leaf's last
// used line repeat the leaf max): a query goes from the directory straight to its leaf
// line (v = chain[c], line j), one dependent access instead of key line + leaf line.
// As in implicit_search_cdir_kernel, items are cut inside one bucket and the bucket's
// 16-bit entries and prefix table are bulk-copied into shared memory per item (plus
// its chain ids).  A single tie can name the line BEFORE the right one (a run of ties,
// including a used line and the padding entries repeating its max, is settled exactly
// by lower_bound16); the leaf then reports "past every real key of the line" (s = P, or
// a MAX padding slot at or past the line's count), which cannot happen on the
// right line of a bucket (q <= sp[b]), so the slot moves to the next line in key order
// (j + 1, or line 0 of the next chain leaf) while inside the bucket.
template <typename K, int F, int THREADS>
__global__ void __launch_bounds__(THREADS)
regular_search_cdir_kernel(const RView rv, const ItemDir d, const K* __restrict__ queries, uint64_t m,
                           uint64_t* __restrict__ out_pf, K* __restrict__ out_v) {
  constexpr int G = 2, NG = 16, QPG = 32 / NG;
  constexpr uint32_t P = Geo<K>::P;
  const uint64_t W = uint64_t(THREADS) * d.rounds;
  const uint32_t B = d.B;
  extern __shared__ __align__(16) uint8_t smem[];
  // [E16: cap | T16: kT16 | chain ids: cap / F + 4, padded to 4 | bucket starts: B + 1 u64 | item starts: B + 1]
  uint16_t* s_E = reinterpret_cast<uint16_t*>(smem);
  uint16_t* s_T = s_E + d.cap;
  uint32_t* s_chain = reinterpret_cast<uint32_t*>(s_T + kT16);
  uint64_t* s_bs = reinterpret_cast<uint64_t*>(s_chain + ((d.cap / F + 4 + 3) & ~3u));
  uint32_t* s_is = reinterpret_cast<uint32_t*>(s_bs + B + 1);
  __shared__ uint64_t bar;
  __shared__ uint32_t s_tmp[32];
  __shared__ uint64_t s_p[2];
  __shared__ BucketDir s_bd;
  const K* gM = static_cast<const K*>(d.M);
  for (uint32_t i = threadIdx.x; i <= B; i += THREADS) s_bs[i] = d.bstart[i];
  __syncthreads();
  for (uint32_t b = threadIdx.x; b < B; b += THREADS) s_is[b] = uint32_t((s_bs[b + 1] - s_bs[b] + W - 1) / W);
  __syncthreads();
  const uint32_t last = s_is[B - 1];
  block_exclusive_scan<THREADS>(s_is, s_is, B, s_tmp);
  if (threadIdx.x == 0) {
    s_is[B] = s_is[B - 1] + last;
    mbar_init(&bar, 1);
    fence_mbar_init();
  }
  __syncthreads();
  const uint32_t items = s_is[B];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int g = lane / G, k = lane % G;
  uint32_t parity = 0;
  for (uint32_t it = blockIdx.x; it < items; it += gridDim.x) {
    if (threadIdx.x == 0) {
      uint32_t lo = 0, hi = B;  // the bucket: largest b with s_is[b] <= it
      while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (s_is[mid] <= it) lo = mid; else hi = mid;
      }
      const uint64_t nb = s_is[lo + 1] - s_is[lo], j = it - s_is[lo];
      const uint64_t c0 = s_bs[lo], cnt = s_bs[lo + 1] - c0;
      s_p[0] = c0 + (cnt * j) / nb;
      s_p[1] = c0 + (cnt * (j + 1)) / nb - 1;
      const BucketDir bd = d.bd[lo];
      s_bd = bd;
      fence_proxy_async_smem();  // the previous item's reads of the directory precede this copy
      const uint32_t eb = ((bd.cnt + 7u) & ~7u) * 2u;
      mbar_expect_tx(&bar, eb + kT16 * 2u);
      bulk_g2s(s_E, d.E16 + bd.off16, eb, &bar);
      bulk_g2s(s_T, d.T16 + uint64_t(lo) * kT16, kT16 * 2u, &bar);
    }
    __syncthreads();
    const uint64_t p0 = s_p[0], p1 = s_p[1];
    const uint64_t e0 = s_bd.u0;  // first entry = first chain leaf * F
    const uint32_t cnt = s_bd.cnt, nc = cnt / F;
    for (uint32_t i = threadIdx.x; i < nc; i += THREADS) s_chain[i] = __ldg(d.chain + e0 / F + i);
    mbar_wait(&bar, parity);
    parity ^= 1u;
    __syncthreads();  // chain ids
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
        // the query of the round after next into the L2 now (as implicit_search_cdir_kernel)
        if (d.qpf && r + 1 + int(d.qpf) < int(d.rounds) && i + d.qpf * (THREADS / 32) * 32 <= p1)
          asm volatile("prefetch.global.L2 [%0];" ::"l"(queries + i + d.qpf * (THREADS / 32) * 32));
      }
      const uint32_t a = lower_bound16(s_E, s_T, cnt, myq, K(s_bd.lo), s_bd.sh, s_bd.top, s_bd.ssh, s_bd.esh,
                                       gM + e0, true);
      const uint32_t e = a < cnt ? a : cnt - 1;
      K q[QPG];
      uint32_t cl[QPG], ln[QPG];
#pragma unroll
      for (int j = 0; j < QPG; ++j) {
        const int src = (j * NG) % 32 + g;
        q[j] = __shfl_sync(0xffffffffu, myq, src);
        const uint32_t ej = __shfl_sync(0xffffffffu, e, src);
        cl[j] = ej / F;
        ln[j] = ej % F;
      }
      // leaf line (v*F + line) by two 256-bit lane loads: keys on lane 0, values on lane 1
      L256<K> lw[QPG];
      uint32_t sl[QPG];
      bool end[QPG];
      K key_s[QPG], val_s[QPG];
      auto probe = [&](int j) {
        const uint32_t v = s_chain[cl[j]];
        ld32(lw[j], rv.leaf + (uint64_t(v) * F + ln[j]) * 64 + k * 32);
      };
      auto settle = [&](int j) {  // every lane shuffles
        const uint32_t v = s_chain[cl[j]];
        uint32_t c = 0;
#pragma unroll
        for (uint32_t x = 0; x < P; ++x) c += lw[j].k[x] < q[j] ? 1u : 0u;
        sl[j] = __shfl_sync(0xffffffffu, c, g * G);
        const uint32_t sc = sl[j] < P ? sl[j] : P - 1;
        const K xk = pick(lw[j].k, sc);
        key_s[j] = __shfl_sync(0xffffffffu, xk, g * G);
        val_s[j] = __shfl_sync(0xffffffffu, xk, g * G + 1);
        bool en = (sl[j] == P);
        if (!en && key_s[j] == key_max<K>()) {
          // MAX slot: padding unless it is a counted entry ("must read the node size")
          const int64_t in_line = int64_t(__ldg(rv.count + v)) - int64_t(ln[j]) * P;
          const int64_t lim = in_line < int64_t(P) ? in_line : int64_t(P);
          en = int64_t(sl[j]) >= lim;
        }
        end[j] = en;
      };
#pragma unroll
      for (int j = 0; j < QPG; ++j) probe(j);
#pragma unroll
      for (int j = 0; j < QPG; ++j) settle(j);
#pragma unroll 1
      for (;;) {
        // past the line's real keys before the bucket's last line: the next line in key order
        uint32_t adv = 0;
#pragma unroll
        for (int j = 0; j < QPG; ++j) {
          if (!end[j]) continue;
          const uint32_t v = s_chain[cl[j]];
          const uint32_t used = (__ldg(rv.count + v) + P - 1) / P;
          if (ln[j] + 1 < used) {
            ++ln[j];
            adv |= 1u << j;
          } else if (cl[j] + 1 < nc) {
            ++cl[j];
            ln[j] = 0;
            adv |= 1u << j;
          }
        }
        if (!__any_sync(0xffffffffu, adv != 0)) break;
#pragma unroll
        for (int j = 0; j < QPG; ++j)
          if ((adv >> j) & 1u) probe(j);
#pragma unroll
        for (int j = 0; j < QPG; ++j) settle(j);  // unchanged slots settle to the same result
      }
      uint64_t my_pf = 0;
      K my_v = 0;
#pragma unroll
      for (int j = 0; j < QPG; ++j) {
        const uint32_t v = s_chain[cl[j]];
        const bool found = !end[j] && key_s[j] == q[j];
        if (j == k) {
          my_pf = end[j] ? kEnd : (((uint64_t(v) * F + ln[j]) * P + sl[j]) | (found ? kFound : 0ull));
          my_v = found ? val_s[j] : K(0);
        }
      }
      const uint64_t o = base + uint64_t(k) * NG + g;
      if (o <= p1)  // 16 B record {pos|found, value}: the bucket gather reads records
        __stcs(reinterpret_cast<ulonglong2*>(out_pf) + o, make_ulonglong2(my_pf, (unsigned long long)my_v));
    }
    __syncthreads();
  }
}

template <typename K, int F, int QPL, int THREADS>
int search_v2_launch(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s) {
  const RegularState& r = t->r;
  auto kern = regular_search_v2<K, F, QPL, THREADS>;
  RView rv{};
  rv.leaf = (const uint8_t*)r.d_leaf;
  rv.count = r.d_count;
  rv.lkeys = (const uint8_t*)r.d_lkeys;
  rv.lidx = (const uint8_t*)r.d_lidx;
  rv.ukeys = (const uint8_t*)r.d_ukeys;
  rv.uidx = (const uint8_t*)r.d_uidx;
  rv.urefs = r.d_urefs;
  for (uint32_t u = 0; u <= r.U; ++u) rv.uoff[u] = r.uoff[u];
  rv.U = r.U;
  RDir rd{};
  rd.T = r.dir_T;
  rd.count = r.dir_count;
  rd.bits = r.dir_bits;
  rd.T_base = r.dir_T < r.U ? r.uoff[r.U - 1 - r.dir_T] : 0;
  const size_t smem = r.dir_bytes;
  static bool attr = false;
  if (!attr) {
    HBT_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
    attr = true;
  }
  static size_t occ_smem = ~size_t(0);
  static int occ_cached = 0;
  if (occ_smem != smem) {
    HBT_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_cached, kern, THREADS, smem));
    occ_smem = smem;
  }
  int occ = occ_cached;
  if (t->cfg.ctas_per_sm && int(t->cfg.ctas_per_sm) < occ) occ = int(t->cfg.ctas_per_sm);
  if (occ < 1) occ = 1;
  const uint64_t rounds = (m + 32 * QPL - 1) / (32 * QPL);
  uint64_t grid = uint64_t(t->num_sms) * occ;
  const uint64_t need = (rounds + THREADS / 32 - 1) / (THREADS / 32);
  if (need < grid) grid = need ? need : 1;
  cudaLaunchConfig_t lc = {};
  lc.gridDim = dim3(unsigned(grid));
  lc.blockDim = dim3(THREADS);
  lc.dynamicSmemBytes = smem;
  lc.stream = s;
  HBT_CUDA_TRY(cudaLaunchKernelEx(&lc, kern, rv, rd, (const uint32_t*)r.d_dir, (const uint32_t*)r.d_chain, (const K*)q,
                                  m, pf, (K*)v));
  return HBT_OK;
}


template <typename K, int F>
int search_cdir_launch(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, const ItemDir& d,
                          cudaStream_t s) {
  constexpr int TH = 1024;
  const RegularState& r = t->r;
  auto kern = regular_search_cdir_kernel<K, F, TH>;
  RView rv{};
  rv.leaf = (const uint8_t*)r.d_leaf;
  rv.count = r.d_count;
  rv.U = r.U;
  const size_t smem = (size_t(d.cap) + kT16) * 2 + ((size_t(d.cap) / F + 4 + 3) & ~size_t(3)) * 4 +
                      (size_t(d.B) + 1) * 12;
  static bool attr = false;
  if (!attr) {
    HBT_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024));
    attr = true;
  }
  ItemDir dd = d;
  dd.rounds = item_rounds(m, t->num_sms, TH, t->cfg.item_rounds ? t->cfg.item_rounds : 16);
  dd.qpf = t->cfg.item_qpf;
  kern<<<t->num_sms, TH, smem, s>>>(rv, dd, (const K*)q, m, pf, (K*)v);
  HBT_CUDA_TRY(cudaGetLastError());
  return HBT_OK;
}

template <typename K, int F>
int search_items_launch(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, const ItemDir& d,
                        cudaStream_t s) {
  if (d.bd) return search_cdir_launch<K, F>(t, q, m, pf, v, d, s);
  constexpr int TH = 1024;
  const RegularState& r = t->r;
  auto kern = regular_search_items_kernel<K, F, TH>;
  RView rv{};
  rv.leaf = (const uint8_t*)r.d_leaf;
  rv.count = r.d_count;
  rv.lkeys = (const uint8_t*)r.d_lkeys;
  rv.lidx = (const uint8_t*)r.d_lidx;
  rv.U = r.U;
  rv.leaf256 = t->cfg.leaf256;
  const size_t smem = (d.B + 1) * 8 + size_t(d.cap) * (sizeof(K) + 4) + ((1u << kPrefixBits) + 1) * 4;
  static bool attr = false;
  if (!attr) {
    HBT_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
    attr = true;
  }
  ItemDir dd = d;
  dd.rounds = item_rounds(m, t->num_sms, TH, t->cfg.item_rounds ? t->cfg.item_rounds : 16);
  uint64_t grid = t->num_sms;
  const uint64_t items = (m + uint64_t(TH) * dd.rounds - 1) / (uint64_t(TH) * dd.rounds);
  if (items < grid) grid = items ? items : 1;
  kern<<<unsigned(grid), TH, smem, s>>>(rv, dd, (const K*)q, m, pf, (K*)v);
  HBT_CUDA_TRY(cudaGetLastError());
  return HBT_OK;
}

template <typename K, int F>
int search_launch(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s) {
  return search_v2_launch<K, F, 1, 1024>(t, q, m, pf, v, s);
}

template <typename K>
int search_t(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s) {
  switch (t->F) {
    case 4: return search_launch<K, 4>(t, q, m, pf, v, s);
    case 8: return search_launch<K, 8>(t, q, m, pf, v, s);
    case 16: return search_launch<K, 16>(t, q, m, pf, v, s);
    case 32: return search_launch<K, 32>(t, q, m, pf, v, s);
  }
  set_error("unsupported fanout");
  return HBT_EINVAL;
}

// ---------------------------------------------------------------- state management

template <typename K>
int alloc_pool(hbt_tree* t, uint64_t cap) {
  RegularState& r = t->r;
  const uint64_t F = t->F, S = sizeof(K);
  HBT_CUDA_TRY(cudaMalloc(&r.d_leaf, cap * F * 64));
  HBT_CUDA_TRY(cudaMalloc(&r.d_count, cap * 4));
  HBT_CUDA_TRY(cudaMalloc(&r.d_lkeys, cap * F * S));
  HBT_CUDA_TRY(cudaMalloc(&r.d_lidx, cap * 32));
  HBT_CUDA_TRY(cudaMalloc(&r.d_chain, cap * 4));
  r.cap = cap;
  return HBT_OK;
}

// grow the big-leaf pool arrays to hold `need` leaves (copying pool entries)
template <typename K>
int grow_pool(hbt_tree* t, uint64_t need, cudaStream_t s) {
  RegularState& r = t->r;
  if (need <= r.cap) return HBT_OK;
  uint64_t cap = r.cap ? r.cap : 1;
  while (cap < need) cap = cap + cap / 2 + 1;
  const uint64_t F = t->F, S = sizeof(K);
  void *leaf = nullptr, *lkeys = nullptr, *lidx = nullptr;
  uint32_t *count = nullptr, *chain = nullptr;
  void* hleaf = nullptr;
  if (r.h_leaf) {  // L-segment placed in host memory: the grown pool stays there
    if (cudaHostAlloc(&hleaf, cap * F * 64, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) {
      cudaGetLastError();
      set_error("cudaHostAlloc of the grown big-leaf pool failed");
      return HBT_ENOMEM;
    }
    HBT_CUDA_TRY(cudaHostGetDevicePointer(&leaf, hleaf, 0));
  } else {
    HBT_CUDA_TRY(cudaMalloc(&leaf, cap * F * 64));
  }
  HBT_CUDA_TRY(cudaMalloc(&count, cap * 4));
  HBT_CUDA_TRY(cudaMalloc(&lkeys, cap * F * S));
  HBT_CUDA_TRY(cudaMalloc(&lidx, cap * 32));
  HBT_CUDA_TRY(cudaMalloc(&chain, cap * 4));
  HBT_CUDA_TRY(cudaMemcpyAsync(leaf, r.d_leaf, r.pool * F * 64, cudaMemcpyDefault, s));
  HBT_CUDA_TRY(cudaMemcpyAsync(count, r.d_count, r.pool * 4, cudaMemcpyDeviceToDevice, s));
  HBT_CUDA_TRY(cudaMemcpyAsync(lkeys, r.d_lkeys, r.pool * F * S, cudaMemcpyDeviceToDevice, s));
  HBT_CUDA_TRY(cudaMemcpyAsync(lidx, r.d_lidx, r.pool * 32, cudaMemcpyDeviceToDevice, s));
  HBT_CUDA_TRY(cudaMemcpyAsync(chain, r.d_chain, r.nchain * 4, cudaMemcpyDeviceToDevice, s));
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  if (r.h_leaf) cudaFreeHost(r.h_leaf); else cudaFree(r.d_leaf);
  cudaFree(r.d_count); cudaFree(r.d_lkeys); cudaFree(r.d_lidx); cudaFree(r.d_chain);
  r.d_leaf = leaf; r.h_leaf = hleaf; r.d_count = count; r.d_lkeys = lkeys; r.d_lidx = lidx; r.d_chain = chain;
  r.cap = cap;
  return HBT_OK;
}

// Upper-level node count for a chain of c big leaves (levels bottom-up).
inline uint64_t upper_nodes_for(uint64_t c, uint32_t F) {
  uint64_t total = 0;
  while (c > 1) {
    c = ceil_div_u64(c, F);
    total += c;
  }
  return total;
}

// Before an update mutates anything: grow every array the update and the rebuild after
// it may need (big-leaf pool, upper levels, chain positions), copying the live contents,
// so that an allocation failure leaves the tree unchanged (hbt.h error contract).
template <typename K>
int reserve_for_update(hbt_tree* t, uint64_t pool_need, uint64_t nchain_bound, cudaStream_t s) {
  RegularState& r = t->r;
  const uint32_t F = t->F;
  int rc = grow_pool<K>(t, pool_need, s);
  if (rc != HBT_OK) return rc;
  const uint64_t total = upper_nodes_for(nchain_bound, F);
  if (total > r.ucap) {
    const uint64_t cap = total + total / 4 + 16;
    void *uk = nullptr, *ui = nullptr;
    uint32_t* ur = nullptr;
    auto undo = [&]() { cudaFree(uk); cudaFree(ui); cudaFree(ur); };
    if (cudaMalloc(&uk, cap * F * sizeof(K)) != cudaSuccess || cudaMalloc(&ui, cap * 32) != cudaSuccess ||
        cudaMalloc(&ur, cap * F * 4) != cudaSuccess) {
      cudaGetLastError();
      undo();
      set_error("no device memory for the grown upper levels");
      return HBT_ENOMEM;
    }
    const uint64_t live = r.uoff[r.U];
    if (live) {
      HBT_CUDA_TRY(cudaMemcpyAsync(uk, r.d_ukeys, live * F * sizeof(K), cudaMemcpyDeviceToDevice, s));
      HBT_CUDA_TRY(cudaMemcpyAsync(ui, r.d_uidx, live * 32, cudaMemcpyDeviceToDevice, s));
      HBT_CUDA_TRY(cudaMemcpyAsync(ur, r.d_urefs, live * F * 4, cudaMemcpyDeviceToDevice, s));
    }
    HBT_CUDA_TRY(cudaStreamSynchronize(s));
    cudaFree(r.d_ukeys); cudaFree(r.d_uidx); cudaFree(r.d_urefs);
    r.d_ukeys = uk; r.d_uidx = ui; r.d_urefs = ur; r.ucap = cap;
  }
  if (r.chainpos_cap < r.cap) {
    uint32_t* cp = nullptr;
    HBT_CUDA_TRY(cudaMalloc(&cp, r.cap * 4));
    HBT_CUDA_TRY(cudaMemsetAsync(cp, 0xFF, r.cap * 4, s));
    if (r.chainpos_cap) HBT_CUDA_TRY(cudaMemcpyAsync(cp, r.d_chainpos, r.chainpos_cap * 4, cudaMemcpyDeviceToDevice, s));
    HBT_CUDA_TRY(cudaStreamSynchronize(s));
    cudaFree(r.d_chainpos);
    r.d_chainpos = cp;
    r.chainpos_cap = r.cap;
  }
  return HBT_OK;
}

// Regroup every upper level from the chain (reading R11).  mx: optional
// scratch of 2 x (nchain + 1) keys (the update passes preallocated scratch, so it
// cannot fail for memory after it has modified the leaves).
template <typename K>
int rebuild_upper(hbt_tree* t, cudaStream_t s, K* mx = nullptr) {
  RegularState& r = t->r;
  const uint32_t F = t->F;
  uint64_t c = r.nchain, total = 0;
  uint32_t U = 0;
  uint64_t unodes[HBT_MAX_LEVELS];
  while (c > 1) {
    c = ceil_div_u64(c, F);
    if (U >= HBT_MAX_LEVELS) { set_error("tree too tall"); return HBT_EUNSUPPORTED; }
    unodes[U++] = c;
    total += c;
  }
  if (total > r.ucap) {
    cudaFree(r.d_ukeys); cudaFree(r.d_uidx); cudaFree(r.d_urefs);
    r.d_ukeys = r.d_uidx = nullptr; r.d_urefs = nullptr; r.ucap = 0;
    const uint64_t cap = total + total / 4 + 16;
    HBT_CUDA_TRY(cudaMalloc(&r.d_ukeys, cap * F * sizeof(K)));
    HBT_CUDA_TRY(cudaMalloc(&r.d_uidx, cap * 32));
    HBT_CUDA_TRY(cudaMalloc(&r.d_urefs, cap * F * 4));
    r.ucap = cap;
  }
  r.U = U;
  r.uoff[0] = 0;
  for (uint32_t u = 0; u < U; ++u) {
    r.unodes[u] = unodes[u];
    r.uoff[u + 1] = r.uoff[u] + unodes[u];
  }
  if (U == 0) return HBT_OK;
  K *mx_a = nullptr, *mx_b = nullptr;
  const bool own = mx == nullptr;
  if (own) {
    HBT_CUDA_TRY(scratch_alloc((void**)&mx_a, r.nchain * sizeof(K), s));
    HBT_CUDA_TRY(scratch_alloc((void**)&mx_b, (unodes[0] + 1) * sizeof(K), s));
  } else {
    mx_a = mx;
    mx_b = mx + r.nchain + 1;
  }
  chain_leaf_max<K><<<grid_for(r.nchain), 256, 0, s>>>((const K*)r.d_leaf, r.d_count, r.d_chain, r.nchain, F, mx_a);
  uint64_t below = r.nchain;
  for (uint32_t u = 0; u < U; ++u) {
    build_upper_level<K><<<grid_for(unodes[u]), 256, 0, s>>>(
        u == 0 ? r.d_chain : nullptr, u == 0 ? 0 : r.uoff[u - 1], mx_a, below, unodes[u], r.uoff[u], F,
        (K*)r.d_ukeys, (K*)r.d_uidx, r.d_urefs, mx_b);
    K* tmp = mx_a; mx_a = mx_b; mx_b = tmp;
    below = unodes[u];
  }
  cudaError_t e = cudaGetLastError();
  if (own) {
    scratch_free(mx_a, s);
    scratch_free(mx_b, s);
  }
  cudaStreamSynchronize(s);
  if (e != cudaSuccess) { set_error("rebuild_upper: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
  return HBT_OK;
}

__global__ void chain_positions(const uint32_t* __restrict__ chain, uint64_t nchain, uint32_t* __restrict__ pos) {
  GRID_STRIDE(i, nchain) pos[chain[i]] = uint32_t(i);
}

template <typename K>
int rebuild_dir(hbt_tree* t, cudaStream_t s) {
  RegularState& r = t->r;
  if (r.chainpos_cap < r.cap) {
    cudaFree(r.d_chainpos);
    r.d_chainpos = nullptr;
    r.chainpos_cap = 0;
    HBT_CUDA_TRY(cudaMalloc(&r.d_chainpos, r.cap * 4));
    HBT_CUDA_TRY(cudaMemsetAsync(r.d_chainpos, 0xFF, r.cap * 4, s));  // dead leaves: no position
    r.chainpos_cap = r.cap;
  }
  chain_positions<<<grid_for(r.nchain), 256, 0, s>>>(r.d_chain, r.nchain, r.d_chainpos);
  const uint32_t F = t->F;
  // root-first level d: d < U -> upper level U-1-d, d == U -> the last level (big leaves)
  auto count_at = [&](uint32_t d) -> uint64_t { return d < r.U ? r.unodes[r.U - 1 - d] : r.nchain; };
  uint32_t T = 0;
  for (uint32_t d = 0; d <= r.U; ++d)
    if (count_at(d) * sizeof(K) <= 64 * 1024 && count_at(d) <= 65535) T = d;
  const uint64_t cnt = count_at(T);
  uint64_t span = 1;
  for (uint32_t e = T; e < r.U; ++e) span *= F;
  uint32_t bits = 1;
  while ((1ull << bits) < 4 * cnt && bits < 13) ++bits;
  const uint64_t bytes = cnt * sizeof(K) + (4ull << bits);
  if (bytes > r.dir_cap) {
    cudaFree(r.d_dir);
    r.d_dir = nullptr;
    r.dir_cap = 0;
    const uint64_t cap = 64 * 1024 + (4ull << 13);  // the largest M_T (64 KB) + directory (32 KB)
    HBT_CUDA_TRY(cudaMalloc(&r.d_dir, cap));
    r.dir_cap = cap;
  }
  r.dir_T = T;
  r.dir_count = uint32_t(cnt);
  r.dir_bits = bits;
  r.dir_bytes = bytes;
  K* M = (K*)r.d_dir;
  uint32_t* dir = (uint32_t*)((uint8_t*)r.d_dir + cnt * sizeof(K));
  reg_dir_max<K><<<grid_for(cnt), 256, 0, s>>>((const K*)r.d_leaf, r.d_count, r.d_chain, r.nchain, F, cnt, span, M);
  reg_dir_table<K><<<grid_for(1ull << bits), 256, 0, s>>>(M, uint32_t(cnt), bits, dir);
  HBT_CUDA_TRY(cudaGetLastError());
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  return HBT_OK;
}

template <typename K>
int build_t(hbt_tree* t, const void* keys, const void* values, uint64_t n, cudaStream_t s) {
  RegularState& r = t->r;
  const uint32_t F = t->F;
  r.kpl = Geo<K>::KPL;
  r.NI = F > r.kpl ? F / r.kpl : 1;
  r.B = F * Geo<K>::P;
  r.b = (3 * r.B) / 4;
  void *kd = nullptr, *vd = nullptr;
  uint64_t nd = 0;
  int rc = sort_dedupe(sizeof(K), keys, values, n, &kd, &vd, &nd, s);
  if (rc != HBT_OK) return rc;
  const uint64_t nb = nd == 0 ? 1 : ceil_div_u64(nd, r.b);
  rc = alloc_pool<K>(t, nb + nb / 8 + 16);
  if (rc != HBT_OK) { scratch_free(kd, s); scratch_free(vd, s); return rc; }
  r.pool = nb;
  r.nchain = nb;
  r.root_leaf = 0;
  t->n = nd;
  pack_big_leaves<K><<<grid_for(nb * r.B), 256, 0, s>>>((const K*)kd, (const K*)vd, nd, nb, F, (K*)r.d_leaf, r.d_count);
  derive_last_level<K><<<grid_for(nb), 256, 0, s>>>((const K*)r.d_leaf, r.d_count, nb, F, nullptr, (K*)r.d_lkeys,
                                                     (K*)r.d_lidx);
  iota_chain<<<grid_for(nb), 256, 0, s>>>(r.d_chain, nb);
  cudaError_t e = cudaGetLastError();
  scratch_free(kd, s);
  scratch_free(vd, s);
  cudaStreamSynchronize(s);
  if (e != cudaSuccess) { set_error("regular build: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
  int rc2 = rebuild_upper<K>(t, s);
  return rc2 != HBT_OK ? rc2 : rebuild_dir<K>(t, s);
}

// ---------------------------------------------------------------- update kernels

// Scalar descent of one op key to its big leaf (stops above the last level).
template <typename K>
__global__ void locate_leaf(const K* __restrict__ keys, uint64_t m, const K* __restrict__ ukeys,
                            const K* __restrict__ uidx, const uint32_t* __restrict__ urefs, uint64_t root,
                            uint32_t U, uint32_t root_leaf, uint32_t F, uint32_t* __restrict__ leaf_of) {
  constexpr uint32_t KPL = Geo<K>::KPL, NIP = Geo<K>::NIP;
  const uint32_t NI = F > KPL ? F / KPL : 1;
  GRID_STRIDE(x, m) {
    const K q = keys[x];
    uint64_t cur = U ? root : root_leaf;
    for (uint32_t l = 0; l < U; ++l) {
      uint32_t base = 0, len = F;
      if (NI > 1) {
        uint32_t t = 0;
        for (uint32_t e = 0; e < NI; ++e) t += uidx[cur * NIP + e] < q;
        base = t * KPL;
        len = KPL;
      }
      uint32_t i = base;
      for (uint32_t e = 0; e < len; ++e) i += ukeys[cur * F + base + e] < q;
      cur = urefs[cur * F + i];
    }
    leaf_of[x] = uint32_t(cur);
  }
}

__global__ void iota_u32(uint32_t* p, uint64_t n) { GRID_STRIDE(i, n) p[i] = uint32_t(i); }

template <typename K>
__global__ void last_of_run(const K* __restrict__ sk, uint64_t n, uint8_t* __restrict__ f) {
  GRID_STRIDE(i, n) f[i] = (i + 1 == n) || (sk[i] != sk[i + 1]);
}

template <typename K>
__global__ void gather_ops(const uint32_t* __restrict__ idx, uint64_t n, const K* __restrict__ bv,
                           const uint8_t* __restrict__ bo, K* __restrict__ ov, uint8_t* __restrict__ oo) {
  GRID_STRIDE(i, n) {
    ov[i] = bv[idx[i]];
    oo[i] = bo[idx[i]];
  }
}

__global__ void segment_flags(const uint32_t* __restrict__ leaf_of, uint64_t m, uint32_t* __restrict__ start_flag) {
  GRID_STRIDE(i, m) start_flag[i] = (i == 0 || leaf_of[i] != leaf_of[i - 1]) ? 1u : 0u;
}

// segment s = ops [seg_off[s], seg_off[s+1]) of leaf seg_leaf[s]
__global__ void segment_tables(const uint32_t* __restrict__ leaf_of, const uint32_t* __restrict__ seg_incl, uint64_t m,
                               uint32_t* __restrict__ seg_off, uint32_t* __restrict__ seg_leaf) {
  GRID_STRIDE(i, m) {
    if (i == 0 || leaf_of[i] != leaf_of[i - 1]) {
      const uint32_t sgi = seg_incl[i] - 1;
      seg_off[sgi] = uint32_t(i);
      seg_leaf[sgi] = leaf_of[i];
    }
    if (i + 1 == m) seg_off[seg_incl[i]] = uint32_t(m);
  }
}

// leaf -> its update segment (tree-owned map, reset to "none" after the update)
__global__ void mark_seg_of_leaf(const uint32_t* __restrict__ seg_leaf, uint64_t nseg, uint32_t* __restrict__ seg_of_leaf) {
  GRID_STRIDE(sg, nseg) seg_of_leaf[seg_leaf[sg]] = uint32_t(sg);
}

// Big-leaf entry e of leaf v (dense order): line e/P, slot e%P.
template <typename K>
__device__ __forceinline__ K leaf_key(const K* leaf, uint64_t v, uint32_t F, uint32_t e) {
  constexpr uint32_t P = Geo<K>::P;
  return leaf[(v * F + e / P) * (2 * P) + e % P];
}

// Per op: lower bound in its leaf, found?, inserted?, count delta.
template <typename K>
__global__ void op_classify(const K* __restrict__ ok, const uint8_t* __restrict__ oo, uint64_t m,
                            const uint32_t* __restrict__ leaf_of, const uint32_t* __restrict__ seg_incl,
                            const K* __restrict__ leaf, const uint32_t* __restrict__ count, uint32_t F,
                            uint32_t* __restrict__ lb, uint32_t* __restrict__ ins, int* __restrict__ seg_delta) {
  GRID_STRIDE(x, m) {
    const uint64_t v = leaf_of[x];
    const K q = ok[x];
    uint32_t lo = 0, hi = count[v];
    while (lo < hi) {
      const uint32_t mid = (lo + hi) / 2;
      if (leaf_key(leaf, v, F, mid) < q) lo = mid + 1; else hi = mid;
    }
    const bool found = lo < count[v] && leaf_key(leaf, v, F, lo) == q;
    lb[x] = lo;
    const bool is_ins = oo[x] == 0 && !found;
    const bool is_del = oo[x] != 0 && found;
    ins[x] = is_ins ? 1u : 0u;
    const int d = is_ins ? 1 : (is_del ? -1 : 0);
    if (d) atomicAdd(seg_delta + (seg_incl[x] - 1), d);
  }
}

__global__ void segment_counts(const uint32_t* __restrict__ seg_leaf, const int* __restrict__ seg_delta, uint64_t nseg,
                               const uint32_t* __restrict__ count, uint32_t B, uint32_t* __restrict__ new_cnt,
                               uint32_t* __restrict__ extra) {
  GRID_STRIDE(s, nseg) {
    const int64_t c = int64_t(count[seg_leaf[s]]) + seg_delta[s];
    new_cnt[s] = uint32_t(c);
    const uint64_t parts = c == 0 ? 0 : (uint64_t(c) + B - 1) / B;
    extra[s] = parts > 1 ? uint32_t(parts - 1) : 0u;
  }
}

// One warp per affected leaf: merge the leaf's entries with its ops and write
// the result evenly split over ceil(c/B) leaves (the first keeps index v, the
// others get new_base[s] + p - 1), padding every slot past each part's count.
template <typename K, int MAXB>
__global__ void merge_write(const uint32_t* __restrict__ seg_leaf, const uint32_t* __restrict__ seg_off, uint64_t nseg,
                            const uint32_t* __restrict__ new_cnt, const uint32_t* __restrict__ new_base,
                            const K* __restrict__ ok, const K* __restrict__ ov, const uint8_t* __restrict__ oo,
                            const uint32_t* __restrict__ lb, const uint32_t* __restrict__ insx,
                            K* __restrict__ leaf, uint32_t* __restrict__ count, uint8_t* __restrict__ dirty,
                            uint32_t F) {
  constexpr uint32_t P = Geo<K>::P;
  constexpr int WARPS = 4;
  __shared__ K s_k[WARPS][MAXB];
  __shared__ K s_v[WARPS][MAXB];
  __shared__ uint32_t s_del[WARPS][MAXB + 1];  // # deleted entries before index i
  const int w = threadIdx.x / 32, lane = threadIdx.x & 31;
  const uint32_t B = F * P;
  for (uint64_t sg = blockIdx.x * uint64_t(WARPS) + w; sg < nseg; sg += uint64_t(gridDim.x) * WARPS) {
    const uint64_t v = seg_leaf[sg];
    const uint32_t c_old = count[v];
    const uint32_t o0 = seg_off[sg], o1 = seg_off[sg + 1];
    const uint32_t ins0 = insx[o0];
    // stage old entries; resolve each against the ops (binary search in [o0, o1))
    for (uint32_t i = lane; i < c_old; i += 32) {
      const K key = leaf_key(leaf, v, F, i);
      s_k[w][i] = key;
      s_v[w][i] = leaf[(v * F + i / P) * (2 * P) + P + i % P];
    }
    __syncwarp();
    // deleted flags + new values
    for (uint32_t base = 0; base < c_old; base += 32) {
      const uint32_t i = base + lane;
      bool del = false;
      if (i < c_old) {
        const K key = s_k[w][i];
        uint32_t lo = o0, hi = o1;
        while (lo < hi) {
          const uint32_t mid = (lo + hi) / 2;
          if (ok[mid] < key) lo = mid + 1; else hi = mid;
        }
        if (lo < o1 && ok[lo] == key) {
          if (oo[lo] != 0) del = true;
          else s_v[w][i] = ov[lo];
        }
        s_del[w][i] = del;  // temporarily the flag
      }
    }
    __syncwarp();
    // exclusive prefix of deletions (chunked ballot scan)
    uint32_t carry = 0;
    for (uint32_t base = 0; base < c_old; base += 32) {
      const uint32_t i = base + lane;
      const bool f = i < c_old && s_del[w][i];
      const unsigned bal = __ballot_sync(0xffffffffu, f);
      const uint32_t before = carry + __popc(bal & ((1u << lane) - 1u));
      __syncwarp();
      if (i < c_old) s_del[w][i] = before;
      carry += __popc(bal);
      __syncwarp();
    }
    if (lane == 0) s_del[w][c_old] = carry;
    __syncwarp();
    const uint32_t c = new_cnt[sg];
    const uint32_t parts = c == 0 ? 0 : (c + B - 1) / B;
    auto dest = [&](uint32_t rnk, uint64_t& leaf_id, uint32_t& local) {
      // part p holds merged ranks [floor(p c/k), floor((p+1) c/k))
      uint32_t p = uint32_t((uint64_t(rnk + 1) * parts + c - 1) / c) - 1;
      while (p + 1 < parts && uint64_t(p + 1) * c / parts <= rnk) ++p;
      while (p > 0 && uint64_t(p) * c / parts > rnk) --p;
      const uint32_t lo = uint32_t(uint64_t(p) * c / parts);
      leaf_id = p == 0 ? v : uint64_t(new_base[sg]) + p - 1;
      local = rnk - lo;
    };
    auto put = [&](uint64_t id, uint32_t e, K key, K val) {
      K* line = leaf + (id * F + e / P) * (2 * P);
      line[e % P] = key;
      line[P + e % P] = val;
    };
    // surviving old entries
    for (uint32_t i = lane; i < c_old; i += 32) {
      const bool del = s_del[w][i + 1] != s_del[w][i];
      if (del) continue;
      const K key = s_k[w][i];
      uint32_t lo = o0, hi = o1;  // first op >= key
      while (lo < hi) {
        const uint32_t mid = (lo + hi) / 2;
        if (ok[mid] < key) lo = mid + 1; else hi = mid;
      }
      // inserted ops with key < entry key = inserted among [o0, lo)
      const uint32_t ins_before = insx[lo] - ins0;
      const uint32_t r2 = (i - s_del[w][i]) + ins_before;
      uint64_t id; uint32_t local;
      dest(r2, id, local);
      put(id, local, key, s_v[w][i]);
    }
    // inserted ops
    for (uint32_t j = o0 + lane; j < o1; j += 32) {
      const uint32_t l = lb[j];
      const bool found = l < c_old && s_k[w][l] == ok[j];
      if (oo[j] != 0 || found) continue;
      const uint32_t r2 = (l - s_del[w][l]) + (insx[j] - ins0);
      uint64_t id; uint32_t local;
      dest(r2, id, local);
      put(id, local, ok[j], ov[j]);
    }
    // padding + counts of every destination leaf
    const uint32_t np = parts ? parts : 1;
    for (uint32_t p = 0; p < np; ++p) {
      const uint64_t id = p == 0 ? v : uint64_t(new_base[sg]) + p - 1;
      const uint32_t cnt = parts ? uint32_t(uint64_t(p + 1) * c / parts - uint64_t(p) * c / parts) : 0;
      for (uint32_t e = cnt + lane; e < B; e += 32) put(id, e, key_max<K>(), K(0));
      if (lane == 0) {
        count[id] = cnt;
        dirty[id] = 1;
      }
    }
    __syncwarp();
  }
}

// new chain: position i of the old chain expands to its parts (0 if emptied)
__global__ void chain_parts(const uint32_t* __restrict__ chain, uint64_t nchain, const uint32_t* __restrict__ seg_of_leaf,
                            const uint32_t* __restrict__ new_cnt, uint32_t B, uint32_t* __restrict__ parts) {
  GRID_STRIDE(i, nchain) {
    const uint32_t s = seg_of_leaf[chain[i]];
    if (s == kNoRef) parts[i] = 1;
    else parts[i] = new_cnt[s] == 0 ? 0 : (new_cnt[s] + B - 1) / B;
  }
}

__global__ void chain_write(const uint32_t* __restrict__ chain, uint64_t nchain, const uint32_t* __restrict__ seg_of_leaf,
                            const uint32_t* __restrict__ parts, const uint32_t* __restrict__ pos,
                            const uint32_t* __restrict__ new_base, uint32_t* __restrict__ out) {
  GRID_STRIDE(i, nchain) {
    const uint32_t v = chain[i];
    const uint32_t s = seg_of_leaf[v];
    for (uint32_t p = 0; p < parts[i]; ++p) out[pos[i] + p] = p == 0 ? v : new_base[s] + p - 1;
  }
}

__global__ void reset_seg_of_leaf(const uint32_t* __restrict__ seg_leaf, uint64_t nseg, uint32_t* __restrict__ seg_of_leaf) {
  GRID_STRIDE(s, nseg) seg_of_leaf[seg_leaf[s]] = kNoRef;
}

__global__ void add_base(uint32_t* __restrict__ x, uint64_t n, uint64_t base) {
  GRID_STRIDE(i, n) x[i] = uint32_t(x[i] + base);
}

template <typename K>
__global__ void clear_leaf0(K* leaf, uint32_t* count, uint32_t* chain, uint32_t F, uint8_t* dirty) {
  constexpr uint32_t P = Geo<K>::P;
  for (uint32_t e = threadIdx.x; e < F * P; e += blockDim.x) {
    leaf[(e / P) * (2 * P) + e % P] = key_max<K>();
    leaf[(e / P) * (2 * P) + P + e % P] = K(0);
  }
  if (threadIdx.x == 0) { count[0] = 0; chain[0] = 0; dirty[0] = 1; }
}

__global__ void chain_count_sum(const uint32_t* __restrict__ chain, uint64_t nchain, const uint32_t* __restrict__ count,
                                unsigned long long* __restrict__ sum) {
  unsigned long long local = 0;
  GRID_STRIDE(i, nchain) local += count[chain[i]];
  if (local) atomicAdd(sum, local);
}

// Update scratch from the stream-ordered pool (freed on the update's stream).
struct DevBuf {
  void* p = nullptr;
  cudaStream_t s = nullptr;
  ~DevBuf() { scratch_free(p, s); }
  template <typename T> T* as() { return static_cast<T*>(p); }
};

template <typename K>
int update_t(hbt_tree* t, const hbt_batch* b, cudaStream_t s) {
  RegularState& r = t->r;
  const uint32_t F = t->F, B = r.B;
  const uint64_t m0 = b->count;
  if (m0 >= (1ull << 32)) { set_error("batch too large"); return HBT_EUNSUPPORTED; }
  // 1. sort ops by key (stable), last op per key wins
  DevBuf sk, sidx, idx, flags, tmp, dk, didx, dv, dop, nsel;
  sk.s = s;
  HBT_CUDA_TRY(scratch_alloc(&sk.p, m0 * sizeof(K), s));
  idx.s = s;
  HBT_CUDA_TRY(scratch_alloc(&idx.p, m0 * 4, s));
  sidx.s = s;
  HBT_CUDA_TRY(scratch_alloc(&sidx.p, m0 * 4, s));
  flags.s = s;
  HBT_CUDA_TRY(scratch_alloc(&flags.p, m0, s));
  dk.s = s;
  HBT_CUDA_TRY(scratch_alloc(&dk.p, m0 * sizeof(K), s));
  didx.s = s;
  HBT_CUDA_TRY(scratch_alloc(&didx.p, m0 * 4, s));
  dv.s = s;
  HBT_CUDA_TRY(scratch_alloc(&dv.p, m0 * sizeof(K), s));
  dop.s = s;
  HBT_CUDA_TRY(scratch_alloc(&dop.p, m0, s));
  nsel.s = s;
  HBT_CUDA_TRY(scratch_alloc(&nsel.p, 8, s));
  iota_u32<<<grid_for(m0), 256, 0, s>>>(idx.as<uint32_t>(), m0);
  size_t tb = 0, tb2 = 0;
  HBT_CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, (const K*)b->keys, sk.as<K>(), idx.as<uint32_t>(),
                                               sidx.as<uint32_t>(), m0, 0, int(8 * sizeof(K)), s));
  HBT_CUDA_TRY(cub::DeviceSelect::Flagged(nullptr, tb2, sk.as<K>(), flags.as<uint8_t>(), dk.as<K>(),
                                          nsel.as<int64_t>(), int64_t(m0), s));
  if (tb2 > tb) tb = tb2;
  tmp.s = s;
  HBT_CUDA_TRY(scratch_alloc(&tmp.p, tb, s));
  HBT_CUDA_TRY(cub::DeviceRadixSort::SortPairs(tmp.p, tb, (const K*)b->keys, sk.as<K>(), idx.as<uint32_t>(),
                                               sidx.as<uint32_t>(), m0, 0, int(8 * sizeof(K)), s));
  last_of_run<K><<<grid_for(m0), 256, 0, s>>>(sk.as<K>(), m0, flags.as<uint8_t>());
  HBT_CUDA_TRY(cub::DeviceSelect::Flagged(tmp.p, tb, sk.as<K>(), flags.as<uint8_t>(), dk.as<K>(), nsel.as<int64_t>(),
                                          int64_t(m0), s));
  HBT_CUDA_TRY(cub::DeviceSelect::Flagged(tmp.p, tb, sidx.as<uint32_t>(), flags.as<uint8_t>(), didx.as<uint32_t>(),
                                          nsel.as<int64_t>(), int64_t(m0), s));
  int64_t hm = 0;
  HBT_CUDA_TRY(cudaMemcpyAsync(&hm, nsel.p, 8, cudaMemcpyDeviceToHost, s));
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  const uint64_t m = uint64_t(hm);
  gather_ops<K><<<grid_for(m), 256, 0, s>>>(didx.as<uint32_t>(), m, (const K*)b->values, b->ops, dv.as<K>(),
                                            dop.as<uint8_t>());
  // 2. locate each op's big leaf through the pre-update tree
  DevBuf leaf_of, start, incl, seg_off, seg_leaf, seg_delta, lb, ins, insx, new_cnt, extra, new_base;
  leaf_of.s = s;
  HBT_CUDA_TRY(scratch_alloc(&leaf_of.p, m * 4, s));
  const uint32_t root_leaf = r.root_leaf;
  locate_leaf<K><<<grid_for(m), 256, 0, s>>>(dk.as<K>(), m, (const K*)r.d_ukeys, (const K*)r.d_uidx, r.d_urefs,
                                             r.U ? r.uoff[r.U] - 1 : 0, r.U, root_leaf, F, leaf_of.as<uint32_t>());
  // 3. segments of ops per leaf (ops are in key order, so are their leaves)
  start.s = s;
  HBT_CUDA_TRY(scratch_alloc(&start.p, m * 4, s));
  incl.s = s;
  HBT_CUDA_TRY(scratch_alloc(&incl.p, m * 4, s));
  segment_flags<<<grid_for(m), 256, 0, s>>>(leaf_of.as<uint32_t>(), m, start.as<uint32_t>());
  tb2 = 0;
  HBT_CUDA_TRY(cub::DeviceScan::InclusiveSum(nullptr, tb2, start.as<uint32_t>(), incl.as<uint32_t>(), m, s));
  DevBuf tmp2;
  tmp2.s = s;
  HBT_CUDA_TRY(scratch_alloc(&tmp2.p, tb2 + 256, s));
  HBT_CUDA_TRY(cub::DeviceScan::InclusiveSum(tmp2.p, tb2, start.as<uint32_t>(), incl.as<uint32_t>(), m, s));
  uint32_t nseg32 = 0;
  HBT_CUDA_TRY(cudaMemcpyAsync(&nseg32, incl.as<uint32_t>() + (m - 1), 4, cudaMemcpyDeviceToHost, s));
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  const uint64_t nseg = nseg32;
  seg_off.s = s;
  HBT_CUDA_TRY(scratch_alloc(&seg_off.p, (nseg + 1) * 4, s));
  seg_leaf.s = s;
  HBT_CUDA_TRY(scratch_alloc(&seg_leaf.p, nseg * 4, s));
  seg_delta.s = s;
  HBT_CUDA_TRY(scratch_alloc(&seg_delta.p, nseg * 4, s));
  HBT_CUDA_TRY(cudaMemsetAsync(seg_delta.p, 0, nseg * 4, s));
  segment_tables<<<grid_for(m), 256, 0, s>>>(leaf_of.as<uint32_t>(), incl.as<uint32_t>(), m, seg_off.as<uint32_t>(),
                                             seg_leaf.as<uint32_t>());
  // 4. classify ops against their leaf; new counts; new pool indices (key order)
  lb.s = s;
  HBT_CUDA_TRY(scratch_alloc(&lb.p, m * 4, s));
  ins.s = s;
  HBT_CUDA_TRY(scratch_alloc(&ins.p, (m + 1) * 4, s));
  insx.s = s;
  HBT_CUDA_TRY(scratch_alloc(&insx.p, (m + 1) * 4, s));
  HBT_CUDA_TRY(cudaMemsetAsync(ins.p, 0, (m + 1) * 4, s));
  op_classify<K><<<grid_for(m), 256, 0, s>>>(dk.as<K>(), dop.as<uint8_t>(), m, leaf_of.as<uint32_t>(),
                                             incl.as<uint32_t>(), (const K*)r.d_leaf, r.d_count, F, lb.as<uint32_t>(),
                                             ins.as<uint32_t>(), seg_delta.as<int>());
  HBT_CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb2, ins.as<uint32_t>(), insx.as<uint32_t>(), m + 1, s));
  DevBuf tmp3;
  tmp3.s = s;
  HBT_CUDA_TRY(scratch_alloc(&tmp3.p, tb2 + 256, s));
  HBT_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp3.p, tb2, ins.as<uint32_t>(), insx.as<uint32_t>(), m + 1, s));
  new_cnt.s = s;
  HBT_CUDA_TRY(scratch_alloc(&new_cnt.p, nseg * 4, s));
  extra.s = s;
  HBT_CUDA_TRY(scratch_alloc(&extra.p, nseg * 4, s));
  new_base.s = s;
  HBT_CUDA_TRY(scratch_alloc(&new_base.p, (nseg + 1) * 4, s));
  segment_counts<<<grid_for(nseg), 256, 0, s>>>(seg_leaf.as<uint32_t>(), seg_delta.as<int>(), nseg, r.d_count, B,
                                                new_cnt.as<uint32_t>(), extra.as<uint32_t>());
  DevBuf tmp4;
  HBT_CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb2, extra.as<uint32_t>(), new_base.as<uint32_t>(), nseg + 0, s));
  tmp4.s = s;
  HBT_CUDA_TRY(scratch_alloc(&tmp4.p, tb2 + 256, s));
  HBT_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp4.p, tb2, extra.as<uint32_t>(), new_base.as<uint32_t>(), nseg, s));
  uint32_t last_base = 0, last_extra = 0;
  HBT_CUDA_TRY(cudaMemcpyAsync(&last_base, new_base.as<uint32_t>() + nseg - 1, 4, cudaMemcpyDeviceToHost, s));
  HBT_CUDA_TRY(cudaMemcpyAsync(&last_extra, extra.as<uint32_t>() + nseg - 1, 4, cudaMemcpyDeviceToHost, s));
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  const uint64_t n_new = uint64_t(last_base) + last_extra;
  const uint64_t old_pool = r.pool;
  if (old_pool + n_new >= (1ull << 32) - 1) { set_error("pool index overflow"); return HBT_EUNSUPPORTED; }
  // ---- every allocation of the update happens before its first change to the tree
  //      (hbt.h: on error the tree is unchanged)
  const uint64_t nchain_bound = r.nchain + n_new;
  int rc = reserve_for_update<K>(t, old_pool + n_new, nchain_bound, s);
  if (rc != HBT_OK) return rc;
  DevBuf dirty, parts, ppos, nchain_buf, tmp5, mxbuf, sum;
  dirty.s = s;
  HBT_CUDA_TRY(scratch_alloc(&dirty.p, old_pool + n_new, s));
  parts.s = s;
  HBT_CUDA_TRY(scratch_alloc(&parts.p, (r.nchain + 1) * 4, s));
  ppos.s = s;
  HBT_CUDA_TRY(scratch_alloc(&ppos.p, (r.nchain + 1) * 4, s));
  nchain_buf.s = s;
  HBT_CUDA_TRY(scratch_alloc(&nchain_buf.p, (nchain_bound + 1) * 4, s));
  tb2 = 0;
  HBT_CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb2, parts.as<uint32_t>(), ppos.as<uint32_t>(), r.nchain, s));
  tmp5.s = s;
  HBT_CUDA_TRY(scratch_alloc(&tmp5.p, tb2 + 256, s));
  mxbuf.s = s;
  HBT_CUDA_TRY(scratch_alloc(&mxbuf.p, 2 * (nchain_bound + 2) * sizeof(K), s));
  sum.s = s;
  HBT_CUDA_TRY(scratch_alloc(&sum.p, 8, s));
  HBT_CUDA_TRY(cudaMemsetAsync(dirty.p, 0, old_pool + n_new, s));
  // ---- mutation starts here
  add_base<<<grid_for(nseg), 256, 0, s>>>(new_base.as<uint32_t>(), nseg, old_pool);
  mark_seg_of_leaf<<<grid_for(nseg), 256, 0, s>>>(seg_leaf.as<uint32_t>(), nseg, r.d_seg_of_leaf);
  r.pool = old_pool + n_new;
  // 5. merge + split + pad, one warp per affected leaf
  {
    constexpr int MAXB = 32 * Geo<K>::P;  // F <= 32
    const uint64_t blocks = (nseg + 3) / 4;
    merge_write<K, MAXB><<<unsigned(blocks < 148 * 64 ? blocks : 148 * 64), 128, 0, s>>>(
        seg_leaf.as<uint32_t>(), seg_off.as<uint32_t>(), nseg, new_cnt.as<uint32_t>(), new_base.as<uint32_t>(),
        dk.as<K>(), dv.as<K>(), dop.as<uint8_t>(), lb.as<uint32_t>(), insx.as<uint32_t>(), (K*)r.d_leaf, r.d_count,
        dirty.as<uint8_t>(), F);
    HBT_CUDA_TRY(cudaGetLastError());
  }
  // 6. new chain (key order): every old position expands to its parts
  chain_parts<<<grid_for(r.nchain), 256, 0, s>>>(r.d_chain, r.nchain, r.d_seg_of_leaf, new_cnt.as<uint32_t>(), B,
                                                 parts.as<uint32_t>());
  HBT_CUDA_TRY(cub::DeviceScan::ExclusiveSum(tmp5.p, tb2, parts.as<uint32_t>(), ppos.as<uint32_t>(), r.nchain, s));
  uint32_t lp = 0, lpart = 0;
  HBT_CUDA_TRY(cudaMemcpyAsync(&lp, ppos.as<uint32_t>() + r.nchain - 1, 4, cudaMemcpyDeviceToHost, s));
  HBT_CUDA_TRY(cudaMemcpyAsync(&lpart, parts.as<uint32_t>() + r.nchain - 1, 4, cudaMemcpyDeviceToHost, s));
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  const uint64_t new_nchain = uint64_t(lp) + lpart;
  chain_write<<<grid_for(r.nchain), 256, 0, s>>>(r.d_chain, r.nchain, r.d_seg_of_leaf, parts.as<uint32_t>(),
                                                 ppos.as<uint32_t>(), new_base.as<uint32_t>(), nchain_buf.as<uint32_t>());
  reset_seg_of_leaf<<<grid_for(nseg), 256, 0, s>>>(seg_leaf.as<uint32_t>(), nseg, r.d_seg_of_leaf);
  if (new_nchain == 0) {  // every key deleted: the empty tree (one empty leaf at index 0)
    r.pool = 1;
    clear_leaf0<K><<<1, 256, 0, s>>>((K*)r.d_leaf, r.d_count, r.d_chain, F, dirty.as<uint8_t>());
    r.nchain = 1;
  } else {
    HBT_CUDA_TRY(cudaMemcpyAsync(r.d_chain, nchain_buf.p, new_nchain * 4, cudaMemcpyDeviceToDevice, s));
    r.nchain = new_nchain;
  }
  // 7. refresh the last-level inner nodes of dirty leaves, then the upper levels
  derive_last_level<K><<<grid_for(r.pool), 256, 0, s>>>((const K*)r.d_leaf, r.d_count, r.pool, F, dirty.as<uint8_t>(),
                                                         (K*)r.d_lkeys, (K*)r.d_lidx);
  HBT_CUDA_TRY(cudaGetLastError());
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  HBT_CUDA_TRY(cudaMemcpyAsync(&r.root_leaf, r.d_chain, 4, cudaMemcpyDeviceToHost, s));
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  rc = rebuild_upper<K>(t, s, mxbuf.as<K>());
  if (rc != HBT_OK) return rc;
  rc = rebuild_dir<K>(t, s);
  if (rc != HBT_OK) return rc;
  // live key count n' = sum of the chain's counts
  {
    HBT_CUDA_TRY(cudaMemsetAsync(sum.p, 0, 8, s));
    chain_count_sum<<<grid_for(r.nchain), 256, 0, s>>>(r.d_chain, r.nchain, r.d_count, sum.as<unsigned long long>());
    uint64_t nn = 0;
    HBT_CUDA_TRY(cudaMemcpyAsync(&nn, sum.p, 8, cudaMemcpyDeviceToHost, s));
    HBT_CUDA_TRY(cudaStreamSynchronize(s));
    t->n = nn;
  }
  return HBT_OK;
}

}  // namespace

int regular_build(hbt_tree* t, const void* keys, const void* values, uint64_t n, cudaStream_t s) {
  int rc = t->width == 4 ? build_t<uint32_t>(t, keys, values, n, s) : build_t<uint64_t>(t, keys, values, n, s);
  if (rc != HBT_OK) return rc;
  // pool-sized map leaf -> update segment (kept at "none" between updates)
  HBT_CUDA_TRY(cudaMalloc(&t->r.d_seg_of_leaf, t->r.cap * 4));
  HBT_CUDA_TRY(cudaMemset(t->r.d_seg_of_leaf, 0xFF, t->r.cap * 4));
  t->r.seg_cap = t->r.cap;
  return HBT_OK;
}

int regular_search_items(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, const ItemDir& d,
                         cudaStream_t s) {
  if (m == 0) return HBT_OK;
  auto go = [&](auto tag) -> int {
    using K = decltype(tag);
    switch (t->F) {
      case 4: return search_items_launch<K, 4>(t, q, m, pf, v, d, s);
      case 8: return search_items_launch<K, 8>(t, q, m, pf, v, d, s);
      case 16: return search_items_launch<K, 16>(t, q, m, pf, v, d, s);
      case 32: return search_items_launch<K, 32>(t, q, m, pf, v, d, s);
    }
    set_error("unsupported fanout %u", t->F);
    return HBT_EINVAL;
  };
  return t->width == 4 ? go(uint32_t{}) : go(uint64_t{});
}

int regular_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s) {
  if (m == 0) return HBT_OK;
  return t->width == 4 ? search_t<uint32_t>(t, q, m, pf, v, s) : search_t<uint64_t>(t, q, m, pf, v, s);
}

int regular_update(hbt_tree* t, const hbt_batch* b, cudaStream_t s) {
  RegularState& r = t->r;
  // the leaf->segment map must cover the pool after growth: size it for the worst case
  const uint64_t worst = r.pool + b->count + 1;
  if (worst > r.seg_cap) {
    uint32_t* nm = nullptr;
    HBT_CUDA_TRY(cudaMalloc(&nm, worst * 4));
    HBT_CUDA_TRY(cudaMemset(nm, 0xFF, worst * 4));
    cudaFree(r.d_seg_of_leaf);
    r.d_seg_of_leaf = nm;
    r.seg_cap = worst;
  }
  return t->width == 4 ? update_t<uint32_t>(t, b, s) : update_t<uint64_t>(t, b, s);
}

int regular_clone(const hbt_tree* src, hbt_tree* dst, cudaStream_t s) {
  const RegularState& a = src->r;
  RegularState& b = dst->r;
  if (a.h_leaf) { set_error("clone of a host-placed big-leaf pool is not supported"); return HBT_EUNSUPPORTED; }
  const uint64_t F = src->F, S = src->width;
  b = a;  // scalars; every device pointer is replaced below
  b.d_leaf = b.d_lkeys = b.d_lidx = b.d_ukeys = b.d_uidx = b.d_dir = nullptr;
  b.d_count = b.d_chain = b.d_urefs = b.d_seg_of_leaf = b.d_chainpos = nullptr;
  b.h_leaf = nullptr;
  // same capacities; only the live prefix of each array is copied (the rest is
  // never read before it is written)
  auto dup = [&](void** d, const void* p, uint64_t cap_bytes, uint64_t live_bytes) -> int {
    if (!p || !cap_bytes) return HBT_OK;
    HBT_CUDA_TRY(cudaMalloc(d, cap_bytes));
    if (live_bytes) HBT_CUDA_TRY(cudaMemcpyAsync(*d, p, live_bytes, cudaMemcpyDeviceToDevice, s));
    return HBT_OK;
  };
  const uint64_t up = a.uoff[a.U];
  int rc;
  if ((rc = dup(&b.d_leaf, a.d_leaf, a.cap * F * 64, a.pool * F * 64)) ||
      (rc = dup((void**)&b.d_count, a.d_count, a.cap * 4, a.pool * 4)) ||
      (rc = dup(&b.d_lkeys, a.d_lkeys, a.cap * F * S, a.pool * F * S)) ||
      (rc = dup(&b.d_lidx, a.d_lidx, a.cap * 32, a.pool * 32)) ||
      (rc = dup((void**)&b.d_chain, a.d_chain, a.cap * 4, a.nchain * 4)) ||
      (rc = dup(&b.d_ukeys, a.d_ukeys, a.ucap * F * S, up * F * S)) ||
      (rc = dup(&b.d_uidx, a.d_uidx, a.ucap * 32, up * 32)) ||
      (rc = dup((void**)&b.d_urefs, a.d_urefs, a.ucap * F * 4, up * F * 4)) ||
      (rc = dup((void**)&b.d_seg_of_leaf, a.d_seg_of_leaf, a.seg_cap * 4, a.seg_cap * 4)) ||
      (rc = dup(&b.d_dir, a.d_dir, a.dir_cap, a.dir_bytes)) ||
      (rc = dup((void**)&b.d_chainpos, a.d_chainpos, a.chainpos_cap * 4, a.chainpos_cap * 4)))
    return rc;
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  return HBT_OK;
}

void regular_free(hbt_tree* t) {
  RegularState& r = t->r;
  if (r.h_leaf) cudaFreeHost(r.h_leaf); else cudaFree(r.d_leaf);
  cudaFree(r.d_count); cudaFree(r.d_lkeys); cudaFree(r.d_lidx); cudaFree(r.d_chain);
  cudaFree(r.d_ukeys); cudaFree(r.d_uidx); cudaFree(r.d_urefs); cudaFree(r.d_seg_of_leaf); cudaFree(r.d_dir);
  cudaFree(r.d_chainpos);
  r = RegularState{};
}


}  // namespace hbt
