// implicit_search.cu — hbt_search for the IMPLICIT tree (the hot path).
//
// One lane GROUP of G = max(2, F*S/16) lanes searches one node: each lane loads
// 16 B (8 B for 16-byte nodes) of the node with one vector load and the group
// counts the node keys smaller than q with __ballot_sync + __popc:
//   i = #{t : sep[t] < q} = the minimum i with q <= sep[i]   (PAPER.md:190,
//       read with the "k is the minimum i" comments of P:520 / P:566; R1)
// and descends to child node*F + i (Snippet 3's (nodeIndex+result)<<3,
// P:689).  No shared flags and no barriers (Snippet 3 needs two __syncthreads
// per level).  Each group keeps QPG queries in flight level-
// synchronously (the GPU form of the paper's software pipelining, Alg. 2,
// P:600-612), so a warp has 32 independent node loads outstanding per level.
// The top SL levels are staged once per persistent CTA in shared memory (the
// I-segment-in-fast-memory principle of P:178); deeper levels and the leaf line
// come from L2/HBM with read-only loads; queries and results stream with
// evict-first (.cs) accesses so they do not displace the tree from L2.
#include "hbt_internal.cuh"

namespace hbt {
namespace {

constexpr uint64_t kEnd = HBT_POS_END;
constexpr uint64_t kFound = HBT_FOUND_BIT;

template <typename K>
__device__ __forceinline__ K key_max() { return K(~K(0)); }

template <typename K, int BYTES>
struct Chunk {
  static constexpr int N = BYTES / int(sizeof(K));
  K k[N];
};

template <typename K, int BYTES>
__device__ __forceinline__ void ld_global(Chunk<K, BYTES>& c, const uint8_t* p) {
  if constexpr (BYTES == 8) {
    uint2 v = __ldg(reinterpret_cast<const uint2*>(p));
    memcpy(&c, &v, 8);
  } else if constexpr (BYTES == 16) {
    uint4 v = __ldg(reinterpret_cast<const uint4*>(p));
    memcpy(&c, &v, 16);
  } else {
    static_assert(BYTES == 32, "chunk size");
    uint4 v0 = __ldg(reinterpret_cast<const uint4*>(p));
    uint4 v1 = __ldg(reinterpret_cast<const uint4*>(p) + 1);
    memcpy(&c, &v0, 16);
    memcpy(reinterpret_cast<uint8_t*>(&c) + 16, &v1, 16);
  }
}

template <typename K, int BYTES>
__device__ __forceinline__ void ld_shared(Chunk<K, BYTES>& c, const uint8_t* p) {
  if constexpr (BYTES == 8) {
    uint2 v = *reinterpret_cast<const uint2*>(p);
    memcpy(&c, &v, 8);
  } else {
    static_assert(BYTES == 16, "chunk size");
    uint4 v = *reinterpret_cast<const uint4*>(p);
    memcpy(&c, &v, 16);
  }
}

__device__ __forceinline__ uint32_t ldcs(const uint32_t* p) { return __ldcs(p); }
__device__ __forceinline__ uint64_t ldcs(const uint64_t* p) {
  return __ldcs(reinterpret_cast<const unsigned long long*>(p));
}
__device__ __forceinline__ void stcs(uint32_t* p, uint32_t v) { __stcs(p, v); }
__device__ __forceinline__ void stcs(uint64_t* p, uint64_t v) {
  __stcs(reinterpret_cast<unsigned long long*>(p), (unsigned long long)v);
}

template <typename K, int F, int QPG_>
struct Cfg {
  static constexpr int S = int(sizeof(K));
  static constexpr int NODE_BYTES = F * S;
  static constexpr int G = NODE_BYTES / 16 < 2 ? 2 : NODE_BYTES / 16;  // lanes per group
  static constexpr int LANE_BYTES = NODE_BYTES / G;                    // 8 or 16
  static constexpr int NG = 32 / G;                                    // groups per warp
  static constexpr int QPG = QPG_;                                     // queries in flight per group
  static constexpr int ROUND = NG * QPG;                               // queries per warp round
  static constexpr int P = 64 / (2 * S);                               // pairs per leaf line
  static constexpr int LL = G < 4 ? G : 4;                             // lanes loading a leaf line
  static constexpr int LB = 64 / LL;                                   // leaf bytes per lane
  static constexpr int KEY_LANES = LL / 2;                             // lanes holding the key half
  static constexpr int LK = LB / S;                                    // leaf entries per lane
  static_assert(QPG <= G && ROUND <= 32, "tiling");
};

template <typename K, int N>
__device__ __forceinline__ uint32_t count_less(const K (&k)[N], K q, unsigned gmask) {
  uint32_t c = 0;
#pragma unroll
  for (int t = 0; t < N; ++t) c += __popc(__ballot_sync(0xffffffffu, k[t] < q) & gmask);
  return c;
}

template <typename K, int N>
__device__ __forceinline__ K pick(const K (&k)[N], uint32_t slot) {
  K r = k[0];
#pragma unroll
  for (int t = 1; t < N; ++t) r = (slot == uint32_t(t)) ? k[t] : r;
  return r;
}

template <typename K, int F, int QPG, int THREADS>
__global__ void __launch_bounds__(THREADS)
implicit_search_kernel(const uint8_t* __restrict__ inner, const uint8_t* __restrict__ leaf,
                       const K* __restrict__ queries, uint64_t m, uint64_t* __restrict__ out_pf,
                       K* __restrict__ out_v, const LevelTable lt, uint64_t n) {
  using C = Cfg<K, F, QPG>;
  extern __shared__ __align__(16) uint8_t smem[];
  const uint32_t SL = lt.SL, H = lt.H;
  {  // stage the top SL levels (root-first, contiguous) once per persistent CTA
    const uint32_t vecs = uint32_t(lt.offset[SL] * C::NODE_BYTES / 16);
    const uint4* src = reinterpret_cast<const uint4*>(inner);
    uint4* dst = reinterpret_cast<uint4*>(smem);
    for (uint32_t i = threadIdx.x; i < vecs; i += THREADS) dst[i] = __ldg(src + i);
  }
  __syncthreads();

  const int lane = threadIdx.x & 31;
  const int g = lane / C::G, k = lane % C::G;
  const unsigned gmask = ((1u << C::G) - 1u) << (g * C::G);
  const uint64_t warp = (uint64_t(blockIdx.x) * THREADS + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * THREADS) >> 5;
  const uint64_t rounds = (m + C::ROUND - 1) / C::ROUND;

  for (uint64_t rd = warp; rd < rounds; rd += nwarps) {
    // Query j of group g is query base + j*NG + g: lane (g, k<QPG) loads query
    // k of its group, so the warp's load and store are one coalesced segment.
    const uint64_t my_i = rd * C::ROUND + uint64_t(k) * C::NG + g;
    const bool my_ok = (k < QPG) && (my_i < m);
    const K myq = my_ok ? ldcs(queries + my_i) : key_max<K>();
    K q[QPG];
    uint32_t node[QPG];
#pragma unroll
    for (int j = 0; j < QPG; ++j) {
      q[j] = __shfl_sync(0xffffffffu, myq, g * C::G + j);
      node[j] = 0;
    }
    // ---- inner levels pinned in shared memory
    for (uint32_t d = 0; d < SL; ++d) {
      const uint8_t* lvl = smem + uint32_t(lt.offset[d]) * C::NODE_BYTES + k * C::LANE_BYTES;
      Chunk<K, C::LANE_BYTES> c[QPG];
#pragma unroll
      for (int j = 0; j < QPG; ++j) ld_shared(c[j], lvl + node[j] * C::NODE_BYTES);
#pragma unroll
      for (int j = 0; j < QPG; ++j) node[j] = node[j] * F + count_less(c[j].k, q[j], gmask);
    }
    // ---- inner levels in L2 / HBM
    for (uint32_t d = SL; d < H; ++d) {
      const uint8_t* lvl = inner + lt.offset[d] * C::NODE_BYTES + k * C::LANE_BYTES;
      Chunk<K, C::LANE_BYTES> c[QPG];
#pragma unroll
      for (int j = 0; j < QPG; ++j) ld_global(c[j], lvl + uint64_t(node[j]) * C::NODE_BYTES);
#pragma unroll
      for (int j = 0; j < QPG; ++j) node[j] = node[j] * F + count_less(c[j].k, q[j], gmask);
    }
    // ---- leaf line: lanes [0, KEY_LANES) hold the P keys, [KEY_LANES, LL) the P values
    Chunk<K, C::LB> lc[QPG];
#pragma unroll
    for (int j = 0; j < QPG; ++j) {
      if (k < C::LL) {
        ld_global(lc[j], leaf + uint64_t(node[j]) * 64 + k * C::LB);
      } else {
#pragma unroll
        for (int t = 0; t < C::LK; ++t) lc[j].k[t] = key_max<K>();
      }
    }
    uint64_t my_pf = 0;
    K my_v = 0;
#pragma unroll
    for (int j = 0; j < QPG; ++j) {
      uint32_t s = 0;
#pragma unroll
      for (int t = 0; t < C::LK; ++t)
        s += __popc(__ballot_sync(0xffffffffu, (k < C::KEY_LANES) && (lc[j].k[t] < q[j])) & gmask);
      const uint32_t sc = s < uint32_t(C::P) ? s : uint32_t(C::P - 1);
      const K sel = pick(lc[j].k, sc % C::LK);
      const int src = g * C::G + int(sc / C::LK);
      const K key_s = __shfl_sync(0xffffffffu, sel, src);
      const K val_s = __shfl_sync(0xffffffffu, sel, src + C::KEY_LANES);
      const uint64_t r = uint64_t(node[j]) * C::P + s;
      const bool found = (s < uint32_t(C::P)) && (r < n) && (key_s == q[j]);
      if (j == k) {
        my_pf = (r < n ? r : kEnd) | (found ? kFound : 0ull);
        my_v = found ? val_s : K(0);
      }
    }
    if (my_ok) {
      stcs(out_pf + my_i, my_pf);
      stcs(out_v + my_i, my_v);
    }
  }
}

constexpr int kThreads = 512;

template <typename K, int F>
struct Launch {
  static constexpr int G = Cfg<K, F, 1>::G;
  static constexpr int QPG = G < 8 ? G : 8;
  using C = Cfg<K, F, QPG>;

  static auto kernel() { return implicit_search_kernel<K, F, QPG, kThreads>; }

  static int run(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s) {
    auto kern = kernel();
    LevelTable lt{};
    for (uint32_t d = 0; d <= t->H; ++d) lt.offset[d] = t->offset[d];
    lt.H = t->H;
    const uint32_t budget = t->cfg.smem_budget ? t->cfg.smem_budget : default_budget();
    lt.SL = smem_levels(t, budget);
    const size_t smem = size_t(lt.offset[lt.SL]) * C::NODE_BYTES;
    static bool attr_set = false;  // per instantiation
    if (!attr_set) {
      HBT_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
      attr_set = true;
    }
    int occ = 0;
    HBT_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kThreads, smem));
    if (t->cfg.ctas_per_sm && int(t->cfg.ctas_per_sm) < occ) occ = int(t->cfg.ctas_per_sm);
    if (occ < 1) occ = 1;
    const uint64_t rounds = (m + C::ROUND - 1) / C::ROUND;
    const uint64_t warps_per_cta = kThreads / 32;
    uint64_t grid = uint64_t(t->num_sms) * occ;
    const uint64_t need = (rounds + warps_per_cta - 1) / warps_per_cta;
    if (need < grid) grid = need ? need : 1;
    kern<<<unsigned(grid), kThreads, smem, s>>>((const uint8_t*)t->d_inner, (const uint8_t*)t->d_leaf,
                                                (const K*)q, m, pf, (K*)v, lt, t->n);
    HBT_CUDA_TRY(cudaGetLastError());
    return HBT_OK;
  }

  static uint32_t default_budget() {
    // Two resident CTAs per SM share the 228 KB carve-out.
    return 100 * 1024;
  }

  static uint32_t smem_levels(const hbt_tree* t, uint32_t budget) {
    uint32_t SL = 0;
    while (SL < t->H && t->offset[SL + 1] * uint64_t(C::NODE_BYTES) <= budget) ++SL;
    return SL;
  }
};

template <typename K>
int dispatch_f(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s) {
  switch (t->F) {
    case 4: return Launch<K, 4>::run(t, q, m, pf, v, s);
    case 8: return Launch<K, 8>::run(t, q, m, pf, v, s);
    case 16: return Launch<K, 16>::run(t, q, m, pf, v, s);
    case 32: return Launch<K, 32>::run(t, q, m, pf, v, s);
  }
  set_error("unsupported fanout %u", t->F);
  return HBT_EINVAL;
}

template <typename K>
uint32_t smem_levels_f(const hbt_tree* t, uint32_t budget) {
  switch (t->F) {
    case 4: return Launch<K, 4>::smem_levels(t, budget);
    case 8: return Launch<K, 8>::smem_levels(t, budget);
    case 16: return Launch<K, 16>::smem_levels(t, budget);
    case 32: return Launch<K, 32>::smem_levels(t, budget);
  }
  return 0;
}

}  // namespace

int implicit_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s) {
  if (m == 0) return HBT_OK;
  return t->width == 4 ? dispatch_f<uint32_t>(t, q, m, pf, v, s) : dispatch_f<uint64_t>(t, q, m, pf, v, s);
}

uint32_t implicit_smem_levels(const hbt_tree* t, uint32_t budget) {
  if (!budget) budget = 100 * 1024;
  return t->width == 4 ? smem_levels_f<uint32_t>(t, budget) : smem_levels_f<uint64_t>(t, budget);
}

}  // namespace hbt
