// bucketed.cu — query bucketing by key range in front of the tree walk
// (BASELINE.json north_star: "Queries pre-sorted or bucketed per batch so
// neighbouring lanes share upper-level nodes"; the paper's batch-of-queries
// problem statement).
//
// For a tree far larger than the L2, every query of an unordered batch pays
// its own DRAM round trips for the bottom inner levels and the leaf line.  A
// batch that is partitioned into B key-range buckets (each bucket covering a
// tree slice that fits in the L2 with room to spare) and searched bucket after
// bucket lets the queries of a bucket share the slice's lines: they are
// fetched from DRAM about once per bucket instead of once per query.
//
// The batch is cut into chunks of kChunk queries.  Per chunk and bucket the
// queries form one contiguous RUN in the bucketed order (bucket-major, chunk
// order inside a bucket), so both reorderings move whole runs:
//   splitters   sp[b] = max key of unit floor((b+1) U / B) - 1 (units = leaf
//               lines of the implicit tree / chain big leaves of the regular
//               tree), sp[B-1] = MAX; bucket(q) = #{sp < q} (a lower bound, the
//               node-search rule R1 of DESIGN.md applied to the splitters)
//   directory   dir[p] = [bucket(p << sh), bucket(((p+1) << sh) - 1)] over the
//               top D bits of the key, so a query binary-searches a short range
//   bk_count    bucket of every query (u16) + per-chunk histograms tab[b][c]
//   scan        gb = exclusive scan of tab in (bucket, chunk) order = the
//               first global slot of every run (CUB)
//   bk_scatter  per chunk: queries ordered by bucket in shared memory, written
//               as runs; linv[i] = position of query i in the chunk's order
//   search      the normal implicit / regular search kernels on the bucketed
//               queries
//   bk_gather   per chunk: result runs read into shared memory, stored in
//               query order through linv
// Results are bit-identical to the unbucketed search (each query is searched
// on its own; only the order in which queries are processed changes).
// Extra HBM traffic per query (u64): 8 + 2 | 2 + 8 + 8 + 2 | - | 2 + 16 + 16.
#include <algorithm>

#include <cub/cub.cuh>

#include "hbt_internal.cuh"

namespace hbt {
namespace {

constexpr uint32_t kMaxBuckets = 1024;  // <= 2 * kThreads (block scan), < 2^16 (u16 bucket ids)
constexpr uint32_t kDirBits = 12;
constexpr int kThreads = 512;
constexpr int kQPT = 16;                      // queries per thread per chunk
constexpr uint32_t kChunk = kThreads * kQPT;  // 8192 queries per chunk (< 2^16: u16 positions)

template <typename K>
__device__ __forceinline__ K kmax() { return K(~K(0)); }

template <typename K>
__device__ __forceinline__ K load_key(const uint8_t* p) { return *reinterpret_cast<const K*>(p); }

// sp[b] for the implicit tree: unit = leaf line, its max key is the key of rank
// min(n, (l+1) P) - 1 (dense L-segment).
template <typename K>
__global__ void bk_splitters_implicit(const uint8_t* __restrict__ leaf, uint64_t n, uint32_t P, uint64_t L0,
                                      uint32_t B, K* __restrict__ sp) {
  const uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= B) return;
  if (b == B - 1 || n == 0) { sp[b] = kmax<K>(); return; }
  uint64_t l = ((uint64_t(b) + 1) * L0) / B;
  l = l ? l - 1 : 0;
  const uint64_t r = std::min<uint64_t>(n, (l + 1) * P) - 1;
  sp[b] = load_key<K>(leaf + (r / P) * 64 + (r % P) * sizeof(K));
}

// sp[b] for the regular tree: unit = big leaf in chain (key) order, its max key
// is entry count-1 (dense lines: line e/P, slot e%P).
template <typename K>
__global__ void bk_splitters_regular(const uint8_t* __restrict__ leaf, const uint32_t* __restrict__ count,
                                     const uint32_t* __restrict__ chain, uint64_t nchain, uint32_t F, uint32_t P,
                                     uint32_t B, K* __restrict__ sp) {
  const uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= B) return;
  if (b == B - 1 || nchain == 0) { sp[b] = kmax<K>(); return; }
  uint64_t c = ((uint64_t(b) + 1) * nchain) / B;
  c = c ? c - 1 : 0;
  const uint32_t v = chain[c];
  const uint32_t cnt = count[v];
  if (cnt == 0) { sp[b] = kmax<K>(); return; }
  const uint32_t e = cnt - 1;
  sp[b] = load_key<K>(leaf + (uint64_t(v) * F + e / P) * 64 + (e % P) * sizeof(K));
}

template <typename K>
__device__ __forceinline__ uint32_t lower_bound_in(const K* sp, uint32_t lo, uint32_t hi, K q) {
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (sp[mid] < q) lo = mid + 1; else hi = mid;
  }
  return lo;
}

template <typename K>
__global__ void bk_directory(const K* __restrict__ sp, uint32_t B, uint32_t* __restrict__ dir) {
  const uint32_t p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= (1u << kDirBits)) return;
  constexpr int sh = 8 * int(sizeof(K)) - int(kDirBits);
  const K lo_key = K(K(p) << sh);
  const K hi_key = K(lo_key | K((K(1) << sh) - 1));
  const uint32_t lo = lower_bound_in(sp, 0, B - 1, lo_key);
  const uint32_t hi = lower_bound_in(sp, 0, B - 1, hi_key);
  dir[p] = lo | (hi << 16);
}

// Bucket of q: directory range, then a lower bound over the splitters in it.
template <typename K>
__device__ __forceinline__ uint32_t bucket_of(K q, const K* s_sp, const uint32_t* s_dir) {
  constexpr int sh = 8 * int(sizeof(K)) - int(kDirBits);
  const uint32_t e = s_dir[uint32_t(q >> sh)];
  return lower_bound_in(s_sp, e & 0xFFFFu, e >> 16, q);
}

// Exclusive scan of s_in[0, B) into s_out (B <= 2 * kThreads) by one CTA; s_tmp
// holds kThreads partial sums.  Ends with a barrier.
__device__ __forceinline__ void block_exclusive_scan(const uint32_t* s_in, uint32_t* s_out, uint32_t B,
                                                     uint32_t* s_tmp) {
  const uint32_t t = threadIdx.x;
  const uint32_t a = 2 * t < B ? s_in[2 * t] : 0u, b = 2 * t + 1 < B ? s_in[2 * t + 1] : 0u;
  s_tmp[t] = a + b;
  __syncthreads();
  for (uint32_t off = 1; off < kThreads; off <<= 1) {
    const uint32_t x = t >= off ? s_tmp[t - off] : 0u;
    __syncthreads();
    s_tmp[t] += x;
    __syncthreads();
  }
  const uint32_t ex = s_tmp[t] - (a + b);
  if (2 * t < B) s_out[2 * t] = ex;
  if (2 * t + 1 < B) s_out[2 * t + 1] = ex + a;
  __syncthreads();
}

// Pass 1: bucket of every query (bq, u16) and the per-chunk histograms, stored
// bucket-major: tab[b * chunks + c] = #queries of chunk c in bucket b.
template <typename K>
__global__ void __launch_bounds__(kThreads) bk_count(const K* __restrict__ q, uint64_t m, const K* __restrict__ sp,
                                                     const uint32_t* __restrict__ dir, uint32_t B, uint64_t chunks,
                                                     uint16_t* __restrict__ bq, uint32_t* __restrict__ tab) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t* s_dir = reinterpret_cast<uint32_t*>(smem);
  uint32_t* s_h = s_dir + (1u << kDirBits);
  K* s_sp = reinterpret_cast<K*>(s_h + kMaxBuckets);
  for (uint32_t i = threadIdx.x; i < B; i += kThreads) s_sp[i] = sp[i];
  for (uint32_t i = threadIdx.x; i < (1u << kDirBits); i += kThreads) s_dir[i] = dir[i];
  for (uint64_t c = blockIdx.x; c < chunks; c += gridDim.x) {
    for (uint32_t i = threadIdx.x; i < B; i += kThreads) s_h[i] = 0;
    __syncthreads();
    const uint64_t lo = c * kChunk;
    K qq[kQPT];
#pragma unroll
    for (int j = 0; j < kQPT; ++j) {
      const uint64_t i = lo + uint64_t(j) * kThreads + threadIdx.x;
      qq[j] = i < m ? __ldcs(q + i) : K(0);
    }
#pragma unroll
    for (int j = 0; j < kQPT; ++j) {
      const uint64_t i = lo + uint64_t(j) * kThreads + threadIdx.x;
      if (i < m) {
        const uint32_t b = bucket_of(qq[j], s_sp, s_dir);
        bq[i] = uint16_t(b);
        atomicAdd(&s_h[b], 1u);
      }
    }
    __syncthreads();
    for (uint32_t b = threadIdx.x; b < B; b += kThreads) tab[uint64_t(b) * chunks + c] = s_h[b];
    __syncthreads();
  }
}

// Per-chunk bucket layout shared by the scatter and the gather: s_cnt (this
// chunk's count per bucket), s_lb (their exclusive scan = the bucket's start in
// the chunk's bucket-sorted order), s_gb (the run's first global slot).
__device__ __forceinline__ void chunk_layout(const uint32_t* __restrict__ tab, const uint32_t* __restrict__ gb,
                                             uint32_t B, uint64_t chunks, uint64_t c, uint32_t* s_cnt,
                                             uint32_t* s_lb, uint32_t* s_gb, uint32_t* s_tmp) {
  for (uint32_t b = threadIdx.x; b < B; b += kThreads) {
    s_cnt[b] = tab[uint64_t(b) * chunks + c];
    s_gb[b] = gb[uint64_t(b) * chunks + c];
  }
  __syncthreads();
  block_exclusive_scan(s_cnt, s_lb, B, s_tmp);
}

// Pass 2: each chunk's queries are ordered by bucket in shared memory, then
// written as B contiguous runs (the run of bucket b at global slot gb[b][c]);
// linv[i] (u16) = the query's position in the chunk's bucket-sorted order.
template <typename K>
__global__ void __launch_bounds__(kThreads, 2) bk_scatter(const K* __restrict__ q, uint64_t m,
                                                       const uint16_t* __restrict__ bq, const uint32_t* __restrict__ tab,
                                                       const uint32_t* __restrict__ gb, uint32_t B, uint64_t chunks,
                                                       K* __restrict__ qs, uint16_t* __restrict__ linv) {
  extern __shared__ __align__(16) uint8_t smem[];
  K* s_q = reinterpret_cast<K*>(smem);
  uint16_t* s_b = reinterpret_cast<uint16_t*>(s_q + kChunk);
  uint32_t* s_cnt = reinterpret_cast<uint32_t*>(s_b + kChunk);
  uint32_t* s_lb = s_cnt + kMaxBuckets;
  uint32_t* s_gb = s_lb + kMaxBuckets;
  uint32_t* s_rank = s_gb + kMaxBuckets;
  uint32_t* s_tmp = s_rank + kMaxBuckets;
  for (uint64_t c = blockIdx.x; c < chunks; c += gridDim.x) {
    const uint64_t lo = c * kChunk;
    const uint32_t nc = uint32_t(m - lo < kChunk ? m - lo : kChunk);
    for (uint32_t b = threadIdx.x; b < B; b += kThreads) s_rank[b] = 0;
    chunk_layout(tab, gb, B, chunks, c, s_cnt, s_lb, s_gb, s_tmp);
    K qq[kQPT];
    uint32_t bb[kQPT];
#pragma unroll
    for (int j = 0; j < kQPT; ++j) {
      const uint32_t t = uint32_t(j) * kThreads + threadIdx.x;
      qq[j] = K(0);
      bb[j] = 0;
      if (t < nc) {
        qq[j] = __ldcs(q + lo + t);
        bb[j] = __ldcs(reinterpret_cast<const unsigned short*>(bq) + lo + t);
      }
    }
#pragma unroll
    for (int j = 0; j < kQPT; ++j) {
      const uint32_t t = uint32_t(j) * kThreads + threadIdx.x;
      if (t < nc) {
        const uint32_t pos = s_lb[bb[j]] + atomicAdd(&s_rank[bb[j]], 1u);
        s_q[pos] = qq[j];
        s_b[pos] = uint16_t(bb[j]);
        __stcs(reinterpret_cast<unsigned short*>(linv) + lo + t, (unsigned short)pos);
      }
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < kQPT; ++j) {
      const uint32_t t = uint32_t(j) * kThreads + threadIdx.x;
      if (t < nc) {
        const uint32_t b = s_b[t];
        qs[uint64_t(s_gb[b]) + (t - s_lb[b])] = s_q[t];
      }
    }
    __syncthreads();
  }
}

// Pass 4: the chunk's results are read back as its B contiguous runs into
// shared memory (bucket-sorted order), then stored in query order through linv.
template <typename K>
__global__ void __launch_bounds__(kThreads, 2) bk_gather(const uint16_t* __restrict__ linv, uint64_t m,
                                                      const uint32_t* __restrict__ tab, const uint32_t* __restrict__ gb,
                                                      uint32_t B, uint64_t chunks, const uint64_t* __restrict__ pf_s,
                                                      const K* __restrict__ v_s, uint64_t* __restrict__ out_pf,
                                                      K* __restrict__ out_v) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint64_t* s_val = reinterpret_cast<uint64_t*>(smem);
  uint16_t* s_b = reinterpret_cast<uint16_t*>(s_val + kChunk);
  uint32_t* s_cnt = reinterpret_cast<uint32_t*>(s_b + kChunk);
  uint32_t* s_lb = s_cnt + kMaxBuckets;
  uint32_t* s_gb = s_lb + kMaxBuckets;
  uint32_t* s_tmp = s_gb + kMaxBuckets;
  for (uint64_t c = blockIdx.x; c < chunks; c += gridDim.x) {
    const uint64_t lo = c * kChunk;
    const uint32_t nc = uint32_t(m - lo < kChunk ? m - lo : kChunk);
    chunk_layout(tab, gb, B, chunks, c, s_cnt, s_lb, s_gb, s_tmp);
    for (uint32_t b = threadIdx.x; b < B; b += kThreads)
      for (uint32_t k = 0, n = s_cnt[b], p = s_lb[b]; k < n; ++k) s_b[p + k] = uint16_t(b);
    __syncthreads();
    const unsigned short* li = reinterpret_cast<const unsigned short*>(linv) + lo;
#pragma unroll 1
    for (int h = 0; h < kQPT; h += 8) {
      uint64_t x[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint32_t t = uint32_t(h + j) * kThreads + threadIdx.x;
        if (t < nc) {
          const uint32_t b = s_b[t];
          x[j] = __ldcs(reinterpret_cast<const unsigned long long*>(pf_s) + s_gb[b] + (t - s_lb[b]));
        }
      }
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint32_t t = uint32_t(h + j) * kThreads + threadIdx.x;
        if (t < nc) s_val[t] = x[j];
      }
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < kQPT; ++j) {
      const uint32_t t = uint32_t(j) * kThreads + threadIdx.x;
      if (t < nc) __stcs(reinterpret_cast<unsigned long long*>(out_pf) + lo + t, (unsigned long long)s_val[__ldg(li + t)]);
    }
    __syncthreads();
#pragma unroll 1
    for (int h = 0; h < kQPT; h += 8) {
      K x[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint32_t t = uint32_t(h + j) * kThreads + threadIdx.x;
        if (t < nc) {
          const uint32_t b = s_b[t];
          x[j] = __ldcs(v_s + uint64_t(s_gb[b]) + (t - s_lb[b]));
        }
      }
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint32_t t = uint32_t(h + j) * kThreads + threadIdx.x;
        if (t < nc) s_val[t] = uint64_t(x[j]);
      }
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < kQPT; ++j) {
      const uint32_t t = uint32_t(j) * kThreads + threadIdx.x;
      if (t < nc) {
        const uint32_t l = __ldcs(li + t);
        if constexpr (sizeof(K) == 8)
          __stcs(reinterpret_cast<unsigned long long*>(out_v) + lo + t, (unsigned long long)s_val[l]);
        else
          __stcs(reinterpret_cast<unsigned int*>(out_v) + lo + t, (unsigned int)s_val[l]);
      }
    }
    __syncthreads();
  }
}

uint64_t tree_bytes(const hbt_tree* t) {
  if (t->form == HBT_IMPLICIT) return t->inner_bytes + t->inner_idx_bytes + t->leaf_bytes;
  const RegularState& r = t->r;
  const uint64_t S = t->width, F = t->F;
  return r.uoff[r.U] * (F * (S + 4) + 32) + r.pool * (F * S + 32) + r.pool * F * 64;
}

// Number of buckets: one per `slice` bytes of tree, at most one per unit and
// kMaxBuckets.
uint32_t pick_buckets(const hbt_tree* t) {
  const uint64_t slice = t->cfg.bucket_slice ? t->cfg.bucket_slice : (16ull << 20);
  const uint64_t units = t->form == HBT_IMPLICIT ? t->L0 : t->r.nchain;
  uint64_t B = (tree_bytes(t) + slice - 1) / slice;
  B = std::min<uint64_t>(B, kMaxBuckets);
  B = std::min<uint64_t>(B, units);
  return uint32_t(std::max<uint64_t>(B, 1));
}

template <typename K>
int prepare_splitters(const hbt_tree* t, cudaStream_t s) {
  BucketState& bs = t->bk;
  const uint32_t B = pick_buckets(t);
  if (bs.valid && bs.B == B) return HBT_OK;
  if (!bs.d_sp) {
    HBT_CUDA_TRY(cudaMalloc(&bs.d_sp, kMaxBuckets * 8));
    HBT_CUDA_TRY(cudaMalloc(&bs.d_dir, (1u << kDirBits) * 4));
  }
  const unsigned gb = (B + 255) / 256;
  if (t->form == HBT_IMPLICIT)
    bk_splitters_implicit<K><<<gb, 256, 0, s>>>((const uint8_t*)t->d_leaf, t->n, t->P, t->L0, B, (K*)bs.d_sp);
  else
    bk_splitters_regular<K><<<gb, 256, 0, s>>>((const uint8_t*)t->r.d_leaf, t->r.d_count, t->r.d_chain,
                                               t->r.nchain, t->F, t->P, B, (K*)bs.d_sp);
  HBT_CUDA_TRY(cudaGetLastError());
  bk_directory<K><<<(1u << kDirBits) / 256, 256, 0, s>>>((const K*)bs.d_sp, B, bs.d_dir);
  HBT_CUDA_TRY(cudaGetLastError());
  bs.B = B;
  bs.valid = true;
  return HBT_OK;
}

template <typename K>
int bucketed_t(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s,
               int (*search)(const hbt_tree*, const void*, uint64_t, uint64_t*, void*, cudaStream_t)) {
  int rc = prepare_splitters<K>(t, s);
  if (rc != HBT_OK) return rc;
  const BucketState& bs = t->bk;
  const uint32_t B = bs.B;
  const uint64_t chunks = (m + kChunk - 1) / kChunk;
  const uint64_t ntab = uint64_t(B) * chunks;
  size_t scan_bytes = 0;
  HBT_CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, scan_bytes, (const uint32_t*)nullptr, (uint32_t*)nullptr,
                                             ntab, s));
  // scratch (stream-ordered pool): qs, pf_s, v_s, bq, linv, tab, gb, scan temp
  auto al = [](uint64_t x) { return (x + 255) & ~uint64_t(255); };
  const uint64_t o_pf = al(m * sizeof(K)), o_v = o_pf + al(m * 8), o_bq = o_v + al(m * sizeof(K)),
                 o_li = o_bq + al(m * 2), o_tab = o_li + al(m * 2), o_gb = o_tab + al(ntab * 4),
                 o_tmp = o_gb + al(ntab * 4), total = o_tmp + al(scan_bytes);
  void* buf = nullptr;
  HBT_CUDA_TRY(scratch_alloc(&buf, total, s));
  uint8_t* base = static_cast<uint8_t*>(buf);
  K* qs = reinterpret_cast<K*>(base);
  uint64_t* pf_s = reinterpret_cast<uint64_t*>(base + o_pf);
  K* v_s = reinterpret_cast<K*>(base + o_v);
  uint16_t* bq = reinterpret_cast<uint16_t*>(base + o_bq);
  uint16_t* linv = reinterpret_cast<uint16_t*>(base + o_li);
  uint32_t* tab = reinterpret_cast<uint32_t*>(base + o_tab);
  uint32_t* gb = reinterpret_cast<uint32_t*>(base + o_gb);
  rc = HBT_OK;
  do {
    const size_t smem_count = (1u << kDirBits) * 4 + kMaxBuckets * 4 + kMaxBuckets * sizeof(K);
    const size_t smem_scatter = kChunk * (sizeof(K) + 2) + kMaxBuckets * 4 * 4 + kThreads * 4;
    const size_t smem_gather = kChunk * (8 + 2) + kMaxBuckets * 4 * 3 + kThreads * 4;
    static bool attr = false;
    if (!attr) {
      const int lim = 120 * 1024;
      cudaFuncSetAttribute(bk_count<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
      cudaFuncSetAttribute(bk_count<uint64_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
      cudaFuncSetAttribute(bk_scatter<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
      cudaFuncSetAttribute(bk_scatter<uint64_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
      cudaFuncSetAttribute(bk_gather<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
      cudaFuncSetAttribute(bk_gather<uint64_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
      attr = true;
    }
    const unsigned grid = unsigned(std::min<uint64_t>(chunks, uint64_t(t->num_sms) * 2));
    bk_count<K><<<grid, kThreads, smem_count, s>>>((const K*)q, m, (const K*)bs.d_sp, bs.d_dir, B, chunks, bq, tab);
    if (cub::DeviceScan::ExclusiveSum(base + o_tmp, scan_bytes, tab, gb, ntab, s) != cudaSuccess) {
      set_error("bucket scan failed");
      rc = HBT_ECUDA;
      break;
    }
    bk_scatter<K><<<grid, kThreads, smem_scatter, s>>>((const K*)q, m, bq, tab, gb, B, chunks, qs, linv);
    if (cudaError_t e = cudaGetLastError(); e != cudaSuccess) {
      set_error("bucketing kernels failed to launch: %s", cudaGetErrorString(e));
      rc = HBT_ECUDA;
      break;
    }
    rc = search(t, qs, m, pf_s, v_s, s);
    if (rc != HBT_OK) break;
    bk_gather<K><<<grid, kThreads, smem_gather, s>>>(linv, m, tab, gb, B, chunks, pf_s, v_s, pf, (K*)v);
    if (cudaError_t e = cudaGetLastError(); e != cudaSuccess) {
      set_error("bucket gather failed to launch: %s", cudaGetErrorString(e));
      rc = HBT_ECUDA;
      break;
    }
  } while (0);
  scratch_free(buf, s);
  return rc;
}

}  // namespace

bool bucketed_enabled(const hbt_tree* t, uint64_t m) {
  const uint32_t mode = t->cfg.bucket;
  if (mode == 0) return false;
  if (m >= (1ull << 32) || pick_buckets(t) < 2) return false;
  if (mode == 1) return true;
  // auto: regular trees well beyond the L2 and batches large enough to share
  // lines (measured, profiles/r01_bucket_*: c3 10.8 -> 15.2 G q/s; the implicit
  // c5 tree under Zipf queries already hits L2 and loses, 23.1 -> 19.6)
  int l2 = 0;
  cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, t->device);
  return t->form == HBT_REGULAR && tree_bytes(t) > 8ull * uint64_t(l2) && m >= (1ull << 22);
}

int bucketed_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s) {
  auto search = t->form == HBT_REGULAR ? regular_search : implicit_search;
  return t->width == 4 ? bucketed_t<uint32_t>(t, q, m, pf, v, s, search)
                       : bucketed_t<uint64_t>(t, q, m, pf, v, s, search);
}

void bucket_free(hbt_tree* t) {
  cudaFree(t->bk.d_sp);
  cudaFree(t->bk.d_dir);
  t->bk = BucketState{};
}

}  // namespace hbt
