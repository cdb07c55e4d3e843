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
// The batch is cut into chunks of kChunk queries, and the chunks into NSEG contiguous
// SEGMENTS, each handled in chunk order by one CTA in every pass.  Per chunk and
// bucket the queries form one contiguous RUN in the bucketed order (bucket-major,
// then segment, then chunk inside a segment), so both reorderings move whole runs:
//   splitters   sp[b] = max key of unit floor((b+1) U / B) - 1 (units = leaf
//               lines of the implicit tree / chain big leaves of the regular
//               tree), sp[B-1] = MAX; bucket(q) = #{sp < q} (a lower bound, the
//               node-search rule R1 of DESIGN.md applied to the splitters)
//   directory   dir[p] = [bucket(p << sh), bucket(((p+1) << sh) - 1)] over the
//               top D bits of the key, so a query binary-searches a short range
//   bk_count    bucket of every query (u16), per-chunk histograms tab[c][b] and
//               per-segment column sums seg[j][b]
//   bk_seg_scan one CTA: run start of every (segment, bucket), segoff[j][b] =
//               sum_{b'<b} total(b') + sum_{j'<j} seg[j'][b], and the bucket starts
//   bk_scatter  per segment, chunk after chunk: queries ordered by bucket in shared
//               memory and written as runs at a running per-bucket offset (segoff +
//               earlier chunks' counts); linv[i] = the query's position in its
//               chunk's bucket-sorted order
//   search      the item searches (bucket-local directory) on the bucketed queries
//   bk_gather   per segment, the same running offsets: result runs read into
//               shared memory, stored in query order through linv
// Results are bit-identical to the unbucketed search (each query is searched
// on its own; only the order in which queries are processed changes).
// Extra HBM traffic per query (u64): 8 + 2 | - | 2 + 8 + 8 + 2 | - | 2 + 16 + 16.
#include <algorithm>
#include <functional>
#include <mutex>
#include <vector>

#include "block_util.cuh"
#include "hbt_internal.cuh"
#include "item_dir.cuh"

namespace hbt {
namespace {

constexpr uint32_t kMaxBuckets = 1024;  // <= 2 * kThreads (block scan), < 2^16 (u16 bucket ids)
constexpr uint32_t kDirBits = 12;
constexpr int kThreads = 512;
constexpr int kQPT = 16;                      // queries per thread per chunk
constexpr uint32_t kChunk = kThreads * kQPT;  // 8192 queries per chunk (< 2^16: u16 positions)
// bk_count pulls its NEXT chunk's queries into the L2 with one bulk prefetch while it
// works on the current one (cp.async.bulk.prefetch.L2; c3 count 0.167 -> 0.158 ms; the
// same in bk_scatter measured no gain)
constexpr bool kStreamPrefetch = true;

template <typename K>
__device__ __forceinline__ K kmax() { return K(~K(0)); }

// Row stride of the chunk-major tables tab / gb: B rounded up to 4 entries, so every
// chunk's row starts 16 B aligned (bulk copies of a row into shared memory).
__host__ __device__ __forceinline__ uint32_t row_stride(uint32_t B) { return (B + 3u) & ~3u; }

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

// Item directory (implicit): M[j] = max key below level node j = the key of rank
// min(n, (j+1) * span * P) - 1 (span = leaf lines per node; dense L-segment).
template <typename K>
__global__ void bk_level_max(const uint8_t* __restrict__ leaf, uint64_t n, uint32_t P, uint64_t span,
                             uint64_t nunits, K* __restrict__ M) {
  for (uint64_t j = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; j < nunits; j += uint64_t(gridDim.x) * blockDim.x) {
    if (n == 0) { M[j] = kmax<K>(); continue; }
    const uint64_t r = std::min<uint64_t>(n, (j + 1) * span * P) - 1;
    M[j] = load_key<K>(leaf + (r / P) * 64 + (r % P) * sizeof(K));
  }
}

// Compressed item directory (ItemDir::bd): one CTA per bucket derives the offset origin
// lo = M[u0], the shift sh that fits M[u0 + cnt - 1] - lo in 32 bits (M' = (M - lo) >> sh),
// the prefix-table slice shift ssh (2^12 slices over [0, top]) and the entry shift esh,
// then writes the 16-bit entries E16 = (M' >> esh) & 0xFFFF (padding to 8 entries: ~0) and
// the prefix table T16[p] = #{M' < p << ssh}, p in [0, 2^12] (padded with cnt).
template <typename K>
__global__ void bk_cdir(const K* __restrict__ M, BucketDir* __restrict__ bd, uint16_t* __restrict__ E16,
                        uint16_t* __restrict__ T16) {
  __shared__ K s_lo;
  __shared__ uint32_t s_sh[3];
  BucketDir* d = bd + blockIdx.x;
  const uint64_t u0 = d->u0, off16 = d->off16;
  const uint32_t cnt = d->cnt;
  if (threadIdx.x == 0) {
    const K lo = M[u0], span = K(M[u0 + cnt - 1] - lo);
    const uint32_t bits = span ? uint32_t(8 * sizeof(K)) - uint32_t(sizeof(K) == 8 ? __clzll((long long)span)
                                                                                 : __clz(int(span)))
                               : 0u;
    const uint32_t sh = bits > 32 ? bits - 32 : 0u;
    const uint32_t top = uint32_t(span >> sh);
    const uint32_t tb = top ? 32u - uint32_t(__clz(int(top))) : 0u;
    const uint32_t ssh = tb > 12 ? tb - 12 : 0u;
    s_lo = lo;
    s_sh[0] = sh;
    s_sh[1] = ssh;
    s_sh[2] = ssh > 16 ? ssh - 16 : 0u;
    d->lo = uint64_t(lo);
    d->sh = sh;
    d->top = top;
    d->ssh = ssh;
    d->esh = s_sh[2];
  }
  __syncthreads();
  const K lo = s_lo;
  const uint32_t sh = s_sh[0], ssh = s_sh[1], esh = s_sh[2];
  auto mp = [&](uint32_t i) { return uint32_t(K(M[u0 + i] - lo) >> sh); };
  const uint32_t padded = (cnt + 7u) & ~7u;
  for (uint32_t i = threadIdx.x; i < padded; i += blockDim.x) E16[off16 + i] = i < cnt ? uint16_t(mp(i) >> esh) : 0xFFFFu;
  for (uint32_t p = threadIdx.x; p < kT16; p += blockDim.x) {
    uint32_t a = 0;
    if (p > 4096u) {
      a = cnt;
    } else {
      const uint64_t key = uint64_t(p) << ssh;  // lower bound of key over M'
      uint32_t len = cnt;
      while (len > 0) {
        const uint32_t half = len >> 1;
        if (uint64_t(mp(a + half)) < key) { a += half + 1; len -= half + 1; } else { len = half; }
      }
    }
    T16[uint64_t(blockIdx.x) * kT16 + p] = uint16_t(a);
  }
}

// Compact nodes of the compressed directory's level (implicit, u64 keys, F = 16; ItemDir::
// cnode): one CTA per bucket.  With M'(x) = (x - lo) >> sh of the bucket (0 below lo), node u
// becomes 32 B: u32 b0 = M'(sep_0), then for slots 1..14 the u16 (M'(sep_i) - b0) >> nsh, or
// 0xFFFF for a MAX slot (slot 15 is always MAX, reading R3); nsh is the bucket's shift that
// keeps every real entry <= 0xFFFE.  Truncation is monotone, so the child the search counts
// from it is the true child or an earlier one (a tie), never a later one; the walk's FIX
// moves on from an early leaf line (descend_and_store).  A DRAM transfer of 128 B brings
// four of them instead of one node.
__global__ void bk_cnode(const uint64_t* __restrict__ lvl, BucketDir* __restrict__ bd,
                         uint4* __restrict__ out) {
  constexpr uint64_t MAXK = ~0ull;
  __shared__ uint32_t s_w[32];
  __shared__ uint32_t s_nsh;
  BucketDir* d = bd + blockIdx.x;
  const uint64_t u0 = d->u0, lo = d->lo;
  const uint32_t cnt = d->cnt, sh = d->sh;
  auto mp = [&](uint64_t x) -> uint32_t {
    if (x <= lo) return 0u;
    const uint64_t y = (x - lo) >> sh;
    return y > 0xFFFFFFFFull ? 0xFFFFFFFFu : uint32_t(y);
  };
  uint32_t w = 0;
  for (uint32_t i = threadIdx.x; i < cnt; i += blockDim.x) {
    const uint64_t* nd = lvl + (u0 + i) * 16;
    if (nd[0] == MAXK) continue;
    const uint32_t b0 = mp(nd[0]);
    for (int j = 14; j >= 1; --j)
      if (nd[j] != MAXK) {
        w = max(w, mp(nd[j]) - b0);
        break;
      }
  }
  for (int o = 16; o > 0; o >>= 1) w = max(w, __shfl_xor_sync(0xffffffffu, w, o));
  if ((threadIdx.x & 31) == 0) s_w[threadIdx.x >> 5] = w;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t m = 0;
    for (uint32_t x = 0; x < blockDim.x / 32; ++x) m = max(m, s_w[x]);
    uint32_t nsh = 0;
    while ((m >> nsh) > 0xFFFEu) ++nsh;
    s_nsh = nsh;
    d->nsh = nsh;
  }
  __syncthreads();
  const uint32_t nsh = s_nsh;
  for (uint32_t i = threadIdx.x; i < cnt; i += blockDim.x) {
    const uint64_t* nd = lvl + (u0 + i) * 16;
    const uint32_t b0 = nd[0] == MAXK ? 0xFFFFFFFFu : mp(nd[0]);
    uint32_t wv[8];
    wv[0] = b0;
    for (int j = 1; j <= 14; ++j) {
      const uint32_t e = nd[j] == MAXK ? 0xFFFFu : ((mp(nd[j]) - b0) >> nsh);
      const int word = (j + 1) / 2, half = (j + 1) & 1;  // u16 slot j at byte 4 + 2 (j - 1)
      if (half == 0) wv[word] = e; else wv[word] |= e << 16;
    }
    uint4* o = out + (u0 + i) * 2;
    o[0] = make_uint4(wv[0], wv[1], wv[2], wv[3]);
    o[1] = make_uint4(wv[4], wv[5], wv[6], wv[7]);
  }
}

// Item directory (regular): M[c * NI + t] = true max key of key line t of the
// last-level node of chain leaf c = the key of entry min(count, (t+1)*KPL*P) - 1
// (KPL separators per 64 B key line, each covering one leaf line of P entries);
// key lines past the leaf's last entry repeat the leaf max (keeps M sorted).
template <typename K>
__global__ void bk_keyline_max(const uint8_t* __restrict__ leaf, const uint32_t* __restrict__ count,
                               const uint32_t* __restrict__ chain, uint64_t nchain, uint32_t F, uint32_t P,
                               uint32_t NI, uint32_t KPL, K* __restrict__ M) {
  const uint64_t total = nchain * NI;
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < total; x += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t v = chain[x / NI], t = uint32_t(x % NI);
    const uint32_t cnt = count[v];
    if (cnt == 0) { M[x] = kmax<K>(); continue; }
    const uint32_t e = std::min<uint32_t>(cnt, (t + 1) * KPL * P) - 1;
    M[x] = load_key<K>(leaf + (uint64_t(v) * F + e / P) * 64 + (e % P) * sizeof(K));
  }
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

// Pass 1: bucket of every query (bq, u16), the per-chunk histograms (chunk-major:
// tab[c * Bp + b] = #queries of chunk c in bucket b, Bp = row_stride(B)) and the per-segment column sums
// seg[j * B + b] (segment j = chunks [j * kps, (j + 1) * kps), in chunk order).
template <typename K>
__global__ void __launch_bounds__(kThreads) bk_count(const K* __restrict__ q, uint64_t m, const K* __restrict__ sp,
                                                     const uint32_t* __restrict__ dir, uint32_t B, uint64_t chunks,
                                                     uint64_t kps, uint64_t nseg, uint16_t* __restrict__ bq,
                                                     uint32_t* __restrict__ tab, uint32_t* __restrict__ seg) {
  extern __shared__ __align__(16) uint8_t smem[];
  uint32_t* s_dir = reinterpret_cast<uint32_t*>(smem);
  uint32_t* s_h = s_dir + (1u << kDirBits);
  uint32_t* s_sh = s_h + kMaxBuckets;
  K* s_sp = reinterpret_cast<K*>(s_sh + kMaxBuckets);
  for (uint32_t i = threadIdx.x; i < B; i += kThreads) s_sp[i] = sp[i];
  for (uint32_t i = threadIdx.x; i < (1u << kDirBits); i += kThreads) s_dir[i] = dir[i];
  for (uint64_t j = blockIdx.x; j < nseg; j += gridDim.x) {
    const uint64_t c0 = j * kps, c1 = c0 + kps < chunks ? c0 + kps : chunks;
    for (uint32_t i = threadIdx.x; i < B; i += kThreads) s_sh[i] = 0;
    for (uint64_t c = c0; c < c1; ++c) {
      if (kStreamPrefetch && threadIdx.x == 0 && c + 1 < c1) {  // next chunk's queries -> L2
        const uint64_t n0 = (c + 1) * kChunk;
        prefetch_l2_range(q + n0, (m - n0 < kChunk ? m - n0 : kChunk) * sizeof(K));
      }
      for (uint32_t i = threadIdx.x; i < B; i += kThreads) s_h[i] = 0;
      __syncthreads();
      const uint64_t lo = c * kChunk;
      K qq[kQPT];
#pragma unroll
      for (int x = 0; x < kQPT; ++x) {
        const uint64_t i = lo + uint64_t(x) * kThreads + threadIdx.x;
        qq[x] = i < m ? __ldcs(q + i) : K(0);
      }
#pragma unroll
      for (int x = 0; x < kQPT; ++x) {
        const uint64_t i = lo + uint64_t(x) * kThreads + threadIdx.x;
        if (i < m) {
          const uint32_t b = bucket_of(qq[x], s_sp, s_dir);
          bq[i] = uint16_t(b);
          atomicAdd(&s_h[b], 1u);
        }
      }
      __syncthreads();
      for (uint32_t b = threadIdx.x; b < B; b += kThreads) {
        tab[c * row_stride(B) + b] = s_h[b];
        s_sh[b] += s_h[b];
      }
      __syncthreads();
    }
    for (uint32_t b = threadIdx.x; b < B; b += kThreads) seg[j * B + b] = s_sh[b];
  }
}

// Run starts (one CTA; B <= 1024): bucket b's runs follow segment after segment,
// buckets in order, so segoff[j * B + b] = bstart[b] + sum_{j' < j} seg[j' * B + b]
// with bstart[b] = the exclusive scan of the bucket totals (bstart[B] = m).
constexpr int kScanThreads = 1024;
__global__ void __launch_bounds__(kScanThreads) bk_seg_scan(const uint32_t* __restrict__ seg, uint32_t B, uint64_t nseg,
                                                            uint64_t m, uint32_t* __restrict__ segoff,
                                                            uint64_t* __restrict__ bstart) {
  __shared__ uint32_t s_T[kScanThreads], s_base[kScanThreads], s_tmp[32];
  const uint32_t b = threadIdx.x;
  uint32_t tot = 0;
  if (b < B) {
#pragma unroll 8
    for (uint64_t j = 0; j < nseg; ++j) tot += seg[j * B + b];
  }
  s_T[b] = tot;
  __syncthreads();
  block_exclusive_scan<kScanThreads>(s_T, s_base, B, s_tmp);
  if (b < B) {
    uint32_t run = s_base[b];
#pragma unroll 8
    for (uint64_t j = 0; j < nseg; ++j) {
      const uint32_t x = seg[j * B + b];
      segoff[j * B + b] = run;
      run += x;
    }
    bstart[b] = s_base[b];
  }
  if (b == 0) bstart[B] = m;
}

// Run start of every (chunk, bucket), chunk-major: gb[c * Bp + b] = segoff[j][b] + the
// counts of segment j's earlier chunks (one CTA per segment walks its chunks in order;
// rows are coalesced).  The scatter and the gather take chunks interleaved over the
// CTAs (c = blockIdx, blockIdx + grid, ...): the runs they write / read at the same
// time are then neighbours in memory and share L2 lines and DRAM pages (contiguous
// per-CTA segments measured slower: c4 scatter 1.95 -> 2.57 ms, gather 2.14 -> 2.44).
__global__ void __launch_bounds__(kScanThreads) bk_run_starts(const uint32_t* __restrict__ tab,
                                                              const uint32_t* __restrict__ segoff, uint32_t B,
                                                              uint64_t chunks, uint64_t kps,
                                                              uint32_t* __restrict__ gb) {
  const uint64_t j = blockIdx.x;
  const uint32_t b = threadIdx.x;
  if (b >= B) return;
  const uint64_t c0 = j * kps, c1 = c0 + kps < chunks ? c0 + kps : chunks;
  uint32_t run = segoff[j * B + b];
#pragma unroll 4
  for (uint64_t c = c0; c < c1; ++c) {
    const uint32_t x = tab[c * row_stride(B) + b];
    gb[c * row_stride(B) + b] = run;
    run += x;
  }
}

// Per-chunk bucket layout shared by the scatter and the gather (tab, gb
// chunk-major): s_cnt (this chunk's count per bucket), s_lb (their exclusive scan = the
// bucket's start in the chunk's bucket-sorted order), s_gb (the run's first global slot).
template <int TH = kThreads>
__device__ __forceinline__ void chunk_layout(const uint32_t* __restrict__ tab, const uint32_t* __restrict__ gb,
                                             uint32_t B, uint64_t c, uint32_t* s_cnt, uint32_t* s_lb, uint32_t* s_gb,
                                             uint32_t* s_tmp) {
  for (uint32_t b = threadIdx.x; b < B; b += TH) {  // chunk-major rows: coalesced
    s_cnt[b] = tab[c * row_stride(B) + b];
    s_gb[b] = gb[c * row_stride(B) + b];
  }
  __syncthreads();
  block_exclusive_scan<TH>(s_cnt, s_lb, B, s_tmp);
}

// Pass 2: each chunk's queries are ordered by bucket in shared memory, then
// written as B contiguous runs (the run of bucket b at global slot gb[c][b]);
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
  // the chunk's queries and bucket ids are loaded before its layout row is scanned,
  // so the two DRAM round trips overlap (loading the NEXT chunk's row into registers and
  // prefetching its queries into L2 measured slower: c4 scatter 1.96 -> 2.45 ms)
  constexpr int LPT = int(kMaxBuckets) / kThreads;  // layout entries per thread
  for (uint64_t c = blockIdx.x; c < chunks; c += gridDim.x) {
    const uint64_t lo = c * kChunk;
    const uint32_t nc = uint32_t(m - lo < kChunk ? m - lo : kChunk);
    K qq[kQPT];
    uint32_t bb[kQPT];
#pragma unroll
    for (int x = 0; x < kQPT; ++x) {
      const uint32_t t = uint32_t(x) * kThreads + threadIdx.x;
      qq[x] = K(0);
      bb[x] = 0;
      if (t < nc) {
        qq[x] = __ldcs(q + lo + t);
        bb[x] = __ldcs(reinterpret_cast<const unsigned short*>(bq) + lo + t);
      }
    }
#pragma unroll
    for (int e = 0; e < LPT; ++e) {
      const uint32_t b = uint32_t(e) * kThreads + threadIdx.x;
      if (b < B) {
        s_rank[b] = 0;
        s_cnt[b] = tab[c * row_stride(B) + b];
        s_gb[b] = gb[c * row_stride(B) + b];
      }
    }
    __syncthreads();
    block_exclusive_scan<kThreads>(s_cnt, s_lb, B, s_tmp);
#pragma unroll
    for (int x = 0; x < kQPT; ++x) {
      const uint32_t t = uint32_t(x) * kThreads + threadIdx.x;
      if (t < nc) {
        const uint32_t pos = s_lb[bb[x]] + atomicAdd(&s_rank[bb[x]], 1u);
        s_q[pos] = qq[x];
        s_b[pos] = uint16_t(bb[x]);
        __stcs(reinterpret_cast<unsigned short*>(linv) + lo + t, (unsigned short)pos);
      }
    }
    __syncthreads();
#pragma unroll
    for (int x = 0; x < kQPT; ++x) {
      const uint32_t t = uint32_t(x) * kThreads + threadIdx.x;
      if (t < nc) {
        const uint32_t b = s_b[t];
        qs[uint64_t(s_gb[b]) + (t - s_lb[b])] = s_q[t];
      }
    }
    __syncthreads();
  }
}

// ---- Pass 2 with bulk-copy staging (default for full chunks).  One elected thread
// streams the NEXT chunk's queries, bucket ids and layout rows (88 KB for u64) into a
// shared staging buffer with cp.async.bulk (TMA 1D bulk copies, completion on an
// mbarrier) while the CTA sorts and writes the current chunk, so no warp waits on
// DRAM for its inputs and no registers hold them in flight.  1024 threads, 8 queries
// each; the sort and the run writes are those of bk_scatter.
constexpr int kTThreads = 1024;
constexpr int kTQPT = int(kChunk) / kTThreads;  // 8 queries per thread

template <typename K>
size_t smem_scatter_tma(uint32_t B) {
  const size_t bp = row_stride(B);
  return kChunk * (sizeof(K) + 2) * 2 + bp * 4 * 2 + kMaxBuckets * 4 * 3 + 32 * 4 + 64;
}

template <typename K>
__global__ void __launch_bounds__(kTThreads, 1) bk_scatter_tma(const K* __restrict__ q, uint64_t m,
                                                               const uint16_t* __restrict__ bq,
                                                               const uint32_t* __restrict__ tab,
                                                               const uint32_t* __restrict__ gb, uint32_t B,
                                                               uint64_t chunks, K* __restrict__ qs,
                                                               uint16_t* __restrict__ linv) {
  extern __shared__ __align__(16) uint8_t smem[];
  const uint32_t BP = row_stride(B);
  // staging: [q | bq | tab row | gb row]; sorted: [s_q | s_b]; layout arrays
  K* st_q = reinterpret_cast<K*>(smem);
  uint16_t* st_b = reinterpret_cast<uint16_t*>(st_q + kChunk);
  uint32_t* st_cnt = reinterpret_cast<uint32_t*>(st_b + kChunk);
  uint32_t* st_gb = st_cnt + BP;
  K* s_q = reinterpret_cast<K*>(st_gb + BP);
  uint16_t* s_b = reinterpret_cast<uint16_t*>(s_q + kChunk);
  uint32_t* s_lb = reinterpret_cast<uint32_t*>(s_b + kChunk);
  uint32_t* s_rank = s_lb + kMaxBuckets;
  uint32_t* s_gb = s_rank + kMaxBuckets;
  uint32_t* s_tmp = s_gb + kMaxBuckets;
  uint64_t* bar = reinterpret_cast<uint64_t*>(s_tmp + 32);
  const uint32_t bytes = uint32_t(kChunk * (sizeof(K) + 2) + 2 * BP * 4);
  auto issue = [&](uint64_t c) {  // one thread: the whole chunk c into the staging buffer
    mbar_expect_tx(bar, bytes);
    bulk_g2s(st_q, q + c * kChunk, uint32_t(kChunk * sizeof(K)), bar);
    bulk_g2s(st_b, bq + c * kChunk, uint32_t(kChunk * 2), bar);
    bulk_g2s(st_cnt, tab + c * BP, BP * 4, bar);
    bulk_g2s(st_gb, gb + c * BP, BP * 4, bar);
  };
  const uint64_t full = m / kChunk;  // chunks served by bulk copies; the tail chunk reads directly
  if (threadIdx.x == 0) {
    mbar_init(bar, 1);
    fence_mbar_init();
  }
  __syncthreads();
  if (threadIdx.x == 0 && blockIdx.x < full) issue(blockIdx.x);
  uint32_t parity = 0;
  for (uint64_t c = blockIdx.x; c < chunks; c += gridDim.x) {
    const uint64_t lo = c * kChunk;
    const uint32_t nc = uint32_t(m - lo < kChunk ? m - lo : kChunk);
    K qq[kTQPT];
    uint32_t bb[kTQPT];
    if (c < full) {
      mbar_wait(bar, parity);
      parity ^= 1u;
#pragma unroll
      for (int x = 0; x < kTQPT; ++x) {
        const uint32_t t = uint32_t(x) * kTThreads + threadIdx.x;
        qq[x] = st_q[t];
        bb[x] = st_b[t];
      }
      for (uint32_t b = threadIdx.x; b < B; b += kTThreads) {
        s_rank[b] = 0;
        s_gb[b] = st_gb[b];
        s_lb[b] = st_cnt[b];  // counts for the scan below (in place)
      }
    } else {
#pragma unroll
      for (int x = 0; x < kTQPT; ++x) {
        const uint32_t t = uint32_t(x) * kTThreads + threadIdx.x;
        qq[x] = K(0);
        bb[x] = 0;
        if (t < nc) {
          qq[x] = __ldcs(q + lo + t);
          bb[x] = __ldcs(reinterpret_cast<const unsigned short*>(bq) + lo + t);
        }
      }
      for (uint32_t b = threadIdx.x; b < B; b += kTThreads) {
        s_rank[b] = 0;
        s_gb[b] = gb[c * BP + b];
        s_lb[b] = tab[c * BP + b];
      }
    }
    __syncthreads();  // the staging buffer is consumed: stream the next chunk into it
    if (threadIdx.x == 0) {
      const uint64_t cn = c + gridDim.x;
      if (cn < full) {
        fence_proxy_async_smem();
        issue(cn);
      }
    }
    block_exclusive_scan<kTThreads>(s_lb, s_lb, B, s_tmp);
#pragma unroll
    for (int x = 0; x < kTQPT; ++x) {
      const uint32_t t = uint32_t(x) * kTThreads + threadIdx.x;
      if (t < nc) {
        const uint32_t pos = s_lb[bb[x]] + atomicAdd(&s_rank[bb[x]], 1u);
        s_q[pos] = qq[x];
        s_b[pos] = uint16_t(bb[x]);
        __stcs(reinterpret_cast<unsigned short*>(linv) + lo + t, (unsigned short)pos);
      }
    }
    __syncthreads();
#pragma unroll
    for (int x = 0; x < kTQPT; ++x) {
      const uint32_t t = uint32_t(x) * kTThreads + threadIdx.x;
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
    chunk_layout(tab, gb, B, c, s_cnt, s_lb, s_gb, s_tmp);
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

// Pass 4 for 16 B result records (the item-directory searches): one pass, the
// chunk's record runs into shared memory, then {pos|found, value} in query
// order.  (Measured: splitting the chunk into two halves for two CTAs per SM
// makes each half's stores partial sectors and costs DRAM read-modify-writes,
// 0.77 -> 0.88 ms on c3.)
constexpr int kGThreads = 1024;
template <typename K, bool REMOTE>
__global__ void __launch_bounds__(kGThreads) bk_gather_rec(const uint16_t* __restrict__ linv, uint64_t m,
                                                           const uint32_t* __restrict__ tab,
                                                           const uint32_t* __restrict__ gb, uint32_t B,
                                                           uint64_t chunks, const ulonglong2* __restrict__ rec,
                                                           uint64_t* __restrict__ out_pf, K* __restrict__ out_v,
                                                           const RemoteOut ro) {
  // B <= kMaxBuckets == kGThreads: thread b owns bucket b's layout entries.  The next
  // chunk's layout row is loaded while this chunk's records are stored, and all of a
  // thread's record and linv loads are issued together (the kernel was latency
  // bound: long-scoreboard stalls 38 per issue, one CTA per SM).  REMOTE (the owner
  // side of the fused sharded exchange): query i of the receive window came from
  // rank s = org[i] >> 40, and its record is stored straight into THAT rank's result
  // window (peer memory) at i - start[s] + dst[s]: consecutive receive slots of one
  // source land on consecutive result slots there (coalesced peer stores).
  static_assert(kMaxBuckets <= kGThreads, "one bucket per thread");
  constexpr int PT = int(kChunk) / kGThreads;
  extern __shared__ __align__(16) uint8_t smem[];
  ulonglong2* s_rec = reinterpret_cast<ulonglong2*>(smem);
  uint16_t* s_b = reinterpret_cast<uint16_t*>(s_rec + kChunk);
  uint32_t* s_cnt = reinterpret_cast<uint32_t*>(s_b + kChunk);
  uint32_t* s_lb = s_cnt + kMaxBuckets;
  uint32_t* s_gb = s_lb + kMaxBuckets;
  uint32_t* s_tmp = s_gb + kMaxBuckets;
  const uint32_t tb = threadIdx.x;
  uint32_t nx_cnt = 0, nx_gb = 0;
  if (blockIdx.x < chunks && tb < B) {
    nx_cnt = tab[uint64_t(blockIdx.x) * row_stride(B) + tb];
    nx_gb = gb[uint64_t(blockIdx.x) * row_stride(B) + tb];
  }
  for (uint64_t c = blockIdx.x; c < chunks; c += gridDim.x) {
    const uint64_t lo = c * kChunk;
    const uint32_t nc = uint32_t(m - lo < kChunk ? m - lo : kChunk);
    if (tb < B) {
      s_cnt[tb] = nx_cnt;
      s_gb[tb] = nx_gb;
    }
    __syncthreads();
    block_exclusive_scan<kGThreads>(s_cnt, s_lb, B, s_tmp);
    if (tb < B)
      for (uint32_t k = 0, n = s_cnt[tb], p = s_lb[tb]; k < n; ++k) s_b[p + k] = uint16_t(tb);
    __syncthreads();
    const unsigned short* li = reinterpret_cast<const unsigned short*>(linv) + lo;
    ulonglong2 x[PT];
    unsigned short l[PT];
#pragma unroll
    for (int j = 0; j < PT; ++j) {
      const uint32_t t = uint32_t(j) * kGThreads + tb;
      if (t < nc) {
        const uint32_t b = s_b[t];
        x[j] = __ldcs(rec + s_gb[b] + (t - s_lb[b]));
        l[j] = __ldcs(li + t);
      }
    }
    {  // next chunk's layout row, in flight during the stores below
      const uint64_t cn = c + gridDim.x;
      if (cn < chunks && tb < B) {
        nx_cnt = tab[cn * row_stride(B) + tb];
        nx_gb = gb[cn * row_stride(B) + tb];
      }
    }
#pragma unroll
    for (int j = 0; j < PT; ++j) {
      const uint32_t t = uint32_t(j) * kGThreads + tb;
      if (t < nc) s_rec[t] = x[j];
    }
    __syncthreads();
    if constexpr (REMOTE) {
      uint64_t o[PT];
#pragma unroll
      for (int j = 0; j < PT; ++j) {
        const uint32_t t = uint32_t(j) * kGThreads + tb;
        o[j] = t < nc ? __ldcs(reinterpret_cast<const unsigned long long*>(ro.org) + lo + t) : 0ull;
      }
#pragma unroll
      for (int j = 0; j < PT; ++j) {
        const uint32_t t = uint32_t(j) * kGThreads + tb;
        if (t < nc) {
          const ulonglong2 r = s_rec[l[j]];
          const uint32_t src = uint32_t(o[j] >> kRemoteOrgShift);
          const uint64_t slot = lo + t - ro.start[src] + ro.dst[src];
          ro.pf[src][slot] = r.x;
          reinterpret_cast<K*>(ro.v[src])[slot] = K(r.y);
        }
      }
    } else {
#pragma unroll
      for (int j = 0; j < PT; ++j) {
        const uint32_t t = uint32_t(j) * kGThreads + tb;
        if (t < nc) {
          const ulonglong2 r = s_rec[l[j]];
          __stcs(reinterpret_cast<unsigned long long*>(out_pf) + lo + t, r.x);
          if constexpr (sizeof(K) == 8)
            __stcs(reinterpret_cast<unsigned long long*>(out_v) + lo + t, r.y);
          else
            __stcs(reinterpret_cast<unsigned int*>(out_v) + lo + t, (unsigned int)r.y);
        }
      }
    }
    __syncthreads();
  }
}

// Dynamic shared memory beyond 48 KB for the partition kernels (once per process).
void set_bucket_attrs() {
  static bool attr = false;
  if (attr) return;
  const int lim = 120 * 1024;
  cudaFuncSetAttribute(bk_count<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
  cudaFuncSetAttribute(bk_count<uint64_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
  cudaFuncSetAttribute(bk_scatter<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
  cudaFuncSetAttribute(bk_scatter<uint64_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
  cudaFuncSetAttribute(bk_scatter_tma<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       int(smem_scatter_tma<uint32_t>(kMaxBuckets)));
  cudaFuncSetAttribute(bk_scatter_tma<uint64_t>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                       int(smem_scatter_tma<uint64_t>(kMaxBuckets)));
  cudaFuncSetAttribute(bk_gather<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
  cudaFuncSetAttribute(bk_gather<uint64_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
  cudaFuncSetAttribute(bk_gather_rec<uint32_t, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  cudaFuncSetAttribute(bk_gather_rec<uint64_t, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  cudaFuncSetAttribute(bk_gather_rec<uint32_t, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  cudaFuncSetAttribute(bk_gather_rec<uint64_t, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  attr = true;
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
  // default 1 MB slices: with the 1024-bucket cap, large trees get the most
  // buckets, which keeps the item directory in shared memory (measured on c3:
  // 16 MB slices 15.0 G q/s, 1 MB 18.6 before the prefix table)
  const uint64_t slice = t->cfg.bucket_slice ? t->cfg.bucket_slice : (1ull << 20);
  const uint64_t units = t->form == HBT_IMPLICIT ? t->L0 : t->r.nchain;
  uint64_t B = (tree_bytes(t) + slice - 1) / slice;
  B = std::min<uint64_t>(B, kMaxBuckets);
  B = std::min<uint64_t>(B, units);
  return uint32_t(std::max<uint64_t>(B, 1));
}

// Units of bucket b at a directory level of `span` leaf lines per unit (the units
// holding leaf lines [floor(bU/B), floor((b+1)U/B) - 1], where b's queries end).
static inline void bucket_units(uint64_t U, uint32_t B, uint32_t b, uint64_t span, uint64_t& u0, uint64_t& u1) {
  u0 = ((uint64_t(b) * U) / B) / span;
  u1 = (((uint64_t(b) + 1) * U) / B - 1) / span;
}

// Entries of the compressed directory per bucket: below 2^16 (16-bit prefix table) and
// within ~160 KB of shared memory per CTA together with the prefix table, the bucket
// and item starts (and, regular trees, one chain id per F entries), so the L1 keeps
// >= 92 KB for the loads in flight (a 200 KB directory measured 30 % slower on c3).
uint64_t item_cap16(uint32_t B, uint32_t per_chain) {
  const uint64_t fixed = uint64_t(kT16) * 2 + (uint64_t(B) + 1) * 12 + 64 + (per_chain ? 32 : 0);
  const uint64_t per = per_chain ? 2 * uint64_t(per_chain) + 4 : 2 * uint64_t(1);  // bytes per `per_chain` entries
  const uint64_t room = (160 * 1024 - fixed) * (per_chain ? per_chain : 1) / per;
  return std::min<uint64_t>(room, 65528);
}

// Shared-memory entries of the item directory (keys; the regular tree also
// stages one u32 chain id per NI entries): ~150 KB per CTA beside the bucket starts.
uint64_t item_cap(const hbt_tree* t, uint32_t B) {
  const uint64_t budget = 150 * 1024 - (uint64_t(B) + 1) * 8;
  const uint64_t per = t->width + (t->form == HBT_REGULAR ? 4 : 0);
  return budget / per;
}

// Splitters, prefix directory and item-directory maxima of one bucket state, derived
// from the tree on first use and after every update / bucketing knob change.  The
// arrays are shared by every search on the tree, so preparation is serialised
// (t->bk_mu) and completes on the HOST before it is marked valid: a search on another
// stream can never read half-written splitters.  A re-preparation rewrites the arrays
// in place, so it first waits for the device to drain (searches in flight on other
// streams may still read the old ones).
template <typename K>
int prepare_splitters(const hbt_tree* t, cudaStream_t s, BucketState& bs, uint32_t B, bool want_items) {
  std::lock_guard<std::mutex> lock(t->bk_mu);
  if (bs.valid && bs.B == B) return HBT_OK;
  bs.valid = false;
  if (bs.d_sp) HBT_CUDA_TRY(cudaDeviceSynchronize());
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
  // Item directory: the deepest unit level whose range for two buckets fits the
  // shared-memory capacity.
  bs.items = false;
  if (want_items && t->cfg.bucket_items) {
    const uint64_t cap = item_cap(t, B);
    uint64_t nunits = 0;
    bs.cdir = false;
    if (t->form == HBT_IMPLICIT) {
      uint64_t span = 1;
      for (int d = int(t->H); d >= 0; --d) {
        const uint64_t units = d == int(t->H) ? t->L0 : t->nodes[d];
        if (2 * ((t->L0 / B) / span + 2) <= cap) {
          bs.level = uint32_t(d);
          bs.span = span;
          nunits = units;
          bs.items = true;
          break;
        }
        span *= t->F;
      }
      // the compressed per-bucket form, where it reaches a deeper level (or when forced)
      if (t->cfg.item_cdir && !t->cfg.bucket_cap) {
        const uint64_t cap16 = item_cap16(B, 0);
        uint64_t span32 = 1;
        for (int d = int(t->H); d >= 0; --d) {
          uint64_t most = 0;
          for (uint32_t b = 0; b < B; ++b) {
            uint64_t u0, u1;
            bucket_units(t->L0, B, b, span32, u0, u1);
            most = std::max<uint64_t>(most, u1 - u0 + 1);
          }
          if (most <= cap16) {
            if (!bs.items || d > int(bs.level) || t->cfg.item_cdir == 2) {
              bs.level = uint32_t(d);
              bs.span = span32;
              nunits = d == int(t->H) ? t->L0 : t->nodes[d];
              bs.items = true;
              bs.cdir = true;
              bs.cap16 = uint32_t((most + 7) & ~uint64_t(7));
            }
            break;
          }
          span32 *= t->F;
        }
      }
    } else {
      const uint32_t KPL = 64 / sizeof(K);
      const uint32_t NI = t->F > KPL ? t->F / KPL : 1;
      if (2 * ((t->r.nchain / B) + 2) * NI <= cap) {
        bs.span = NI;
        nunits = t->r.nchain * NI;
        bs.items = true;
      }
      // the compressed per-bucket form on the LEAF LINES (F per chain leaf): the search
      // goes from the directory straight to the leaf line (regular_search_items32_kernel)
      if (t->cfg.item_cdir && !t->cfg.bucket_cap) {
        uint64_t most = 0;
        for (uint32_t b = 0; b < B; ++b) {
          uint64_t c0, c1;
          bucket_units(t->r.nchain, B, b, 1, c0, c1);
          most = std::max<uint64_t>(most, (c1 - c0 + 1) * t->F);
        }
        if (most + 8 <= item_cap16(B, t->F)) {
          bs.span = t->F;
          nunits = t->r.nchain * t->F;
          bs.items = true;
          bs.cdir = true;
          bs.cap16 = uint32_t((most + 7) & ~uint64_t(7));
        }
      }
    }
    if (bs.items) {
      const uint64_t bytes = std::max<uint64_t>(nunits, 1) * sizeof(K);
      if (bs.M_cap < bytes) {
        cudaFree(bs.d_M);
        bs.d_M = nullptr;
        bs.M_cap = 0;
        HBT_CUDA_TRY(cudaMalloc(&bs.d_M, bytes));
        bs.M_cap = bytes;
      }
      bs.nunits = nunits;
      if (t->form == HBT_IMPLICIT)
        bk_level_max<K><<<t->num_sms * 4, 256, 0, s>>>((const uint8_t*)t->d_leaf, t->n, t->P, bs.span, nunits,
                                                        (K*)bs.d_M);
      else  // key lines (NI per leaf, KPL lines of P each) or, compressed form, leaf lines (F, 1)
        bk_keyline_max<K><<<t->num_sms * 4, 256, 0, s>>>((const uint8_t*)t->r.d_leaf, t->r.d_count, t->r.d_chain,
                                                          t->r.nchain, t->F, t->P, uint32_t(bs.span),
                                                          bs.cdir ? 1u : uint32_t(64 / sizeof(K)), (K*)bs.d_M);
      HBT_CUDA_TRY(cudaGetLastError());
    }
    if (bs.cdir) {
      std::vector<BucketDir> h(B);
      uint64_t total = 0;
      for (uint32_t b = 0; b < B; ++b) {
        uint64_t u0, u1;
        if (t->form == HBT_IMPLICIT) {
          bucket_units(t->L0, B, b, bs.span, u0, u1);
        } else {  // the lines of chain leaves [c0, c1]
          bucket_units(t->r.nchain, B, b, 1, u0, u1);
          u0 *= t->F;
          u1 = u1 * t->F + t->F - 1;
        }
        h[b] = BucketDir{u0, total, 0, uint32_t(u1 - u0 + 1), 0, 0, 0, 0, 0};
        total += (u1 - u0 + 1 + 7) & ~uint64_t(7);
      }
      if (!bs.d_bd) HBT_CUDA_TRY(cudaMalloc(&bs.d_bd, kMaxBuckets * sizeof(BucketDir)));
      const uint64_t bytes = total * 2 + uint64_t(B) * kT16 * 2;
      if (bs.E16_cap < bytes) {
        cudaFree(bs.d_E16);
        bs.d_E16 = nullptr;
        bs.E16_cap = 0;
        HBT_CUDA_TRY(cudaMalloc(&bs.d_E16, bytes));
        bs.E16_cap = bytes;
      }
      bs.d_T16 = bs.d_E16 + total;
      HBT_CUDA_TRY(cudaMemcpyAsync(bs.d_bd, h.data(), B * sizeof(BucketDir), cudaMemcpyHostToDevice, s));
      bk_cdir<K><<<B, 256, 0, s>>>((const K*)bs.d_M, (BucketDir*)bs.d_bd, bs.d_E16, bs.d_T16);
      HBT_CUDA_TRY(cudaGetLastError());
      // compact copies of the directory level's nodes where that level is read as whole
      // nodes from HBM (c4: the last inner level, 4 GB -> 1 GB)
      bs.cnode = false;
      // (the last inner level only: a tie there puts the walk at most a few leaf lines early)
      if (t->form == HBT_IMPLICIT && sizeof(K) == 8 && t->F == 16 && t->H >= 1 && bs.level == t->H - 1 &&
          t->cfg.item_cnode) {
        bool full = t->cfg.item_cnode == 2;
        if (!full) {
          uint64_t cum = 0;
          const uint64_t budget = t->cfg.l2_levels_bytes ? t->cfg.l2_levels_bytes : (32ull << 20);
          for (uint32_t x = bs.level; x < t->H; ++x) cum += t->nodes[x] * uint64_t(16 * 8 + 32);
          full = cum > budget;
        }
        if (full) {
          const uint64_t bytes = t->nodes[bs.level] * 32;
          if (bs.cnode_cap < bytes) {
            cudaFree(bs.d_cnode);
            bs.d_cnode = nullptr;
            bs.cnode_cap = 0;
            HBT_CUDA_TRY(cudaMalloc(&bs.d_cnode, bytes));
            bs.cnode_cap = bytes;
          }
          bk_cnode<<<B, 256, 0, s>>>(reinterpret_cast<const uint64_t*>(static_cast<const uint8_t*>(t->d_inner) +
                                                                         t->offset[bs.level] * 128),
                                     (BucketDir*)bs.d_bd, reinterpret_cast<uint4*>(bs.d_cnode));
          HBT_CUDA_TRY(cudaGetLastError());
          bs.cnode = true;
        }
      }
    }
  }
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  bs.B = B;
  bs.valid = true;
  return HBT_OK;
}

// Scratch layout and geometry of one partitioned batch (stream-ordered pool).
struct Part {
  uint32_t B = 0;
  uint64_t chunks = 0, kps = 0, nseg = 0;
  uint8_t* base = nullptr;
  uint64_t o_pf = 0, o_v = 0, o_bq = 0, o_li = 0, o_tab = 0, o_gb = 0, o_seg = 0, o_so = 0, o_bs = 0, total = 0;
  template <typename T> T* at(uint64_t o) const { return reinterpret_cast<T*>(base + o); }
};

// qs (m x S) | results: pf_s (m x 8) + v_s (m x 8), or 16 B records over the same
// 16 m bytes | bq (u16) | linv (u16) | tab, gb (chunks x B) | seg, segoff (nseg x B) |
// bucket starts (B + 1)
template <typename K>
Part part_layout(uint64_t m, uint32_t B, uint32_t sms) {
  Part p;
  p.B = B;
  p.chunks = (m + kChunk - 1) / kChunk;
  const uint64_t want = std::min<uint64_t>(p.chunks, uint64_t(sms) * 2);
  p.kps = (p.chunks + want - 1) / want;
  p.nseg = (p.chunks + p.kps - 1) / p.kps;
  auto al = [](uint64_t x) { return (x + 255) & ~uint64_t(255); };
  p.o_pf = al(m * sizeof(K));
  p.o_v = p.o_pf + al(m * 8);
  p.o_bq = p.o_v + al(m * 8);
  p.o_li = p.o_bq + al(m * 2);
  p.o_tab = p.o_li + al(m * 2);
  p.o_gb = p.o_tab + al(p.chunks * row_stride(B) * 4);
  p.o_seg = p.o_gb + al(p.chunks * row_stride(B) * 4);
  p.o_so = p.o_seg + al(p.nseg * B * 4);
  p.o_bs = p.o_so + al(p.nseg * B * 4);
  p.total = p.o_bs + al((uint64_t(B) + 1) * 8);
  return p;
}

constexpr size_t kSmemCount = (1u << kDirBits) * 4 + kMaxBuckets * 4 * 2 + kMaxBuckets * 8;
template <typename K>
constexpr size_t smem_scatter() { return kChunk * (sizeof(K) + 2) + kMaxBuckets * 4 * 4 + kThreads * 4; }
constexpr size_t kSmemGather = kChunk * (8 + 2) + kMaxBuckets * 4 * 3 + kThreads * 4;
constexpr size_t kSmemGatherRec = kChunk * (16 + 2) + kMaxBuckets * 4 * 3 + kGThreads * 4;

// count -> run starts -> scatter: the batch q in bucket order at qs (Part::base).
template <typename K>
int partition(const hbt_tree* t, const BucketState& bs, const void* q, uint64_t m, const Part& p, cudaStream_t s,
              const std::function<void(int)>& mark) {
  NvtxRange nvtx_("bucket.partition");
  set_bucket_attrs();
  const unsigned grid = unsigned(std::min<uint64_t>(p.nseg, uint64_t(t->num_sms) * 2));
  mark(0);
  bk_count<K><<<grid, kThreads, kSmemCount, s>>>((const K*)q, m, (const K*)bs.d_sp, bs.d_dir, p.B, p.chunks, p.kps,
                                                 p.nseg, p.at<uint16_t>(p.o_bq), p.at<uint32_t>(p.o_tab),
                                                 p.at<uint32_t>(p.o_seg));
  mark(1);
  bk_seg_scan<<<1, kScanThreads, 0, s>>>(p.at<uint32_t>(p.o_seg), p.B, p.nseg, m, p.at<uint32_t>(p.o_so),
                                         p.at<uint64_t>(p.o_bs));
  bk_run_starts<<<unsigned(p.nseg), kScanThreads, 0, s>>>(p.at<uint32_t>(p.o_tab), p.at<uint32_t>(p.o_so), p.B,
                                                          p.chunks, p.kps, p.at<uint32_t>(p.o_gb));
  mark(2);
  if (t->cfg.scatter_tma && m >= kChunk && (reinterpret_cast<uintptr_t>(q) & 15u) == 0) {
    const unsigned sgrid = unsigned(std::min<uint64_t>(p.chunks, uint64_t(t->num_sms)));
    bk_scatter_tma<K><<<sgrid, kTThreads, smem_scatter_tma<K>(p.B), s>>>(
        (const K*)q, m, p.at<uint16_t>(p.o_bq), p.at<uint32_t>(p.o_tab), p.at<uint32_t>(p.o_gb), p.B, p.chunks,
        p.at<K>(0), p.at<uint16_t>(p.o_li));
  } else {
    const unsigned sgrid = unsigned(std::min<uint64_t>(p.chunks, uint64_t(t->num_sms) * 2));
    bk_scatter<K><<<sgrid, kThreads, smem_scatter<K>(), s>>>((const K*)q, m, p.at<uint16_t>(p.o_bq),
                                                             p.at<uint32_t>(p.o_tab), p.at<uint32_t>(p.o_gb), p.B,
                                                             p.chunks, p.at<K>(0), p.at<uint16_t>(p.o_li));
  }
  if (cudaError_t e = cudaGetLastError(); e != cudaSuccess) {
    set_error("bucketing kernels failed to launch: %s", cudaGetErrorString(e));
    return HBT_ECUDA;
  }
  mark(3);
  return HBT_OK;
}

template <typename K>
int bucketed_t(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t pos_base,
               cudaStream_t s, const RemoteOut* ro) {
  int rc = prepare_splitters<K>(t, s, t->bk, pick_buckets(t), true);
  if (rc != HBT_OK) return rc;
  const BucketState& bs = t->bk;
  if (ro && !bs.items) {
    set_error("remote result stores need the bucket-local item directory");
    return HBT_EUNSUPPORTED;
  }
  Part p = part_layout<K>(m, bs.B, uint32_t(t->num_sms));
  void* buf = nullptr;
  HBT_CUDA_TRY(scratch_alloc(&buf, p.total, s));
  p.base = static_cast<uint8_t*>(buf);
  K* qs = p.at<K>(0);
  uint64_t* pf_s = p.at<uint64_t>(p.o_pf);
  K* v_s = p.at<K>(p.o_v);
  BucketState& bw = t->bk;
  const bool timing = t->cfg.phase_timing != 0;
  if (timing && !bw.ev[0])
    for (auto& e : bw.ev) HBT_CUDA_TRY(cudaEventCreate(&e));
  auto mark = [&](int i) {
    if (timing) cudaEventRecord(bw.ev[i], s);
  };
  do {
    if ((rc = partition<K>(t, bs, q, m, p, s, mark)) != HBT_OK) break;
    if (bs.items) {
      ItemDir d;
      d.M = bs.d_M;
      d.chain = t->form == HBT_REGULAR ? t->r.d_chain : nullptr;
      d.bstart = p.at<uint64_t>(p.o_bs);
      d.B = p.B;
      d.U = t->form == HBT_IMPLICIT ? t->L0 : t->r.nchain;
      d.level = bs.level;
      d.span = bs.span;
      d.nunits = bs.nunits;
      d.pos_base = pos_base;
      d.cap = t->cfg.bucket_cap ? std::min<uint32_t>(t->cfg.bucket_cap, uint32_t(item_cap(t, p.B)))
                                : uint32_t(item_cap(t, p.B));
      if (bs.cdir) {
        d.bd = static_cast<const BucketDir*>(bs.d_bd);
        d.E16 = bs.d_E16;
        d.T16 = bs.d_T16;
        d.cap = bs.cap16;
        if (bs.cnode) d.cnode = bs.d_cnode;
      }
      rc = t->form == HBT_IMPLICIT ? implicit_search_items(t, qs, m, pf_s, v_s, d, s)
                                   : regular_search_items(t, qs, m, pf_s, v_s, d, s);
    } else {
      rc = t->form == HBT_REGULAR ? regular_search(t, qs, m, pf_s, v_s, s)
                                  : implicit_search_base(t, qs, m, pf_s, v_s, pos_base, s);
    }
    if (rc != HBT_OK) break;
    mark(4);
    const uint16_t* linv = p.at<uint16_t>(p.o_li);
    const uint32_t* tab = p.at<uint32_t>(p.o_tab);
    const uint32_t* gb = p.at<uint32_t>(p.o_gb);
    if (bs.items) {
      const unsigned g = unsigned(std::min<uint64_t>(p.chunks, t->num_sms));
      const ulonglong2* rec = reinterpret_cast<const ulonglong2*>(pf_s);
      if (ro)
        bk_gather_rec<K, true><<<g, kGThreads, kSmemGatherRec, s>>>(linv, m, tab, gb, p.B, p.chunks, rec, nullptr,
                                                                    nullptr, *ro);
      else
        bk_gather_rec<K, false><<<g, kGThreads, kSmemGatherRec, s>>>(linv, m, tab, gb, p.B, p.chunks, rec, pf, (K*)v,
                                                                     RemoteOut{});
    } else {
      const unsigned g = unsigned(std::min<uint64_t>(p.chunks, uint64_t(t->num_sms) * 2));
      bk_gather<K><<<g, kThreads, kSmemGather, s>>>(linv, m, tab, gb, p.B, p.chunks, pf_s, v_s, pf, (K*)v);
    }
    if (cudaError_t e = cudaGetLastError(); e != cudaSuccess) {
      set_error("bucket gather failed to launch: %s", cudaGetErrorString(e));
      rc = HBT_ECUDA;
      break;
    }
    mark(5);
    bw.launches = 6;  // count, run-start scan, run starts, scatter, search, gather
    bw.timed = timing;
  } while (0);
  scratch_free(buf, s);
  return rc;
}

// ---- streamed host L-segment (the paper's bucket pipeline with double
// buffering, turned around: the BATCH is bucketed on the GPU and the
// L-SEGMENT slices stream host -> HBM).  With the L-segment in pinned host memory a
// batch that touches most of it is cheaper to serve by copying each bucket's leaf
// slice into HBM at the link's copy rate than by one random 64 B zero-copy read per
// query (measured 22 GB/s vs a 55 GB/s copy rate).  Bucket b's queries all answer in
// the leaf lines [floor(bU/B), floor((b+1)U/B)) (sp[b-1] < q <= sp[b], DESIGN.md
// 'Bucketed search'), so its search reads only that staged slice; the inner levels
// stay in HBM.  Slice copies (one stream) alternate between two staging slots and
// overlap the previous bucket's search; results are identical.
uint64_t stream_slice_bytes(const hbt_tree* t) {
  return t->cfg.stream_slice ? t->cfg.stream_slice : (8ull << 20);
}

uint32_t pick_stream_buckets(const hbt_tree* t) {
  uint64_t B = (t->leaf_bytes + stream_slice_bytes(t) - 1) / stream_slice_bytes(t);
  B = std::min<uint64_t>(B, kMaxBuckets);
  B = std::min<uint64_t>(B, t->L0);
  return uint32_t(std::max<uint64_t>(B, 1));
}

template <typename K>
int streamed_t(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t pos_base,
               cudaStream_t s) {
  // one user of the staging slots at a time (not pipe.mu: hbt_search_host holds it
  // while its chunks come through here)
  std::lock_guard<std::mutex> lock(t->stream_mu);
  BucketState& bs = t->bks;
  const uint32_t B = pick_stream_buckets(t);
  int rc = prepare_splitters<K>(t, s, bs, B, false);
  if (rc != HBT_OK) return rc;
  const uint64_t U = t->L0;
  const uint64_t slice_lines = (U + B - 1) / B + 1;
  if (bs.stage_cap < slice_lines * 64) {
    cudaFree(bs.d_stage[0]);
    bs.d_stage[0] = bs.d_stage[1] = nullptr;
    bs.stage_cap = 0;
    HBT_CUDA_TRY(cudaMalloc(&bs.d_stage[0], 2 * slice_lines * 64));
    bs.d_stage[1] = static_cast<uint8_t*>(bs.d_stage[0]) + slice_lines * 64;
    bs.stage_cap = slice_lines * 64;
  }
  if (!bs.cs) {
    HBT_CUDA_TRY(cudaStreamCreateWithFlags(&bs.cs, cudaStreamNonBlocking));
    for (int i = 0; i < 2; ++i) {
      HBT_CUDA_TRY(cudaEventCreateWithFlags(&bs.ev_copy[i], cudaEventDisableTiming));
      HBT_CUDA_TRY(cudaEventCreateWithFlags(&bs.ev_done[i], cudaEventDisableTiming));
      HBT_CUDA_TRY(cudaEventRecord(bs.ev_done[i], s));  // slots start free
    }
  }
  Part p = part_layout<K>(m, B, uint32_t(t->num_sms));
  void* buf = nullptr;
  HBT_CUDA_TRY(scratch_alloc(&buf, p.total, s));
  p.base = static_cast<uint8_t*>(buf);
  K* qs = p.at<K>(0);
  uint64_t* pf_s = p.at<uint64_t>(p.o_pf);
  K* v_s = p.at<K>(p.o_v);
  std::vector<uint64_t> hb(B + 1);
  do {
    if ((rc = partition<K>(t, bs, q, m, p, s, [](int) {})) != HBT_OK) break;
    // the bucket boundaries drive the host loop below (one sync per batch)
    HBT_CUDA_TRY(cudaMemcpyAsync(hb.data(), p.at<uint64_t>(p.o_bs), (B + 1) * 8, cudaMemcpyDeviceToHost, s));
    HBT_CUDA_TRY(cudaStreamSynchronize(s));
    const uint8_t* hl = static_cast<const uint8_t*>(t->h_leaf);
    uint32_t j = 0;
    for (uint32_t b = 0; b < B && rc == HBT_OK; ++b) {
      const uint64_t cnt = hb[b + 1] - hb[b];
      if (!cnt) continue;
      const uint64_t u_lo = (uint64_t(b) * U) / B, u_hi = ((uint64_t(b) + 1) * U) / B;
      const int slot = int(j++ & 1);
      uint8_t* st = static_cast<uint8_t*>(bs.d_stage[slot]);
      HBT_CUDA_TRY(cudaStreamWaitEvent(bs.cs, bs.ev_done[slot], 0));
      HBT_CUDA_TRY(cudaMemcpyAsync(st, hl + u_lo * 64, (u_hi - u_lo) * 64, cudaMemcpyHostToDevice, bs.cs));
      HBT_CUDA_TRY(cudaEventRecord(bs.ev_copy[slot], bs.cs));
      HBT_CUDA_TRY(cudaStreamWaitEvent(s, bs.ev_copy[slot], 0));
      rc = implicit_search_leaf(t, qs + hb[b], cnt, pf_s + hb[b], v_s + hb[b], pos_base,
                                st - int64_t(u_lo) * 64, s);
      HBT_CUDA_TRY(cudaEventRecord(bs.ev_done[slot], s));
    }
    if (rc != HBT_OK) break;
    const unsigned g = unsigned(std::min<uint64_t>(p.chunks, uint64_t(t->num_sms) * 2));
    bk_gather<K><<<g, kThreads, kSmemGather, s>>>(p.at<uint16_t>(p.o_li), m, p.at<uint32_t>(p.o_tab),
                                                 p.at<uint32_t>(p.o_gb), B, p.chunks, pf_s, v_s, pf, (K*)v);
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

bool leaf_stream_enabled(const hbt_tree* t, uint64_t m) {
  if (t->form != HBT_IMPLICIT || !t->h_leaf || m == 0 || m >= (1ull << 32)) return false;
  const uint32_t mode = t->cfg.leaf_stream;
  if (mode == 0 || pick_stream_buckets(t) < 2) return false;
  if (mode == 1) return true;
  // auto: stream when the batch's random 64 B link reads (~22 GB/s measured) would
  // cost more than copying the whole L-segment (~55 GB/s): m * 64 / 22 > L / 55
  return m * 160 > t->leaf_bytes;
}

int streamed_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t pos_base,
                    cudaStream_t s) {
  return t->width == 4 ? streamed_t<uint32_t>(t, q, m, pf, v, pos_base, s)
                       : streamed_t<uint64_t>(t, q, m, pf, v, pos_base, s);
}

bool bucketed_enabled(const hbt_tree* t, uint64_t m) {
  const uint32_t mode = t->cfg.bucket;
  if (mode == 0 || m >= (1ull << 32)) return false;
  if (mode == 2 && m < (1ull << 22)) return false;  // auto: small batches never (no host calls)
  if (pick_buckets(t) < 2) return false;
  if (mode == 1) return true;
  // auto: batches large enough to share lines, trees beyond 8x the L2 (measured: c3
  // regular 10.9 -> 24 G q/s; c5 implicit Zipf 2^27 keys 2.84 -> 2.71 ms once the scatter
  // used bulk-copy staging, profiles/r02_c5_c2_bucket_ab.jsonl; c2's 150 MB tree stays
  // unbucketed: 0.41 vs 0.66 ms)
  static int l2 = 0;  // one device model per process
  if (!l2) cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, t->device);
  return tree_bytes(t) > 8ull * uint64_t(l2);
}

int bucketed_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t pos_base,
                    cudaStream_t s, const RemoteOut* ro) {
  return t->width == 4 ? bucketed_t<uint32_t>(t, q, m, pf, v, pos_base, s, ro)
                       : bucketed_t<uint64_t>(t, q, m, pf, v, pos_base, s, ro);
}

int shard_local_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t pos_base,
                       cudaStream_t s) {
  if (bucketed_enabled(t, m)) return bucketed_search(t, q, m, pf, v, pos_base, s);
  return implicit_search_base(t, q, m, pf, v, pos_base, s);
}

static void bucket_state_free(BucketState& b) {
  for (auto& e : b.ev)
    if (e) cudaEventDestroy(e);
  for (int i = 0; i < 2; ++i) {
    if (b.ev_copy[i]) cudaEventDestroy(b.ev_copy[i]);
    if (b.ev_done[i]) cudaEventDestroy(b.ev_done[i]);
  }
  if (b.cs) cudaStreamDestroy(b.cs);
  cudaFree(b.d_stage[0]);
  cudaFree(b.d_sp);
  cudaFree(b.d_dir);
  cudaFree(b.d_M);
  cudaFree(b.d_bd);
  cudaFree(b.d_E16);
  cudaFree(b.d_cnode);
  b = BucketState{};
}

void bucket_free(hbt_tree* t) {
  bucket_state_free(t->bk);
  bucket_state_free(t->bks);
}

}  // namespace hbt
