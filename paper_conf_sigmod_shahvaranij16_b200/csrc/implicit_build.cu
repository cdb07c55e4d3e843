// implicit_build.cu — hbt_bulk_build / hbt_bulk_update for the IMPLICIT tree.
//
// Layout:
//   L-segment: L0 = max(1, ceil(n'/P)) lines of 64 B = [P keys | P values],
//              rank r at line r/P slot r%P, padding (MAX, 0)
//   I-segment: inner levels root-first, node = F keys of S bytes (F*S-byte
//              aligned), child i of node j at level d+1 index j*F + i;
//              key slot i = max key of child i's subtree for i < cnt-1, else MAX
//              (reading R3; slot F-1 always MAX).
// The separators are gathered with the closed form
//   sep(h, j, i) = Kd[min(n', (j*F + i + 1) * F^(h-1) * P) - 1]
// from the sorted distinct key array (one kernel for all levels), so the build
// is: CUB radix sort (stable) -> keep-last-of-run compaction -> pack -> gather.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_select.cuh>

#include "hbt_internal.cuh"

namespace hbt {
namespace {

template <typename K>
__host__ __device__ constexpr K key_max() { return K(~K(0)); }

template <typename K>
__global__ void last_of_run_flags(const K* __restrict__ sk, uint64_t n, uint8_t* __restrict__ flags) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
    flags[i] = (i + 1 == n) || (sk[i] != sk[i + 1]);
}

template <typename K>
__global__ void pack_leaf_lines(const K* __restrict__ kd, const K* __restrict__ vd, uint64_t nd, uint64_t L0,
                                K* __restrict__ leaf) {
  constexpr uint32_t P = 64 / (2 * sizeof(K));
  const uint64_t total = L0 * P;
  for (uint64_t r = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; r < total; r += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t line = r / P, s = r % P;
    K* L = leaf + line * (2 * P);
    L[s] = r < nd ? kd[r] : key_max<K>();
    L[P + s] = r < nd ? vd[r] : K(0);
  }
}

template <typename K>
__global__ void gather_separators(const K* __restrict__ kd, uint64_t nd, const LevelTable lt, uint64_t L0,
                                  uint32_t F, K* __restrict__ inner) {
  constexpr uint32_t P = 64 / (2 * sizeof(K));
  const uint32_t H = lt.H;
  const uint64_t total = lt.offset[H] * F;
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < total; x += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t node = x / F;
    const uint32_t i = uint32_t(x % F);
    uint32_t d = 0;
    while (node >= lt.offset[d + 1]) ++d;
    const uint64_t j = node - lt.offset[d];
    const uint32_t h = H - d;  // height >= 1
    const uint64_t below = (d + 1 < H) ? (lt.offset[d + 2] - lt.offset[d + 1]) : L0;
    const uint64_t first = j * F;
    const uint64_t cnt = (below - first < F) ? (below - first) : F;
    K key = key_max<K>();
    if (i + 1 < cnt) {
      uint64_t span = P;  // ranks covered by one child: F^(h-1) * P
      for (uint32_t e = 1; e < h; ++e) span *= F;
      uint64_t end = (first + i + 1) * span;
      if (end > nd) end = nd;
      key = kd[end - 1];
    }
    inner[x] = key;
  }
}

// Index sector of every inner node: entry t = node key t*KPS + KPS - 1 (the max
// key of the node's t-th 32 B sector), entries >= NSEC are MAX.
template <typename K>
__global__ void derive_inner_index(const K* __restrict__ inner, uint64_t nodes, uint32_t F, uint32_t idx_entries,
                                   K* __restrict__ idx) {
  constexpr uint32_t KPS = 32 / sizeof(K);
  const uint32_t nsec = F / KPS;
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < nodes * idx_entries;
       x += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t node = x / idx_entries;
    const uint32_t t = uint32_t(x % idx_entries);
    idx[x] = t < nsec ? inner[node * F + t * KPS + KPS - 1] : key_max<K>();
  }
}

// Directory (search mode 2).  The descent through levels 0..T-1 reaches the
// FIRST level-T node whose subtree max key is >= q (or the last node): at every
// level the child picked is #{sep < q} with sep = child max keys and the last
// slot MAX (R1, R3).  So node_T(q) = lower_bound(M_T, q) with M_T[j] = the max
// key below node j and M_T[last] = MAX.  dir[p] = [node_T(p << shift),
// node_T(((p + 1) << shift) - 1)] bounds that lower bound for every q of prefix p
// (node_T is monotone in q), so the search = one dir lookup + a binary search of
// M_T restricted to that range.  Exact for any key distribution.
template <typename K>
__global__ void build_dir_max(const K* __restrict__ leaf, uint64_t nd, uint64_t count, uint64_t span,
                              K* __restrict__ M) {
  constexpr uint32_t P = 64 / (2 * sizeof(K));
  for (uint64_t j = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; j < count; j += uint64_t(gridDim.x) * blockDim.x) {
    if (j + 1 == count || nd == 0) {
      M[j] = key_max<K>();
    } else {
      uint64_t end = (j + 1) * span;
      if (end > nd) end = nd;
      const uint64_t r = end - 1;
      M[j] = leaf[(r / P) * (2 * P) + r % P];
    }
  }
}

template <typename K>
__device__ __forceinline__ uint32_t lower_bound_dev(const K* M, uint32_t count, K q) {
  uint32_t lo = 0, hi = count - 1;  // M[count-1] = MAX >= q
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (M[mid] < q) lo = mid + 1; else hi = mid;
  }
  return lo;
}

template <typename K>
__global__ void build_dir_table(const K* __restrict__ M, uint32_t count, uint32_t bits, uint32_t* __restrict__ dir) {
  const uint32_t shift = 8 * sizeof(K) - bits;
  for (uint64_t p = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; p < (1ull << bits); p += uint64_t(gridDim.x) * blockDim.x) {
    const K first = K(K(p) << shift);
    const K last = K(first | K((K(1) << shift) - 1));
    const uint32_t lo = lower_bound_dev(M, count, first);
    const uint32_t hi = lower_bound_dev(M, count, last);
    dir[p] = lo | (hi << 16);
  }
}


template <typename K>
__global__ void unpack_leaf_lines(const K* __restrict__ leaf, uint64_t nd, K* __restrict__ kd, K* __restrict__ vd) {
  constexpr uint32_t P = 64 / (2 * sizeof(K));
  for (uint64_t r = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; r < nd; r += uint64_t(gridDim.x) * blockDim.x) {
    const K* L = leaf + (r / P) * (2 * P);
    kd[r] = L[r % P];
    vd[r] = L[P + r % P];
  }
}

// Update merge: concatenated (base ++ batch) sorted stably by key; the last
// element of each key run decides (base entry: keep; UPSERT: keep with the
// op's value; DELETE: drop).  Batch entries follow base entries in the
// concatenation, so "last" = the batch's last op on the key (reading R12).
template <typename K>
__global__ void merge_flags(const K* __restrict__ sk, const uint32_t* __restrict__ sidx, uint64_t total,
                            uint64_t n_base, const uint8_t* __restrict__ ops, uint8_t* __restrict__ flags) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < total; i += uint64_t(gridDim.x) * blockDim.x) {
    const bool last = (i + 1 == total) || (sk[i] != sk[i + 1]);
    const uint64_t src = sidx[i];
    const bool del = src >= n_base && ops[src - n_base] != 0;
    flags[i] = last && !del;
  }
}

template <typename K>
__global__ void merge_gather_values(const uint32_t* __restrict__ sidx, uint64_t total, uint64_t n_base,
                                    const K* __restrict__ base_v, const K* __restrict__ batch_v,
                                    K* __restrict__ out_v) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < total; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t src = sidx[i];
    out_v[i] = src < n_base ? base_v[src] : batch_v[src - n_base];
  }
}

__global__ void iota_u32(uint32_t* p, uint64_t n) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
    p[i] = uint32_t(i);
}

inline unsigned grid_for(uint64_t n) {
  uint64_t g = (n + 255) / 256;
  if (g > 148 * 64) g = 148 * 64;
  return unsigned(g ? g : 1);
}

// 1 if keys[] is strictly increasing (already sorted and distinct), else 0.
template <typename K>
__global__ void strictly_increasing(const K* __restrict__ k, uint64_t n, int* __restrict__ bad) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i + 1 < n; i += uint64_t(gridDim.x) * blockDim.x)
    if (!(k[i] < k[i + 1])) { *bad = 1; return; }
}

template <typename K>
int is_sorted_distinct(const void* keys, uint64_t n, bool* out, cudaStream_t s) {
  *out = false;
  int* d = nullptr;
  HBT_CUDA_TRY(cudaMalloc(&d, sizeof(int)));
  cudaMemsetAsync(d, 0, sizeof(int), s);
  strictly_increasing<K><<<grid_for(n), 256, 0, s>>>((const K*)keys, n, d);
  int h = 1;
  cudaMemcpyAsync(&h, d, sizeof(int), cudaMemcpyDeviceToHost, s);
  cudaError_t e = cudaStreamSynchronize(s);
  cudaFree(d);
  if (e != cudaSuccess) { set_error("sorted check: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
  *out = (h == 0);
  return HBT_OK;
}

template <typename K>
int sort_dedupe_t(const void* keys, const void* values, uint64_t n, void** out_k, void** out_v, uint64_t* nd,
                  cudaStream_t s) {
  *out_k = *out_v = nullptr;
  *nd = 0;
  if (n == 0) return HBT_OK;
  K *sk = nullptr, *sv = nullptr, *kd = nullptr, *vd = nullptr;
  uint8_t* flags = nullptr;
  void* tmp = nullptr;
  int64_t* d_nsel = nullptr;
  size_t tb = 0, tb2 = 0;
  int rc = HBT_OK;
  auto fail = [&](int code) {
    scratch_free(sk, s); scratch_free(sv, s); scratch_free(kd, s); scratch_free(vd, s); scratch_free(flags, s);
    scratch_free(tmp, s); scratch_free(d_nsel, s);
    return code;
  };
#define TRY(x)                                                                          \
  do {                                                                                  \
    cudaError_t _e = (x);                                                               \
    if (_e != cudaSuccess) {                                                            \
      set_error("%s:%d %s: %s", __FILE__, __LINE__, #x, cudaGetErrorString(_e));         \
      return fail(_e == cudaErrorMemoryAllocation ? HBT_ENOMEM : HBT_ECUDA);            \
    }                                                                                   \
  } while (0)
  TRY(scratch_alloc((void**)&sk, n * sizeof(K), s));
  TRY(scratch_alloc((void**)&sv, n * sizeof(K), s));
  TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, (const K*)keys, sk, (const K*)values, sv, n, 0,
                                      int(8 * sizeof(K)), s));
  TRY(cub::DeviceSelect::Flagged(nullptr, tb2, sk, flags, kd, d_nsel, int64_t(n), s));
  if (tb2 > tb) tb = tb2;
  TRY(scratch_alloc((void**)&tmp, tb, s));
  // Stable LSD radix sort: equal keys keep input order, so the last element of
  // each run is the key's last occurrence (dedupe-last-wins, reading R4).
  TRY(cub::DeviceRadixSort::SortPairs(tmp, tb, (const K*)keys, sk, (const K*)values, sv, n, 0,
                                      int(8 * sizeof(K)), s));
  TRY(scratch_alloc((void**)&flags, n, s));
  TRY(scratch_alloc((void**)&d_nsel, sizeof(int64_t), s));
  last_of_run_flags<K><<<grid_for(n), 256, 0, s>>>(sk, n, flags);
  TRY(cudaGetLastError());
  TRY(scratch_alloc((void**)&kd, n * sizeof(K), s));
  TRY(scratch_alloc((void**)&vd, n * sizeof(K), s));
  TRY(cub::DeviceSelect::Flagged(tmp, tb, sk, flags, kd, d_nsel, int64_t(n), s));
  TRY(cub::DeviceSelect::Flagged(tmp, tb, sv, flags, vd, d_nsel, int64_t(n), s));
  int64_t h_nsel = 0;
  TRY(cudaMemcpyAsync(&h_nsel, d_nsel, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  TRY(cudaStreamSynchronize(s));
#undef TRY
  scratch_free(sk, s); scratch_free(sv, s); scratch_free(flags, s); scratch_free(tmp, s); scratch_free(d_nsel, s);
  *out_k = kd;
  *out_v = vd;
  *nd = uint64_t(h_nsel);
  (void)rc;
  return HBT_OK;
}

template <typename K>
int build_sorted_t(hbt_tree* t, const K* kd, const K* vd, uint64_t nd, cudaStream_t s) {
  const uint32_t P = 64 / (2 * sizeof(K));
  const uint32_t F = t->F;
  t->P = P;
  t->n = nd;
  t->L0 = nd == 0 ? 1 : ceil_div_u64(nd, P);
  uint64_t c[HBT_MAX_LEVELS + 2];
  uint32_t H = 0;
  c[0] = t->L0;
  while (c[H] > 1) {
    if (H + 1 >= HBT_MAX_LEVELS) { set_error("tree too tall"); return HBT_EUNSUPPORTED; }
    c[H + 1] = ceil_div_u64(c[H], F);
    ++H;
  }
  t->H = H;
  t->offset[0] = 0;
  for (uint32_t d = 0; d < H; ++d) {
    t->nodes[d] = c[H - d];
    t->offset[d + 1] = t->offset[d] + t->nodes[d];
  }
  t->inner_bytes = t->offset[H] * F * sizeof(K);
  t->leaf_bytes = t->L0 * 64;
  HBT_CUDA_TRY(cudaMalloc(&t->d_leaf, t->leaf_bytes));
  // I-segment and its derived index share ONE allocation so that a single L2
  // access-policy window can cover both (search: "l2_persist").
  t->idx_stride = H ? implicit_idx_stride(F, sizeof(K)) : 0;
  t->inner_idx_bytes = t->offset[H] * t->idx_stride;
  const uint64_t inner_al = (t->inner_bytes + 255) & ~uint64_t(255);
  if (t->inner_bytes) HBT_CUDA_TRY(cudaMalloc(&t->d_inner, inner_al + t->inner_idx_bytes));
  t->d_inner_idx = t->inner_idx_bytes ? (uint8_t*)t->d_inner + inner_al : nullptr;
  pack_leaf_lines<K><<<grid_for(t->L0 * P), 256, 0, s>>>(kd, vd, nd, t->L0, (K*)t->d_leaf);
  HBT_CUDA_TRY(cudaGetLastError());
  if (H) {
    LevelTable lt{};
    for (uint32_t d = 0; d <= H; ++d) lt.offset[d] = t->offset[d];
    lt.H = H;
    lt.SL = 0;
    gather_separators<K><<<grid_for(t->offset[H] * F), 256, 0, s>>>(kd, nd, lt, t->L0, F, (K*)t->d_inner);
    HBT_CUDA_TRY(cudaGetLastError());
    if (t->idx_stride) {
      const uint32_t ie = t->idx_stride / sizeof(K);
      derive_inner_index<K><<<grid_for(t->offset[H] * ie), 256, 0, s>>>((const K*)t->d_inner, t->offset[H], F, ie,
                                                                         (K*)t->d_inner_idx);
      HBT_CUDA_TRY(cudaGetLastError());
    }
  }
  // level-T directory: T = the deepest level whose max-key array fits 64 KB
  {
    uint32_t T = 0;
    for (uint32_t d = 0; d <= H; ++d) {
      const uint64_t cnt = d < H ? t->nodes[d] : t->L0;
      if (cnt * sizeof(K) <= 64 * 1024 && cnt <= 65535) T = d;
    }
    const uint64_t cnt = T < H ? t->nodes[T] : t->L0;
    uint64_t span = P;  // ranks below one level-T node: P * F^(H-T)
    for (uint32_t e = T; e < H; ++e) span *= F;
    uint32_t bits = 1;
    while ((1ull << bits) < 4 * cnt && bits < 13) ++bits;
    t->dir_T = T;
    t->dir_count = uint32_t(cnt);
    t->dir_bits = bits;
    t->dir_bytes = cnt * sizeof(K) + (4ull << bits);
    HBT_CUDA_TRY(cudaMalloc(&t->d_dir, t->dir_bytes));
    K* M = (K*)t->d_dir;
    uint32_t* dir = (uint32_t*)((uint8_t*)t->d_dir + cnt * sizeof(K));
    build_dir_max<K><<<grid_for(cnt), 256, 0, s>>>((const K*)t->d_leaf, nd, cnt, span, M);
    HBT_CUDA_TRY(cudaGetLastError());
    build_dir_table<K><<<grid_for(1ull << bits), 256, 0, s>>>(M, uint32_t(cnt), bits, dir);
    HBT_CUDA_TRY(cudaGetLastError());
  }
  HBT_CUDA_TRY(cudaStreamSynchronize(s));
  return HBT_OK;
}

// Merge the batch into t's sorted pairs (read from its L-segment) and build the result
// into the EMPTY tree `nt` (form / width / F / device set by the caller); t is not
// modified.  hbt_bulk_update swaps nt into t; a versioned tree keeps t as the version
// that searches still read (versioned.cu).
template <typename K>
int implicit_merge_rebuild_t(const hbt_tree* t, const hbt_batch* b, hbt_tree* nt, cudaStream_t s) {
  const uint64_t nb = t->n, m = b->count, total = nb + m;
  if (total >= (1ull << 32)) { set_error("update: n + batch must be < 2^32"); return HBT_EUNSUPPORTED; }
  K *ck = nullptr, *sk = nullptr, *base_v = nullptr, *mv = nullptr, *kd = nullptr, *vd = nullptr;
  uint32_t *idx = nullptr, *sidx = nullptr;
  uint8_t* flags = nullptr;
  int64_t* d_nsel = nullptr;
  void* tmp = nullptr;
  size_t tb = 0, tb2 = 0;
  auto cleanup = [&]() {
    scratch_free(ck, s); scratch_free(sk, s); scratch_free(base_v, s); scratch_free(mv, s); scratch_free(kd, s);
    scratch_free(vd, s); scratch_free(idx, s); scratch_free(sidx, s); scratch_free(flags, s); scratch_free(d_nsel, s);
    scratch_free(tmp, s);
  };
#define TRY(x)                                                                          \
  do {                                                                                  \
    cudaError_t _e = (x);                                                               \
    if (_e != cudaSuccess) {                                                            \
      set_error("%s:%d %s: %s", __FILE__, __LINE__, #x, cudaGetErrorString(_e));         \
      cleanup();                                                                        \
      return _e == cudaErrorMemoryAllocation ? HBT_ENOMEM : HBT_ECUDA;                  \
    }                                                                                   \
  } while (0)
  TRY(scratch_alloc((void**)&ck, total * sizeof(K), s));
  TRY(scratch_alloc((void**)&sk, total * sizeof(K), s));
  TRY(scratch_alloc((void**)&base_v, (nb ? nb : 1) * sizeof(K), s));
  TRY(scratch_alloc((void**)&mv, total * sizeof(K), s));
  TRY(scratch_alloc((void**)&idx, total * sizeof(uint32_t), s));
  TRY(scratch_alloc((void**)&sidx, total * sizeof(uint32_t), s));
  TRY(scratch_alloc((void**)&flags, total, s));
  TRY(scratch_alloc((void**)&d_nsel, sizeof(int64_t), s));
  if (nb) {
    unpack_leaf_lines<K><<<grid_for(nb), 256, 0, s>>>((const K*)t->d_leaf, nb, ck, base_v);
    TRY(cudaGetLastError());
  }
  TRY(cudaMemcpyAsync(ck + nb, b->keys, m * sizeof(K), cudaMemcpyDeviceToDevice, s));
  iota_u32<<<grid_for(total), 256, 0, s>>>(idx, total);
  TRY(cudaGetLastError());
  TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb, ck, sk, idx, sidx, total, 0, int(8 * sizeof(K)), s));
  TRY(cub::DeviceSelect::Flagged(nullptr, tb2, sk, flags, ck, d_nsel, int64_t(total), s));
  if (tb2 > tb) tb = tb2;
  TRY(scratch_alloc((void**)&tmp, tb, s));
  TRY(cub::DeviceRadixSort::SortPairs(tmp, tb, ck, sk, idx, sidx, total, 0, int(8 * sizeof(K)), s));
  merge_flags<K><<<grid_for(total), 256, 0, s>>>(sk, sidx, total, nb, b->ops, flags);
  TRY(cudaGetLastError());
  merge_gather_values<K><<<grid_for(total), 256, 0, s>>>(sidx, total, nb, base_v, (const K*)b->values, mv);
  TRY(cudaGetLastError());
  TRY(scratch_alloc((void**)&kd, total * sizeof(K), s));
  TRY(scratch_alloc((void**)&vd, total * sizeof(K), s));
  TRY(cub::DeviceSelect::Flagged(tmp, tb, sk, flags, kd, d_nsel, int64_t(total), s));
  TRY(cub::DeviceSelect::Flagged(tmp, tb, mv, flags, vd, d_nsel, int64_t(total), s));
  int64_t h_nsel = 0;
  TRY(cudaMemcpyAsync(&h_nsel, d_nsel, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  TRY(cudaStreamSynchronize(s));
#undef TRY
  // Rebuild into a fresh layout.
  int rc = build_sorted_t<K>(nt, kd, vd, uint64_t(h_nsel), s);
  cleanup();
  if (rc != HBT_OK) {
    cudaFree(nt->d_leaf); cudaFree(nt->d_inner); cudaFree(nt->d_dir);
    nt->d_leaf = nt->d_inner = nt->d_inner_idx = nt->d_dir = nullptr;
  }
  return rc;
}

template <typename K>
int implicit_update_t(hbt_tree* t, const hbt_batch* b, cudaStream_t s) {
  hbt_tree nt;
  nt.form = t->form; nt.width = t->width; nt.F = t->F; nt.device = t->device; nt.num_sms = t->num_sms;
  int rc = implicit_merge_rebuild_t<K>(t, b, &nt, s);
  if (rc != HBT_OK) return rc;
  const uint32_t where = t->leaf_where;
  leaf_free(t);
  cudaFree(t->d_inner);  // also holds the derived index
  cudaFree(t->d_dir);
  t->n = nt.n; t->L0 = nt.L0; t->H = nt.H; t->P = nt.P;
  for (int d = 0; d < HBT_MAX_LEVELS; ++d) t->nodes[d] = nt.nodes[d];
  for (int d = 0; d <= HBT_MAX_LEVELS; ++d) t->offset[d] = nt.offset[d];
  t->d_leaf = nt.d_leaf; t->leaf_bytes = nt.leaf_bytes;
  t->d_inner = nt.d_inner; t->inner_bytes = nt.inner_bytes;
  t->d_inner_idx = nt.d_inner_idx; t->inner_idx_bytes = nt.inner_idx_bytes; t->idx_stride = nt.idx_stride;
  t->d_dir = nt.d_dir; t->dir_bytes = nt.dir_bytes; t->dir_T = nt.dir_T; t->dir_count = nt.dir_count;
  t->dir_bits = nt.dir_bits;
  nt.d_leaf = nt.d_inner = nt.d_inner_idx = nt.d_dir = nullptr;
  // the rebuilt L-segment goes back where the caller placed the old one
  return where ? leaf_place(t, where) : HBT_OK;
}

}  // namespace

int sort_dedupe(uint32_t width, const void* keys, const void* values, uint64_t n, void** out_k, void** out_v,
                uint64_t* nd, cudaStream_t s) {
  return width == 4 ? sort_dedupe_t<uint32_t>(keys, values, n, out_k, out_v, nd, s)
                    : sort_dedupe_t<uint64_t>(keys, values, n, out_k, out_v, nd, s);
}

int implicit_build_sorted(hbt_tree* t, const void* kd, const void* vd, uint64_t nd, cudaStream_t s) {
  return t->width == 4 ? build_sorted_t<uint32_t>(t, (const uint32_t*)kd, (const uint32_t*)vd, nd, s)
                       : build_sorted_t<uint64_t>(t, (const uint64_t*)kd, (const uint64_t*)vd, nd, s);
}

int implicit_build(hbt_tree* t, const void* keys, const void* values, uint64_t n, cudaStream_t s) {
  // Presorted distinct input (e.g. c4's stratified keys): build straight from it
  // (no sort workspace: 2^31 u64 pairs would otherwise need ~100 GB of temporaries).
  bool sorted = false;
  int rc = n ? (t->width == 4 ? is_sorted_distinct<uint32_t>(keys, n, &sorted, s)
                              : is_sorted_distinct<uint64_t>(keys, n, &sorted, s))
             : HBT_OK;
  if (rc != HBT_OK) return rc;
  if (sorted) return implicit_build_sorted(t, keys, values, n, s);
  void *kd = nullptr, *vd = nullptr;
  uint64_t nd = 0;
  rc = sort_dedupe(t->width, keys, values, n, &kd, &vd, &nd, s);
  if (rc != HBT_OK) return rc;
  rc = implicit_build_sorted(t, kd, vd, nd, s);
  scratch_free(kd, s);
  scratch_free(vd, s);
  cudaStreamSynchronize(s);
  return rc;
}

int implicit_update(hbt_tree* t, const hbt_batch* b, cudaStream_t s) {
  return t->width == 4 ? implicit_update_t<uint32_t>(t, b, s) : implicit_update_t<uint64_t>(t, b, s);
}

int implicit_merge_rebuild(const hbt_tree* t, const hbt_batch* b, hbt_tree* nt, cudaStream_t s) {
  return t->width == 4 ? implicit_merge_rebuild_t<uint32_t>(t, b, nt, s) : implicit_merge_rebuild_t<uint64_t>(t, b, nt, s);
}

}  // namespace hbt
