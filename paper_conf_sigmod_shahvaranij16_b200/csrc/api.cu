// api.cu — the C ABI of libhbt.so (include/hbt.h): argument validation,
// handle ownership, dispatch to the implicit / regular paths, the chunked
// host-buffer pipeline and error reporting.  Every compute step runs in this
// library's CUDA kernels (or CUB device primitives for the build's sort); there
// is no CPU fallback.
#include <stdarg.h>
#include <stdio.h>

#include <algorithm>
#include <string>

#include "hbt_internal.cuh"

namespace hbt {

static thread_local std::string g_err;

void set_error(const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
}

cudaError_t scratch_alloc(void** p, size_t bytes, cudaStream_t s) {
  static thread_local int configured = -1;
  int dev = 0;
  cudaGetDevice(&dev);
  if (configured != dev) {
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
      // keep up to a quarter of the device between calls: a bucketed search of
      // 2^28 queries needs 7.5 GB of scratch, and returning it to the driver
      // after every call costs ~100 ms (c4, measured)
      size_t free_b = 0, total_b = 0;
      cudaMemGetInfo(&free_b, &total_b);
      uint64_t keep = std::max<uint64_t>(4ull << 30, uint64_t(total_b) / 4);
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
    }
    configured = dev;
  }
  *p = nullptr;
  return cudaMallocAsync(p, bytes ? bytes : 1, s);
}

void scratch_free(void* p, cudaStream_t s) {
  if (p) cudaFreeAsync(p, s);
}

static bool is_device_ptr_uncached(const void* p) {
  if (!p) return false;
  cudaPointerAttributes a;
  cudaError_t e = cudaPointerGetAttributes(&a, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// The search entry points validate three pointers per call; cudaPointerGetAttributes
// costs ~1 us each, which dominates small batches (c1: 2^16 queries in ~5 us of
// device time).  A pointer that validated once stays in a small per-thread cache:
// device virtual addresses are never handed out to pageable host memory, so a stale
// entry can at worst admit a pinned/managed buffer, which the device can read.
static bool is_device_ptr(const void* p) {
  constexpr int kN = 8;
  thread_local const void* cache[kN] = {};
  thread_local int next = 0;
  if (!p) return false;
  for (int i = 0; i < kN; ++i)
    if (cache[i] == p) return true;
  if (!is_device_ptr_uncached(p)) return false;
  cache[next] = p;
  next = (next + 1) % kN;
  return true;
}

void leaf_free(hbt_tree* t) {
  if (t->h_leaf) cudaFreeHost(t->h_leaf);
  else cudaFree(t->d_leaf);
  t->h_leaf = nullptr;
  t->d_leaf = nullptr;
}

// Move one pool between HBM and pinned, mapped host memory: *d is the device-visible
// pointer (the host allocation's device alias when on the host), *h the host
// allocation or NULL.
static int move_pool(void** d, void** h, uint64_t bytes, uint32_t where) {
  if (where == 1) {
    void* hh = nullptr;
    void* dd = nullptr;
    if (cudaHostAlloc(&hh, bytes ? bytes : 64, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) {
      cudaGetLastError();
      set_error("cudaHostAlloc of %llu bytes for the L-segment failed", (unsigned long long)bytes);
      return HBT_ENOMEM;
    }
    if (bytes) {
      cudaError_t e = cudaMemcpy(hh, *d, bytes, cudaMemcpyDefault);
      if (e != cudaSuccess) { cudaFreeHost(hh); set_error("L-segment copy: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
    }
    cudaError_t e = cudaHostGetDevicePointer(&dd, hh, 0);
    if (e != cudaSuccess) { cudaFreeHost(hh); set_error("no device alias of the host L-segment: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
    cudaFree(*d);
    *h = hh;
    *d = dd;
  } else {
    void* dd = nullptr;
    HBT_CUDA_TRY(cudaMalloc(&dd, bytes ? bytes : 64));
    if (bytes) {
      cudaError_t e = cudaMemcpy(dd, *h, bytes, cudaMemcpyDefault);
      if (e != cudaSuccess) { cudaFree(dd); set_error("L-segment copy: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
    }
    cudaFreeHost(*h);
    *h = nullptr;
    *d = dd;
  }
  return HBT_OK;
}

// Move the L-segment (implicit: the leaf lines; regular: the big-leaf pool) between
// HBM and pinned, mapped host memory.  The kernels read (and the regular update
// kernels write) leaf lines through the device-visible pointer either way — zero-copy
// accesses over the host link when it lives on the host — so results are identical.
int leaf_place(hbt_tree* t, uint32_t where) {
  if (t->form == HBT_REGULAR) {
    RegularState& r = t->r;
    if ((where == 1) == (r.h_leaf != nullptr)) { t->leaf_where = where; return HBT_OK; }
    const int rc = move_pool(&r.d_leaf, &r.h_leaf, r.cap * uint64_t(t->F) * 64, where);
    if (rc == HBT_OK) t->leaf_where = where;
    return rc;
  }
  const bool on_host = t->h_leaf != nullptr;
  if ((where == 1) == on_host) { t->leaf_where = where; return HBT_OK; }
  const uint64_t bytes = t->leaf_bytes ? t->leaf_bytes : 64;
  if (where == 1) {
    void* h = nullptr;
    void* d = nullptr;
    if (cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) {
      cudaGetLastError();
      set_error("cudaHostAlloc of %llu bytes for the L-segment failed", (unsigned long long)bytes);
      return HBT_ENOMEM;
    }
    if (t->leaf_bytes) {
      cudaError_t e = cudaMemcpy(h, t->d_leaf, t->leaf_bytes, cudaMemcpyDefault);
      if (e != cudaSuccess) { cudaFreeHost(h); set_error("L-segment copy: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
    }
    cudaError_t e = cudaHostGetDevicePointer(&d, h, 0);
    if (e != cudaSuccess) { cudaFreeHost(h); set_error("no device alias of the host L-segment: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
    cudaFree(t->d_leaf);
    t->h_leaf = h;
    t->d_leaf = d;
  } else {
    void* d = nullptr;
    HBT_CUDA_TRY(cudaMalloc(&d, bytes));
    if (t->leaf_bytes) {
      cudaError_t e = cudaMemcpy(d, t->h_leaf, t->leaf_bytes, cudaMemcpyDefault);
      if (e != cudaSuccess) { cudaFree(d); set_error("L-segment copy: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
    }
    cudaFreeHost(t->h_leaf);
    t->h_leaf = nullptr;
    t->d_leaf = d;
  }
  t->leaf_where = where;
  return HBT_OK;
}

void free_tree(hbt_tree* t) {
  if (!t) return;
  cudaFree(t->d_inner);  // also holds d_inner_idx
  cudaFree(t->d_dir);
  leaf_free(t);
  regular_free(t);
  shard_free(t);
  fused_free(t);
  range_free(t);
  bucket_free(t);
  cudaFree(t->pipe.d_q);
  cudaFree(t->pipe.d_pf);
  cudaFree(t->pipe.d_v);
  for (int i = 0; i < kHostBufs; ++i) {
    if (t->pipe.s[i]) cudaStreamDestroy(t->pipe.s[i]);
    if (t->pipe.ev[i]) cudaEventDestroy(t->pipe.ev[i]);
  }
  delete t;
}

// Mark the bucket states stale (re-derived by the next bucketed search, bucketed.cu).
void invalidate_buckets(hbt_tree* t) {
  std::lock_guard<std::mutex> lock(t->bk_mu);
  t->bk.valid = false;
  t->bks.valid = false;
}

int device_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s) {
  if (t->h_leaf && leaf_stream_enabled(t, m)) return streamed_search(t, q, m, pf, v, 0, s);
  if (bucketed_enabled(t, m)) return bucketed_search(t, q, m, pf, v, 0, s);
  return t->form == HBT_REGULAR ? regular_search(t, q, m, pf, v, s) : implicit_search(t, q, m, pf, v, s);
}

}  // namespace hbt

using namespace hbt;

extern "C" {

const char* hbt_last_error(void) { return g_err.c_str(); }

const char* hbt_version(void) { return "hbt 0.1 (HB+-tree lookups, sm_100a)"; }

int hbt_bulk_build(const void* keys, const void* values, uint64_t n, uint32_t fanout, uint32_t layout,
                   void* stream, hbt_tree** out) {
  NvtxRange nvtx_("hbt_bulk_build");
  g_err.clear();
  if (!out) { set_error("out is NULL"); return HBT_EINVAL; }
  *out = nullptr;
  const uint32_t form = layout & 0x1;
  const uint32_t wbits = layout & 0xF0;
  if ((layout & ~0x11u) != 0 || (wbits != HBT_KEY32 && wbits != HBT_KEY64)) {
    set_error("bad layout word 0x%x", layout);
    return HBT_EINVAL;
  }
  if (fanout != 4 && fanout != 8 && fanout != 16 && fanout != 32) {
    set_error("fanout must be 4, 8, 16 or 32 (got %u)", fanout);
    return HBT_EINVAL;
  }
  if (n >= (1ull << 32)) { set_error("n must be < 2^32"); return HBT_EUNSUPPORTED; }
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) { set_error("no CUDA device: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
  if (n > 0 && (!is_device_ptr(keys) || !is_device_ptr(values))) {
    set_error("keys/values must be device pointers");
    return HBT_EINVAL;
  }
  hbt_tree* t = new hbt_tree();
  t->form = form;
  t->width = wbits == HBT_KEY64 ? 8 : 4;
  t->F = fanout;
  t->P = 64 / (2 * t->width);
  t->device = dev;
  cudaDeviceGetAttribute(&t->num_sms, cudaDevAttrMultiProcessorCount, dev);
  cudaStream_t s = (cudaStream_t)stream;
  int rc = form == HBT_REGULAR ? regular_build(t, keys, values, n, s) : implicit_build(t, keys, values, n, s);
  if (rc != HBT_OK) {
    free_tree(t);
    return rc;
  }
  *out = t;
  return HBT_OK;
}

int hbt_search(const hbt_tree* t, const void* queries, uint64_t m, hbt_out out, void* stream) {
  NvtxRange nvtx_("hbt_search");
  if (!t) { set_error("tree is NULL"); return HBT_EINVAL; }
  if (m == 0) return HBT_OK;
  if (!is_device_ptr(queries) || !is_device_ptr(out.pos_found) || !is_device_ptr(out.values)) {
    set_error("queries/out must be device pointers");
    return HBT_EINVAL;
  }
  return device_search(t, queries, m, out.pos_found, out.values, (cudaStream_t)stream);
}

int hbt_search_host(const hbt_tree* t, const void* host_queries, uint64_t m, uint64_t* host_pos_found,
                    void* host_values, void* stream) {
  NvtxRange nvtx_("hbt_search_host");
  if (!t) { set_error("tree is NULL"); return HBT_EINVAL; }
  if (m == 0) return HBT_OK;
  if (!host_queries || !host_pos_found || !host_values) { set_error("NULL host buffer"); return HBT_EINVAL; }
  HostPipe& p = t->pipe;
  std::lock_guard<std::mutex> lock(p.mu);
  const uint64_t S = t->width;
  const uint64_t chunk = uint64_t(1) << t->cfg.host_chunk_log2;  // queries per bucket (default 4 Mi)
  const int nbuf = int(t->cfg.host_bufs);
  if (p.chunk != chunk || p.nbuf != nbuf) {
    for (int i = 0; i < p.nbuf && p.chunk; ++i) HBT_CUDA_TRY(cudaStreamSynchronize(p.s[i]));
    cudaFree(p.d_q);
    cudaFree(p.d_pf);
    cudaFree(p.d_v);
    p.d_q = p.d_v = nullptr;
    p.d_pf = nullptr;
    p.chunk = 0;
    HBT_CUDA_TRY(cudaMalloc(&p.d_q, nbuf * chunk * S));
    HBT_CUDA_TRY(cudaMalloc(&p.d_pf, nbuf * chunk * sizeof(uint64_t)));
    HBT_CUDA_TRY(cudaMalloc(&p.d_v, nbuf * chunk * S));
    for (int i = 0; i < kHostBufs; ++i) {
      if (p.s[i]) continue;
      HBT_CUDA_TRY(cudaStreamCreateWithFlags(&p.s[i], cudaStreamNonBlocking));
      HBT_CUDA_TRY(cudaEventCreateWithFlags(&p.ev[i], cudaEventDisableTiming));
    }
    p.chunk = chunk;
    p.nbuf = nbuf;
  }
  // Order after the caller's stream.
  cudaStream_t cs = (cudaStream_t)stream;
  HBT_CUDA_TRY(cudaEventRecord(p.ev[0], cs));
  for (int i = 0; i < nbuf; ++i) HBT_CUDA_TRY(cudaStreamWaitEvent(p.s[i], p.ev[0], 0));
  // Buckets rotate over nbuf (stream, buffer) pairs: bucket c+1's H2D copy overlaps
  // bucket c's search and bucket c-1's D2H copy.
  const char* hq = (const char*)host_queries;
  char* hv = (char*)host_values;
  uint64_t c = 0;
  for (uint64_t off = 0; off < m; off += chunk, ++c) {
    const uint64_t len = (m - off < chunk) ? (m - off) : chunk;
    const int b = int(c % uint64_t(nbuf));
    cudaStream_t s = p.s[b];
    char* dq = (char*)p.d_q + b * chunk * S;
    uint64_t* dpf = p.d_pf + b * chunk;
    char* dv = (char*)p.d_v + b * chunk * S;
    HBT_CUDA_TRY(cudaMemcpyAsync(dq, hq + off * S, len * S, cudaMemcpyHostToDevice, s));
    int rc = device_search(t, dq, len, dpf, dv, s);
    if (rc != HBT_OK) return rc;
    HBT_CUDA_TRY(cudaMemcpyAsync(host_pos_found + off, dpf, len * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    HBT_CUDA_TRY(cudaMemcpyAsync(hv + off * S, dv, len * S, cudaMemcpyDeviceToHost, s));
  }
  for (int i = 0; i < nbuf; ++i) HBT_CUDA_TRY(cudaStreamSynchronize(p.s[i]));
  return HBT_OK;
}

int hbt_range(const hbt_tree* t, const void* lo, const void* hi, uint64_t m, uint32_t k, void* out_keys,
              void* out_values, uint32_t* out_count, void* stream) {
  NvtxRange nvtx_("hbt_range");
  if (!t) { set_error("tree is NULL"); return HBT_EINVAL; }
  if (m == 0) return HBT_OK;
  if (k == 0 || k > 4096) { set_error("k must be in [1, 4096]"); return HBT_EINVAL; }
  if (!is_device_ptr(lo) || !is_device_ptr(hi) || !is_device_ptr(out_keys) || !is_device_ptr(out_values) ||
      !is_device_ptr(out_count)) {
    set_error("range arrays must be device pointers");
    return HBT_EINVAL;
  }
  return range_scan(t, lo, hi, m, k, out_keys, out_values, out_count, (cudaStream_t)stream);
}

int hbt_bulk_update(hbt_tree* t, const hbt_batch* batch, void* stream) {
  NvtxRange nvtx_("hbt_bulk_update");
  if (!t || !batch) { set_error("tree/batch is NULL"); return HBT_EINVAL; }
  if (batch->count == 0) return HBT_OK;
  if (!is_device_ptr(batch->keys) || !is_device_ptr(batch->values) || !is_device_ptr(batch->ops)) {
    set_error("batch arrays must be device pointers");
    return HBT_EINVAL;
  }
  if (t->shard.G >= 1) {
    // a shard's (n', base, max) are part of every rank's routing table: a local update
    // would leave the other ranks routing by stale maxima and bases
    set_error("bulk update of a key-range shard is not supported (rebuild the sharded tree)");
    return HBT_EUNSUPPORTED;
  }
  cudaStream_t s = (cudaStream_t)stream;
  invalidate_buckets(t);  // bucket splitters follow the tree
  return t->form == HBT_REGULAR ? regular_update(t, batch, s) : implicit_update(t, batch, s);
}

int hbt_destroy(hbt_tree* t) {
  if (!t) return HBT_EINVAL;
  cudaDeviceSynchronize();
  free_tree(t);
  return HBT_OK;
}

int hbt_info(const hbt_tree* t, hbt_info_t* info) {
  if (!t || !info) { set_error("NULL argument"); return HBT_EINVAL; }
  *info = hbt_info_t{};
  info->layout = t->form;
  info->width = t->width;
  info->fanout = t->F;
  info->pairs_per_line = t->P;
  info->n_distinct = t->n;
  if (t->form == HBT_IMPLICIT) {
    info->height = t->H;
    info->smem_levels = t->dir_T;
    for (uint32_t d = 0; d < t->H; ++d) info->level_nodes[d] = t->nodes[d];
    info->leaf_lines = t->L0;
    info->chain_len = t->L0;
    info->inner_bytes = t->inner_bytes + t->inner_idx_bytes;
    info->leaf_bytes = t->leaf_bytes;
  } else {
    const RegularState& r = t->r;
    info->height = r.U + 1;
    info->smem_levels = r.dir_T;
    for (uint32_t u = 0; u < r.U; ++u) info->level_nodes[u] = r.unodes[u];
    info->leaf_lines = r.pool;
    info->chain_len = r.nchain;
    const uint64_t nip = 32 / t->width;
    info->inner_bytes = r.uoff[r.U] * (uint64_t(t->F) * (t->width + 4) + 32) + r.pool * (uint64_t(t->F) * t->width + nip * t->width);
    info->leaf_bytes = r.pool * uint64_t(t->F) * 64;
  }
  return HBT_OK;
}

int hbt_export(const hbt_tree* t, uint32_t segment, void* dst, uint64_t bytes, uint64_t* written) {
  if (!t || !dst) { set_error("NULL argument"); return HBT_EINVAL; }
  const void* src = nullptr;
  uint64_t len = 0;
  const uint64_t S = t->width, F = t->F;
  const RegularState& r = t->r;
  const uint64_t nip = 32 / S;  // index entries padded to one 32 B sector
  if (t->form == HBT_IMPLICIT) {
    if (segment == HBT_SEG_INNER) { src = t->d_inner; len = t->inner_bytes; }
    else if (segment == HBT_SEG_LEAF) { src = t->d_leaf; len = t->leaf_bytes; }
    else if (segment == HBT_SEG_INNER_IDX) { src = t->d_inner_idx; len = t->inner_idx_bytes; }
    else { set_error("segment %u not in an implicit tree", segment); return HBT_EINVAL; }
  } else {
    switch (segment) {
      case HBT_SEG_LEAF: src = r.d_leaf; len = r.pool * F * 64; break;
      case HBT_SEG_COUNT: src = r.d_count; len = r.pool * 4; break;
      case HBT_SEG_LAST_KEYS: src = r.d_lkeys; len = r.pool * F * S; break;
      case HBT_SEG_LAST_IDX: src = r.d_lidx; len = r.pool * nip * S; break;
      case HBT_SEG_UPPER_KEYS: src = r.d_ukeys; len = r.uoff[r.U] * F * S; break;
      case HBT_SEG_UPPER_IDX: src = r.d_uidx; len = r.uoff[r.U] * nip * S; break;
      case HBT_SEG_UPPER_REFS: src = r.d_urefs; len = r.uoff[r.U] * F * 4; break;
      case HBT_SEG_CHAIN: src = r.d_chain; len = r.nchain * 4; break;
      default: set_error("segment %u not in a regular tree", segment); return HBT_EINVAL;
    }
  }
  if (written) *written = len;
  if (bytes < len) { set_error("destination too small: need %llu bytes", (unsigned long long)len); return HBT_EINVAL; }
  if (len) HBT_CUDA_TRY(cudaMemcpy(dst, src, len, cudaMemcpyDefault));  // src may be the mapped host L-segment
  return HBT_OK;
}

int hbt_set_leaf_placement(hbt_tree* t, uint32_t where) {
  g_err.clear();
  if (!t) { set_error("tree is NULL"); return HBT_EINVAL; }
  if (where > 1) { set_error("placement must be 0 (HBM) or 1 (host)"); return HBT_EINVAL; }
  if (t->shard.G > 1) { set_error("leaf placement: not for sharded trees"); return HBT_EUNSUPPORTED; }
  HBT_CUDA_TRY(cudaDeviceSynchronize());  // no search may be reading the old copy
  return leaf_place(t, where);
}

int hbt_get_leaf_placement(const hbt_tree* t, uint32_t* where) {
  if (!t || !where) { set_error("NULL argument"); return HBT_EINVAL; }
  *where = (t->form == HBT_REGULAR ? t->r.h_leaf : t->h_leaf) ? 1u : 0u;
  return HBT_OK;
}

int hbt_last_phases(const hbt_tree* t, hbt_phase_times* out) {
  if (!t || !out) { set_error("NULL argument"); return HBT_EINVAL; }
  const BucketState& bs = t->bk;
  if (!bs.timed) { set_error("no timed bucketed search on this tree"); return HBT_EINVAL; }
  *out = hbt_phase_times{};
  HBT_CUDA_TRY(cudaEventSynchronize(bs.ev[5]));
  out->phases = 5;
  out->launches = bs.launches;
  for (int i = 0; i < 5; ++i) HBT_CUDA_TRY(cudaEventElapsedTime(&out->ms[i], bs.ev[i], bs.ev[i + 1]));
  return HBT_OK;
}

int hbt_set_param(hbt_tree* t, const char* name, int64_t value) {
  if (!t || !name) { set_error("NULL argument"); return HBT_EINVAL; }
  const std::string n(name);
  SearchConfig& c = t->cfg;
  if (n == "ctas_per_sm" && value >= 0 && value <= 32) c.ctas_per_sm = uint32_t(value);
  else if (n == "smem_mode" && (value == 2 || value == 3)) c.mode = uint32_t(value);
  else if (n == "small_batch" && value >= 0) c.small_batch = uint64_t(value);
  else if (n == "l2_levels_bytes" && value >= 0) c.l2_levels_bytes = uint64_t(value);
  else if (n == "full_levels" && value >= 0 && value <= 0xFFFFFFFFll) c.full_levels = uint32_t(value);
  else if (n == "exchange" && (value == 0 || value == 1)) c.exchange = uint32_t(value);
  else if (n == "exchange_chunks" && value >= 1 && value <= 4) c.exchange_chunks = uint32_t(value);
  else if (n == "g1_direct" && (value == 0 || value == 1)) c.g1_direct = uint32_t(value);
  else if (n == "bucket" && value >= 0 && value <= 2) c.bucket = uint32_t(value);
  else if (n == "bucket_slice" && value >= 0) { c.bucket_slice = uint64_t(value); invalidate_buckets(t); }
  else if (n == "bucket_items" && (value == 0 || value == 1)) { c.bucket_items = uint32_t(value); invalidate_buckets(t); }
  else if (n == "bucket_cap" && value >= 0 && value < (1 << 20)) { c.bucket_cap = uint32_t(value); invalidate_buckets(t); }
  else if (n == "item_rounds" && value >= 0 && value <= 64) c.item_rounds = uint32_t(value);
  else if (n == "scatter_tma" && (value == 0 || value == 1)) c.scatter_tma = uint32_t(value);
  else if (n == "phase_timing" && (value == 0 || value == 1)) c.phase_timing = uint32_t(value);
  else if (n == "leaf_stream" && value >= 0 && value <= 2) c.leaf_stream = uint32_t(value);
  else if (n == "stream_slice" && value >= 0) { c.stream_slice = uint64_t(value); invalidate_buckets(t); }
  else if (n == "host_chunk_log2" && value >= 12 && value <= 26) c.host_chunk_log2 = uint32_t(value);
  else if (n == "host_bufs" && value >= 2 && value <= kHostBufs) c.host_bufs = uint32_t(value);
  else if (n == "leaf256" && (value == 0 || value == 1)) c.leaf256 = uint32_t(value);
  else if (n == "full256" && (value == 0 || value == 1)) c.full256 = uint32_t(value);
  else if (n == "l2_hint" && value >= 0 && value <= 4) c.l2_hint = uint32_t(value);
  else if (n == "item_l2_hint" && value >= 0 && value <= 3) c.item_l2_hint = uint32_t(value);
  else if (n == "item_qpf" && value >= 0 && value <= 6) c.item_qpf = uint32_t(value);
  else if (n == "item_cnode" && value >= 0 && value <= 2) { c.item_cnode = uint32_t(value); invalidate_buckets(t); }
  else if (n == "item_cdir" && value >= 0 && value <= 2) { c.item_cdir = uint32_t(value); invalidate_buckets(t); }
  else {
    set_error("bad parameter %s = %lld", name, (long long)value);
    return HBT_EINVAL;
  }
  return HBT_OK;
}

}  // extern "C"
