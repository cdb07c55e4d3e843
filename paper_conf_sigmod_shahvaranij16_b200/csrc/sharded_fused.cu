// sharded_fused.cu — the key-range-sharded search with a FUSED exchange over
// peer memory (NVLink 5 / NVSwitch): no NCCL and no host collective on the data path.
//
// Every rank owns one window (one cudaMalloc, exported with CUDA IPC and
// mapped by every peer):
//   [flags: 64 x u32 | matrix: 2 x 64 x 64 u64 (parity of the batch) | res_pf: cap_m u64
//    | res_v: cap_m x S | recv_q: cap_r x S | recv_org: cap_r u64]
// Per batch b (all kernels stream-ordered; barriers are device-side flag exchanges
// over peer memory):
//   1. f_count (the owner rule of sharded.cu) counts queries per destination, and
//      f_publish stores this rank's count row into EVERY peer's matrix[b & 1]
//                                                                 -> barrier
//   2. the host reads its own matrix[b & 1] (the full G x G count matrix, one small
//      D2H) to size the owner search; every rank sees the same matrix, so a window
//      regrowth is decided identically everywhere (a collective re-export)
//   3. f_put: every query is stored straight into its owner's receive window at
//      (earlier sources' counts) + a CTA-reserved slot, with its origin (rank, index)
//                                                                 -> barrier
//   4. the owner searches its receive window (pos_base = its first global rank); the
//      bucketed search's final gather stores each result straight into the
//      REQUESTER's result window, the owner's run of that requester's queries as one
//      contiguous run (coalesced peer stores; bucketed.cu, RemoteOut); small batches
//      search into scratch and f_return stores them the same way  -> barrier
//   5. the requester moves its result window (one run per owner) into query order
//      through rpos[i], the result slot f_put recorded for query i (f_collect).
// The matrix is double-buffered by batch parity, so step 1 of batch b+1 (stores into
// the peers' other matrix) cannot disturb a peer still reading batch b's.  The same
// kernels run for G virtual shards on one GPU (peer table = local windows, barriers =
// stream order), which is how they are tested on one device.
#include <nccl.h>

#include <vector>

#include "hbt_internal.cuh"

namespace hbt {
namespace {

constexpr int kMaxG = 64;
constexpr int kThreads = 256;
constexpr uint64_t kOrgShift = kRemoteOrgShift;  // recv_org = (source rank << 40) | origin index
constexpr uint64_t kMat = uint64_t(kMaxG) * kMaxG;  // one count matrix [src][dst]
constexpr int kMaxChunks = 4;                       // exchange chunks per batch (overlap, see below)
constexpr uint64_t kMatAll = 2 * kMaxChunks * kMat; // [parity][chunk] matrices per window

struct Win {
  uint32_t* flags;
  unsigned long long* matrix;  // [parity][chunk][src][dst]
  uint64_t* res_pf;
  uint8_t* res_v;
  uint8_t* recv_q;
  uint64_t* recv_org;
};

struct PeerTable {
  Win w[kMaxG];
  int G;
};

struct RouteTab {
  uint64_t max[kMaxG];
  uint32_t id[kMaxG];
  uint32_t n;
};

inline unsigned grid_for(uint64_t n) {
  uint64_t g = (n + kThreads - 1) / kThreads;
  if (g > 148 * 16) g = 148 * 16;
  return unsigned(g ? g : 1);
}

uint64_t win_bytes(uint64_t cap_m, uint64_t cap_r, uint32_t S) {
  auto al = [](uint64_t x) { return (x + 255) & ~uint64_t(255); };
  return al(kMaxG * 4) + al(kMatAll * 8) + al(cap_m * 8) + al(cap_m * S) + al(cap_r * S) + al(cap_r * 8);
}

Win carve(uint8_t* base, uint64_t cap_m, uint64_t cap_r, uint32_t S) {
  auto al = [](uint64_t x) { return (x + 255) & ~uint64_t(255); };
  Win w;
  uint64_t o = 0;
  w.flags = (uint32_t*)(base + o); o += al(kMaxG * 4);
  w.matrix = (unsigned long long*)(base + o); o += al(kMatAll * 8);
  w.res_pf = (uint64_t*)(base + o); o += al(cap_m * 8);
  w.res_v = base + o; o += al(cap_m * S);
  w.recv_q = base + o; o += al(cap_r * S);
  w.recv_org = (uint64_t*)(base + o);
  return w;
}

template <typename K>
__device__ __forceinline__ uint32_t owner(K q, const RouteTab& rt) {
  if (rt.n == 0) return 0;
  uint32_t c = 0;
  for (uint32_t i = 0; i < rt.n; ++i) c += (K(rt.max[i]) < q) ? 1u : 0u;
  return rt.id[c < rt.n ? c : rt.n - 1];
}

template <typename K>
__global__ void __launch_bounds__(kThreads) f_count(const K* __restrict__ q, uint64_t m, const RouteTab rt, int G,
                                                    uint8_t* __restrict__ dest, unsigned long long* __restrict__ cnt) {
  __shared__ unsigned int h[kMaxG];
  for (int i = threadIdx.x; i < G; i += blockDim.x) h[i] = 0;
  __syncthreads();
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < m; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t o = owner(q[i], rt);
    dest[i] = uint8_t(o);
    atomicAdd(&h[o], 1u);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < G; i += blockDim.x)
    if (h[i]) atomicAdd(cnt + i, (unsigned long long)h[i]);
}

// Store this rank's count rows (one per chunk) into every peer's matrix[parity][chunk]
// (row `me`).  cnt: chunk c's counts at cnt[c * 2 * kMaxG].
__global__ void f_publish(const PeerTable pt, int me, const unsigned long long* __restrict__ cnt, int parity,
                          int nchunks) {
  const int G = pt.G;
  for (int x = threadIdx.x; x < nchunks * G * G; x += blockDim.x) {
    const int ch = x / (G * G), d = (x / G) % G, c = x % G;
    pt.w[d].matrix[(uint64_t(parity) * kMaxChunks + ch) * kMat + me * kMaxG + c] = cnt[ch * 2 * kMaxG + c];
  }
}

// Where one chunk's put lands: rbase[d] = the chunk's region in owner d's receive window
// (earlier chunks' receives), qbase = the chunk's first query (result slots follow the
// batch's chunks in order).
struct PutOff {
  uint64_t rbase[kMaxG];
  uint64_t qbase;
};

// Route + put: queries go straight into their owner's receive window.  Each CTA
// reserves one block per destination for its chunk of the batch and fills it in SOURCE
// ORDER (warp match + a per-destination prefix over the CTA's warps), so a run of the
// owner's window holds one source chunk's queries in index order and the results the
// owner stores back into the requester's window land on nearly consecutive indices.
// rpos[i] = where query i's result will land in this rank's result window: the owner
// stores its run of our queries back as one run starting at (our earlier destinations'
// counts), in the order of its receive slots.
template <typename K>
__global__ void __launch_bounds__(kThreads) f_put(const K* __restrict__ q, uint64_t m, const uint8_t* __restrict__ dest,
                                                  const PeerTable pt, int me,
                                                  const unsigned long long* __restrict__ M, const PutOff off,
                                                  unsigned long long* __restrict__ cursor, uint64_t chunk,
                                                  uint32_t* __restrict__ rpos) {
  constexpr int W = kThreads / 32;
  __shared__ unsigned int h[kMaxG];
  __shared__ unsigned long long base[kMaxG];
  __shared__ unsigned long long roff[kMaxG];  // base[d] - (start of our share of d) + (our row prefix)
  __shared__ unsigned int wc[W][kMaxG];
  const int G = pt.G;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint64_t lo = blockIdx.x * chunk;
  const uint64_t hi = lo + chunk < m ? lo + chunk : m;
  for (int i = threadIdx.x; i < G; i += blockDim.x) h[i] = 0;
  __syncthreads();
  for (uint64_t i = lo + threadIdx.x; i < hi; i += blockDim.x) atomicAdd(&h[dest[i]], 1u);
  __syncthreads();
  // M = this chunk's full matrix in our own window (every row published)
  for (int d = threadIdx.x; d < G; d += blockDim.x) {
    unsigned long long start = off.rbase[d];  // earlier chunks, then earlier sources, at destination d
    for (int s = 0; s < me; ++s) start += M[s * kMaxG + d];
    unsigned long long row = 0;    // our queries to earlier destinations
    for (int x = 0; x < d; ++x) row += M[me * kMaxG + x];
    const unsigned long long o = h[d] ? atomicAdd(cursor + d, (unsigned long long)h[d]) : 0ull;
    base[d] = start + o;
    roff[d] = off.qbase + row + o;
    h[d] = 0;  // from here on: queries of this chunk already placed, per destination
  }
  for (uint64_t r0 = lo; r0 < hi; r0 += blockDim.x) {
    __syncwarp();  // every lane of this warp has read its row of the previous round
    for (int d = lane; d < G; d += 32) wc[w][d] = 0;
    __syncthreads();  // base / h ready (first round), previous round's slots read
    const uint64_t i = r0 + threadIdx.x;
    const bool v = i < hi;
    const uint32_t d = v ? dest[i] : 0xFFu;
    const unsigned peers = __match_any_sync(0xffffffffu, d);
    const unsigned before = peers & ((1u << lane) - 1u);
    if (v && before == 0) wc[w][d] = __popc(peers);
    __syncthreads();
    if (threadIdx.x < G) {  // exclusive prefix over the warps, continuing the chunk's count
      unsigned run = h[threadIdx.x];
      for (int x = 0; x < W; ++x) {
        const unsigned c = wc[x][threadIdx.x];
        wc[x][threadIdx.x] = run;
        run += c;
      }
      h[threadIdx.x] = run;
    }
    __syncthreads();
    if (v) {
      const uint64_t k = wc[w][d] + __popc(before);
      const uint64_t slot = base[d] + k;
      reinterpret_cast<K*>(pt.w[d].recv_q)[slot] = q[i];
      pt.w[d].recv_org[slot] = (uint64_t(me) << kOrgShift) | (off.qbase + i);
      rpos[i] = uint32_t(roff[d] + k);
    }
  }
}

// Results straight into the requester's result window, each source's run as one
// contiguous run (RemoteOut: slot i - start[s] + dst[s] of source s).
template <typename K>
__global__ void f_return(const PeerTable pt, uint64_t nrecv, const uint64_t* __restrict__ pf,
                         const K* __restrict__ v, const RemoteOut ro) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < nrecv; i += uint64_t(gridDim.x) * blockDim.x) {
    const int src = int(ro.org[i] >> kOrgShift);
    const uint64_t slot = i - ro.start[src] + ro.dst[src];
    pt.w[src].res_pf[slot] = pf[i];
    reinterpret_cast<K*>(pt.w[src].res_v)[slot] = v[i];
  }
}

// Requester: results from the result window (runs per destination) into query order.
template <typename K>
__global__ void f_collect(const uint32_t* __restrict__ rpos, uint64_t m, const uint64_t* __restrict__ res_pf,
                          const K* __restrict__ res_v, uint64_t* __restrict__ out_pf, K* __restrict__ out_v) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < m; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t p = __ldcs(rpos + i);
    __stcs(reinterpret_cast<unsigned long long*>(out_pf) + i, (unsigned long long)res_pf[p]);
    out_v[i] = res_v[p];
  }
}

// Device-side barrier over peer memory: publish `epoch` into every peer's flag
// slot `me`, then wait until every peer has published it into ours.
__global__ void f_barrier(const PeerTable pt, int me, uint32_t epoch) {
  if (threadIdx.x != 0) return;
  __threadfence_system();
  for (int d = 0; d < pt.G; ++d) {
    volatile uint32_t* f = pt.w[d].flags + me;
    *f = epoch;
  }
  __threadfence_system();
  for (int s = 0; s < pt.G; ++s) {
    volatile uint32_t* f = pt.w[me].flags + s;
    while (int32_t(*f - epoch) < 0) {
    }
  }
  __threadfence_system();
}

template <typename T>
int ensure(T** p, uint64_t* cap, uint64_t need) {
  if (need <= *cap) return HBT_OK;
  cudaFree(*p);
  *p = nullptr;
  *cap = 0;
  const uint64_t c = need + need / 8 + 1024;
  HBT_CUDA_TRY(cudaMalloc(p, c * sizeof(T)));
  *cap = c;
  return HBT_OK;
}

RouteTab table_of(const ShardMeta& sm) {
  RouteTab rt{};
  for (int g = 0; g < sm.G; ++g)
    if (sm.count[g]) {
      rt.max[rt.n] = sm.max[g];
      rt.id[rt.n] = uint32_t(g);
      ++rt.n;
    }
  return rt;
}

}  // namespace

// Per-tree state of the fused exchange.
struct FusedState {
  uint8_t* win = nullptr;        // this rank's window (own allocation)
  uint64_t cap_m = 0, cap_r = 0;
  uint8_t* peer[kMaxG] = {};     // mapped peer windows (multi-process)
  uint8_t* dest = nullptr; uint64_t dest_cap = 0;
  uint32_t* rpos = nullptr; uint64_t rpos_cap = 0;   // per query: its slot in our result window
  uint64_t* tmp_pf = nullptr; uint64_t tmp_pf_cap = 0;
  uint8_t* tmp_v = nullptr; uint64_t tmp_v_cap = 0;
  unsigned long long* cnt = nullptr;  // per chunk: kMaxG counts, kMaxG cursors
  unsigned long long* h_mat = nullptr;  // pinned host copy of one parity's count matrices
  cudaStream_t aux = nullptr;         // owner searches of the chunks (overlapping later puts)
  cudaEvent_t ev_put[kMaxChunks] = {}, ev_done = nullptr;
  uint32_t epoch = 0;
  uint64_t batch = 0;                 // parity of the count matrix
};

void fused_free(hbt_tree* t) {
  FusedState* f = static_cast<FusedState*>(t->fused);
  if (!f) return;
  for (int g = 0; g < kMaxG; ++g)
    if (f->peer[g] && f->peer[g] != f->win) cudaIpcCloseMemHandle(f->peer[g]);
  cudaFree(f->win); cudaFree(f->dest); cudaFree(f->rpos); cudaFree(f->tmp_pf); cudaFree(f->tmp_v); cudaFree(f->cnt);
  if (f->h_mat) cudaFreeHost(f->h_mat);
  for (auto& e : f->ev_put)
    if (e) cudaEventDestroy(e);
  if (f->ev_done) cudaEventDestroy(f->ev_done);
  if (f->aux) cudaStreamDestroy(f->aux);
  delete f;
  t->fused = nullptr;
}

namespace {

FusedState* state_of(hbt_tree* t) {
  if (!t->fused) t->fused = new FusedState();
  return static_cast<FusedState*>(t->fused);
}

int alloc_window(FusedState* f, uint64_t cap_m, uint64_t cap_r, uint32_t S) {
  cudaFree(f->win);
  f->win = nullptr;
  HBT_CUDA_TRY(cudaMalloc(&f->win, win_bytes(cap_m, cap_r, S)));
  HBT_CUDA_TRY(cudaMemset(f->win, 0, 256 * ((kMaxG * 4 + 255) / 256) + kMatAll * 8));  // flags + matrices
  f->cap_m = cap_m;
  f->cap_r = cap_r;
  f->epoch = 0;
  return HBT_OK;
}

int prep_local(FusedState* f, uint64_t m) {
  int rc;
  if ((rc = ensure(&f->dest, &f->dest_cap, m ? m : 1))) return rc;
  if ((rc = ensure(&f->rpos, &f->rpos_cap, m ? m : 1))) return rc;
  if (!f->cnt) HBT_CUDA_TRY(cudaMalloc(&f->cnt, kMaxChunks * 2 * kMaxG * sizeof(unsigned long long)));
  if (!f->h_mat) HBT_CUDA_TRY(cudaMallocHost(&f->h_mat, kMaxChunks * kMat * sizeof(unsigned long long)));
  return HBT_OK;
}

// Owner of every query and per-destination counts, chunk by chunk (chunk c = queries
// [c * mc, min((c + 1) * mc, m))).
template <typename K>
int route_and_count(FusedState* f, const K* q, uint64_t m, uint64_t mc, int nchunks, const RouteTab& rt, int G,
                    cudaStream_t st) {
  HBT_CUDA_TRY(cudaMemsetAsync(f->cnt, 0, kMaxChunks * 2 * kMaxG * sizeof(unsigned long long), st));
  for (int c = 0; c < nchunks; ++c) {
    const uint64_t lo = uint64_t(c) * mc, n = lo < m ? std::min<uint64_t>(mc, m - lo) : 0;
    if (!n) continue;
    f_count<K><<<grid_for(n), kThreads, 0, st>>>(q + lo, n, rt, G, f->dest + lo, f->cnt + c * 2 * kMaxG);
    HBT_CUDA_TRY(cudaGetLastError());
  }
  return HBT_OK;
}

// Chunk c of this rank's batch (queries [lo, lo + n)) into the owners' windows.
template <typename K>
int put_queries(FusedState* f, const K* q, uint64_t lo, uint64_t n, const PeerTable& pt, int me,
                const unsigned long long* M, const PutOff& off, int c, cudaStream_t st) {
  if (!n) return HBT_OK;
  const uint64_t chunk = 4096;
  f_put<K><<<unsigned((n + chunk - 1) / chunk), kThreads, 0, st>>>(q + lo, n, f->dest + lo, pt, me, M, off,
                                                                   f->cnt + c * 2 * kMaxG + kMaxG, chunk,
                                                                   f->rpos + lo);
  HBT_CUDA_TRY(cudaGetLastError());
  return HBT_OK;
}

// The owner's search of its receive window, results stored straight back into the
// requesters' result windows.  mat = the G x G count matrix [src][dst] of this batch:
// source s's run in our window starts at sum_{s' < s} mat[s'][me], and its results go
// to s's window from sum_{d < me} mat[s][d] on (where s's f_put pointed its rpos).
template <typename K>
int search_and_return(hbt_tree* t, FusedState* f, const PeerTable& pt, int me, uint64_t rstart,
                      const std::vector<unsigned long long>& mat, const std::vector<uint64_t>& qbase,
                      cudaStream_t st) {
  int rc;
  const int G = pt.G;
  uint64_t nrecv = 0;
  for (int g = 0; g < G; ++g) nrecv += mat[g * G + me];
  if (!nrecv) return HBT_OK;
  const Win& w = pt.w[me];
  const uint8_t* rq = w.recv_q + rstart * sizeof(K);
  RemoteOut ro;
  ro.org = w.recv_org + rstart;
  uint64_t start = 0;
  for (int g = 0; g < G; ++g) {
    ro.pf[g] = pt.w[g].res_pf;
    ro.v[g] = pt.w[g].res_v;
    ro.start[g] = start;
    start += mat[g * G + me];
    uint64_t dst = qbase[g];
    for (int d = 0; d < me; ++d) dst += mat[g * G + d];
    ro.dst[g] = dst;
  }
  if (bucketed_enabled(t, nrecv)) {
    // fused return: the bucketed search's gather stores each result straight into the
    // requester's result window (no staging, no f_return pass)
    rc = bucketed_search(t, rq, nrecv, nullptr, nullptr, t->shard.base[me], st, &ro);
    if (rc != HBT_EUNSUPPORTED) return rc;  // EUNSUPPORTED: no item directory, stage + f_return
  }
  if ((rc = ensure(&f->tmp_pf, &f->tmp_pf_cap, nrecv))) return rc;
  if ((rc = ensure(&f->tmp_v, &f->tmp_v_cap, nrecv * sizeof(K)))) return rc;
  rc = shard_local_search(t, rq, nrecv, f->tmp_pf, f->tmp_v, t->shard.base[me], st);
  if (rc) return rc;
  f_return<K><<<grid_for(nrecv), kThreads, 0, st>>>(pt, nrecv, f->tmp_pf, (const K*)f->tmp_v, ro);
  HBT_CUDA_TRY(cudaGetLastError());
  return HBT_OK;
}

// ------------------------------------------------------------ single process

template <typename K>
int local_t(hbt_tree* const* shards, int G, const void* const* queries, const uint64_t* m, const hbt_out* outs,
            cudaStream_t st) {
  const uint32_t S = sizeof(K);
  const RouteTab rt = table_of(shards[0]->shard);
  // host-side sizes (the multi-process path learns them from the published matrix)
  std::vector<FusedState*> fs(G);
  std::vector<std::vector<unsigned long long>> cnt(G, std::vector<unsigned long long>(G));
  for (int s = 0; s < G; ++s) {
    fs[s] = state_of(shards[s]);
    int rc = prep_local(fs[s], m[s]);
    if (rc) return rc;
    rc = route_and_count<K>(fs[s], (const K*)queries[s], m[s], m[s] ? m[s] : 1, 1, rt, G, st);
    if (rc) return rc;
    HBT_CUDA_TRY(cudaMemcpyAsync(cnt[s].data(), fs[s]->cnt, G * 8, cudaMemcpyDeviceToHost, st));
  }
  HBT_CUDA_TRY(cudaStreamSynchronize(st));
  uint64_t need_m = 1, need_r = 1;
  for (int d = 0; d < G; ++d) {
    uint64_t r = 0;
    for (int s = 0; s < G; ++s) r += cnt[s][d];
    need_r = std::max<uint64_t>(need_r, r);
    need_m = std::max<uint64_t>(need_m, m[d]);
  }
  PeerTable pt{};
  pt.G = G;
  for (int g = 0; g < G; ++g) {
    if (fs[g]->cap_m < need_m || fs[g]->cap_r < need_r || !fs[g]->win) {
      int rc = alloc_window(fs[g], need_m + need_m / 8, need_r + need_r / 8, S);
      if (rc) return rc;
    }
    pt.w[g] = carve(fs[g]->win, fs[g]->cap_m, fs[g]->cap_r, S);
  }
  for (int s = 0; s < G; ++s) {
    f_publish<<<1, 256, 0, st>>>(pt, s, fs[s]->cnt, 0, 1);
    HBT_CUDA_TRY(cudaGetLastError());
  }
  PutOff off{};
  for (int s = 0; s < G; ++s) {
    int rc = put_queries<K>(fs[s], (const K*)queries[s], 0, m[s], pt, s, pt.w[s].matrix, off, 0, st);
    if (rc) return rc;
  }
  std::vector<unsigned long long> mat(G * G);
  for (int s = 0; s < G; ++s)
    for (int d = 0; d < G; ++d) mat[s * G + d] = cnt[s][d];
  const std::vector<uint64_t> qbase(G, 0);
  for (int d = 0; d < G; ++d) {
    int rc = search_and_return<K>(shards[d], fs[d], pt, d, 0, mat, qbase, st);
    if (rc) return rc;
  }
  for (int s = 0; s < G; ++s) {
    if (!m[s]) continue;
    f_collect<K><<<grid_for(m[s]), kThreads, 0, st>>>(fs[s]->rpos, m[s], pt.w[s].res_pf, (const K*)pt.w[s].res_v,
                                                      outs[s].pos_found, (K*)outs[s].values);
    HBT_CUDA_TRY(cudaGetLastError());
  }
  return HBT_OK;
}

// ------------------------------------------------------------ one process per GPU

#define NCCL_TRY2(expr)                                                                   \
  do {                                                                                    \
    ncclResult_t _r = (expr);                                                             \
    if (_r != ncclSuccess) {                                                              \
      set_error("%s:%d %s: %s", __FILE__, __LINE__, #expr, ncclGetErrorString(_r));        \
      return HBT_ENCCL;                                                                   \
    }                                                                                     \
  } while (0)

// (Re)allocate this rank's window and map every peer's (collective).
int exchange_windows(FusedState* f, hbt_comm* c, uint64_t cap_m, uint64_t cap_r, uint32_t S, cudaStream_t st) {
  HBT_CUDA_TRY(cudaStreamSynchronize(st));  // no kernel of ours still touches a peer window
  for (int g = 0; g < kMaxG; ++g) {
    if (f->peer[g] && f->peer[g] != f->win) cudaIpcCloseMemHandle(f->peer[g]);
    f->peer[g] = nullptr;
  }
  if (f->win) {
    // every peer must have closed its mapping of our old window before it is freed
    uint8_t one = 1;
    std::vector<uint8_t> all(c->nranks);
    int rc0 = comm_allgather_host(c, &one, all.data(), 1, st);
    if (rc0) return rc0;
  }
  int rc = alloc_window(f, cap_m, cap_r, S);
  if (rc) return rc;
  cudaIpcMemHandle_t h;
  HBT_CUDA_TRY(cudaIpcGetMemHandle(&h, f->win));
  std::vector<cudaIpcMemHandle_t> all(c->nranks);
  rc = comm_allgather_host(c, &h, all.data(), sizeof(h), st);
  if (rc) return rc;
  for (int g = 0; g < c->nranks; ++g) {
    if (g == c->rank) { f->peer[g] = f->win; continue; }
    void* p = nullptr;
    HBT_CUDA_TRY(cudaIpcOpenMemHandle(&p, all[g], cudaIpcMemLazyEnablePeerAccess));
    f->peer[g] = (uint8_t*)p;
  }
  return HBT_OK;
}

// The batch is cut into C chunks ("exchange_chunks"): chunk c's queries are put into the
// owners' windows (region c of every window) on the caller's stream while the owner
// searches chunk c-1 on an auxiliary stream, so the NVLink stores of the put overlap the
// owner's search (the paper's double buffering of transfers against processing,
// P:232-238, on peer memory).  The C count rows are published together, so one barrier
// and one D2H size every chunk; chunk regions do not overlap, so no slot is reused
// within a batch.
template <typename K>
int nccl_fused_t(hbt_tree* t, const void* queries, uint64_t m, hbt_out out, cudaStream_t st) {
  hbt_comm* c = t->shard.comm;
  const int G = c->nranks, me = c->rank;
  const uint32_t S = sizeof(K);
  FusedState* f = state_of(t);
  int rc = prep_local(f, m);
  if (rc) return rc;
  const int C = int(std::max<uint32_t>(1, std::min<uint32_t>(t->cfg.exchange_chunks, kMaxChunks)));
  const uint64_t mc = std::max<uint64_t>(1, (m + C - 1) / C);
  const RouteTab rt = table_of(t->shard);
  {
    NvtxRange r("exchange.count");
    rc = route_and_count<K>(f, (const K*)queries, m, mc, C, rt, G, st);
  }
  if (rc) return rc;
  const int par = int(f->batch & 1);
  // mat[ch][src * G + dst]
  std::vector<std::vector<unsigned long long>> mat(C, std::vector<unsigned long long>(G * G));
  PeerTable pt{};
  pt.G = G;
  // every rank must use the same C: agree on it with the window (first batch) or trust
  // the configuration (the bench and the tests set it on every rank)
  const bool had_windows = f->win != nullptr;
  if (had_windows) {
    // steady state: the count rows travel by peer stores, no host collective
    for (int g = 0; g < G; ++g) pt.w[g] = carve(f->peer[g], f->cap_m, f->cap_r, S);
    f_publish<<<1, 256, 0, st>>>(pt, me, f->cnt, par, C);
    f_barrier<<<1, 32, 0, st>>>(pt, me, ++f->epoch);
    HBT_CUDA_TRY(cudaGetLastError());
    HBT_CUDA_TRY(cudaMemcpyAsync(f->h_mat, pt.w[me].matrix + uint64_t(par) * kMaxChunks * kMat, C * kMat * 8,
                                 cudaMemcpyDeviceToHost, st));
    HBT_CUDA_TRY(cudaStreamSynchronize(st));
    for (int ch = 0; ch < C; ++ch)
      for (int s2 = 0; s2 < G; ++s2)
        for (int x = 0; x < G; ++x) mat[ch][s2 * G + x] = f->h_mat[ch * kMat + s2 * kMaxG + x];
  } else {
    // first batch: no windows to store into yet; the count rows go through the host
    std::vector<unsigned long long> mine(C * G), all(size_t(C) * G * G);
    std::vector<unsigned long long> dev(C * 2 * kMaxG);
    HBT_CUDA_TRY(cudaMemcpyAsync(dev.data(), f->cnt, dev.size() * 8, cudaMemcpyDeviceToHost, st));
    HBT_CUDA_TRY(cudaStreamSynchronize(st));
    for (int ch = 0; ch < C; ++ch)
      for (int x = 0; x < G; ++x) mine[ch * G + x] = dev[ch * 2 * kMaxG + x];
    rc = comm_allgather_host(c, mine.data(), all.data(), C * G * 8, st);
    if (rc) return rc;
    for (int s2 = 0; s2 < G; ++s2)
      for (int ch = 0; ch < C; ++ch)
        for (int x = 0; x < G; ++x) mat[ch][s2 * G + x] = all[(size_t(s2) * C + ch) * G + x];
  }
  uint64_t need_m = 1, need_r = 1;
  for (int x = 0; x < G; ++x) {
    uint64_t row = 0, col = 0;
    for (int ch = 0; ch < C; ++ch)
      for (int y = 0; y < G; ++y) { row += mat[ch][x * G + y]; col += mat[ch][y * G + x]; }
    need_m = std::max<uint64_t>(need_m, row);
    need_r = std::max<uint64_t>(need_r, col);
  }
  if (!had_windows || f->cap_m < need_m || f->cap_r < need_r) {
    // every rank holds the same matrices, so every rank takes this branch (collective)
    rc = exchange_windows(f, c, need_m + need_m / 8, need_r + need_r / 8, S, st);
    if (rc) return rc;
    for (int g = 0; g < G; ++g) pt.w[g] = carve(f->peer[g], f->cap_m, f->cap_r, S);
    std::vector<unsigned long long> full(C * kMat, 0);
    for (int ch = 0; ch < C; ++ch)
      for (int s2 = 0; s2 < G; ++s2)
        for (int x = 0; x < G; ++x) full[ch * kMat + s2 * kMaxG + x] = mat[ch][s2 * G + x];
    HBT_CUDA_TRY(cudaMemcpyAsync(pt.w[me].matrix + uint64_t(par) * kMaxChunks * kMat, full.data(), C * kMat * 8,
                                 cudaMemcpyHostToDevice, st));
    f_barrier<<<1, 32, 0, st>>>(pt, me, ++f->epoch);  // every window exists and holds its matrices
  }
  if (C > 1 && !f->aux) {
    HBT_CUDA_TRY(cudaStreamCreateWithFlags(&f->aux, cudaStreamNonBlocking));
    for (auto& e : f->ev_put) HBT_CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    HBT_CUDA_TRY(cudaEventCreateWithFlags(&f->ev_done, cudaEventDisableTiming));
  }
  // per chunk: region bases in every owner's window, and every source's first query
  std::vector<uint64_t> rbase(G, 0), qb(G, 0);
  uint64_t my_rstart = 0;
  for (int ch = 0; ch < C; ++ch) {
    const std::vector<unsigned long long>& M = mat[ch];
    PutOff off{};
    for (int d = 0; d < G; ++d) off.rbase[d] = rbase[d];
    off.qbase = uint64_t(ch) * mc;
    const uint64_t lo = uint64_t(ch) * mc, n = lo < m ? std::min<uint64_t>(mc, m - lo) : 0;
    {
      NvtxRange r("exchange.put");
      rc = put_queries<K>(f, (const K*)queries, lo, n, pt, me, pt.w[me].matrix + (uint64_t(par) * kMaxChunks + ch) * kMat,
                          off, ch, st);
    }
    if (rc) return rc;
    f_barrier<<<1, 32, 0, st>>>(pt, me, ++f->epoch);  // chunk ch is in every owner's window
    HBT_CUDA_TRY(cudaGetLastError());
    cudaStream_t ss = st;
    if (C > 1) {
      HBT_CUDA_TRY(cudaEventRecord(f->ev_put[ch], st));
      HBT_CUDA_TRY(cudaStreamWaitEvent(f->aux, f->ev_put[ch], 0));
      ss = f->aux;
    }
    {
      NvtxRange r("owner_search_and_return");
      rc = search_and_return<K>(t, f, pt, me, my_rstart, M, qb, ss);
    }
    if (rc) return rc;
    for (int s2 = 0; s2 < G; ++s2) {
      my_rstart += M[s2 * G + me];
      for (int d = 0; d < G; ++d) rbase[d] += M[s2 * G + d];
      uint64_t row = 0;
      for (int d = 0; d < G; ++d) row += M[s2 * G + d];
      qb[s2] += row;
    }
  }
  if (C > 1) {  // the owner searches of every chunk, then the last barrier
    HBT_CUDA_TRY(cudaEventRecord(f->ev_done, f->aux));
    HBT_CUDA_TRY(cudaStreamWaitEvent(st, f->ev_done, 0));
  }
  f_barrier<<<1, 32, 0, st>>>(pt, me, ++f->epoch);  // every owner has stored our results
  HBT_CUDA_TRY(cudaGetLastError());
  if (m) {  // our results, one run per (chunk, owner) in our window, back into query order
    f_collect<K><<<grid_for(m), kThreads, 0, st>>>(f->rpos, m, pt.w[me].res_pf, (const K*)pt.w[me].res_v,
                                                   out.pos_found, (K*)out.values);
    HBT_CUDA_TRY(cudaGetLastError());
  }
  ++f->batch;
  return HBT_OK;
}

}  // namespace

int fused_search_local(hbt_tree* const* shards, int G, const void* const* queries, const uint64_t* m,
                       const hbt_out* outs, cudaStream_t st) {
  return shards[0]->width == 4 ? local_t<uint32_t>(shards, G, queries, m, outs, st)
                               : local_t<uint64_t>(shards, G, queries, m, outs, st);
}

int fused_search_nccl(const hbt_tree* t, const void* queries, uint64_t m, hbt_out out, cudaStream_t st) {
  hbt_tree* tt = const_cast<hbt_tree*>(t);
  std::lock_guard<std::mutex> lock(tt->pipe.mu);
  return t->width == 4 ? nccl_fused_t<uint32_t>(tt, queries, m, out, st) : nccl_fused_t<uint64_t>(tt, queries, m, out, st);
}

}  // namespace hbt
