// sharded.cu — key-range-sharded implicit trees over G GPUs.
//
// Shard g holds a contiguous key range (ranks in key order).  A query goes to
//   owner(q) = #(shard_max < q)   over the non-empty shards (clamped to the last)
// — the max-separator rule of the node search (R1/R3) applied one level
// above the shard roots, which also routes a missing key to the shard holding
// its successor.  Per batch:
//   route_count    owner of every query + per-destination counts (smem histogram)
//   [counts all-to-all]
//   route_scatter  queries grouped by destination (CTA-reserved blocks)
//   [queries all-to-all]  -> the owner's receive buffer, segmented by source
//   implicit search with pos_base = the shard's first global rank
//   [results all-to-all back, in the same order]
//   unpermute      out[origin[i]] = result[i]
// The exchanges are NCCL send/recv over NVLink (north_star: "results returned by
// NCCL all-to-all").  hbt_search_sharded_local runs the SAME kernels for G
// shards on one GPU with device-to-device copies as the exchange, which is how
// the pipeline is tested on a single B200.
#include <nccl.h>

#include <vector>

#include "hbt_internal.cuh"

namespace hbt {
namespace {

#define NCCL_TRY(expr)                                                         \
  do {                                                                         \
    ncclResult_t _r = (expr);                                                  \
    if (_r != ncclSuccess) {                                                   \
      set_error("%s:%d %s: %s", __FILE__, __LINE__, #expr, ncclGetErrorString(_r)); \
      return HBT_ENCCL;                                                        \
    }                                                                          \
  } while (0)

constexpr int kMaxShards = 64;
constexpr int kThreads = 256;

struct RouteTable {
  uint64_t max[kMaxShards];  // maxima of the non-empty shards, in shard order
  uint32_t id[kMaxShards];   // their shard ids
  uint32_t n;                // non-empty shards (0: every query goes to shard 0)
};

template <typename K>
__device__ __forceinline__ uint32_t owner_of(K q, const RouteTable& rt) {
  if (rt.n == 0) return 0;
  uint32_t c = 0;
  for (uint32_t i = 0; i < rt.n; ++i) c += (K(rt.max[i]) < q) ? 1u : 0u;
  return rt.id[c < rt.n ? c : rt.n - 1];
}

template <typename K>
__global__ void __launch_bounds__(kThreads) route_count(const K* __restrict__ q, uint64_t m, const RouteTable rt,
                                                        uint32_t G, uint8_t* __restrict__ dest,
                                                        unsigned long long* __restrict__ counts) {
  __shared__ unsigned int h[kMaxShards];
  for (uint32_t i = threadIdx.x; i < G; i += blockDim.x) h[i] = 0;
  __syncthreads();
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < m; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t o = owner_of(q[i], rt);
    dest[i] = uint8_t(o);
    atomicAdd(&h[o], 1u);
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < G; i += blockDim.x)
    if (h[i]) atomicAdd(counts + i, (unsigned long long)h[i]);
}

// Scatter: each CTA counts its slice per destination, reserves a block in each
// destination segment with one atomic, then places its queries there.
template <typename K>
__global__ void __launch_bounds__(kThreads) route_scatter(const K* __restrict__ q, uint64_t m,
                                                          const uint8_t* __restrict__ dest, uint32_t G,
                                                          unsigned long long* __restrict__ cursor,
                                                          K* __restrict__ send_q, uint32_t* __restrict__ origin,
                                                          uint64_t chunk) {
  __shared__ unsigned int h[kMaxShards];
  __shared__ unsigned long long base[kMaxShards];
  const uint64_t lo = blockIdx.x * chunk;
  const uint64_t hi = lo + chunk < m ? lo + chunk : m;
  for (uint32_t i = threadIdx.x; i < G; i += blockDim.x) h[i] = 0;
  __syncthreads();
  for (uint64_t i = lo + threadIdx.x; i < hi; i += blockDim.x) atomicAdd(&h[dest[i]], 1u);
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < G; i += blockDim.x) {
    base[i] = h[i] ? atomicAdd(cursor + i, (unsigned long long)h[i]) : 0ull;
    h[i] = 0;
  }
  __syncthreads();
  for (uint64_t i = lo + threadIdx.x; i < hi; i += blockDim.x) {
    const uint32_t d = dest[i];
    const uint64_t slot = base[d] + atomicAdd(&h[d], 1u);
    send_q[slot] = q[i];
    origin[slot] = uint32_t(i);
  }
}

template <typename K>
__global__ void unpermute(const uint32_t* __restrict__ origin, uint64_t m, const uint64_t* __restrict__ pf,
                          const K* __restrict__ v, uint64_t* __restrict__ out_pf, K* __restrict__ out_v) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < m; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t o = origin[i];
    out_pf[o] = pf[i];
    out_v[o] = v[i];
  }
}

inline unsigned grid_for(uint64_t n) {
  uint64_t g = (n + kThreads - 1) / kThreads;
  if (g > 148 * 16) g = 148 * 16;
  return unsigned(g ? g : 1);
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

int prepare(Scratch& s, uint64_t m, uint64_t recv, uint32_t S) {
  int rc;
  if ((rc = ensure(&s.dest, &s.dest_cap, m ? m : 1))) return rc;
  if ((rc = ensure(&s.send_q, &s.send_cap, (m ? m : 1) * S))) return rc;
  if ((rc = ensure(&s.origin, &s.origin_cap, m ? m : 1))) return rc;
  if ((rc = ensure(&s.recv_q, &s.recv_cap, (recv ? recv : 1) * S))) return rc;
  if ((rc = ensure(&s.res_pf, &s.res_pf_cap, recv ? recv : 1))) return rc;
  if ((rc = ensure(&s.res_v, &s.res_v_cap, (recv ? recv : 1) * S))) return rc;
  if ((rc = ensure(&s.back_pf, &s.back_pf_cap, m ? m : 1))) return rc;
  if ((rc = ensure(&s.back_v, &s.back_v_cap, (m ? m : 1) * S))) return rc;
  if (!s.counts) HBT_CUDA_TRY(cudaMalloc(&s.counts, 2 * kMaxShards * sizeof(unsigned long long)));
  return HBT_OK;
}

void free_scratch(Scratch& s) {
  cudaFree(s.dest); cudaFree(s.send_q); cudaFree(s.origin); cudaFree(s.recv_q); cudaFree(s.res_pf);
  cudaFree(s.res_v); cudaFree(s.back_pf); cudaFree(s.back_v); cudaFree(s.counts);
  s = Scratch{};
}

// route_count + route_scatter for one source; counts[0..G) receive the per-destination counts
template <typename K>
int route(const K* q, uint64_t m, const RouteTable& rt, uint32_t G, Scratch& s, cudaStream_t st,
          std::vector<unsigned long long>& h_counts) {
  HBT_CUDA_TRY(cudaMemsetAsync(s.counts, 0, 2 * kMaxShards * sizeof(unsigned long long), st));
  if (m) {
    route_count<K><<<grid_for(m), kThreads, 0, st>>>(q, m, rt, G, s.dest, s.counts);
    HBT_CUDA_TRY(cudaGetLastError());
  }
  h_counts.assign(G, 0);
  HBT_CUDA_TRY(cudaMemcpyAsync(h_counts.data(), s.counts, G * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
  HBT_CUDA_TRY(cudaStreamSynchronize(st));
  if (m) {
    std::vector<unsigned long long> off(G, 0);
    for (uint32_t g = 1; g < G; ++g) off[g] = off[g - 1] + h_counts[g - 1];
    HBT_CUDA_TRY(cudaMemcpyAsync(s.counts + kMaxShards, off.data(), G * sizeof(unsigned long long),
                                 cudaMemcpyHostToDevice, st));
    const uint64_t chunk = 4096;
    const uint64_t blocks = (m + chunk - 1) / chunk;
    route_scatter<K><<<unsigned(blocks), kThreads, 0, st>>>(q, m, s.dest, G, s.counts + kMaxShards, (K*)s.send_q,
                                                           s.origin, chunk);
    HBT_CUDA_TRY(cudaGetLastError());
  }
  return HBT_OK;
}

RouteTable make_table(const ShardMeta& sm) {
  RouteTable rt{};
  rt.n = 0;
  for (int g = 0; g < sm.G; ++g)
    if (sm.count[g]) {
      rt.max[rt.n] = sm.max[g];
      rt.id[rt.n] = uint32_t(g);
      ++rt.n;
    }
  return rt;
}

int first_last_keys(const hbt_tree* t, uint64_t* kmin, uint64_t* kmax) {
  *kmin = *kmax = 0;
  if (t->n == 0) return HBT_OK;
  const uint32_t S = t->width, P = t->P;
  const uint64_t last = t->n - 1;
  uint64_t a = 0, b = 0;
  HBT_CUDA_TRY(cudaMemcpy(&a, (const uint8_t*)t->d_leaf, S, cudaMemcpyDefault));
  HBT_CUDA_TRY(cudaMemcpy(&b, (const uint8_t*)t->d_leaf + (last / P) * 64 + (last % P) * S, S, cudaMemcpyDefault));
  *kmin = a;
  *kmax = b;
  return HBT_OK;
}

int validate_and_set(ShardMeta& sm, const std::vector<uint64_t>& cnt, const std::vector<uint64_t>& mn,
                     const std::vector<uint64_t>& mx, int G) {
  sm.G = G;
  uint64_t base = 0;
  bool have_prev = false;
  uint64_t prev_max = 0;
  for (int g = 0; g < G; ++g) {
    sm.count[g] = cnt[g];
    sm.base[g] = base;
    sm.max[g] = mx[g];
    if (cnt[g]) {
      if (have_prev && mn[g] <= prev_max) {
        set_error("shard %d's keys overlap an earlier shard's range (shards must be in key order)", g);
        return HBT_EINVAL;
      }
      have_prev = true;
      prev_max = mx[g];
    }
    base += cnt[g];
  }
  return HBT_OK;
}

template <typename K>
int search_local_t(hbt_tree* const* shards, int G, const void* const* queries, const uint64_t* m,
                   const hbt_out* outs, cudaStream_t st) {
  const uint32_t S = sizeof(K);
  const RouteTable rt = make_table(shards[0]->shard);
  std::vector<std::vector<unsigned long long>> cnt(G);
  // 1. route on every source
  for (int s = 0; s < G; ++s) {
    Scratch& sc = shards[s]->shard_scratch;
    int rc = prepare(sc, m[s], 0, S);
    if (rc) return rc;
    rc = route<K>((const K*)queries[s], m[s], rt, uint32_t(G), sc, st, cnt[s]);
    if (rc) return rc;
  }
  // 2. "all-to-all" of queries: destination d receives segments from s = 0..G-1 in order
  std::vector<uint64_t> recv(G, 0);
  for (int d = 0; d < G; ++d)
    for (int s = 0; s < G; ++s) recv[d] += cnt[s][d];
  for (int d = 0; d < G; ++d) {
    int rc = prepare(shards[d]->shard_scratch, m[d], recv[d], S);
    if (rc) return rc;
  }
  for (int d = 0; d < G; ++d) {
    uint64_t roff = 0;
    for (int s = 0; s < G; ++s) {
      uint64_t soff = 0;
      for (int e = 0; e < d; ++e) soff += cnt[s][e];
      if (cnt[s][d])
        HBT_CUDA_TRY(cudaMemcpyAsync(shards[d]->shard_scratch.recv_q + roff * S, shards[s]->shard_scratch.send_q + soff * S,
                                     cnt[s][d] * S, cudaMemcpyDeviceToDevice, st));
      roff += cnt[s][d];
    }
  }
  // 3. owners search with their global rank base
  for (int d = 0; d < G; ++d) {
    Scratch& sc = shards[d]->shard_scratch;
    int rc = shard_local_search(shards[d], sc.recv_q, recv[d], sc.res_pf, sc.res_v, shards[d]->shard.base[d], st);
    if (rc) return rc;
  }
  // 4. results back in send order, 5. unpermute
  for (int s = 0; s < G; ++s) {
    uint64_t soff = 0;
    for (int d = 0; d < G; ++d) {
      uint64_t roff = 0;
      for (int e = 0; e < s; ++e) roff += cnt[e][d];
      if (cnt[s][d]) {
        HBT_CUDA_TRY(cudaMemcpyAsync(shards[s]->shard_scratch.back_pf + soff, shards[d]->shard_scratch.res_pf + roff,
                                     cnt[s][d] * 8, cudaMemcpyDeviceToDevice, st));
        HBT_CUDA_TRY(cudaMemcpyAsync(shards[s]->shard_scratch.back_v + soff * S, shards[d]->shard_scratch.res_v + roff * S,
                                     cnt[s][d] * S, cudaMemcpyDeviceToDevice, st));
      }
      soff += cnt[s][d];
    }
    Scratch& sc = shards[s]->shard_scratch;
    if (m[s]) {
      unpermute<K><<<grid_for(m[s]), kThreads, 0, st>>>(sc.origin, m[s], sc.back_pf, (const K*)sc.back_v,
                                                        outs[s].pos_found, (K*)outs[s].values);
      HBT_CUDA_TRY(cudaGetLastError());
    }
  }
  return HBT_OK;
}

ncclDataType_t u8() { return ncclUint8; }

// Poll the communicator's asynchronous error state (a peer failure or a network error
// surfaces here, not in the enqueue calls' return codes).
int nccl_async_ok(ncclComm_t comm) {
  ncclResult_t a = ncclSuccess;
  ncclResult_t r = ncclCommGetAsyncError(comm, &a);
  if (r != ncclSuccess) { set_error("ncclCommGetAsyncError: %s", ncclGetErrorString(r)); return HBT_ENCCL; }
  if (a != ncclSuccess && a != ncclInProgress) {
    set_error("NCCL asynchronous error: %s", ncclGetErrorString(a));
    return HBT_ENCCL;
  }
  return HBT_OK;
}

template <typename K>
int search_nccl_t(const hbt_tree* tc, const void* queries, uint64_t m, hbt_out out, cudaStream_t st) {
  hbt_tree* t = const_cast<hbt_tree*>(tc);
  const ShardMeta& sm = t->shard;
  hbt_comm* c = sm.comm;
  const int G = c->nranks, me = c->rank;
  const uint32_t S = sizeof(K);
  Scratch& sc = t->shard_scratch;
  std::lock_guard<std::mutex> lock(t->pipe.mu);
  int rc = prepare(sc, m, 0, S);
  if (rc) return rc;
  const RouteTable rt = make_table(sm);
  std::vector<unsigned long long> scnt;
  rc = route<K>((const K*)queries, m, rt, uint32_t(G), sc, st, scnt);
  if (rc) return rc;
  // counts all-to-all (one u64 per peer)
  HBT_CUDA_TRY(cudaMemcpyAsync(sc.counts, scnt.data(), G * 8, cudaMemcpyHostToDevice, st));
  NCCL_TRY(ncclAlltoAll(sc.counts, sc.counts + kMaxShards, 1, ncclUint64, c->comm, st));
  std::vector<unsigned long long> rcnt(G, 0);
  HBT_CUDA_TRY(cudaMemcpyAsync(rcnt.data(), sc.counts + kMaxShards, G * 8, cudaMemcpyDeviceToHost, st));
  HBT_CUDA_TRY(cudaStreamSynchronize(st));
  if ((rc = nccl_async_ok(c->comm))) return rc;
  uint64_t recv = 0;
  for (int g = 0; g < G; ++g) recv += rcnt[g];
  if ((rc = prepare(sc, m, recv, S))) return rc;
  // queries out, grouped by destination
  NCCL_TRY(ncclGroupStart());
  uint64_t so = 0, ro = 0;
  for (int p = 0; p < G; ++p) {
    if (scnt[p]) NCCL_TRY(ncclSend(sc.send_q + so * S, scnt[p] * S, u8(), p, c->comm, st));
    if (rcnt[p]) NCCL_TRY(ncclRecv(sc.recv_q + ro * S, rcnt[p] * S, u8(), p, c->comm, st));
    so += scnt[p];
    ro += rcnt[p];
  }
  NCCL_TRY(ncclGroupEnd());
  rc = shard_local_search(t, sc.recv_q, recv, sc.res_pf, sc.res_v, sm.base[me], st);
  if (rc) return rc;
  // results back, in the order they came
  NCCL_TRY(ncclGroupStart());
  so = ro = 0;
  for (int p = 0; p < G; ++p) {
    if (rcnt[p]) {
      NCCL_TRY(ncclSend(sc.res_pf + ro, rcnt[p] * 8, u8(), p, c->comm, st));
      NCCL_TRY(ncclSend(sc.res_v + ro * S, rcnt[p] * S, u8(), p, c->comm, st));
    }
    if (scnt[p]) {
      NCCL_TRY(ncclRecv(sc.back_pf + so, scnt[p] * 8, u8(), p, c->comm, st));
      NCCL_TRY(ncclRecv(sc.back_v + so * S, scnt[p] * S, u8(), p, c->comm, st));
    }
    so += scnt[p];
    ro += rcnt[p];
  }
  NCCL_TRY(ncclGroupEnd());
  if (m) {
    unpermute<K><<<grid_for(m), kThreads, 0, st>>>(sc.origin, m, sc.back_pf, (const K*)sc.back_v, out.pos_found,
                                                   (K*)out.values);
    HBT_CUDA_TRY(cudaGetLastError());
  }
  return nccl_async_ok(c->comm);
}

}  // namespace

int comm_allgather_host(hbt_comm* c, const void* send, void* recv, uint64_t bytes, cudaStream_t st) {
  if (c->host_allgather) {
    if (c->host_allgather(send, recv, bytes, c->host_ctx) != 0) {
      set_error("host all-gather callback failed");
      return HBT_ENCCL;
    }
    return HBT_OK;
  }
  uint8_t* d = nullptr;
  HBT_CUDA_TRY(cudaMalloc(&d, bytes * (c->nranks + 1)));
  cudaMemcpyAsync(d, send, bytes, cudaMemcpyHostToDevice, st);
  ncclResult_t r = ncclAllGather(d, d + bytes, bytes, ncclUint8, c->comm, st);
  if (r == ncclSuccess) cudaMemcpyAsync(recv, d + bytes, bytes * c->nranks, cudaMemcpyDeviceToHost, st);
  cudaError_t e = cudaStreamSynchronize(st);
  cudaFree(d);
  if (r != ncclSuccess) { set_error("ncclAllGather: %s", ncclGetErrorString(r)); return HBT_ENCCL; }
  if (e != cudaSuccess) { set_error("all-gather: %s", cudaGetErrorString(e)); return HBT_ECUDA; }
  return nccl_async_ok(c->comm);
}

void shard_free(hbt_tree* t) { free_scratch(t->shard_scratch); }

}  // namespace hbt

using namespace hbt;

extern "C" {

int hbt_comm_unique_id(void* id128) {
  if (!id128) { set_error("NULL id"); return HBT_EINVAL; }
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  NCCL_TRY(ncclGetUniqueId(reinterpret_cast<ncclUniqueId*>(id128)));
  return HBT_OK;
}

int hbt_comm_init(int nranks, int rank, const void* id128, hbt_comm** out) {
  if (!out || !id128 || nranks < 1 || nranks > kMaxShards || rank < 0 || rank >= nranks) {
    set_error("bad communicator arguments");
    return HBT_EINVAL;
  }
  *out = nullptr;
  hbt_comm* c = new hbt_comm();
  ncclUniqueId id;
  memcpy(&id, id128, sizeof(id));
  ncclResult_t r = ncclCommInitRank(&c->comm, nranks, id, rank);
  if (r != ncclSuccess) {
    set_error("ncclCommInitRank: %s", ncclGetErrorString(r));
    delete c;
    return HBT_ENCCL;
  }
  c->nranks = nranks;
  c->rank = rank;
  *out = c;
  return HBT_OK;
}

int hbt_comm_init_host(int nranks, int rank, hbt_allgather_fn fn, void* ctx, hbt_comm** out) {
  if (!out || !fn || nranks < 1 || nranks > kMaxShards || rank < 0 || rank >= nranks) {
    set_error("bad communicator arguments");
    return HBT_EINVAL;
  }
  hbt_comm* c = new hbt_comm();
  c->nranks = nranks;
  c->rank = rank;
  c->host_allgather = fn;
  c->host_ctx = ctx;
  *out = c;
  return HBT_OK;
}

int hbt_comm_destroy(hbt_comm* c) {
  if (!c) return HBT_EINVAL;
  if (c->comm) ncclCommDestroy(c->comm);
  delete c;
  return HBT_OK;
}

int hbt_comm_shard_table(hbt_comm* c, uint64_t n_local, uint64_t kmin, uint64_t kmax, uint64_t* counts,
                         uint64_t* bases, uint64_t* maxima) {
  if (!c || !counts || !bases || !maxima) { set_error("NULL argument"); return HBT_EINVAL; }
  NvtxRange nvtx_("hbt_comm_shard_table");
  const int G = c->nranks;
  uint64_t mine[3] = {n_local, kmin, kmax};
  std::vector<uint64_t> all(3 * G);
  int rc = comm_allgather_host(c, mine, all.data(), sizeof(mine), nullptr);
  if (rc) return rc;
  std::vector<uint64_t> cn(G), mnv(G), mxv(G);
  for (int g = 0; g < G; ++g) { cn[g] = all[3 * g]; mnv[g] = all[3 * g + 1]; mxv[g] = all[3 * g + 2]; }
  ShardMeta sm;
  if ((rc = validate_and_set(sm, cn, mnv, mxv, G))) return rc;
  for (int g = 0; g < G; ++g) {
    counts[g] = sm.count[g];
    bases[g] = sm.base[g];
    maxima[g] = sm.max[g];
  }
  return HBT_OK;
}

int hbt_bulk_build_sharded(hbt_comm* c, const void* keys_local, const void* values_local, uint64_t n_local,
                           uint32_t fanout, uint32_t layout, void* stream, hbt_tree** out) {
  NvtxRange nvtx_("hbt_bulk_build_sharded");
  if (!c || !out) { set_error("NULL argument"); return HBT_EINVAL; }
  if ((layout & 0x1) != HBT_IMPLICIT) { set_error("sharded trees are implicit"); return HBT_EUNSUPPORTED; }
  int rc = hbt_bulk_build(keys_local, values_local, n_local, fanout, layout, stream, out);
  if (rc) return rc;
  hbt_tree* t = *out;
  const int G = c->nranks;
  uint64_t mn = 0, mx = 0;
  if ((rc = first_last_keys(t, &mn, &mx))) { hbt_destroy(t); *out = nullptr; return rc; }
  // all-gather (n', min, max) of every shard, validate the key order, set the routing table
  std::vector<uint64_t> cn(G), bs(G), mxv(G);
  if ((rc = hbt_comm_shard_table(c, t->n, mn, mx, cn.data(), bs.data(), mxv.data()))) {
    hbt_destroy(t);
    *out = nullptr;
    return rc;
  }
  t->shard.G = G;
  for (int g = 0; g < G; ++g) {
    t->shard.count[g] = cn[g];
    t->shard.base[g] = bs[g];
    t->shard.max[g] = mxv[g];
  }
  t->shard.comm = c;
  t->shard.rank = c->rank;
  return HBT_OK;
}

int hbt_search_sharded(const hbt_tree* t, const void* queries_local, uint64_t m_local, hbt_out out_local,
                       void* stream) {
  NvtxRange nvtx_("hbt_search_sharded");
  if (!t || !t->shard.comm) { set_error("not a sharded tree"); return HBT_EINVAL; }
  cudaStream_t st = (cudaStream_t)stream;
  if (t->shard.G == 1 && t->cfg.exchange == 0 && t->cfg.g1_direct) {
    // One shard owns every key: routing would send every query to this rank and the
    // exchange would only copy, so search in place (global pos = the shard's base rank).
    if (m_local == 0) return HBT_OK;
    if (!queries_local || !out_local.pos_found || !out_local.values) { set_error("NULL buffer"); return HBT_EINVAL; }
    return shard_local_search(t, queries_local, m_local, out_local.pos_found, out_local.values, t->shard.base[0], st);
  }
  if (t->cfg.exchange == 0) return fused_search_nccl(t, queries_local, m_local, out_local, st);
  if (!t->shard.comm->comm) { set_error("exchange=1 needs an NCCL communicator"); return HBT_EUNSUPPORTED; }
  return t->width == 4 ? search_nccl_t<uint32_t>(t, queries_local, m_local, out_local, st)
                       : search_nccl_t<uint64_t>(t, queries_local, m_local, out_local, st);
}

int hbt_shard_local_init(hbt_tree* const* shards, int G) {
  if (!shards || G < 1 || G > kMaxShards) { set_error("bad shard list"); return HBT_EINVAL; }
  std::vector<uint64_t> cn(G), mn(G), mx(G);
  for (int g = 0; g < G; ++g) {
    if (!shards[g] || shards[g]->form != HBT_IMPLICIT || shards[g]->width != shards[0]->width) {
      set_error("shards must be implicit trees of one key width");
      return HBT_EINVAL;
    }
    cn[g] = shards[g]->n;
    int rc = first_last_keys(shards[g], &mn[g], &mx[g]);
    if (rc) return rc;
  }
  ShardMeta sm;
  int rc = validate_and_set(sm, cn, mn, mx, G);
  if (rc) return rc;
  for (int g = 0; g < G; ++g) {
    shards[g]->shard = sm;
    shards[g]->shard.rank = g;
    shards[g]->shard.comm = nullptr;
  }
  return HBT_OK;
}

int hbt_search_sharded_local(hbt_tree* const* shards, int G, const void* const* queries, const uint64_t* m,
                             const hbt_out* outs, void* stream) {
  if (!shards || !queries || !m || !outs || G < 1 || G > kMaxShards || shards[0]->shard.G != G) {
    set_error("bad arguments (call hbt_shard_local_init first)");
    return HBT_EINVAL;
  }
  cudaStream_t st = (cudaStream_t)stream;
  if (shards[0]->cfg.exchange == 0) return fused_search_local(shards, G, queries, m, outs, st);
  return shards[0]->width == 4 ? search_local_t<uint32_t>(shards, G, queries, m, outs, st)
                               : search_local_t<uint64_t>(shards, G, queries, m, outs, st);
}

}  // extern "C"
