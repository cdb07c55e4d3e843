// tools/probe.cu — in-run bandwidth probes for bench.py's roofline (libhbtprobe.so).
// Not part of the method: an all-SM random-read probe of L2 at the tree's
// access granularities (32 / 64 / 128 B chunks, 16 B per lane, read-only with a
// checksum), as SURVEY §8(d) "L2 bandwidth microbenchmark" asks for.
#include <cuda_runtime.h>
#include <stdint.h>

#define PROBE_API extern "C" __attribute__((visibility("default")))

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// Each group of CHUNK/16 lanes reads one random CHUNK-byte aligned chunk per
// iteration; UNROLL independent chunks in flight per lane.
template <int CHUNK, int UNROLL>
__global__ void __launch_bounds__(512) l2_random_read(const uint4* __restrict__ buf, uint64_t nchunks, uint64_t iters,
                                                      uint64_t seed, uint4* __restrict__ sink) {
  constexpr int G = CHUNK / 16;
  const int lane = threadIdx.x & 31;
  const uint64_t gid = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) / G;
  const int k = lane % G;
  uint4 acc = make_uint4(0, 0, 0, 0);
  uint64_t state = mix64(gid ^ seed);
  for (uint64_t it = 0; it < iters; ++it) {
    uint4 v[UNROLL];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      state = mix64(state);
      const uint64_t c = __umul64hi(state, nchunks);
      v[u] = __ldg(buf + c * G + k);
    }
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      acc.x ^= v[u].x; acc.y ^= v[u].y; acc.z ^= v[u].z; acc.w ^= v[u].w;
    }
  }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x12345678u) sink[threadIdx.x] = acc;
}

// Returns achieved GB/s for the given chunk size (32, 64 or 128 B) over a
// `bytes`-sized buffer (keep it below L2 for an L2 figure), or <0 on error.
PROBE_API int probe_set_l2_fetch(int bytes) {
  return int(cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, size_t(bytes)));
}

PROBE_API int probe_get_l2_fetch(void) {
  size_t v = 0;
  cudaDeviceGetLimit(&v, cudaLimitMaxL2FetchGranularity);
  return int(v);
}

PROBE_API double probe_random_read_gbs(uint64_t bytes, int chunk, int reps) {
  uint4* buf = nullptr;
  uint4* sink = nullptr;
  if (cudaMalloc(&buf, bytes) != cudaSuccess) return -1;
  cudaMalloc(&sink, 512 * sizeof(uint4));
  cudaMemset(buf, 1, bytes);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint64_t nchunks = bytes / chunk;
  const uint64_t iters = 256;
  const unsigned grid = sms * 4;
  const unsigned threads = 512;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best_ms = 1e30f;
  for (int r = 0; r < reps + 1; ++r) {
    cudaEventRecord(a);
    if (chunk == 32) l2_random_read<32, 8><<<grid, threads>>>(buf, nchunks, iters, r, sink);
    else if (chunk == 64) l2_random_read<64, 8><<<grid, threads>>>(buf, nchunks, iters, r, sink);
    else if (chunk == 256) l2_random_read<256, 8><<<grid, threads>>>(buf, nchunks, iters, r, sink);
    else l2_random_read<128, 8><<<grid, threads>>>(buf, nchunks, iters, r, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    if (r > 0 && ms < best_ms) best_ms = ms;  // first launch is warm-up
  }
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(buf);
  cudaFree(sink);
  if (cudaGetLastError() != cudaSuccess) return -2;
  const double total = double(grid) * threads * iters * 8 * 16;  // bytes read
  return total / (best_ms * 1e-3) / 1e9;
}

// Die-affinity experiment: the SMs are split into two halves by `map` applied
// to %smid (0 = no split, 1 = smid < nsm/2, 2 = smid & 1, 3 = (smid >> 1) & 1,
// 4 = (smid >> 2) & 1, 5 = (smid >> 3) & 1); each half reads random chunks of
// its own half of the buffer only.  If L2 capacity for all-SM random reads is
// lost to cross-die duplication, the right split restores it.
__device__ __forceinline__ uint32_t smid() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

template <int CHUNK, int UNROLL>
__global__ void __launch_bounds__(512) l2_random_read_aff(const uint4* __restrict__ buf, uint64_t nchunks,
                                                          uint64_t iters, uint64_t seed, int map, uint32_t nsm,
                                                          const uint8_t* __restrict__ die, uint4* __restrict__ sink) {
  constexpr int G = CHUNK / 16;
  const int lane = threadIdx.x & 31;
  const uint64_t gid = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) / G;
  const int k = lane % G;
  const uint32_t s = smid();
  uint32_t half = 0;
  switch (map) {
    case 1: half = s >= nsm / 2; break;
    case 2: half = s & 1; break;
    case 3: half = (s >> 1) & 1; break;
    case 4: half = (s >> 2) & 1; break;
    case 5: half = (s >> 3) & 1; break;
    case 6: half = die[s]; break;
    default: half = 0;
  }
  const uint64_t span = map ? nchunks / 2 : nchunks;
  const uint64_t off = uint64_t(half) * span;
  uint4 acc = make_uint4(0, 0, 0, 0);
  uint64_t state = mix64(gid ^ seed);
  for (uint64_t it = 0; it < iters; ++it) {
    uint4 v[UNROLL];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      state = mix64(state);
      const uint64_t c = off + __umul64hi(state, span);
      v[u] = __ldg(buf + c * G + k);
    }
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      acc.x ^= v[u].x; acc.y ^= v[u].y; acc.z ^= v[u].z; acc.w ^= v[u].w;
    }
  }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x12345678u) sink[threadIdx.x] = acc;
}

PROBE_API double probe_random_read_aff_gbs(uint64_t bytes, int chunk, int map, int reps, const uint8_t* die_host) {
  uint4* buf = nullptr;
  uint8_t* die = nullptr;
  cudaMalloc(&die, 1024);
  cudaMemset(die, 0, 1024);
  if (die_host) cudaMemcpy(die, die_host, 256, cudaMemcpyHostToDevice);
  uint4* sink = nullptr;
  if (cudaMalloc(&buf, bytes) != cudaSuccess) return -1;
  cudaMalloc(&sink, 512 * sizeof(uint4));
  cudaMemset(buf, 1, bytes);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint64_t nchunks = bytes / chunk;
  const uint64_t iters = 256;
  const unsigned grid = sms * 4;
  const unsigned threads = 512;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best_ms = 1e30f;
  for (int r = 0; r < reps + 1; ++r) {
    cudaEventRecord(a);
    if (chunk == 32) l2_random_read_aff<32, 8><<<grid, threads>>>(buf, nchunks, iters, r, map, sms, die, sink);
    else l2_random_read_aff<64, 8><<<grid, threads>>>(buf, nchunks, iters, r, map, sms, die, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    if (r > 0 && ms < best_ms) best_ms = ms;
  }
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(buf);
  cudaFree(sink);
  cudaFree(die);
  if (cudaGetLastError() != cudaSuccess) return -2;
  const double total = double(grid) * threads * iters * 8 * 16;
  return total / (best_ms * 1e-3) / 1e9;
}

// SM -> die discovery: one CTA per SM, one thread, times a dependent L2 hit to
// each of NA addresses (warm); lines homed on the far die's L2 take longer.
constexpr int kNA = 64;
__global__ void sm_latency(const uint64_t* __restrict__ buf, uint64_t stride_words, uint32_t* __restrict__ out,
                           uint32_t* __restrict__ sm_of_cta) {
  if (threadIdx.x) return;
  const uint32_t s = smid();
  sm_of_cta[blockIdx.x] = s;
  uint64_t x = 0;
  for (int rep = 0; rep < 2; ++rep) {
    for (int a = 0; a < kNA; ++a) {
      const uint64_t* p = buf + uint64_t(a) * stride_words + (x & 1);
      const long long t0 = clock64();
      uint64_t v;
      asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
      x += v;
      const long long t1 = clock64() + (long long)(x & 0);  // depends on v
      if (rep == 1) out[blockIdx.x * kNA + a] = uint32_t(t1 - t0);
    }
  }
  if (x == 12345) out[0] = 0;
}

PROBE_API int probe_sm_latency(uint32_t* host_lat, uint32_t* host_sm, int nctas) {
  uint64_t* buf = nullptr;
  uint32_t *lat = nullptr, *sm = nullptr;
  const uint64_t stride_words = 4096 / 8 + 4;  // 4 KB + 32 B apart
  cudaMalloc(&buf, kNA * stride_words * 8 + 64);
  cudaMemset(buf, 0, kNA * stride_words * 8 + 64);
  cudaMalloc(&lat, sizeof(uint32_t) * kNA * nctas);
  cudaMalloc(&sm, sizeof(uint32_t) * nctas);
  sm_latency<<<nctas, 32>>>(buf, stride_words, lat, sm);
  cudaMemcpy(host_lat, lat, sizeof(uint32_t) * kNA * nctas, cudaMemcpyDeviceToHost);
  cudaMemcpy(host_sm, sm, sizeof(uint32_t) * nctas, cudaMemcpyDeviceToHost);
  cudaFree(buf);
  cudaFree(lat);
  cudaFree(sm);
  return int(cudaGetLastError());
}

// Address -> home-die discovery: every CTA (one per SM) times a dependent L2 hit
// to each of na addresses `stride` bytes apart (second pass, warm).
__global__ void addr_latency(const uint8_t* __restrict__ buf, uint64_t stride, int na, uint16_t* __restrict__ out,
                             uint32_t* __restrict__ sm_of_cta) {
  if (threadIdx.x) return;
  sm_of_cta[blockIdx.x] = smid();
  uint64_t x = 0;
  for (int rep = 0; rep < 2; ++rep) {
    for (int a = 0; a < na; ++a) {
      const uint64_t* p = reinterpret_cast<const uint64_t*>(buf + uint64_t(a) * stride) + (x & 1);
      const long long t0 = clock64();
      uint64_t v;
      asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
      x += v;
      const long long t1 = clock64() + (long long)(x & 0);
      if (rep == 1) out[uint64_t(blockIdx.x) * na + a] = uint16_t(min(t1 - t0, 65535ll));
    }
  }
  if (x == 12345) out[0] = 0;
}

PROBE_API int probe_addr_latency(uint16_t* host_lat, uint32_t* host_sm, int nctas, uint64_t stride, int na) {
  uint8_t* buf = nullptr;
  uint16_t* lat = nullptr;
  uint32_t* sm = nullptr;
  cudaMalloc(&buf, stride * na + 64);
  cudaMemset(buf, 0, stride * na + 64);
  cudaMalloc(&lat, sizeof(uint16_t) * na * nctas);
  cudaMalloc(&sm, sizeof(uint32_t) * nctas);
  addr_latency<<<nctas, 32>>>(buf, stride, na, lat, sm);
  cudaMemcpy(host_lat, lat, sizeof(uint16_t) * na * nctas, cudaMemcpyDeviceToHost);
  cudaMemcpy(host_sm, sm, sizeof(uint32_t) * nctas, cudaMemcpyDeviceToHost);
  cudaFree(buf);
  cudaFree(lat);
  cudaFree(sm);
  return int(cudaGetLastError());
}

// Home die of every 256 B chunk of a buffer: each CTA (thread 0) touches its
// chunks once (miss) and times a second, L2-hit access; the latency compared
// with the CTA's own die says near (same die) or far.
__global__ void chunk_home(const uint8_t* __restrict__ buf, uint64_t nchunks, const uint8_t* __restrict__ die,
                           uint8_t* __restrict__ home, uint32_t thresh) {
  if (threadIdx.x) return;
  const uint32_t d = die[smid()];
  uint64_t x = 0;
  for (uint64_t c = blockIdx.x; c < nchunks; c += gridDim.x) {
    const uint64_t* p = reinterpret_cast<const uint64_t*>(buf + c * 256);
    uint64_t v;
    asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    x += v;
    const uint64_t* p2 = p + (x & 1);
    const long long t0 = clock64();
    asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p2) : "memory");
    x += v;
    const long long t1 = clock64() + (long long)(x & 0);
    const bool near = uint32_t(t1 - t0) < thresh;
    home[c] = uint8_t(near ? d : 1 - d);
  }
  if (x == 12345) home[0] = 7;
}

template <int UNROLL>
__global__ void __launch_bounds__(512) l2_random_read_home(const uint4* __restrict__ buf, uint64_t nchunks,
                                                           const uint32_t* __restrict__ homebits, int mode,
                                                           uint64_t iters, uint64_t seed, const uint8_t* __restrict__ die,
                                                           uint4* __restrict__ sink) {
  extern __shared__ uint32_t sbits[];
  const uint32_t nw = uint32_t((nchunks + 31) / 32);
  for (uint32_t i = threadIdx.x; i < nw; i += blockDim.x) sbits[i] = homebits[i];
  __syncthreads();
  const uint64_t gid = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) / 2;
  const int k = threadIdx.x & 1;
  const uint32_t want = mode == 1 ? die[smid()] : 1u - die[smid()];
  uint4 acc = make_uint4(0, 0, 0, 0);
  uint64_t state = mix64(gid ^ seed);
  for (uint64_t it = 0; it < iters; ++it) {
    uint4 v[UNROLL];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      uint64_t c;
      for (;;) {  // both lanes of the pair draw the same sequence
        state = mix64(state);
        c = __umul64hi(state, nchunks);
        if (mode == 0 || ((sbits[c >> 5] >> (c & 31)) & 1u) == want) break;
      }
      const uint32_t sec = uint32_t(state) & 7u;
      v[u] = __ldg(buf + c * 16 + sec * 2 + k);
    }
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      acc.x ^= v[u].x; acc.y ^= v[u].y; acc.z ^= v[u].z; acc.w ^= v[u].w;
    }
  }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x12345678u) sink[threadIdx.x] = acc;
}

// mode 0: both SM groups read random sectors of the whole buffer;
// mode 1: each group reads only chunks homed on its own die;
// mode 2: each group reads only chunks homed on the OTHER die.
PROBE_API double probe_affinity_read_gbs(uint64_t bytes, int mode, const uint8_t* die_host, uint32_t thresh,
                                         double* frac_home0) {
  uint8_t *buf = nullptr, *die = nullptr, *home = nullptr;
  uint4* sink = nullptr;
  const uint64_t nchunks = bytes / 256;
  if (cudaMalloc(&buf, bytes) != cudaSuccess) return -1;
  cudaMemset(buf, 1, bytes);
  cudaMalloc(&die, 256);
  cudaMemcpy(die, die_host, 256, cudaMemcpyHostToDevice);
  cudaMalloc(&home, nchunks);
  cudaMalloc(&sink, 512 * sizeof(uint4));
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  chunk_home<<<sms, 32>>>(buf, nchunks, die, home, thresh);
  uint8_t* h = new uint8_t[nchunks];
  cudaMemcpy(h, home, nchunks, cudaMemcpyDeviceToHost);
  const uint64_t nw = (nchunks + 31) / 32;
  uint32_t* hb = new uint32_t[nw]();
  uint64_t n0 = 0;
  for (uint64_t c = 0; c < nchunks; ++c) {
    n0 += h[c] == 0;
    if (h[c] == 1) hb[c >> 5] |= 1u << (c & 31);
  }
  *frac_home0 = double(n0) / double(nchunks);
  uint32_t* dl = nullptr;
  cudaMalloc(&dl, nw * 4);
  cudaMemcpy(dl, hb, nw * 4, cudaMemcpyHostToDevice);
  if (nw * 4 > 200 * 1024) return -3;
  cudaFuncSetAttribute(l2_random_read_home<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 210 * 1024);
  const uint64_t iters = 256;
  const unsigned grid = sms, threads = 512;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best_ms = 1e30f;
  for (int r = 0; r < 3; ++r) {
    cudaEventRecord(a);
    l2_random_read_home<8><<<grid, threads, nw * 4>>>((const uint4*)buf, nchunks, dl, mode, iters, r, die, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    if (r > 0 && ms < best_ms) best_ms = ms;
  }
  delete[] h;
  delete[] hb;
  cudaFree(buf);
  cudaFree(die);
  cudaFree(home);
  cudaFree(sink);
  cudaFree(dl);
  if (cudaGetLastError() != cudaSuccess) return -2;
  return double(grid) * threads * iters * 8 * 16 / (best_ms * 1e-3) / 1e9;
}

// ---- Random 64 B line gather from a DRAM-resident buffer (round-2 item-search design
// probe): how many random line reads per second the SMs sustain as a function of the
// lines in flight per SM and of how they land.
//   mode 0: a lane pair per line, one 256-bit load per lane (the item search's leaf read);
//           U lines in flight per pair.
//   mode 1: every lane issues cp.async.bulk (TMA) copies of its own lines (64 B each) into
//           a shared-memory slot; one mbarrier per warp and stage; U lines per lane.
__device__ __forceinline__ void pb_mbar_init(uint64_t* bar, uint32_t n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(uint32_t(__cvta_generic_to_shared(bar))), "r"(n));
}
__device__ __forceinline__ void pb_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(uint32_t(__cvta_generic_to_shared(bar))),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void pb_bulk(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          uint32_t(__cvta_generic_to_shared(dst))),
      "l"(src), "r"(bytes), "r"(uint32_t(__cvta_generic_to_shared(bar)))
      : "memory");
}
__device__ __forceinline__ void pb_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}\n" ::"r"(
          uint32_t(__cvta_generic_to_shared(bar))),
      "r"(parity)
      : "memory");
}

// wlines > 0: every line of iteration `it` lies in the window of wlines lines starting at
// (it * wlines) mod nlines (all SMs move through the buffer window by window: locality
// at the DRAM-row / L2 level, not within a warp)
template <int U>
__global__ void gather64_ldg(const uint8_t* __restrict__ buf, uint64_t nlines, uint64_t iters, uint64_t seed,
                             uint64_t* __restrict__ sink, uint64_t wlines = 0) {
  const int lane = threadIdx.x & 31, k = lane & 1;
  const uint64_t gid = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 1;
  uint64_t state = mix64(gid ^ seed), acc = 0;
  for (uint64_t it = 0; it < iters; ++it) {
    unsigned long long v[U][4];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      state = mix64(state);
      const uint64_t line = wlines ? ((it * wlines) % (nlines - wlines + 1)) + __umul64hi(state, wlines)
                                   : __umul64hi(state, nlines);
      const uint8_t* p = buf + line * 64 + k * 32;
      asm volatile("ld.global.nc.v4.u64 {%0, %1, %2, %3}, [%4];"
                   : "=l"(v[u][0]), "=l"(v[u][1]), "=l"(v[u][2]), "=l"(v[u][3])
                   : "l"(p));
    }
#pragma unroll
    for (int u = 0; u < U; ++u) acc ^= v[u][0] ^ v[u][1] ^ v[u][2] ^ v[u][3];
  }
  if (acc == 0x1234567890ull) sink[threadIdx.x] = acc;
}

template <int U>
__global__ void gather64_tma(const uint8_t* __restrict__ buf, uint64_t nlines, uint64_t iters, uint64_t seed,
                             uint64_t* __restrict__ sink) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint64_t bars[32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint8_t* slot = smem + (size_t(threadIdx.x) * U) * 64;
  if (lane == 0) pb_mbar_init(&bars[wid], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
  uint64_t state = mix64((uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) ^ seed), acc = 0;
  uint32_t parity = 0;
  for (uint64_t it = 0; it < iters; ++it) {
    if (lane == 0) pb_expect_tx(&bars[wid], 32u * U * 64u);
    __syncwarp();
#pragma unroll
    for (int u = 0; u < U; ++u) {
      state = mix64(state);
      pb_bulk(slot + u * 64, buf + __umul64hi(state, nlines) * 64, 64, &bars[wid]);
    }
    pb_wait(&bars[wid], parity);
    parity ^= 1u;
#pragma unroll
    for (int u = 0; u < U; ++u) acc ^= *reinterpret_cast<const uint64_t*>(slot + u * 64 + (lane & 7) * 8);
    __syncwarp();
  }
  if (acc == 0x1234567890ull) sink[threadIdx.x] = acc;
}

// Returns random 64 B lines per second (G lines/s) over a `bytes` buffer.
PROBE_API double probe_gather64(uint64_t bytes, int mode, int u, int threads, int ctas_per_sm, int reps) {
  uint8_t* buf = nullptr;
  uint64_t* sink = nullptr;
  if (cudaMalloc(&buf, bytes) != cudaSuccess) return -1;
  cudaMalloc(&sink, 1024 * 8);
  cudaMemset(buf, 1, bytes);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint64_t nlines = bytes / 64, iters = 64;
  const unsigned grid = sms * ctas_per_sm;
  const size_t smem = mode == 1 ? size_t(threads) * u * 64 : 0;
  auto launch = [&](int r) {
    if (mode == 0) {
      switch (u) {
        case 1: gather64_ldg<1><<<grid, threads>>>(buf, nlines, iters, r, sink); break;
        case 2: gather64_ldg<2><<<grid, threads>>>(buf, nlines, iters, r, sink); break;
        case 4: gather64_ldg<4><<<grid, threads>>>(buf, nlines, iters, r, sink); break;
        default: gather64_ldg<8><<<grid, threads>>>(buf, nlines, iters, r, sink); break;
      }
    } else {
      switch (u) {
        case 1: cudaFuncSetAttribute(gather64_tma<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
                gather64_tma<1><<<grid, threads, smem>>>(buf, nlines, iters, r, sink); break;
        case 2: cudaFuncSetAttribute(gather64_tma<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
                gather64_tma<2><<<grid, threads, smem>>>(buf, nlines, iters, r, sink); break;
        case 4: cudaFuncSetAttribute(gather64_tma<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
                gather64_tma<4><<<grid, threads, smem>>>(buf, nlines, iters, r, sink); break;
        default: cudaFuncSetAttribute(gather64_tma<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
                gather64_tma<8><<<grid, threads, smem>>>(buf, nlines, iters, r, sink); break;
      }
    }
  };
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best_ms = 1e30f;
  for (int r = 0; r < reps + 1; ++r) {
    cudaEventRecord(a);
    launch(r);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    if (r > 0 && ms < best_ms) best_ms = ms;
  }
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(buf);
  cudaFree(sink);
  if (cudaGetLastError() != cudaSuccess) return -2;
  const double lines = mode == 0 ? double(grid) * threads / 2 * iters * u : double(grid) * threads * iters * u;
  return lines / (best_ms * 1e-3) / 1e9;
}

// The windowed form of probe_gather64 mode 0 (u = 2, 1024 threads, 1 CTA per SM): G lines/s.
PROBE_API double probe_gather64_window(uint64_t bytes, uint64_t window_bytes, int reps) {
  uint8_t* buf = nullptr;
  uint64_t* sink = nullptr;
  if (cudaMalloc(&buf, bytes) != cudaSuccess) return -1;
  cudaMalloc(&sink, 1024 * 8);
  cudaMemset(buf, 1, bytes);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint64_t nlines = bytes / 64, iters = 64, wl = window_bytes / 64;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best_ms = 1e30f;
  for (int r = 0; r < reps + 1; ++r) {
    cudaEventRecord(a);
    gather64_ldg<2><<<sms, 1024>>>(buf, nlines, iters, r, sink, wl);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    if (r > 0 && ms < best_ms) best_ms = ms;
  }
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(buf);
  cudaFree(sink);
  if (cudaGetLastError() != cudaSuccess) return -2;
  return double(sms) * 1024 / 2 * iters * 2 / (best_ms * 1e-3) / 1e9;
}
