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
