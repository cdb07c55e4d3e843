// gen/gen.cu — device twin of gen/__init__.py's integer streams (libhbtgen.so).
// Counter-based, so every element is a pure function of (index, seed): the
// device and numpy generators produce identical arrays (tests/test_gpu_gen.py).
// Holds no arithmetic of the method (no sort, no tree, no search).
#include <cuda_runtime.h>
#include <stdint.h>

#define HBTGEN_API extern "C" __attribute__((visibility("default")))

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__device__ __forceinline__ uint32_t fmix32(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85EBCA6Bu;
  h ^= h >> 13;
  h *= 0xC2B2AE35u;
  h ^= h >> 16;
  return h;
}

// K_i = mixS(i ^ seed)
template <typename K>
__device__ __forceinline__ K mix_stream(uint64_t i, uint64_t seed);
template <>
__device__ __forceinline__ uint64_t mix_stream<uint64_t>(uint64_t i, uint64_t seed) { return mix64(i ^ seed); }
template <>
__device__ __forceinline__ uint32_t mix_stream<uint32_t>(uint64_t i, uint64_t seed) {
  return fmix32(uint32_t(i ^ seed));
}

template <typename K>
__global__ void k_mix_stream(K* out, uint64_t start, uint64_t n, uint64_t seed) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
    out[i] = mix_stream<K>(start + i, seed);
}

// q_j = K_u with u = mulhi64(mix64(j ^ seed_q), range) and K_u = mixS(u ^ seed_k)
template <typename K>
__global__ void k_uniform_queries(K* out, uint64_t start, uint64_t m, uint64_t range, uint64_t seed_q,
                                  uint64_t seed_k) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < m; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t u = __umul64hi(mix64((start + i) ^ seed_q), range);
    out[i] = mix_stream<K>(u, seed_k);
  }
}

__device__ __forceinline__ uint64_t strat(uint64_t i, uint64_t seed) {
  return (i << 33) | (mix64(i ^ seed) & ((1ull << 33) - 1));
}

__global__ void k_stratified(uint64_t* out, uint64_t start, uint64_t n, uint64_t seed) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
    out[i] = strat(start + i, seed);
}

__global__ void k_stratified_queries(uint64_t* out, uint64_t start, uint64_t m, uint64_t range, uint64_t seed_q,
                                     uint64_t seed_k) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < m; i += uint64_t(gridDim.x) * blockDim.x)
    out[i] = strat(__umul64hi(mix64((start + i) ^ seed_q), range), seed_k);
}

static unsigned grid_for(uint64_t n) {
  uint64_t g = (n + 255) / 256;
  if (g > 148 * 32) g = 148 * 32;
  return unsigned(g ? g : 1);
}

HBTGEN_API int hbtgen_mix_stream(void* out, uint64_t start, uint64_t n, uint32_t width, uint64_t seed, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  if (width == 8) k_mix_stream<uint64_t><<<grid_for(n), 256, 0, s>>>((uint64_t*)out, start, n, seed);
  else k_mix_stream<uint32_t><<<grid_for(n), 256, 0, s>>>((uint32_t*)out, start, n, seed);
  return int(cudaGetLastError());
}

HBTGEN_API int hbtgen_uniform_queries(void* out, uint64_t start, uint64_t m, uint64_t range, uint32_t width,
                                      uint64_t seed_q, uint64_t seed_k, void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  if (width == 8)
    k_uniform_queries<uint64_t><<<grid_for(m), 256, 0, s>>>((uint64_t*)out, start, m, range, seed_q, seed_k);
  else
    k_uniform_queries<uint32_t><<<grid_for(m), 256, 0, s>>>((uint32_t*)out, start, m, range, seed_q, seed_k);
  return int(cudaGetLastError());
}

HBTGEN_API int hbtgen_stratified_keys(uint64_t* out, uint64_t start, uint64_t n, uint64_t seed, void* stream) {
  k_stratified<<<grid_for(n), 256, 0, (cudaStream_t)stream>>>(out, start, n, seed);
  return int(cudaGetLastError());
}

HBTGEN_API int hbtgen_stratified_queries(uint64_t* out, uint64_t start, uint64_t m, uint64_t range, uint64_t seed_q,
                                         uint64_t seed_k, void* stream) {
  k_stratified_queries<<<grid_for(m), 256, 0, (cudaStream_t)stream>>>(out, start, m, range, seed_q, seed_k);
  return int(cudaGetLastError());
}
