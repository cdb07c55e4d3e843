// block_util.cuh — CTA-level helpers shared by the bucketing kernels (bucketed.cu)
// and the item searches (implicit_search.cu): 1D bulk copies global -> shared
// memory (cp.async.bulk, the TMA unit's non-tensor form) completing on an
// mbarrier, and an exclusive block scan.
#pragma once

#include <stdint.h>

namespace hbt {

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return uint32_t(__cvta_generic_to_shared(p)); }

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      " .reg .pred p;\n"
      "WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// bytes: a multiple of 16, src and dst 16 B aligned.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
// Orders this CTA's earlier generic-proxy shared-memory accesses before later
// async-proxy (bulk copy) writes to the same bytes.
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

// Exclusive scan of s_in[0, B) into s_out (B <= 2 * TH) by one CTA of TH threads:
// two elements per thread, a shuffle scan per warp, the warp totals (s_tmp, TH / 32
// entries) scanned by warp 0.  In place is allowed.  Ends with a barrier.
template <int TH>
__device__ __forceinline__ void block_exclusive_scan(const uint32_t* s_in, uint32_t* s_out, uint32_t B,
                                                     uint32_t* s_tmp) {
  const uint32_t t = threadIdx.x, lane = t & 31, wid = t >> 5;
  const uint32_t a = 2 * t < B ? s_in[2 * t] : 0u, b = 2 * t + 1 < B ? s_in[2 * t + 1] : 0u;
  uint32_t x = a + b;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= uint32_t(o)) x += y;
  }
  if (lane == 31) s_tmp[wid] = x;
  __syncthreads();
  if (wid == 0) {
    uint32_t w = lane < uint32_t(TH / 32) ? s_tmp[lane] : 0u;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, w, o);
      if (lane >= uint32_t(o)) w += y;
    }
    if (lane < uint32_t(TH / 32)) s_tmp[lane] = w;
  }
  __syncthreads();
  const uint32_t ex = x - (a + b) + (wid ? s_tmp[wid - 1] : 0u);
  if (2 * t < B) s_out[2 * t] = ex;
  if (2 * t + 1 < B) s_out[2 * t + 1] = ex + a;
  __syncthreads();
}

}  // namespace hbt
