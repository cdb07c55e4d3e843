// range.cu — hbt_range: range scans ("search for the first key in
// the range and then traverse leaf nodes until the last key is found"; the
// paper's range-query experiment, returns 1..32 keys per query).
//
// Step 1 is the tree's own lower-bound search of the range start (the hot
// path).  Step 2: one warp per query walks forward 32 entries at a time —
// implicit: consecutive ranks of the contiguous L-segment ("leaf nodes
// are arranged sequentially"); regular: the entries of big leaf v, then the next
// big leaf in key order (the chain, the paper's linked leaves).  Keys are sorted,
// so the entries <= hi form a prefix of each chunk: popc(ballot(key <= hi)).
#include "hbt_internal.cuh"

namespace hbt {
namespace {

constexpr uint64_t kEnd = HBT_POS_END;

template <typename K>
__device__ __forceinline__ K key_max() { return K(~K(0)); }

// L lanes per query (L = next power of two >= min(k, 32)), 32/L queries per warp;
// every sub-group walks its own query, chunk by chunk, until done or k reached.
template <typename K>
__global__ void range_implicit(const K* __restrict__ leaf, uint64_t n, const uint64_t* __restrict__ pf,
                               const K* __restrict__ hi, uint64_t m, uint32_t k, uint32_t L, K* __restrict__ ok,
                               K* __restrict__ ov, uint32_t* __restrict__ oc) {
  constexpr uint32_t P = 64 / (2 * sizeof(K));
  const uint32_t lane = threadIdx.x & 31, sub = lane % L, grp = lane / L, QW = 32 / L;
  const unsigned gmask = (L == 32 ? 0xffffffffu : ((1u << L) - 1u)) << (grp * L);
  const uint64_t w0 = (blockIdx.x * uint64_t(blockDim.x) + threadIdx.x) >> 5;
  const uint64_t nw = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  for (uint64_t xb = w0 * QW; xb < m; xb += nw * QW) {
    const uint64_t x = xb + grp;
    const bool live = x < m;
    const uint64_t r0 = live ? (pf[x] & kEnd) : kEnd;
    const K h = live ? hi[x] : K(0);
    uint32_t c = 0;
    bool done = (r0 == kEnd);
    for (uint32_t base = 0; base < k; base += L) {
      const uint32_t i = base + sub;
      bool valid = false;
      K key = key_max<K>(), val = K(0);
      if (!done && i < k) {
        const uint64_t r = r0 + i;
        if (r < n) {
          key = leaf[(r / P) * (2 * P) + r % P];
          val = leaf[(r / P) * (2 * P) + P + r % P];
          valid = key <= h;
        }
      }
      const unsigned b = __ballot_sync(0xffffffffu, valid) & gmask;
      if (live && i < k) {
        ok[x * k + i] = valid ? key : key_max<K>();
        ov[x * k + i] = valid ? val : K(0);
      }
      c += __popc(b);
      if (b != gmask) done = true;
    }
    if (live && sub == 0) oc[x] = c;
  }
}

template <typename K>
__global__ void range_regular(const K* __restrict__ leaf, const uint32_t* __restrict__ count,
                              const uint32_t* __restrict__ chain, const uint32_t* __restrict__ chainpos,
                              uint64_t nchain, uint32_t F, const uint64_t* __restrict__ pf,
                              const K* __restrict__ hi, uint64_t m, uint32_t k, uint32_t L, K* __restrict__ ok,
                              K* __restrict__ ov, uint32_t* __restrict__ oc) {
  constexpr uint32_t P = 64 / (2 * sizeof(K));
  const uint64_t FP = uint64_t(F) * P;
  const uint32_t lane = threadIdx.x & 31, sub = lane % L, grp = lane / L, QW = 32 / L;
  const unsigned gmask = (L == 32 ? 0xffffffffu : ((1u << L) - 1u)) << (grp * L);
  const uint64_t w0 = (blockIdx.x * uint64_t(blockDim.x) + threadIdx.x) >> 5;
  const uint64_t nw = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  for (uint64_t xb = w0 * QW; xb < m; xb += nw * QW) {
    const uint64_t x = xb + grp;
    const bool live = x < m;
    const uint64_t pos = live ? (pf[x] & kEnd) : kEnd;
    const K h = live ? hi[x] : K(0);
    if (live)
      for (uint32_t i = sub; i < k; i += L) {
        ok[x * k + i] = key_max<K>();
        ov[x * k + i] = K(0);
      }
    uint32_t c = 0;
    bool active = pos != kEnd;
    uint64_t v = active ? pos / FP : 0, ci = active ? chainpos[v] : 0;
    uint32_t e = active ? uint32_t(pos % FP) : 0;  // dense packing: line j slot s = entry j*P + s
    while (__any_sync(0xffffffffu, active)) {
      uint32_t take = 0;
      bool valid = false;
      K key = key_max<K>(), val = K(0);
      if (active) {
        const uint32_t cnt = count[v];
        const uint32_t take0 = cnt - e < L ? cnt - e : L;
        take = take0 < k - c ? take0 : k - c;
        if (sub < take) {
          const uint32_t en = e + sub;
          key = leaf[(v * F + en / P) * (2 * P) + en % P];
          val = leaf[(v * F + en / P) * (2 * P) + P + en % P];
          valid = key <= h;
        }
      }
      const unsigned b = __ballot_sync(0xffffffffu, valid) & gmask;
      if (active) {
        if (valid) {
          ok[x * k + c + sub] = key;
          ov[x * k + c + sub] = val;
        }
        const uint32_t got = __popc(b);
        c += got;
        e += take;
        if (got < take || c >= k) {
          active = false;                    // passed hi, or k reached
        } else if (e >= count[v]) {          // next big leaf in key order
          if (++ci >= nchain) active = false;
          else { v = chain[ci]; e = 0; }
        }
      }
    }
    if (live && sub == 0) oc[x] = c;
  }
}

inline unsigned warps_grid(uint64_t m, uint32_t L) {
  const uint64_t warps = (m + 32 / L - 1) / (32 / L);
  uint64_t g = (warps + 7) / 8;  // 8 warps per 256-thread block
  if (g > 148 * 32) g = 148 * 32;
  return unsigned(g ? g : 1);
}

template <typename K>
int range_t(hbt_tree* t, const void* lo, const void* hi, uint64_t m, uint32_t k, void* ok, void* ov, uint32_t* oc,
            cudaStream_t s) {
  // lower bounds of the range starts in per-call scratch from the stream-ordered pool:
  // concurrent range scans on other streams each get their own
  void* buf = nullptr;
  const uint64_t off_v = (m * 8 + 255) & ~uint64_t(255);
  HBT_CUDA_TRY(scratch_alloc(&buf, off_v + m * sizeof(K), s));
  uint64_t* rpf = static_cast<uint64_t*>(buf);
  K* rv = reinterpret_cast<K*>(static_cast<uint8_t*>(buf) + off_v);
  int rc = t->form == HBT_REGULAR ? regular_search(t, lo, m, rpf, rv, s) : implicit_search(t, lo, m, rpf, rv, s);
  if (rc) {
    scratch_free(buf, s);
    return rc;
  }
  uint32_t L = 1;
  while (L < k && L < 32) L <<= 1;
  if (t->form == HBT_REGULAR) {
    const RegularState& r = t->r;
    range_regular<K><<<warps_grid(m, L), 256, 0, s>>>((const K*)r.d_leaf, r.d_count, r.d_chain, r.d_chainpos,
                                                      r.nchain, t->F, rpf, (const K*)hi, m, k, L, (K*)ok,
                                                      (K*)ov, oc);
  } else {
    range_implicit<K><<<warps_grid(m, L), 256, 0, s>>>((const K*)t->d_leaf, t->n, rpf, (const K*)hi, m, k, L,
                                                       (K*)ok, (K*)ov, oc);
  }
  const cudaError_t e = cudaGetLastError();
  scratch_free(buf, s);
  if (e != cudaSuccess) {
    set_error("range scan launch: %s", cudaGetErrorString(e));
    return HBT_ECUDA;
  }
  return HBT_OK;
}

}  // namespace

void range_free(hbt_tree*) {}

int range_scan(const hbt_tree* tc, const void* lo, const void* hi, uint64_t m, uint32_t k, void* ok, void* ov,
               uint32_t* oc, cudaStream_t s) {
  hbt_tree* t = const_cast<hbt_tree*>(tc);
  return t->width == 4 ? range_t<uint32_t>(t, lo, hi, m, k, ok, ov, oc, s) : range_t<uint64_t>(t, lo, hi, m, k, ok, ov, oc, s);
}

}  // namespace hbt
