// hbt_internal.cuh — shared internals of libhbt.so (the CUDA path).
// Nothing here is shared with oracle/ (test infrastructure); see DESIGN.md §4.
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>
#include <nvtx3/nvToolsExt.h>
#include <stdint.h>

#include <mutex>
#include <string>

#include "../../include/hbt.h"

namespace hbt {

void set_error(const char* fmt, ...);

#define HBT_CUDA_TRY(expr)                                                              \
  do {                                                                                  \
    cudaError_t _e = (expr);                                                            \
    if (_e != cudaSuccess) {                                                            \
      ::hbt::set_error("%s:%d %s: %s", __FILE__, __LINE__, #expr, cudaGetErrorString(_e)); \
      return _e == cudaErrorMemoryAllocation ? HBT_ENOMEM : HBT_ECUDA;                  \
    }                                                                                   \
  } while (0)

static inline uint64_t ceil_div_u64(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

// NVTX range around a host-side phase (build, search, update, exchange steps): shows
// up in nsys / ncu --nvtx timelines; free when no tool is attached (NVTX v3 is
// header-only and does nothing until a tool injects itself).
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange&) = delete;
  NvtxRange& operator=(const NvtxRange&) = delete;
};

// Scratch of builds and updates comes from the device's stream-ordered pool
// (cudaMallocAsync): after the first use, repeated updates allocate without
// cudaMalloc / cudaFree (which synchronise the device).  The pool keeps up to
// a quarter of the device between calls (api.cu sets the release threshold once).
cudaError_t scratch_alloc(void** p, size_t bytes, cudaStream_t s);
void scratch_free(void* p, cudaStream_t s);

// Level table passed by value to the search kernels (root-first, node units).
struct LevelTable {
  uint64_t offset[HBT_MAX_LEVELS + 1];
  uint32_t H;   // inner levels
  uint32_t SL;  // first level walked by lane groups (the directory level T, or the item directory's level)
  uint32_t dcount;  // nodes at level T (directory entries)
  uint32_t dbits;   // directory prefix bits
  uint32_t full_mask;  // bit d: read level d's nodes whole (not index + sector)
  uint32_t leaf256;    // leaf line read as one 64 B request (two 256-bit lane loads)
  uint32_t full256;    // whole-node levels read by 256-bit lane loads (half the load instructions)
  uint32_t l2_hint;    // bit 0: leaf lines loaded L2::evict_first; bit 1: whole-node levels L2::evict_last
};

// Search / bucketing configuration of one tree (hbt_set_param, include/hbt.h).  Results
// never depend on it.  Variants measured slower in round 1 and 2 were removed; their
// numbers stay in DESIGN.md §8.
struct SearchConfig {
  uint32_t ctas_per_sm = 0;      // 0 = occupancy-derived
  uint32_t mode = 2;             // implicit directory: 2 = staged in shared memory, 3 = read in place
  uint64_t small_batch = 1u << 16;  // mode 2: batches up to this size read the directory in place (mode 3)
  uint64_t l2_levels_bytes = 0;  // L2-resident budget for index+sector levels (0 = default 32 MB)
  uint32_t full_levels = 0;      // implicit: bit d = read level d's nodes whole (0 = by the L2 budget)
  uint32_t exchange = 0;         // sharded search: 0 = fused peer-memory exchange, 1 = NCCL send/recv
  uint32_t exchange_chunks = 1;  // fused exchange: chunks per batch (the put of chunk c+1 overlaps the owner
                                 // search of chunk c on a second stream); every rank of a communicator must
                                 // use the same value.  1 by default: with the ranks sharing one GPU (the only
                                 // multi-rank setup measured) 2 / 3 chunks ran 11.6 -> 10.3 / 9.5 G q/s
  uint32_t g1_direct = 1;        // sharded search with ONE shard: search directly (no route / exchange)
  uint32_t bucket = 2;           // query bucketing (bucketed.cu): 0 = off, 1 = on, 2 = auto
  uint64_t bucket_slice = 0;     // tree bytes per bucket (0 = default 1 MB)
  uint32_t bucket_items = 1;     // bucketed search: bucket-local shared-memory directory (ItemDir)
  uint32_t bucket_cap = 0;       // item directory: shared-memory entries (0 = derived; tests force the fallback)
  uint32_t item_rounds = 0;      // item searches: most warp rounds per work item (0 = 16)
  uint32_t scatter_tma = 1;      // bucketed scatter: inputs streamed into shared memory by bulk copies (1)
  uint32_t phase_timing = 0;     // bucketed search: CUDA events around each phase (hbt_last_phases)
  uint32_t leaf_stream = 2;      // host L-segment: 0 = zero-copy leaf reads, 1 = stream bucket slices
                                 // into HBM (bucketed, double-buffered copies), 2 = auto (by batch size)
  uint64_t stream_slice = 0;     // host L-segment bytes per streamed bucket (0 = 8 MB)
  uint32_t host_chunk_log2 = 20;  // hbt_search_host: queries per pipeline bucket (log2; c2 e2e 2.78 -> 3.00 G q/s vs 2^22)
  uint32_t host_bufs = 2;        // hbt_search_host: (stream, buffer) pairs in flight (2..4)
  uint32_t leaf256 = 1;          // leaf line by two 256-bit lane loads (one 64 B request per group)
  uint32_t full256 = 1;          // implicit whole-node levels by 256-bit lane loads
  uint32_t l2_hint = 4;          // implicit search: L2 eviction-priority hints (LevelTable::l2_hint);
                                 // 4 = auto: leaf lines evict-first iff the I-segment fits in L2 / 4
  uint32_t item_l2_hint = 1;     // implicit bucketed item search (c4 item search 10.96 -> 9.50 ms)
  uint32_t item_qpf = 1;         // see ItemDir::qpf
  uint32_t item_cnode = 1;       // compact 32 B directory-level nodes (u64, F = 16): 0 = off, 1 = when that level
                                 // is read as whole nodes (beyond the L2 budget), 2 = always
  uint32_t item_cdir = 1;        // item directory in the compressed per-bucket form (ItemDir::bd): 0 = never,
                                 // 1 = where it reaches a deeper level (regular: always fits-permitting),
                                 // 2 = always (implicit: even at the same level)
};

// Bucket-local directory of the bucketed search (bucketed.cu): after the
// partition, the queries of a work item (kItem consecutive bucketed queries)
// fall in the key range of a few consecutive buckets, so the item stages the
// maxima of that range's UNITS into shared memory and finds each query's unit
// by one lower bound there, skipping every level above it.
//   implicit: unit = node of level `level` (level H = leaf lines), M[j] = max
//             key below node j; the search continues at that level.
//   regular:  unit = key line t of the last-level node of chain leaf c
//             (entry c*span + t), M = its true max key; chain[c] = the leaf.
struct ItemDir {
  const void* M = nullptr;
  const uint32_t* chain = nullptr;  // regular: chain ids
  const uint64_t* bstart = nullptr; // B + 1 bucket starts in the bucketed order (bstart[B] = m)
  uint32_t B = 0;
  uint64_t U = 0;      // splitter units (implicit: leaf lines, regular: chain leaves)
  uint32_t level = 0;  // implicit: level of the directory units
  uint64_t span = 1;   // implicit: leaf lines per unit; regular: entries per chain leaf
  uint64_t nunits = 0; // entries of M
  uint32_t cap = 0;    // shared-memory entries (larger ranges search M in global memory)
  uint64_t pos_base = 0;  // implicit: added to every reported position (key-range shards)
  uint32_t rounds = 16;   // warp rounds per work item (fewer for small batches: every SM gets items)
  // Compressed per-bucket directory (implicit trees whose directory level has too many
  // units per bucket for 8 B keys in shared memory; regular trees: the leaf lines of the
  // chain leaves): with M' = (M - bd[b].lo) >> bd[b].sh (32 bits), a prefix table over
  // 2^12 slices T16[b * kT16 + p] = #{M' < p << ssh} and 16-bit entries
  // E16[bd[b].off16 + i] = (M'_i >> esh) & 0xFFFF; items are cut inside one bucket
  // (item search).
  const struct BucketDir* bd = nullptr;
  const uint16_t* E16 = nullptr;
  const uint16_t* T16 = nullptr;
  bool fix = false;  // single ties of the truncated maxima resolved by the walk
  // compact 32 B copies of the directory level's nodes (u64 keys, F = 16; bk_cnode): u32
  // M'(sep_0) + 14 u16 (M'(sep_i) - M'(sep_0)) >> nsh (0xFFFF = MAX slot); null = off
  const uint8_t* cnode = nullptr;
  uint32_t qpf = 0;  // compressed-directory items: each lane prefetches its query qpf rounds after the next into
                     // the L2 (0 = off; 1 measured best, 2-4 slower: profiles/r02s_item_query_prefetch_ab.jsonl)
};

constexpr uint32_t kT16 = 4104;  // per-bucket prefix table: 2^12 + 1 entries, padded to 16 B

// One bucket of the compressed item directory (ItemDir::bd).
struct BucketDir {
  uint64_t u0;     // first directory unit of the bucket
  uint64_t off16;  // its first entry in E16 (a multiple of 8: 16 B aligned bulk copies)
  uint64_t lo;     // M[u0]: the offset origin
  uint32_t cnt;    // units u0 .. u0 + cnt - 1 (< 2^16)
  uint32_t sh;     // right shift that makes M[u0 + cnt - 1] - lo fit 32 bits
  uint32_t top;    // (M[u0 + cnt - 1] - lo) >> sh
  uint32_t ssh;    // prefix-table slice p holds M' in [p << ssh, (p + 1) << ssh)
  uint32_t esh;    // entry = (M' >> esh) & 0xFFFF (ssh - 16, or 0)
  uint32_t nsh;    // compact directory-level nodes (ItemDir::cnode): entry = (M'(sep) - M'(sep_0)) >> nsh
};

// Owner side of the fused sharded exchange (sharded_fused.cu): the bucketed search's
// gather stores each received query's result straight into the REQUESTER's result
// window (mapped peer memory).  Receive slot j of source s (s = org[j] >> 40) goes to
// slot j - start[s] + dst[s] there: the owner's run of s's queries comes back as ONE
// contiguous run (coalesced peer stores); the requester maps it to query order.
constexpr int kRemoteOrgShift = 40;  // org = (source rank << 40) | index at the source
struct RemoteOut {
  const uint64_t* org = nullptr;  // per received query (receive-window order)
  uint64_t* pf[64] = {};          // per source rank: its result window
  uint8_t* v[64] = {};
  uint64_t start[64] = {};        // per source: first slot of its run in the owner's window
  uint64_t dst[64] = {};          // per source: where this owner's results start in its window
};

// Query-bucketing state (bucketed.cu): B splitter keys and a prefix directory,
// derived from the tree on first use and after every update.
struct BucketState {
  bool valid = false;
  uint32_t B = 0;
  void* d_sp = nullptr;          // B keys
  uint32_t* d_dir = nullptr;     // 2^12 x (u16 lo, u16 hi)
  void* d_M = nullptr;           // item-directory unit maxima (ItemDir::M)
  uint64_t M_cap = 0;            // bytes allocated
  uint32_t level = 0;            // implicit: directory level
  uint64_t span = 1, nunits = 0;
  bool items = false;            // the item directory is in use
  bool cdir = false;             // ... in its compressed per-bucket form (ItemDir::bd)
  void* d_bd = nullptr;          // B x BucketDir
  uint16_t* d_E16 = nullptr;     // entries | prefix tables
  uint16_t* d_T16 = nullptr;
  uint64_t E16_cap = 0;          // bytes allocated
  uint32_t cap16 = 0;            // largest bucket's unit count, rounded up to 8
  uint8_t* d_cnode = nullptr;    // compact directory-level nodes (ItemDir::cnode), 32 B per unit
  uint64_t cnode_cap = 0;        // bytes allocated
  bool cnode = false;            // in use
  cudaEvent_t ev[6] = {};        // phase boundaries of the last timed bucketed search
  bool timed = false;
  uint32_t launches = 0;
  // streamed host L-segment (bucketed.cu, streamed_t): two HBM staging slots for
  // bucket leaf slices, a copy stream and the events that order slot reuse
  void* d_stage[2] = {};
  uint64_t stage_cap = 0;
  cudaStream_t cs = nullptr;
  cudaEvent_t ev_copy[2] = {}, ev_done[2] = {};
};

// Regular-tree device state.  All pools are SoA arrays
// indexed by pool index (node fragmentation).
struct RegularState {
  uint32_t kpl = 0, NI = 0, B = 0, b = 0;
  uint64_t pool = 0, cap = 0;            // big leaves allocated / capacity
  void* d_leaf = nullptr;                // cap x F lines x 64 B (device alias of h_leaf when on the host)
  void* h_leaf = nullptr;                // pinned mapped host pool (hbt_set_leaf_placement), else NULL
  uint32_t* d_count = nullptr;           // cap
  void* d_lkeys = nullptr;               // cap x F keys (last-level inner node)
  void* d_lidx = nullptr;                // cap x NIP index entries (padded to 32 B)
  uint64_t nchain = 0;
  uint32_t* d_chain = nullptr;           // cap
  uint32_t U = 0;                        // upper levels
  uint64_t unodes[HBT_MAX_LEVELS] = {};  // bottom-up
  uint64_t uoff[HBT_MAX_LEVELS + 1] = {};
  uint64_t ucap = 0;
  void* d_ukeys = nullptr;               // ucap x F keys
  void* d_uidx = nullptr;                // ucap x NIP
  uint32_t* d_urefs = nullptr;           // ucap x F
  uint32_t* d_seg_of_leaf = nullptr;     // pool-sized: leaf -> update segment (0xFFFFFFFF = none)
  uint64_t seg_cap = 0;
  uint32_t root_leaf = 0;                // chain[0] (the root when U == 0)
  // directory over root-first level T (search mode 2), rebuilt with the upper levels:
  // d_dir = [M_T: dir_count keys | 2^dir_bits x (u16 lo, u16 hi)]
  void* d_dir = nullptr;
  uint64_t dir_bytes = 0, dir_cap = 0;
  uint32_t dir_T = 0, dir_count = 0, dir_bits = 0;
  uint32_t* d_chainpos = nullptr;        // pool-sized: big leaf -> position in the chain (range scans)
  uint64_t chainpos_cap = 0;
};

constexpr int kHostBufs = 4;  // most (stream, buffer) pairs of the host pipeline
struct HostPipe {
  std::mutex mu;
  void* d_q = nullptr;                   // nbuf x chunk queries
  uint64_t* d_pf = nullptr;              // nbuf x chunk
  void* d_v = nullptr;                   // nbuf x chunk
  uint64_t chunk = 0;
  int nbuf = 0;
  cudaStream_t s[kHostBufs] = {};
  cudaEvent_t ev[kHostBufs] = {};
};

// Key-range shard metadata (sharded.cu): shard g holds global ranks
// [base[g], base[g] + count[g]) with largest key max[g].
struct ShardMeta {
  int G = 0;
  int rank = 0;
  ::hbt_comm* comm = nullptr;  // NULL for single-process (virtual) shard groups
  uint64_t count[64] = {};
  uint64_t base[64] = {};
  uint64_t max[64] = {};
};

// Per-tree scratch of the sharded search (grown on demand).
struct Scratch {
  uint8_t* dest = nullptr; uint64_t dest_cap = 0;
  uint8_t* send_q = nullptr; uint64_t send_cap = 0;      // elements of S bytes
  uint32_t* origin = nullptr; uint64_t origin_cap = 0;
  uint8_t* recv_q = nullptr; uint64_t recv_cap = 0;
  uint64_t* res_pf = nullptr; uint64_t res_pf_cap = 0;   // receive order
  uint8_t* res_v = nullptr; uint64_t res_v_cap = 0;
  uint64_t* back_pf = nullptr; uint64_t back_pf_cap = 0; // send order
  uint8_t* back_v = nullptr; uint64_t back_v_cap = 0;
  unsigned long long* counts = nullptr;                  // 2 x 64
};

}  // namespace hbt

struct hbt_comm {
  ncclComm_t comm = nullptr;          // NULL for a host-callback communicator
  int nranks = 1;
  int rank = 0;
  hbt_allgather_fn host_allgather = nullptr;  // host all-gather (hbt_comm_init_host)
  void* host_ctx = nullptr;
};

namespace hbt {
// All-gather `bytes` of host memory from every rank into recv (rank order),
// through the host callback if the communicator has one, else through NCCL.
int comm_allgather_host(hbt_comm* c, const void* send, void* recv, uint64_t bytes, cudaStream_t st);
}  // namespace hbt

struct hbt_tree {
  uint32_t form = HBT_IMPLICIT;  // HBT_IMPLICIT | HBT_REGULAR
  uint32_t width = 8;            // S
  uint32_t F = 16;
  uint32_t P = 4;                // 64 / (2S)
  uint64_t n = 0;                // n' distinct keys
  int device = 0;
  int num_sms = 148;
  // ---- implicit ----
  uint32_t H = 0;
  uint64_t nodes[HBT_MAX_LEVELS] = {};       // root-first
  uint64_t offset[HBT_MAX_LEVELS + 1] = {};  // root-first, node units
  void* d_inner = nullptr;
  uint64_t inner_bytes = 0;
  // derived per-node index sector ("I_s = K_8s" applied to implicit nodes
  // wider than one 32 B sector): entry t = max key of sector t, MAX-padded
  void* d_inner_idx = nullptr;
  uint64_t inner_idx_bytes = 0;
  uint32_t idx_stride = 0;  // bytes of index per node (0 = nodes fit one sector)
  // Level-T directory (search mode 2): d_dir = [M_T: count_T keys | dir: 2^dir_bits x (u16 lo, u16 hi)]
  // M_T[j] = max key below level-T node j (MAX for the last node); dir[p] = the
  // range of level-T nodes that queries with key prefix p can reach.
  void* d_dir = nullptr;
  uint64_t dir_bytes = 0;
  uint32_t dir_T = 0;       // target level (H = leaf lines)
  uint32_t dir_count = 0;   // nodes at level T
  uint32_t dir_bits = 0;
  void* d_leaf = nullptr;
  uint64_t L0 = 0;
  uint64_t leaf_bytes = 0;
  // L-segment placement (hbt_set_leaf_placement): 0 = HBM; 1 = pinned host memory
  // mapped into the device address space (h_leaf = its host address, d_leaf = the
  // device alias), the paper's I-segment-on-GPU / L-segment-in-host split
  uint32_t leaf_where = 0;
  void* h_leaf = nullptr;
  // ---- regular ----
  hbt::RegularState r;
  // ---- key-range sharding ----
  hbt::ShardMeta shard;
  hbt::Scratch shard_scratch;
  void* fused = nullptr;  // sharded_fused.cu state (peer windows)
  // ---- search ----
  hbt::SearchConfig cfg;
  mutable hbt::HostPipe pipe;
  mutable hbt::BucketState bk;
  mutable hbt::BucketState bks;  // streamed host L-segment (own bucket count)
  mutable std::mutex stream_mu;   // one user of the streamed staging slots at a time
  // serialises (re)preparation of the bucket splitters / item directory (bucketed.cu):
  // preparation completes on the host before any search may use them
  mutable std::mutex bk_mu;
};

namespace hbt {
// implicit_build.cu
int implicit_build(hbt_tree* t, const void* keys, const void* values, uint64_t n, cudaStream_t s);
int implicit_build_sorted(hbt_tree* t, const void* sk, const void* sv, uint64_t n_sorted_distinct,
                          cudaStream_t s);
// sort (stable) + dedupe-last-wins into fresh device arrays; *nd = distinct count
int sort_dedupe(uint32_t width, const void* keys, const void* values, uint64_t n, void** out_k,
                void** out_v, uint64_t* nd, cudaStream_t s);
int implicit_update(hbt_tree* t, const hbt_batch* b, cudaStream_t s);
// merge t's pairs with the batch and build the result into the empty tree nt (t unchanged)
int implicit_merge_rebuild(const hbt_tree* t, const hbt_batch* b, hbt_tree* nt, cudaStream_t s);
// api.cu: the search dispatch of hbt_search (streamed / bucketed / plain), tree teardown,
// bucket-state invalidation
int device_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s);
void free_tree(hbt_tree* t);
void invalidate_buckets(hbt_tree* t);
// regular.cu: deep copy of a regular tree's device state into the empty tree dst
int regular_clone(const hbt_tree* src, hbt_tree* dst, cudaStream_t s);
// implicit_search.cu
int implicit_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s);
// same, reporting global positions base + rank (sharded trees)
// implicit search reading leaf lines at leafp + line * 64 (a staged slice's base
// minus its first line; only lines inside the slice are dereferenced)
int implicit_search_leaf(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t pos_base,
                         const void* leafp, cudaStream_t s);
bool leaf_stream_enabled(const hbt_tree* t, uint64_t m);
int streamed_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t pos_base,
                    cudaStream_t s);
int implicit_search_base(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t pos_base,
                         cudaStream_t s);
void shard_free(hbt_tree* t);
// range.cu
void range_free(hbt_tree* t);
int range_scan(const hbt_tree* t, const void* lo, const void* hi, uint64_t m, uint32_t k, void* ok, void* ov,
               uint32_t* oc, cudaStream_t s);
// sharded_fused.cu
void fused_free(hbt_tree* t);
int fused_search_local(hbt_tree* const* shards, int G, const void* const* queries, const uint64_t* m,
                       const hbt_out* outs, cudaStream_t st);
int fused_search_nccl(const hbt_tree* t, const void* queries, uint64_t m, hbt_out out, cudaStream_t st);
// index bytes per implicit node (0 when F*S <= 32)
uint32_t implicit_idx_stride(uint32_t F, uint32_t S);
// regular_*.cu
int regular_build(hbt_tree* t, const void* keys, const void* values, uint64_t n, cudaStream_t s);
int regular_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, cudaStream_t s);
int regular_update(hbt_tree* t, const hbt_batch* b, cudaStream_t s);
void regular_free(hbt_tree* t);
// Item-directory searches write 16 B records {pos|found, value (zero-extended)}
// at pf (v is unused): rec[i] = (pf[2i], pf[2i+1]).
int implicit_search_items(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v,
                          const ItemDir& d, cudaStream_t s);
int regular_search_items(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v,
                         const ItemDir& d, cudaStream_t s);
// bucketed.cu
bool bucketed_enabled(const hbt_tree* t, uint64_t m);
int bucketed_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t pos_base,
                    cudaStream_t s, const RemoteOut* ro = nullptr);
// the owner-side search of the sharded paths: bucketed when enabled, positions + pos_base
int shard_local_search(const hbt_tree* t, const void* q, uint64_t m, uint64_t* pf, void* v, uint64_t pos_base,
                       cudaStream_t s);
void bucket_free(hbt_tree* t);
// implicit L-segment placement (api.cu): free the current L-segment wherever it lives;
// move it to HBM (0) or mapped pinned host memory (1)
void leaf_free(hbt_tree* t);
int leaf_place(hbt_tree* t, uint32_t where);
}  // namespace hbt
