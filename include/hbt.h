/* include/hbt.h — C ABI of the B200-native HB+-tree lookup library (libhbt.so).
 *
 * What it computes (Shahvarani & Jacobsen, SIGMOD'16; /root/reference/PAPER.md
 * cited as P:<line>): batched point / lower-bound lookups of unsigned 32- or
 * 64-bit keys in a B+-tree whose inner levels form the I-segment and whose
 * leaves form the L-segment (Fig. 1), in two forms:
 *   - IMPLICIT: breadth-first array, child j of node i of level m at
 *     Offset[m+1] + i*F + j; inner node = F keys, last key MAX;
 *     leaf = one 64-byte line of P = 64/(2S) (key, value) pairs.
 *   - REGULAR: inner node = index entries + keys + child references, searched in
 *     three accesses; big leaves of F lines sharing the pool index
 *     of their last-level inner node.
 * Empty key slots hold MAX = 2^n - 1.  Keys compare UNSIGNED
 * (reading R2).  Values have the key's width (S covers "a key or a
 * value").
 *
 * Result of a lookup of q: let Kd be the sorted
 * distinct keys (duplicates in the input collapse to their LAST occurrence) and
 * r = lower_bound(Kd, q).
 *   found  = r < n' && Kd[r] == q
 *   value  = found ? value of Kd[r] : 0
 *   pos    = IMPLICIT: r (the dense L-segment slot) or HBT_POS_END if r == n';
 *            REGULAR : the physical slot (v*F + j)*P + s of Kd[r] (big leaf v,
 *            line j, slot s), or HBT_POS_END if r == n'.
 *   pos_found[i] = pos | (found ? HBT_FOUND_BIT : 0)
 *
 * Ownership / memory: every pointer passed to hbt_bulk_build, hbt_search and
 * hbt_bulk_update is a caller-owned DEVICE pointer (cudaMalloc / torch CUDA
 * tensor on the current device).  hbt_search_host is the one entry point taking
 * HOST pointers (pinned recommended).  A tree owns its device memory until
 * hbt_destroy.  Device pointers are validated with cudaPointerGetAttributes
 * (pageable host pointers -> HBT_EINVAL); the last 8 pointers that validated are
 * remembered per thread, so small batches do not pay the check on every call.
 *
 * Streams: `stream` is a cudaStream_t passed as void* (NULL = legacy default
 * stream).  hbt_bulk_build and hbt_bulk_update are host-synchronous on return;
 * hbt_search is asynchronous on `stream`; hbt_search_host is synchronous.
 * Concurrent hbt_search calls on one tree are allowed (read-only);
 * hbt_bulk_update must not overlap any search on the same tree.
 *
 * Errors: every call returns an hbt_status; nothing throws across the ABI.  On
 * error the tree is unchanged (for build, *out = NULL) and hbt_last_error()
 * returns a thread-local message.  There is NO CPU fallback: without a CUDA
 * device every compute entry point fails with HBT_ECUDA.
 */
#ifndef HBT_H
#define HBT_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define HBT_API __attribute__((visibility("default")))
#else
#define HBT_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct hbt_tree hbt_tree;

typedef enum {
  HBT_OK = 0,
  HBT_EINVAL = -1,        /* bad argument (NULL, host pointer where device expected, bad fanout/layout) */
  HBT_ENOMEM = -2,        /* device allocation failed */
  HBT_ECUDA = -3,         /* CUDA runtime error (message in hbt_last_error) */
  HBT_ENCCL = -4,         /* NCCL error (sharded calls) */
  HBT_EUNSUPPORTED = -5   /* valid but not supported by this build */
} hbt_status;

/* layout word: bit 0 = tree form, bits 4.. = key (= value) width */
enum { HBT_IMPLICIT = 0x0, HBT_REGULAR = 0x1, HBT_KEY32 = 0x00, HBT_KEY64 = 0x10 };

#define HBT_POS_END   0x7FFFFFFFFFFFFFFFull
#define HBT_FOUND_BIT 0x8000000000000000ull

/* Caller-owned device output arrays of length m: pos_found (uint64) and values
 * (uint32 for HBT_KEY32, uint64 for HBT_KEY64). */
typedef struct {
  uint64_t* pos_found;
  void* values;
} hbt_out;

/* A batch of updates: keys/values of the tree's width and one op
 * byte per entry, 0 = UPSERT (insert or overwrite), 1 = DELETE (no-op if the key
 * is absent).  The last op per key wins (reading R12).  Device pointers. */
typedef struct {
  const void* keys;
  const void* values;
  const uint8_t* ops;
  uint64_t count;
} hbt_batch;

#define HBT_MAX_LEVELS 32

typedef struct {
  uint32_t layout;          /* HBT_IMPLICIT | HBT_REGULAR */
  uint32_t width;           /* S in bytes: 4 or 8 */
  uint32_t fanout;          /* F key slots per inner node */
  uint32_t pairs_per_line;  /* P = 64 / (2S) */
  uint64_t n_distinct;      /* n' live keys */
  uint32_t height;          /* implicit: inner levels H; regular: upper levels U + 1 (last level) */
  uint32_t smem_levels;     /* top levels the search kernel stages in shared memory */
  uint64_t level_nodes[HBT_MAX_LEVELS]; /* implicit: nodes per inner level, root first;
                                           regular: nodes per upper level, bottom first */
  uint64_t leaf_lines;      /* implicit: L0 64-byte lines; regular: big-leaf pool size */
  uint64_t chain_len;       /* regular: live big leaves; implicit: = leaf_lines */
  uint64_t inner_bytes;     /* I-segment bytes on the device */
  uint64_t leaf_bytes;      /* L-segment bytes on the device */
} hbt_info_t;

/* Segments copied out by hbt_export (for bitwise build parity in tests). */
enum {
  HBT_SEG_INNER = 0,       /* implicit: root-first node array, F keys of S bytes per node       */
  HBT_SEG_LEAF = 1,        /* implicit: L0 lines of [P keys | P values];
                              regular : pool x F lines of [P keys | P values]                    */
  HBT_SEG_COUNT = 2,       /* regular: uint32 count per big leaf                                 */
  HBT_SEG_LAST_KEYS = 3,   /* regular: pool x F separator keys of the last-level inner nodes      */
  HBT_SEG_LAST_IDX = 4,    /* regular: pool x NI index entries of the last-level inner nodes      */
  HBT_SEG_UPPER_KEYS = 5,  /* regular: upper pool x F keys                                        */
  HBT_SEG_UPPER_IDX = 6,   /* regular: upper pool x NI index entries                              */
  HBT_SEG_UPPER_REFS = 7,  /* regular: upper pool x F uint32 child references                     */
  HBT_SEG_CHAIN = 8,       /* regular: uint32 big-leaf pool indices in key order                  */
  HBT_SEG_INNER_IDX = 9    /* implicit: per-node index sector (max key of each 32 B key sector,
                              MAX-padded to max(16, F*S/32*S) bytes) for nodes wider than 32 B   */
};

/* Build a tree from n (key, value) pairs.  keys/values: device
 * arrays of n elements of width S (unsorted; duplicates allowed, last wins).
 * fanout in {4, 8, 16, 32}; layout = HBT_IMPLICIT|HBT_REGULAR combined with
 * HBT_KEY32|HBT_KEY64.  n = 0 builds the empty tree.  The inputs are copied;
 * they may be freed after return.  Host-synchronous. */
HBT_API int hbt_bulk_build(const void* keys, const void* values, uint64_t n, uint32_t fanout,
                   uint32_t layout, void* stream, hbt_tree** out);

/* Look up m queries (device array of width S) into out (device arrays, length
 * m): the paper's batched search (the problem statement of §4.1; node
 * search rule P:190, reading R1; implicit child index P:126; regular node P:134-138).
 * Asynchronous on `stream`.  m = 0 is a no-op.  Large batches over trees far beyond the
 * L2 are partitioned by key range first ("bucket"); results are identical either way. */
HBT_API int hbt_search(const hbt_tree* t, const void* queries, uint64_t m, hbt_out out, void* stream);

/* End-to-end lookup with HOST buffers: copies queries host->device, searches and
 * copies results device->host, chunked so copies overlap the search (the
 * paper's bucket pipelining + double buffering, re-done with CUDA
 * streams).  Pinned host memory gives full PCIe/C2C bandwidth.  Synchronous;
 * calls on one tree are serialised. */
HBT_API int hbt_search_host(const hbt_tree* t, const void* host_queries, uint64_t m,
                    uint64_t* host_pos_found, void* host_values, void* stream);

/* L-segment placement (the paper's split: the I-segment on the GPU, the
 * L-segment in host memory).  where = 0: HBM (default);
 * 1: pinned host memory mapped into the device address space — the search, range
 * and bucketing kernels then read each query's leaf line with zero-copy loads over
 * the host link (PCIe / NVLink-C2C), so a tree's leaves may exceed HBM while its
 * inner levels stay in HBM.  Results are identical in both placements.
 * IMPLICIT: the leaf lines; a batch that touches most of them may instead be served
 * by streaming bucket slices into HBM ("leaf_stream"); a rebuild by hbt_bulk_update
 * keeps the placement.  REGULAR: the big-leaf pool (zero-copy only); the update
 * kernels write leaves over the link and pool growth stays in host memory.
 * HBT_EUNSUPPORTED for multi-shard trees.  Synchronises the device (no search may be
 * in flight); HBT_ENOMEM when the pinned allocation fails (the tree is unchanged). */
HBT_API int hbt_set_leaf_placement(hbt_tree* t, uint32_t where);
HBT_API int hbt_get_leaf_placement(const hbt_tree* t, uint32_t* where);

/* Range scan (the range-query experiment of P:392): for each of the m
 * queries, the first up-to-k pairs with lo[i] <= key <= hi[i] in key order.
 * lo/hi: device arrays (width S, length m).  out_keys/out_values: device arrays
 * of m*k elements (row i = query i; slots past the count are (MAX, 0));
 * out_count: device uint32[m].  k in [1, 4096].  Asynchronous on `stream`.
 * IMPLICIT scans consecutive ranks of the contiguous L-segment; REGULAR scans
 * the big leaf, then the next big leaves in key order. */
HBT_API int hbt_range(const hbt_tree* t, const void* lo, const void* hi, uint64_t m, uint32_t k,
                      void* out_keys, void* out_values, uint32_t* out_count, void* stream);

/* Apply a batch of UPSERT/DELETE ops.  IMPLICIT: merge into the
 * sorted pairs and rebuild.  REGULAR: per-big-leaf merge on the GPU,
 * splits into new pool indices, removal of emptied leaves, then the upper
 * levels are regrouped (reading R11).  Host-synchronous. */
HBT_API int hbt_bulk_update(hbt_tree* t, const hbt_batch* batch, void* stream);

HBT_API int hbt_destroy(hbt_tree* t);
HBT_API int hbt_info(const hbt_tree* t, hbt_info_t* info);

/* Copy one segment of the tree's device layout into host memory `dst` of
 * `bytes` bytes (HBT_EINVAL if too small); *written receives the byte count. */
HBT_API int hbt_export(const hbt_tree* t, uint32_t segment, void* dst, uint64_t bytes, uint64_t* written);

/* Tune the search and bucketing of one tree; results never depend on it.  name / value:
 *   "ctas_per_sm" cap on resident CTAs per SM (0 = occupancy-derived)
 *   "smem_mode"   implicit level-T directory (lower_bound over the level-T maxima plus a prefix
 *                 table): 2 = staged in shared memory once per CTA (default), 3 = read in place
 *                 from L2 (used automatically for batches <= "small_batch")
 *   "small_batch" batches of at most this many queries use smem_mode 3 (default 65536)
 *   "l2_levels_bytes" implicit: inner levels below the directory are read as index sector + one
 *                 key sector while their cumulative bytes fit this L2 budget, as whole nodes
 *                 beyond it (0 = default 32 MB; 1 = every level whole)
 *   "full_levels" implicit: bit d set = level d's nodes are read whole (0 = by the budget above)
 *   "exchange"    sharded search: 0 = fused peer-memory exchange (CUDA IPC windows, device
 *                 barriers, count rows and queries by peer stores; default), 1 = NCCL send/recv
 *                 (multi-process) / device copies (hbt_search_sharded_local)
 *   "exchange_chunks" fused exchange: the batch is exchanged in 1..4 chunks; the owner searches
 *                 chunk c on a second stream while chunk c+1 is put (overlap of NVLink stores and
 *                 search).  Default 1; every rank of a communicator must set the same value.
 *   "g1_direct"   hbt_search_sharded on a ONE-shard tree with exchange 0: 1 (default) = search
 *                 in place (nothing to route or exchange), 0 = run the full fused pipeline
 *   "bucket"      query bucketing before the tree walk (north_star "queries bucketed per batch"):
 *                 0 = off, 1 = on, 2 = auto (default: trees larger than 8x the L2, batches of
 *                 >= 4 Mi queries: c3, c4, c5).  The batch is
 *                 partitioned into B key-range buckets, searched bucket after bucket, and the
 *                 results are gathered back to query order; outputs are identical.
 *   "bucket_slice" tree bytes per bucket (0 = default 1 MB; B <= 1024)
 *   "bucket_items" bucketed search through a bucket-local shared-memory directory (1, default)
 *                 or the normal search kernel on the bucketed queries (0)
 *   "bucket_cap"  item-directory shared-memory entries (0 = derived; small values force the
 *                 global-memory fallback, for tests)
 *   "item_rounds" bucketed item searches: most warp rounds per work item (0 = default 16,
 *                 or 8 for the compressed-directory implicit search when the leaf lines its
 *                 in-flight items reach exceed 2x the L2; fewer are used when the batch would
 *                 leave SMs idle)
 *   "phase_timing" 1 = record CUDA events around the phases of each bucketed search (read
 *                 them with hbt_last_phases), 0 = off (default)
 *   "leaf_stream" L-segment in host memory (hbt_set_leaf_placement): 0 = zero-copy leaf
 *                 reads; 1 = bucket the batch and stream each bucket's leaf slice into HBM
 *                 (double-buffered copies overlapping the previous bucket's search);
 *                 2 = auto (default: stream when 160 B x m exceeds the L-segment bytes)
 *   "stream_slice" host L-segment bytes per streamed bucket (0 = default 8 MB; <= 1024 buckets)
 *   "host_chunk_log2" hbt_search_host: queries per pipeline bucket, log2 in [12, 26] (default 20)
 *   "host_bufs"   hbt_search_host: (stream, buffer) pairs in flight, 2..4 (default 2)
 *   "leaf256"     1 (default) = the leaf line (and the regular item search's key line) is read
 *                 by two lanes' 256-bit loads, one 64 B request per lane group; 0 = 16 B loads
 *   "full256"     implicit whole-node levels: 256-bit lane loads (1, default) or 16 B loads (0)
 *   "l2_hint"     implicit search: L2 eviction-priority hints (createpolicy + ld ...
 *                 L2::cache_hint); bit 0 = leaf lines evict-first, bit 1 = whole-node levels
 *                 evict-last; 4 = auto (default: bit 0 iff the I-segment fits in a quarter of
 *                 the L2 -- measured c2 0.426 -> 0.415 ms, c5 Zipf 2.84 -> 3.00 ms with it on)
 *   "item_l2_hint" the same bits for the implicit bucketed item search (default 1: c4 item
 *                 search 10.96 -> 9.50 ms, DRAM reads 171 -> 148 B/query)
 *   "item_cdir"   item directory in its compressed per-bucket form (16-bit entries under a
 *                 per-bucket prefix table, items cut inside one bucket; regular trees: the
 *                 leaf lines): 0 = never, 1 = where it reaches a deeper tree level than 8 B
 *                 keys and fits (default), 2 = always where it fits
 *   "item_qpf"    compressed-directory item searches: each lane prefetches its query this many
 *                 rounds beyond the next into the L2 (0 = off, 1 = default; 0..6)
 *   "item_cnode"  compact 32 B copies of the last inner level's nodes for the bucketed implicit
 *                 search (u64 keys, F = 16, directory on the last inner level): 0 = off,
 *                 1 = where that level is read as whole nodes (default), 2 = always
 * Variants measured slower were removed (DESIGN.md §8 keeps their numbers).  Unknown
 * names or out-of-range values return HBT_EINVAL. */
HBT_API int hbt_set_param(hbt_tree* t, const char* name, int64_t value);

/* Device time of the phases of the tree's last BUCKETED search (hbt_search with
 * "bucket" in effect and "phase_timing" = 1), in milliseconds, measured with
 * CUDA events recorded on the search's stream:
 *   ms[0] bucket count   ms[1] scan   ms[2] scatter   ms[3] tree search   ms[4] gather
 * `launches` = kernel launches of that search.  Synchronises on the last event.
 * HBT_EINVAL if no timed bucketed search has run on this tree. */
typedef struct {
  uint32_t phases;    /* valid entries of ms (5) */
  uint32_t launches;  /* kernels launched by the search */
  float ms[8];
} hbt_phase_times;
HBT_API int hbt_last_phases(const hbt_tree* t, hbt_phase_times* out);

/* ---- key-range sharding over G GPUs (one process per GPU), SURVEY §8(e) ----
 * Shard g holds a contiguous key range; shards are numbered in key order (the
 * keys of shard g are all larger than those of every non-empty shard < g; keys
 * may be unsorted within a shard).  A query goes to owner(q) = #(shard_max < q)
 * over the non-empty shards (the max-separator rule of the node search applied
 * above the shard roots), is searched there, and its result comes back to the
 * rank that asked; pos is GLOBAL: the shard's first global rank + local rank.
 * Implicit trees only. */
typedef struct hbt_comm hbt_comm;

/* Host all-gather used by communicators created with hbt_comm_init_host:
 * gather `bytes` from every rank's `send` into `recv` (nranks * bytes, rank
 * order); return 0 on success. */
typedef int (*hbt_allgather_fn)(const void* send, void* recv, uint64_t bytes, void* ctx);

/* ncclGetUniqueId into a 128-byte buffer (rank 0; broadcast it to all ranks). */
HBT_API int hbt_comm_unique_id(void* id128);
/* ncclCommInitRank over nranks processes (one GPU each, current device). */
HBT_API int hbt_comm_init(int nranks, int rank, const void* id128, hbt_comm** out);
/* A communicator WITHOUT NCCL: the few small host-side exchanges of the sharded
 * calls (shard ranges, per-batch counts, IPC window handles) go through the
 * caller's all-gather callback; the data path is the fused peer-memory exchange
 * (exchange = 0).  Works with any number of ranks per GPU. */
HBT_API int hbt_comm_init_host(int nranks, int rank, hbt_allgather_fn fn, void* ctx, hbt_comm** out);
HBT_API int hbt_comm_destroy(hbt_comm* c);
/* Collective, host only (no device work): all-gather every rank's (n', min key, max key)
 * through the communicator and check that the non-empty shards are in key order.
 * Writes, per rank g (arrays of nranks entries): counts[g] = n'_g, bases[g] = the
 * shard's first global rank (sum of earlier counts), maxima[g] = its max key (the
 * routing table of owner(q) = #(shard_max < q)).  HBT_EINVAL if ranges overlap or are
 * out of order.  hbt_bulk_build_sharded calls it after building the local shard. */
HBT_API int hbt_comm_shard_table(hbt_comm* c, uint64_t n_local, uint64_t kmin, uint64_t kmax, uint64_t* counts,
                                 uint64_t* bases, uint64_t* maxima);
/* Collective: every rank builds its shard from its local (device) pairs, then the
 * ranks all-gather (n', min, max).  HBT_EINVAL if shard ranges overlap. */
HBT_API int hbt_bulk_build_sharded(hbt_comm* c, const void* keys_local, const void* values_local,
                                   uint64_t n_local, uint32_t fanout, uint32_t layout, void* stream,
                                   hbt_tree** out);
/* Collective: every rank searches its local batch (the north_star's routed search,
 * SURVEY §8(e).2, P:186-196 per shard).  Exchange "exchange" = 0 (default): the fused
 * peer-memory exchange — count rows and queries are stored straight into the owners'
 * IPC-mapped windows, device flag barriers order the steps, and the owner's bucketed
 * gather stores each result into the requester's window (sharded_fused.cu); 1: NCCL
 * send/recv of counts, queries and results (an all-to-all) + unpermute.  One small D2H
 * of the count matrix per batch (host-synchronous there).  A ONE-shard tree searches in
 * place ("g1_direct").  Positions are global (shard base rank + local rank). */
HBT_API int hbt_search_sharded(const hbt_tree* t, const void* queries_local, uint64_t m_local,
                               hbt_out out_local, void* stream);
/* Single-process shard group on ONE device (tests, capacity planning): mark G
 * implicit trees built from key-ordered disjoint ranges as shards 0..G-1 ... */
HBT_API int hbt_shard_local_init(hbt_tree* const* shards, int G);
/* ... and run the sharded search for G query batches with the same route /
 * search / unpermute kernels, the exchange being device-to-device copies. */
HBT_API int hbt_search_sharded_local(hbt_tree* const* shards, int G, const void* const* queries,
                                     const uint64_t* m, const hbt_out* outs, void* stream);

/* ---- versioned trees: searches concurrent with bulk updates (
 * the paper's concurrent search/update queries, App. B.3, and its batch
 * update, §5.6) ----
 * A versioned handle owns a sequence of immutable tree versions 0, 1, 2, ...
 * hbt_versioned_search reads the version that is current when it is called (its number
 * goes to *version, may be NULL), asynchronously on `stream`, exactly like hbt_search.
 * hbt_versioned_update derives version k+1 from the current version k on `stream`
 * (IMPLICIT: merge + rebuild into fresh arrays; REGULAR: a device copy of
 * version k, then the in-place batch update of hbt_bulk_update), host-synchronously,
 * while searches on OTHER streams and threads keep reading version k; then publishes
 * k+1 (*version).  Updates are serialised; searches never block on one.  A replaced
 * version is freed once no call is inside it and every search launched on it has
 * completed (CUDA events), so device memory peaks at two versions during an update.
 * Error: the current version is unchanged.  Not for key-range shards or trees whose
 * L-segment is in host memory (HBT_EUNSUPPORTED). */
typedef struct hbt_versioned hbt_versioned;
/* Takes ownership of t (it becomes version 0; do not hbt_destroy it). */
HBT_API int hbt_versioned_create(hbt_tree* t, hbt_versioned** out);
HBT_API int hbt_versioned_search(hbt_versioned* v, const void* queries, uint64_t m, hbt_out out, void* stream,
                                 uint64_t* version);
HBT_API int hbt_versioned_update(hbt_versioned* v, const hbt_batch* batch, void* stream, uint64_t* version);
/* The current version's tree (borrowed: valid until the next update retires it; for
 * hbt_info / hbt_export / hbt_set_param on the current version). */
HBT_API int hbt_versioned_current(hbt_versioned* v, hbt_tree** t, uint64_t* version);
HBT_API int hbt_versioned_destroy(hbt_versioned* v);

HBT_API const char* hbt_last_error(void);
/* Library version string, e.g. "hbt 0.1 sm_100a". */
HBT_API const char* hbt_version(void);

#ifdef __cplusplus
}
#endif
#endif /* HBT_H */
