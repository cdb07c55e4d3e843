/* oracle/oracle.c — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU implementation of what the HB+-tree hot
 * path computes (Shahvarani & Jacobsen, "A Hybrid B+-tree as Solution for
 * In-Memory Indexing on CPU-GPU Heterogeneous Computing Platforms", SIGMOD'16;
 * text at /root/reference/PAPER.md, cited as P:<line>).  It follows the paper's
 * definitions step by step, with the readings of DESIGN.md §3 where the paper is
 * silent or garbled.  No blocking, no SIMD, no prefetch: scalar linear node scans
 * (the paper's "sequential search" baseline).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg may load
 * this library.  It shares no code, header, table or helper with the CUDA path
 * (paper_conf_sigmod_shahvaranij16_b200/csrc); neither includes the other.
 *
 * Parity pins (tests/test_oracle_*.py): lower_bound over the sorted keys
 * (numpy.searchsorted / bisect), brute-force scans, hand-worked golden trees in
 * tests/golden/, B+-tree invariants, a Python dict as the textbook map after
 * updates.  No function here is "parity unpinned".
 */
#include "oracle.h"

#include <stdlib.h>
#include <string.h>

static uint64_t kmax_of(uint32_t width) { return width == 4 ? 0xFFFFFFFFull : 0xFFFFFFFFFFFFFFFFull; }
static uint64_t ceil_div(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

/* ---------------------------------------------------------------------------
 * Dedupe (reading R4 = SURVEY §8c A4): stable sort by unsigned key,
 * duplicates collapse to their LAST occurrence (UPSERT semantics).
 * The sort is the C library's qsort on (key, input index), which makes it stable.
 * ------------------------------------------------------------------------- */
typedef struct { uint64_t key; uint64_t idx; } kv_idx;

static int cmp_kv_idx(const void* a, const void* b) {
  const kv_idx* x = (const kv_idx*)a;
  const kv_idx* y = (const kv_idx*)b;
  if (x->key != y->key) return x->key < y->key ? -1 : 1;
  if (x->idx != y->idx) return x->idx < y->idx ? -1 : 1;
  return 0;
}

uint64_t orc_dedupe(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                    uint64_t* out_keys, uint64_t* out_vals) {
  if (n == 0) return 0;
  kv_idx* a = (kv_idx*)malloc(n * sizeof(kv_idx));
  for (uint64_t i = 0; i < n; ++i) { a[i].key = keys[i]; a[i].idx = i; }
  qsort(a, n, sizeof(kv_idx), cmp_kv_idx);
  uint64_t m = 0;
  for (uint64_t i = 0; i < n; ++i) {
    int last_of_run = (i + 1 == n) || (a[i + 1].key != a[i].key);
    if (last_of_run) {
      out_keys[m] = a[i].key;
      out_vals[m] = vals[a[i].idx];
      ++m;
    }
  }
  free(a);
  return m;
}

/* ---------------------------------------------------------------------------
 * Node search (P:190 read with P:520 / P:566, reading R1 = "minimum i such that
 * key <= array[i]"): the number of node keys strictly smaller than q.  Keys
 * compare as UNSIGNED integers (reading R2).
 * ------------------------------------------------------------------------- */
static uint32_t count_less(const uint64_t* a, uint32_t len, uint64_t q) {
  uint32_t c = 0;
  for (uint32_t t = 0; t < len; ++t)
    if (a[t] < q) ++c;
  return c;
}

/* ---------------------------------------------------------------------------
 * Plain definition: r = lower_bound(Kd, q); found = Kd[r]==q.
 * ------------------------------------------------------------------------- */
void orc_lower_bound(const uint64_t* Kd, const uint64_t* Vd, uint64_t n,
                     const uint64_t* q, uint64_t m, uint64_t* pos_found, uint64_t* vals,
                     int nthreads) {
  (void)nthreads;
#pragma omp parallel for schedule(static) num_threads(nthreads > 0 ? nthreads : 1)
  for (uint64_t j = 0; j < m; ++j) {
    uint64_t lo = 0, hi = n; /* invariant: Kd[<lo] < q <= Kd[>=hi] */
    while (lo < hi) {
      uint64_t mid = lo + (hi - lo) / 2;
      if (Kd[mid] < q[j]) lo = mid + 1; else hi = mid;
    }
    int found = lo < n && Kd[lo] == q[j];
    pos_found[j] = (lo < n ? lo : ORC_END) | (found ? ORC_FOUND : 0);
    vals[j] = found ? Vd[lo] : 0;
  }
}

/* ===========================================================================
 * Implicit tree.  P:126: "If the node A is the i-th node of a tree at level m
 * in breadth first order, then the j-th child of A is at position
 * Offset[m+1] + i*F_I + j".  Leaf = one 64 B line of P = 64/(2S) pairs
 * (P:126).  Inner node = F keys, last key = MAX; key slot i of a
 * node = the max key of child i's subtree for i < cnt-1, MAX otherwise
 * (reading R3).  Empty key slots = MAX.
 * ========================================================================= */
orc_itree* orc_itree_build(const uint64_t* Kd, const uint64_t* Vd, uint64_t n,
                           uint32_t F, uint32_t width) {
  orc_itree* t = (orc_itree*)calloc(1, sizeof(orc_itree));
  t->kmax = kmax_of(width);
  t->F = F;
  t->P = 64 / (2 * width);
  t->n = n;
  const uint64_t P = t->P;
  t->L0 = n == 0 ? 1 : ceil_div(n, P);

  /* L-segment: line l holds Kd[lP .. lP+P), padded with (MAX, 0). */
  t->lkeys = (uint64_t*)malloc(t->L0 * P * sizeof(uint64_t));
  t->lvals = (uint64_t*)malloc(t->L0 * P * sizeof(uint64_t));
  for (uint64_t l = 0; l < t->L0; ++l)
    for (uint64_t s = 0; s < P; ++s) {
      uint64_t r = l * P + s;
      t->lkeys[l * P + s] = r < n ? Kd[r] : t->kmax;
      t->lvals[l * P + s] = r < n ? Vd[r] : 0;
    }

  /* Level sizes bottom-up: c[0] = L0 leaf lines, c[h] = ceil(c[h-1]/F) until 1. */
  uint64_t c[ORC_MAXLEV + 1];
  uint32_t H = 0;
  c[0] = t->L0;
  while (c[H] > 1) { c[H + 1] = ceil_div(c[H], F); ++H; }
  t->H = H;
  /* Root-first numbering: level d (d = 0 root) is height H-d; Offset[] in nodes. */
  t->offset[0] = 0;
  for (uint32_t d = 0; d < H; ++d) {
    t->nodes[d] = c[H - d];
    t->offset[d + 1] = t->offset[d] + t->nodes[d];
  }
  t->inner = (uint64_t*)malloc((t->offset[H] ? t->offset[H] : 1) * F * sizeof(uint64_t));

  /* maxkey per node, computed bottom-up by explicit child enumeration. */
  uint64_t* mk_below = (uint64_t*)malloc(t->L0 * sizeof(uint64_t));
  for (uint64_t l = 0; l < t->L0; ++l) {
    uint64_t last = (l + 1) * P < n ? (l + 1) * P : n; /* one past the line's last real key */
    mk_below[l] = last > 0 ? Kd[last - 1] : t->kmax;
  }
  for (uint32_t h = 1; h <= H; ++h) {
    uint32_t d = H - h;
    uint64_t* mk = (uint64_t*)malloc(c[h] * sizeof(uint64_t));
    for (uint64_t j = 0; j < c[h]; ++j) {
      uint64_t first_child = j * F;
      uint64_t cnt = c[h - 1] - first_child < F ? c[h - 1] - first_child : F;
      uint64_t* node = t->inner + (t->offset[d] + j) * F;
      for (uint64_t i = 0; i < F; ++i)
        node[i] = (i + 1 < cnt) ? mk_below[first_child + i] : t->kmax;
      mk[j] = mk_below[first_child + cnt - 1];
    }
    free(mk_below);
    mk_below = mk;
  }
  free(mk_below);
  return t;
}

void orc_itree_free(orc_itree* t) {
  if (!t) return;
  free(t->inner); free(t->lkeys); free(t->lvals); free(t);
}

void orc_itree_search(const orc_itree* t, const uint64_t* q, uint64_t m,
                      uint64_t* pos_found, uint64_t* vals, int nthreads) {
  const uint32_t F = t->F, P = t->P;
#pragma omp parallel for schedule(static) num_threads(nthreads > 0 ? nthreads : 1)
  for (uint64_t j = 0; j < m; ++j) {
    uint64_t node = 0; /* root */
    for (uint32_t d = 0; d < t->H; ++d) {
      const uint64_t* keys = t->inner + (t->offset[d] + node) * F;
      uint32_t i = count_less(keys, F, q[j]);
      node = node * F + i; /* Offset[d+1] + node*F + i, in level-relative form */
    }
    uint64_t l = node;
    const uint64_t* lk = t->lkeys + l * P;
    uint32_t s = count_less(lk, P, q[j]);
    uint64_t r = l * P + s;
    int found = (r < t->n) && (s < P) && (lk[s] == q[j]);
    pos_found[j] = (r < t->n ? r : ORC_END) | (found ? ORC_FOUND : 0);
    vals[j] = found ? t->lvals[l * P + s] : 0;
  }
}

/* Sort + dedupe a batch of ops (last op per key wins, reading R12). */
static uint64_t dedupe_ops(const uint64_t* ok, const uint64_t* ov, const uint8_t* op, uint64_t nops,
                           uint64_t** dk, uint64_t** dv, uint8_t** dop) {
  kv_idx* a = (kv_idx*)malloc((nops ? nops : 1) * sizeof(kv_idx));
  for (uint64_t i = 0; i < nops; ++i) { a[i].key = ok[i]; a[i].idx = i; }
  qsort(a, nops, sizeof(kv_idx), cmp_kv_idx);
  *dk = (uint64_t*)malloc((nops ? nops : 1) * sizeof(uint64_t));
  *dv = (uint64_t*)malloc((nops ? nops : 1) * sizeof(uint64_t));
  *dop = (uint8_t*)malloc(nops ? nops : 1);
  uint64_t m = 0;
  for (uint64_t i = 0; i < nops; ++i) {
    if (i + 1 == nops || a[i + 1].key != a[i].key) {
      (*dk)[m] = a[i].key; (*dv)[m] = ov[a[i].idx]; (*dop)[m] = op[a[i].idx]; ++m;
    }
  }
  free(a);
  return m;
}

orc_itree* orc_itree_update(const orc_itree* t, const uint64_t* ok, const uint64_t* ov,
                            const uint8_t* op, uint64_t nops) {
  uint64_t *dk, *dv; uint8_t* dop;
  uint64_t m = dedupe_ops(ok, ov, op, nops, &dk, &dv, &dop);
  /* The dense L-segment holds Kd[0..n) in its first n slots. */
  uint64_t cap = t->n + m;
  uint64_t* nk = (uint64_t*)malloc((cap ? cap : 1) * sizeof(uint64_t));
  uint64_t* nv = (uint64_t*)malloc((cap ? cap : 1) * sizeof(uint64_t));
  uint64_t a = 0, b = 0, o = 0;
  while (a < t->n || b < m) {
    if (b == m || (a < t->n && t->lkeys[a] < dk[b])) {        /* key untouched */
      nk[o] = t->lkeys[a]; nv[o] = t->lvals[a]; ++o; ++a;
    } else if (a == t->n || dk[b] < t->lkeys[a]) {             /* key only in batch */
      if (dop[b] == 0) { nk[o] = dk[b]; nv[o] = dv[b]; ++o; }
      ++b;
    } else {                                                    /* key in both */
      if (dop[b] == 0) { nk[o] = dk[b]; nv[o] = dv[b]; ++o; }
      ++a; ++b;
    }
  }
  uint32_t width = t->kmax == 0xFFFFFFFFull ? 4 : 8;
  orc_itree* r = orc_itree_build(nk, nv, o, t->F, width);
  free(nk); free(nv); free(dk); free(dv); free(dop);
  return r;
}

/* ===========================================================================
 * Regular tree (P:134 inner node = index line + key lines + refs; P:136 node
 * fragmentation + MAX padding; P:138 big leaves sharing the pool index of their
 * last-level inner node).  Generalised to fanout F (reading R7/R8):
 *   kpl = 64/S keys per 64 B key line, NI = F/kpl index entries (no index step
 *   when F <= kpl), big-leaf capacity B = F*P, build fill b = floor(3B/4) (R11).
 * ========================================================================= */
static void rt_grow(orc_rtree* t, uint64_t need) {
  if (need <= t->cap) return;
  uint64_t nc = t->cap ? t->cap : 1;
  while (nc < need) nc *= 2;
  const uint64_t FP = (uint64_t)t->F * t->P;
  t->lkeys = (uint64_t*)realloc(t->lkeys, nc * FP * sizeof(uint64_t));
  t->lvals = (uint64_t*)realloc(t->lvals, nc * FP * sizeof(uint64_t));
  t->lcount = (uint32_t*)realloc(t->lcount, nc * sizeof(uint32_t));
  t->lsep = (uint64_t*)realloc(t->lsep, nc * t->F * sizeof(uint64_t));
  t->lidx = (uint64_t*)realloc(t->lidx, nc * t->NI * sizeof(uint64_t));
  t->chain = (uint64_t*)realloc(t->chain, nc * sizeof(uint64_t));
  t->cap = nc;
}

/* Write `cnt` sorted pairs densely into big leaf v: line j holds entries [jP, jP+P). */
static void rt_pack_leaf(orc_rtree* t, uint64_t v, const uint64_t* k, const uint64_t* val, uint64_t cnt) {
  const uint64_t FP = (uint64_t)t->F * t->P;
  for (uint64_t s = 0; s < FP; ++s) {
    t->lkeys[v * FP + s] = s < cnt ? k[s] : t->kmax;
    t->lvals[v * FP + s] = s < cnt ? val[s] : 0;
  }
  t->lcount[v] = (uint32_t)cnt;
}

/* Last-level inner node v: sep[j] = max real key of line j for j < lines_v-1,
 * MAX otherwise; index entry idx[t] = sep[t*kpl + kpl - 1] ("I_s = K_8s"). */
static void rt_derive_last_level(orc_rtree* t, uint64_t v) {
  const uint64_t F = t->F, P = t->P;
  uint64_t cnt = t->lcount[v];
  uint64_t lines = cnt == 0 ? 1 : ceil_div(cnt, P);
  uint64_t* sep = t->lsep + v * F;
  for (uint64_t j = 0; j < F; ++j) {
    if (j + 1 < lines) {
      uint64_t mx = 0;
      for (uint64_t s = 0; s < P; ++s)
        if (j * P + s < cnt) mx = t->lkeys[v * F * P + j * P + s];
      sep[j] = mx;
    } else {
      sep[j] = t->kmax;
    }
  }
  for (uint64_t i = 0; i < t->NI; ++i) {
    uint64_t slot = i * t->kpl + t->kpl - 1;
    if (slot > F - 1) slot = F - 1;
    t->lidx[v * t->NI + i] = sep[slot];
  }
}

/* Upper levels regrouped from the leaf chain, F children per node in key order,
 * the last node of a level partial; pool indices bottom-up, left to right.
 * Node key slot i = max key of child i for i < cnt-1, MAX otherwise. */
static void rt_build_upper(orc_rtree* t) {
  const uint64_t F = t->F;
  free(t->ukeys); free(t->uidx); free(t->urefs);
  t->ukeys = NULL; t->uidx = NULL; t->urefs = NULL;
  uint64_t cnt_below = t->nchain;
  uint64_t total = 0, c = cnt_below;
  uint32_t U = 0;
  while (c > 1) { c = ceil_div(c, F); t->unodes[U] = c; total += c; ++U; }
  t->U = U;
  t->uoff[0] = 0;
  for (uint32_t u = 0; u < U; ++u) t->uoff[u + 1] = t->uoff[u] + t->unodes[u];
  if (U == 0) return;
  t->ukeys = (uint64_t*)malloc(total * F * sizeof(uint64_t));
  t->uidx = (uint64_t*)malloc(total * t->NI * sizeof(uint64_t));
  t->urefs = (uint32_t*)malloc(total * F * sizeof(uint32_t));
  uint64_t* child_id = (uint64_t*)malloc(cnt_below * sizeof(uint64_t));
  uint64_t* child_mx = (uint64_t*)malloc(cnt_below * sizeof(uint64_t));
  for (uint64_t i = 0; i < cnt_below; ++i) {
    uint64_t v = t->chain[i];
    child_id[i] = v;
    child_mx[i] = t->lkeys[v * F * t->P + t->lcount[v] - 1]; /* chain leaves are non-empty when nchain > 1 */
  }
  for (uint32_t u = 0; u < U; ++u) {
    uint64_t nodes = t->unodes[u];
    uint64_t* nid = (uint64_t*)malloc(nodes * sizeof(uint64_t));
    uint64_t* nmx = (uint64_t*)malloc(nodes * sizeof(uint64_t));
    for (uint64_t j = 0; j < nodes; ++j) {
      uint64_t first = j * F;
      uint64_t cnt = cnt_below - first < F ? cnt_below - first : F;
      uint64_t id = t->uoff[u] + j;
      uint64_t* keys = t->ukeys + id * F;
      uint32_t* refs = t->urefs + id * F;
      for (uint64_t i = 0; i < F; ++i) {
        keys[i] = (i + 1 < cnt) ? child_mx[first + i] : t->kmax;
        refs[i] = (i < cnt) ? (uint32_t)child_id[first + i] : 0xFFFFFFFFu;
      }
      for (uint64_t i = 0; i < t->NI; ++i) {
        uint64_t slot = i * t->kpl + t->kpl - 1;
        if (slot > F - 1) slot = F - 1;
        t->uidx[id * t->NI + i] = keys[slot];
      }
      nid[j] = id;
      nmx[j] = child_mx[first + cnt - 1];
    }
    free(child_id); free(child_mx);
    child_id = nid; child_mx = nmx; cnt_below = nodes;
  }
  free(child_id); free(child_mx);
}

static void rt_derive_all(orc_rtree* t) {
  uint64_t n = 0;
  for (uint64_t v = 0; v < t->pool; ++v) rt_derive_last_level(t, v);
  for (uint64_t i = 0; i < t->nchain; ++i) n += t->lcount[t->chain[i]];
  t->n = n;
  rt_build_upper(t);
}

orc_rtree* orc_rtree_build(const uint64_t* Kd, const uint64_t* Vd, uint64_t n,
                           uint32_t F, uint32_t width) {
  orc_rtree* t = (orc_rtree*)calloc(1, sizeof(orc_rtree));
  t->kmax = kmax_of(width);
  t->F = F;
  t->P = 64 / (2 * width);
  t->kpl = 64 / width;
  t->NI = F > t->kpl ? F / t->kpl : 1;
  t->B = F * t->P;
  t->b = (3 * t->B) / 4;
  uint64_t nb = n == 0 ? 1 : ceil_div(n, t->b);
  rt_grow(t, nb);
  t->pool = nb;
  for (uint64_t v = 0; v < nb; ++v) {
    /* big leaf v holds Kd[floor(v n/nb) .. floor((v+1) n/nb)) */
    uint64_t lo = (uint64_t)(((unsigned __int128)v * n) / nb);
    uint64_t hi = (uint64_t)(((unsigned __int128)(v + 1) * n) / nb);
    rt_pack_leaf(t, v, Kd + lo, Vd + lo, hi - lo);
    t->chain[v] = v;
  }
  t->nchain = nb;
  rt_derive_all(t);
  return t;
}

void orc_rtree_free(orc_rtree* t) {
  if (!t) return;
  free(t->lkeys); free(t->lvals); free(t->lcount); free(t->lsep); free(t->lidx);
  free(t->chain); free(t->ukeys); free(t->uidx); free(t->urefs); free(t);
}

/* Three-step inner node search: index entries -> one key line -> ref. */
static uint32_t rt_node_slot(const orc_rtree* t, const uint64_t* keys, const uint64_t* idx, uint64_t q) {
  if (t->NI > 1) {
    uint32_t line = count_less(idx, t->NI, q);
    return line * t->kpl + count_less(keys + (uint64_t)line * t->kpl, t->kpl, q);
  }
  return count_less(keys, t->F, q);
}

/* Descend to the big leaf (= last-level inner node) of q. */
static uint64_t rt_find_leaf(const orc_rtree* t, uint64_t q) {
  if (t->U == 0) return t->chain[0];
  uint64_t u = t->uoff[t->U] - 1; /* root */
  for (int lev = (int)t->U - 1; lev >= 0; --lev) {
    uint32_t i = rt_node_slot(t, t->ukeys + u * t->F, t->uidx + u * t->NI, q);
    uint64_t child = t->urefs[u * t->F + i];
    if (lev == 0) return child;
    u = child;
  }
  return 0; /* unreachable */
}

void orc_rtree_search(const orc_rtree* t, const uint64_t* q, uint64_t m,
                      uint64_t* pos_found, uint64_t* vals, int nthreads) {
  const uint64_t F = t->F, P = t->P;
#pragma omp parallel for schedule(static) num_threads(nthreads > 0 ? nthreads : 1)
  for (uint64_t x = 0; x < m; ++x) {
    uint64_t v = rt_find_leaf(t, q[x]);
    uint64_t j = rt_node_slot(t, t->lsep + v * F, t->lidx + v * t->NI, q[x]);
    const uint64_t* lk = t->lkeys + v * F * P + j * P;
    uint32_t s = count_less(lk, (uint32_t)P, q[x]);
    int64_t in_line = (int64_t)t->lcount[v] - (int64_t)(j * P);
    int64_t lim = in_line < (int64_t)P ? in_line : (int64_t)P;
    if (s == P || (lk[s] == t->kmax && (int64_t)s >= lim)) {
      pos_found[x] = ORC_END;   /* no successor (MAX is padding unless counted) */
      vals[x] = 0;
    } else {
      int found = lk[s] == q[x];
      pos_found[x] = ((v * F + j) * P + s) | (found ? ORC_FOUND : 0);
      vals[x] = found ? t->lvals[v * F * P + j * P + s] : 0;
    }
  }
}

int orc_rtree_update(orc_rtree* t, const uint64_t* ok, const uint64_t* ov,
                     const uint8_t* op, uint64_t nops) {
  uint64_t *dk, *dv; uint8_t* dop;
  uint64_t m = dedupe_ops(ok, ov, op, nops, &dk, &dv, &dop);
  const uint64_t F = t->F, P = t->P, B = t->B, FP = F * P;

  /* Locate every op's big leaf by descent through the PRE-update tree. */
  uint64_t* leaf_of = (uint64_t*)malloc((m ? m : 1) * sizeof(uint64_t));
  for (uint64_t i = 0; i < m; ++i) leaf_of[i] = rt_find_leaf(t, dk[i]);

  uint64_t* old_chain = (uint64_t*)malloc(t->nchain * sizeof(uint64_t));
  memcpy(old_chain, t->chain, t->nchain * sizeof(uint64_t));
  uint64_t old_n = t->nchain;
  uint64_t* new_chain = (uint64_t*)malloc((old_n + m + 1) * sizeof(uint64_t));
  uint64_t nn = 0;
  uint64_t* mk = (uint64_t*)malloc((FP + m + 1) * sizeof(uint64_t));
  uint64_t* mv = (uint64_t*)malloc((FP + m + 1) * sizeof(uint64_t));

  uint64_t b = 0; /* op cursor: ops are in key order, so are their leaves in the chain */
  for (uint64_t ci = 0; ci < old_n; ++ci) {
    uint64_t v = old_chain[ci];
    uint64_t b0 = b;
    while (b < m && leaf_of[b] == v) ++b;
    if (b == b0) { new_chain[nn++] = v; continue; }
    /* merge leaf entries with ops [b0, b) */
    uint64_t cnt = t->lcount[v], a = 0, o = 0, x = b0;
    const uint64_t* lk = t->lkeys + v * FP;
    const uint64_t* lv = t->lvals + v * FP;
    while (a < cnt || x < b) {
      if (x == b || (a < cnt && lk[a] < dk[x])) { mk[o] = lk[a]; mv[o] = lv[a]; ++o; ++a; }
      else if (a == cnt || dk[x] < lk[a]) { if (dop[x] == 0) { mk[o] = dk[x]; mv[o] = dv[x]; ++o; } ++x; }
      else { if (dop[x] == 0) { mk[o] = dk[x]; mv[o] = dv[x]; ++o; } ++a; ++x; }
    }
    if (o == 0) {                       /* emptied: removed, index not reused (R11) */
      rt_pack_leaf(t, v, mk, mv, 0);
    } else if (o <= B) {                /* dense re-pack in place */
      rt_pack_leaf(t, v, mk, mv, o);
      new_chain[nn++] = v;
    } else {                            /* split evenly into ceil(o/B) leaves */
      uint64_t k = ceil_div(o, B);
      for (uint64_t p = 0; p < k; ++p) {
        uint64_t lo = p * o / k, hi = (p + 1) * o / k;
        uint64_t id = v;
        if (p > 0) { rt_grow(t, t->pool + 1); id = t->pool++; }
        rt_pack_leaf(t, id, mk + lo, mv + lo, hi - lo);
        new_chain[nn++] = id;
      }
    }
  }
  if (b != m) { /* routing must have been monotone in key order */
    free(leaf_of); free(old_chain); free(new_chain); free(mk); free(mv);
    free(dk); free(dv); free(dop);
    return -1;
  }
  if (nn == 0) {                        /* every key deleted: the empty tree */
    t->pool = 1;
    rt_pack_leaf(t, 0, mk, mv, 0);
    new_chain[nn++] = 0;
  }
  rt_grow(t, nn);
  memcpy(t->chain, new_chain, nn * sizeof(uint64_t));
  t->nchain = nn;
  rt_derive_all(t);
  free(leaf_of); free(old_chain); free(new_chain); free(mk); free(mv);
  free(dk); free(dv); free(dop);
  return 0;
}

/* ===========================================================================
 * Range scan.  Implicit: the leaves are contiguous in key order,
 * so after the descent the scan walks ranks r, r+1, ... of the L-segment.
 * Regular: the scan walks the big leaf's entries, then the next big leaves in
 * key order (the chain; the paper's linked leaves).
 * ========================================================================= */
void orc_itree_range(const orc_itree* t, const uint64_t* lo, const uint64_t* hi, uint64_t m, uint32_t k,
                     uint64_t* out_keys, uint64_t* out_vals, uint32_t* out_count) {
  uint64_t* pf = (uint64_t*)malloc((m ? m : 1) * sizeof(uint64_t));
  uint64_t* vv = (uint64_t*)malloc((m ? m : 1) * sizeof(uint64_t));
  orc_itree_search(t, lo, m, pf, vv, 1);
  for (uint64_t x = 0; x < m; ++x) {
    uint64_t r = pf[x] & ORC_END;
    uint32_t c = 0;
    for (uint32_t i = 0; i < k; ++i) {
      out_keys[x * k + i] = t->kmax;
      out_vals[x * k + i] = 0;
    }
    while (r != ORC_END && r < t->n && c < k && t->lkeys[r] <= hi[x]) {
      out_keys[x * k + c] = t->lkeys[r];
      out_vals[x * k + c] = t->lvals[r];
      ++c;
      ++r;
    }
    out_count[x] = c;
  }
  free(pf);
  free(vv);
}

void orc_rtree_range(const orc_rtree* t, const uint64_t* lo, const uint64_t* hi, uint64_t m, uint32_t k,
                     uint64_t* out_keys, uint64_t* out_vals, uint32_t* out_count) {
  const uint64_t FP = (uint64_t)t->F * t->P;
  for (uint64_t x = 0; x < m; ++x) {
    for (uint32_t i = 0; i < k; ++i) {
      out_keys[x * k + i] = t->kmax;
      out_vals[x * k + i] = 0;
    }
    uint32_t c = 0;
    /* the first entry >= lo: descend to its big leaf, then scan forward */
    uint64_t v = rt_find_leaf(t, lo[x]);
    uint64_t ci = 0;
    while (t->chain[ci] != v) ++ci;   /* position of v in key order */
    uint64_t e = 0;
    while (e < t->lcount[v] && t->lkeys[v * FP + e] < lo[x]) ++e;
    while (c < k && ci < t->nchain) {
      v = t->chain[ci];
      if (e >= t->lcount[v]) { ++ci; e = 0; continue; }
      if (t->lkeys[v * FP + e] > hi[x]) break;
      out_keys[x * k + c] = t->lkeys[v * FP + e];
      out_vals[x * k + c] = t->lvals[v * FP + e];
      ++c;
      ++e;
    }
    out_count[x] = c;
  }
}
