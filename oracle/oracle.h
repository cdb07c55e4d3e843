/* oracle/oracle.h — TEST INFRASTRUCTURE ONLY (see oracle.c header).
 *
 * Plain CPU oracle of the HB+-tree (Shahvarani & Jacobsen, SIGMOD'16).
 * Every key/value is carried as uint64_t; `kmax` (2^32-1 or 2^64-1) is the
 * key width's MAX = 2^n - 1 used for padding (§4.1).
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg may
 * load liboracle.so.  Shares no code with paper_conf_sigmod_shahvaranij16_b200/.
 */
#ifndef HBT_ORACLE_H
#define HBT_ORACLE_H
#include <stdint.h>

#define ORC_END 0x7FFFFFFFFFFFFFFFull
#define ORC_FOUND 0x8000000000000000ull
#define ORC_MAXLEV 64

/* ---- dedupe: stable sort by unsigned key, last occurrence wins -------------- */
uint64_t orc_dedupe(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                    uint64_t* out_keys, uint64_t* out_vals);

/* ---- implicit tree -------------------------------- */
typedef struct {
  uint64_t kmax;
  uint32_t F, P;            /* key slots per inner node, pairs per 64 B leaf line */
  uint64_t n;               /* n' distinct keys */
  uint32_t H;               /* inner levels (0: the root is the single leaf line) */
  uint64_t L0;              /* leaf lines */
  uint64_t nodes[ORC_MAXLEV];      /* nodes at level d, d = 0 is the ROOT      */
  uint64_t offset[ORC_MAXLEV + 1]; /* Offset[d] in node units, root-first      */
  uint64_t* inner;          /* offset[H] * F keys                              */
  uint64_t* lkeys;          /* L0 * P                                          */
  uint64_t* lvals;          /* L0 * P                                          */
} orc_itree;

orc_itree* orc_itree_build(const uint64_t* Kd, const uint64_t* Vd, uint64_t n,
                           uint32_t F, uint32_t width);
void orc_itree_free(orc_itree* t);
void orc_itree_search(const orc_itree* t, const uint64_t* q, uint64_t m,
                      uint64_t* pos_found, uint64_t* vals, int nthreads);
/* implicit batch update = apply ops to the sorted arrays, then rebuild */
orc_itree* orc_itree_update(const orc_itree* t, const uint64_t* ok, const uint64_t* ov,
                            const uint8_t* op, uint64_t nops);

/* ---- regular tree -------------------------- */
typedef struct {
  uint64_t kmax;
  uint32_t F, P, kpl, NI, B, b; /* fanout, pairs/line, keys per 64 B key line, index entries,
                                   big-leaf capacity F*P, build fill floor(3B/4) */
  uint64_t n;                    /* live keys */
  /* big-leaf pool + last-level inner nodes (same pool index) */
  uint64_t pool, cap;
  uint64_t* lkeys;   /* [cap][F*P] */
  uint64_t* lvals;   /* [cap][F*P] */
  uint32_t* lcount;  /* [cap]      */
  uint64_t* lsep;    /* [cap][F]   last-level inner node keys  */
  uint64_t* lidx;    /* [cap][NI]  last-level inner node index */
  uint64_t nchain;
  uint64_t* chain;   /* live big leaves in key order */
  /* upper levels (above the last inner level), pool indices bottom-up, left to right */
  uint32_t U;
  uint64_t unodes[ORC_MAXLEV]; /* level u = 0 is the level right above the last inner level */
  uint64_t uoff[ORC_MAXLEV + 1];
  uint64_t* ukeys;   /* [uoff[U]][F]  */
  uint64_t* uidx;    /* [uoff[U]][NI] */
  uint32_t* urefs;   /* [uoff[U]][F]  */
} orc_rtree;

orc_rtree* orc_rtree_build(const uint64_t* Kd, const uint64_t* Vd, uint64_t n,
                           uint32_t F, uint32_t width);
void orc_rtree_free(orc_rtree* t);
void orc_rtree_search(const orc_rtree* t, const uint64_t* q, uint64_t m,
                      uint64_t* pos_found, uint64_t* vals, int nthreads);
/* in-place regular batch update (SURVEY §8(c).2 "Regular update"); returns 0 */
int orc_rtree_update(orc_rtree* t, const uint64_t* ok, const uint64_t* ov,
                     const uint8_t* op, uint64_t nops);

/* Range scan ("search for the first key in the range and then traverse
 * leaf nodes until the last key is found"): for query i, the first up-to-k
 * pairs with lo[i] <= key <= hi[i] in key order.  out_keys/out_vals are m x k
 * row-major; unused slots are (MAX, 0); out_count[i] = pairs written. */
void orc_itree_range(const orc_itree* t, const uint64_t* lo, const uint64_t* hi, uint64_t m, uint32_t k,
                     uint64_t* out_keys, uint64_t* out_vals, uint32_t* out_count);
void orc_rtree_range(const orc_rtree* t, const uint64_t* lo, const uint64_t* hi, uint64_t m, uint32_t k,
                     uint64_t* out_keys, uint64_t* out_vals, uint32_t* out_count);

/* plain definition: lower_bound over sorted distinct keys */
void orc_lower_bound(const uint64_t* Kd, const uint64_t* Vd, uint64_t n,
                     const uint64_t* q, uint64_t m, uint64_t* pos_found, uint64_t* vals,
                     int nthreads);
#endif
