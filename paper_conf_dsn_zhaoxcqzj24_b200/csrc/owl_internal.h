/*
 * owl_internal.h — internal declarations of libowl (CUDA kernels <-> host runtime).  Not part of the ABI.
 *
 * Device A-DCFG tables are open-addressing hash tables of 32-byte cells {key_hi, key_lo, count, pad}
 * (one L2 sector per cell: probe, claim and count update touch one sector).  Keys pack the canonical
 * key so that ascending (key_hi, key_lo) as unsigned integers IS the canonical order:
 *   node   hi = slot<<32 | bb                         lo = 0
 *   edge   hi = slot<<32 | src                        lo = dst
 *   triple hi = slot<<32 | bb                         lo = prev<<32 | next
 *   addr   hi = slot<<48 | bb<<30 | ins<<22 | j       lo = x (the full 64-bit address word)
 * Field limits: slot < 0xFFFF, bb < 2^18 (record format), ins < 2^8, j < 2^22.  A real key never has
 * key_hi == ~0, so (~0, ~0) marks an empty cell.
 */
#ifndef OWL_INTERNAL_H
#define OWL_INTERNAL_H

#include <cuda_runtime.h>
#include <stdint.h>

#include <vector>

#include "owl.h"

#define OWL_EMPTY_KEY 0xFFFFFFFFFFFFFFFFull
#define OWL_MAX_SLOT 0xFFFEu
#define OWL_MAX_J ((1u << 22) - 1u)
#define OWL_NONE_BB 0xFFFFFFFEu /* "no basic block entered yet" */

enum { T_NODE = 0, T_EDGE = 1, T_TRIPLE = 2, T_ADDR = 3, T_NUM = 4 };

/* error codes written by kernels (low 3 bits of the packed error word) */
enum {
  KERR_NONE = 0,
  KERR_GWARP = 1,     /* gwarp >= n_warps                                  */
  KERR_BBFIELDS = 2,  /* BB_ENTRY with non-zero addr / lane / ins          */
  KERR_MTYPE = 3,     /* memory type > 8                                   */
  KERR_NOBB = 4,      /* MEM before the warp's first BB_ENTRY              */
  KERR_BBMISMATCH = 5 /* MEM bb != the warp's current BB                   */
};

/* Buckets of two cells, 64 B: both keys in the first 32-byte L2 sector (one 256-bit load probes the
   bucket), the two counts in the second.  Cell i = slot (i & 1) of bucket (i >> 1). */
struct owl_bucket {
  unsigned long long key[2][2]; /* [slot][hi, lo] */
  unsigned long long count[2];
  unsigned long long pad[2];
};

struct DevTable {
  owl_bucket* b;            /* cap / 2 buckets */
  unsigned long long* fill; /* number of claimed cells (device counter) */
  uint64_t cap;             /* cells: power of two, 2 .. 2^31 */
};
#define OWL_MAX_TABLE_CELLS (1ull << 31)

/* Shared device status of one fold launch */
struct FoldStatus {
  unsigned long long first_error;   /* min over errors of (seg<<40 | idx<<3 | code), ~0 = none      */
  unsigned long long not_warp_major;/* min (seg<<32 | gwarp) of a warp seen twice, ~0 = none         */
  unsigned int overflow;            /* bitmask of tables that exceeded their load limit             */
  unsigned int limit;               /* bitmask: 1 = slot/j field limit exceeded, 2 = visits map full */
  unsigned long long tile_counter;  /* persistent-kernel work counter                               */
  unsigned long long n_flush;       /* shared-memory pages allocated (all CTAs)                     */
  unsigned long long n_bypass;      /* address lane-adds served by shared-memory pages              */
  unsigned long long n_claim;       /* shared-table cells claimed                                   */
  unsigned long long dbg[8];        /* OWL_FOLD_STATS builds: fast / slow chunks, directory misses,
                                       directory claims, page admits, broadcast / page / global chunks */
};

/* One segment as the fold kernel sees it */
struct FoldSeg {
  const uint4* rec;   /* 16-byte records (device) */
  uint64_t n;         /* records */
  uint64_t tile0;     /* first global tile index of this segment */
  uint32_t slot;      /* evidence slot of this invocation */
  uint32_t n_warps;
  uint32_t* seen;     /* bitmap of n_warps bits (warp-major check), zeroed */
  unsigned long long* walked; /* records the fold walked in this segment, zeroed; = n iff every record was
                                 walked exactly once (with `seen`: the warp-major check) */
  uint32_t seg_index; /* position in the build's (run, seq)-sorted segment list */
  uint32_t _pad;
};

/* A channel-order segment walked in place (N2, fold_burst_kernel): its bursts in warp-major order (stable by stream
   position within a warp).  Burst k starts at virtual (warp-major) record bvs[k] and at physical record bpo[k] of
   FoldSeg::rec; bk[k] = its gwarp clamped to n_warps; nb bursts (FoldSeg::n = its records). */
struct FoldBurst {
  const uint32_t* bvs;
  const uint32_t* bpo;
  const uint32_t* bk;
  uint64_t nb;
};

/* A work item of the fold is (segment, tile position p): one warp folds the traced warps starting in tile p.
   The items of segment first_seg are item0 .. item0 + its number of tiles - 1. */
struct FoldGroup {
  uint64_t item0;     /* first work-item id of the segment */
  uint32_t first_seg; /* the segment's index in FoldArgs::segs */
  uint32_t _pad;
};

struct FoldArgs {
  const FoldSeg* segs;
  const FoldGroup* groups;
  uint32_t n_groups;
  uint32_t tile_shift;   /* tile = 1 << tile_shift records */
  uint64_t n_items;
  DevTable tab[T_NUM];
  FoldStatus* status;
  uint32_t* vmap; /* per-warp overflow visit maps (owl_fold_scratch_bytes(grid) bytes of device scratch) */
  uint32_t mode; /* experiment switch (OWL_FOLD_MODE): 0 normal, 1 no address inserts, 2 stream only */
};

/* ---- launchers (owl_fold.cu, owl_tables.cu, owl_ks.cu, owl_exchange.cu) ---- */
cudaError_t owl_launch_fold(const FoldArgs& a, int grid, cudaStream_t st);
/* in-place channel-order segments: bursts[i] describes a.segs[i] (owl_fold_burst.cu) */
cudaError_t owl_launch_fold_bursts(const FoldArgs& a, const FoldBurst* bursts, int grid, cudaStream_t st);
int owl_fold_ctas_per_sm();
size_t owl_fold_scratch_bytes(int grid);
int owl_fold_max_bbs(); /* distinct BBs one traced warp may visit */

struct Key128 {
  unsigned long long hi, lo;
};
/* A table compacted and sorted by (hi, lo): the canonical order.  Device arrays owned by the holder. */
struct SortedTable {
  Key128* k = nullptr;
  unsigned long long* c = nullptr;
  uint64_t n = 0;
};

cudaError_t owl_table_alloc(DevTable* t, uint64_t cap, cudaStream_t st);
void owl_table_free(DevTable* t);
cudaError_t owl_tables_sorted(const DevTable* t, int ntab, SortedTable* out, cudaStream_t st);
void owl_sorted_free(SortedTable* s);
/* inserts every cell of a sorted table into a hash table (evidence merge of partial builds / absorb) */
cudaError_t owl_table_insert_sorted(const DevTable& t, int tbl, const Key128* k, const unsigned long long* c,
                                    uint64_t n, FoldStatus* st_dev, cudaStream_t st);

/* A5 over all tables at once (canonical order), into malloc'd host rows with room for extra_rows more */
cudaError_t owl_diff_rows(const SortedTable* A, const SortedTable* B, int ntab, owl_diff** rows, uint64_t* n_rows,
                          size_t extra_rows, cudaStream_t st);

/* order-independent 128-bit fingerprint of the cells of ntab sorted tables (input-class filtering, N1) */
cudaError_t owl_tables_fingerprint(const SortedTable* tabs, int ntab, unsigned long long fp[2], cudaStream_t st);

/* Channel-order segments of one fold launch, bucketed by warp together (reading R17, N2): segment s's records in
   warp-major order at out + off[s]; per sorted burst, its source start (global index in the concatenation of the
   callers' segments) and its destination start in out. */
struct BucketedSet {
  uint4* out = nullptr;     /* copy mode: the segments' records in warp-major order, back to back */
  uint64_t* bsrc = nullptr;
  uint64_t* bdst = nullptr;
  uint64_t nb = 0;
  std::vector<uint64_t> off;
  /* in-place mode (out == nullptr): per sorted burst, segment-relative virtual start / physical start / clamped
     gwarp (u32: every segment < 2^32 records), and each segment's first sorted burst (bfirst[ns] = nb) */
  uint32_t* bvs = nullptr;
  uint32_t* bpo = nullptr;
  uint32_t* bk = nullptr;
  std::vector<uint64_t> bfirst;
  std::vector<const uint4*> rec; /* the callers' (or staged) segment arrays */
};
/* copy = false: the in-place burst index only (no warp-major copy); requires every segment < 2^32 records */
cudaError_t owl_bucket_segments(const std::vector<const uint4*>& rec, const std::vector<uint64_t>& n,
                                const std::vector<uint32_t>& n_warps, BucketedSet* out, cudaStream_t st,
                                bool copy = true);
void owl_bucketed_free(BucketedSet* b);
/* the first malformed record (caller's index in segment seg << 3 | KERR code, ~0 if none) of a bucketed set */
cudaError_t owl_first_bad_record(const BucketedSet& b, uint32_t seg, uint32_t n_warps, unsigned long long* idx_code,
                                 cudaStream_t st);

/* KS tests over one table kind (T_TRIPLE: H_cf per node; T_ADDR: H_addr per (bb, ins, j)) */
struct KsOutRow {
  unsigned long long hi_f, hi_r; /* attribute keys (fix / rnd side) */
  unsigned long long n, m, K_lo, K_hi;
  double D, p;
  uint32_t fail, _pad;
};
cudaError_t owl_ks_run(int tbl, const SortedTable& f, const SortedTable& r, const std::vector<uint32_t>& slot_f2r,
                       double significance, int hcf_reading, std::vector<KsOutRow>& rows, cudaStream_t st);

/* multi-GPU: pack every cell of the four sorted tables by owner rank */
struct ExchangeCell {
  unsigned long long hi, lo, count;
  uint32_t tbl, _pad;
};
cudaError_t owl_partition_cells(const SortedTable* tabs, int world, ExchangeCell** d_send, uint64_t* counts,
                                cudaStream_t st);
/* the same straight from the (unsorted) hash tables: no canonical sort before the exchange */
cudaError_t owl_partition_tables(const DevTable* tabs, int world, ExchangeCell** d_send, uint64_t* counts,
                                 cudaStream_t st);
cudaError_t owl_absorb_cells(const DevTable* tabs, const ExchangeCell* cells, uint64_t n, FoldStatus* st_dev,
                             cudaStream_t st);

/* device memory helpers (owl_tables.cu) */
void* owl_dev_alloc(size_t bytes);
void owl_dev_free(void* p);
void owl_dev_trim(int device); /* return cached blocks to CUDA */
void* owl_host_alloc(size_t bytes); /* pinned (cached) host block for result rows; owl_host_free releases it */
void owl_host_free(void* p);        /* pinned pool block or plain malloc block */

/* host-side key helpers */
static inline uint64_t owl_mix64(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return x;
}

#endif
