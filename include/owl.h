/*
 * owl.h — C ABI of the B200-native hot path of Owl's differential side-channel detector
 * (Zhao et al., "Owl: Differential-based Side-Channel Leakage Detection for CUDA Applications",
 * DSN 2024).  Citations "P:L<n>" refer to lines of the paper text and name the
 * section / equation they fall in.  Readings of ambiguous passages are numbered R1..R20 and listed in
 * DESIGN.md §3 (they follow SURVEY.md §8(c)).
 *
 * The library (libowl.so) implements the data-parallel path
 *     records --(A1 ingest, A2 warp context, A3 group-by)--> per-run A-DCFG / class evidence
 *             --(A4 Myers run merge)--> E_fix, E_rnd --(A5 diff)--> differences
 *             --(A6 KS tests, A7 kernel test + localization)--> located leaks
 * with hand-written sm_100a CUDA kernels.  No torch types cross this boundary: every argument is a
 * plain pointer or size.  Every call returns an owl_status, never throws, and on error writes no
 * output; the cause is available from owl_last_error().
 *
 * Threading: one owl_ctx per GPU / rank, driven by one host thread at a time.
 */
#ifndef OWL_H
#define OWL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* owl_stream_t; /* == cudaStream_t; NULL = the legacy default stream */

typedef enum {
  OWL_OK = 0,
  OWL_ERR_INVALID_ARG = 1,     /* a NULL/ill-formed argument or an inconsistent segment set          */
  OWL_ERR_MALFORMED_TRACE = 2, /* a record violates the trace model of P:L185-191       */
  OWL_ERR_OUT_OF_MEMORY = 3,   /* device or host allocation failed                                   */
  OWL_ERR_CUDA = 4,            /* a CUDA runtime error (message has the CUDA error string)           */
  OWL_ERR_NCCL = 5,            /* reserved: collectives are issued by the caller (torch.distributed) */
  OWL_ERR_STATE = 6,           /* call not valid in the current state (e.g. run not ingested)        */
  OWL_ERR_CAPACITY = 7         /* a table or key field limit was exceeded even after regrowing       */
} owl_status;

/* ------------------------------------------------------------------------------------------------
 * Trace record (16 bytes, 16-byte aligned, little-endian; one 128-bit vector load on the GPU).
 *
 * Owl's device tracer emits one event when a warp enters a basic block (BB offset, warp ID, block ID)
 * and one per active thread per memory access (address, memory type) (§V.C).  Warps are
 * identified by (warp ID, block ID); addresses are converted to offsets inside their
 * cudaMalloc allocation.
 *
 *   addr   MEM:      [63:60] memory type (P:L219 fn.4 order: 0 None, 1 Local, 2 Generic, 3 Global,
 *                            4 Shared, 5 Constant, 6 Global_to_Shared, 7 Surface, 8 Texture; 9..15
 *                            are invalid) | [59:44] allocation id | [43:0] byte offset in allocation
 *          BB_ENTRY: 0
 *   gwarp  block_linear_id * warps_per_block + warp_in_block; must be < the segment's n_warps
 *   meta   [31]    kind: 0 = BB_ENTRY (one per warp per basic-block entry), 1 = MEM (one per active
 *                  thread per memory instruction)
 *          [30:26] lane (MEM; 0 for BB_ENTRY)
 *          [25:8]  bb: basic-block index inside the kernel (an 18-bit id, reading R18)
 *          [7:0]   ins: memory-instruction index inside bb (MEM; 0 for BB_ENTRY)
 * ---------------------------------------------------------------------------------------------- */
typedef struct {
  uint64_t addr;
  uint32_t gwarp;
  uint32_t meta;
} owl_record;

#define OWL_SENTINEL 0xFFFFFFFFu /* the special start/end basic block S (reading R7) */

enum { OWL_FIXED = 0, OWL_RANDOM = 1 }; /* input classes of the leakage-analysis phase */

enum {
  /* Records of each traced warp are contiguous in the buffer (any warp order).  Without this flag only
     per-warp program order is guaranteed (reading R17, a tracer channel's order) and the build first buckets
     the records by gwarp on the device: the runs of consecutive records of one warp ("bursts") are found in
     one streaming pass, the bursts (not the records) are sorted stably by warp and copied whole into a
     warp-major scratch buffer (the segment's bytes again, plus 9 B per burst). */
  OWL_SEG_WARP_MAJOR = 1u,
  /* `records` is a HOST pointer (pinned for asynchronous copies; pageable works but copies synchronously).
     owl_build_adcfg stages host segments in waves of at most owl_config.host_chunk_bytes (a wave holds at
     least one whole segment) through two device buffers: the copy of the next wave overlaps the fold of the
     current one, so device memory for host records stays at 2 x the largest wave.  A channel-order host
     segment is additionally bucketed by warp (its bytes again of scratch until the build returns). */
  OWL_SEG_HOST_RECORDS = 2u
};

/* One kernel invocation T_{k_i} of one run's program trace T_P. */
typedef struct {
  uint32_t run;               /* global run index; runs of a class are merged in ascending order   */
  uint32_t input_class;       /* OWL_FIXED / OWL_RANDOM                                           */
  uint32_t seq;               /* invocation index within the run (chronological order)    */
  uint32_t n_warps;           /* warps of the grid; every record has gwarp < n_warps              */
  uint64_t kernel_id;         /* call-stack hash at cuLaunchKernel                        */
  uint64_t n_records;
  const owl_record* records;  /* borrowed: caller owns; must stay valid until the build consuming it
                                 returns.  Device pointer unless OWL_SEG_HOST_RECORDS.              */
  uint32_t flags;             /* OWL_SEG_*                                                         */
  uint32_t _reserved;
} owl_segment;

typedef struct owl_ctx owl_ctx;
typedef struct owl_adcfg owl_adcfg; /* device-resident A-DCFG of one run, or a class evidence */

typedef struct {
  uint64_t addr_capacity;   /* initial hash capacity for address cells (0 = automatic)            */
  uint64_t cf_capacity;     /* initial hash capacity for node / edge / triple cells (0 = auto)    */
  uint32_t max_regrow;      /* times a build may double a full table and re-run (default 6)       */
  uint32_t fold_ctas_per_sm;/* 0 = automatic                                                      */
  uint64_t host_chunk_bytes;/* staging wave for OWL_SEG_HOST_RECORDS (0 = 256 MiB), see above        */
  uint32_t hcf_reading;     /* y-values of H_cf (SURVEY reading 5): OWL_HCF_COUNTS (0,
                               default) = joint counts c_ij; OWL_HCF_ROW_NORMALIZED (1) = the elements
                               a_ij = c_ij / x_i of the transition matrix A (Eqs. 7-8).  Other values:
                               OWL_ERR_INVALID_ARG from owl_ctx_set_config.                          */
  uint32_t channel_order;   /* segments without OWL_SEG_WARP_MAJOR (a tracer channel's order, reading R17,
                               P:L183, L211) are bucketed by warp on the device, by bursts
                               of consecutive records of one warp.  OWL_CHANNEL_AUTO (0, default) and
                               OWL_CHANNEL_IN_PLACE (2): no copy, the fold reads every record through the
                               burst index (needs every segment < 2^32 records, else the copy is used);
                               OWL_CHANNEL_COPY (1): the bursts are copied to a warp-major buffer first
                               (16 B per record of scratch).  Other values: OWL_ERR_INVALID_ARG.        */
} owl_config;
enum { OWL_CHANNEL_AUTO = 0u, OWL_CHANNEL_COPY = 1u, OWL_CHANNEL_IN_PLACE = 2u };

/* H_cf readings.  R2 weights each (src, dst) cell of a node by a_ij = c_ij / x_i, with
   x_i = sum_j c_ij the src count of Eq. 5, and tests F(t) = sum_{cells <= t} a / k (k = number of srcs,
   the sum of all a_ij) on both sides; D is fp64 (not an exact integer ratio), the KS row's K_lo = K_hi
   = 0, and n, m remain the node counts of Eq. 5. */
enum { OWL_HCF_COUNTS = 0, OWL_HCF_ROW_NORMALIZED = 1 };

/* Tables of an A-DCFG (§V.B).  Canonical key order in brackets. */
enum {
  OWL_TABLE_NODE = 0,   /* node (slot,bb): warp visits of the basic block                [slot,bb]           */
  OWL_TABLE_EDGE = 1,   /* edge (slot,src,dst): transitions incl. S->first, last->S      [slot,src,dst]      */
  OWL_TABLE_TRIPLE = 2, /* (slot,bb,prev,next): edge + its previous edge; H_cf cells
                           (Eqs. 5-8)                                                    [slot,bb,prev,next] */
  OWL_TABLE_ADDR = 3,   /* (slot,bb,ins,j,x): thread accesses of address x by instruction ins on the j-th
                           visit of bb (m_j)                               [slot,bb,ins,j,x]   */
  OWL_TABLE_SLOT = 4    /* (slot, kernel_id) -> invocation count (evidence)                           */
};

typedef struct {
  uint32_t input_class;
  uint32_t n_runs;
  uint32_t n_slots;
  uint32_t _pad;
  uint64_t n_cells[4];      /* node, edge, triple, addr */
  uint64_t n_records;       /* records folded into this A-DCFG */
} owl_adcfg_info;

/* One differing cell of two A-DCFGs (full outer join). Unused key fields = UINT32_MAX / 0. */
typedef struct {
  uint32_t table;           /* OWL_TABLE_* */
  uint32_t slot, bb, ins, j, prev, next, _pad;   /* edge rows: prev = src, next = dst */
  uint64_t x;               /* ADDR: address; SLOT: kernel_id */
  uint64_t count_a, count_b;
} owl_diff;

typedef enum { OWL_LEAK_KERNEL = 0, OWL_LEAK_CONTROL_FLOW = 1, OWL_LEAK_DATA_FLOW = 2 } owl_leak_kind;

/* One located leak (§VII.C). */
typedef struct {
  uint32_t kind;            /* owl_leak_kind */
  uint32_t slot_fix, slot_rnd;  /* UINT32_MAX where unaligned */
  uint32_t bb, ins, j;      /* UINT32_MAX where not applicable; DF: j = the min-p failing visit    */
  uint64_t kernel_id;
  uint64_t n, m;            /* KS sample sizes (kernel leaks: invocation counts fix / rnd)         */
  uint64_t K_lo, K_hi;      /* K = max_t |A_t*m - B_t*n| (exact, 128-bit)                          */
  double D, p;              /* KS statistic (Eq. 2) and Eq.-4 p-value; NaN for kernel leaks        */
} owl_leak;

/* One KS test (all tests, passing or failing), for inspection and parity checks. */
typedef struct {
  uint32_t kind;            /* OWL_LEAK_CONTROL_FLOW (H_cf per node) or OWL_LEAK_DATA_FLOW (H_addr) */
  uint32_t slot_fix, slot_rnd, bb, ins, j;  /* CF: ins = j = UINT32_MAX */
  uint64_t n, m, K_lo, K_hi;
  double D, p;
  uint32_t fail, _pad;
} owl_ks_row;

/* ---- context ----------------------------------------------------------------------------------- */
owl_status owl_ctx_create(int cuda_device, owl_ctx** out);
owl_status owl_ctx_destroy(owl_ctx* ctx);
owl_status owl_ctx_set_config(owl_ctx* ctx, const owl_config* cfg); /* NULL resets to defaults */

/* ---- A1: ingest ---------------------------------------------------------------------------------
 * Registers n_segs kernel invocations.  No record is read here; records are streamed by
 * the build.  (run, seq) must be unique; all segments of a run share input_class.  A run's segments
 * may arrive over several calls; its kernel sequence is the set of its segments ordered by seq.
 * All later device work of the context is enqueued on `stream`. */
owl_status owl_ingest_traces(owl_ctx* ctx, const owl_segment* segs, size_t n_segs, owl_stream_t stream);
/* Drops the registered segments of the given runs (so their buffers can be reused). */
owl_status owl_forget_runs(owl_ctx* ctx, const uint32_t* runs, size_t n_runs);

/* ---- A2-A4: build -------------------------------------------------------------------------------
 * Folds the records of the given runs (all of one input class) thread -> warp -> kernel into A-DCFGs
 * and merges the runs, in ascending run order, into one evidence with the Myers
 * alignment of their kernel sequences (reading R11).  One run gives that run's per-run
 * A-DCFG (slot = seq).  Synchronizes the context stream.  Malformed records fail the build with
 * OWL_ERR_MALFORMED_TRACE; the message names the segment and record index. */
owl_status owl_build_adcfg(owl_ctx* ctx, const uint32_t* runs, size_t n_runs, owl_adcfg** out);
/* Merges more runs (same class, every run > the runs already merged) into an existing evidence. */
owl_status owl_adcfg_accumulate(owl_ctx* ctx, owl_adcfg* g, const uint32_t* runs, size_t n_runs);
owl_status owl_adcfg_info_get(const owl_adcfg* g, owl_adcfg_info* info);
/* Canonical host dump (format in DESIGN.md §5): header, slot table in evidence order, then the four
 * tables sorted by key.  Writes to path if non-NULL; returns a library-allocated blob if host_blob is
 * non-NULL (free with owl_free). */
owl_status owl_adcfg_export(const owl_adcfg* g, const char* path_or_null, void** host_blob, size_t* bytes);
owl_status owl_adcfg_destroy(owl_adcfg* g);

/* ---- A5: diff -----------------------------------------------------------------------------------
 * Full outer join of two A-DCFGs on canonical keys; rows where the counts differ, in canonical order
 * (table, key).  Zero rows <=> identical traces (§VI). */
owl_status owl_diff_adcfg(owl_ctx* ctx, const owl_adcfg* a, const owl_adcfg* b, owl_diff** rows, size_t* n_rows);

/* ---- N1: input-class filtering -----------------------------------------------------
 * "inputs that generate identical traces [are] the same class ... the program [is] side-channel
 * leakage-free when there is only one class" (§VI).  Builds each run's A-DCFG (all of its
 * ingested segments; their input_class is ignored) and partitions the runs by identical A-DCFGs (same
 * kernel sequence, same node / edge / triple / address tables and counts).  Runs are visited in the
 * given order; class ids are assigned in order of first appearance, so a class's representative is its
 * first run (the paper picks one at random; reading R21).  class_of[i] receives the class of runs[i]
 * (caller-allocated, n_runs entries); *n_classes the number of classes (1 <=> leakage-free for these
 * inputs).  A 128-bit order-independent fingerprint of each run's cells buckets the runs on the device;
 * every membership is then confirmed by an exact comparison with the representative (A5 with zero
 * rows and equal slot tables), so the partition is exact.  Errors: INVALID_ARG (NULL, a run not
 * ingested or repeated), MALFORMED_TRACE / CAPACITY as for the build, CUDA. */
owl_status owl_filter_inputs(owl_ctx* ctx, const uint32_t* runs, size_t n_runs, uint32_t* class_of,
                             uint32_t* n_classes);

/* ---- A6-A7: leakage test ------------------------------------------------------------------------
 * Kernel test, then for every aligned slot pair one KS test (Eqs. 1-4) per node's
 * H_cf (Eqs. 5-8) and per (bb, ins, j) H_addr, both sides present.  A test fails
 * iff p < significance (reading R1: pass 0.05 for confidence 0.95).  Returns the located leaks sorted
 * kernel, CF, DF, each by (alignment position, bb, ins). */
owl_status owl_leak_test(owl_ctx* ctx, const owl_adcfg* e_fix, const owl_adcfg* e_rnd, double significance,
                         owl_leak** leaks, size_t* n_leaks);
/* Same tests, returning every KS row (pass or fail) in (alignment position, kind, bb, ins, j) order. */
owl_status owl_ks_tests(owl_ctx* ctx, const owl_adcfg* e_fix, const owl_adcfg* e_rnd, double significance,
                        owl_ks_row** rows, size_t* n_rows);

/* ---- multi-GPU (the collective is issued by the caller through torch.distributed / NCCL) ----------
 * owl_partition_evidence packs every cell of a partial evidence into `world` contiguous device buckets
 * by owner(attr) = mix64(attr) mod world, attr = bb for node/edge-by-src/triple cells and (bb,ins,j)
 * for address cells (no slot: both sides of an aligned fix/rnd slot pair meet on one rank whatever
 * their slot ids).  *d_send is a device buffer owned by the adcfg (valid until it is
 * destroyed); send_bytes[world] receives the bucket sizes (bytes, multiple of 32).
 * owl_absorb_evidence sums received buckets (laid out back to back in d_recv, recv_bytes[world]) into
 * a new evidence `owned` holding exactly the attributes this rank owns.  Slot ids must agree across
 * ranks (same runs' kernel sequences, see owl_assign_slots).  Integer sums: bit-identical to world=1.*/
owl_status owl_partition_evidence(owl_ctx* ctx, const owl_adcfg* partial, int world, void** d_send,
                                  uint64_t* send_bytes);
owl_status owl_absorb_evidence(owl_ctx* ctx, const owl_adcfg* like, const void* d_recv, const uint64_t* recv_bytes,
                               int world, int rank, owl_adcfg** owned);
/* Merge of the owners' result rows into the one-GPU result.  parts: the concatenation
 * of every owner's owl_leak_test rows (any order).  e_fix / e_rnd: this rank's evidences (any of them: the
 * slot tables are replicated).  Output, as owl_leak_test on one GPU: the kernel-leak rows (recomputed from
 * the slot tables), then CF rows, then DF rows, each by (alignment position, bb, ins); a DF location
 * whose visits j were tested on several owners keeps its min-p row, ties -> smallest j (reading
 * R14).  Errors: INVALID_ARG for a NULL argument or a row whose fix slot is not aligned in e_fix. */
owl_status owl_merge_leaks(owl_ctx* ctx, const owl_adcfg* e_fix, const owl_adcfg* e_rnd, const owl_leak* parts,
                           size_t n_parts, owl_leak** leaks, size_t* n_leaks);
/* Same for owl_diff_adcfg rows: the owners' table rows (disjoint) in canonical (table, key) order, then the
 * slot rows recomputed from a's and b's slot tables.  INVALID_ARG for a NULL argument or a bad table id. */
owl_status owl_merge_diffs(owl_ctx* ctx, const owl_adcfg* a, const owl_adcfg* b, const owl_diff* parts,
                           size_t n_parts, owl_diff** rows, size_t* n_rows);
/* Registers the kernel sequences of runs this rank does not hold (gathered from the other ranks) so
 * that Myers slot assignment (A4) sees every run of the class in global order. kernel_ids is the
 * concatenation of the runs' sequences; seq_len[i] is run i's length. */
owl_status owl_register_remote_runs(owl_ctx* ctx, const uint32_t* runs, const uint32_t* classes,
                                    const uint32_t* seq_len, const uint64_t* kernel_ids, size_t n_runs);

/* ---- measurement ---------------------------------------------------------------------------------
 * Fold-kernel statistics of the context: launches, the duration of the last fold launch measured with
 * CUDA events on the context stream, and the records it folded (plus running totals). */
owl_status owl_get_stats(const owl_ctx* ctx, uint64_t* fold_launches, double* last_fold_ms, uint64_t* last_fold_records,
                         double* total_fold_ms, uint64_t* total_fold_records);
owl_status owl_reset_stats(owl_ctx* ctx);

void owl_free(void* host_ptr);       /* frees rows / leaks / blobs allocated by the library */
const char* owl_last_error(void);    /* thread-local message for the last non-OK status      */
const char* owl_version(void);

#ifdef __cplusplus
}
#endif
#endif /* OWL_H */
