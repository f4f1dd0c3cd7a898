/*
 * owl_fold_body.cuh — A1-A3: stream trace records once and fold them thread -> warp -> kernel into the
 * A-DCFG hash tables (§V.A-B).
 *
 * Design v16 (the variants and their measurements: profiles/r01_v4_ab.txt, and for the round-2
 * redesign attempts profiles/r02_fold_experiments.txt).  The fold is an HBM stream whose per-record work must
 * fit the issue budget; at 24 warps per SM the register budget (80) binds, so every choice below minimises
 * instructions per 32-record chunk and live registers (what ptxas still spills stays in L1: the shared memory
 * below fits the 196 KB carve-out, see carveout()):
 *
 *  * persistent CTAs of FOLD_WARPS independent warps; a warp pops one work item (segment, tile of 2^15
 *    records) at a time from a global counter.  A tile holds the traced warps whose first record lies in
 *    it: the warp finds the first such start with a 33-ary warp-cooperative search and finishes the last
 *    traced warp past the tile end.  Every segment's walked records are counted (= n iff the warp-major
 *    layout held) and every traced warp start is marked in a bitmap (a warp seen twice is not warp-major);
 *  * a warp walks its traced warp FOLD_U chunks of 32 records at a time (one 128-bit streaming load per
 *    lane and chunk), with cp.async.bulk.prefetch.L2 keeping the next granules of its stream in flight;
 *  * A2: a chunk of 32 well-formed MEM records of the current basic block is the fast path (context
 *    warp-uniform).  A BB_ENTRY in lane 0 (chunks start on instruction boundaries) is consumed alone,
 *    inline: node / edge / triple cells go to per-kind shared tables (three lanes), the visit ordinal j
 *     comes from a visit map held in registers (lane l: one BB and its count; more than 32 BBs
 *    spill to a per-warp map in global scratch), and the rest of the step is realigned with a funnel
 *    shift across lanes instead of a reload.  Anything else (several entries, warp end, malformed
 *    records) takes the generic noinline slow path, which mirrors the oracle walk;
 *  * A3, "merging identical thread traces" before any global atomic: a broadcast chunk (32
 *    equal keys) is one add of 32; every lane then looks its key up on its own in the CTA directory
 *    (hot broadcast cells hold their count there; a hot 1 KB address window of one attribute owns a page
 *    of keyless 4-byte bins and the lane adds 1 to its bin).  Keys enter the directory on their ADMIT-th
 *    (6th) sighting, counted in a 4-way bucketed filter, so one-off windows never take pages.  Lanes that
 *    miss insert into the global open-addressing table: first probes of the step's chunks in flight
 *    together, counts added with fire-and-forget RED.64 in L2.
 *    The shared directory / pages / CF cells are exact partial sums, flushed to the global tables when the
 *    CTA finishes.  Directory and page counters close at SHARED_TOTAL_LIMIT walked records per CTA; the CF
 *    cells' 32-bit counters are bounded by the BB entries a CTA walks in one launch (< 2^32 for any launch
 *    that fits in device memory: at most 180 GB / 16 B = 1.1e10 records).
 * Malformed records are reported with the minimum (segment, index) and skipped (state unaffected),
 * exactly as the oracle does (bucketed channel-order segments are mapped back to the caller's order by
 * owl_first_bad_record after the fold).
 */
#include <cuda_runtime.h>
#include <stdint.h>

#include "owl_device.cuh"
#include "owl_internal.h"

using namespace owl_dev;

#define FULL 0xFFFFFFFFu
#ifndef FOLD_WARPS
#define FOLD_WARPS 24 /* profiles/r01_v4_ab.txt: U2 W24 beat U1-4 x W16-32 */
#endif
#ifndef FOLD_L1PF
#define FOLD_L1PF 1 /* prefetch each warp's next step into L1 (room for it since the 196 KB carve-out) */
#endif
#ifndef L1PF_STEPS
#define L1PF_STEPS 1 /* steps ahead */
#endif
#ifndef L1PF_LANES
#define L1PF_LANES 8 /* lanes 0..L1PF_LANES prefetch one 128 B line each */
#endif
#ifndef STEPS_IN_ST
#define STEPS_IN_ST 1 /* the per-step accounting counter lives in the high bits of the walker's state word (bits 8..31), not in a
                          register of its own: it was the one spill reloaded every step (profiles/r02_fold_experiments.txt #22) */
#endif
#ifndef FOLD_U
#define FOLD_U 2 /* chunks of 32 records per warp and step */
#endif
/* experiment modes (OWL_FOLD_MODE at run time in -DFOLD_RUNTIME_MODE builds, tools/): 1 no global-table
   inserts, 2 stream + walk only, 3 no L2 prefetch, 8 no shared counting; the product is mode 0 */
#ifdef FOLD_RUNTIME_MODE
#define FOLD_MODE_OF(a) ((a).mode)
#else
#define FOLD_MODE_OF(a) 0u
#endif
#define FOLD_THREADS (FOLD_WARPS * 32)
#define CFK 128      /* shared cells per CF table kind (node, edge, triple) */
#define CFK_LIMIT 96
#define VCAP 1024    /* per-warp overflow visit map in global scratch (BBs beyond the 32 held in registers) */
#define VGEN_MAX 0x3FFFu /* visit-map entry = gen<<18 | bb: a new generation per traced warp, 0 = empty */
#ifndef PF_LOG
#define PF_LOG 12    /* L2 bulk prefetch granule: 4 KB (256 records) */
#endif
#ifndef PF_DIST
#define PF_DIST 2    /* granules prefetched ahead of the walk */
#endif
#define PROBE_LIMIT 4096u
#ifndef NPAGE
#define NPAGE 160 /* with FILTER_LOG 10 the CTA's shared memory (198 KB) fits the 196 KB carve-out step (see carveout()) */
#endif
#define PAGE_BINS 256 /* 4-byte bins: one page counts the 1 KB address window x>>10 of one attribute */
#ifndef DIR_LOG
#define DIR_LOG 10
#endif
#ifndef FILTER_LOG
#define FILTER_LOG 10 /* admission filter: sightings of keys not (yet) in the directory */
#endif
#define DIRCAP (1 << DIR_LOG)
#define PAGE_TAG (3ull << 62) /* directory key lo of a page window: (x>>10) | PAGE_TAG (never a valid x) */
/* directory value of a page window: PV_PAGE | page id, or no page (0 while being admitted, PV_NONE
   once pages ran out); of a broadcast cell: its count */
#ifndef ADMIT
#define ADMIT 6u     /* a key enters the directory on its ADMIT-th sighting: recurring keys, not one-offs (sweep 2..32:
                        2 2345, 4 2392, 6 2388, 8 2375, 12 2346, 16 2317 GB/s on the C2 bench) */
#endif
#define PV_NONE 0x40000000u
#define PV_PAGE 0x80000000u
/* a CTA stops using shared counters once it has walked this many records (every shared counter is
   bounded by the records walked, so no 32-bit counter can wrap) */
#define SHARED_TOTAL_LIMIT (1ull << 31)

#ifdef OWL_FOLD_STATS
#define STAT(i) (++stat[i])
#else
#define STAT(i) ((void)0)
#endif

namespace {

/* per-warp fields read only at traced-warp / tile boundaries, in the slow path and on errors */
struct RunDesc {
  const uint4* rec; /* segment base */
  uint32_t* vk;     /* overflow visit map of this warp (global scratch): VCAP keys, then VCAP counts */
  const uint4* tile_end; /* traced warps starting at or after this belong to the next tile */
  uint32_t prev, curj;   /* walk context read only at BB entries (cur and khi stay in registers) */
  uint32_t gen;          /* generation of the traced warp in the overflow visit map */
  const uint4* p_acc;    /* records walked since the last accounting start here */
  uint32_t* seen;
  unsigned long long* seg_walked; /* records walked in this segment (all CTAs): must end = n */
  uint32_t slot, n_warps, seg_index;
#if FOLD_BURST
  /* in-place channel order (N2): rec / p_acc / tile_end are virtual (warp-major) positions; the segment's burst
     index; the warp's window of 32 bursts starts at burst wb (their starts / physical offsets sit in the walker's
     registers ws / wp), wend = the start of burst wb + 32 (or n) */
  const uint32_t* bvs;
  const uint32_t* bpo;
  const uint4* prec; /* the segment's physical records */
  uint64_t nb, wb;
  uint32_t n, wend;
#endif
};

struct __align__(16) FoldSmem {
  uint32_t page[NPAGE][PAGE_BINS];
  ulonglong2 dir_key[DIRCAP]; /* (attribute key hi, x) broadcast cell, or (hi, x>>10 | PAGE_TAG) window */
  uint32_t dir_val[DIRCAP];
  uint32_t filt[1 << FILTER_LOG]; /* 4-way buckets of tag<<8 | sightings of keys not in the directory */
  uint16_t page_dir[NPAGE];   /* page -> directory slot (final flush) */
  ulonglong2 cf_key[3][CFK];  /* node / edge / triple cells, one table per kind */
  unsigned int cf_cnt[3][CFK];
  unsigned int cf_fill[3];
  RunDesc rd[FOLD_WARPS];
  unsigned long long walked; /* records walked by the CTA */
  unsigned int npages;
  unsigned int off;          /* 1: shared counting closed (total limit, or experiment mode 8) */
};

/* Streaming record load: L1 bypassed, no L2 eviction hint (v16: the evict_first hint cost 1.8% once the bulk
   prefetch kept the stream ahead) */
__device__ __forceinline__ uint4 ld_stream(const uint4* p, uint64_t) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

/* L2 prefetch with normal eviction priority: the lines must survive until the walk's demand loads */
__device__ __forceinline__ void l2_prefetch_bulk(const void* p, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

/* 16-byte key load from L2 (.cg: no L1 allocation, so no stale copies of a cell claimed meanwhile) */
__device__ __forceinline__ ulonglong2 ld_key_weak(const unsigned long long* c) {
  ulonglong2 k;
  asm volatile("ld.global.cg.v2.u64 {%0, %1}, [%2];" : "=l"(k.x), "=l"(k.y) : "l"(c));
  return k;
}

__device__ __forceinline__ void red_add(unsigned long long* p, unsigned long long v) {
  asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

/* both keys of a bucket: one 256-bit load of its first 32-byte sector (predicated, no branch) */
__device__ __forceinline__ ulonglong4 ld_bucket_keys_if(bool pred, const owl_bucket* b) {
  ulonglong4 k;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %5, 0;\n\t"
      "mov.b64 %0, -1;\n\t"
      "mov.b64 %1, -1;\n\t"
      "mov.b64 %2, -1;\n\t"
      "mov.b64 %3, -1;\n\t"
      "@p ld.global.cg.v4.u64 {%0, %1, %2, %3}, [%4];\n\t}"
      : "=l"(k.x), "=l"(k.y), "=l"(k.z), "=l"(k.w)
      : "l"(b), "r"((int)pred));
  return k;
}
__device__ __forceinline__ void red_add_if(bool pred, unsigned long long* p, unsigned long long v) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %2, 0;\n\t"
      "@p red.relaxed.gpu.global.add.u64 [%0], %1;\n\t}" ::"l"(p),
      "l"(v), "r"((int)pred)
      : "memory");
}

/* probe continuation of an address-cell insert whose first probe (home bucket) missed; returns cells
   claimed */
__device__ __noinline__ uint32_t addr_insert_slow(const DevTable t, uint64_t h, uint64_t hi, uint64_t lo,
                                                  uint64_t c, FoldStatus* st) {
  const uint64_t mask = t.cap - 1;
  for (uint32_t probe = 0; probe < PROBE_LIMIT; ++probe) {
    unsigned long long* key = cell_key(t, h);
    const ulonglong2 k = ld_key_weak(key);
    if (k.x == hi && k.y == lo) {
      red_add(cell_count(t, h), c);
      return 0;
    }
    if (k.x == OWL_EMPTY_KEY || k.x == hi) { /* empty, being claimed, or a torn read: resolve with the CAS */
      const ulonglong2 o = cas128_global(key, OWL_EMPTY_KEY, OWL_EMPTY_KEY, hi, lo);
      if ((o.x == OWL_EMPTY_KEY && o.y == OWL_EMPTY_KEY) || (o.x == hi && o.y == lo)) {
        red_add(cell_count(t, h), c);
        return (o.x == OWL_EMPTY_KEY && o.y == OWL_EMPTY_KEY) ? 1u : 0u;
      }
    }
    h = (h + 1) & mask;
  }
  atomicOr(&st->overflow, 1u << T_ADDR); /* pathological clustering: regrow */
  return 0;
}

/* node / edge / triple cell += 1 in the CTA's table of kind `tbl` (T_NODE / T_EDGE / T_TRIPLE); lanes of
   one call may insert concurrently as long as they use different kinds (different arrays) */
__device__ __noinline__ void cf_insert(FoldSmem& s, const FoldArgs& a, int tbl, uint64_t hi, uint64_t lo) {
  ulonglong2* K = s.cf_key[tbl];
  uint32_t h = (((uint32_t)hi * 0x9E3779B1u) ^ ((uint32_t)(hi >> 32) * 0x85EBCA77u) ^ ((uint32_t)lo * 0xC2B2AE3Du) ^
                (uint32_t)(lo >> 32)) >> 25; /* CFK = 128 */
  for (int probe = 0; probe < CFK; ++probe) {
    const ulonglong2 k = K[h];
    if (k.x == hi && k.y == lo) {
      atomicAdd(&s.cf_cnt[tbl][h], 1u);
      return;
    }
    if (k.x == OWL_EMPTY_KEY) {
      if (*(volatile unsigned int*)&s.cf_fill[tbl] >= CFK_LIMIT) break;
      const ulonglong2 o = cas128_shared(&K[h], OWL_EMPTY_KEY, OWL_EMPTY_KEY, hi, lo);
      if ((o.x == OWL_EMPTY_KEY && o.y == OWL_EMPTY_KEY) || (o.x == hi && o.y == lo)) {
        if (o.x == OWL_EMPTY_KEY) atomicAdd(&s.cf_fill[tbl], 1u);
        atomicAdd(&s.cf_cnt[tbl][h], 1u);
        return;
      }
    }
    h = (h + 1) & (CFK - 1);
  }
  g_insert(a.tab[tbl], tbl, hi, lo, 1, a.status);
}

/* 32-bit mixed hash of a directory key: top DIR_LOG bits = home slot, low FILTER_LOG bits = filter slot */
__device__ __forceinline__ uint32_t dir_hash(uint64_t hi, uint64_t lo) {
  /* the keys of one program differ in few low bits (ins, j, window): a sum of multiplicative hashes of the
     four 32-bit words, then a finishing mix (xor-shift, multiply, xor-shift) so the top bits (home slot)
     depend on all of them */
  uint32_t h = (uint32_t)hi + (uint32_t)(hi >> 32) * 0x9E3779B1u + (uint32_t)lo * 0x85EBCA77u +
               (uint32_t)(lo >> 32) * 0xC2B2AE3Du;
  h ^= h >> 16;
  h *= 0x2C1B3C6Du;
  h ^= h >> 13;
  return h;
}
#ifndef DIR_PROBES
#define DIR_PROBES 4
#endif

/* Admission of a recurring key into the CTA directory (lane 0): claims the first free slot of h ..
   h+DIR_PROBES-1 (the slots lookups probe); a window then gets the next free page.  A key already
   present, or full slots, leave the directory unchanged. */
__device__ __noinline__ int dir_admit(FoldSmem& s, uint64_t hi, uint64_t lo, uint32_t h, bool window) {
  for (int probe = 0; probe < DIR_PROBES; ++probe) {
    const uint32_t hh = (h + probe) & (DIRCAP - 1);
    const ulonglong2 o = cas128_shared(&s.dir_key[hh], OWL_EMPTY_KEY, OWL_EMPTY_KEY, hi, lo);
    if (o.x == OWL_EMPTY_KEY && o.y == OWL_EMPTY_KEY) {
      if (window) {
        const unsigned n = atomicAdd(&s.npages, 1u);
        if (n < NPAGE) s.page_dir[n] = (uint16_t)hh;
        atomicExch(&s.dir_val[hh], n < NPAGE ? (PV_PAGE | n) : PV_NONE); /* pages were zeroed */
      }
      return 1;
    }
    if (o.x == hi && o.y == lo) return 2 + probe;
  }
  return 0;
}

__device__ __forceinline__ void report(FoldStatus* st, uint32_t seg_index, uint64_t idx, uint32_t code) {
  atomicMin(&st->first_error, ((unsigned long long)seg_index << 40) | (idx << 3) | code);
}

/* visits[b] += 1 in the warp's map; returns the new visit ordinal j (reading R8).  Entries of
   older generations (earlier traced warps) count as empty. */
__device__ __forceinline__ uint32_t visits_inc(uint32_t* vk, uint32_t* vc, uint32_t b, uint32_t gen, int lane,
                                               FoldStatus* st) {
  const uint32_t key = (gen << 18) | b;
  const uint32_t h = (b * 0x9E3779B1u) >> (32 - __ffs(VCAP) + 1); /* top log2(VCAP) bits */
  for (int w = 0; w < VCAP / 32; ++w) {
    const uint32_t pos = (h + w * 32 + lane) & (VCAP - 1);
    const uint32_t k = vk[pos];
    const unsigned found = __ballot_sync(FULL, k == key);
    const unsigned empty = __ballot_sync(FULL, (k >> 18) != gen);
    if (found | empty) {
      const bool hit = found && (!empty || __ffs(found) < __ffs(empty));
      const uint32_t p = (h + w * 32 + __ffs(hit ? found : empty) - 1) & (VCAP - 1);
      uint32_t j = 1;
      if (lane == 0) {
        if (hit) {
          j = vc[p] + 1;
          vc[p] = j;
        } else {
          vk[p] = key;
          vc[p] = 1;
        }
      }
      __syncwarp();
      return __shfl_sync(FULL, j, 0);
    }
  }
  if (lane == 0) atomicOr(&st->limit, 2u);
  return 1;
}

/* First traced-warp start in [b, e), or e if the tile begins inside a traced warp running past e. */
__device__ __forceinline__ uint64_t first_warp_start(const uint4* rec, uint64_t b, uint64_t e, int lane) {
  if (b == 0) return 0;
  const uint32_t gp = __ldg(&rec[b - 1].z);
  if (__ldg(&rec[b].z) != gp) return b;
  if (__ldg(&rec[e - 1].z) == gp) return e;
  uint64_t lo = b, hi = e - 1; /* rec[lo] == gp, rec[hi] != gp */
  while (hi - lo > 1) {
    const uint64_t p = lo + ((hi - lo) * (uint64_t)(lane + 1)) / 33u;
    const bool same = (p <= lo) ? true : (p >= hi ? false : (__ldg(&rec[p].z) == gp));
    const unsigned m = __ballot_sync(FULL, same);
    const unsigned nm = ~m;
    if (m && nm && 31 - __clz(m) > __ffs(nm) - 1) return b; /* not one contiguous run: not warp-major */
    const uint64_t plo = __shfl_sync(FULL, p, m ? 31 - __clz(m) : 0);
    const uint64_t phi = __shfl_sync(FULL, p, nm ? __ffs(nm) - 1 : 0);
    if (m && plo > lo) lo = plo;
    if (nm && phi < hi) hi = phi;
  }
  return hi;
}

/* Admissions of the keys whose sightings reached ADMIT (rare): one distinct key at a time, by lane 0. */
__device__ __noinline__ void admit_ready(FoldSmem& s, bool ready, uint64_t hi, uint64_t lo, uint32_t h0, uint32_t fi,
                                         bool window, int lane) {
  unsigned rm = __ballot_sync(FULL, ready);
  while (rm) {
    const int L = __ffs(rm) - 1;
    const uint64_t ah = __shfl_sync(FULL, hi, L), al = __shfl_sync(FULL, lo, L);
    const uint32_t ahh = __shfl_sync(FULL, h0, L), afi = __shfl_sync(FULL, fi, L);
    if (lane == 0) {
      dir_admit(s, ah, al, ahh, window);
      s.filt[afi] = 0;
    }
    rm &= ~__ballot_sync(FULL, hi == ah && lo == al);
  }
}

enum { W_INWARP = 2u, W_SKIP = 4u };

/* Per-warp walk state in registers (warp-uniform except vb / vn). */
struct Walker {
  const uint4* p;  /* next record */
  uint64_t khi;    /* slot<<48 | cur<<30 | curj: address key of the current context (ins added per chunk) */
  uint32_t g0, cur;
  uint32_t want;   /* meta of a fast-path record modulo lane and ins: MEM | cur<<8 (impossible when skipping) */
  uint32_t st;
  uint32_t vb, vn; /* visit map in registers: lane l holds BB vb and its visit count vn (32 BBs / warp) */
#if FOLD_BURST
  uint32_t ws, wp;  /* burst window: lane l holds the virtual start / physical offset of burst wb + l (n past nb) */
#endif
};

/* visits[b] += 1 for the traced warp; returns the new visit ordinal j (reading R8).  The first
   32 distinct BBs of a traced warp live in registers (one per lane), further ones in the shared map. */
__device__ __forceinline__ uint32_t visit(Walker& w, const RunDesc& d, uint32_t b, int lane,
                                          FoldStatus* st) {
  const unsigned m = __ballot_sync(FULL, w.vb == b);
  if (m) {
    const int L = __ffs(m) - 1;
    const uint32_t j = __shfl_sync(FULL, w.vn, L) + 1;
    if (lane == L) w.vn = j;
    return j;
  }
  const unsigned used = __ballot_sync(FULL, w.vb != 0xFFFFFFFFu);
  if (used != FULL) {
    if (lane == __ffs(~used) - 1) {
      w.vb = b;
      w.vn = 1;
    }
    return 1;
  }
  uint32_t* vk = d.vk;
  return visits_inc(vk, vk + VCAP, b, d.gen, lane, st);
}

struct SlowRes {
  Walker w;
  uint64_t khi, lo; /* key of this lane's record if good */
  int nproc;        /* records consumed */
  int good;
};

/* noinline (and everything by value): the slow path is rare, and keeping it out of the unrolled fast
   loop keeps the kernel within the instruction cache */
__device__ __noinline__ SlowRes slow_chunk(const uint4 r, const unsigned vm, Walker w, RunDesc& d,
                                           const FoldArgs& a, FoldSmem& s,
                                           const int lane) {
  bool good;
  uint64_t khi_out, lo_out;
  const int nvalid = vm == FULL ? 32 : __ffs(~vm) - 1;
  const bool active = lane < nvalid;
  int nproc = nvalid;
  const uint64_t idx = (uint64_t)(w.p - d.rec) + lane;
  const uint64_t addr = (uint64_t)r.x | ((uint64_t)r.y << 32);
  const uint32_t meta = r.w;
  const uint32_t bbf = (meta >> 8) & 0x3FFFFu;
  const uint32_t ins = meta & 0xFFu;
  good = false;
  khi_out = lo_out = 0;
  if (!(w.st & W_SKIP)) {
    const bool isbb = active && (meta >> 31) == 0;
    const bool bbbad = isbb && (addr != 0 || (meta & 0x7C0000FFu) != 0);
    if (bbbad) report(a.status, d.seg_index, idx, KERR_BBFIELDS);
    const unsigned bbmask = __ballot_sync(FULL, isbb && !bbbad);
    const uint32_t cur0 = w.cur, j0 = d.curj;
    uint32_t myj = 0;
    if (bbmask) {
      uint32_t prev = d.prev, curj = j0;
      const uint64_t slot_hi = (uint64_t)d.slot << 32;
      unsigned m = bbmask;
      while (m) {
        const int k = __ffs(m) - 1;
        m &= m - 1;
        const uint32_t b = __shfl_sync(FULL, bbf, k);
        if (FOLD_MODE_OF(a) == 0 && lane < 3) { /* node, edge, triple cell of this entry: one lane (and table) each */
          if (lane == T_NODE) cf_insert(s, a, T_NODE, slot_hi | b, 0);
          else if (lane == T_EDGE) /* S -> first BB, else cur -> b */
            cf_insert(s, a, T_EDGE, slot_hi | (w.cur == OWL_NONE_BB ? OWL_SENTINEL : w.cur), b);
          else if (w.cur != OWL_NONE_BB)
            cf_insert(s, a, T_TRIPLE, slot_hi | w.cur, ((uint64_t)prev << 32) | b);
        }
        if (w.cur != OWL_NONE_BB) prev = w.cur;
        w.cur = b;
        curj = visit(w, d, b, lane, a.status);
        if (lane == k) myj = curj;
      }
      w.khi = ((uint64_t)d.slot << 48) | ((uint64_t)w.cur << 30) | (uint64_t)curj;
      w.want = 0x80000000u | (w.cur << 8);
      if (curj > OWL_MAX_J && lane == 0) atomicOr(&a.status->limit, 1u);
      __syncwarp();
      d.prev = prev; /* every lane writes the same value */
      d.curj = curj;
      nproc = 32 - __clz(bbmask); /* consume up to the last BB_ENTRY: the next chunk starts aligned */
    }
    const bool ismem = lane < nproc && (meta >> 31) != 0;
    const unsigned lt = bbmask & ((1u << lane) - 1u);
    const int L = lt ? 31 - __clz(lt) : lane;
    uint32_t cbb = __shfl_sync(FULL, bbf, L);
    uint32_t cj = __shfl_sync(FULL, myj, L);
    if (!lt) {
      cbb = cur0;
      cj = j0;
    }
    uint32_t code = 0;
    if (ismem) {
      if ((addr >> 60) > 8) code = KERR_MTYPE;
      else if (cbb == OWL_NONE_BB) code = KERR_NOBB;
      else if (bbf != cbb) code = KERR_BBMISMATCH;
      if (code) report(a.status, d.seg_index, idx, code);
    }
    good = ismem && code == 0;
    if (good && cj > OWL_MAX_J) atomicOr(&a.status->limit, 1u);
    khi_out = ((uint64_t)d.slot << 48) | ((uint64_t)cbb << 30) | ((uint64_t)ins << 22) | cj;
    lo_out = addr;
  }
  w.p += nproc;
  if (nvalid < 32 && nproc == nvalid) { /* warp end: last BB -> S */
    if (FOLD_MODE_OF(a) == 0 && !(w.st & W_SKIP) && w.cur != OWL_NONE_BB && (lane == T_EDGE || lane == T_TRIPLE)) {
      const uint64_t hi = ((uint64_t)d.slot << 32) | w.cur;
      if (lane == T_EDGE) cf_insert(s, a, T_EDGE, hi, OWL_SENTINEL);
      else cf_insert(s, a, T_TRIPLE, hi, ((uint64_t)d.prev << 32) | OWL_SENTINEL);
    }
    w.st &= ~W_INWARP;
  }
  SlowRes res;
  res.w = w;
  res.khi = khi_out;
  res.lo = lo_out;
  res.nproc = nproc;
  res.good = good;
  return res;
}

#if FOLD_BURST
/* First traced-warp start (a burst index) in [b, e) of the sorted bursts, or e (bk: gwarp of each burst, clamped) */
__device__ __forceinline__ uint64_t first_burst_start(const uint32_t* bk, uint64_t b, uint64_t e, int lane) {
  if (b == 0) return 0;
  const uint32_t gp = __ldg(&bk[b - 1]);
  if (__ldg(&bk[b]) != gp) return b;
  if (__ldg(&bk[e - 1]) == gp) return e;
  uint64_t lo = b, hi = e - 1; /* bk[lo] == gp, bk[hi] != gp: the sorted keys of one warp are contiguous */
  while (hi - lo > 1) {
    const uint64_t p = lo + ((hi - lo) * (uint64_t)(lane + 1)) / 33u;
    const bool same = (p <= lo) ? true : (p >= hi ? false : (__ldg(&bk[p]) == gp));
    const unsigned m = __ballot_sync(FULL, same);
    const unsigned nm = ~m;
    const uint64_t plo = __shfl_sync(FULL, p, m ? 31 - __clz(m) : 0);
    const uint64_t phi = __shfl_sync(FULL, p, nm ? __ffs(nm) - 1 : 0);
    if (m && plo > lo) lo = plo;
    if (nm && phi < hi) hi = phi;
  }
  return hi;
}

/* (re)loads the warp's burst window at burst k */
__device__ __forceinline__ void burst_window_load(Walker& w, RunDesc& d, uint64_t k, int lane) {
  const bool in = k + lane < d.nb;
  w.ws = in ? __ldg(&d.bvs[k + lane]) : d.n;
  w.wp = in ? __ldg(&d.bpo[k + lane]) : 0u;
  const uint32_t we = k + 32 < d.nb ? __ldg(&d.bvs[k + 32]) : d.n;
  __syncwarp();
  d.wb = k; /* every lane writes the same values */
  d.wend = we;
  __syncwarp();
  /* L2 prefetch of the window's bursts 1..31: the window moves on when the walk reaches its burst BURST_SLIDE, so
     (but for the first window of a work item) every burst is prefetched at least 31 - BURST_SLIDE bursts ahead.
     Lane l prefetches the first 5 lines of burst l (a 32-record burst), one prefetch.global.L2 per line: per-lane
     cp.async.bulk.prefetch is serialised over the lanes. */
  const uint32_t e = __shfl_down_sync(FULL, w.ws, 1);
  const uint32_t end = lane == 31 ? we : e;
  if (lane >= 1 && w.ws < d.n) {
    const char* b0 = (const char*)(d.prec + w.wp);
    const char* b1 = (const char*)(d.prec + w.wp + (end - w.ws));
#pragma unroll
    for (int k = 0; k < 5; ++k)
      if (b0 + k * 128 < b1) asm volatile("prefetch.global.L2 [%0];" ::"l"(b0 + k * 128));
  }
}

/* the window position (0..31) of the burst holding virtual record v, the window moved to start there when v + 64
   would run past it (cold: about once per 32 bursts) */
__device__ __noinline__ int burst_slide(Walker& w, RunDesc& d, uint32_t v, int lane) {
  uint64_t k;
  if (v >= d.wend || __shfl_sync(FULL, w.ws, 0) > v) { /* v outside the window: binary search */
    uint64_t lo = 0, hi = d.nb; /* last burst with bvs <= v */
    while (hi - lo > 1) {
      const uint64_t mid = (lo + hi) >> 1;
      if (__ldg(&d.bvs[mid]) <= v) lo = mid; else hi = mid;
    }
    k = lo;
  } else {
    const unsigned m = __ballot_sync(FULL, w.ws <= v);
    k = d.wb + (31 - __clz(m));
  }
  burst_window_load(w, d, k, lane);
  return 0;
}

#ifndef BURST_SLIDE
#define BURST_SLIDE 24 /* the window also moves once the walk reaches its BURST_SLIDE-th burst (8 and 16 measured
                          slower: more window loads) */
#endif
__device__ __forceinline__ int burst_at(Walker& w, RunDesc& d, uint32_t v, int lane) {
  const uint32_t wend = d.wend;
  const unsigned m = __ballot_sync(FULL, w.ws <= v);
  const int j = 31 - __clz(m);
  if (m == 0 || j >= BURST_SLIDE || (wend <= v + 32 * FOLD_U - 1 && wend < d.n)) return burst_slide(w, d, v, lane);
  return j;
}

/* per-lane physical pointers of the step's FOLD_U chunks at virtual record v0 (nullptr at or past the segment end).
   Common case, the step within the three bursts from the one holding v0: their starts and physical offsets are
   shuffled from the window and each lane selects.  Otherwise (shorter bursts) the burst starts inside the step are
   one 64-bit mask (two warp OR-reductions), a lane's burst is the one holding v0 plus the starts at or before it. */
__device__ __forceinline__ void burst_step(Walker& w, RunDesc& d, uint32_t v0, int lane, const uint4* (&q)[FOLD_U]) {
  const int j0 = burst_at(w, d, v0, lane);
  const uint32_t n = d.n, wend = d.wend;
  { /* the step within three bursts (j0, j0 + 1, j0 + 2: bursts of at least ~21 records): a select per lane */
    const uint32_t s0 = __shfl_sync(FULL, w.ws, j0), p0 = __shfl_sync(FULL, w.wp, j0);
    const uint32_t a1 = __shfl_sync(FULL, w.ws, (j0 + 1) & 31), p1 = __shfl_sync(FULL, w.wp, (j0 + 1) & 31);
    const uint32_t a2 = __shfl_sync(FULL, w.ws, (j0 + 2) & 31), p2 = __shfl_sync(FULL, w.wp, (j0 + 2) & 31);
    const uint32_t a3 = __shfl_sync(FULL, w.ws, (j0 + 3) & 31);
    const uint32_t e0 = j0 + 1 < 32 ? a1 : wend, e1 = j0 + 2 < 32 ? a2 : wend, e2 = j0 + 3 < 32 ? a3 : wend;
    if (e2 >= v0 + 32 * FOLD_U || e2 >= n) {
#pragma unroll
      for (int u = 0; u < FOLD_U; ++u) {
        const uint32_t t = v0 + 32 * u + lane;
        const uint32_t off = t < e0 ? p0 + (t - s0) : (t < e1 ? p1 + (t - e0) : p2 + (t - e1));
        q[u] = t < n ? d.prec + off : nullptr;
      }
      return;
    }
  }
  const uint32_t rel = w.ws - v0;
  const bool inb = lane > j0 && rel < 32 * FOLD_U;
  const uint32_t blo = __reduce_or_sync(FULL, inb && rel < 32 ? 1u << (rel & 31) : 0u);
#if FOLD_U == 2
  const uint32_t bhi = __reduce_or_sync(FULL, inb && rel >= 32 ? 1u << (rel & 31) : 0u);
#endif
  const uint32_t le = (2u << lane) - 1u; /* lanes 0..lane */
#pragma unroll
  for (int u = 0; u < FOLD_U; ++u) {
    const uint32_t t = v0 + 32 * u + lane;
#if FOLD_U == 2
    const int src = j0 + (u == 0 ? __popc(blo & le) : __popc(blo) + __popc(bhi & le));
#else
    const int src = j0 + __popc(blo & le);
#endif
    const uint32_t sj = __shfl_sync(FULL, w.ws, src & 31), pj = __shfl_sync(FULL, w.wp, src & 31);
    q[u] = t >= n ? nullptr : d.prec + (pj + (t - sj));
    if (t < n && t >= wend) { /* past the window (bursts shorter than 2 records): this lane on its own */
      uint64_t lo = 0, hi = d.nb;
      while (hi - lo > 1) {
        const uint64_t mid = (lo + hi) >> 1;
        if (__ldg(&d.bvs[mid]) <= t) lo = mid; else hi = mid;
      }
      q[u] = d.prec + __ldg(&d.bpo[lo]) + (t - __ldg(&d.bvs[lo]));
    }
  }

}
#endif

__device__ __forceinline__ void begin_traced_warp(Walker& w, RunDesc& d, const FoldArgs& a,
                                                  int lane) {
#if FOLD_BURST
  {
    const uint32_t v = (uint32_t)(w.p - d.rec);
    const int j = burst_at(w, d, v, lane);
    w.g0 = __ldg(&d.prec[__shfl_sync(FULL, w.wp, j) + (v - __shfl_sync(FULL, w.ws, j))].z);
  }
#else
  w.g0 = __ldg(&w.p->z);
#endif
#if STEPS_IN_ST
  w.st = (w.st & ~0xFFu) | W_INWARP; /* (bits 8..31: steps since the last accounting) */
#else
  w.st = W_INWARP;
#endif
  if (w.g0 >= d.n_warps) { /* every record of this warp is malformed (the first one is reported) */
    if (lane == 0) report(a.status, d.seg_index, (uint64_t)(w.p - d.rec), KERR_GWARP);
    w.st |= W_SKIP;
  } else if (lane == 0) {
    const uint32_t bit = 1u << (w.g0 & 31);
    if (atomicOr(&d.seen[w.g0 >> 5], bit) & bit)
      atomicMin(&a.status->not_warp_major, ((unsigned long long)d.seg_index << 32) | w.g0);
  }
  __syncwarp();
  uint32_t gen = d.gen + 1;
  if (gen > VGEN_MAX) { /* generations wrapped: clear the map */
    for (int i = lane; i < VCAP; i += 32) d.vk[i] = 0;
    gen = 1;
  }
  __syncwarp();
  d.gen = gen; /* every lane writes the same values */
  d.prev = OWL_SENTINEL;
  d.curj = 0;
  __syncwarp();
  w.vb = 0xFFFFFFFFu;
  w.vn = 0;
  w.cur = OWL_NONE_BB;
  w.khi = 0;
  w.want = 1u; /* no record matches until the first BB_ENTRY (and never while skipping) */
}

__device__ __forceinline__ const FoldGroup& group_of(const FoldArgs& a, unsigned long long item) {
  uint32_t lo = 0, hi = a.n_groups; /* last group with item0 <= item */
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (a.groups[mid].item0 <= item) lo = mid; else hi = mid;
  }
  return a.groups[lo];
}

/* lane i of the result = record (i + k) of the 64-record window (lo, hi), 0 < k < 32 */
__device__ __forceinline__ uint4 funnel(const uint4 lo, const uint4 hi, int k, int lane) {
  const int src = (lane + k) & 31;
  const bool from_lo = lane + k < 32;
  uint4 r;
  const uint32_t ax = __shfl_sync(FULL, lo.x, src), bx = __shfl_sync(FULL, hi.x, src);
  const uint32_t ay = __shfl_sync(FULL, lo.y, src), by = __shfl_sync(FULL, hi.y, src);
  const uint32_t az = __shfl_sync(FULL, lo.z, src), bz = __shfl_sync(FULL, hi.z, src);
  const uint32_t aw = __shfl_sync(FULL, lo.w, src), bw = __shfl_sync(FULL, hi.w, src);
  r.x = from_lo ? ax : bx;
  r.y = from_lo ? ay : by;
  r.z = from_lo ? az : bz;
  r.w = from_lo ? aw : bw;
  return r;
}

#if FOLD_BURST
/* In-place channel-order segments (N2): the walk runs over each segment's virtual warp-major stream (its bursts
   sorted by warp, bursts[i] for segs[i]); loads go through the burst index; work items are blocks of
   2^tile_shift bursts.  Virtual positions are offsets from VBASE, never dereferenced. */
#define VBASE (reinterpret_cast<const uint4*>((uintptr_t)1 << 20))
__global__ void __launch_bounds__(FOLD_THREADS, 1) fold_burst_kernel(const FoldArgs args, const FoldBurst* bursts) {
#else
__global__ void __launch_bounds__(FOLD_THREADS, 1) fold_kernel(const FoldArgs args) {
#endif
  extern __shared__ __align__(16) unsigned char smem_raw[];
  FoldSmem& s = *reinterpret_cast<FoldSmem*>(smem_raw);
  __shared__ FoldArgs a; /* shared copy: helpers take it by reference without a local-memory copy */
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    a = args;
    s.npages = 0;
    s.off = FOLD_MODE_OF(args) == 8 ? 1u : 0u; /* experiment mode 8: global table only */
    s.walked = 0;
  }
  if (threadIdx.x < 3) s.cf_fill[threadIdx.x] = 0;
  for (int i = threadIdx.x; i < 3 * CFK; i += FOLD_THREADS) {
    (&s.cf_key[0][0])[i] = make_ulonglong2(OWL_EMPTY_KEY, OWL_EMPTY_KEY);
    (&s.cf_cnt[0][0])[i] = 0;
  }
  for (int i = threadIdx.x; i < NPAGE * PAGE_BINS / 4; i += FOLD_THREADS)
    reinterpret_cast<uint4*>(&s.page[0][0])[i] = make_uint4(0, 0, 0, 0);
  for (int i = threadIdx.x; i < DIRCAP; i += FOLD_THREADS) {
    s.dir_key[i] = make_ulonglong2(OWL_EMPTY_KEY, OWL_EMPTY_KEY);
    s.dir_val[i] = 0;
  }
  /* overflow visit map of this warp (global scratch, L1-cached; only this warp touches it) */
  {
    uint32_t* vk = args.vmap + ((size_t)blockIdx.x * FOLD_WARPS + warp) * (2 * VCAP);
    for (int i = lane; i < VCAP; i += 32) vk[i] = 0;
    if (lane == 0) {
      s.rd[warp].vk = vk;
      s.rd[warp].gen = 0;
    }
  }
  for (int i = threadIdx.x; i < (1 << FILTER_LOG); i += FOLD_THREADS) s.filt[i] = 0;
  __syncthreads();
  const uint64_t tile = 1ull << a.tile_shift;
  owl_bucket* const tab_b = a.tab[T_ADDR].b; /* the rest of the table descriptor is read from shared */
  const uint32_t shift = tab_shift(a.tab[T_ADDR].cap);
  RunDesc& d = s.rd[warp];
  uint32_t claims = 0;
#ifdef OWL_FOLD_STATS
  unsigned long long stat[8] = {0, 0, 0, 0, 0, 0, 0, 0};
#endif

  for (;;) {
    unsigned long long item = 0;
    if (lane == 0) {
      item = atomicAdd(&a.status->tile_counter, 1ull);
      if (*(volatile unsigned int*)&a.status->overflow) item = a.n_items;
    }
    item = __shfl_sync(FULL, item, 0);
    if (item >= a.n_items) break;
    const FoldGroup& g = group_of(a, item);
    const uint64_t b = (item - g.item0) * tile;
    const FoldSeg& sg = a.segs[g.first_seg];
#if FOLD_BURST
    const FoldBurst& sb = bursts[g.first_seg];
    if (b >= sb.nb) continue;
    const uint64_t e = b + tile < sb.nb ? b + tile : sb.nb;
    if (lane == 0) {
      d.rec = VBASE;
      d.seen = sg.seen;
      d.seg_walked = sg.walked;
      d.slot = sg.slot;
      d.n_warps = sg.n_warps;
      d.seg_index = sg.seg_index;
      d.bvs = sb.bvs;
      d.bpo = sb.bpo;
      d.prec = sg.rec;
      d.nb = sb.nb;
      d.n = (uint32_t)sg.n;
    }
    const uint4* const end = VBASE + sg.n;
    Walker w;
    {
      const uint64_t kb = first_burst_start(sb.bk, b, e, lane);
      const uint64_t ve = e < sb.nb ? __ldg(&sb.bvs[e]) : sg.n;
      if (lane == 0) d.tile_end = VBASE + ve;
      __syncwarp();
      burst_window_load(w, d, kb < sb.nb ? kb : sb.nb - 1, lane);
      w.p = VBASE + (kb < sb.nb ? __shfl_sync(FULL, w.ws, 0) : sg.n);
    }
#else
    if (b >= sg.n) continue;
    const uint64_t e = b + tile < sg.n ? b + tile : sg.n;
    if (lane == 0) {
      d.rec = sg.rec;
      d.seen = sg.seen;
      d.seg_walked = sg.walked;
      d.slot = sg.slot;
      d.n_warps = sg.n_warps;
      d.seg_index = sg.seg_index;
    }
    const uint4* const end = sg.rec + sg.n;
    if (lane == 0) d.tile_end = sg.rec + e;
    Walker w;
    w.p = sg.rec + first_warp_start(sg.rec, b, e, lane);
#endif
#if !STEPS_IN_ST
    uint32_t steps = 0; /* steps since the last accounting (a step walks <= 32 * FOLD_U records) */
#endif
    if (lane == 0) d.p_acc = w.p;
    w.st = 0;
    w.g0 = w.cur = 0;
    w.khi = 0;
    w.want = 1u;
    w.vb = 0xFFFFFFFFu;
    w.vn = 0;
    /* shared counting stays open while the CTA's walked records cannot wrap a 32-bit counter */
    bool shared_on = !*(volatile unsigned int*)&s.off;
    if (!FOLD_BURST && lane < PF_DIST && FOLD_MODE_OF(a) != 3) { /* prime the L2 prefetch window */
      const char* q = (const char*)(((((uintptr_t)w.p) >> PF_LOG) + lane) << PF_LOG);
      if (q < (const char*)end) {
        const uint64_t left = (uint64_t)((const char*)end - q);
        l2_prefetch_bulk(q, left < (1u << PF_LOG) ? (uint32_t)left : (1u << PF_LOG));
      }
    }
    __syncwarp();

    for (;;) {
      if (!(w.st & W_INWARP)) {
        if (w.p >= d.tile_end) break;
        begin_traced_warp(w, d, a, lane);
      }
#if STEPS_IN_ST
      if ((w.st += 256u) >= (1u << 24)) { /* very long traced warp: account as we go (steps in w.st bits 8..31) */
#else
      if (++steps >= (1u << 16)) { /* very long traced warp: account as we go */
#endif
        __syncwarp();
        if (lane == 0) {
          const unsigned long long n = (unsigned long long)(w.p - d.p_acc);
          if (atomicAdd(&s.walked, n) + n > SHARED_TOTAL_LIMIT) s.off = 1;
          atomicAdd(d.seg_walked, n);
          d.p_acc = w.p;
        }
        __syncwarp();
#if STEPS_IN_ST
        w.st &= 0xFFu;
#else
        steps = 0;
#endif
        shared_on = !*(volatile unsigned int*)&s.off;
      }
      uint4 rr[FOLD_U];
      const uint64_t pol = 0;
#if FOLD_BURST
      {
        const uint4* q[FOLD_U];
        burst_step(w, d, (uint32_t)(w.p - VBASE), lane, q);
#pragma unroll
        for (int u = 0; u < FOLD_U; ++u) rr[u] = q[u] ? ld_stream(q[u], pol) : make_uint4(0, 0, 0xFFFFFFFFu, 0);
      }
#else
      if (w.p + 32 * FOLD_U <= end) {
#pragma unroll
        for (int u = 0; u < FOLD_U; ++u) rr[u] = ld_stream(w.p + u * 32 + lane, pol);
      } else {
#pragma unroll
        for (int u = 0; u < FOLD_U; ++u) {
          const uint4* q = w.p + u * 32 + lane;
          rr[u] = q < end ? ld_stream(q, pol) : make_uint4(0, 0, 0xFFFFFFFFu, 0);
        }
      }
#endif
#if FOLD_L1PF && !FOLD_BURST
      { /* the next step's records into L1 (lanes 0..8: one 128 B line each); the streaming loads do not allocate in
           L1 but hit what is there (profiles/r02_fold_experiments.txt #25) */
        const char* q = (const char*)((((uintptr_t)(w.p + 32 * FOLD_U * L1PF_STEPS)) & ~(uintptr_t)127) +
                                      (uintptr_t)lane * 128);
        if (lane <= L1PF_LANES && q < (const char*)end) asm volatile("prefetch.global.L1 [%0];" ::"l"(q));
      }
#endif
      if (!FOLD_BURST && FOLD_MODE_OF(a) != 3) { /* keep PF_DIST granules of the stream in flight to L2 */
        const uintptr_t g1 = ((uintptr_t)(w.p + 32 * FOLD_U)) >> PF_LOG;
        if (g1 != (((uintptr_t)w.p) >> PF_LOG) && lane == 0) {
          const char* q = (const char*)((g1 + PF_DIST - 1) << PF_LOG);
          if (q < (const char*)end) {
            const uint64_t left = (uint64_t)((const char*)end - q);
            l2_prefetch_bulk(q, left < (1u << PF_LOG) ? (uint32_t)left : (1u << PF_LOG));
          }
        }
      }
      bool lead[FOLD_U];
      uint32_t cnt[FOLD_U];
      uint64_t khi[FOLD_U], klo[FOLD_U];
      bool stop = false; /* the traced warp ended inside the step: the rest is reloaded */
#pragma unroll
      for (int u = 0; u < FOLD_U; ++u) {
        lead[u] = false;
        cnt[u] = 1;
        if (stop) continue;
        const uint4 r = rr[u];
        /* fast path: a well-formed MEM record of the current BB of this traced warp */
        const bool ok = r.z == w.g0 && (r.w & 0x83FFFF00u) == w.want && r.y < 0x90000000u;
        if (__all_sync(FULL, ok)) {
          STAT(0);
          w.p += 32;
          khi[u] = w.khi | ((uint64_t)(r.w & 0xFFu) << 22);
          klo[u] = ((uint64_t)r.y << 32) | r.x;
          lead[u] = true;
          if (FOLD_MODE_OF(a) == 2) { /* experiment: stream + walk only */
            lead[u] = false;
            continue;
          }
          const uint32_t m0 = __shfl_sync(FULL, r.w, 0);
          const uint32_t x0l = __shfl_sync(FULL, r.x, 0), x0h = __shfl_sync(FULL, r.y, 0);
          const bool bc = __all_sync(FULL, ((r.w ^ m0) & 0xFFu) == 0 && r.x == x0l && r.y == x0h);
          if (bc) { /* broadcast: one cell, 32 adds (lane 0) */
            lead[u] = lane == 0;
            cnt[u] = 32;
          }
          if (shared_on) {
            /* per lane: the CTA directory holds (attribute, x) of hot broadcast cells and
               (attribute, x>>10) of hot 1 KB windows, each window owning a page of keyless 4-byte bins.
               Every lane decides for itself (no vote): a lane that misses goes to the global table. */
            const uint64_t lo = bc ? klo[u] : ((klo[u] >> 10) | PAGE_TAG);
            const uint32_t mh = dir_hash(khi[u], lo);
            const uint32_t h0 = mh >> (32 - DIR_LOG);
            uint32_t h = h0;
            ulonglong2 k = s.dir_key[h];
            bool f = k.x == khi[u] && k.y == lo;
            for (int probe = 1; probe < DIR_PROBES && !f && k.x != OWL_EMPTY_KEY; ++probe) {
              h = (h0 + probe) & (DIRCAP - 1);
              k = s.dir_key[h];
              f = k.x == khi[u] && k.y == lo;
            }
            if (f) {
              if (bc) {
                if (lane == 0) atomicAdd(&s.dir_val[h], 32u);
                lead[u] = false;
              } else {
                const uint32_t v = s.dir_val[h];
                if ((v & PV_PAGE) && (r.x & 3u) == 0) {
                  atomicAdd(&s.page[v & 0xFFFFu][(r.x >> 2) & (PAGE_BINS - 1)], 1u);
                  lead[u] = false;
                  STAT(6);
                }
              }
            }
            /* a key not in the directory: count a sighting, admit recurring keys (one vote skips it all
               for the usual chunk, whose lanes all hit) */
            const bool miss = !f && (!bc || lane == 0);
            if (__any_sync(FULL, miss)) {
            bool ready = false;
            uint32_t fi = 0;
            if (miss) {
              STAT(2);
              /* 4-way filter bucket: the key's entry, else the entry with the fewest sightings is replaced
                 (hot keys sharing a bucket do not evict each other); racy updates: counts are approximate */
              const uint32_t tag = mh & 0xFFFFFF00u;
              const uint32_t bi = mh & ((1u << (FILTER_LOG - 2)) - 1);
              const uint4 bk = reinterpret_cast<const uint4*>(s.filt)[bi];
              const uint32_t e0 = bk.x, e1 = bk.y, e2 = bk.z, e3 = bk.w;
              uint32_t way, ne;
              if ((e0 & 0xFFFFFF00u) == tag) { way = 0; ne = e0 + 1; }
              else if ((e1 & 0xFFFFFF00u) == tag) { way = 1; ne = e1 + 1; }
              else if ((e2 & 0xFFFFFF00u) == tag) { way = 2; ne = e2 + 1; }
              else if ((e3 & 0xFFFFFF00u) == tag) { way = 3; ne = e3 + 1; }
              else {
                const uint32_t c01 = min(e0 & 0xFFu, e1 & 0xFFu), c23 = min(e2 & 0xFFu, e3 & 0xFFu);
                way = c01 <= c23 ? ((e0 & 0xFFu) <= (e1 & 0xFFu) ? 0u : 1u) : ((e2 & 0xFFu) <= (e3 & 0xFFu) ? 2u : 3u);
                ne = tag | 1u;
              }
              fi = bi * 4 + way;
              s.filt[fi] = ne;
              ready = (ne & 0xFFu) >= ADMIT;
            }
            if (__any_sync(FULL, ready)) admit_ready(s, ready, khi[u], lo, h0, fi, !bc, lane);
            }
          }
        } else if (__shfl_sync(FULL, r.z == w.g0 && (r.w & 0xFC0000FFu) == 0 && r.x == 0 && r.y == 0, 0) &&
                   !(w.st & W_SKIP) && FOLD_MODE_OF(a) == 0) {
          /* the common slow chunk: a well-formed BB_ENTRY in lane 0 (chunks start on instruction
             boundaries).  Consume it alone, then realign the rest of the step. */
          STAT(1);
          const uint32_t b = (__shfl_sync(FULL, r.w, 0) >> 8) & 0x3FFFFu;
          const uint64_t slot_hi = (uint64_t)d.slot << 32;
          if (lane < 3) { /* node / edge / triple cell of this entry, one lane (and table) each */
            const bool first = w.cur == OWL_NONE_BB;
            const uint64_t hi = slot_hi | (lane == T_NODE ? b : (first ? OWL_SENTINEL : w.cur));
            const uint64_t lo = lane == T_NODE ? 0 : (lane == T_EDGE ? (uint64_t)b : (((uint64_t)d.prev << 32) | b));
            if (lane != T_TRIPLE || !first) cf_insert(s, a, lane, hi, lo);
          }
          __syncwarp();
          if (w.cur != OWL_NONE_BB) d.prev = w.cur; /* every lane writes the same value */
          w.cur = b;
          const uint32_t j = visit(w, d, b, lane, a.status);
          d.curj = j;
          if (j > OWL_MAX_J && lane == 0) atomicOr(&a.status->limit, 1u);
          w.khi = ((uint64_t)d.slot << 48) | ((uint64_t)b << 30) | (uint64_t)j;
          w.want = 0x80000000u | (b << 8);
          w.p += 1;
#pragma unroll
          for (int c = FOLD_U - 1; c > u; --c) rr[c] = funnel(rr[c - 1], rr[c], 1, lane);
        } else {
          STAT(1);
          const SlowRes sr = slow_chunk(r, __ballot_sync(FULL, r.z == w.g0 && w.p + lane < end), w, d, a, s,
                                        lane);
          w = sr.w;
          lead[u] = sr.good;
          khi[u] = sr.khi;
          klo[u] = sr.lo;
          const int k = sr.nproc;
          if (!(w.st & W_INWARP)) {
            stop = true;
          } else if (k < 32) {
            /* realign the rest of the step to the record after the consumed ones (no reload) */
#pragma unroll
            for (int c = FOLD_U - 1; c > u; --c) rr[c] = funnel(rr[c - 1], rr[c], k, lane);
          }
        }
      }
      bool mine = false; /* one vote per step: does any lane of any chunk go to the global table? */
#pragma unroll
      for (int u = 0; u < FOLD_U; ++u) mine = mine || lead[u];
      if (!__any_sync(FULL, mine) || FOLD_MODE_OF(a) == 1) continue;
      /* global table: first probes of all chunks in flight together, predicated REDs, rare misses */
      uint32_t home[FOLD_U];
      ulonglong4 kk[FOLD_U];
#pragma unroll
      for (int u = 0; u < FOLD_U; ++u) {
        home[u] = tab_index(khi[u], klo[u], shift);
        kk[u] = ld_bucket_keys_if(lead[u], tab_b + (home[u] >> 1));
      }
      bool missed = false;
#pragma unroll
      for (int u = 0; u < FOLD_U; ++u) {
        const bool h0 = kk[u].x == khi[u] && kk[u].y == klo[u];
        const bool h1 = kk[u].z == khi[u] && kk[u].w == klo[u];
        const bool hit = lead[u] && (h0 || h1);
        red_add_if(hit, &tab_b[home[u] >> 1].count[h1 ? 1 : 0], cnt[u]);
        lead[u] = lead[u] && !hit; /* now: missed (absent, or displaced past the home bucket) */
        missed = missed || lead[u];
      }
      if (__any_sync(FULL, missed)) {
#pragma unroll
        for (int u = 0; u < FOLD_U; ++u)
          if (lead[u]) claims += addr_insert_slow(a.tab[T_ADDR], home[u], khi[u], klo[u], cnt[u], a.status);
      }
    }
    /* records walked by this item bound every shared counter it touched */
    __syncwarp();
    if (lane == 0) {
      const unsigned long long n = (unsigned long long)(w.p - d.p_acc);
      if (atomicAdd(&s.walked, n) + n > SHARED_TOTAL_LIMIT) s.off = 1;
      if (n) atomicAdd(d.seg_walked, n);
    }
    /* cells claimed by this item -> table fill; past the load limit the build stops and regrows */
    if (__any_sync(FULL, claims != 0)) {
#pragma unroll
      for (int o = 16; o; o >>= 1) claims += __shfl_xor_sync(FULL, claims, o);
      if (lane == 0) {
        const DevTable& tab = a.tab[T_ADDR];
        const unsigned long long f = atomicAdd(tab.fill, (unsigned long long)claims) + claims;
        if (f > (tab.cap >> 1) + (tab.cap >> 2)) atomicOr(&a.status->overflow, 1u << T_ADDR);
        atomicAdd(&a.status->n_claim, (unsigned long long)claims);
      }
      claims = 0;
    }
  }
#ifdef OWL_FOLD_STATS
  if (lane == 0)
    for (int i = 0; i < 8; ++i) atomicAdd(&a.status->dbg[i], stat[i]);
#endif
  __syncthreads();
  /* flush the CTA's exact partial sums: pages, broadcast cells, CF cells */
  const unsigned np = s.npages < NPAGE ? s.npages : NPAGE;
  if (threadIdx.x == 0) atomicAdd(&a.status->n_flush, (unsigned long long)np);
  for (unsigned i = threadIdx.x; i < np * PAGE_BINS; i += FOLD_THREADS) {
    const unsigned pg = i / PAGE_BINS, b = i % PAGE_BINS;
    const uint32_t c = s.page[pg][b];
    if (c) {
      const ulonglong2 k = s.dir_key[s.page_dir[pg]];
      g_insert(a.tab[T_ADDR], T_ADDR, k.x, ((k.y & ~PAGE_TAG) << 10) | ((uint64_t)b << 2), c, a.status);
    }
  }
  for (int i = threadIdx.x; i < DIRCAP; i += FOLD_THREADS) {
    const ulonglong2 k = s.dir_key[i];
    const uint32_t c = s.dir_val[i];
    if (k.x != OWL_EMPTY_KEY && (k.y & PAGE_TAG) != PAGE_TAG && c) g_insert(a.tab[T_ADDR], T_ADDR, k.x, k.y, c, a.status);
  }
  for (int i = threadIdx.x; i < 3 * CFK; i += FOLD_THREADS) {
    const int tbl = i / CFK;
    const ulonglong2 k = s.cf_key[tbl][i % CFK];
    if (k.x != OWL_EMPTY_KEY) g_insert(a.tab[tbl], tbl, k.x, k.y, s.cf_cnt[tbl][i % CFK], a.status);
  }
}

}  // namespace

/* Preferred shared-memory carve-out (percent of the 228 KB maximum): the smallest that holds the CTA's shared memory
   (+ the static copy of the arguments and the 1 KB the system reserves), so the rest of the 256 KB per SM is L1.
   FoldSmem is sized to fit the 196 KB step (L1 ~60 KB instead of ~28 KB at 228 KB): +3-5% on C2 / C3 / C5
   (profiles/r02_fold_experiments.txt #20). */
static int carveout(size_t smem) { return (int)((smem + 2048) * 100 / (228 * 1024)); }
static_assert(sizeof(FoldSmem) + sizeof(FoldArgs) + 1024 <= 196 * 1024,
              "the fold's shared memory must fit the 196 KB carve-out step (else L1 shrinks to ~28 KB)");

#if FOLD_BURST
cudaError_t owl_launch_fold_bursts(const FoldArgs& a, const FoldBurst* bursts, int grid, cudaStream_t st) {
  const size_t smem = sizeof(FoldSmem);
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(fold_burst_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(fold_burst_kernel, cudaFuncAttributePreferredSharedMemoryCarveout, carveout(smem));
    if (e != cudaSuccess) return e;
    attr = true;
  }
  fold_burst_kernel<<<grid, FOLD_THREADS, smem, st>>>(a, bursts);
  return cudaGetLastError();
}
#else
int owl_fold_ctas_per_sm() { return 1; }
size_t owl_fold_scratch_bytes(int grid) { return (size_t)grid * FOLD_WARPS * 2 * VCAP * sizeof(uint32_t); }
int owl_fold_max_bbs() { return 32 + VCAP; }

cudaError_t owl_launch_fold(const FoldArgs& a, int grid, cudaStream_t st) {
  const size_t smem = sizeof(FoldSmem);
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(fold_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess) e = cudaFuncSetAttribute(fold_kernel, cudaFuncAttributePreferredSharedMemoryCarveout, carveout(smem));
    if (e != cudaSuccess) return e;
    attr = true;
  }
  fold_kernel<<<grid, FOLD_THREADS, smem, st>>>(a);
  return cudaGetLastError();
}
#endif
