/*
 * owl_fold.cu — A1-A3: stream trace records once and fold them thread -> warp -> kernel into the
 * A-DCFG hash tables (§V.A-B).
 *
 * Design (measurements in profiles/):
 *
 *  * persistent CTAs of FOLD_WARPS independent warps; a warp pops one work item at a time from a global
 *    counter.  A work item is (group, tile p): a group holds up to FOLD_R segments of one evidence slot
 *    (consecutive runs of one class), and the warp walks tile p of every member AT ONCE — FOLD_R walkers
 *    whose state is warp-uniform and lives in registers, one 128-bit record load per lane per walker and
 *    step, so FOLD_R x 512 B are in flight per warp besides the L2 bulk prefetch that runs ahead;
 *  * a tile holds the traced warps whose first record lies in it: a walker that starts inside a traced
 *    warp finds the next warp start with a 33-ary warp-cooperative search, and the walker that owns a
 *    traced warp finishes it past the tile end;
 *  * per traced warp a walker takes the records 32 at a time (one per lane):
 *      A2  fast path: 32 MEM records of the current basic block — the key of lane i is
 *          (slot, cur, ins_i, j, x_i); the context (cur, j) is warp-uniform.  Chunks holding a BB_ENTRY,
 *          a warp end or a malformed record take the slow path, which applies the BB entries in lane
 *          order with warp-uniform state (cur, prev, the per-warp visit ordinal j of each BB in a
 *          shared-memory map), counts node / edge / triple cells in a small shared-memory table,
 *          and gives every MEM lane the context of the last BB_ENTRY lane before it;
 *      A3  "merging identical thread traces" at two levels before any atomic:
 *          - across runs: a fast-path chunk of walker r that is bit-identical to walker 0's chunk under
 *            the same context (same slot, BB, visit) adds its counts to walker 0's (exact: the records
 *            and the context ARE the key) — every FIX run of a deterministic program folds as one;
 *          - across lanes: consecutive lanes with equal keys (broadcast loads) form one add of their
 *            count;
 *          then one insert per distinct key into the global open-addressing table (32-byte cells, one L2
 *          sector each): the key probe is a plain (L1-cacheable) load — keys are immutable once
 *          claimed, a stale "empty" only sends the lane to the 128-bit CAS — and the count update is a
 *          fire-and-forget RED.64 in L2, where the hot cells of a trace stay resident (the record stream
 *          is loaded L2::evict_first).
 * Malformed records are reported with the minimum (segment, index) and skipped (state unaffected), exactly
 * as the oracle does.
 */
#include <cuda_runtime.h>
#include <stdint.h>
#ifdef OWL_DEBUG_CHECKS
#include <cstdio>
#endif

#include "owl_device.cuh"
#include "owl_internal.h"

using namespace owl_dev;

#define FULL 0xFFFFFFFFu
#ifndef FOLD_WARPS
#define FOLD_WARPS 16
#endif
#ifndef FOLD_U
#define FOLD_U 4 /* chunks of 32 records per warp and step */
#endif
#define FOLD_R 1
#define FOLD_THREADS (FOLD_WARPS * 32)
#define CF_CAP 512   /* shared node / edge / triple cells */
#define CF_LIMIT 384
#define VCAP 128     /* per-walker visit map (distinct BBs of one traced warp) */
#ifndef PF_LOG
#define PF_LOG 12    /* L2 bulk prefetch granule: 4 KB (256 records) */
#endif
#ifndef PF_DIST
#define PF_DIST 2    /* granules prefetched ahead of the walk */
#endif
#define PROBE_LIMIT 4096u
/* shared-memory paged histogram (keyless counting of hot narrow-range attributes) */
#ifndef NPAGE
#define NPAGE 168
#endif
#define PAGE_BINS 256       /* 4-byte bins: one page covers 1 KB of one attribute's address range */
#define DIR_LOG 10
#define DIRCAP (1 << DIR_LOG)
#define FILTER_CAP 1024
#define PAGE_TOTAL_LIMIT (1ull << 31)

namespace {

/* per-walker fields read only at traced-warp / tile boundaries and on errors */
struct RunDesc {
  const uint4* rec;      /* segment base */
  const uint4* end;      /* segment end */
  const uint4* tile_end; /* traced warps starting at or after this belong to the next tile */
  uint32_t* seen;
  uint32_t slot, n_warps, seg_index;
  uint32_t prev, curj;   /* walk context read only by the slow path (cur and khi stay in registers) */
};

struct __align__(16) FoldSmem {
  uint32_t page[NPAGE][PAGE_BINS]; /* keyless counters: bin b of page (attr, pg) counts x = pg<<10 | b<<2 */
  ulonglong2 dir_key[DIRCAP];      /* page directory: (address-key hi, x >> 10) -> page */
  int dir_page[DIRCAP];            /* -1: no page (yet) */
  uint32_t filter[FILTER_CAP];     /* second-touch admission: fingerprints of page keys seen once */
  uint16_t page_dir[NPAGE];        /* page -> directory slot (for the final flush) */
  ulonglong2 cf_key[CF_CAP];
  unsigned int cf_cnt[CF_CAP];
  uint32_t vkey[FOLD_WARPS][FOLD_R][VCAP];
  uint32_t vcnt[FOLD_WARPS][FOLD_R][VCAP];
  RunDesc rd[FOLD_WARPS][FOLD_R];
  unsigned long long page_total;   /* sum of all page adds: pages are closed before a counter could wrap */
  unsigned int cf_fill;
  unsigned int npages;
  unsigned int pages_off;
};

__device__ __forceinline__ uint64_t evict_first_policy() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}

__device__ __forceinline__ uint4 ld_stream(const uint4* p, uint64_t pol) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p), "l"(pol));
  return r;
}

/* L2 prefetch with normal eviction priority: the lines must survive until the walk's demand loads (which
   then mark them evict_first) */
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

/* predicated forms (no divergent branch around them) */
/* both keys of a bucket: one 256-bit load of its first 32-byte sector */
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

/* probe continuation of an address-cell insert whose first probe at `h` missed; returns cells claimed */
__device__ __noinline__ uint32_t addr_insert_slow(const DevTable t, uint32_t shift, uint64_t h, uint64_t hi,
                                                  uint64_t lo, uint64_t c, FoldStatus* st) {
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
  (void)shift;
  return 0;
}

/* node / edge / triple cells (the table id rides in key bits 62-63; slot < 2^16) */
__device__ __noinline__ void cf_insert(FoldSmem& s, const FoldArgs& a, int tbl, uint64_t hi, uint64_t lo) {
  const uint64_t thi = hi | ((uint64_t)tbl << 62);
  if (*(volatile unsigned int*)&s.cf_fill < CF_LIMIT) {
    uint32_t h = (uint32_t)(hmix(thi, lo) & (CF_CAP - 1));
    for (int probe = 0; probe < CF_CAP; ++probe) {
      const ulonglong2 o = cas128_shared(&s.cf_key[h], OWL_EMPTY_KEY, OWL_EMPTY_KEY, thi, lo);
      if (o.x == OWL_EMPTY_KEY && o.y == OWL_EMPTY_KEY) {
        atomicAdd(&s.cf_fill, 1u);
        atomicAdd(&s.cf_cnt[h], 1u);
        return;
      }
      if (o.x == thi && o.y == lo) {
        atomicAdd(&s.cf_cnt[h], 1u);
        return;
      }
      h = (h + 1) & (CF_CAP - 1);
    }
  }
  g_insert(a.tab[tbl], tbl, hi, lo, 1, a.status);
}

__device__ __forceinline__ uint32_t dir_hash(uint64_t hi, uint64_t pg) {
  return ((uint32_t)hi * 0x9E3779B1u) ^ ((uint32_t)(hi >> 32) * 0x85EBCA77u) ^ ((uint32_t)pg * 0xC2B2AE3Du) ^
         ((uint32_t)(pg >> 32) * 0x27D4EB2Fu);
}

/* Warp-uniform (every lane passes the same key): claims a page for page key (hi, pg), absent from its
   directory slots h, h+1, on the key's second sighting while pages last; -1 = none (the chunk goes to
   the global table).  Lane 0 decides, every lane gets its answer. */
__device__ __noinline__ int page_alloc(FoldSmem& s, uint64_t hi, uint64_t pg, uint32_t h, int lane) {
  int res = -1;
  if (lane == 0 && *(volatile unsigned int*)&s.npages < NPAGE && !*(volatile unsigned int*)&s.pages_off) {
    const uint32_t fp = dir_hash(hi, pg);
    volatile uint32_t* f = &s.filter[fp & (FILTER_CAP - 1)];
    if (*f != fp) {
      *f = fp; /* first sighting: remember it, count this chunk globally */
    } else {
      for (int probe = 0; probe < 2; ++probe) {
        const uint32_t hh = (h + probe) & (DIRCAP - 1);
        const ulonglong2 o = cas128_shared(&s.dir_key[hh], OWL_EMPTY_KEY, OWL_EMPTY_KEY, hi, pg);
        if (o.x == OWL_EMPTY_KEY && o.y == OWL_EMPTY_KEY) {
          const unsigned n = atomicAdd(&s.npages, 1u);
          if (n < NPAGE) {
            res = (int)n;
            s.page_dir[n] = (uint16_t)hh;
          }
          *(volatile int*)&s.dir_page[hh] = res; /* pages were zeroed at kernel start */
          break;
        }
        if (o.x == hi && o.y == pg) break; /* claimed meanwhile by another warp: its page id may not be
                                              published yet; this chunk goes global */
      }
    }
  }
  return __shfl_sync(FULL, res, 0);
}

__device__ __forceinline__ void report(FoldStatus* st, uint32_t seg_index, uint64_t idx, uint32_t code) {
  atomicMin(&st->first_error, ((unsigned long long)seg_index << 40) | (idx << 3) | code);
}

/* visits[b] += 1 in the walker's map; returns the new visit ordinal j (reading R8) */
__device__ __forceinline__ uint32_t visits_inc(uint32_t* vk, uint32_t* vc, uint32_t b, int lane, FoldStatus* st) {
  const uint32_t h = (b * 0x9E3779B1u) >> 25; /* VCAP = 128 */
  for (int w = 0; w < VCAP / 32; ++w) {
    const uint32_t pos = (h + w * 32 + lane) & (VCAP - 1);
    const uint32_t k = vk[pos];
    const unsigned found = __ballot_sync(FULL, k == b);
    const unsigned empty = __ballot_sync(FULL, k == 0xFFFFFFFFu);
    if (found | empty) {
      const bool hit = found && (!empty || __ffs(found) < __ffs(empty));
      const uint32_t p = (h + w * 32 + __ffs(hit ? found : empty) - 1) & (VCAP - 1);
      uint32_t j = 1;
      if (lane == 0) {
        if (hit) {
          j = vc[p] + 1;
          vc[p] = j;
        } else {
          vk[p] = b;
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
    const uint64_t plo = __shfl_sync(FULL, p, m ? 31 - __clz(m) : 0);
    const uint64_t phi = __shfl_sync(FULL, p, nm ? __ffs(nm) - 1 : 0);
    if (m && plo > lo) lo = plo;
    if (nm && phi < hi) hi = phi;
  }
  return hi;
}

enum { W_ACTIVE = 1u, W_INWARP = 2u, W_SKIP = 4u };

/* Per-walker state in registers (warp-uniform). */
struct Walker {
  const uint4* p;   /* next record */
  uint64_t khi;     /* slot<<48 | cur<<30 | curj: the address key of the current context (ins added per lane) */
  uint32_t g0, cur;
  uint32_t st;
};

/* Slow path of one chunk (BB entries, warp end, malformed records): applies the BB entries, computes the
   key of every good MEM lane, advances the walker.  Mirrors the oracle walk. */
__device__ __forceinline__ void slow_chunk(const uint4 r, const unsigned vm, Walker& w, RunDesc& d,
                                           const FoldArgs& a, FoldSmem& s, uint32_t* vk, uint32_t* vc,
                                           const int lane, bool& good, uint64_t& khi_out, uint64_t& lo_out) {
  const int nvalid = vm == FULL ? 32 : __ffs(~vm) - 1;
  const bool active = lane < nvalid;
  int nproc = nvalid; /* records consumed: up to the last BB_ENTRY, so the next chunk starts on an
                         instruction boundary (one attribute per fast chunk) */
  const uint64_t idx = (uint64_t)(w.p - d.rec) + lane;
  const uint64_t addr = (uint64_t)r.x | ((uint64_t)r.y << 32);
  const uint32_t meta = r.w;
  const uint32_t bbf = (meta >> 8) & 0x3FFFFu;
  const uint32_t ins = meta & 0xFFu;
  good = false;
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
        if (a.mode == 0 && lane == 0) {
          if (w.cur == OWL_NONE_BB) {
            cf_insert(s, a, T_EDGE, slot_hi | OWL_SENTINEL, b); /* S -> first BB */
          } else {
            cf_insert(s, a, T_EDGE, slot_hi | w.cur, b);       /* cur -> b */
            cf_insert(s, a, T_TRIPLE, slot_hi | w.cur, ((uint64_t)prev << 32) | b);
          }
          cf_insert(s, a, T_NODE, slot_hi | b, 0);
        }
        if (w.cur != OWL_NONE_BB) prev = w.cur;
        w.cur = b;
        curj = visits_inc(vk, vc, b, lane, a.status);
        if (lane == k) myj = curj;
      }
      w.khi = ((uint64_t)d.slot << 48) | ((uint64_t)w.cur << 30) | (uint64_t)curj;
      if (curj > OWL_MAX_J && lane == 0) atomicOr(&a.status->limit, 1u);
      __syncwarp();
      if (lane == 0) {
        d.prev = prev;
        d.curj = curj;
      }
      __syncwarp();
    }
    if (bbmask) nproc = 32 - __clz(bbmask);
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
    if (a.mode == 0 && !(w.st & W_SKIP) && w.cur != OWL_NONE_BB && lane == 0) {
      cf_insert(s, a, T_EDGE, ((uint64_t)d.slot << 32) | w.cur, OWL_SENTINEL);
      cf_insert(s, a, T_TRIPLE, ((uint64_t)d.slot << 32) | w.cur, ((uint64_t)d.prev << 32) | OWL_SENTINEL);
    }
    w.st &= ~W_INWARP;
  }
}

__device__ __forceinline__ void begin_traced_warp(Walker& w, RunDesc& d, const FoldArgs& a, uint32_t* vk,
                                                  int lane) {
  w.g0 = __ldg(&w.p->z);
  w.st = (w.st & ~W_SKIP) | W_INWARP;
  if (w.g0 >= d.n_warps) { /* every record of this warp is malformed (the first one is reported) */
    if (lane == 0) report(a.status, d.seg_index, (uint64_t)(w.p - d.rec), KERR_GWARP);
    w.st |= W_SKIP;
  } else if (lane == 0) {
    const uint32_t bit = 1u << (w.g0 & 31);
    if (atomicOr(&d.seen[w.g0 >> 5], bit) & bit)
      atomicMin(&a.status->not_warp_major, ((unsigned long long)d.seg_index << 32) | w.g0);
  }
  for (int i = lane; i < VCAP; i += 32) vk[i] = 0xFFFFFFFFu;
  if (lane == 0) {
    d.prev = OWL_SENTINEL;
    d.curj = 0;
  }
  __syncwarp();
  w.cur = OWL_NONE_BB;
  w.khi = 0;
}

__device__ __forceinline__ const FoldGroup& group_of(const FoldArgs& a, unsigned long long item) {
  uint32_t lo = 0, hi = a.n_groups; /* last group with item0 <= item */
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (a.groups[mid].item0 <= item) lo = mid; else hi = mid;
  }
  return a.groups[lo];
}

__global__ void __launch_bounds__(FOLD_THREADS, 1) fold_kernel(const FoldArgs args) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  FoldSmem& s = *reinterpret_cast<FoldSmem*>(smem_raw);
  __shared__ FoldArgs a; /* shared copy: helpers take it by reference without a local-memory copy */
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    a = args;
    s.cf_fill = 0;
    s.npages = 0;
    s.pages_off = args.mode == 8 ? 1u : 0u; /* experiment mode 8: global table only */
    s.page_total = 0;
  }
  for (int i = threadIdx.x; i < CF_CAP; i += FOLD_THREADS) {
    s.cf_key[i] = make_ulonglong2(OWL_EMPTY_KEY, OWL_EMPTY_KEY);
    s.cf_cnt[i] = 0;
  }
  for (int i = threadIdx.x; i < NPAGE * PAGE_BINS; i += FOLD_THREADS) (&s.page[0][0])[i] = 0;
  for (int i = threadIdx.x; i < DIRCAP; i += FOLD_THREADS) {
    s.dir_key[i] = make_ulonglong2(OWL_EMPTY_KEY, OWL_EMPTY_KEY);
    s.dir_page[i] = -1;
  }
  for (int i = threadIdx.x; i < FILTER_CAP; i += FOLD_THREADS) s.filter[i] = 0;
  __syncthreads();
  const uint64_t pol = evict_first_policy();
  const uint64_t tile = 1ull << a.tile_shift;
  const DevTable tab = a.tab[T_ADDR];
  const uint32_t shift = tab_shift(tab.cap);
  RunDesc& d = s.rd[warp][0];
  uint32_t* vk = s.vkey[warp][0];
  uint32_t* vc = s.vcnt[warp][0];
  uint32_t claims = 0;
  unsigned long long ptot = 0; /* this warp's page adds since the last item end */
  uint32_t padds = 0;          /* lane-adds served by pages (statistics) */

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
    if (b >= sg.n) continue;
    const uint64_t e = b + tile < sg.n ? b + tile : sg.n;
    if (lane == 0) {
      d.rec = sg.rec;
      d.end = sg.rec + sg.n;
      d.tile_end = sg.rec + e;
      d.seen = sg.seen;
      d.slot = sg.slot;
      d.n_warps = sg.n_warps;
      d.seg_index = sg.seg_index;
    }
    const uint4* const end = sg.rec + sg.n;
#ifdef OWL_DEBUG_CHECKS
    if (b > sg.n || e > sg.n) { printf("bad tile b %llu e %llu n %llu\n", (unsigned long long)b, (unsigned long long)e, (unsigned long long)sg.n); __trap(); }
#endif
    const uint4* const tile_end = sg.rec + e;
    Walker w;
    w.p = sg.rec + first_warp_start(sg.rec, b, e, lane);
    w.st = W_ACTIVE;
    w.g0 = w.cur = 0;
    w.khi = 0;
    if (lane < PF_DIST && a.mode != 3) { /* prime the L2 prefetch window */
      const char* q = (const char*)(((((uintptr_t)w.p) >> PF_LOG) + lane) << PF_LOG);
      if (q < (const char*)end) {
        const uint64_t left = (uint64_t)((const char*)end - q);
        l2_prefetch_bulk(q, left < (1u << PF_LOG) ? (uint32_t)left : (1u << PF_LOG));
      }
    }
    __syncwarp();

    for (;;) {
      if (!(w.st & W_INWARP)) {
        if (w.p >= tile_end) break;
        begin_traced_warp(w, d, a, vk, lane);
      }
      /* FOLD_U chunks of 32 records: one 128-bit load per lane per chunk */
      uint4 rr[FOLD_U];
#pragma unroll
      for (int u = 0; u < FOLD_U; ++u) {
        const uint4* q = w.p + u * 32 + lane;
        rr[u] = q < end ? ld_stream(q, pol) : make_uint4(0, 0, 0xFFFFFFFFu, 0);
      }
      if (a.mode != 3) { /* keep PF_DIST granules of the stream in flight to L2 */
        const uintptr_t g1 = ((uintptr_t)(w.p + 32 * FOLD_U)) >> PF_LOG;
        if (g1 != (((uintptr_t)w.p) >> PF_LOG) && lane == 0) {
          const char* q = (const char*)((g1 + PF_DIST - 1) << PF_LOG);
          if (q < (const char*)end) {
            const uint64_t left = (uint64_t)((const char*)end - q);
            l2_prefetch_bulk(q, left < (1u << PF_LOG) ? (uint32_t)left : (1u << PF_LOG));
          }
        }
      }
      /* fast path: every record of the U chunks is a well-formed MEM record of the current BB */
      const uint32_t want = 0x80000000u | (w.cur << 8);
      bool ok = !(w.st & W_SKIP) && (w.p + 32 * FOLD_U <= end);
#pragma unroll
      for (int u = 0; u < FOLD_U; ++u)
        ok = ok && rr[u].z == w.g0 && (rr[u].w & 0x83FFFF00u) == want && rr[u].y < 0x90000000u;
      bool good[FOLD_U], fastc[FOLD_U];
      uint64_t khi[FOLD_U], klo[FOLD_U];
      if (__all_sync(FULL, ok)) {
#pragma unroll
        for (int u = 0; u < FOLD_U; ++u) {
          good[u] = fastc[u] = true;
          khi[u] = w.khi | ((uint64_t)(rr[u].w & 0xFFu) << 22);
          klo[u] = (uint64_t)rr[u].x | ((uint64_t)rr[u].y << 32);
        }
        w.p += 32 * FOLD_U;
      } else {
        bool live = true; /* false once the traced warp ended inside this batch: later chunks are reloaded */
#pragma unroll
        for (int u = 0; u < FOLD_U; ++u) {
          good[u] = fastc[u] = false;
          khi[u] = klo[u] = 0;
          if (!live) continue;
          const bool valid = (w.p + lane < end) && rr[u].z == w.g0;
          const bool fast_ok = valid && (rr[u].w & 0x83FFFF00u) == want && rr[u].y < 0x90000000u;
          if (__all_sync(FULL, fast_ok) && !(w.st & W_SKIP)) {
            good[u] = fastc[u] = true;
            khi[u] = w.khi | ((uint64_t)(rr[u].w & 0xFFu) << 22);
            klo[u] = (uint64_t)rr[u].x | ((uint64_t)rr[u].y << 32);
            w.p += 32;
          } else {
            const uint4* p0 = w.p;
            slow_chunk(rr[u], __ballot_sync(FULL, valid), w, d, a, s, vk, vc, lane, good[u], khi[u], klo[u]);
            live = (w.st & W_INWARP) != 0 && w.p == p0 + 32; /* else later chunks are reloaded */
          }
        }
      }
      if (a.mode != 0 && a.mode < 5) continue; /* experiment modes: 5 probe only, 6 RED only, 7 no RED */

      /* A3, "merge identical thread traces" before any atomic:
         - a fast chunk whose 32 keys are equal (broadcast access) is one add of 32;
         - otherwise the chunk (one attribute after realignment) looks its page key up in the CTA's
           page directory (branch-free 2-slot probe, same address for every lane: a broadcast read) and
           the lanes of that page add into shared-memory bins; a missing page is allocated on the key's
           second sighting (lane 0, rare);
         - what is left (slow chunks, pages exhausted, wide-range or unaligned addresses) goes to the
           global table: first probes of all chunks in flight together, predicated REDs, rare misses. */
      bool lead[FOLD_U];
      uint32_t cnt[FOLD_U];
      unsigned any_lead = 0;
#pragma unroll
      for (int u = 0; u < FOLD_U; ++u) {
        lead[u] = good[u];
        cnt[u] = 1;
        if (fastc[u]) { /* the key's upper word is warp-uniform on a fast chunk */
          const uint32_t x0l = __shfl_sync(FULL, (uint32_t)klo[u], 0);
          const uint32_t x0h = __shfl_sync(FULL, (uint32_t)(klo[u] >> 32), 0);
          const uint32_t h0l = __shfl_sync(FULL, (uint32_t)khi[u], 0);
          const bool eq_ins = (uint32_t)khi[u] == h0l;
          if (__all_sync(FULL, eq_ins && (uint32_t)klo[u] == x0l && (uint32_t)(klo[u] >> 32) == x0h)) {
            lead[u] = lane == 0;
            cnt[u] = 32;
          } else if (!*(volatile unsigned int*)&s.pages_off) {
            const uint64_t Kh = (khi[u] & 0xFFFFFFFF00000000ull) | h0l;
            const uint64_t Kp = (((uint64_t)x0h << 32) | x0l) >> 10;
            const bool mine = eq_ins && (klo[u] >> 10) == Kp && (klo[u] & 3u) == 0;
            const uint32_t h = dir_hash(Kh, Kp) >> (32 - DIR_LOG);
            const ulonglong2 k0 = s.dir_key[h], k1 = s.dir_key[(h + 1) & (DIRCAP - 1)];
            const bool f0 = k0.x == Kh && k0.y == Kp, f1 = k1.x == Kh && k1.y == Kp;
            int pid = f0 ? s.dir_page[h] : (f1 ? s.dir_page[(h + 1) & (DIRCAP - 1)] : -1);
            if (__any_sync(FULL, !f0 && !f1 && (k0.x == OWL_EMPTY_KEY || k1.x == OWL_EMPTY_KEY)))
              pid = page_alloc(s, Kh, Kp, h, lane);
            if (pid >= 0 && mine) {
              atomicAdd(&s.page[pid][(klo[u] >> 2) & (PAGE_BINS - 1)], 1u);
              ++ptot;
              ++padds;
              lead[u] = false;
            }
          }
        }
        any_lead |= __ballot_sync(FULL, lead[u]);
      }
      if (!any_lead) continue;
      uint32_t home[FOLD_U];
      ulonglong4 kk[FOLD_U];
#pragma unroll
      for (int u = 0; u < FOLD_U; ++u) {
        home[u] = tab_index(khi[u], klo[u], shift);
#ifdef OWL_DEBUG_CHECKS
        if (lead[u] && home[u] >= tab.cap) { printf("bad home %u cap %llu shift %u\n", home[u], (unsigned long long)tab.cap, shift); __trap(); }
#endif
        kk[u] = ld_bucket_keys_if(lead[u] && a.mode != 6, tab.b + (home[u] >> 1));
      }
      if (a.mode == 5) { /* experiment: probe loads only */
        unsigned sink = 0;
#pragma unroll
        for (int u = 0; u < FOLD_U; ++u) sink |= (unsigned)(kk[u].x == khi[u]);
        if (__all_sync(FULL, sink == 7u)) claims += 1;
        continue;
      }
      if (a.mode == 6) { /* experiment: REDs to the home cells only (counts are wrong) */
#pragma unroll
        for (int u = 0; u < FOLD_U; ++u) red_add_if(lead[u], &tab.b[home[u] >> 1].count[0], cnt[u]);
        continue;
      }
      unsigned miss_any = 0;
#pragma unroll
      for (int u = 0; u < FOLD_U; ++u) {
        const bool h0 = kk[u].x == khi[u] && kk[u].y == klo[u];
        const bool h1 = kk[u].z == khi[u] && kk[u].w == klo[u];
        const bool hit = lead[u] && (h0 || h1);
        red_add_if(hit && a.mode != 7, &tab.b[home[u] >> 1].count[h1 ? 1 : 0], cnt[u]);
        lead[u] = lead[u] && !hit; /* now: missed (absent, or displaced past the home bucket) */
        miss_any |= __ballot_sync(FULL, lead[u]);
      }
      if (miss_any) {
#pragma unroll
        for (int u = 0; u < FOLD_U; ++u)
          if (lead[u]) claims += addr_insert_slow(tab, shift, home[u], khi[u], klo[u], cnt[u], a.status);
      }
    }
    if (__any_sync(FULL, ptot != 0)) { /* close the pages before any counter could wrap */
#pragma unroll
      for (int o = 16; o; o >>= 1) ptot += __shfl_xor_sync(FULL, ptot, o);
      if (lane == 0 && atomicAdd(&s.page_total, ptot) + ptot > PAGE_TOTAL_LIMIT) s.pages_off = 1;
      ptot = 0;
    }
    /* cells claimed by this item -> table fill; past the load limit the build stops and regrows */
    if (__any_sync(FULL, claims != 0)) {
#pragma unroll
      for (int o = 16; o; o >>= 1) claims += __shfl_xor_sync(FULL, claims, o);
      if (lane == 0) {
        const unsigned long long f = atomicAdd(tab.fill, (unsigned long long)claims) + claims;
        if (f > (tab.cap >> 1) + (tab.cap >> 2)) atomicOr(&a.status->overflow, 1u << T_ADDR);
        atomicAdd(&a.status->n_claim, (unsigned long long)claims);
      }
      claims = 0;
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) padds += __shfl_xor_sync(FULL, padds, o);
  if (lane == 0) atomicAdd(&a.status->n_bypass, (unsigned long long)padds);
  __syncthreads();
  const unsigned np = s.npages < NPAGE ? s.npages : NPAGE;
  if (threadIdx.x == 0) atomicAdd(&a.status->n_flush, (unsigned long long)np);
  for (unsigned i = threadIdx.x; i < np * PAGE_BINS; i += FOLD_THREADS) {
    const unsigned pg = i / PAGE_BINS, b = i % PAGE_BINS;
    const uint32_t c = s.page[pg][b];
    if (c) {
      const ulonglong2 k = s.dir_key[s.page_dir[pg]];
      g_insert(tab, T_ADDR, k.x, (k.y << 10) | ((uint64_t)b << 2), c, a.status);
    }
  }
  for (int i = threadIdx.x; i < CF_CAP; i += FOLD_THREADS) {
    const ulonglong2 k = s.cf_key[i];
    if (k.x != OWL_EMPTY_KEY) {
      const int tbl = (int)(k.x >> 62);
      g_insert(a.tab[tbl], tbl, k.x & ~(3ull << 62), k.y, s.cf_cnt[i], a.status);
    }
  }
}

}  // namespace

int owl_fold_ctas_per_sm() { return 1; }
int owl_fold_runs_per_warp() { return 1; }

cudaError_t owl_launch_fold(const FoldArgs& a, int grid, cudaStream_t st) {
  const size_t smem = sizeof(FoldSmem);
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(fold_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  fold_kernel<<<grid, FOLD_THREADS, smem, st>>>(a);
  return cudaGetLastError();
}
