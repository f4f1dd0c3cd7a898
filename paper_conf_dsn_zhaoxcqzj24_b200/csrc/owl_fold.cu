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

#include "owl_device.cuh"
#include "owl_internal.h"

using namespace owl_dev;

#define FULL 0xFFFFFFFFu
#ifndef FOLD_WARPS
#define FOLD_WARPS 24
#endif
#ifndef FOLD_R
#define FOLD_R 2 /* walkers (runs) per warp */
#endif
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
  ulonglong2 cf_key[CF_CAP];
  unsigned int cf_cnt[CF_CAP];
  uint32_t vkey[FOLD_WARPS][FOLD_R][VCAP];
  uint32_t vcnt[FOLD_WARPS][FOLD_R][VCAP];
  RunDesc rd[FOLD_WARPS][FOLD_R];
  unsigned int cf_fill;
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
__device__ __forceinline__ ulonglong2 ld_key_weak(const owl_cell* c) {
  ulonglong2 k;
  asm volatile("ld.global.cg.v2.u64 {%0, %1}, [%2];" : "=l"(k.x), "=l"(k.y) : "l"(c));
  return k;
}

__device__ __forceinline__ void red_add(unsigned long long* p, unsigned long long v) {
  asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

/* predicated forms (no divergent branch around them) */
__device__ __forceinline__ ulonglong2 ld_key_if(bool pred, const owl_cell* c) {
  ulonglong2 k;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %3, 0;\n\t"
      "mov.b64 %0, -1;\n\t"
      "mov.b64 %1, -1;\n\t"
      "@p ld.global.cg.v2.u64 {%0, %1}, [%2];\n\t}"
      : "=l"(k.x), "=l"(k.y)
      : "l"(c), "r"((int)pred));
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
    owl_cell* cell = t.cells + h;
    const ulonglong2 k = ld_key_weak(cell);
    if (k.x == hi && k.y == lo) {
      red_add(&cell->count, c);
      return 0;
    }
    if (k.x == OWL_EMPTY_KEY || k.x == hi) { /* empty, being claimed, or a torn read: resolve with the CAS */
      const ulonglong2 o = cas128_global(&cell->hi, OWL_EMPTY_KEY, OWL_EMPTY_KEY, hi, lo);
      if ((o.x == OWL_EMPTY_KEY && o.y == OWL_EMPTY_KEY) || (o.x == hi && o.y == lo)) {
        red_add(&cell->count, c);
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
    const bool ismem = active && (meta >> 31) != 0;
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
  w.p += nvalid;
  if (nvalid < 32) { /* warp end: last BB -> S */
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

/* table index of a key: multiplicative hash, top bits (same function as owl_device.cuh::tab_index) */
__device__ __forceinline__ uint64_t addr_index(uint64_t hi, uint64_t lo, uint32_t shift) {
  return tab_hash(hi, lo) >> shift;
}

__global__ void __launch_bounds__(FOLD_THREADS, 1) fold_kernel(const FoldArgs args) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  FoldSmem& s = *reinterpret_cast<FoldSmem*>(smem_raw);
  __shared__ FoldArgs a; /* shared copy: helpers take it by reference without a local-memory copy */
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    a = args;
    s.cf_fill = 0;
  }
  for (int i = threadIdx.x; i < CF_CAP; i += FOLD_THREADS) {
    s.cf_key[i] = make_ulonglong2(OWL_EMPTY_KEY, OWL_EMPTY_KEY);
    s.cf_cnt[i] = 0;
  }
  __syncthreads();
  const uint64_t pol = evict_first_policy();
  const uint64_t tile = 1ull << a.tile_shift;
  const DevTable tab = a.tab[T_ADDR];
  const uint32_t shift = tab_shift(tab.cap);
  uint32_t claims = 0;

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
    Walker w[FOLD_R];
#pragma unroll
    for (int r = 0; r < FOLD_R; ++r) {
      w[r].st = 0;
      w[r].p = nullptr;
      w[r].g0 = w[r].cur = 0;
      w[r].khi = 0;
      if (r < (int)g.n_members) {
        const FoldSeg& sg = a.segs[g.first_seg + r];
        if (b < sg.n) {
          RunDesc& d = s.rd[warp][r];
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
          w[r].p = sg.rec + first_warp_start(sg.rec, b, e, lane);
          w[r].st = W_ACTIVE;
          const uint4* end = sg.rec + sg.n;
          if (lane < PF_DIST && a.mode != 3) { /* prime the L2 prefetch window */
            const uintptr_t g0 = (((uintptr_t)w[r].p) >> PF_LOG) + lane;
            const char* q = (const char*)(g0 << PF_LOG);
            if (q < (const char*)end) {
              const uint64_t left = (uint64_t)((const char*)end - q);
              l2_prefetch_bulk(q, left < (1u << PF_LOG) ? (uint32_t)left : (1u << PF_LOG));
            }
          }
        }
      }
    }
    __syncwarp();

    for (;;) {
      /* traced-warp starts and tile ends */
      unsigned any = 0;
#pragma unroll
      for (int r = 0; r < FOLD_R; ++r) {
        if ((w[r].st & (W_ACTIVE | W_INWARP)) == W_ACTIVE) {
          RunDesc& d = s.rd[warp][r];
          if (w[r].p >= d.tile_end) w[r].st = 0;
          else begin_traced_warp(w[r], d, a, s.vkey[warp][r], lane);
        }
        any |= w[r].st;
      }
      if (!any) break;

      /* loads: one 128-bit record per lane per walker */
      uint4 rr[FOLD_R];
      const uint4* end[FOLD_R];
#pragma unroll
      for (int r = 0; r < FOLD_R; ++r) {
        end[r] = s.rd[warp][r].end;
        const uint4* q = w[r].p + lane;
        rr[r] = (w[r].st && q < end[r]) ? ld_stream(q, pol) : make_uint4(0, 0, 0xFFFFFFFFu, 0);
      }
      /* L2 prefetch PF_DIST granules ahead when the walk enters a new granule */
#pragma unroll
      for (int r = 0; r < FOLD_R; ++r) {
        if (w[r].st && a.mode != 3) {
          const uintptr_t g1 = (((uintptr_t)(w[r].p + 32)) >> PF_LOG);
          if (g1 != (((uintptr_t)w[r].p) >> PF_LOG) && lane == 0) {
            const char* q = (const char*)((g1 + PF_DIST - 1) << PF_LOG);
            if (q < (const char*)end[r]) {
              const uint64_t left = (uint64_t)((const char*)end[r] - q);
              l2_prefetch_bulk(q, left < (1u << PF_LOG) ? (uint32_t)left : (1u << PF_LOG));
            }
          }
        }
      }

      /* classify + keys */
      bool good[FOLD_R];
      uint64_t khi[FOLD_R], klo[FOLD_R];
      uint32_t mult[FOLD_R];
      bool fast[FOLD_R];
#pragma unroll
      for (int r = 0; r < FOLD_R; ++r) {
        good[r] = false;
        fast[r] = false;
        mult[r] = 1;
        khi[r] = 0;
        klo[r] = 0;
        if (!w[r].st) continue;
        const bool valid = (w[r].p + lane < end[r]) && rr[r].z == w[r].g0;
        const uint64_t addr = (uint64_t)rr[r].x | ((uint64_t)rr[r].y << 32);
        const bool fast_ok = valid && (rr[r].w >> 31) != 0 && ((rr[r].w >> 8) & 0x3FFFFu) == w[r].cur &&
                             (addr >> 60) <= 8;
        const unsigned vm = __ballot_sync(FULL, valid);
        if (__all_sync(FULL, fast_ok) && !(w[r].st & W_SKIP)) {
          fast[r] = true;
          good[r] = true;
          khi[r] = w[r].khi | ((uint64_t)(rr[r].w & 0xFFu) << 22);
          klo[r] = addr;
          w[r].p += 32;
        } else {
          slow_chunk(rr[r], vm, w[r], s.rd[warp][r], a, s, s.vkey[warp][r], s.vcnt[warp][r], lane, good[r],
                     khi[r], klo[r]);
        }
      }
      if (a.mode != 0) continue;

      /* merge chunks of other runs whose 32 keys equal walker 0's into walker 0 (exact: equal keys) */
#pragma unroll
      for (int r = 1; r < FOLD_R; ++r) {
        if (fast[0] && fast[r]) {
          const bool eq = khi[r] == khi[0] && klo[r] == klo[0];
          if (__all_sync(FULL, eq)) {
            mult[0] += 1;
            mult[r] = 0;
          }
        }
      }

      /* one insert per run of equal keys over consecutive lanes: leaders, counts, first probes for every
         walker (loads in flight together), then predicated REDs; misses take a rare uniform branch */
      bool lead[FOLD_R];
      uint32_t cnt[FOLD_R];
      owl_cell* cell[FOLD_R];
      ulonglong2 kk[FOLD_R];
#pragma unroll
      for (int r = 0; r < FOLD_R; ++r) {
        const uint64_t phi = __shfl_up_sync(FULL, khi[r], 1), plo = __shfl_up_sync(FULL, klo[r], 1);
        const bool pgood = __shfl_up_sync(FULL, (int)good[r], 1) != 0;
        const bool same = lane > 0 && good[r] && pgood && phi == khi[r] && plo == klo[r];
        const unsigned brk = __ballot_sync(FULL, !same);
        const unsigned above = brk & ~((2u << lane) - 1u);
        const uint32_t nxt = above ? __ffs(above) - 1 : 32;
        lead[r] = good[r] && !same && mult[r] != 0;
        cnt[r] = (nxt - lane) * mult[r];
        cell[r] = tab.cells + addr_index(khi[r], klo[r], shift);
        kk[r] = ld_key_if(lead[r], cell[r]);
      }
      unsigned miss_any = 0;
#pragma unroll
      for (int r = 0; r < FOLD_R; ++r) {
        const bool hit = lead[r] && kk[r].x == khi[r] && kk[r].y == klo[r];
        red_add_if(hit, &cell[r]->count, cnt[r]);
        lead[r] = lead[r] && !hit; /* now: missed */
        miss_any |= __ballot_sync(FULL, lead[r]);
      }
      if (miss_any) {
#pragma unroll
        for (int r = 0; r < FOLD_R; ++r)
          if (lead[r])
            claims += addr_insert_slow(tab, shift, (uint64_t)(cell[r] - tab.cells), khi[r], klo[r], cnt[r], a.status);
      }
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
  __syncthreads();
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
int owl_fold_runs_per_warp() { return FOLD_R; }

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
