/*
 * owl_fold.cu — A1-A3: stream trace records once and fold them thread -> warp -> kernel into the
 * A-DCFG hash tables (§V.A-B).
 *
 * Design (measured in profiles/r01_microbench.txt): L2 RED.64 saturates at ~1.9e11/s, so
 * one global atomic per record cannot reach half of HBM bandwidth, while shared-memory atomics run at ~4
 * per SM-cycle; __match_any_sync on 64-bit keys costs ~33 SM-cycles and is not used.  Hence:
 *
 *  * one persistent CTA of 32 warps per SM owns a shared-memory hash table (8192 cells of 128-bit key +
 *    u32 count) that caches address cells; the exact global table (owl_device.cuh::g_insert) is only
 *    touched when the CTA flushes (table half full at a round barrier) or bypasses (table 3/4 full);
 *  * run batching: a work item is (group of up to 32 segments of one slot, tile position p); warp w folds
 *    tile p of segment w.  Runs of one class repeat most addresses (all of them for FIX), so the 32 warps
 *    hit the same cells at the same time and merge them in shared memory;
 *  * a tile holds the traced warps whose first record lies in it; a warp that starts a tile inside a traced
 *    warp finds the next warp start with a 33-ary warp-cooperative search, and the owner of a traced warp
 *    finishes it past the tile end;
 *  * per traced warp one CUDA warp walks the records 32 at a time (one 128-bit load per lane, 4 chunks in
 *    flight):
 *      A2  BB_ENTRY lanes are rare; they are applied in lane order with warp-uniform state (cur, prev, the
 *          per-warp visit ordinal j of each BB in a shared-memory map) and count node / edge /
 *          triple cells in a second, small shared-memory table.  Each MEM lane takes its context (bb, j)
 *          from the last BB_ENTRY lane before it (ballot + clz), or from the state carried into the chunk.
 *      A3  MEM lanes add 1 to their (bb, ins, j, x) cell; a chunk whose lanes share one key (broadcast
 *          loads) adds the lane count once (the paper's merge of identical thread traces).
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
#define FOLD_WARPS 24 /* 24 warps x 80 registers: no spills (32 warps x 64 registers spill) */
#endif
#define FOLD_THREADS (FOLD_WARPS * 32)
#define SCAP 8192          /* shared address-cell cache */
#define SCAP_FLUSH 3072    /* request a CTA flush at this fill (37.5%) */
#define SCAP_BYPASS 5120   /* above this fill new keys go straight to the global table */
#define CF_CAP 512         /* shared node / edge / triple cells */
#define CF_LIMIT 384
#define VCAP 128           /* per-warp visit map (distinct BBs of one traced warp) */
#ifndef PF
#define PF 2
#endif
#define PF_AHEAD 512       /* records prefetched into L2 ahead of the walk (8 KB per warp) */
#define PF_BULK 256        /* records per bulk prefetch (4 KB) */
#define PF_DOC               /* chunks of 32 records in flight per warp */

namespace {

struct WarpTile {
  const uint4* rec;
  uint64_t n, e;      /* segment records, tile end */
  uint32_t* seen;
  uint32_t slot, n_warps, seg_index, _pad;
};

struct __align__(16) FoldSmem {
  ulonglong2 key[SCAP];
  unsigned int cnt[SCAP];
  ulonglong2 cf_key[CF_CAP];
  unsigned int cf_cnt[CF_CAP];
  uint32_t vkey[FOLD_WARPS][VCAP];
  uint32_t vcnt[FOLD_WARPS][VCAP];
  WarpTile wt[FOLD_WARPS]; /* per-warp tile description (read per chunk, broadcast) */
  unsigned long long qword;  /* CTA work queue: item << QSHIFT | next member */
  unsigned int fill;
  unsigned int cf_fill;
  unsigned int flush_req;
  unsigned int done_count;
  unsigned int n_flush, n_bypass, n_claim;
};

__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

__device__ __forceinline__ uint32_t shash(uint64_t hi, uint64_t lo) {
  return (uint32_t)((lo * 0x9E3779B97F4A7C15ull + hi * 0xC2B2AE3D27D4EB4Full) >> 51); /* 13 bits: SCAP */
}

/* address cell += c in the CTA cache (triangular probing); bypass to the exact global table when the cache
   is full.  The cache is an exact partial sum: every cell is eventually added to the global table. */
__device__ __forceinline__ void s_insert(FoldSmem& s, const FoldArgs& a, uint64_t hi, uint64_t lo, uint32_t c) {
  uint32_t h = shash(hi, lo);
#pragma unroll 1
  for (uint32_t probe = 1; probe <= 24; ++probe) {
    const ulonglong2 k = s.key[h];
    if (k.x == hi && k.y == lo) {
      atomicAdd(&s.cnt[h], c);
      return;
    }
    if (k.x == OWL_EMPTY_KEY) {
      if (*(volatile unsigned int*)&s.fill >= SCAP_BYPASS) break;
      const ulonglong2 o = cas128_shared(&s.key[h], OWL_EMPTY_KEY, OWL_EMPTY_KEY, hi, lo);
      if (o.x == OWL_EMPTY_KEY && o.y == OWL_EMPTY_KEY) {
        if (atomicAdd(&s.fill, 1u) + 1 == SCAP_FLUSH) s.flush_req = 1;
        atomicAdd(&s.cnt[h], c);
        return;
      }
      if (o.x == hi && o.y == lo) {
        atomicAdd(&s.cnt[h], c);
        return;
      }
    }
    h = (h + probe) & (SCAP - 1);
  }
  atomicAdd(&s.n_bypass, 1u);
  g_insert(a.tab[T_ADDR], T_ADDR, hi, lo, c, a.status);
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

/* visits[b] += 1 in the warp's map; returns the new visit ordinal j (reading R8) */
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

/* Per-warp walker state in registers (warp-uniform); the tile description lives in FoldSmem::wt[warp] */
struct Walker {
  uint64_t pos;  /* next record */
  uint64_t pf;   /* records below pf have been prefetched into L2 */
  uint64_t khi;  /* slot<<48 | cur<<30 | curj<<0: the address key of the current context (ins added per record) */
  uint32_t g0, cur, prev, curj;
  bool active, in_warp, skip;
};

__device__ __forceinline__ void process_chunk(const uint4 r, const bool active, const uint64_t idx, Walker& w,
                                              const WarpTile& t, const FoldArgs& a, FoldSmem& s, uint32_t* vk,
                                              uint32_t* vc, const int lane) {
  const uint64_t addr = (uint64_t)r.x | ((uint64_t)r.y << 32);
  const uint32_t meta = r.w;
  const uint32_t bbf = (meta >> 8) & 0x3FFFFu;
  const uint32_t ins = meta & 0xFFu;
  const bool isbb = active && (meta >> 31) == 0;
  const bool bbbad = isbb && (addr != 0 || (meta & 0x7C0000FFu) != 0);
  if (bbbad) report(a.status, t.seg_index, idx, KERR_BBFIELDS);
  const unsigned bbmask = __ballot_sync(FULL, isbb && !bbbad);
  const uint32_t cur0 = w.cur, j0 = w.curj;
  uint32_t myj = 0;
  if (bbmask) {
    const uint64_t slot_hi = (uint64_t)t.slot << 32;
    unsigned m = bbmask;
    while (m) {
      const int k = __ffs(m) - 1;
      m &= m - 1;
      const uint32_t b = __shfl_sync(FULL, bbf, k);
      if (lane == 0) {
        if (w.cur == OWL_NONE_BB) {
          cf_insert(s, a, T_EDGE, slot_hi | OWL_SENTINEL, b); /* S -> first BB */
        } else {
          cf_insert(s, a, T_EDGE, slot_hi | w.cur, b);       /* cur -> b */
          cf_insert(s, a, T_TRIPLE, slot_hi | w.cur, ((uint64_t)w.prev << 32) | b);
        }
        cf_insert(s, a, T_NODE, slot_hi | b, 0);
      }
      if (w.cur != OWL_NONE_BB) w.prev = w.cur;
      w.cur = b;
      w.curj = visits_inc(vk, vc, b, lane, a.status);
      if (lane == k) myj = w.curj;
    }
    w.khi = ((uint64_t)t.slot << 48) | ((uint64_t)w.cur << 30) | (uint64_t)w.curj;
    if (w.curj > OWL_MAX_J && lane == 0) atomicOr(&a.status->limit, 1u);
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
    if (code) report(a.status, t.seg_index, idx, code);
  }
  const bool good = ismem && code == 0;
  const unsigned gm = __ballot_sync(FULL, good);
  if (!gm) return;
  if (good && cj > OWL_MAX_J) atomicOr(&a.status->limit, 1u);
  const uint64_t khi = ((uint64_t)t.slot << 48) | ((uint64_t)cbb << 30) | ((uint64_t)ins << 22) | cj;
  const int first = __ffs(gm) - 1;
  const uint64_t hi0 = __shfl_sync(FULL, khi, first);
  const uint64_t lo0 = __shfl_sync(FULL, addr, first);
  const bool uniform = __ballot_sync(FULL, good && (khi != hi0 || addr != lo0)) == 0;
  if (a.mode != 0) return;
  if (uniform) { /* one key for the whole chunk (broadcast access): one add of the lane count */
    if (lane == first) s_insert(s, a, hi0, lo0, __popc(gm));
  } else if (good) {
    s_insert(s, a, khi, addr, 1);
  }
}

/* warp end: last BB -> S */
__device__ __forceinline__ void end_traced_warp(Walker& w, const WarpTile& t, const FoldArgs& a, FoldSmem& s,
                                                int lane) {
  if (!w.skip && w.cur != OWL_NONE_BB && lane == 0) {
    cf_insert(s, a, T_EDGE, ((uint64_t)t.slot << 32) | w.cur, OWL_SENTINEL);
    cf_insert(s, a, T_TRIPLE, ((uint64_t)t.slot << 32) | w.cur, ((uint64_t)w.prev << 32) | OWL_SENTINEL);
  }
  w.in_warp = false;
}

__device__ __forceinline__ void begin_traced_warp(Walker& w, const WarpTile& t, const FoldArgs& a, uint32_t* vk,
                                                  int lane) {
  w.g0 = __ldg(&t.rec[w.pos].z);
  w.skip = false;
  if (w.g0 >= t.n_warps) { /* every record of this warp is malformed (the first one is reported) */
    if (lane == 0) report(a.status, t.seg_index, w.pos, KERR_GWARP);
    w.skip = true;
  } else if (lane == 0) {
    const uint32_t bit = 1u << (w.g0 & 31);
    if (atomicOr(&t.seen[w.g0 >> 5], bit) & bit)
      atomicMin(&a.status->not_warp_major, ((unsigned long long)t.seg_index << 32) | w.g0);
  }
  for (int i = lane; i < VCAP; i += 32) vk[i] = 0xFFFFFFFFu;
  __syncwarp();
  w.cur = OWL_NONE_BB;
  w.prev = OWL_SENTINEL;
  w.curj = 0;
  w.khi = 0;
  w.in_warp = true;
}

/* Keeps the next PF_AHEAD records of the warp's stream in flight to L2 (one bulk prefetch instruction
   per PF_BULK records): the demand loads of the walk then hit L2, which hides DRAM latency without
   spending registers or shared memory on staging. */
__device__ __forceinline__ void l2_prefetch(Walker& w, const WarpTile& t, int lane) {
  if (w.pf < w.pos) w.pf = w.pos;
  while (w.pf < t.n && w.pf < w.pos + PF_AHEAD) {
    uint64_t nrec = t.n - w.pf < PF_BULK ? t.n - w.pf : PF_BULK;
    if (lane == 0)
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(t.rec + w.pf), "r"((uint32_t)(nrec * 16))
                   : "memory");
    w.pf += nrec;
  }
}

/* One step: up to PF chunks of the warp's tile; clears w.active when the tile is finished. */
__device__ __forceinline__ void walk_step(Walker& w, const WarpTile& t, const FoldArgs& a, FoldSmem& s, uint32_t* vk,
                                          uint32_t* vc, int lane) {
  if (!w.in_warp) {
    if (w.pos >= t.e) {
      w.active = false;
      return;
    }
    begin_traced_warp(w, t, a, vk, lane);
  }
  if (a.mode != 3) l2_prefetch(w, t, lane);
  uint4 r[PF];
#pragma unroll
  for (int u = 0; u < PF; ++u) {
    const uint64_t i = w.pos + (uint64_t)u * 32 + lane;
    r[u] = i < t.n ? ld_stream(t.rec + i) : make_uint4(0, 0, 0xFFFFFFFFu, 0);
  }
#pragma unroll
  for (int u = 0; u < PF; ++u) {
    if (!w.in_warp) continue;
    const uint64_t base = w.pos;
    const bool valid = (base + lane < t.n) && r[u].z == w.g0;
    const unsigned vm = __ballot_sync(FULL, valid);
    /* fast path: 32 MEM records of the current BB, well-formed (the common case: BB entries are < 1%) */
    const uint64_t addr = (uint64_t)r[u].x | ((uint64_t)r[u].y << 32);
    const bool fast_ok = (r[u].w >> 31) != 0 && ((r[u].w >> 8) & 0x3FFFFu) == w.cur && (addr >> 60) <= 8;
    if (vm == FULL && __all_sync(FULL, fast_ok) && !w.skip && a.mode == 0) {
      const uint32_t ins = r[u].w & 0xFFu;
      const uint64_t khi = w.khi | ((uint64_t)ins << 22);
      const uint32_t ins0 = __shfl_sync(FULL, ins, 0);
      const uint32_t alo0 = __shfl_sync(FULL, r[u].x, 0), ahi0 = __shfl_sync(FULL, r[u].y, 0);
      if (__all_sync(FULL, ins == ins0 && r[u].x == alo0 && r[u].y == ahi0)) {
        if (lane == 0) s_insert(s, a, khi, addr, 32u); /* broadcast access: one add of the lane count */
      } else {
        s_insert(s, a, khi, addr, 1u);
      }
      w.pos = base + 32;
      continue;
    }
    const int nvalid = vm == FULL ? 32 : __ffs(~vm) - 1;
    if (!w.skip && a.mode < 2) process_chunk(r[u], lane < nvalid, base + lane, w, t, a, s, vk, vc, lane);
    w.pos = base + nvalid;
    if (nvalid < 32) end_traced_warp(w, t, a, s, lane);
  }
}

/* warp-uniform read of a shared flag (every lane must take the same branch before warp-synchronous code) */
__device__ __forceinline__ unsigned uniform_read(const unsigned int* p) {
  unsigned v = 0;
  if ((threadIdx.x & 31) == 0) v = *(volatile const unsigned int*)p;
  return __shfl_sync(FULL, v, 0);
}

__device__ __forceinline__ void named_barrier() { asm volatile("bar.sync 1, %0;" ::"n"(FOLD_THREADS) : "memory"); }

/* All 32 warps: move every cached address cell to the global table and clear the cache. */
__device__ __noinline__ void cta_flush(FoldSmem& s, const FoldArgs& a) {
  named_barrier(); /* every warp is here: no insert is in flight */
  for (int i = threadIdx.x; i < SCAP; i += FOLD_THREADS) {
    const ulonglong2 k = s.key[i];
    if (k.x != OWL_EMPTY_KEY) {
      g_insert(a.tab[T_ADDR], T_ADDR, k.x, k.y, s.cnt[i], a.status);
      s.key[i] = make_ulonglong2(OWL_EMPTY_KEY, OWL_EMPTY_KEY);
      s.cnt[i] = 0;
    }
  }
  named_barrier();
  if (threadIdx.x == 0) {
    s.n_claim += s.fill;
    s.fill = 0;
    s.flush_req = 0;
    s.n_flush += 1;
  }
  named_barrier();
}

__device__ __forceinline__ const FoldGroup& group_of(const FoldArgs& a, unsigned long long item) {
  uint32_t lo = 0, hi = a.n_groups; /* last group with item0 <= item */
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (a.groups[mid].item0 <= item) lo = mid; else hi = mid;
  }
  return a.groups[lo];
}

#define QSHIFT 8 /* member field: <= 32 pops + 1 refill + 31 waiting warps per epoch < 256 */
#define NO_ITEM (~0ull >> QSHIFT)

/* Pops (item, member) from the CTA queue; refills it from the global counter.  Returns false when the
   global work is exhausted.  Run batching: the CTA's warps take the members of one item together. */
__device__ bool pop_work(FoldSmem& s, const FoldArgs& a, int lane, unsigned long long& item, uint32_t& member) {
  for (;;) {
    unsigned long long old = 0;
    if (lane == 0) old = atomicAdd(&s.qword, 1ull);
    old = __shfl_sync(FULL, old, 0);
    item = old >> QSHIFT;
    member = (uint32_t)(old & ((1u << QSHIFT) - 1));
    if (item == NO_ITEM) return false;
    const uint32_t nm = group_of(a, item).n_members;
    if (member < nm) return true;
    if (member == nm) { /* this warp refills the queue */
      if (lane == 0) {
        unsigned long long nxt = atomicAdd(&a.status->tile_counter, 1ull);
        if (nxt >= a.n_items || *(volatile unsigned int*)&a.status->overflow) nxt = NO_ITEM;
        atomicExch(&s.qword, nxt << QSHIFT);
      }
      __syncwarp();
      continue;
    }
    /* another warp is refilling: wait for the item to change */
    if (lane == 0)
      while ((*(volatile unsigned long long*)&s.qword >> QSHIFT) == item) __nanosleep(64);
    __syncwarp();
  }
}

__global__ void __launch_bounds__(FOLD_THREADS, 1) fold_kernel(const FoldArgs args) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  FoldSmem& s = *reinterpret_cast<FoldSmem*>(smem_raw);
  __shared__ FoldArgs a; /* shared copy: helpers take it by reference without a local-memory copy */
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    a = args;
    s.fill = 0;
    s.cf_fill = 0;
    s.flush_req = 0;
    s.done_count = 0;
    s.n_flush = s.n_bypass = s.n_claim = 0;
    unsigned long long first = atomicAdd(&args.status->tile_counter, 1ull);
    s.qword = (first >= args.n_items ? NO_ITEM : first) << QSHIFT;
  }
  for (int i = threadIdx.x; i < SCAP; i += FOLD_THREADS) {
    s.key[i] = make_ulonglong2(OWL_EMPTY_KEY, OWL_EMPTY_KEY);
    s.cnt[i] = 0;
  }
  for (int i = threadIdx.x; i < CF_CAP; i += FOLD_THREADS) {
    s.cf_key[i] = make_ulonglong2(OWL_EMPTY_KEY, OWL_EMPTY_KEY);
    s.cf_cnt[i] = 0;
  }
  __syncthreads();
  uint32_t* vk = s.vkey[warp];
  uint32_t* vc = s.vcnt[warp];
  WarpTile& t = s.wt[warp];
  const uint64_t tile = 1ull << a.tile_shift;
  Walker w;
  w.active = false;
  w.in_warp = false;
  for (;;) {
    if (uniform_read(&s.flush_req)) {
      cta_flush(s, a);
      continue;
    }
    if (!w.active) {
      unsigned long long item;
      uint32_t member;
      if (!pop_work(s, a, lane, item, member)) break;
      const FoldGroup& g = group_of(a, item);
      const FoldSeg& sg = a.segs[g.first_seg + member];
      const uint64_t b = (item - g.item0) * tile;
      if (b >= sg.n) continue;
      if (lane == 0) {
        t.rec = sg.rec;
        t.n = sg.n;
        t.e = b + tile < sg.n ? b + tile : sg.n;
        t.seen = sg.seen;
        t.slot = sg.slot;
        t.n_warps = sg.n_warps;
        t.seg_index = sg.seg_index;
      }
      __syncwarp();
      w.pos = first_warp_start(sg.rec, b, t.e, lane);
      w.pf = w.pos;
      w.active = true;
      w.in_warp = false;
    }
    walk_step(w, t, a, s, vk, vc, lane);
  }
  /* out of work: keep answering flush requests until every warp is out of work */
  if (lane == 0) atomicAdd(&s.done_count, 1u);
  for (;;) {
    if (uniform_read(&s.flush_req)) {
      cta_flush(s, a);
      continue;
    }
    if (uniform_read(&s.done_count) == FOLD_WARPS) break;
    __nanosleep(200);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    s.n_claim += s.fill;
    atomicAdd(&a.status->n_flush, (unsigned long long)s.n_flush);
    atomicAdd(&a.status->n_bypass, (unsigned long long)s.n_bypass);
    atomicAdd(&a.status->n_claim, (unsigned long long)s.n_claim);
  }
  for (int i = threadIdx.x; i < SCAP; i += FOLD_THREADS) {
    const ulonglong2 k = s.key[i];
    if (k.x != OWL_EMPTY_KEY) g_insert(a.tab[T_ADDR], T_ADDR, k.x, k.y, s.cnt[i], a.status);
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
