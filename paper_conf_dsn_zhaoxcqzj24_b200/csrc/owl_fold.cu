/*
 * owl_fold.cu — A1-A3: stream trace records once and fold them thread -> warp -> kernel into the
 * A-DCFG hash tables (§V.A-B).
 *
 * Work decomposition: the records of every segment are cut into fixed tiles of
 * 2^tile_shift records; a persistent grid of CTAs (8 warps each) pulls tiles from a global counter.  A
 * CUDA warp owns every traced warp whose first record lies in its tile (tiles hold whole traced warps
 * only at their start, so a traced warp that crosses the tile end is finished by the owner; a tile whose
 * first record continues a traced warp finds the next warp start with a 33-ary warp-cooperative search).
 *
 * Per traced warp, one CUDA warp walks the records 32 at a time (one 128-bit load per lane, 4 chunks in
 * flight):
 *   A2  BB_ENTRY lanes are rare; they are applied in lane order with warp-uniform state (cur, prev, the
 *       visit ordinal j of each BB kept in a per-warp shared-memory map) and update the node /
 *       edge / triple cells of a CTA-private shared-memory table (flushed once per CTA).  Each MEM lane
 *       takes its context (bb, j) from the last BB_ENTRY lane before it (ballot + clz), or from the
 *       state carried into the chunk.
 *   A3  MEM lanes with identical (bb, ins, j, x) keys are merged with __match_any_sync (the paper's
 *       "merge identical thread traces") and the leader adds the lane count to the
 *       address cell in the global table (128-bit CAS claim, 64-bit atomic count).
 * Malformed records are reported with the minimum (segment, index) and skipped (state unaffected),
 * exactly as the oracle does.
 */
#include <cuda_runtime.h>
#include <stdint.h>

#include "owl_device.cuh"
#include "owl_internal.h"

using namespace owl_dev;

#define FULL 0xFFFFFFFFu
#define FOLD_WARPS 8
#define FOLD_THREADS (FOLD_WARPS * 32)
#define VCAP 256          /* per-warp visit map entries (distinct BBs of one traced warp) */
#define CF_CAP 1024       /* CTA shared-memory table for node / edge / triple cells */
#define CF_LOAD_LIMIT 700 /* above this fill, CF cells go straight to the global table */
#define PF 4              /* chunks of 32 records in flight per warp */

namespace {

struct __align__(16) CfSmem {
  ulonglong2 key[CF_CAP];
  unsigned long long cnt[CF_CAP];
  uint32_t vkey[FOLD_WARPS][VCAP];
  uint32_t vcnt[FOLD_WARPS][VCAP];
  unsigned int fill;
};

__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

/* CTA-private node / edge / triple aggregation (the table id rides in key bits 62-63; slot < 2^16). */
__device__ void cf_insert(CfSmem& s, const FoldArgs& a, int tbl, uint64_t hi, uint64_t lo) {
  const uint64_t thi = hi | ((uint64_t)tbl << 62);
  if (*(volatile unsigned int*)&s.fill < CF_LOAD_LIMIT) {
    uint32_t h = (uint32_t)hmix(thi, lo) & (CF_CAP - 1);
    for (int probe = 0; probe < CF_CAP; ++probe) {
      ulonglong2 o = cas128_shared(&s.key[h], OWL_EMPTY_KEY, OWL_EMPTY_KEY, thi, lo);
      if (o.x == OWL_EMPTY_KEY && o.y == OWL_EMPTY_KEY) {
        atomicAdd(&s.fill, 1u);
        atomicAdd(&s.cnt[h], 1ull);
        return;
      }
      if (o.x == thi && o.y == lo) {
        atomicAdd(&s.cnt[h], 1ull);
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

/* visits[b] += 1 in the warp's map; returns the new visit ordinal j (reading R8). */
__device__ uint32_t visits_inc(uint32_t* vk, uint32_t* vc, uint32_t b, int lane, FoldStatus* st) {
  const uint32_t h = (b * 0x9E3779B1u) >> 24; /* VCAP = 256 */
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

/* First traced-warp start in [b, e) of a warp-major segment, or e if the tile starts inside a traced
   warp that runs past e.  33-ary warp-cooperative search over the monotone predicate gwarp == gprev. */
__device__ uint64_t first_warp_start(const uint4* rec, uint64_t b, uint64_t e, int lane) {
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
    const int last_same = 31 - __clz(m | 0u); /* m may be 0 */
    uint64_t nlo = lo, nhi = hi;
    if (m) nlo = __shfl_sync(FULL, p, last_same);
    else __shfl_sync(FULL, p, 0);
    if (nm) nhi = __shfl_sync(FULL, p, __ffs(nm) - 1);
    else __shfl_sync(FULL, p, 0);
    if (nlo > lo) lo = nlo;
    if (nhi < hi) hi = nhi;
  }
  return hi;
}

struct WarpState {
  uint32_t cur, prev, curj;
};

/* Applies one chunk of up to 32 records (lanes < nvalid belong to the traced warp). */
__device__ __forceinline__ void process_chunk(const uint4 r, const bool active, const uint64_t idx, WarpState& ws,
                                              const FoldSeg& sg, const FoldArgs& a, CfSmem& s, uint32_t* vk,
                                              uint32_t* vc, const int lane) {
  const uint64_t addr = (uint64_t)r.x | ((uint64_t)r.y << 32);
  const uint32_t meta = r.w;
  const uint32_t kind = meta >> 31;
  const uint32_t bbf = (meta >> 8) & 0x3FFFFu;
  const uint32_t ins = meta & 0xFFu;
  const uint32_t lf = (meta >> 26) & 31u;
  const bool isbb = active && kind == 0;
  const bool bbbad = isbb && (addr != 0 || ins != 0 || lf != 0);
  if (bbbad) report(a.status, sg.seg_index, idx, KERR_BBFIELDS);
  const unsigned bbmask = __ballot_sync(FULL, isbb && !bbbad);
  const uint32_t cur0 = ws.cur, j0 = ws.curj;
  uint32_t myj = 0;
  const uint64_t slot_hi = (uint64_t)sg.slot << 32;
  if (bbmask) {
    unsigned m = bbmask;
    while (m) {
      const int k = __ffs(m) - 1;
      m &= m - 1;
      const uint32_t b = __shfl_sync(FULL, bbf, k);
      if (lane == 0) {
        if (ws.cur == OWL_NONE_BB) {
          cf_insert(s, a, T_EDGE, slot_hi | OWL_SENTINEL, b); /* S -> first BB */
        } else {
          cf_insert(s, a, T_EDGE, slot_hi | ws.cur, b);       /* cur -> b */
          cf_insert(s, a, T_TRIPLE, slot_hi | ws.cur, ((uint64_t)ws.prev << 32) | b);
        }
        cf_insert(s, a, T_NODE, slot_hi | b, 0);
      }
      if (ws.cur != OWL_NONE_BB) ws.prev = ws.cur;
      ws.cur = b;
      ws.curj = visits_inc(vk, vc, b, lane, a.status);
      if (lane == k) myj = ws.curj;
    }
  }
  const bool ismem = active && kind == 1;
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
    if (code) report(a.status, sg.seg_index, idx, code);
  }
  const bool good = ismem && code == 0;
  if (good && cj > OWL_MAX_J) atomicOr(&a.status->limit, 1u);
  const unsigned gm = __ballot_sync(FULL, good);
  if (gm) {
    const uint64_t khi = ((uint64_t)sg.slot << 48) | ((uint64_t)cbb << 30) | ((uint64_t)ins << 22) | cj;
    const unsigned peers = __match_any_sync(FULL, addr) & __match_any_sync(FULL, khi) & gm;
    if (good && __ffs(peers) - 1 == lane) g_insert(a.tab[T_ADDR], T_ADDR, khi, addr, __popc(peers), a.status);
  }
}

/* Folds the traced warp starting at `start`; returns the index one past its last record. */
__device__ uint64_t fold_traced_warp(const FoldSeg& sg, uint64_t start, const FoldArgs& a, CfSmem& s, uint32_t* vk,
                                     uint32_t* vc, const int lane) {
  const uint4* rec = sg.rec;
  const uint64_t n = sg.n;
  const uint32_t g0 = __ldg(&rec[start].z);
  bool skip = false;
  if (g0 >= sg.n_warps) { /* every record of this warp is malformed (the first one is reported) */
    if (lane == 0) report(a.status, sg.seg_index, start, KERR_GWARP);
    skip = true;
  } else if (lane == 0) {
    const uint32_t bit = 1u << (g0 & 31);
    if (atomicOr(&sg.seen[g0 >> 5], bit) & bit)
      atomicMin(&a.status->not_warp_major, ((unsigned long long)sg.seg_index << 32) | g0);
  }
  for (int i = lane; i < VCAP; i += 32) vk[i] = 0xFFFFFFFFu;
  __syncwarp();
  WarpState ws{OWL_NONE_BB, OWL_SENTINEL, 0};
  uint64_t pos = start;
  for (;;) {
    uint4 r[PF];
#pragma unroll
    for (int u = 0; u < PF; ++u) {
      const uint64_t i = pos + (uint64_t)u * 32 + lane;
      r[u] = i < n ? ld_stream(rec + i) : make_uint4(0, 0, 0xFFFFFFFFu, 0);
    }
#pragma unroll
    for (int u = 0; u < PF; ++u) {
      const uint64_t base = pos + (uint64_t)u * 32;
      const bool valid = (base + lane < n) && r[u].z == g0;
      const unsigned vm = __ballot_sync(FULL, valid);
      const int nvalid = vm == FULL ? 32 : __ffs(~vm) - 1;
      if (!skip) process_chunk(r[u], lane < nvalid, base + lane, ws, sg, a, s, vk, vc, lane);
      if (nvalid < 32) {
        const uint64_t end = base + nvalid;
        if (!skip && ws.cur != OWL_NONE_BB && lane == 0) { /* warp end: last BB -> S */
          cf_insert(s, a, T_EDGE, ((uint64_t)sg.slot << 32) | ws.cur, OWL_SENTINEL);
          cf_insert(s, a, T_TRIPLE, ((uint64_t)sg.slot << 32) | ws.cur, ((uint64_t)ws.prev << 32) | OWL_SENTINEL);
        }
        return end;
      }
    }
    pos += (uint64_t)PF * 32;
  }
}

__global__ void __launch_bounds__(FOLD_THREADS) fold_kernel(const FoldArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  CfSmem& s = *reinterpret_cast<CfSmem*>(smem_raw);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < CF_CAP; i += FOLD_THREADS) {
    s.key[i] = make_ulonglong2(OWL_EMPTY_KEY, OWL_EMPTY_KEY);
    s.cnt[i] = 0;
  }
  if (threadIdx.x == 0) s.fill = 0;
  __syncthreads();
  uint32_t* vk = s.vkey[warp];
  uint32_t* vc = s.vcnt[warp];
  const uint64_t tile = 1ull << a.tile_shift;
  for (;;) {
    unsigned long long t = 0;
    if (lane == 0) t = atomicAdd(&a.status->tile_counter, 1ull);
    t = __shfl_sync(FULL, t, 0);
    if (t >= a.n_tiles) break;
    if (*(volatile unsigned int*)&a.status->overflow) break;
    /* segment of tile t: last seg with tile0 <= t (binary search, warp-uniform) */
    uint32_t lo = 0, hi = a.n_segs;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (a.segs[mid].tile0 <= t) lo = mid; else hi = mid;
    }
    const FoldSeg sg = a.segs[lo];
    const uint64_t b = (t - sg.tile0) * tile;
    const uint64_t e = b + tile < sg.n ? b + tile : sg.n;
    uint64_t start = first_warp_start(sg.rec, b, e, lane);
    while (start < e) start = fold_traced_warp(sg, start, a, s, vk, vc, lane);
  }
  __syncthreads();
  /* flush the CTA's node / edge / triple cells */
  for (int i = threadIdx.x; i < CF_CAP; i += FOLD_THREADS) {
    const ulonglong2 k = s.key[i];
    if (k.x != OWL_EMPTY_KEY) {
      const int tbl = (int)(k.x >> 62);
      g_insert(a.tab[tbl], tbl, k.x & ~(3ull << 62), k.y, s.cnt[i], a.status);
    }
  }
}

}  // namespace

int owl_fold_ctas_per_sm() { return 4; }

cudaError_t owl_launch_fold(const FoldArgs& a, int grid, cudaStream_t st) {
  const size_t smem = sizeof(CfSmem);
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(fold_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  fold_kernel<<<grid, FOLD_THREADS, smem, st>>>(a);
  return cudaGetLastError();
}
