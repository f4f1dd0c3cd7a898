/*
 * owl_ks.cu — A6: batched two-sample Kolmogorov-Smirnov tests (Eqs. 1-4), one warp per
 * attribute pair, on the canonical (sorted) tables of E_fix and E_rnd.
 *
 *   H_cf  per node (Eqs. 5-8): the node's triple cells (prev, next), row-major with S last
 *         (reading R6) — exactly the sorted triple table's order inside one key_hi = (slot, bb).
 *   H_addr per (bb, ins, j): the address cells — the sorted addr table's order inside one
 *         key_hi = (slot, bb, ins, j).
 * An attribute is tested only when it is present on both sides of an aligned slot pair (reading R9).
 *
 * Samples are histogram x-values repeated by their counts (R4).  With A_t, B_t the fix / rnd counts at or
 * below t, F_X(t) = A_t/n and F_Y(t) = B_t/m, so D = sup|F_X - F_Y| = K/(n m), K = max_t |A_t m - B_t n|,
 * evaluated exactly in 128-bit integers at every x of either side (each lane: own cell's prefix sum plus a
 * binary search of the other side).  Then, in fp64 with round-to-nearest intrinsics and no FMA, in the
 * fixed order of DESIGN.md §3: D = K/(n*m); w = (n*m)/(n+m); x = (2*(D*D))*w; p = 2*exp(-x);
 * fail = p < significance.
 */
#include <cub/cub.cuh>
#include <cuda_runtime.h>

#include "owl_internal.h"

namespace {

typedef unsigned __int128 u128;

__global__ void extract_hi_kernel(const Key128* k, uint64_t n, unsigned long long* hi, unsigned char* start) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long h = k[i].hi;
    hi[i] = h;
    start[i] = (i == 0 || k[i - 1].hi != h) ? 1 : 0;
  }
}

__device__ __forceinline__ uint32_t slot_of(int tbl, unsigned long long hi) {
  return tbl == T_ADDR ? (uint32_t)(hi >> 48) : (uint32_t)(hi >> 32);
}
__device__ __forceinline__ unsigned long long with_slot(int tbl, unsigned long long hi, uint32_t s) {
  return tbl == T_ADDR ? ((hi & 0x0000FFFFFFFFFFFFull) | ((unsigned long long)s << 48))
                       : ((hi & 0xFFFFFFFFull) | ((unsigned long long)s << 32));
}

/* pairs (attribute index on fix side, attribute index on rnd side) */
__global__ void pair_kernel(int tbl, const unsigned long long* hif, const uint64_t* stf, uint64_t naf,
                            const unsigned long long* hir, const uint64_t* str, uint64_t nar, const uint32_t* map,
                            uint32_t nmap, uint2* pairs, unsigned long long* npairs) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < naf; i += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long hf = hif[stf[i]];
    const uint32_t sf = slot_of(tbl, hf);
    if (sf >= nmap || map[sf] == 0xFFFFFFFFu) continue;
    const unsigned long long hr = with_slot(tbl, hf, map[sf]);
    uint64_t lo = 0, hi = nar;
    while (lo < hi) {
      const uint64_t mid = (lo + hi) >> 1;
      if (hir[str[mid]] < hr) lo = mid + 1; else hi = mid;
    }
    if (lo < nar && hir[str[lo]] == hr) {
      const unsigned long long o = atomicAdd(npairs, 1ull);
      pairs[o] = make_uint2((uint32_t)i, (uint32_t)lo);
    }
  }
}

/* exact round-to-nearest-even conversion of an unsigned 128-bit integer to double */
__device__ double u128_to_double_rn(u128 v) {
  const unsigned long long hi = (unsigned long long)(v >> 64);
  if (hi == 0) return __ull2double_rn((unsigned long long)v);
  const int lz = __clzll(hi);
  const u128 x = v << lz; /* bit 127 set */
  const unsigned long long top = (unsigned long long)(x >> 64);
  const bool sticky = (unsigned long long)x != 0;
  unsigned long long mant = top >> 11;
  const unsigned long long rb = top & 0x7FFull;
  int e = 127 - lz - 52;
  if (rb > 0x400ull || (rb == 0x400ull && (sticky || (mant & 1ull)))) {
    ++mant;
    if (mant == (1ull << 53)) { mant >>= 1; ++e; }
  }
  return scalbn((double)mant, e);
}

__device__ __forceinline__ u128 absdiff(u128 a, u128 b) { return a > b ? a - b : b - a; }

__global__ void ks_kernel(const Key128* fk, const unsigned long long* fpre, uint64_t nf, const uint64_t* stf, uint64_t naf,
                          const Key128* rk, const unsigned long long* rpre, uint64_t nr, const uint64_t* str, uint64_t nar,
                          const uint2* pairs, uint64_t npairs, double significance, KsOutRow* out) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp0 = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t w = warp0; w < npairs; w += nwarps) {
    const uint2 pr = pairs[w];
    const uint64_t fb = stf[pr.x], fe = pr.x + 1 < naf ? stf[pr.x + 1] : nf;
    const uint64_t rb = str[pr.y], re = pr.y + 1 < nar ? str[pr.y + 1] : nr;
    const unsigned long long n = fpre[fe - 1], m = rpre[re - 1];
    u128 K = 0;
    for (uint64_t i = fb + lane; i < fe; i += 32) {
      const unsigned long long x = fk[i].lo;
      uint64_t lo = rb, hi = re; /* first rnd cell with lo > x */
      while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (rk[mid].lo <= x) lo = mid + 1; else hi = mid;
      }
      const unsigned long long B = lo > rb ? rpre[lo - 1] : 0ull;
      const u128 d = absdiff((u128)fpre[i] * m, (u128)B * n);
      if (d > K) K = d;
    }
    for (uint64_t i = rb + lane; i < re; i += 32) {
      const unsigned long long x = rk[i].lo;
      uint64_t lo = fb, hi = fe;
      while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (fk[mid].lo <= x) lo = mid + 1; else hi = mid;
      }
      const unsigned long long A = lo > fb ? fpre[lo - 1] : 0ull;
      const u128 d = absdiff((u128)A * m, (u128)rpre[i] * n);
      if (d > K) K = d;
    }
    for (int o = 16; o > 0; o >>= 1) {
      const unsigned long long khi = __shfl_xor_sync(0xFFFFFFFFu, (unsigned long long)(K >> 64), o);
      const unsigned long long klo = __shfl_xor_sync(0xFFFFFFFFu, (unsigned long long)K, o);
      const u128 other = ((u128)khi << 64) | klo;
      if (other > K) K = other;
    }
    if (lane == 0) {
      const double nd = __ull2double_rn(n), md = __ull2double_rn(m);
      const double nm = __dmul_rn(nd, md);
      const double D = __ddiv_rn(u128_to_double_rn(K), nm);
      const double wgt = __ddiv_rn(nm, __dadd_rn(nd, md));
      const double x = __dmul_rn(__dmul_rn(2.0, __dmul_rn(D, D)), wgt);
      const double p = __dmul_rn(2.0, exp(-x));
      KsOutRow r;
      r.hi_f = fk[fb].hi;
      r.hi_r = rk[rb].hi;
      r.n = n;
      r.m = m;
      r.K_lo = (unsigned long long)K;
      r.K_hi = (unsigned long long)(K >> 64);
      r.D = D;
      r.p = p;
      r.fail = p < significance ? 1u : 0u;
      r._pad = 0;
      out[w] = r;
    }
  }
}

struct Side {
  unsigned long long* hi = nullptr;
  unsigned char* st = nullptr;
  unsigned long long* pre = nullptr;
  uint64_t* starts = nullptr;
  unsigned long long* nattr = nullptr;
  uint64_t na = 0;
  void free_all() {
    cudaFree(hi); cudaFree(st); cudaFree(pre); cudaFree(starts); cudaFree(nattr);
  }
};

int grid_for(uint64_t n, int block) {
  uint64_t g = (n + block - 1) / block;
  if (g > 148ull * 16) g = 148ull * 16;
  return g ? (int)g : 1;
}

cudaError_t prepare(const SortedTable& t, Side& s, cudaStream_t st) {
  const uint64_t n = t.n;
  if (cudaMalloc(&s.hi, (n + 1) * 8) || cudaMalloc(&s.st, n + 1) || cudaMalloc(&s.pre, (n + 1) * 8) ||
      cudaMalloc(&s.starts, (n + 1) * 8) || cudaMalloc(&s.nattr, 8))
    return cudaErrorMemoryAllocation;
  if (!n) return cudaSuccess;
  extract_hi_kernel<<<grid_for(n, 256), 256, 0, st>>>(t.k, n, s.hi, s.st);
  size_t t1 = 0, t2 = 0;
  cub::DeviceSelect::Flagged(nullptr, t1, cub::CountingInputIterator<uint64_t>(0), s.st, s.starts, s.nattr, (int64_t)n, st);
  cub::DeviceScan::InclusiveSumByKey(nullptr, t2, s.hi, t.c, s.pre, (int64_t)n, cub::Equality(), st);
  void* tmp = nullptr;
  if (cudaMalloc(&tmp, (t1 > t2 ? t1 : t2) + 16)) return cudaErrorMemoryAllocation;
  cudaError_t e = cub::DeviceSelect::Flagged(tmp, t1, cub::CountingInputIterator<uint64_t>(0), s.st, s.starts, s.nattr,
                                             (int64_t)n, st);
  if (e == cudaSuccess) e = cub::DeviceScan::InclusiveSumByKey(tmp, t2, s.hi, t.c, s.pre, (int64_t)n, cub::Equality(), st);
  unsigned long long na = 0;
  if (e == cudaSuccess) e = cudaMemcpyAsync(&na, s.nattr, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  cudaFree(tmp);
  s.na = na;
  return e;
}

}  // namespace

cudaError_t owl_ks_run(int tbl, const SortedTable& f, const SortedTable& r, const std::vector<uint32_t>& slot_f2r,
                       double significance, std::vector<KsOutRow>& rows, cudaStream_t st) {
  rows.clear();
  if (!f.n || !r.n || slot_f2r.empty()) return cudaSuccess;
  Side sf, sr;
  uint32_t* dmap = nullptr;
  uint2* pairs = nullptr;
  unsigned long long* npairs = nullptr;
  KsOutRow* dout = nullptr;
  cudaError_t e = prepare(f, sf, st);
  if (e == cudaSuccess) e = prepare(r, sr, st);
  unsigned long long np = 0;
  if (e == cudaSuccess && cudaMalloc(&dmap, slot_f2r.size() * 4)) e = cudaErrorMemoryAllocation;
  if (e == cudaSuccess && (cudaMalloc(&pairs, (sf.na + 1) * sizeof(uint2)) || cudaMalloc(&npairs, 8)))
    e = cudaErrorMemoryAllocation;
  if (e == cudaSuccess) {
    cudaMemcpyAsync(dmap, slot_f2r.data(), slot_f2r.size() * 4, cudaMemcpyHostToDevice, st);
    cudaMemsetAsync(npairs, 0, 8, st);
    pair_kernel<<<grid_for(sf.na, 256), 256, 0, st>>>(tbl, sf.hi, sf.starts, sf.na, sr.hi, sr.starts, sr.na, dmap,
                                                      (uint32_t)slot_f2r.size(), pairs, npairs);
    e = cudaMemcpyAsync(&np, npairs, 8, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  }
  if (e == cudaSuccess && np) {
    if (cudaMalloc(&dout, np * sizeof(KsOutRow))) e = cudaErrorMemoryAllocation;
    if (e == cudaSuccess) {
      ks_kernel<<<grid_for(np * 32, 256), 256, 0, st>>>(f.k, sf.pre, f.n, sf.starts, sf.na, r.k, sr.pre, r.n, sr.starts,
                                                        sr.na, pairs, np, significance, dout);
      rows.resize(np);
      e = cudaMemcpyAsync(rows.data(), dout, np * sizeof(KsOutRow), cudaMemcpyDeviceToHost, st);
      if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    }
  }
  sf.free_all();
  sr.free_all();
  cudaFree(dmap); cudaFree(pairs); cudaFree(npairs); cudaFree(dout);
  if (e == cudaSuccess) e = cudaGetLastError();
  return e;
}
