/*
 * owl_ks.cu — A6: batched two-sample Kolmogorov-Smirnov tests (Eqs. 1-4) on the canonical
 * (sorted) tables of E_fix and E_rnd.
 *
 *   H_cf  per node (Eqs. 5-8): the node's triple cells (prev, next), row-major with S last
 *         (reading R6) — exactly the sorted triple table's order inside one key_hi = (slot, bb).
 *   H_addr per (bb, ins, j): the address cells — the sorted addr table's order inside one
 *         key_hi = (slot, bb, ins, j).
 * An attribute is tested only when it is present on both sides of an aligned slot pair (reading R9).
 *
 * Samples are histogram x-values repeated by their counts (R4).  With A_t, B_t the fix / rnd counts at or
 * below t, F_X(t) = A_t/n and F_Y(t) = B_t/m, so D = sup|F_X - F_Y| = K/(n m) with the exact 128-bit
 * K = max_t |A_t m - B_t n|, evaluated at every distinct x of the union of both sides.
 *
 * Work decomposition: the sorted union of an attribute pair's two cell lists is cut into units of 1024
 * union positions; one warp per unit, each lane walks 32 consecutive union positions starting from a
 * merge-path split (binary search), carrying the segmented prefix sums A and B, and evaluates |A m - B n|
 * after the last occurrence of each x.  Unit maxima are reduced per pair, then D and p are computed in
 * fp64 with round-to-nearest intrinsics and no FMA, in the fixed order of DESIGN.md §3:
 *   D = K/(n*m); w = (n*m)/(n+m); x = (2*(D*D))*w; p = 2*exp(-x); fail = p < significance.
 */
#include <cub/cub.cuh>
#include <thrust/iterator/counting_iterator.h>
#include <cuda_runtime.h>

#include "owl_internal.h"

namespace {

typedef unsigned __int128 u128;
#define UNIT 1024u
#define PER_LANE (UNIT / 32u)

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

/* pairs (attribute index on the fix side, attribute index on the rnd side) */
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

struct Range {
  uint64_t fb, fe, rb, re;
};
__device__ __forceinline__ Range range_of(const uint2 pr, const uint64_t* stf, uint64_t naf, uint64_t nf,
                                          const uint64_t* str, uint64_t nar, uint64_t nr) {
  Range r;
  r.fb = stf[pr.x];
  r.fe = pr.x + 1 < naf ? stf[pr.x + 1] : nf;
  r.rb = str[pr.y];
  r.re = pr.y + 1 < nar ? str[pr.y + 1] : nr;
  return r;
}

__global__ void units_kernel(const uint2* pairs, uint64_t np, const uint64_t* stf, uint64_t naf, uint64_t nf,
                             const uint64_t* str, uint64_t nar, uint64_t nr, unsigned long long* nunits) {
  for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < np; p += (uint64_t)gridDim.x * blockDim.x) {
    const Range r = range_of(pairs[p], stf, naf, nf, str, nar, nr);
    const uint64_t U = (r.fe - r.fb) + (r.re - r.rb);
    nunits[p] = (U + UNIT - 1) / UNIT;
  }
}

__device__ __forceinline__ u128 absdiff(u128 a, u128 b) { return a > b ? a - b : b - a; }

/* one warp per unit: partial K of union positions [u*UNIT, (u+1)*UNIT) of one pair */
__global__ void ks_unit_kernel(const Key128* fk, const unsigned long long* fpre, uint64_t nf, const uint64_t* stf,
                               uint64_t naf, const Key128* rk, const unsigned long long* rpre, uint64_t nr,
                               const uint64_t* str, uint64_t nar, const uint2* pairs, uint64_t np,
                               const unsigned long long* uoff, uint64_t total_units, u128* partial) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp0 = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t u = warp0; u < total_units; u += nwarps) {
    uint64_t lo = 0, hi = np; /* pair of unit u: last p with uoff[p] <= u */
    while (hi - lo > 1) {
      const uint64_t mid = (lo + hi) >> 1;
      if (uoff[mid] <= u) lo = mid; else hi = mid;
    }
    const Range r = range_of(pairs[lo], stf, naf, nf, str, nar, nr);
    const uint64_t nfa = r.fe - r.fb, nra = r.re - r.rb;
    const unsigned long long n = fpre[r.fe - 1], m = rpre[r.re - 1];
    const uint64_t d0 = (u - uoff[lo]) * UNIT + (uint64_t)lane * PER_LANE;
    const uint64_t d1 = d0 + PER_LANE < nfa + nra ? d0 + PER_LANE : nfa + nra;
    u128 K = 0;
    if (d0 < d1) {
      /* merge-path split: i fix elements among the first d0 union positions (ties: fix first) */
      uint64_t a = d0 > nra ? d0 - nra : 0, b = d0 < nfa ? d0 : nfa;
      while (a < b) {
        const uint64_t mid = (a + b) >> 1;
        if (fk[r.fb + mid].lo <= rk[r.rb + (d0 - mid - 1)].lo) a = mid + 1; else b = mid;
      }
      uint64_t i = a, j = d0 - a;
      unsigned long long A = i ? fpre[r.fb + i - 1] : 0ull, B = j ? rpre[r.rb + j - 1] : 0ull;
      for (uint64_t d = d0; d < d1; ++d) {
        unsigned long long x;
        if (i < nfa && (j >= nra || fk[r.fb + i].lo <= rk[r.rb + j].lo)) {
          x = fk[r.fb + i].lo;
          A = fpre[r.fb + i];
          ++i;
        } else {
          x = rk[r.rb + j].lo;
          B = rpre[r.rb + j];
          ++j;
        }
        /* evaluate after the last occurrence of x in the union */
        const bool more_f = i < nfa && fk[r.fb + i].lo == x;
        const bool more_r = j < nra && rk[r.rb + j].lo == x;
        if (!more_f && !more_r) {
          const u128 dd = absdiff((u128)A * m, (u128)B * n);
          if (dd > K) K = dd;
        }
      }
    }
    for (int o = 16; o > 0; o >>= 1) {
      const unsigned long long khi = __shfl_xor_sync(0xFFFFFFFFu, (unsigned long long)(K >> 64), o);
      const unsigned long long klo = __shfl_xor_sync(0xFFFFFFFFu, (unsigned long long)K, o);
      const u128 other = ((u128)khi << 64) | klo;
      if (other > K) K = other;
    }
    if (lane == 0) partial[u] = K;
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

/* ---- H_cf reading R2 (Eqs. 5-8) --------------------------------------------
 * The node's cells (prev, next) are weighted by a_ij = c_ij / x_i (x_i = the row's total, Eq. 5, so that
 * I.A = O, Eq. 7) and H = (a_11, ..., a_kp) (Eq. 8) is tested as a weighted sample: F(t) = sum_{cells<=t} a / k
 * with k = number of rows (= sum of all a).  Cells are row-major, so at a union position t = (p, q) a side's
 * F is (rows before p + cum_p(q) / x_p) / k when it has row p, else (rows before p) / k: one division per
 * side and position, in this fixed order.  One thread per attribute pair walks the two sorted lists (nodes
 * hold at most a few hundred cells; this is latency-bound, not a roofline kernel). */
struct R2State {
  uint64_t i, e;
  uint32_t rows, cur;
  bool have;
  unsigned long long cum, x;
};

__device__ __forceinline__ uint32_t prev_of(const Key128& k) { return (uint32_t)(k.lo >> 32); }

__device__ uint32_t r2_rows(const Key128* k, uint64_t b, uint64_t e) {
  uint32_t r = 0;
  for (uint64_t i = b; i < e; ++i) r += (i == b || prev_of(k[i]) != prev_of(k[i - 1])) ? 1u : 0u;
  return r;
}

__device__ void r2_step(const Key128* k, const unsigned long long* c, R2State& s, unsigned long long t) {
  if (s.i >= s.e || k[s.i].lo != t) return;
  const uint32_t p = (uint32_t)(t >> 32);
  if (!s.have || p != s.cur) {
    if (s.have) ++s.rows;
    s.have = true;
    s.cur = p;
    s.cum = 0;
    s.x = 0;
    for (uint64_t i = s.i; i < s.e && prev_of(k[i]) == p; ++i) s.x += c[i];
  }
  s.cum += c[s.i];
  ++s.i;
}

__device__ double r2_F(const R2State& s, uint32_t tp, double kd) {
  if (!s.have) return 0.0;
  if (s.cur == tp)
    return __ddiv_rn(__dadd_rn(__uint2double_rn(s.rows), __ddiv_rn(__ull2double_rn(s.cum), __ull2double_rn(s.x))),
                     kd);
  return __ddiv_rn(__uint2double_rn(s.rows + 1u), kd); /* its row before tp is complete */
}

__device__ __forceinline__ void ks_p_value(unsigned long long n, unsigned long long m, double D, double significance,
                                           double& pv, uint32_t& fail) {
  const double nd = __ull2double_rn(n), md = __ull2double_rn(m);
  const double nm = __dmul_rn(nd, md);
  const double wgt = __ddiv_rn(nm, __dadd_rn(nd, md));
  const double x = __dmul_rn(__dmul_rn(2.0, __dmul_rn(D, D)), wgt);
  pv = __dmul_rn(2.0, exp(-x));
  fail = pv < significance ? 1u : 0u;
}

__global__ void ks_r2_kernel(const Key128* fk, const unsigned long long* fc, const unsigned long long* fpre, uint64_t nf,
                             const uint64_t* stf, uint64_t naf, const Key128* rk, const unsigned long long* rc,
                             const unsigned long long* rpre, uint64_t nr, const uint64_t* str, uint64_t nar,
                             const uint2* pairs, uint64_t np, double significance, KsOutRow* out) {
  for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < np; p += (uint64_t)gridDim.x * blockDim.x) {
    const Range r = range_of(pairs[p], stf, naf, nf, str, nar, nr);
    const unsigned long long n = fpre[r.fe - 1], m = rpre[r.re - 1];
    const double kf = __uint2double_rn(r2_rows(fk, r.fb, r.fe)), kr = __uint2double_rn(r2_rows(rk, r.rb, r.re));
    R2State a{r.fb, r.fe, 0u, 0u, false, 0ull, 0ull}, b{r.rb, r.re, 0u, 0u, false, 0ull, 0ull};
    double D = 0.0;
    while (a.i < a.e || b.i < b.e) {
      const unsigned long long t =
          (a.i < a.e && (b.i >= b.e || fk[a.i].lo <= rk[b.i].lo)) ? fk[a.i].lo : rk[b.i].lo;
      r2_step(fk, fc, a, t);
      r2_step(rk, rc, b, t);
      const uint32_t tp = (uint32_t)(t >> 32);
      const double d = fabs(__dsub_rn(r2_F(a, tp, kf), r2_F(b, tp, kr)));
      if (d > D) D = d;
    }
    KsOutRow o;
    o.hi_f = fk[r.fb].hi;
    o.hi_r = rk[r.rb].hi;
    o.n = n;
    o.m = m;
    o.K_lo = 0;
    o.K_hi = 0;
    o.D = D;
    ks_p_value(n, m, D, significance, o.p, o.fail);
    o._pad = 0;
    out[p] = o;
  }
}

__global__ void ks_final_kernel(const Key128* fk, const unsigned long long* fpre, uint64_t nf, const uint64_t* stf,
                                uint64_t naf, const Key128* rk, const unsigned long long* rpre, uint64_t nr,
                                const uint64_t* str, uint64_t nar, const uint2* pairs, uint64_t np,
                                const unsigned long long* uoff, const unsigned long long* nunits, const u128* partial,
                                double significance, KsOutRow* out) {
  for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < np; p += (uint64_t)gridDim.x * blockDim.x) {
    const Range r = range_of(pairs[p], stf, naf, nf, str, nar, nr);
    const unsigned long long n = fpre[r.fe - 1], m = rpre[r.re - 1];
    u128 K = 0;
    for (unsigned long long q = 0; q < nunits[p]; ++q)
      if (partial[uoff[p] + q] > K) K = partial[uoff[p] + q];
    const double nd = __ull2double_rn(n), md = __ull2double_rn(m);
    const double nm = __dmul_rn(nd, md);
    const double D = __ddiv_rn(u128_to_double_rn(K), nm);
    const double wgt = __ddiv_rn(nm, __dadd_rn(nd, md));
    const double x = __dmul_rn(__dmul_rn(2.0, __dmul_rn(D, D)), wgt);
    const double pv = __dmul_rn(2.0, exp(-x));
    KsOutRow o;
    o.hi_f = fk[r.fb].hi;
    o.hi_r = rk[r.rb].hi;
    o.n = n;
    o.m = m;
    o.K_lo = (unsigned long long)K;
    o.K_hi = (unsigned long long)(K >> 64);
    o.D = D;
    o.p = pv;
    o.fail = pv < significance ? 1u : 0u;
    o._pad = 0;
    out[p] = o;
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
    owl_dev_free(hi); owl_dev_free(st); owl_dev_free(pre); owl_dev_free(starts); owl_dev_free(nattr);
  }
};

int grid_for(uint64_t n, int block) {
  uint64_t g = (n + block - 1) / block;
  if (g > 148ull * 16) g = 148ull * 16;
  return g ? (int)g : 1;
}

cudaError_t prepare(const SortedTable& t, Side& s, cudaStream_t st) {
  const uint64_t n = t.n;
  s.hi = (unsigned long long*)owl_dev_alloc((n + 1) * 8);
  s.st = (unsigned char*)owl_dev_alloc(n + 1);
  s.pre = (unsigned long long*)owl_dev_alloc((n + 1) * 8);
  s.starts = (uint64_t*)owl_dev_alloc((n + 1) * 8);
  s.nattr = (unsigned long long*)owl_dev_alloc(8);
  if (!s.hi || !s.st || !s.pre || !s.starts || !s.nattr) return cudaErrorMemoryAllocation;
  if (!n) return cudaSuccess;
  extract_hi_kernel<<<grid_for(n, 256), 256, 0, st>>>(t.k, n, s.hi, s.st);
  size_t t1 = 0, t2 = 0;
  cub::DeviceSelect::Flagged(nullptr, t1, thrust::counting_iterator<uint64_t>(0), s.st, s.starts, s.nattr, (int64_t)n, st);
  cub::DeviceScan::InclusiveSumByKey(nullptr, t2, s.hi, t.c, s.pre, (int64_t)n, cub::Equality(), st);
  void* tmp = owl_dev_alloc((t1 > t2 ? t1 : t2) + 16);
  if (!tmp) return cudaErrorMemoryAllocation;
  cudaError_t e = cub::DeviceSelect::Flagged(tmp, t1, thrust::counting_iterator<uint64_t>(0), s.st, s.starts, s.nattr,
                                             (int64_t)n, st);
  if (e == cudaSuccess) e = cub::DeviceScan::InclusiveSumByKey(tmp, t2, s.hi, t.c, s.pre, (int64_t)n, cub::Equality(), st);
  unsigned long long na = 0;
  if (e == cudaSuccess) e = cudaMemcpyAsync(&na, s.nattr, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  owl_dev_free(tmp);
  s.na = na;
  return e;
}

}  // namespace

cudaError_t owl_ks_run(int tbl, const SortedTable& f, const SortedTable& r, const std::vector<uint32_t>& slot_f2r,
                       double significance, int hcf_reading, std::vector<KsOutRow>& rows, cudaStream_t st) {
  rows.clear();
  if (!f.n || !r.n || slot_f2r.empty()) return cudaSuccess;
  Side sf, sr;
  uint32_t* dmap = nullptr;
  uint2* pairs = nullptr;
  unsigned long long *npairs = nullptr, *nunits = nullptr, *uoff = nullptr;
  u128* partial = nullptr;
  KsOutRow* dout = nullptr;
  void* tmp = nullptr;
  cudaError_t e = prepare(f, sf, st);
  if (e == cudaSuccess) e = prepare(r, sr, st);
  unsigned long long np = 0;
  if (e == cudaSuccess) {
    dmap = (uint32_t*)owl_dev_alloc(slot_f2r.size() * 4);
    pairs = (uint2*)owl_dev_alloc((sf.na + 1) * sizeof(uint2));
    npairs = (unsigned long long*)owl_dev_alloc(8);
    if (!dmap || !pairs || !npairs) e = cudaErrorMemoryAllocation;
  }
  if (e == cudaSuccess) {
    cudaMemcpyAsync(dmap, slot_f2r.data(), slot_f2r.size() * 4, cudaMemcpyHostToDevice, st);
    cudaMemsetAsync(npairs, 0, 8, st);
    pair_kernel<<<grid_for(sf.na, 256), 256, 0, st>>>(tbl, sf.hi, sf.starts, sf.na, sr.hi, sr.starts, sr.na, dmap,
                                                      (uint32_t)slot_f2r.size(), pairs, npairs);
    e = cudaMemcpyAsync(&np, npairs, 8, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  }
  if (e == cudaSuccess && np && tbl == T_TRIPLE && hcf_reading == OWL_HCF_ROW_NORMALIZED) {
    dout = (KsOutRow*)owl_dev_alloc(np * sizeof(KsOutRow));
    if (!dout) e = cudaErrorMemoryAllocation;
    if (e == cudaSuccess) {
      ks_r2_kernel<<<grid_for(np, 128), 128, 0, st>>>(f.k, f.c, sf.pre, f.n, sf.starts, sf.na, r.k, r.c, sr.pre, r.n,
                                                      sr.starts, sr.na, pairs, np, significance, dout);
      rows.resize(np);
      e = cudaMemcpyAsync(rows.data(), dout, np * sizeof(KsOutRow), cudaMemcpyDeviceToHost, st);
      if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    }
  } else if (e == cudaSuccess && np) {
    nunits = (unsigned long long*)owl_dev_alloc(np * 8);
    uoff = (unsigned long long*)owl_dev_alloc((np + 1) * 8);
    dout = (KsOutRow*)owl_dev_alloc(np * sizeof(KsOutRow));
    if (!nunits || !uoff || !dout) e = cudaErrorMemoryAllocation;
    unsigned long long total = 0;
    if (e == cudaSuccess) {
      units_kernel<<<grid_for(np, 256), 256, 0, st>>>(pairs, np, sf.starts, sf.na, f.n, sr.starts, sr.na, r.n, nunits);
      size_t tb = 0;
      cub::DeviceScan::InclusiveSum(nullptr, tb, nunits, uoff + 1, (int64_t)np, st);
      tmp = owl_dev_alloc(tb + 16);
      if (!tmp) e = cudaErrorMemoryAllocation;
      if (e == cudaSuccess) {
        cudaMemsetAsync(uoff, 0, 8, st);
        e = cub::DeviceScan::InclusiveSum(tmp, tb, nunits, uoff + 1, (int64_t)np, st);
      }
      if (e == cudaSuccess) e = cudaMemcpyAsync(&total, uoff + np, 8, cudaMemcpyDeviceToHost, st);
      if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    }
    if (e == cudaSuccess) {
      partial = (u128*)owl_dev_alloc((total + 1) * sizeof(u128));
      if (!partial) e = cudaErrorMemoryAllocation;
    }
    if (e == cudaSuccess) {
      ks_unit_kernel<<<grid_for(total * 32, 256), 256, 0, st>>>(f.k, sf.pre, f.n, sf.starts, sf.na, r.k, sr.pre, r.n,
                                                                  sr.starts, sr.na, pairs, np, uoff, total, partial);
      ks_final_kernel<<<grid_for(np, 128), 128, 0, st>>>(f.k, sf.pre, f.n, sf.starts, sf.na, r.k, sr.pre, r.n, sr.starts,
                                                         sr.na, pairs, np, uoff, nunits, partial, significance, dout);
      rows.resize(np);
      e = cudaMemcpyAsync(rows.data(), dout, np * sizeof(KsOutRow), cudaMemcpyDeviceToHost, st);
      if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    }
  }
  sf.free_all();
  sr.free_all();
  owl_dev_free(dmap); owl_dev_free(pairs); owl_dev_free(npairs); owl_dev_free(nunits); owl_dev_free(uoff);
  owl_dev_free(dout); owl_dev_free(partial); owl_dev_free(tmp);
  if (e == cudaSuccess) e = cudaGetLastError();
  return e;
}
