/*
 * owl_tables.cu — A-DCFG table management: allocation, canonical export order (compaction + 128-bit radix
 * sort), table merge (evidence accumulation / absorb), the A5 diff (full outer join on canonical keys,
 * P:L227-229), and stable bucketing of channel-order input by warp (reading R17).
 */
#include <cub/cub.cuh>
#include <thrust/iterator/counting_iterator.h>
#include <cuda/std/tuple>
#include <cuda_runtime.h>

#include <map>
#include <mutex>
#include <vector>

#include "owl_device.cuh"
#include "owl_internal.h"

using namespace owl_dev;

namespace {

struct KeyDecomp {
  __host__ __device__ ::cuda::std::tuple<unsigned long long&, unsigned long long&> operator()(Key128& k) const {
    return {k.hi, k.lo}; /* most significant first */
  }
};

__global__ void clear_kernel(owl_bucket* b, uint64_t nb) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nb; i += (uint64_t)gridDim.x * blockDim.x) {
    reinterpret_cast<ulonglong4*>(&b[i])[0] = make_ulonglong4(OWL_EMPTY_KEY, OWL_EMPTY_KEY, OWL_EMPTY_KEY, OWL_EMPTY_KEY);
    reinterpret_cast<ulonglong4*>(&b[i])[1] = make_ulonglong4(0, 0, 0, 0);
  }
}

/* compaction of non-empty cells (order is irrelevant: a sort follows) */
__global__ void compact_kernel(const owl_bucket* c, uint64_t cap, Key128* k, unsigned long long* cnt,
                               unsigned long long* n_out) {
  const int lane = threadIdx.x & 31;
  for (uint64_t base = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) & ~31ull; base < cap;
       base += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t i = base + lane;
    unsigned long long vhi = OWL_EMPTY_KEY, vlo = 0, vc = 0;
    bool live = false;
    if (i < cap) {
      vhi = c[i >> 1].key[i & 1][0];
      vlo = c[i >> 1].key[i & 1][1];
      vc = c[i >> 1].count[i & 1];
      live = vhi != OWL_EMPTY_KEY;
    }
    const unsigned m = __ballot_sync(0xFFFFFFFFu, live);
    unsigned long long b = 0;
    if (lane == 0 && m) b = atomicAdd(n_out, (unsigned long long)__popc(m));
    b = __shfl_sync(0xFFFFFFFFu, b, 0);
    if (live) {
      const uint64_t o = b + __popc(m & ((1u << lane) - 1u));
      k[o].hi = vhi;
      k[o].lo = vlo;
      cnt[o] = vc;
    }
  }
}

__global__ void insert_sorted_kernel(DevTable t, int tbl, const Key128* k, const unsigned long long* c, uint64_t n,
                                     FoldStatus* st) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    g_insert(t, tbl, k[i].hi, k[i].lo, c[i], st);
}

__device__ __forceinline__ bool key_less(const Key128& a, const Key128& b) {
  return a.hi < b.hi || (a.hi == b.hi && a.lo < b.lo);
}

/* index of key in sorted array, or n */
__device__ uint64_t find_key(const Key128* k, uint64_t n, const Key128& q) {
  uint64_t lo = 0, hi = n;
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (key_less(k[mid], q)) lo = mid + 1; else hi = mid;
  }
  return (lo < n && k[lo].hi == q.hi && k[lo].lo == q.lo) ? lo : n;
}

/* A side: flag cells absent from B or with a different count; B side: flag cells absent from A */
__global__ void diff_flag_kernel(const Key128* ak, const unsigned long long* ac, uint64_t na, const Key128* bk,
                                 const unsigned long long* bc, uint64_t nb, unsigned char* fa, unsigned long long* cb_of_a,
                                 unsigned char* fb) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < na; i += stride) {
    const uint64_t j = find_key(bk, nb, ak[i]);
    const unsigned long long cbv = j < nb ? bc[j] : 0ull;
    cb_of_a[i] = cbv;
    fa[i] = (j >= nb || cbv != ac[i]) ? 1 : 0;
  }
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nb; i += stride)
    fb[i] = find_key(ak, na, bk[i]) >= na ? 1 : 0;
}

__global__ void gather_diff_kernel(const uint64_t* idx, const unsigned long long* nsel, const Key128* k,
                                   const unsigned long long* c, const unsigned long long* other, int a_side,
                                   DiffCell* out) {
  const uint64_t n = *nsel;
  for (uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; t < n; t += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t i = idx[t];
    DiffCell d;
    d.k = k[i];
    if (a_side) { d.ca = c[i]; d.cb = other[i]; }
    else { d.ca = 0; d.cb = c[i]; }
    out[t] = d;
  }
}

__global__ void bucket_keys_kernel(const uint4* rec, uint64_t n, uint32_t* gw, uint64_t* idx) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    gw[i] = rec[i].z;
    idx[i] = i;
  }
}

__global__ void gather_records_kernel(const uint4* rec, const uint64_t* perm, uint64_t n, uint4* out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = rec[perm[i]];
}

int grid_for(uint64_t n, int block) {
  uint64_t g = (n + block - 1) / block;
  if (g > 148ull * 16) g = 148ull * 16;
  return g ? (int)g : 1;
}

}  // namespace

/* Caching device allocator: blocks are rounded up to a power of two (>= 256 B) and recycled per device,
   so the per-call scratch of build / sort / diff / KS never hits cudaMalloc / cudaFree (which synchronize
   the device) in steady state.  All library work of a context runs on its one stream, so a block freed
   by one call and reused by the next is ordered by that stream. */
namespace {
std::mutex g_pool_mu;
std::map<std::pair<int, size_t>, std::vector<void*>> g_pool;   /* (device, size) -> free blocks */
std::map<void*, std::pair<int, size_t>> g_live;                /* block -> (device, size) */
}  // namespace

void* owl_dev_alloc(size_t bytes) {
  size_t sz = 256;
  while (sz < bytes) sz <<= 1;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(g_pool_mu);
  auto it = g_pool.find({dev, sz});
  void* p = nullptr;
  if (it != g_pool.end() && !it->second.empty()) {
    p = it->second.back();
    it->second.pop_back();
  } else if (cudaMalloc(&p, sz) != cudaSuccess) {
    cudaGetLastError();
    for (auto& f : g_pool) /* release cached blocks of this device and retry once */
      if (f.first.first == dev) {
        for (void* q : f.second) cudaFree(q);
        f.second.clear();
      }
    if (cudaMalloc(&p, sz) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
  }
  g_live[p] = {dev, sz};
  return p;
}

void owl_dev_free(void* p) {
  if (!p) return;
  std::lock_guard<std::mutex> lk(g_pool_mu);
  auto it = g_live.find(p);
  if (it == g_live.end()) return;
  g_pool[it->second].push_back(p);
  g_live.erase(it);
}

void owl_dev_trim(int dev) {
  std::lock_guard<std::mutex> lk(g_pool_mu);
  for (auto& f : g_pool)
    if (f.first.first == dev) {
      for (void* q : f.second) cudaFree(q);
      f.second.clear();
    }
}

cudaError_t owl_table_alloc(DevTable* t, uint64_t cap, cudaStream_t st) {
  if (cap < 2 || cap > OWL_MAX_TABLE_CELLS || (cap & (cap - 1))) return cudaErrorInvalidValue;
  t->cap = cap;
  t->b = (owl_bucket*)owl_dev_alloc((cap / 2) * sizeof(owl_bucket));
  t->fill = (unsigned long long*)owl_dev_alloc(sizeof(unsigned long long));
  if (!t->b || !t->fill) {
    owl_table_free(t);
    return cudaErrorMemoryAllocation;
  }
  clear_kernel<<<grid_for(cap / 2, 256), 256, 0, st>>>(t->b, cap / 2);
  cudaMemsetAsync(t->fill, 0, sizeof(unsigned long long), st);
  return cudaGetLastError();
}

void owl_table_free(DevTable* t) {
  owl_dev_free(t->b);
  owl_dev_free(t->fill);
  t->b = nullptr;
  t->fill = nullptr;
  t->cap = 0;
}

void owl_sorted_free(SortedTable* s) {
  owl_dev_free(s->k);
  owl_dev_free(s->c);
  s->k = nullptr;
  s->c = nullptr;
  s->n = 0;
}

cudaError_t owl_table_sorted(const DevTable& t, SortedTable* out, cudaStream_t st) {
  unsigned long long n = 0;
  cudaError_t e = cudaMemcpyAsync(&n, t.fill, sizeof n, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return e;
  Key128* k0 = (Key128*)owl_dev_alloc(n * sizeof(Key128));
  unsigned long long* c0 = (unsigned long long*)owl_dev_alloc(n * sizeof(unsigned long long));
  out->k = (Key128*)owl_dev_alloc(n * sizeof(Key128));
  out->c = (unsigned long long*)owl_dev_alloc(n * sizeof(unsigned long long));
  unsigned long long* dn = (unsigned long long*)owl_dev_alloc(sizeof(unsigned long long));
  if (!k0 || !c0 || !out->k || !out->c || !dn) {
    owl_dev_free(k0); owl_dev_free(c0); owl_dev_free(dn); owl_sorted_free(out);
    return cudaErrorMemoryAllocation;
  }
  cudaMemsetAsync(dn, 0, sizeof(unsigned long long), st);
  compact_kernel<<<grid_for(t.cap, 256), 256, 0, st>>>(t.b, t.cap, k0, c0, dn);
  size_t tmp = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, tmp, k0, out->k, c0, out->c, (int64_t)n, KeyDecomp{}, st);
  void* dt = owl_dev_alloc(tmp);
  if (!dt) e = cudaErrorMemoryAllocation;
  else e = cub::DeviceRadixSort::SortPairs(dt, tmp, k0, out->k, c0, out->c, (int64_t)n, KeyDecomp{}, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  owl_dev_free(dt); owl_dev_free(k0); owl_dev_free(c0); owl_dev_free(dn);
  out->n = n;
  return e;
}

cudaError_t owl_table_insert_sorted(const DevTable& t, int tbl, const Key128* k, const unsigned long long* c,
                                    uint64_t n, FoldStatus* st_dev, cudaStream_t st) {
  if (!n) return cudaSuccess;
  insert_sorted_kernel<<<grid_for(n, 256), 256, 0, st>>>(t, tbl, k, c, n, st_dev);
  return cudaGetLastError();
}

cudaError_t owl_diff_sorted(const SortedTable& a, const SortedTable& b, std::vector<DiffCell>& out, cudaStream_t st) {
  out.clear();
  const uint64_t na = a.n, nb = b.n;
  unsigned char* fa = (unsigned char*)owl_dev_alloc(na + 1);
  unsigned char* fb = (unsigned char*)owl_dev_alloc(nb + 1);
  unsigned long long* cboa = (unsigned long long*)owl_dev_alloc((na + 1) * 8);
  uint64_t* ia = (uint64_t*)owl_dev_alloc((na + 1) * 8);
  uint64_t* ib = (uint64_t*)owl_dev_alloc((nb + 1) * 8);
  unsigned long long* nsel = (unsigned long long*)owl_dev_alloc(16);
  DiffCell* da = (DiffCell*)owl_dev_alloc((na + 1) * sizeof(DiffCell));
  DiffCell* db = (DiffCell*)owl_dev_alloc((nb + 1) * sizeof(DiffCell));
  cudaError_t e = cudaSuccess;
  void* dt = nullptr;
  if (!fa || !fb || !cboa || !ia || !ib || !nsel || !da || !db) e = cudaErrorMemoryAllocation;
  if (e == cudaSuccess) {
    diff_flag_kernel<<<grid_for(na > nb ? na : nb, 256), 256, 0, st>>>(a.k, a.c, na, b.k, b.c, nb, fa, cboa, fb);
    size_t tmp = 0, tmp2 = 0;
    cub::DeviceSelect::Flagged(nullptr, tmp, thrust::counting_iterator<uint64_t>(0), fa, ia, nsel, (int64_t)na, st);
    cub::DeviceSelect::Flagged(nullptr, tmp2, thrust::counting_iterator<uint64_t>(0), fb, ib, nsel + 1, (int64_t)nb, st);
    if (tmp2 > tmp) tmp = tmp2;
    dt = owl_dev_alloc(tmp);
    if (!dt) e = cudaErrorMemoryAllocation;
  }
  unsigned long long hn[2] = {0, 0};
  if (e == cudaSuccess) {
    size_t tmp = 0;
    cub::DeviceSelect::Flagged(nullptr, tmp, thrust::counting_iterator<uint64_t>(0), fa, ia, nsel, (int64_t)na, st);
    e = cub::DeviceSelect::Flagged(dt, tmp, thrust::counting_iterator<uint64_t>(0), fa, ia, nsel, (int64_t)na, st);
    tmp = 0;
    cub::DeviceSelect::Flagged(nullptr, tmp, thrust::counting_iterator<uint64_t>(0), fb, ib, nsel + 1, (int64_t)nb, st);
    if (e == cudaSuccess)
      e = cub::DeviceSelect::Flagged(dt, tmp, thrust::counting_iterator<uint64_t>(0), fb, ib, nsel + 1, (int64_t)nb, st);
    if (e == cudaSuccess) {
      gather_diff_kernel<<<grid_for(na, 256), 256, 0, st>>>(ia, nsel, a.k, a.c, cboa, 1, da);
      gather_diff_kernel<<<grid_for(nb, 256), 256, 0, st>>>(ib, nsel + 1, b.k, b.c, nullptr, 0, db);
      e = cudaMemcpyAsync(hn, nsel, 16, cudaMemcpyDeviceToHost, st);
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  }
  std::vector<DiffCell> ha(hn[0]), hb(hn[1]);
  if (e == cudaSuccess && hn[0]) e = cudaMemcpy(ha.data(), da, hn[0] * sizeof(DiffCell), cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && hn[1]) e = cudaMemcpy(hb.data(), db, hn[1] * sizeof(DiffCell), cudaMemcpyDeviceToHost);
  if (e == cudaSuccess) { /* merge the two canonical-order lists */
    out.reserve(ha.size() + hb.size());
    size_t i = 0, j = 0;
    while (i < ha.size() || j < hb.size()) {
      if (j >= hb.size() || (i < ha.size() && (ha[i].k.hi < hb[j].k.hi ||
                                                (ha[i].k.hi == hb[j].k.hi && ha[i].k.lo < hb[j].k.lo))))
        out.push_back(ha[i++]);
      else
        out.push_back(hb[j++]);
    }
  }
  owl_dev_free(fa); owl_dev_free(fb); owl_dev_free(cboa); owl_dev_free(ia); owl_dev_free(ib);
  owl_dev_free(nsel); owl_dev_free(da); owl_dev_free(db); owl_dev_free(dt);
  return e;
}

cudaError_t owl_bucket_by_warp(const uint4* rec, uint64_t n, uint32_t n_warps, uint4* out, uint64_t* perm,
                               cudaStream_t st) {
  if (!n) return cudaSuccess;
  uint32_t* gw = (uint32_t*)owl_dev_alloc(n * 4);
  uint32_t* gw2 = (uint32_t*)owl_dev_alloc(n * 4);
  uint64_t* idx = (uint64_t*)owl_dev_alloc(n * 8);
  cudaError_t e = (gw && gw2 && idx) ? cudaSuccess : cudaErrorMemoryAllocation;
  void* dt = nullptr;
  if (e == cudaSuccess) {
    bucket_keys_kernel<<<grid_for(n, 256), 256, 0, st>>>(rec, n, gw, idx);
    int bits = 1;
    while (bits < 32 && (1ull << bits) <= (uint64_t)n_warps) ++bits; /* gwarp >= n_warps sorts last (bit 31) */
    bits = 32;  /* records with out-of-range gwarp must keep their relative order too */
    size_t tmp = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, tmp, gw, gw2, idx, perm, (int64_t)n, 0, bits, st);
    dt = owl_dev_alloc(tmp);
    if (!dt) e = cudaErrorMemoryAllocation;
    else e = cub::DeviceRadixSort::SortPairs(dt, tmp, gw, gw2, idx, perm, (int64_t)n, 0, bits, st);
    if (e == cudaSuccess) gather_records_kernel<<<grid_for(n, 256), 256, 0, st>>>(rec, perm, n, out);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  }
  owl_dev_free(gw); owl_dev_free(gw2); owl_dev_free(idx); owl_dev_free(dt);
  return e == cudaSuccess ? cudaGetLastError() : e;
}
