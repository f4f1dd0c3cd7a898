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

/* compaction of non-empty cells (order is irrelevant: a sort follows); also the bitwise OR and AND of the
   live keys (bits that vary across the table: the radix sort needs only those) */
__global__ void compact_kernel(const owl_bucket* c, uint64_t cap, Key128* k, unsigned long long* cnt,
                               unsigned long long* n_out, unsigned long long* masks /* or_hi, or_lo, and_hi, and_lo */) {
  /* each warp takes CW x 32 cells at a time and claims their output slots with ONE atomic (the table is mostly
     empty: one atomic per 32 cells serialised on n_out) */
  constexpr int CW = 8;
  const int lane = threadIdx.x & 31;
  unsigned long long ohi = 0, olo = 0, ahi = ~0ull, alo = ~0ull;
  const uint64_t step = (uint64_t)gridDim.x * blockDim.x * CW;
  for (uint64_t base = ((blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) & ~31ull) * CW; base < cap; base += step) {
    ulonglong2 kv[CW];
    unsigned long long cv[CW];
    unsigned m[CW];
    unsigned tot = 0;
#pragma unroll
    for (int u = 0; u < CW; ++u) {
      const uint64_t i = base + u * 32 + lane;
      kv[u] = make_ulonglong2(OWL_EMPTY_KEY, 0);
      cv[u] = 0;
      if (i < cap) {
        kv[u] = *reinterpret_cast<const ulonglong2*>(&c[i >> 1].key[i & 1][0]);
        cv[u] = c[i >> 1].count[i & 1];
      }
    }
#pragma unroll
    for (int u = 0; u < CW; ++u) {
      m[u] = __ballot_sync(0xFFFFFFFFu, kv[u].x != OWL_EMPTY_KEY);
      tot += __popc(m[u]);
    }
    if (!tot) continue;
    unsigned long long b = 0;
    if (lane == 0) b = atomicAdd(n_out, (unsigned long long)tot);
    b = __shfl_sync(0xFFFFFFFFu, b, 0);
#pragma unroll
    for (int u = 0; u < CW; ++u) {
      if (kv[u].x != OWL_EMPTY_KEY) {
        const uint64_t o = b + __popc(m[u] & ((1u << lane) - 1u));
        k[o].hi = kv[u].x;
        k[o].lo = kv[u].y;
        cnt[o] = cv[u];
        ohi |= kv[u].x;
        olo |= kv[u].y;
        ahi &= kv[u].x;
        alo &= kv[u].y;
      }
      b += __popc(m[u]);
    }
  }
  for (int o = 16; o; o >>= 1) {
    ohi |= __shfl_xor_sync(0xFFFFFFFFu, ohi, o);
    olo |= __shfl_xor_sync(0xFFFFFFFFu, olo, o);
    ahi &= __shfl_xor_sync(0xFFFFFFFFu, ahi, o);
    alo &= __shfl_xor_sync(0xFFFFFFFFu, alo, o);
  }
  if (lane == 0) {
    atomicOr(&masks[0], ohi);
    atomicOr(&masks[1], olo);
    atomicAnd(&masks[2], ahi);
    atomicAnd(&masks[3], alo);
  }
}

/* Order-preserving key compaction for the radix sort: the bits that vary across a table's keys, packed
   (hi's above lo's, each in significance order) into one u64 — equal constant bits make the packed
   order the (hi, lo) order.  Runs are (shift, length) of the varying-bit mask, packed from the top. */
struct PackRuns {
  int n;
  unsigned char word[48], shift[48], len[48], pos[48];
};

__global__ void pack_kernel(const Key128* k, uint64_t n, PackRuns r, unsigned long long* ck, uint32_t* idx) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const Key128 q = k[i];
    unsigned long long v = 0;
    for (int t = 0; t < r.n; ++t) {
      const unsigned long long w = r.word[t] ? q.lo : q.hi;
      const unsigned long long f = (w >> r.shift[t]) & (r.len[t] == 64 ? ~0ull : ((1ull << r.len[t]) - 1));
      v |= f << r.pos[t];
    }
    ck[i] = v;
    idx[i] = (uint32_t)i;
  }
}

__global__ void gather_sorted_kernel(const Key128* k0, const unsigned long long* c0, const uint32_t* idx, uint64_t n,
                                     Key128* k, unsigned long long* c) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t j = idx[i];
    k[i] = k0[j];
    c[i] = c0[j];
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

int grid_for(uint64_t n, int block) {
  uint64_t g = (n + block - 1) / block;
  if (g > 148ull * 16) g = 148ull * 16;
  return g ? (int)g : 1;
}

}  // namespace

/* Caching device allocator: blocks are rounded up to a power of two (>= 256 B; above 1 GiB to a multiple of
   1 GiB, so a 22 GB scratch does not hold 32 GB) and recycled per device,
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
  if (bytes > (1ull << 30)) sz = (bytes + (1ull << 30) - 1) & ~((1ull << 30) - 1);
  else while (sz < bytes) sz <<= 1;
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

/* Pinned host blocks for result rows (diff rows can be millions): a D2H copy into pinned memory runs at PCIe
   speed, into fresh pageable memory it is staged and page-faulted.  Blocks are cached by power-of-two size
   class (at most kHostCache bytes kept); owl_host_free returns them, and frees plain malloc blocks. */
namespace {
std::mutex g_host_mu;
std::map<size_t, std::vector<void*>> g_host_pool;
std::map<void*, size_t> g_host_live;
size_t g_host_cached = 0;
const size_t kHostCache = 4ull << 30;
}  // namespace

void* owl_host_alloc(size_t bytes) {
  size_t sz = 4096;
  while (sz < bytes) sz <<= 1;
  std::lock_guard<std::mutex> lk(g_host_mu);
  auto it = g_host_pool.find(sz);
  void* p = nullptr;
  if (it != g_host_pool.end() && !it->second.empty()) {
    p = it->second.back();
    it->second.pop_back();
    g_host_cached -= sz;
  } else if (cudaMallocHost(&p, sz) != cudaSuccess) {
    cudaGetLastError();
    return malloc(bytes ? bytes : 1); /* not pinned: owl_host_free frees it */
  }
  g_host_live[p] = sz;
  return p;
}

void owl_host_free(void* p) {
  if (!p) return;
  std::lock_guard<std::mutex> lk(g_host_mu);
  auto it = g_host_live.find(p);
  if (it == g_host_live.end()) {
    free(p);
    return;
  }
  const size_t sz = it->second;
  g_host_live.erase(it);
  if (g_host_cached + sz <= kHostCache) {
    g_host_pool[sz].push_back(p);
    g_host_cached += sz;
  } else {
    cudaFreeHost(p);
  }
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

/* varying-bit runs of (hi, lo) masks, packed from bit nb-1 down; false if more than 64 bits vary */
static bool pack_runs(unsigned long long mhi, unsigned long long mlo, PackRuns* r, int* nb) {
  const int total = __builtin_popcountll(mhi) + __builtin_popcountll(mlo);
  if (total > 64) return false;
  r->n = 0;
  int top = total;
  for (int word = 0; word < 2; ++word) {
    unsigned long long m = word ? mlo : mhi;
    /* most significant run first */
    while (m) {
      const int hb = 63 - __builtin_clzll(m);
      int lb = hb;
      while (lb > 0 && ((m >> (lb - 1)) & 1)) --lb;
      const int len = hb - lb + 1;
      if (r->n >= 48) return false;
      top -= len;
      r->word[r->n] = (unsigned char)word;
      r->shift[r->n] = (unsigned char)lb;
      r->len[r->n] = (unsigned char)len;
      r->pos[r->n] = (unsigned char)top;
      ++r->n;
      m &= (len == 64) ? 0ull : ~(((1ull << len) - 1) << lb);
    }
  }
  *nb = total;
  return true;
}

/* Canonical order of ntab tables at once (compaction, then a radix sort of the packed varying key bits,
   or of the full 128-bit keys for small tables); three host synchronisations in all. */
/* Small tables sorted by one CTA: keys (distinct) and counts in shared memory, padded to a power of two with
   all-ones keys, bitonic sort by (hi, lo) unsigned (the canonical order), then written out. */
#define SMALL_SORT_MAX 4096
namespace {
__global__ void __launch_bounds__(1024) small_sort_kernel(const Key128* k, const unsigned long long* c, uint64_t n,
                                                          uint32_t np2, Key128* ko, unsigned long long* co) {
  extern __shared__ __align__(16) unsigned char sm[];
  Key128* sk = reinterpret_cast<Key128*>(sm);
  unsigned long long* sc = reinterpret_cast<unsigned long long*>(sk + np2);
  for (uint32_t i = threadIdx.x; i < np2; i += blockDim.x) {
    if (i < n) {
      sk[i] = k[i];
      sc[i] = c[i];
    } else {
      sk[i].hi = ~0ull;
      sk[i].lo = ~0ull;
      sc[i] = 0;
    }
  }
  __syncthreads();
  for (uint32_t size = 2; size <= np2; size <<= 1)
    for (uint32_t stride = size >> 1; stride; stride >>= 1) {
      for (uint32_t t = threadIdx.x; t < np2 / 2; t += blockDim.x) {
        const uint32_t lo = 2 * t - (t & (stride - 1)), hi = lo + stride; /* the pair (lo, hi) of this step */
        const bool up = (lo & size) == 0;
        const Key128 a = sk[lo], b = sk[hi];
        const bool gt = a.hi > b.hi || (a.hi == b.hi && a.lo > b.lo);
        if (gt == up) {
          sk[lo] = b;
          sk[hi] = a;
          const unsigned long long x = sc[lo];
          sc[lo] = sc[hi];
          sc[hi] = x;
        }
      }
      __syncthreads();
    }
  for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
    ko[i] = sk[i];
    co[i] = sc[i];
  }
}
}  // namespace

static cudaError_t small_sort(const Key128* k, const unsigned long long* c, uint64_t n, Key128* ko,
                              unsigned long long* co, cudaStream_t st) {
  uint32_t np2 = 2;
  while (np2 < n) np2 <<= 1;
  const size_t smem = (size_t)np2 * (sizeof(Key128) + 8);
  static bool attr = false;
  if (!attr) {
    const cudaError_t e = cudaFuncSetAttribute(small_sort_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                               (int)(SMALL_SORT_MAX * (sizeof(Key128) + 8)));
    if (e != cudaSuccess) return e;
    attr = true;
  }
  small_sort_kernel<<<1, 1024, smem, st>>>(k, c, n, np2, ko, co);
  return cudaGetLastError();
}

cudaError_t owl_tables_sorted(const DevTable* t, int ntab, SortedTable* out, cudaStream_t st) {
  std::vector<unsigned long long> n(ntab, 0);
  cudaError_t e = cudaSuccess;
  for (int i = 0; i < ntab && e == cudaSuccess; ++i) e = cudaMemcpyAsync(&n[i], t[i].fill, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return e;
  std::vector<void*> scratch;
  auto alloc = [&](size_t bytes) { void* p = owl_dev_alloc(bytes); scratch.push_back(p); return p; };
  std::vector<Key128*> k0(ntab);
  std::vector<unsigned long long*> c0(ntab);
  unsigned long long* dn = (unsigned long long*)alloc(5 * 8 * ntab);
  if (!dn) e = cudaErrorMemoryAllocation;
  std::vector<unsigned long long> init(5 * ntab);
  for (int i = 0; i < ntab; ++i) {
    init[5 * i] = init[5 * i + 1] = init[5 * i + 2] = 0;
    init[5 * i + 3] = init[5 * i + 4] = ~0ull;
  }
  if (e == cudaSuccess) e = cudaMemcpyAsync(dn, init.data(), 5 * 8 * ntab, cudaMemcpyHostToDevice, st);
  bool any_large = false;
  for (int i = 0; i < ntab && e == cudaSuccess; ++i) {
    k0[i] = (Key128*)alloc(n[i] * sizeof(Key128));
    c0[i] = (unsigned long long*)alloc(n[i] * 8);
    out[i].k = (Key128*)owl_dev_alloc(n[i] * sizeof(Key128));
    out[i].c = (unsigned long long*)owl_dev_alloc(n[i] * 8);
    out[i].n = n[i];
    if (!k0[i] || !c0[i] || !out[i].k || !out[i].c) { e = cudaErrorMemoryAllocation; break; }
    compact_kernel<<<grid_for(t[i].cap, 256), 256, 0, st>>>(t[i].b, t[i].cap, k0[i], c0[i], dn + 5 * i, dn + 5 * i + 1);
    any_large |= n[i] > 4096;
  }
  std::vector<unsigned long long> masks(5 * ntab, 0);
  if (e == cudaSuccess && any_large) {
    e = cudaMemcpyAsync(masks.data(), dn, 5 * 8 * ntab, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  }
  for (int i = 0; i < ntab && e == cudaSuccess; ++i) {
    if (!n[i]) continue;
    const unsigned long long* m = &masks[5 * i + 1]; /* or_hi, or_lo, and_hi, and_lo */
    PackRuns runs;
    int nb = 0;
    if (n[i] > 4096 && pack_runs(m[0] ^ m[2], m[1] ^ m[3], &runs, &nb)) {
      /* large table: radix-sort the packed varying bits (a few passes instead of 16) and gather */
      unsigned long long* ck = (unsigned long long*)alloc(n[i] * 8);
      unsigned long long* ck2 = (unsigned long long*)alloc(n[i] * 8);
      uint32_t* ix = (uint32_t*)alloc(n[i] * 4);
      uint32_t* ix2 = (uint32_t*)alloc(n[i] * 4);
      if (!ck || !ck2 || !ix || !ix2) { e = cudaErrorMemoryAllocation; break; }
      pack_kernel<<<grid_for(n[i], 256), 256, 0, st>>>(k0[i], n[i], runs, ck, ix);
      size_t tmp = 0;
      const int eb = nb > 0 ? nb : 1;
      cub::DeviceRadixSort::SortPairs(nullptr, tmp, ck, ck2, ix, ix2, (int64_t)n[i], 0, eb, st);
      void* dt = alloc(tmp);
      if (!dt) { e = cudaErrorMemoryAllocation; break; }
      e = cub::DeviceRadixSort::SortPairs(dt, tmp, ck, ck2, ix, ix2, (int64_t)n[i], 0, eb, st);
      if (e == cudaSuccess)
        gather_sorted_kernel<<<grid_for(n[i], 256), 256, 0, st>>>(k0[i], c0[i], ix2, n[i], out[i].k, out[i].c);
    } else if (n[i] <= SMALL_SORT_MAX) {
      /* small table (the node / edge / triple tables): one CTA, bitonic in shared memory */
      e = small_sort(k0[i], c0[i], n[i], out[i].k, out[i].c, st);
    } else {
      size_t tmp = 0;
      cub::DeviceRadixSort::SortPairs(nullptr, tmp, k0[i], out[i].k, c0[i], out[i].c, (int64_t)n[i], KeyDecomp{}, st);
      void* dt = alloc(tmp);
      if (!dt) { e = cudaErrorMemoryAllocation; break; }
      e = cub::DeviceRadixSort::SortPairs(dt, tmp, k0[i], out[i].k, c0[i], out[i].c, (int64_t)n[i], KeyDecomp{}, st);
    }
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  for (void* p : scratch) owl_dev_free(p);
  if (e != cudaSuccess)
    for (int i = 0; i < ntab; ++i) owl_sorted_free(&out[i]);
  return e;
}

cudaError_t owl_table_insert_sorted(const DevTable& t, int tbl, const Key128* k, const unsigned long long* c,
                                    uint64_t n, FoldStatus* st_dev, cudaStream_t st) {
  if (!n) return cudaSuccess;
  insert_sorted_kernel<<<grid_for(n, 256), 256, 0, st>>>(t, tbl, k, c, n, st_dev);
  return cudaGetLastError();
}

namespace {

__device__ __forceinline__ bool key_lt(const Key128& a, const Key128& b) {
  return a.hi < b.hi || (a.hi == b.hi && a.lo < b.lo);
}

/* number of selected keys (k[idx[0..n)]) less than q */
__device__ uint64_t count_less(const Key128* k, const uint64_t* idx, uint64_t n, const Key128& q) {
  uint64_t lo = 0, hi = n;
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (key_lt(k[idx[mid]], q)) lo = mid + 1; else hi = mid;
  }
  return lo;
}

__global__ void diff_base_kernel(const unsigned long long* nsel, int ntab, unsigned long long* base) {
  unsigned long long b = 0;
  for (int t = 0; t < ntab; ++t) {
    base[t] = b;
    b += nsel[2 * t] + nsel[2 * t + 1];
  }
  base[ntab] = b;
}

/* the differing cells of table t as owl_diff rows, in canonical order: A-side rows (in B with another count,
   or absent from B) and B-only rows merged by key (binary search of each in the other list) */
__global__ void diff_rows_kernel(int t, const Key128* ak, const unsigned long long* ac, const unsigned long long* cboa,
                                 const uint64_t* ia, const Key128* bk, const unsigned long long* bc, const uint64_t* ib,
                                 const unsigned long long* nsel, const unsigned long long* base, owl_diff* out) {
  const uint64_t nA = nsel[2 * t], nB = nsel[2 * t + 1];
  const uint32_t NA = 0xFFFFFFFFu;
  for (uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; r < nA + nB; r += (uint64_t)gridDim.x * blockDim.x) {
    Key128 k;
    unsigned long long ca, cb;
    uint64_t pos;
    if (r < nA) {
      const uint64_t i = ia[r];
      k = ak[i];
      ca = ac[i];
      cb = cboa[i];
      pos = r + count_less(bk, ib, nB, k);
    } else {
      const uint64_t i = ib[r - nA];
      k = bk[i];
      ca = 0;
      cb = bc[i];
      pos = (r - nA) + count_less(ak, ia, nA, k);
    }
    owl_diff d;
    d.table = (uint32_t)t;
    d.bb = d.ins = d.j = d.prev = d.next = NA;
    d._pad = 0;
    d.x = 0;
    if (t == T_ADDR) {
      d.slot = (uint32_t)(k.hi >> 48);
      d.bb = (uint32_t)((k.hi >> 30) & 0x3FFFFu);
      d.ins = (uint32_t)((k.hi >> 22) & 0xFFu);
      d.j = (uint32_t)(k.hi & OWL_MAX_J);
      d.x = k.lo;
    } else {
      d.slot = (uint32_t)(k.hi >> 32);
      const uint32_t a = (uint32_t)k.hi, b = (uint32_t)(k.lo >> 32), c = (uint32_t)k.lo;
      if (t == T_NODE) d.bb = a;
      else if (t == T_EDGE) { d.prev = a; d.next = c; }
      else { d.bb = a; d.prev = b; d.next = c; }
    }
    d.count_a = ca;
    d.count_b = cb;
    out[base[t] + pos] = d;
  }
}

}  // namespace

/* A5 over all tables at once: the rows of every table in canonical (table, key) order, returned in host
   memory allocated with malloc (caller frees); two host synchronisations in all. */
cudaError_t owl_diff_rows(const SortedTable* A, const SortedTable* B, int ntab, owl_diff** rows, uint64_t* n_rows,
                          size_t extra_rows, cudaStream_t st) {
  *rows = nullptr;
  *n_rows = 0;
  std::vector<void*> scratch;
  auto alloc = [&](size_t bytes) { void* p = owl_dev_alloc(bytes); scratch.push_back(p); return p; };
  unsigned long long* nsel = (unsigned long long*)alloc(2 * ntab * 8 + 8);
  unsigned long long* base = (unsigned long long*)alloc((ntab + 1) * 8);
  cudaError_t e = (nsel && base) ? cudaSuccess : cudaErrorMemoryAllocation;
  if (e == cudaSuccess) e = cudaMemsetAsync(nsel, 0, 2 * ntab * 8, st);
  uint64_t max_rows = 0;
  std::vector<unsigned char*> fa(ntab), fb(ntab);
  std::vector<unsigned long long*> cboa(ntab);
  std::vector<uint64_t*> ia(ntab), ib(ntab);
  for (int t = 0; t < ntab && e == cudaSuccess; ++t) {
    const uint64_t na = A[t].n, nb = B[t].n;
    max_rows += na + nb;
    fa[t] = (unsigned char*)alloc(na + 1);
    fb[t] = (unsigned char*)alloc(nb + 1);
    cboa[t] = (unsigned long long*)alloc((na + 1) * 8);
    ia[t] = (uint64_t*)alloc((na + 1) * 8);
    ib[t] = (uint64_t*)alloc((nb + 1) * 8);
    if (!fa[t] || !fb[t] || !cboa[t] || !ia[t] || !ib[t]) { e = cudaErrorMemoryAllocation; break; }
    if (na || nb)
      diff_flag_kernel<<<grid_for(na > nb ? na : nb, 256), 256, 0, st>>>(A[t].k, A[t].c, na, B[t].k, B[t].c, nb, fa[t],
                                                                           cboa[t], fb[t]);
    size_t tmp = 0, tmp2 = 0;
    cub::DeviceSelect::Flagged(nullptr, tmp, thrust::counting_iterator<uint64_t>(0), fa[t], ia[t], nsel + 2 * t, (int64_t)na, st);
    cub::DeviceSelect::Flagged(nullptr, tmp2, thrust::counting_iterator<uint64_t>(0), fb[t], ib[t], nsel + 2 * t + 1, (int64_t)nb, st);
    void* dt = alloc(tmp > tmp2 ? tmp : tmp2);
    if (!dt) { e = cudaErrorMemoryAllocation; break; }
    if (na) e = cub::DeviceSelect::Flagged(dt, tmp, thrust::counting_iterator<uint64_t>(0), fa[t], ia[t], nsel + 2 * t, (int64_t)na, st);
    if (e == cudaSuccess && nb)
      e = cub::DeviceSelect::Flagged(dt, tmp2, thrust::counting_iterator<uint64_t>(0), fb[t], ib[t], nsel + 2 * t + 1, (int64_t)nb, st);
  }
  owl_diff* drows = nullptr;
  if (e == cudaSuccess) {
    drows = (owl_diff*)alloc((max_rows + 1) * sizeof(owl_diff));
    if (!drows) e = cudaErrorMemoryAllocation;
  }
  if (e == cudaSuccess) {
    diff_base_kernel<<<1, 1, 0, st>>>(nsel, ntab, base);
    for (int t = 0; t < ntab; ++t)
      if (A[t].n + B[t].n)
        diff_rows_kernel<<<grid_for(A[t].n + B[t].n, 256), 256, 0, st>>>(t, A[t].k, A[t].c, cboa[t], ia[t], B[t].k, B[t].c,
                                                                          ib[t], nsel, base, drows);
  }
  unsigned long long total = 0;
  if (e == cudaSuccess) e = cudaMemcpyAsync(&total, base + ntab, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e == cudaSuccess) {
    *rows = (owl_diff*)owl_host_alloc((total + extra_rows + 1) * sizeof(owl_diff));
    if (!*rows) e = cudaErrorMemoryAllocation;
  }
  if (e == cudaSuccess && total) e = cudaMemcpyAsync(*rows, drows, total * sizeof(owl_diff), cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  for (void* p : scratch) owl_dev_free(p);
  if (e != cudaSuccess) {
    owl_host_free(*rows);
    *rows = nullptr;
    return e;
  }
  *n_rows = total;
  return cudaSuccess;
}

namespace {

__device__ __forceinline__ unsigned long long fmix64(unsigned long long x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return x;
}

/* sums (mod 2^64) of two independent mixes of every (table, key, count): equal multisets of cells give
   equal fingerprints whatever their order */
__global__ void fingerprint_kernel(const Key128* k, const unsigned long long* c, uint64_t n, int t,
                                   unsigned long long* fp) {
  unsigned long long a = 0, b = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long h = fmix64(k[i].hi ^ ((unsigned long long)t << 62)) ^ fmix64(k[i].lo + 0x9E3779B97F4A7C15ull);
    a += fmix64(h ^ c[i]);
    b += fmix64(h + c[i] * 0xC2B2AE3D27D4EB4Full + 1);
  }
  for (int o = 16; o; o >>= 1) {
    a += __shfl_xor_sync(0xFFFFFFFFu, a, o);
    b += __shfl_xor_sync(0xFFFFFFFFu, b, o);
  }
  if ((threadIdx.x & 31) == 0) {
    atomicAdd(&fp[0], a);
    atomicAdd(&fp[1], b);
  }
}

}  // namespace

cudaError_t owl_tables_fingerprint(const SortedTable* tabs, int ntab, unsigned long long fp[2], cudaStream_t st) {
  unsigned long long* d = (unsigned long long*)owl_dev_alloc(16);
  if (!d) return cudaErrorMemoryAllocation;
  cudaError_t e = cudaMemsetAsync(d, 0, 16, st);
  for (int t = 0; t < ntab && e == cudaSuccess; ++t)
    if (tabs[t].n) fingerprint_kernel<<<grid_for(tabs[t].n, 256), 256, 0, st>>>(tabs[t].k, tabs[t].c, tabs[t].n, t, d);
  if (e == cudaSuccess) e = cudaMemcpyAsync(fp, d, 16, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  owl_dev_free(d);
  return e;
}

namespace {
/* Channel-order bucketing by bursts (N2).  A tracer's channel delivers each warp's records in runs ("bursts") of
   consecutive records of one warp.  All channel-order segments of a fold launch are bucketed together and by
   bursts, not records: one streaming pass marks burst heads (key = (segment, gwarp clamped to n_warps): out-of-
   range gwarps share one key and keep their stream order), the heads are compacted, the burst keys radix-sorted
   stably, and every burst is copied whole (coalesced) to its warp-major position in one buffer holding the
   segments back to back.  Per sorted burst the source start is kept, so a malformed record can be mapped back
   to the caller's index (owl_first_bad_record) without a per-record permutation. */
struct BucketArgs {
  const uint4* const* rec; /* per segment */
  const uint64_t* off;     /* per segment: first global record index; off[n_seg] = total */
  const uint32_t* n_warps; /* per segment */
  uint32_t n_seg;
  uint32_t warp_bits;      /* key bits of the clamped gwarp */
};

/* burst heads of all the launch's channel-order segments in one streaming pass: each warp scans a tile of 1024
   records of one segment (tile t belongs to the last segment with tile0 <= t; 32 coalesced loads of the gwarp
   words, 8 in flight per lane), keeps its heads in stream order in the tile's slot range of `slots` with their
   sort keys (segment, gwarp clamped to n_warps) in `skey`, and the count in tile_cnt; the tiles are concatenated
   afterwards (burst_gather_kernel) */
#define BT_LOG 10
__global__ void burst_head_kernel(const BucketArgs a, const uint64_t* tile0, uint64_t ntile, uint64_t* slots,
                                  unsigned long long* skey, uint32_t* tile_cnt) {
  const int lane = threadIdx.x & 31;
  const uint64_t wid = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t t = wid; t < ntile; t += nw) {
    uint32_t lo = 0, hi = a.n_seg; /* the tile's segment */
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (tile0[mid] <= t) lo = mid; else hi = mid;
    }
    const uint32_t sg = lo;
    const uint4* rec = a.rec[sg];
    const uint64_t n = a.off[sg + 1] - a.off[sg], goff = a.off[sg];
    const uint32_t n_warps = a.n_warps[sg];
    const unsigned long long kseg = (unsigned long long)sg << a.warp_bits;
    const uint64_t b = (t - tile0[sg]) << BT_LOG;
    uint32_t prev = b == 0 ? 0xFFFFFFFFu : min(__ldg(&rec[b - 1].z), n_warps);
    uint32_t cnt = 0;
    uint64_t* out = slots + (t << BT_LOG);
    unsigned long long* kout = skey + (t << BT_LOG);
    for (int it0 = 0; it0 < (1 << BT_LOG) / 32; it0 += 8) {
      uint32_t gg[8]; /* 8 loads in flight per lane */
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint64_t i = b + (it0 + u) * 32 + lane;
        gg[u] = i < n ? __ldg(&rec[i].z) : 0xFFFFFFFEu;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint64_t i = b + (it0 + u) * 32 + lane;
        const uint32_t g = i < n ? min(gg[u], n_warps) : 0xFFFFFFFEu;
        uint32_t left = __shfl_up_sync(0xFFFFFFFFu, g, 1);
        if (lane == 0) left = prev;
        const bool head = i < n && (i == 0 || g != left);
        const unsigned m = __ballot_sync(0xFFFFFFFFu, head);
        if (head) {
          const uint32_t k = cnt + __popc(m & ((1u << lane) - 1));
          out[k] = goff + i;
          kout[k] = kseg | g;
        }
        cnt += __popc(m);
        prev = __shfl_sync(0xFFFFFFFFu, g, 31);
      }
    }
    if (lane == 0) tile_cnt[t] = cnt;
  }
}

/* concatenation of the tiles' heads (tile_off = exclusive scan of tile_cnt): global burst starts in stream order,
   their sort keys, and the original burst ids (the sort's values) */
__global__ void burst_gather_kernel(const uint64_t* slots, const unsigned long long* skey, const uint32_t* tile_cnt,
                                    const uint64_t* tile_off, uint64_t ntile, uint64_t* start, unsigned long long* key,
                                    uint32_t* id) {
  const int lane = threadIdx.x & 31;
  const uint64_t wid = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t t = wid; t < ntile; t += nw) {
    const uint32_t c = tile_cnt[t];
    const uint64_t o = tile_off[t];
    for (uint32_t k = lane; k < c; k += 32) {
      start[o + k] = slots[(t << BT_LOG) + k];
      key[o + k] = skey[(t << BT_LOG) + k];
      id[o + k] = (uint32_t)(o + k);
    }
  }
}

__global__ void widen_kernel(const uint32_t* in, uint64_t n, uint64_t* out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) out[i] = in[i];
}

/* per sorted burst: its length (a segment's first record is a head: bursts never span segments), source start
   (global stream index) and source pointer */
__global__ void burst_sorted_kernel(const BucketArgs a, const uint32_t* sid, const unsigned long long* key2,
                                    const uint64_t* start, const unsigned long long* nb_p, uint64_t* slen,
                                    uint64_t* bsrc, const uint4** sptr) {
  const uint64_t nb = *nb_p, total = a.off[a.n_seg];
  for (uint64_t b = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; b < nb; b += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t i = sid[b];
    const uint64_t g = start[i];
    const uint32_t sg = (uint32_t)(key2[b] >> a.warp_bits);
    slen[b] = (i + 1 < nb ? start[i + 1] : total) - g;
    bsrc[b] = g;
    sptr[b] = a.rec[sg] + (g - a.off[sg]);
  }
}

/* sorted bursts copied to their warp-major offsets: each warp takes 4 bursts per round and issues all their
   loads before the stores (memory-level parallelism); lane k of a burst copies its records k, k + 32, ... */
__global__ void burst_copy_kernel(const uint4* const* sptr, const uint64_t* slen, const uint64_t* bdst,
                                  const unsigned long long* nb_p, uint4* out) {
  const uint64_t nb = *nb_p;
  const int lane = threadIdx.x & 31;
  const uint64_t wid = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t b0 = wid * 4; b0 < nb; b0 += nw * 4) {
    const uint4* src[4];
    uint64_t l[4], d[4];
    uint4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint64_t b = b0 + u;
      l[u] = b < nb ? slen[b] : 0;
      d[u] = b < nb ? bdst[b] : 0;
      src[u] = b < nb ? sptr[b] : nullptr;
      if (lane < l[u]) v[u] = src[u][lane];
    }
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (lane < l[u]) out[d[u] + lane] = v[u];
#pragma unroll
    for (int u = 0; u < 4; ++u)
      for (uint64_t k = lane + 32; k < l[u]; k += 32) out[d[u] + k] = src[u][k]; /* bursts longer than 32 */
  }
}

/* Error report of a bucketed segment: every malformed record, by the rules of the warp walk (SURVEY §8(b)
   conventions; the fold's slow path), mapped back to the caller's index through its burst; the minimum wins.  One
   thread per traced warp (start detected on the gwarp change), walking it in order; records with gwarp >=
   n_warps are checked one by one.  Only launched after a fold reported an error in such a segment. */
__device__ __forceinline__ uint64_t caller_index(uint64_t d, const uint64_t* bsrc, const uint64_t* bdst, uint64_t nb,
                                                 uint64_t seg_off) {
  uint64_t lo = 0, hi = nb; /* last burst with bdst <= d */
  while (hi - lo > 1) {
    const uint64_t mid = (lo + hi) >> 1;
    if (bdst[mid] <= d) lo = mid; else hi = mid;
  }
  return bsrc[lo] + (d - bdst[lo]) - seg_off;
}

/* rec: the warp-major copy (copy mode), or nullptr with caller = the segment's own array (in-place mode: the
   record at warp-major index i is read through its burst) */
__global__ void first_bad_kernel(const uint4* rec, const uint4* caller, uint64_t n, uint32_t n_warps,
                                 const uint64_t* bsrc, const uint64_t* bdst, uint64_t nb, uint64_t seg_off,
                                 unsigned long long* out) {
  auto at = [&](uint64_t i) -> uint4 {
    return rec ? rec[i] : caller[caller_index(seg_off + i, bsrc, bdst, nb, seg_off)];
  };
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t g = at(i).z;
    if (g >= n_warps) {
      atomicMin(out, ((unsigned long long)caller_index(seg_off + i, bsrc, bdst, nb, seg_off) << 3) | KERR_GWARP);
      continue;
    }
    if (i > 0 && at(i - 1).z == g) continue;
    uint32_t cur = OWL_NONE_BB;
    for (uint64_t k = i; k < n; ++k) {
      const uint4 r = at(k);
      if (r.z != g) break;
      const uint32_t bb = (r.w >> 8) & 0x3FFFFu;
      uint32_t code = KERR_NONE;
      if ((r.w >> 31) == 0) {
        if (r.x != 0 || r.y != 0 || (r.w & 0x7C0000FFu) != 0) code = KERR_BBFIELDS;
        else cur = bb;
      } else if ((r.y >> 28) > 8) code = KERR_MTYPE;
      else if (cur == OWL_NONE_BB) code = KERR_NOBB;
      else if (bb != cur) code = KERR_BBMISMATCH;
      if (code) atomicMin(out, ((unsigned long long)caller_index(seg_off + k, bsrc, bdst, nb, seg_off) << 3) | code);
    }
  }
}

/* in-place burst index (N2): per sorted burst its segment-relative virtual start, physical start and clamped gwarp */
__global__ void burst_inplace_kernel(const unsigned long long* key2, const uint64_t* bsrc, const uint64_t* bdst,
                                     const uint64_t* off, uint32_t warp_bits, const unsigned long long* nb_p,
                                     uint32_t* bvs, uint32_t* bpo, uint32_t* bk) {
  const uint64_t nb = *nb_p;
  for (uint64_t b = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; b < nb; b += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = key2[b];
    const uint64_t so = off[k >> warp_bits];
    bvs[b] = (uint32_t)(bdst[b] - so);
    bpo[b] = (uint32_t)(bsrc[b] - so);
    bk[b] = (uint32_t)(k & ((1ull << warp_bits) - 1));
  }
}

/* first sorted burst of every segment: lower bound of (s << warp_bits) in the sorted keys; first[ns] = nb */
__global__ void seg_first_kernel(const unsigned long long* key2, const unsigned long long* nb_p, uint32_t ns,
                                 uint32_t warp_bits, uint64_t* first) {
  const uint64_t nb = *nb_p;
  for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s <= ns; s += gridDim.x * blockDim.x) {
    const unsigned long long want = (unsigned long long)s << warp_bits;
    uint64_t lo = 0, hi = nb;
    while (lo < hi) {
      const uint64_t mid = (lo + hi) >> 1;
      if (key2[mid] < want) lo = mid + 1; else hi = mid;
    }
    first[s] = s == ns ? nb : lo;
  }
}
}  // namespace

void owl_bucketed_free(BucketedSet* b) {
  owl_dev_free(b->out);
  owl_dev_free(b->bsrc);
  owl_dev_free(b->bdst);
  owl_dev_free(b->bvs);
  owl_dev_free(b->bpo);
  owl_dev_free(b->bk);
  *b = BucketedSet{};
}

cudaError_t owl_bucket_segments(const std::vector<const uint4*>& rec, const std::vector<uint64_t>& n,
                                const std::vector<uint32_t>& n_warps, BucketedSet* out, cudaStream_t st, bool copy) {
  *out = BucketedSet{};
  out->rec = rec;
  const uint32_t ns = (uint32_t)rec.size();
  std::vector<uint64_t> off(ns + 1, 0);
  uint32_t maxw = 1;
  for (uint32_t i = 0; i < ns; ++i) {
    off[i + 1] = off[i] + n[i];
    maxw = std::max(maxw, n_warps[i]);
  }
  const uint64_t total = off[ns];
  out->off = off;
  if (!total) return cudaSuccess;
  std::vector<void*> scratch;
  auto alloc = [&](size_t bytes) { void* p = owl_dev_alloc(bytes); scratch.push_back(p); return p; };
  uint32_t warp_bits = 1;
  while (warp_bits < 32 && (1ull << warp_bits) <= (uint64_t)maxw) ++warp_bits; /* keys 0..n_warps */
  int seg_bits = 1;
  while (seg_bits < 32 && (1ull << seg_bits) < (uint64_t)ns) ++seg_bits;
  std::vector<uint64_t> tile0(ns + 1, 0);
  for (uint32_t i = 0; i < ns; ++i) tile0[i + 1] = tile0[i] + ((n[i] + (1u << BT_LOG) - 1) >> BT_LOG);
  const uint64_t ntile = tile0[ns];
  uint64_t* slots = (uint64_t*)alloc((ntile << BT_LOG) * 8); /* worst case: every record starts a burst */
  unsigned long long* skey = (unsigned long long*)alloc((ntile << BT_LOG) * 8);
  uint64_t* dtile0 = (uint64_t*)alloc((ns + 1) * 8);
  uint32_t* tile_cnt = (uint32_t*)alloc(ntile * 4 + 4);
  uint64_t* tile_cnt64 = (uint64_t*)alloc(ntile * 8 + 8);
  uint64_t* tile_off = (uint64_t*)alloc(ntile * 8 + 8);
  const uint4** drec = (const uint4**)alloc(ns * sizeof(void*));
  uint64_t* doff = (uint64_t*)alloc((ns + 1) * 8);
  uint32_t* dnw = (uint32_t*)alloc(ns * 4);
  unsigned long long* nb_d = (unsigned long long*)alloc(8);
  cudaError_t e = (slots && skey && dtile0 && tile_cnt && tile_cnt64 && tile_off && drec && doff && dnw && nb_d)
                      ? cudaSuccess : cudaErrorMemoryAllocation;
  if (e == cudaSuccess) e = cudaMemcpyAsync(drec, rec.data(), ns * sizeof(void*), cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync(doff, off.data(), (ns + 1) * 8, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync(dnw, n_warps.data(), ns * 4, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) e = cudaMemcpyAsync(dtile0, tile0.data(), (ns + 1) * 8, cudaMemcpyHostToDevice, st);
  BucketArgs a{drec, doff, dnw, ns, warp_bits};
  if (e == cudaSuccess && ntile)
    burst_head_kernel<<<grid_for(ntile * 32, 256), 256, 0, st>>>(a, dtile0, ntile, slots, skey, tile_cnt);
  if (e == cudaSuccess) {
    widen_kernel<<<grid_for(ntile, 256), 256, 0, st>>>(tile_cnt, ntile, tile_cnt64);
    size_t tmp = 0;
    cub::DeviceScan::InclusiveSum(nullptr, tmp, tile_cnt64, tile_off + 1, (int64_t)ntile, st);
    void* dt = alloc(tmp);
    if (!dt) e = cudaErrorMemoryAllocation;
    else {
      e = cudaMemsetAsync(tile_off, 0, 8, st);
      if (e == cudaSuccess) e = cub::DeviceScan::InclusiveSum(dt, tmp, tile_cnt64, tile_off + 1, (int64_t)ntile, st);
    }
  }
  if (e == cudaSuccess) e = cudaMemcpyAsync(nb_d, tile_off + ntile, 8, cudaMemcpyDeviceToDevice, st);
  unsigned long long nb = 0;
  if (e == cudaSuccess) e = cudaMemcpyAsync(&nb, nb_d, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e == cudaSuccess) {
    uint64_t* start = (uint64_t*)alloc(nb * 8 + 8);
    unsigned long long* key = (unsigned long long*)alloc(nb * 8);
    unsigned long long* key2 = (unsigned long long*)alloc(nb * 8);
    uint32_t* id = (uint32_t*)alloc(nb * 4);
    uint32_t* sid = (uint32_t*)alloc(nb * 4);
    uint64_t* slen = (uint64_t*)alloc(nb * 8);
    const uint4** sptr = (const uint4**)alloc(nb * sizeof(void*));
    out->bsrc = (uint64_t*)owl_dev_alloc(nb * 8);
    out->bdst = (uint64_t*)owl_dev_alloc(nb * 8);
    if (copy) {
      out->out = (uint4*)owl_dev_alloc(total * 16);
    } else {
      out->bvs = (uint32_t*)owl_dev_alloc(nb * 4 + 4);
      out->bpo = (uint32_t*)owl_dev_alloc(nb * 4 + 4);
      out->bk = (uint32_t*)owl_dev_alloc(nb * 4 + 4);
    }
    out->nb = nb;
    if (!start || !key || !key2 || !id || !sid || !slen || !sptr || !out->bsrc || !out->bdst ||
        (copy ? !out->out : (!out->bvs || !out->bpo || !out->bk)))
      e = cudaErrorMemoryAllocation;
    if (e == cudaSuccess) {
      burst_gather_kernel<<<grid_for(ntile * 32, 256), 256, 0, st>>>(slots, skey, tile_cnt, tile_off, ntile, start,
                                                                    key, id);
      size_t tmp = 0;
      const int bits = (int)warp_bits + seg_bits;
      cub::DeviceRadixSort::SortPairs(nullptr, tmp, key, key2, id, sid, (int64_t)nb, 0, bits, st);
      void* dt = alloc(tmp);
      if (!dt) e = cudaErrorMemoryAllocation;
      else e = cub::DeviceRadixSort::SortPairs(dt, tmp, key, key2, id, sid, (int64_t)nb, 0, bits, st);
    }
    if (e == cudaSuccess) {
      burst_sorted_kernel<<<grid_for(nb, 256), 256, 0, st>>>(a, sid, key2, start, nb_d, slen, out->bsrc, sptr);
      size_t tmp = 0;
      cub::DeviceScan::ExclusiveSum(nullptr, tmp, slen, out->bdst, (int64_t)nb, st);
      void* dt = alloc(tmp);
      if (!dt) e = cudaErrorMemoryAllocation;
      else e = cub::DeviceScan::ExclusiveSum(dt, tmp, slen, out->bdst, (int64_t)nb, st);
    }
    if (e == cudaSuccess && copy)
      burst_copy_kernel<<<grid_for((nb + 3) / 4 * 32, 256), 256, 0, st>>>(sptr, slen, out->bdst, nb_d, out->out);
    if (e == cudaSuccess && !copy) {
      burst_inplace_kernel<<<grid_for(nb, 256), 256, 0, st>>>(key2, out->bsrc, out->bdst, doff, warp_bits, nb_d,
                                                              out->bvs, out->bpo, out->bk);
      uint64_t* dfirst = (uint64_t*)alloc((ns + 1) * 8);
      if (!dfirst) e = cudaErrorMemoryAllocation;
      else {
        seg_first_kernel<<<grid_for(ns + 1, 128), 128, 0, st>>>(key2, nb_d, ns, warp_bits, dfirst);
        out->bfirst.assign(ns + 1, 0);
        e = cudaMemcpyAsync(out->bfirst.data(), dfirst, (ns + 1) * 8, cudaMemcpyDeviceToHost, st);
      }
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(st); /* the scratch (drec, slen) is freed below */
  }
  for (void* p : scratch) owl_dev_free(p);
  if (e != cudaSuccess) owl_bucketed_free(out);
  return e == cudaSuccess ? cudaGetLastError() : e;
}

cudaError_t owl_first_bad_record(const BucketedSet& b, uint32_t seg, uint32_t n_warps, unsigned long long* idx_code,
                                 cudaStream_t st) {
  unsigned long long* d = (unsigned long long*)owl_dev_alloc(8);
  if (!d) return cudaErrorMemoryAllocation;
  const uint64_t n = b.off[seg + 1] - b.off[seg];
  cudaError_t e = cudaMemsetAsync(d, 0xFF, 8, st);
  if (e == cudaSuccess && n)
    first_bad_kernel<<<grid_for(n, 256), 256, 0, st>>>(b.out ? b.out + b.off[seg] : nullptr, b.rec[seg], n, n_warps,
                                                       b.bsrc, b.bdst, b.nb, b.off[seg], d);
  if (e == cudaSuccess) e = cudaMemcpyAsync(idx_code, d, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  owl_dev_free(d);
  return e;
}
