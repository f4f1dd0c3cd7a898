/*
 * owl_exchange.cu — the one data exchange of the multi-GPU path: every cell of
 * a rank's partial evidence goes to owner(attr) = mix64(attr) mod world, attr = bb for node, edge-by-src and
 * triple cells and (bb, ins, j) for address cells (the slot is left out: fix and rnd slots of one aligned
 * pair may differ), so all cells of one KS attribute (a node's H_cf, an instruction-visit's H_addr) of
 * both evidences meet on one rank.  The payload is exchanged by the caller
 * with torch.distributed all_to_all_single (NCCL over NVLink); the owner sums it into its tables (integer
 * sums: bit-identical to one GPU).
 */
#include <cuda_runtime.h>

#include "owl_device.cuh"
#include "owl_internal.h"

using namespace owl_dev;

namespace {

/* owner of a cell: a hash of its attribute WITHOUT the slot field.  The two evidences number their slots
   independently and the KS pairs fix slot s with rnd slot f2r[s] (owl_ks.cu), so both sides of one attribute
   must meet on one rank whatever their slot ids: (bb) for node / edge-by-src / triple cells, (bb, ins, j)
   for address cells (owl_internal.h key layout). */
__device__ __forceinline__ uint32_t owner_of(unsigned long long hi, int tbl, int world) {
  unsigned long long x = tbl == T_ADDR ? (hi & ((1ull << 48) - 1)) : (hi & 0xFFFFFFFFull);
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return (uint32_t)(x % (unsigned long long)world);
}

__global__ void count_owner_kernel(const Key128* k, uint64_t n, int tbl, int world, unsigned long long* counts) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    atomicAdd(&counts[owner_of(k[i].hi, tbl, world)], 1ull);
}

__global__ void scatter_owner_kernel(const Key128* k, const unsigned long long* c, uint64_t n, int tbl, int world,
                                     const unsigned long long* offs, unsigned long long* cursor, ExchangeCell* out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t o = owner_of(k[i].hi, tbl, world);
    const unsigned long long pos = offs[o] + atomicAdd(&cursor[o], 1ull);
    ExchangeCell e;
    e.hi = k[i].hi;
    e.lo = k[i].lo;
    e.count = c[i];
    e.tbl = (uint32_t)tbl;
    e._pad = 0;
    out[pos] = e;
  }
}

/* the same two passes straight over a hash table's buckets (no canonical sort first): empty cells skipped */
__global__ void count_owner_table_kernel(const owl_bucket* b, uint64_t cap, int tbl, int world,
                                         unsigned long long* counts) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < cap; i += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long hi = b[i >> 1].key[i & 1][0];
    if (hi != OWL_EMPTY_KEY) atomicAdd(&counts[owner_of(hi, tbl, world)], 1ull);
  }
}

__global__ void scatter_owner_table_kernel(const owl_bucket* b, uint64_t cap, int tbl, int world,
                                           const unsigned long long* offs, unsigned long long* cursor,
                                           ExchangeCell* out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < cap; i += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long hi = b[i >> 1].key[i & 1][0];
    if (hi == OWL_EMPTY_KEY) continue;
    const uint32_t o = owner_of(hi, tbl, world);
    const unsigned long long pos = offs[o] + atomicAdd(&cursor[o], 1ull);
    ExchangeCell e;
    e.hi = hi;
    e.lo = b[i >> 1].key[i & 1][1];
    e.count = b[i >> 1].count[i & 1];
    e.tbl = (uint32_t)tbl;
    e._pad = 0;
    out[pos] = e;
  }
}

__global__ void absorb_kernel(DevTable t0, DevTable t1, DevTable t2, DevTable t3, const ExchangeCell* cells, uint64_t n,
                              FoldStatus* st) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const ExchangeCell e = cells[i];
    const DevTable& t = e.tbl == 0 ? t0 : e.tbl == 1 ? t1 : e.tbl == 2 ? t2 : t3;
    g_insert(t, (int)e.tbl, e.hi, e.lo, e.count, st);
  }
}

int grid_for(uint64_t n, int block) {
  uint64_t g = (n + block - 1) / block;
  if (g > 148ull * 16) g = 148ull * 16;
  return g ? (int)g : 1;
}

}  // namespace

cudaError_t owl_partition_cells(const SortedTable* tabs, int world, ExchangeCell** d_send, uint64_t* counts,
                                cudaStream_t st) {
  unsigned long long *dcnt = nullptr, *doff = nullptr, *dcur = nullptr;
  uint64_t total = 0;
  for (int t = 0; t < T_NUM; ++t) total += tabs[t].n;
  dcnt = (unsigned long long*)owl_dev_alloc(world * 8);
  doff = (unsigned long long*)owl_dev_alloc(world * 8);
  dcur = (unsigned long long*)owl_dev_alloc(world * 8);
  *d_send = (ExchangeCell*)owl_dev_alloc((total + 1) * sizeof(ExchangeCell));
  if (!dcnt || !doff || !dcur || !*d_send) {
    owl_dev_free(dcnt); owl_dev_free(doff); owl_dev_free(dcur); owl_dev_free(*d_send);
    return cudaErrorMemoryAllocation;
  }
  cudaMemsetAsync(dcnt, 0, world * 8, st);
  cudaMemsetAsync(dcur, 0, world * 8, st);
  for (int t = 0; t < T_NUM; ++t)
    if (tabs[t].n) count_owner_kernel<<<grid_for(tabs[t].n, 256), 256, 0, st>>>(tabs[t].k, tabs[t].n, t, world, dcnt);
  std::vector<unsigned long long> h(world), off(world);
  cudaError_t e = cudaMemcpyAsync(h.data(), dcnt, world * 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  unsigned long long acc = 0;
  for (int w = 0; w < world; ++w) { off[w] = acc; acc += h[w]; counts[w] = h[w]; }
  if (e == cudaSuccess) e = cudaMemcpyAsync(doff, off.data(), world * 8, cudaMemcpyHostToDevice, st);
  for (int t = 0; t < T_NUM && e == cudaSuccess; ++t)
    if (tabs[t].n)
      scatter_owner_kernel<<<grid_for(tabs[t].n, 256), 256, 0, st>>>(tabs[t].k, tabs[t].c, tabs[t].n, t, world, doff,
                                                                     dcur, *d_send);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  owl_dev_free(dcnt); owl_dev_free(doff); owl_dev_free(dcur);
  return e == cudaSuccess ? cudaGetLastError() : e;
}

cudaError_t owl_partition_tables(const DevTable* tabs, int world, ExchangeCell** d_send, uint64_t* counts,
                                 cudaStream_t st) {
  unsigned long long *dcnt = nullptr, *doff = nullptr, *dcur = nullptr;
  std::vector<unsigned long long> fill(T_NUM, 0);
  cudaError_t e = cudaSuccess;
  for (int t = 0; t < T_NUM && e == cudaSuccess; ++t)
    if (tabs[t].b) e = cudaMemcpyAsync(&fill[t], tabs[t].fill, 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return e;
  uint64_t total = 0;
  for (int t = 0; t < T_NUM; ++t) total += fill[t];
  dcnt = (unsigned long long*)owl_dev_alloc(world * 8);
  doff = (unsigned long long*)owl_dev_alloc(world * 8);
  dcur = (unsigned long long*)owl_dev_alloc(world * 8);
  *d_send = (ExchangeCell*)owl_dev_alloc((total + 1) * sizeof(ExchangeCell));
  if (!dcnt || !doff || !dcur || !*d_send) {
    owl_dev_free(dcnt); owl_dev_free(doff); owl_dev_free(dcur); owl_dev_free(*d_send);
    return cudaErrorMemoryAllocation;
  }
  cudaMemsetAsync(dcnt, 0, world * 8, st);
  cudaMemsetAsync(dcur, 0, world * 8, st);
  for (int t = 0; t < T_NUM; ++t)
    if (tabs[t].b && fill[t])
      count_owner_table_kernel<<<grid_for(tabs[t].cap, 256), 256, 0, st>>>(tabs[t].b, tabs[t].cap, t, world, dcnt);
  std::vector<unsigned long long> h(world), off(world);
  e = cudaMemcpyAsync(h.data(), dcnt, world * 8, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  unsigned long long acc = 0;
  for (int w = 0; w < world; ++w) { off[w] = acc; acc += h[w]; counts[w] = h[w]; }
  if (e == cudaSuccess) e = cudaMemcpyAsync(doff, off.data(), world * 8, cudaMemcpyHostToDevice, st);
  for (int t = 0; t < T_NUM && e == cudaSuccess; ++t)
    if (tabs[t].b && fill[t])
      scatter_owner_table_kernel<<<grid_for(tabs[t].cap, 256), 256, 0, st>>>(tabs[t].b, tabs[t].cap, t, world, doff,
                                                                             dcur, *d_send);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  owl_dev_free(dcnt); owl_dev_free(doff); owl_dev_free(dcur);
  return e == cudaSuccess ? cudaGetLastError() : e;
}

cudaError_t owl_absorb_cells(const DevTable* tabs, const ExchangeCell* cells, uint64_t n, FoldStatus* st_dev,
                             cudaStream_t st) {
  if (!n) return cudaSuccess;
  absorb_kernel<<<grid_for(n, 256), 256, 0, st>>>(tabs[0], tabs[1], tabs[2], tabs[3], cells, n, st_dev);
  return cudaGetLastError();
}
