// microbench.cu — B200 measurements that decide the fold design: streaming read bandwidth,
// L2-resident RED.ADD.64 and load+RED throughput, shared-memory atomics, MATCH.ANY.U64 issue cost.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o microbench microbench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ uint64_t mix(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33; return x;
}

__global__ void stream_read(const uint4* __restrict__ p, uint64_t n, unsigned* out) {
  unsigned acc = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p + i));
    acc ^= v.x ^ v.w;
  }
  if (acc == 0x12345678) out[0] = acc;
}

// each thread: `iters` random RED.ADD.64 into a table of `cells` 32-byte cells
__global__ void red_random(unsigned long long* cells, uint64_t mask, int iters, uint64_t seed) {
  uint64_t s = seed ^ (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x);
  for (int i = 0; i < iters; ++i) {
    s = mix(s + i);
    atomicAdd(&cells[(s & mask) * 4 + 2], 1ull);
  }
}

// load the 16-byte key of a random cell, compare, then RED the count (the g_insert hit path)
__global__ void load_red_random(unsigned long long* cells, uint64_t mask, int iters, uint64_t seed, unsigned* out) {
  uint64_t s = seed ^ (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x);
  unsigned miss = 0;
  for (int i = 0; i < iters; ++i) {
    s = mix(s + i);
    uint64_t h = s & mask;
    ulonglong2 k;
    asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(k.x), "=l"(k.y) : "l"(cells + h * 4) : "memory");
    if (k.x == h) atomicAdd(&cells[h * 4 + 2], 1ull); else ++miss;
  }
  if (miss == 12345) out[0] = miss;
}

// same with 4 independent probes in flight per thread
__global__ void load_red_random4(unsigned long long* cells, uint64_t mask, int iters, uint64_t seed, unsigned* out) {
  uint64_t s = seed ^ (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x);
  unsigned miss = 0;
  for (int i = 0; i < iters; i += 4) {
    uint64_t h[4]; ulonglong2 k[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) { s = mix(s + i + u); h[u] = s & mask; }
#pragma unroll
    for (int u = 0; u < 4; ++u)
      asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(k[u].x), "=l"(k[u].y) : "l"(cells + h[u] * 4) : "memory");
#pragma unroll
    for (int u = 0; u < 4; ++u) { if (k[u].x == h[u]) atomicAdd(&cells[h[u] * 4 + 2], 1ull); else ++miss; }
  }
  if (miss == 12345) out[0] = miss;
}

__global__ void smem_atomic(int iters, unsigned* out, int cells_log2) {
  extern __shared__ unsigned sm[];
  const unsigned mask = (1u << cells_log2) - 1;
  for (unsigned i = threadIdx.x; i <= mask; i += blockDim.x) sm[i] = 0;
  __syncthreads();
  uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  for (int i = 0; i < iters; ++i) { s = mix(s + i); atomicAdd(&sm[s & mask], 1u); }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = sm[0];
}

// non-atomic shared RMW (ld + st) at random distinct-ish addresses
__global__ void smem_rmw(int iters, unsigned* out, int cells_log2) {
  extern __shared__ unsigned sm[];
  const unsigned mask = (1u << cells_log2) - 1;
  for (unsigned i = threadIdx.x; i <= mask; i += blockDim.x) sm[i] = 0;
  __syncthreads();
  uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  for (int i = 0; i < iters; ++i) { s = mix(s + i); volatile unsigned* p = &sm[s & mask]; *p = *p + 1; }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = sm[0];
}

__global__ void match_cost(int iters, unsigned* out) {
  uint64_t v = (threadIdx.x & 7) * 0x1234567890ull;
  unsigned acc = 0;
  for (int i = 0; i < iters; ++i) { acc += __match_any_sync(0xFFFFFFFFu, v); v += acc & 1; }
  if (acc == 7) out[0] = acc;
}
__global__ void match32_cost(int iters, unsigned* out) {
  unsigned v = (threadIdx.x & 7) * 0x12345u;
  unsigned acc = 0;
  for (int i = 0; i < iters; ++i) { acc += __match_any_sync(0xFFFFFFFFu, v); v += acc & 1; }
  if (acc == 7) out[0] = acc;
}

int main() {
  int sms = 148;
  cudaDeviceProp pr; cudaGetDeviceProperties(&pr, 0); sms = pr.multiProcessorCount;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float ms;
  unsigned* out; CK(cudaMalloc(&out, 1 << 20));
  // 1. stream read 16 GB
  uint64_t n = (16ull << 30) / 16;
  uint4* buf; CK(cudaMalloc(&buf, n * 16)); CK(cudaMemset(buf, 1, n * 16));
  for (int blocks_per_sm : {4, 8, 16}) {
    stream_read<<<sms * blocks_per_sm, 256>>>(buf, n, out);
    cudaEventRecord(a); stream_read<<<sms * blocks_per_sm, 256>>>(buf, n, out); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    printf("stream_read bps=%d: %.1f GB/s\n", blocks_per_sm, n * 16 / ms / 1e6);
  }
  CK(cudaFree(buf));
  // 2. RED into tables of various sizes
  unsigned long long* cells; CK(cudaMalloc(&cells, (1ull << 26) * 32)); CK(cudaMemset(cells, 0, (1ull << 26) * 32));
  const int iters = 256;
  for (int lg : {12, 16, 20, 22, 26}) {
    uint64_t mask = (1ull << lg) - 1;
    red_random<<<sms * 8, 256>>>(cells, mask, iters, 1);
    cudaEventRecord(a); red_random<<<sms * 8, 256>>>(cells, mask, iters, 2); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    double ops = (double)sms * 8 * 256 * iters;
    printf("RED.64 random cells=2^%d (%.1f MB): %.3g ops/s\n", lg, (1ull << lg) * 32 / 1e6, ops / ms * 1e3);
    load_red_random<<<sms * 8, 256>>>(cells, mask, iters, 1, out);
    cudaEventRecord(a); load_red_random<<<sms * 8, 256>>>(cells, mask, iters, 3, out); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    printf("  load16+RED (MLP 1/thread): %.3g ops/s\n", ops / ms * 1e3);
    load_red_random4<<<sms * 8, 256>>>(cells, mask, iters, 1, out);
    cudaEventRecord(a); load_red_random4<<<sms * 8, 256>>>(cells, mask, iters, 4, out); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    printf("  load16+RED (MLP 4/thread): %.3g ops/s\n", ops / ms * 1e3);
  }
  // 3. shared-memory atomics / RMW
  for (int lg : {10, 14}) {
    cudaFuncSetAttribute(smem_atomic, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
    cudaFuncSetAttribute(smem_rmw, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
    smem_atomic<<<sms * 4, 256, 4 << lg>>>(1024, out, lg);
    cudaEventRecord(a); smem_atomic<<<sms * 4, 256, 4 << lg>>>(1024, out, lg); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    double ops = (double)sms * 4 * 256 * 1024;
    printf("ATOMS.ADD random cells=2^%d: %.3g ops/s (%.2f per SM-cycle @1.9GHz)\n", lg, ops / ms * 1e3, ops / ms * 1e3 / sms / 1.9e9);
    smem_rmw<<<sms * 4, 256, 4 << lg>>>(1024, out, lg);
    cudaEventRecord(a); smem_rmw<<<sms * 4, 256, 4 << lg>>>(1024, out, lg); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    printf("LDS+STS random cells=2^%d: %.3g ops/s (%.2f per SM-cycle)\n", lg, ops / ms * 1e3, ops / ms * 1e3 / sms / 1.9e9);
  }
  // 4. match_any
  match_cost<<<sms * 8, 256>>>(4096, out);
  cudaEventRecord(a); match_cost<<<sms * 8, 256>>>(4096, out); cudaEventRecord(b); cudaEventSynchronize(b);
  cudaEventElapsedTime(&ms, a, b);
  double wi = (double)sms * 8 * 8 * 4096;
  printf("MATCH.ANY.U64: %.3g warp-instr/s = %.2f per SM-cycle\n", wi / ms * 1e3, wi / ms * 1e3 / sms / 1.9e9);
  match32_cost<<<sms * 8, 256>>>(4096, out);
  cudaEventRecord(a); match32_cost<<<sms * 8, 256>>>(4096, out); cudaEventRecord(b); cudaEventSynchronize(b);
  cudaEventElapsedTime(&ms, a, b);
  printf("MATCH.ANY.U32: %.3g warp-instr/s = %.2f per SM-cycle\n", wi / ms * 1e3, wi / ms * 1e3 / sms / 1.9e9);
  return 0;
}
