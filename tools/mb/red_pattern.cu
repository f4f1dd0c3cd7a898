// RED.64 throughput for fold-like address patterns (B200).  nvcc -gencode arch=compute_100a,code=sm_100a -O3
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s\n", cudaGetErrorString(e)); return 1; } } while (0)
__device__ __forceinline__ uint64_t mix(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33; return x;
}
__device__ __forceinline__ uint32_t cell_of(uint32_t attr, uint32_t x, uint32_t shift) {
  return ((x * 0x9E3779B1u) ^ (attr * 0xC2B2AE3Du)) >> shift;
}
// mode 0: 32 lanes pick random bytes of one attribute (duplicates ~2 pairs/instr)
// mode 1: lane-distinct bytes (lane + 32*k) of one attribute
// mode 2: random cells over the whole hot set (attr random per lane)
// mode 3: random cells over the whole table
__global__ void red_pat(unsigned long long* cells, uint32_t shift, uint32_t n_attr, int iters, int mode, uint64_t seed) {
  const int lane = threadIdx.x & 31;
  uint64_t s = seed ^ mix(blockIdx.x * (uint64_t)blockDim.x + threadIdx.x);
  const uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  for (int i = 0; i < iters; ++i) {
    s = mix(s + i);
    uint32_t attr = (w * 7 + i) % n_attr, x = 0, c;
    if (mode == 0) x = (uint32_t)s & 255u;
    else if (mode == 1) x = (lane + 32u * (uint32_t)(i & 7)) & 255u;
    else if (mode == 2) { attr = (uint32_t)(s >> 40) % n_attr; x = (uint32_t)s & 255u; }
    if (mode == 3) c = (uint32_t)(s >> 8) >> shift; else c = cell_of(attr, 4u * x, shift);
    atomicAdd(&cells[(uint64_t)c * 4 + 2], 1ull);
  }
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b); float ms;
  unsigned long long* cells; CK(cudaMalloc(&cells, (1ull << 24) * 32)); CK(cudaMemset(cells, 0, (1ull << 24) * 32));
  const int iters = 512;
  for (int lg : {16, 20, 24}) for (int mode = 0; mode < 4; ++mode) for (int bpsm : {4, 8}) {
    const uint32_t shift = 32 - lg;
    red_pat<<<sms * bpsm, 256>>>(cells, shift, 160, iters, mode, 1);
    cudaEventRecord(a); red_pat<<<sms * bpsm, 256>>>(cells, shift, 160, iters, mode, 2); cudaEventRecord(b);
    CK(cudaEventSynchronize(b)); cudaEventElapsedTime(&ms, a, b);
    double ops = (double)sms * bpsm * 256 * iters;
    printf("table 2^%d mode %d blocks/SM %d: %.3g RED/s\n", lg, mode, bpsm, ops / ms * 1e3);
  }
  return 0;
}
