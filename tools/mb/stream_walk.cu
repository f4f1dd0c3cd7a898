// stream_walk.cu — which record-staging scheme lets a per-warp sequential walk (the fold's access pattern:
// one warp walks one 2^15-record tile, 32 records = 512 B per step) stream at HBM rate on B200, and how much
// per-chunk ALU work it tolerates.  Schemes:
//   0  LDG: U chunks of 32 records per step loaded into registers, consumed at once
//   1  LDG pipelined: the next step's U chunks are loaded before the current ones are consumed
//   2  cp.async ring: per-warp ring of D blocks x 512 B, one commit group per block
//   3  TMA bulk ring: per-warp ring of D blocks x B bytes (cp.async.bulk + mbarrier complete_tx)
// each optionally with cp.async.bulk.prefetch.L2 of 4 KB granules PF granules ahead.  Per chunk: a checksum
// plus W dependent ALU instructions (the fold's per-chunk work).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o stream_walk stream_walk.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)
#define FULL 0xFFFFFFFFu

struct Args {
  const uint4* rec;
  uint64_t n;       // records
  uint32_t tile_shift;
  unsigned long long* counter;
  unsigned* out;
  int W, PF, D, B;  // work, prefetch granules, ring depth, TMA block bytes
};

__device__ __forceinline__ void pf(const void* p, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}
__device__ __forceinline__ uint4 ldg(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint32_t work(uint4 r, uint32_t acc, int W) {
  uint32_t x = r.x ^ r.y ^ r.z ^ r.w;
  for (int i = 0; i < W; ++i) x = x * 0x9E3779B1u + (x >> 7);
  return acc + x;
}
__device__ __forceinline__ void prefetch_step(const uint4* p, const uint4* end, int PF, int lane) {
  // when p crosses a 4 KB granule, prefetch granule +PF
  if (PF && lane == 0) {
    const char* q = (const char*)((((uintptr_t)p >> 12) + PF) << 12);
    if (q < (const char*)end) pf(q, 4096);
  }
}

template <int U>
__global__ void k_ldg(Args a) {
  const int lane = threadIdx.x & 31;
  uint32_t acc = 0;
  for (;;) {
    unsigned long long item = 0;
    if (lane == 0) item = atomicAdd(a.counter, 1ull);
    item = __shfl_sync(FULL, item, 0);
    const uint64_t b = item << a.tile_shift;
    if (b >= a.n) break;
    const uint4* p = a.rec + b;
    const uint4* end = a.rec + (b + (1ull << a.tile_shift) < a.n ? b + (1ull << a.tile_shift) : a.n);
    if (a.PF && lane < a.PF) { const char* q = (const char*)((((uintptr_t)p >> 12) + lane) << 12); if (q < (const char*)end) pf(q, 4096); }
    while (p + 32 * U <= end) {
      uint4 r[U];
#pragma unroll
      for (int u = 0; u < U; ++u) r[u] = ldg(p + 32 * u + lane);
      if (((uintptr_t)(p + 32 * U) >> 12) != ((uintptr_t)p >> 12)) prefetch_step(p + 32 * U, end, a.PF, lane);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        acc = work(r[u], acc, a.W);
        if (__all_sync(FULL, r[u].z == 0xFFFFFFFFu)) acc += 1;
      }
      p += 32 * U;
    }
  }
  if (acc == 0x12345678) a.out[0] = acc;
}

template <int U>
__global__ void k_ldg_pipe(Args a) {
  const int lane = threadIdx.x & 31;
  uint32_t acc = 0;
  for (;;) {
    unsigned long long item = 0;
    if (lane == 0) item = atomicAdd(a.counter, 1ull);
    item = __shfl_sync(FULL, item, 0);
    const uint64_t b = item << a.tile_shift;
    if (b >= a.n) break;
    const uint4* p = a.rec + b;
    const uint4* end = a.rec + (b + (1ull << a.tile_shift) < a.n ? b + (1ull << a.tile_shift) : a.n);
    if (a.PF && lane < a.PF) { const char* q = (const char*)((((uintptr_t)p >> 12) + lane) << 12); if (q < (const char*)end) pf(q, 4096); }
    uint4 nx[U];
#pragma unroll
    for (int u = 0; u < U; ++u) nx[u] = p + 32 * u + lane < end ? ldg(p + 32 * u + lane) : make_uint4(0, 0, 0, 0);
    while (p + 32 * U <= end) {
      uint4 r[U];
#pragma unroll
      for (int u = 0; u < U; ++u) r[u] = nx[u];
      const uint4* q = p + 32 * U;
#pragma unroll
      for (int u = 0; u < U; ++u) nx[u] = q + 32 * u + lane < end ? ldg(q + 32 * u + lane) : make_uint4(0, 0, 0, 0);
      if (((uintptr_t)(q) >> 12) != ((uintptr_t)p >> 12)) prefetch_step(q, end, a.PF, lane);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        acc = work(r[u], acc, a.W);
        if (__all_sync(FULL, r[u].z == 0xFFFFFFFFu)) acc += 1;
      }
      p = q;
    }
  }
  if (acc == 0x12345678) a.out[0] = acc;
}

__device__ __forceinline__ void cpa(uint4* dst, const uint4* src, const uint4* end) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(dst);
  const uint32_t n = src < end ? 16u : 0u;
  if (src >= end) src = end - 1;
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n\tcp.async.commit_group;" ::"r"(d), "l"(src), "r"(n) : "memory");
}
template <int N> __device__ __forceinline__ void cpw() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

template <int D>
__global__ void k_cpasync(Args a) {
  extern __shared__ __align__(16) uint4 sm[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint4* ring = sm + warp * D * 32;
  uint32_t acc = 0;
  for (;;) {
    unsigned long long item = 0;
    if (lane == 0) item = atomicAdd(a.counter, 1ull);
    item = __shfl_sync(FULL, item, 0);
    const uint64_t b = item << a.tile_shift;
    if (b >= a.n) break;
    const uint4* p = a.rec + b;
    const uint4* end = a.rec + (b + (1ull << a.tile_shift) < a.n ? b + (1ull << a.tile_shift) : a.n);
    if (a.PF && lane < a.PF) { const char* q = (const char*)((((uintptr_t)p >> 12) + lane) << 12); if (q < (const char*)end) pf(q, 4096); }
    const uint4* f = p;
    int fs = 0, rs = 0;
#pragma unroll
    for (int k = 0; k < D; ++k) { cpa(ring + fs * 32 + lane, f + lane, end); f += 32; fs = fs + 1 == D ? 0 : fs + 1; }
    while (p + 32 <= end) {
      cpw<D - 1>();
      __syncwarp();
      const uint4 r = ring[rs * 32 + lane];
      acc = work(r, acc, a.W);
      if (__all_sync(FULL, r.z == 0xFFFFFFFFu)) acc += 1;
      __syncwarp();
      cpa(ring + fs * 32 + lane, f + lane, end);
      if (((uintptr_t)(f + 32) >> 12) != ((uintptr_t)f >> 12)) prefetch_step(f + 32, end, a.PF, lane);
      f += 32;
      fs = fs + 1 == D ? 0 : fs + 1;
      rs = rs + 1 == D ? 0 : rs + 1;
      p += 32;
    }
    cpw<0>();
  }
  if (acc == 0x12345678) a.out[0] = acc;
}

__device__ __forceinline__ void mb_init(uint64_t* mb) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(mb)) : "memory");
}
__device__ __forceinline__ void tma_load(void* dst, const void* src, uint32_t bytes, uint64_t* mb) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(dst), m = (uint32_t)__cvta_generic_to_shared(mb);
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(m), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d), "l"(src),
               "r"(bytes), "r"(m) : "memory");
}
__device__ __forceinline__ void mb_wait(uint64_t* mb, uint32_t parity) {
  const uint32_t m = (uint32_t)__cvta_generic_to_shared(mb);
  asm volatile(
      "{\n\t.reg .pred P;\n\tWAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra WAIT_%=;\n\t}" ::"r"(m), "r"(parity) : "memory");
}

// ring of D blocks of B bytes per warp; mbarriers after the rings
__global__ void k_tma(Args a) {
  extern __shared__ __align__(128) unsigned char smb[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const int D = a.D, B = a.B, CH = B / 512;
  unsigned char* ring = smb + (size_t)warp * D * B;
  uint64_t* mb = (uint64_t*)(smb + (size_t)nw * D * B) + warp * D;
  if (lane < D) mb_init(&mb[lane]);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  uint32_t phase = 0;  // bit k: parity of block slot k
  uint32_t acc = 0;
  for (;;) {
    unsigned long long item = 0;
    if (lane == 0) item = atomicAdd(a.counter, 1ull);
    item = __shfl_sync(FULL, item, 0);
    const uint64_t b = item << a.tile_shift;
    if (b >= a.n) break;
    const uint4* p = a.rec + b;
    const uint64_t tn = (b + (1ull << a.tile_shift) < a.n ? (1ull << a.tile_shift) : a.n - b);
    const uint4* end = p + tn;
    const int nblk = (int)((tn * 16) / B);  // full blocks only (tile multiple of B)
    if (a.PF && lane < a.PF) { const char* q = (const char*)((((uintptr_t)p >> 12) + lane) << 12); if (q < (const char*)end) pf(q, 4096); }
    if (lane == 0)
      for (int k = 0; k < D && k < nblk; ++k) tma_load(ring + k * B, (const char*)p + (size_t)k * B, B, &mb[k]);
    for (int bi = 0; bi < nblk; ++bi) {
      const int slot = bi % D;
      mb_wait(&mb[slot], (phase >> slot) & 1u);
      phase ^= 1u << slot;
      const uint4* blk = (const uint4*)(ring + slot * B);
      for (int c = 0; c < CH; ++c) {
        const uint4 r = blk[c * 32 + lane];
        acc = work(r, acc, a.W);
        if (__all_sync(FULL, r.z == 0xFFFFFFFFu)) acc += 1;
      }
      __syncwarp();
      if (lane == 0 && bi + D < nblk) {
        const char* src = (const char*)p + (size_t)(bi + D) * B;
        if (a.PF && ((uintptr_t)src >> 12) != (((uintptr_t)src - B) >> 12)) {
          const char* q = (const char*)((((uintptr_t)src >> 12) + a.PF) << 12);
          if (q < (const char*)end) pf(q, 4096);
        }
        tma_load(ring + slot * B, src, B, &mb[slot]);
      }
    }
  }
  if (acc == 0x12345678) a.out[0] = acc;
}

int main(int argc, char** argv) {
  const uint64_t n = (argc > 1 ? strtoull(argv[1], 0, 10) : (1ull << 30));  // records (16 GB)
  uint4* rec;
  CK(cudaMalloc(&rec, n * 16));
  CK(cudaMemset(rec, 0x11, n * 16));
  unsigned long long* ctr;
  unsigned* out;
  CK(cudaMalloc(&ctr, 8));
  CK(cudaMalloc(&out, 4));
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto run = [&](const char* name, void (*k)(Args), int warps, size_t smem, int W, int PF, int D, int B) {
    Args a{rec, n, 15, ctr, out, W, PF, D, B};
    if (smem > 48 * 1024) CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    float best = 1e30f;
    for (int it = 0; it < 4; ++it) {
      CK(cudaMemset(ctr, 0, 8));
      cudaEventRecord(e0);
      k<<<nsm, warps * 32, smem>>>(a);
      cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1));
      CK(cudaGetLastError());
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (it && ms < best) best = ms;
    }
    printf("%-10s warps %2d W %3d PF %d D %d B %5d smem %6zu: %7.1f GB/s\n", name, warps, W, PF, D, B, smem,
           n * 16 / (best * 1e-3) / 1e9);
    fflush(stdout);
  };
  const int Ws[] = {0, 64, 128};
  for (int W : Ws) {
    for (int PF : {0, 2, 4}) {
      run("ldg_u2", k_ldg<2>, 24, 0, W, PF, 0, 0);
      run("ldg_u4", k_ldg<4>, 24, 0, W, PF, 0, 0);
      run("pipe_u1", k_ldg_pipe<1>, 24, 0, W, PF, 0, 0);
      run("pipe_u2", k_ldg_pipe<2>, 24, 0, W, PF, 0, 0);
      run("cpa_d4", k_cpasync<4>, 24, 24 * 4 * 512, W, PF, 0, 0);
      run("cpa_d8", k_cpasync<8>, 24, 24 * 8 * 512, W, PF, 0, 0);
      run("tma_2x1k", k_tma, 24, 24 * (2 * 1024 + 16), W, PF, 2, 1024);
      run("tma_3x1k", k_tma, 24, 24 * (3 * 1024 + 24), W, PF, 3, 1024);
      run("tma_2x2k", k_tma, 24, 24 * (2 * 2048 + 16), W, PF, 2, 2048);
      run("tma_4x1k", k_tma, 16, 16 * (4 * 1024 + 32), W, PF, 4, 1024);
    }
    run("ldg_u2", k_ldg<2>, 32, 0, W, 2, 0, 0);
    run("pipe_u2", k_ldg_pipe<2>, 32, 0, W, 2, 0, 0);
    run("cpa_d4", k_cpasync<4>, 32, 32 * 4 * 512, W, 2, 0, 0);
  }
  return 0;
}
