/* gen_device.cu — device build of the synthetic trace generator (libowlgen_cuda.so).  TEST / BENCH
 * INFRASTRUCTURE (untimed): generates the same records as gen_host.c directly into HBM, so that the
 * 44-184 GB workloads never cross PCIe.  One thread per traced warp. */
#include <cuda_runtime.h>

#include "owl_gen_core.h"

#define OG_API extern "C" __attribute__((visibility("default")))

__global__ void og_count_kernel(og_params p, uint32_t r, uint32_t seq, uint32_t nw, uint64_t* counts) {
  uint32_t w = blockIdx.x * blockDim.x + threadIdx.x;
  if (w < nw) counts[w] = og_warp(&p, r, seq, w, nullptr);
}

/* exclusive scan of nw counts into offs[0..nw] (single block; nw is at most a few thousand) */
__global__ void og_scan_kernel(const uint64_t* counts, uint32_t nw, uint64_t* offs) {
  __shared__ uint64_t part[1024];
  uint32_t t = threadIdx.x, per = (nw + blockDim.x - 1) / blockDim.x;
  uint32_t b = t * per, e = b + per < nw ? b + per : nw;
  uint64_t s = 0;
  for (uint32_t i = b; i < e; ++i) s += counts[i];
  part[t] = s;
  __syncthreads();
  if (t == 0) {
    uint64_t acc = 0;
    for (uint32_t i = 0; i < blockDim.x; ++i) { uint64_t v = part[i]; part[i] = acc; acc += v; }
    offs[nw] = acc;
  }
  __syncthreads();
  uint64_t acc = part[t];
  for (uint32_t i = b; i < e; ++i) { offs[i] = acc; acc += counts[i]; }
}

__global__ void og_gen_kernel(og_params p, uint32_t r, uint32_t seq, uint32_t nw, const uint64_t* offs,
                              og_record* out) {
  uint32_t w = blockIdx.x * blockDim.x + threadIdx.x;
  if (w < nw) og_warp(&p, r, seq, w, out + offs[w]);
}

/* d_offs: device array of n_warps+1 u64 (scratch d_counts: n_warps u64). Returns a cudaError_t. */
OG_API int ogd_seq_offsets(const og_params* p, uint32_t r, uint32_t seq, uint64_t* d_counts, uint64_t* d_offs,
                           void* stream) {
  cudaStream_t st = (cudaStream_t)stream;
  uint32_t nw = og_seq_n_warps(p, r, seq);
  og_count_kernel<<<(nw + 127) / 128, 128, 0, st>>>(*p, r, seq, nw, d_counts);
  og_scan_kernel<<<1, 1024, 0, st>>>(d_counts, nw, d_offs);
  return (int)cudaGetLastError();
}

OG_API int ogd_seq_generate(const og_params* p, uint32_t r, uint32_t seq, const uint64_t* d_offs, og_record* d_out,
                            void* stream) {
  cudaStream_t st = (cudaStream_t)stream;
  uint32_t nw = og_seq_n_warps(p, r, seq);
  og_gen_kernel<<<(nw + 63) / 64, 64, 0, st>>>(*p, r, seq, nw, d_offs, d_out);
  return (int)cudaGetLastError();
}
