// Full-mode ("dense") aggregation on CUDA cores — the paper's §IV-C kernel
// (L183-L187: one block pair per thread block, dense edge tile staged in
// shared memory, consecutive threads over consecutive feature dimensions,
// register accumulation).  On B200 the product full mode is the tcgen05
// kernel (dense_tc.cu); this fp32 kernel is selected with
// dense_prec = PCGCN_DENSE_FP32_SIMT and serves as the exact-fp32 cross-check
// of the bit-tile layout.
//
// One CTA per 128-row destination tile; for every 128x32 bit chunk of the
// tile, the 32 source rows (prescaled Y) are staged in smem and each thread
// accumulates its fixed set of (row, float4) outputs in chunk order.
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.h"

namespace pcgcn {
namespace {

__global__ void __launch_bounds__(256) dense_simt_kernel(DenseArgs a, const float* __restrict__ y,
                                                         int64_t ldy, int nvec) {
  extern __shared__ float4 sm[];  // [32][nvec] source rows
  __shared__ uint32_t sbits[128];
  const int64_t t = blockIdx.x;
  const int tid = threadIdx.x;
  const int npairs = 128 * nvec;
  float4 acc[16];
#pragma unroll
  for (int s = 0; s < 16; ++s) acc[s] = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int64_t c = a.rt_cptr[t]; c < a.rt_cptr[t + 1]; ++c) {
    const int64_t col0 = a.ch_col0[c];
    __syncthreads();
    if (tid < 128) sbits[tid] = a.bits[c * 128 + tid];
    for (int e = tid; e < 32 * nvec; e += 256) {
      int b = e / nvec, q = e % nvec;
      int64_t src = col0 + b;
      sm[e] = src < a.n_src ? *reinterpret_cast<const float4*>(y + src * ldy + 4 * q)
                        : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    __syncthreads();
#pragma unroll
    for (int s = 0; s < 16; ++s) {
      const int pr = tid + 256 * s;
      if (pr < npairs) {
        const int rr = pr / nvec, q = pr % nvec;
        uint32_t w = sbits[rr];
        while (w) {
          const int b = __ffs(w) - 1;
          w &= w - 1;
          float4 v = sm[b * nvec + q];
          acc[s].x += v.x; acc[s].y += v.y; acc[s].z += v.z; acc[s].w += v.w;
        }
      }
    }
  }
#pragma unroll
  for (int s = 0; s < 16; ++s) {
    const int pr = tid + 256 * s;
    if (pr < npairs) {
      const int rr = pr / nvec, q = pr % nvec;
      *reinterpret_cast<float4*>(a.zd + (t * 128 + rr) * a.ldzd + 4 * q) = acc[s];
    }
  }
}

}  // namespace

cudaError_t launch_dense_simt_y(const DenseArgs& a, const float* y, int64_t ldy, int F,
                                cudaStream_t s) {
  if (a.nrt <= 0) return cudaSuccess;
  const int nvec = (F + 3) / 4;
  if (nvec > 32) return cudaErrorInvalidValue;  // 16 pairs/thread x 256 threads = 128 rows x 32 float4
  dense_simt_kernel<<<unsigned(a.nrt), 256, 32 * nvec * sizeof(float4), s>>>(a, y, ldy, nvec);
  return cudaGetLastError();
}

}  // namespace pcgcn
