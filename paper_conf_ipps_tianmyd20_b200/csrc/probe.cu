// Measurement helper (not on the hot path): read bandwidth of the L2->SM path
// (buffer << 126 MB) or of HBM (buffer >> 126 MB), used by bench.py to put
// the gather kernels on a measured roofline.
#include <cuda_runtime.h>

#include <cstdint>
#include <string>

#include "plan_internal.h"

namespace {

__global__ void __launch_bounds__(512) read_kernel(const float4* __restrict__ p, int64_t n4, int iters,
                                                   float* __restrict__ sink) {
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  const int64_t stride = int64_t(gridDim.x) * blockDim.x;
  for (int it = 0; it < iters; ++it) {
    // rotate the starting block every pass so each SM streams different lines
    const int64_t start = (int64_t(blockIdx.x + it * 37) % gridDim.x) * blockDim.x + threadIdx.x;
    for (int64_t i = start; i < n4; i += stride) {
      const float4 v = __ldcg(p + i);
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
  }
  if (acc.x + acc.y + acc.z + acc.w == 1234.5678f) *sink = acc.x;  // keep the loads alive
}

}  // namespace

extern "C" pcgcn_status pcgcn_probe_read_gbs(int64_t bytes, int32_t iters, float* gbs) {
  if (bytes < (1 << 20) || iters < 1 || !gbs) {
    pcgcn::set_error("probe: bad arguments");
    return PCGCN_EINVAL;
  }
  float4* buf = nullptr;
  float* sink = nullptr;
  cudaEvent_t a, b;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (cudaMalloc(&buf, bytes) != cudaSuccess || cudaMalloc(&sink, 4) != cudaSuccess) {
    pcgcn::set_error("probe: allocation failed");
    return PCGCN_ENOMEM;
  }
  cudaMemset(buf, 0, bytes);
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int64_t n4 = bytes / 16;
  read_kernel<<<sms * 4, 512>>>(buf, n4, 1, sink);  // warm-up (and L2 fill)
  cudaEventRecord(a);
  read_kernel<<<sms * 4, 512>>>(buf, n4, iters, sink);
  cudaEventRecord(b);
  cudaError_t e = cudaEventSynchronize(b);
  float ms = 0.f;
  if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, a, b);
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(buf);
  cudaFree(sink);
  if (e != cudaSuccess) {
    pcgcn::set_error(std::string("probe: ") + cudaGetErrorString(e));
    return PCGCN_ECUDA;
  }
  *gbs = float(double(n4) * 16.0 * iters / (double(ms) * 1e-3) / 1e9);
  return PCGCN_OK;
}
