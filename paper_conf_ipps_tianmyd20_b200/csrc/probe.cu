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

// Random-row gather: the selective kernel's access pattern without its index
// stream.  A warp's 32 lanes form 32/G slots of G = row_bytes/16 lanes; every
// step each slot reads one pseudo-random row (LCG per slot, power-of-two row
// count) with plain cached 16-byte loads, 8 steps in flight per lane.  The
// buffer size picks the level that serves the rows: L1 (<= ~128 KB), L2
// (<< 126 MB) or HBM (>> 126 MB).
template <int G>
__global__ void __launch_bounds__(256) gather_kernel(const char* __restrict__ p, uint32_t row_mask,
                                                     uint32_t row_bytes, int steps, float* __restrict__ sink) {
  const int lane = threadIdx.x & 31;
  const uint32_t slot = uint32_t(lane / G);
  const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  uint32_t st = (gw * 32u + slot) * 2654435761u + 12345u;
  const int q = lane % G;
  const char* base = p + (16u * q < row_bytes ? 16 * q : 0);  // lanes past the row re-read its first 16 B
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int k = 0; k < steps; k += 8) {
    float4 v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      st = st * 1664525u + 1013904223u;
      const uint32_t j = (st >> 7) & row_mask;
      v[u] = __ldg(reinterpret_cast<const float4*>(base + size_t(j) * row_bytes));
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w;
    }
  }
  if (acc.x + acc.y + acc.z + acc.w == 1234.5678f) *sink = acc.x;
}

}  // namespace

extern "C" pcgcn_status pcgcn_probe_gather_gbs(int64_t bytes, int32_t row_bytes, int32_t steps, float* gbs) {
  if (bytes < (16 << 10) || steps < 8 || !gbs || row_bytes < 16 || row_bytes > 512 || (row_bytes & 15)) {
    pcgcn::set_error("probe_gather: bad arguments (row_bytes a multiple of 16 in [16, 512], steps >= 8)");
    return PCGCN_EINVAL;
  }
  int64_t rows = 1;
  while (rows * 2 * row_bytes <= bytes) rows *= 2;
  char* buf = nullptr;
  float* sink = nullptr;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (cudaMalloc(&buf, size_t(rows) * row_bytes) != cudaSuccess || cudaMalloc(&sink, 4) != cudaSuccess) {
    pcgcn::set_error("probe_gather: allocation failed");
    return PCGCN_ENOMEM;
  }
  cudaMemset(buf, 0, size_t(rows) * row_bytes);
  int G = 1;
  while (G * 16 < row_bytes) G *= 2;  // narrowest power-of-two slot covering the row (as the kernel)
  const int blocks = sms * 4;  // 4 CTAs x 8 warps per SM: the selective kernel's occupancy
  auto go = [&](int n) {
    switch (G) {
      case 1: gather_kernel<1><<<blocks, 256>>>(buf, uint32_t(rows - 1), row_bytes, n, sink); break;
      case 2: gather_kernel<2><<<blocks, 256>>>(buf, uint32_t(rows - 1), row_bytes, n, sink); break;
      case 4: gather_kernel<4><<<blocks, 256>>>(buf, uint32_t(rows - 1), row_bytes, n, sink); break;
      case 8: gather_kernel<8><<<blocks, 256>>>(buf, uint32_t(rows - 1), row_bytes, n, sink); break;
      case 16: gather_kernel<16><<<blocks, 256>>>(buf, uint32_t(rows - 1), row_bytes, n, sink); break;
      default: gather_kernel<32><<<blocks, 256>>>(buf, uint32_t(rows - 1), row_bytes, n, sink); break;
    }
  };
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  go(8);  // warm-up
  cudaEventRecord(a);
  go(steps);
  cudaEventRecord(b);
  cudaError_t e = cudaEventSynchronize(b);
  float ms = 0.f;
  if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, a, b);
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(buf);
  cudaFree(sink);
  if (e != cudaSuccess) {
    pcgcn::set_error(std::string("probe_gather: ") + cudaGetErrorString(e));
    return PCGCN_ECUDA;
  }
  // rows gathered: every slot of every warp reads one row of row_bytes per step
  const double warps = double(blocks) * 8.0;
  const double per_row = double(row_bytes);
  *gbs = float(warps * (32.0 / G) * (steps / 8 * 8) * per_row / (double(ms) * 1e-3) / 1e9);
  return PCGCN_OK;
}

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
