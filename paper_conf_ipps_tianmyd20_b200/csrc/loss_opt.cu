// Loss and optimiser of the 2-layer GCN step (Kipf's model as used by the
// paper, L203; readings #14): softmax cross-entropy over the train mask with
// its gradient (scaled by r for the prescaled backward aggregation), Adam and
// SGD.  Deterministic: per-CTA partial sums in a fixed order, then one CTA
// sums the partials in index order.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "kernels.h"

namespace pcgcn {
namespace {

constexpr int CE_BLOCKS = 592;  // 4 x 148 SMs, all resident (launch bounds: 4 CTAs/SM); <= PCGCN_CE_WORK_FLOATS

// one warp per row, RPW rows per warp step with all their loads issued up
// front (a row is short: C <= 32*8 logits; at C5's 33.5M rows one row per
// step left the kernel latency-bound, ~11.6 ms); grid-stride over row groups.
constexpr int RPW = 4;
template <int NT>  // 32-logit slices per row (C <= 32 * NT)
__global__ void __launch_bounds__(256, 4) softmax_ce_kernel(
    const float* __restrict__ L, int64_t ld, const int32_t* __restrict__ labels,
    const uint8_t* __restrict__ train, int64_t M, int C, float inv_nT, const float* __restrict__ s,
    float* __restrict__ dL, float* __restrict__ partial) {
  __shared__ float wsum[8];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  float my = 0.f;  // lane 0 of each warp accumulates its rows' losses in row order
  for (int64_t row0 = (int64_t(blockIdx.x) * 8 + w) * RPW; row0 < M; row0 += int64_t(gridDim.x) * 8 * RPW) {
    float v[RPW][NT];
    int y[RPW];
    float scale[RPW];
    bool tr[RPW];
#pragma unroll
    for (int k = 0; k < RPW; ++k) {
      const int64_t row = row0 + k;
      const bool ok = row < M;
      const float* Lr = L + row * ld;
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        const int c = lane + 32 * t;
        v[k][t] = (ok && c < C) ? __ldg(Lr + c) : -INFINITY;
      }
      y[k] = ok ? __ldg(labels + row) : 0;
      tr[k] = ok && __ldg(train + row) != 0;
      scale[k] = ok ? (s ? __ldg(s + row) : 1.f) : 0.f;
    }
#pragma unroll
    for (int k = 0; k < RPW; ++k) {
      const int64_t row = row0 + k;
      float mx = -INFINITY;
#pragma unroll
      for (int t = 0; t < NT; ++t) mx = fmaxf(mx, v[k][t]);
#pragma unroll
      for (int off = 16; off; off >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, off));
      float se = 0.f, ly = 0.f;
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        const int c = lane + 32 * t;
        if (c == y[k]) ly = v[k][t];
        v[k][t] = c < C ? expf(v[k][t] - mx) : 0.f;
        se += v[k][t];
      }
#pragma unroll
      for (int off = 16; off; off >>= 1) {
        se += __shfl_xor_sync(0xffffffffu, se, off);
        ly += __shfl_xor_sync(0xffffffffu, ly, off);  // the label's logit (one lane holds it)
      }
      if (row < M) {
        const float sc = (tr[k] ? inv_nT : 0.f) * scale[k];
        const float inv = 1.f / se;
#pragma unroll
        for (int t = 0; t < NT; ++t) {
          const int c = lane + 32 * t;
          if (c < C) dL[row * ld + c] = (v[k][t] * inv - (c == y[k] ? 1.f : 0.f)) * sc;
        }
        if (lane == 0 && tr[k]) my += (mx + logf(se) - ly);
      }
    }
  }
  if (lane == 0) wsum[w] = my;
  __syncthreads();
  if (threadIdx.x == 0) {
    float t = 0.f;
    for (int i = 0; i < 8; ++i) t += wsum[i];
    partial[blockIdx.x] = t;
  }
}

__global__ void finish_loss_kernel(const float* __restrict__ partial, int nb, float inv_nT,
                                   float* __restrict__ loss) {
  __shared__ float sh[1024];
  float t = 0.f;
  for (int i = threadIdx.x; i < nb; i += blockDim.x) t += partial[i];
  sh[threadIdx.x] = t;
  __syncthreads();
  for (int h = blockDim.x / 2; h > 0; h >>= 1) {
    if (threadIdx.x < h) sh[threadIdx.x] += sh[threadIdx.x + h];
    __syncthreads();
  }
  if (threadIdx.x == 0) *loss = sh[0] * inv_nT;
}

__global__ void adam_kernel(float* __restrict__ th, const float* __restrict__ g, float* __restrict__ m,
                            float* __restrict__ v, int64_t n, float lr, float b1, float b2, float eps,
                            const int32_t* __restrict__ step) {
  const int t = *step + 1;
  const float c1 = 1.f - powf(b1, float(t));
  const float c2 = 1.f - powf(b2, float(t));
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x) {
    float gi = g[i];
    float mi = b1 * m[i] + (1.f - b1) * gi;
    float vi = b2 * v[i] + (1.f - b2) * gi * gi;
    m[i] = mi;
    v[i] = vi;
    th[i] -= lr * (mi / c1) / (sqrtf(vi / c2) + eps);
  }
}

__global__ void step_inc_kernel(int32_t* step) { *step += 1; }

__global__ void sgd_kernel(float* __restrict__ th, const float* __restrict__ g, int64_t n, float lr) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x)
    th[i] -= lr * g[i];
}

}  // namespace

cudaError_t launch_softmax_ce(const float* L, int64_t ld, const int32_t* labels,
                              const uint8_t* train, int64_t M, int C, float inv_nT, const float* s,
                              float* dL, float* loss, float* work, cudaStream_t st) {
  if (C > 256) return cudaErrorInvalidValue;
  const int nt = (C + 31) / 32;
  if (nt <= 1) softmax_ce_kernel<1><<<CE_BLOCKS, 256, 0, st>>>(L, ld, labels, train, M, C, inv_nT, s, dL, work);
  else if (nt <= 2) softmax_ce_kernel<2><<<CE_BLOCKS, 256, 0, st>>>(L, ld, labels, train, M, C, inv_nT, s, dL, work);
  else if (nt <= 4) softmax_ce_kernel<4><<<CE_BLOCKS, 256, 0, st>>>(L, ld, labels, train, M, C, inv_nT, s, dL, work);
  else softmax_ce_kernel<8><<<CE_BLOCKS, 256, 0, st>>>(L, ld, labels, train, M, C, inv_nT, s, dL, work);
  finish_loss_kernel<<<1, 1024, 0, st>>>(work, CE_BLOCKS, inv_nT, loss);
  return cudaGetLastError();
}

cudaError_t launch_adam(float* th, const float* g, float* m, float* v, int64_t n, float lr, float b1,
                        float b2, float eps, int32_t* step, cudaStream_t st) {
  int blocks = int(std::min<int64_t>(1024, (n + 255) / 256));
  adam_kernel<<<blocks, 256, 0, st>>>(th, g, m, v, n, lr, b1, b2, eps, step);
  step_inc_kernel<<<1, 1, 0, st>>>(step);
  return cudaGetLastError();
}

cudaError_t launch_sgd(float* th, const float* g, int64_t n, float lr, cudaStream_t st) {
  int blocks = int(std::min<int64_t>(1024, (n + 255) / 256));
  sgd_kernel<<<blocks, 256, 0, st>>>(th, g, n, lr);
  return cudaGetLastError();
}

}  // namespace pcgcn
