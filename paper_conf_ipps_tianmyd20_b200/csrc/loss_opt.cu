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

// C <= 32: four lanes per row (8 logits each as two float4), eight rows per
// warp step — the reductions take 2 shuffle rounds instead of 5 and every
// instruction serves 8 rows (C5: 33.5 M rows of 32 logits; the warp-per-row
// kernel was issue-bound at 74%).  Rows need ld % 4 == 0 (16-byte rows).
__global__ void __launch_bounds__(256) softmax_ce_c32_kernel(
    const float* __restrict__ L, int64_t ld, const int32_t* __restrict__ labels,
    const uint8_t* __restrict__ train, int64_t M, int C, float inv_nT, const float* __restrict__ s,
    float* __restrict__ dL, float* __restrict__ partial) {
  __shared__ float wsum[8];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int q = lane & 3, rsub = lane >> 2;  // 4 lanes per row, 8 rows per warp step
  const int c0 = 8 * q;                      // this lane's first logit
  float my = 0.f;                            // lane q == 0 of each row group: its rows' losses, in order
  for (int64_t row0 = (int64_t(blockIdx.x) * 8 + w) * 8; row0 < M; row0 += int64_t(gridDim.x) * 64) {
    const int64_t row = row0 + rsub;
    const bool ok = row < M;
    float v[8];
    const float* Lr = L + row * ld + c0;
    if (ok && c0 + 8 <= C) {
      const float4 a = __ldg(reinterpret_cast<const float4*>(Lr));
      const float4 b = __ldg(reinterpret_cast<const float4*>(Lr + 4));
      v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
    } else {
#pragma unroll
      for (int e = 0; e < 8; ++e) v[e] = (ok && c0 + e < C) ? __ldg(Lr + e) : -INFINITY;
    }
    const int y = ok ? __ldg(labels + row) : -1;
    const bool tr = ok && __ldg(train + row) != 0;
    const float scale = ok ? (s ? __ldg(s + row) : 1.f) : 0.f;
    float mx = v[0];
#pragma unroll
    for (int e = 1; e < 8; ++e) mx = fmaxf(mx, v[e]);
    mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 1));
    mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 2));
    float se = 0.f, ly = 0.f;
#pragma unroll
    for (int e = 0; e < 8; ++e) {
      if (c0 + e == y) ly = v[e];
      v[e] = (c0 + e < C) ? expf(v[e] - mx) : 0.f;
      se += v[e];
    }
    se += __shfl_xor_sync(0xffffffffu, se, 1);
    se += __shfl_xor_sync(0xffffffffu, se, 2);
    ly += __shfl_xor_sync(0xffffffffu, ly, 1);
    ly += __shfl_xor_sync(0xffffffffu, ly, 2);
    if (ok) {
      const float sc = (tr ? inv_nT : 0.f) * scale;
      const float inv = 1.f / se;
      float o[8];
#pragma unroll
      for (int e = 0; e < 8; ++e) o[e] = (v[e] * inv - (c0 + e == y ? 1.f : 0.f)) * sc;
      float* Dr = dL + row * ld + c0;
      if (c0 + 8 <= C) {
        *reinterpret_cast<float4*>(Dr) = make_float4(o[0], o[1], o[2], o[3]);
        *reinterpret_cast<float4*>(Dr + 4) = make_float4(o[4], o[5], o[6], o[7]);
      } else {
#pragma unroll
        for (int e = 0; e < 8; ++e)
          if (c0 + e < C) Dr[e] = o[e];
      }
    }
    // this step's 8 row losses, summed in row order by lane 0
    const float lrow = (tr && q == 0) ? (mx + logf(se) - ly) : 0.f;
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const float x = __shfl_sync(0xffffffffu, lrow, 4 * k);
      if (lane == 0) my += x;
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
  if (nt <= 1 && ld % 4 == 0 && (reinterpret_cast<uintptr_t>(L) & 15) == 0 && (reinterpret_cast<uintptr_t>(dL) & 15) == 0)
    softmax_ce_c32_kernel<<<CE_BLOCKS, 256, 0, st>>>(L, ld, labels, train, M, C, inv_nT, s, dL, work);
  else if (nt <= 1) softmax_ce_kernel<1><<<CE_BLOCKS, 256, 0, st>>>(L, ld, labels, train, M, C, inv_nT, s, dL, work);
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
