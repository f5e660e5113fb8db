// Feature-transform GEMMs of the 2-layer GCN step (Alg. 1 a^l = h^{l-1} w^l,
// L114; the paper runs these as TF MatMul / cuBLAS, L203) and their backward
// counterparts (the paper is silent on the backward, reading A4).
//
// xw and xtg run on the tcgen05 engine (tc_engine.cu) in 3xTF32 when the
// operands are 16-byte aligned (ld % 4 == 0) and a workspace is given; the
// fp32 CUDA-core tiles below (64x64 output tile per CTA, 4x4 register
// micro-tiles) serve the remaining shapes and dwt, with fused epilogues:
//   xw : Y = diag(s)·(X·W)                      (a4, a7: source prescaling)
//   dwt: O = diag(s)·((D·Wᵀ) ⊙ mask)            (a11: ReLU' via the bit mask)
//   xtg: G = Xᵀ·D, split over M into fixed slices + fixed-order reduction
//        (a11, a13: deterministic, no atomics)
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstdint>

#include "kernels.h"

namespace pcgcn {
namespace {

constexpr int BM = 64, BN = 64, BK = 16;

// C[m][n] = Σ_k opA(m,k)·opB(k,n) over k in [k0,k1)
//   opA(m,k) = AT ? A[k*lda+m] : A[m*lda+k]
//   opB(k,n) = BT ? B[n*ldb+k] : B[k*ldb+n]
// Epilogue: optional row scale s[m], optional mask bits (row stride mw), store
// to C[m*ldc+n] (+ z*zstride for split partials).
template <bool AT, bool BT>
__global__ void __launch_bounds__(256) gemm_simt_kernel(
    const float* __restrict__ A, int64_t lda, const float* __restrict__ B, int64_t ldb,
    float* __restrict__ C, int64_t ldc, int64_t M, int N, int64_t K, int64_t kslice,
    const float* __restrict__ s, const uint32_t* __restrict__ mask, int mw, int64_t zstride) {
  __shared__ float As[BK][BM + 4];
  __shared__ float Bs[BK][BN + 4];
  const int tid = threadIdx.x;
  const int tx = tid % 16, ty = tid / 16;
  const int64_t m0 = int64_t(blockIdx.x) * BM;
  const int n0 = blockIdx.y * BN;
  const int64_t kb = int64_t(blockIdx.z) * kslice;
  const int64_t ke = (kb + kslice < K) ? kb + kslice : K;
  float acc[4][4] = {};
  for (int64_t k0 = kb; k0 < ke; k0 += BK) {
    // load A tile (BM x BK) -> As[k][m]
#pragma unroll
    for (int t = 0; t < (BM * BK) / 256; ++t) {
      int e = tid + t * 256;
      int mm, kk;
      if (AT) { mm = e % BM; kk = e / BM; } else { kk = e % BK; mm = e / BK; }
      int64_t gm = m0 + mm, gk = k0 + kk;
      float v = 0.f;
      if (gm < M && gk < ke) v = AT ? A[gk * lda + gm] : A[gm * lda + gk];
      As[kk][mm] = v;
    }
#pragma unroll
    for (int t = 0; t < (BN * BK) / 256; ++t) {
      int e = tid + t * 256;
      int nn, kk;
      if (BT) { kk = e % BK; nn = e / BK; } else { nn = e % BN; kk = e / BN; }
      int gn = n0 + nn;
      int64_t gk = k0 + kk;
      float v = 0.f;
      if (gn < N && gk < ke) v = BT ? B[int64_t(gn) * ldb + gk] : B[gk * ldb + gn];
      Bs[kk][nn] = v;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[kk][ty + 16 * i];
#pragma unroll
      for (int j = 0; j < 4; ++j) b[j] = Bs[kk][tx + 16 * j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
  float* Cz = C + int64_t(blockIdx.z) * zstride;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    int64_t gm = m0 + ty + 16 * i;
    if (gm >= M) continue;
    float sc = s ? s[gm] : 1.f;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int gn = n0 + tx + 16 * j;
      if (gn >= N) continue;
      float v = acc[i][j];
      if (mask) v = ((mask[gm * mw + (gn >> 5)] >> (gn & 31)) & 1u) ? v : 0.f;
      Cz[gm * ldc + gn] = v * sc;
    }
  }
}

__global__ void reduce_slices_kernel(const float* __restrict__ part, int nslices, int64_t count,
                                     float* __restrict__ out) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < count;
       i += int64_t(gridDim.x) * blockDim.x) {
    float a = 0.f;
    for (int z = 0; z < nslices; ++z) a += part[int64_t(z) * count + i];
    out[i] = a;
  }
}

// zero the pad columns [N, ldc) of the first M rows (outputs' pad must be 0)
__global__ void zero_pad_kernel(float* C, int64_t ldc, int64_t M, int N) {
  const int w = int(ldc) - N;
  if (w <= 0) return;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < M * w;
       i += int64_t(gridDim.x) * blockDim.x)
    C[(i / w) * ldc + N + (i % w)] = 0.f;
}

// PCGCN_XTG_PRESPLIT=1: the feature-major split pass + engine instead of the
// in-kernel conversion of D (A/B knob, benchmarks only)
bool xtg_presplit() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("PCGCN_XTG_PRESPLIT");
    v = e ? (atoi(e) != 0) : 0;
  }
  return v != 0;
}
int xtg_slices(int64_t M) { return int(std::min<int64_t>(296, std::max<int64_t>(1, (M + 1023) / 1024))); }

}  // namespace

int64_t r32(int64_t x) { return (x + 31) / 32 * 32; }
int npad16(int n) { return (n + 15) / 16 * 16; }

int64_t gemm_xw_work_floats(int K, int N) { return 2 * int64_t(npad16(N)) * r32(K); }

cudaError_t launch_gemm_xw(const float* X, int64_t ldx, const float* W, int64_t ldw, const float* s,
                           float* Y, int64_t ldy, int64_t M, int K, int N, float* work, cudaStream_t st,
                           const WindowOut* wo) {
  if (work && ldx % 4 == 0 && ldy % 4 == 0 && N <= 256 && M > 0) {
    // tcgen05 3xTF32: Wᵀ split hi/lo (feature-major), then the engine
    const int np = npad16(N);
    const int64_t ldT = r32(K);
    float* hi = work;
    float* lo = work + int64_t(np) * ldT;
    cudaError_t e = launch_split_transpose(W, ldw, K, N, np, hi, lo, ldT, st);
    if (e != cudaSuccess) return e;
    e = launch_tc_gemm_xw(X, ldx, hi, lo, ldT, s, Y, ldy, M, K, N, st, nullptr, 0, wo);
    if (e != cudaSuccess) return e;
    if (ldy > np) zero_pad_kernel<<<256, 256, 0, st>>>(Y, ldy, M, np);
    return cudaGetLastError();
  }
  dim3 grid(unsigned((M + BM - 1) / BM), unsigned((N + BN - 1) / BN), 1);
  gemm_simt_kernel<false, false><<<grid, 256, 0, st>>>(X, ldx, W, ldw, Y, ldy, M, N, K, K, s,
                                                       nullptr, 0, 0);
  if (ldy > N) zero_pad_kernel<<<256, 256, 0, st>>>(Y, ldy, M, N);
  return cudaGetLastError();
}

int64_t gemm_xtg_work_floats(int64_t M, int K, int N) {
  const int64_t simt = int64_t(xtg_slices(M)) * K * N;
  // the in-engine B conversion (npad <= 128) needs only the slice partials; the
  // pre-split path also a feature-major hi/lo copy of D (2 x npad x M floats)
  const bool raw = npad16(N) <= 128 && !xtg_presplit();
  const int64_t tc = (raw ? 0 : 2 * int64_t(npad16(N)) * r32(M)) + tc_xtg_slices(M, K) * int64_t(K) * npad16(N);
  return simt > tc ? simt : tc;
}

__global__ void reduce_slices_ld_kernel(const float* __restrict__ part, int nslices, int64_t rows, int N,
                                        int ldp, float* __restrict__ out) {
  const int64_t count = rows * N;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < count;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = i / N;
    const int c = int(i - r * N);
    float a = 0.f;
    for (int z = 0; z < nslices; ++z) a += part[int64_t(z) * rows * ldp + r * ldp + c];
    out[i] = a;
  }
}

cudaError_t launch_gemm_xtg(const float* X, int64_t ldx, const float* D, int64_t ldd, float* G,
                            int64_t M, int K, int N, float* work, cudaStream_t st) {
  if (ldx % 4 == 0 && ldd % 4 == 0 && N <= 256 && M > 0) {
    // tcgen05 3xTF32: Dᵀ split hi/lo (feature-major), engine over fixed row
    // slices, then a fixed-order sum of the slice partials
    const int np = npad16(N);
    const int64_t ldT = r32(M);
    const bool raw = np <= 128 && !xtg_presplit();
    float* hi = work;
    float* lo = work + int64_t(np) * ldT;
    float* part = raw ? work : lo + int64_t(np) * ldT;
    cudaError_t e;
    if (raw) {
      // B converted inside the engine (D read once; no split pass)
      e = launch_tc_gemm_xtg_raw(X, ldx, D, ldd, part, M, K, N, st);
    } else {
      e = launch_split_transpose(D, ldd, M, N, np, hi, lo, ldT, st);
      if (e != cudaSuccess) return e;
      e = launch_tc_gemm_xtg(X, ldx, hi, lo, ldT, part, M, K, N, st);
    }
    if (e != cudaSuccess) return e;
    const int64_t cnt = int64_t(K) * N;
    reduce_slices_ld_kernel<<<unsigned(std::max<int64_t>(1, std::min<int64_t>(1024, (cnt + 255) / 256))), 256, 0, st>>>(
        part, int(tc_xtg_slices(M, K)), K, N, np, G);
    return cudaGetLastError();
  }
  // G[K x N] = Xᵀ D : output rows = K (A = X transposed), reduction over M
  const int ns = xtg_slices(M);
  int64_t kslice = ((M + ns - 1) / ns + BK - 1) / BK * BK;
  dim3 grid(unsigned((K + BM - 1) / BM), unsigned((N + BN - 1) / BN), unsigned(ns));
  gemm_simt_kernel<true, false><<<grid, 256, 0, st>>>(X, ldx, D, ldd, work, N, K, N, M, kslice,
                                                      nullptr, nullptr, 0, int64_t(K) * N);
  reduce_slices_kernel<<<std::max<int64_t>(1, std::min<int64_t>(1024, (int64_t(K) * N + 255) / 256)), 256, 0, st>>>(
      work, ns, int64_t(K) * N, G);
  return cudaGetLastError();
}

// tf32 hi/lo split of W [K x N] (ld ldw) kept row-major = feature-major for
// the engine's B operand of O = D·Wᵀ: hi/lo [np x ldT], rows >= K and
// columns >= N zero
__global__ void split_rows_kernel(const float* __restrict__ W, int64_t ldw, int K, int N, int np, int64_t ldT,
                                  float* __restrict__ hi, float* __restrict__ lo) {
  const int64_t total = int64_t(np) * ldT;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < total;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = i / ldT, c = i - r * ldT;
    const float v = (r < K && c < N) ? W[r * ldw + c] : 0.f;
    const float h = __uint_as_float(__float_as_uint(v) & 0xffffe000u);
    hi[i] = h;
    lo[i] = v - h;
  }
}

int64_t gemm_dwt_work_floats(int K, int N) { return 2 * int64_t(npad16(K)) * r32(N); }

cudaError_t launch_gemm_dwt(const float* D, int64_t ldd, const float* W, const uint32_t* mask,
                            const float* s, float* O, int64_t ldo, int64_t M, int N, int K,
                            float* work, cudaStream_t st, const WindowOut* wo) {
  if (work && ldd % 4 == 0 && ldo % 4 == 0 && K <= 256 && M > 0) {
    // tcgen05 3xTF32 (the xw engine with D as A, W rows as the feature-major
    // B, and the ReLU' bit mask + row scale in the epilogue)
    const int np = npad16(K);
    const int64_t ldT = r32(N);
    float* hi = work;
    float* lo = work + int64_t(np) * ldT;
    split_rows_kernel<<<unsigned(std::min<int64_t>(256, (np * ldT + 255) / 256)), 256, 0, st>>>(
        W, N, K, N, np, ldT, hi, lo);
    cudaError_t e = launch_tc_gemm_xw(D, ldd, hi, lo, ldT, s, O, ldo, M, N, K, st, mask, (K + 31) / 32, wo);
    if (e != cudaSuccess) return e;
    if (ldo > np) zero_pad_kernel<<<256, 256, 0, st>>>(O, ldo, M, np);
    return cudaGetLastError();
  }
  // O[M x K] = D[M x N] · Wᵀ  with W [K x N] row-major: opB(n, k) = W[k*N + n]
  dim3 grid(unsigned((M + BM - 1) / BM), unsigned((K + BN - 1) / BN), 1);
  gemm_simt_kernel<false, true><<<grid, 256, 0, st>>>(D, ldd, W, N, O, ldo, M, K, N, N, s, mask,
                                                      (K + 31) / 32, 0);
  if (ldo > K) zero_pad_kernel<<<256, 256, 0, st>>>(O, ldo, M, K);
  return cudaGetLastError();
}

}  // namespace pcgcn
