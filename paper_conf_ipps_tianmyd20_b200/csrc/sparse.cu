// Selective-mode ("sparse") aggregation of PCGCN on sm_100a, plus the input
// prescale / tf32-split pass that feeds both modes.
//
// Paper: §III-B.a (L137, L149) and §IV-B (L177-L181, Fig. 6).  The selective
// blocks of all partition pairs are merged into one CSR (L179); per edge the
// kernel decodes the source index, fetches the source feature row, multiplies
// by the edge value and accumulates into the destination (L149); "consecutive
// threads process consecutive dimensions of the feature vector and update the
// accumulated intermediate data in registers" and each destination row is
// written once (L181).
//
// B200 design:
//   * one warp per destination row; the 32 lanes split into S = 32/G edge
//     slots of G lanes, each lane owning one float4 of the row (F <= 128) or
//     two (F <= 256) — full lane use for narrow F (41 -> G=16, S=2);
//   * the warp loads 32 source indices with one coalesced load and broadcasts
//     them by shuffle; the unrolled loop keeps up to 32/S independent 16-byte
//     row loads in flight per lane (the gather is L2-bandwidth bound);
//   * edge values are not stored: Â_ij = r_i r_j, with r_j folded into the
//     producer (IN_PRESCALED) and r_i applied once in the epilogue;
//   * fused epilogue: + dense-mode partial sum Zd (mode combine, L193),
//     × r_i, optional second × r_i, ReLU and the bit-packed ReLU mask;
//   * fixed summation order (4 interleaved accumulators, then a butterfly over
//     slots): bitwise reproducible run to run.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>

#include "kernels.h"

namespace pcgcn {
namespace {

__device__ __forceinline__ float4 ld_f4(const float* p) {
  return __ldg(reinterpret_cast<const float4*>(p));
}
// L2 eviction policies for the gather loads; see gather_hint() for the
// measured choice (the once-read index stream is marked evict_first)
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ float4 ld_f4_hint(const float* p, uint64_t pol) {
  float4 v;
  asm volatile("ld.global.nc.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ float4 ld_f4_na_hint(const float* p, uint64_t pol) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ int ld_idx_hint(const int* p, uint64_t pol) {
  int v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ void add4(float4& a, const float4& b) {
  a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w;
}

template <int G, int V, bool HAS_ZD, int HINT, int MINB>
__global__ void __launch_bounds__(256, MINB) sparse_agg_kernel(AggArgs a) {
  constexpr int S = 32 / G;                 // edges in flight per warp step (slots)
  constexpr int STEPS = 32 / S;             // steps per 32-index batch
  // steps whose loads are all issued before any is consumed: a power of two
  // dividing STEPS with UNR*V <= 8 float4 in flight per lane (16 measured
  // slower on C3: the register cost lowers occupancy more than ILP gains)
  constexpr int UCAP = 8 / V;
  constexpr int UNR = (UCAP >= 16 && STEPS >= 16) ? 16
                    : (UCAP >= 8 && STEPS >= 8) ? 8
                    : (UCAP >= 4 && STEPS >= 4) ? 4
                    : (UCAP >= 2 && STEPS >= 2) ? 2 : 1;
  constexpr int NACC = V >= 3 ? 1 : (V == 2 ? 2 : 4);                        // interleaved partial sums
  const int64_t row = int64_t(blockIdx.x) * 8 + (threadIdx.x >> 5);
  if (row >= a.rows) return;
  const int lane = threadIdx.x & 31;
  const int slot = lane / G, l = lane % G;
  const int nvec = (a.F + 3) >> 2;
  const int64_t e0 = a.rowptr[row], e1 = a.rowptr[row + 1];
  // per-lane column offsets (loop invariant); lanes past F read the zero row
  int qoff[V];
#pragma unroll
  for (int v = 0; v < V; ++v) qoff[v] = (l + G * v) < nvec ? 4 * (l + G * v) : -1;
  float4 acc[NACC][V];
#pragma unroll
  for (int u = 0; u < NACC; ++u)
#pragma unroll
    for (int v = 0; v < V; ++v) acc[u][v] = make_float4(0.f, 0.f, 0.f, 0.f);

  // Branch-free batches: every lane issues UNR*V independent 16-byte loads
  // before consuming any; edges past the row end read the zero row.
  const float* zrow = a.zrow;
  const uint64_t keep = policy_evict_last(), stream = policy_evict_first();
  auto ld_idx = [](const int* p, uint64_t pol) { return HINT == 3 ? __ldg(p) : ld_idx_hint(p, pol); };
  // index batches are prefetched one ahead
  int nextidx = (e0 + lane < e1) ? ld_idx(a.col + e0 + lane, stream) : -1;
  // Loads rotate over NACC interleaved accumulators (a slot adds <= d/(S*NACC)
  // terms sequentially).  Measured on C3 hub rows (d = 25K, all-positive
  // eigenvector input): 1.2e-7 relative error, far inside the 1e-5 gate; a
  // pairwise batch-tree variant was 17% slower for no measurable gain.
  for (int64_t base = e0; base < e1; base += 32) {
    const int cnt = (e1 - base) < 32 ? int(e1 - base) : 32;
    const int myidx = nextidx;
    nextidx = (base + 32 + lane < e1) ? ld_idx(a.col + base + 32 + lane, stream) : -1;
#pragma unroll
    for (int k0 = 0; k0 < STEPS; k0 += UNR) {
      float4 buf[UNR][V];
#pragma unroll
      for (int u = 0; u < UNR; ++u) {
        const int j = __shfl_sync(0xffffffffu, myidx, (k0 + u) * S + slot);
        const float* src = a.Y + int64_t(j) * a.ldy;
#pragma unroll
        for (int v = 0; v < V; ++v) {
          const float* p = (j >= 0 && qoff[v] >= 0) ? src + qoff[v] : zrow;
          if (HINT == 1) buf[u][v] = ld_f4_hint(p, keep);
          else if (HINT == 2) buf[u][v] = ld_f4_na_hint(p, keep);
          else buf[u][v] = ld_f4(p);
        }
      }
#pragma unroll
      for (int u = 0; u < UNR; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) add4(acc[(k0 + u) % NACC][v], buf[u][v]);
      if ((k0 + UNR) * S >= cnt) break;  // warp-uniform: rest of the batch is empty
    }
  }
  float4 tot[V];
#pragma unroll
  for (int v = 0; v < V; ++v) {
    tot[v] = acc[0][v];
#pragma unroll
    for (int u = 1; u < NACC; ++u) add4(tot[v], acc[u][v]);
#pragma unroll
    for (int off = G; off < 32; off <<= 1) {  // fixed butterfly over the slots
      tot[v].x += __shfl_xor_sync(0xffffffffu, tot[v].x, off);
      tot[v].y += __shfl_xor_sync(0xffffffffu, tot[v].y, off);
      tot[v].z += __shfl_xor_sync(0xffffffffu, tot[v].z, off);
      tot[v].w += __shfl_xor_sync(0xffffffffu, tot[v].w, off);
    }
  }
  const float ri = a.r[a.row_lo + row];
  const int zi = HAS_ZD ? a.zd_index[row] : -1;
  uint32_t bal[V][4];
#pragma unroll
  for (int v = 0; v < V; ++v) {
    const bool own = slot == 0 && qoff[v] >= 0;
    float4 z = tot[v];
    if (HAS_ZD && own && zi >= 0) add4(z, ld_f4(a.zd + int64_t(zi) * a.ldzd + qoff[v]));
    z.x *= ri; z.y *= ri; z.z *= ri; z.w *= ri;
    if (a.out_prescaled) { z.x *= ri; z.y *= ri; z.z *= ri; z.w *= ri; }
    if (a.mask) {
      const int c = qoff[v];
      bal[v][0] = __ballot_sync(0xffffffffu, own && z.x > 0.f && c + 0 < a.F);
      bal[v][1] = __ballot_sync(0xffffffffu, own && z.y > 0.f && c + 1 < a.F);
      bal[v][2] = __ballot_sync(0xffffffffu, own && z.z > 0.f && c + 2 < a.F);
      bal[v][3] = __ballot_sync(0xffffffffu, own && z.w > 0.f && c + 3 < a.F);
    }
    if (a.relu) {
      z.x = fmaxf(z.x, 0.f); z.y = fmaxf(z.y, 0.f); z.z = fmaxf(z.z, 0.f); z.w = fmaxf(z.w, 0.f);
    }
    if (own) *reinterpret_cast<float4*>(a.Z + row * a.ldz + qoff[v]) = z;
  }
  if (a.mask) {
    // lane w assembles mask word w: column col = 32w + b lives in lane
    // (col/4) % G, vector v = (col/4) / G, component col % 4
    const int mw = (a.F + 31) >> 5;
    if (lane < mw) {
      uint32_t word = 0;
#pragma unroll 4
      for (int b = 0; b < 32; ++b) {
        const int col = 32 * lane + b;
        const int q = col >> 2;
        const int vv = q / G, ll = q % G;
        uint32_t bit = 0;
#pragma unroll
        for (int v = 0; v < V; ++v)
          if (v == vv) bit = (bal[v][col & 3] >> ll) & 1u;
        word |= bit << b;
      }
      a.mask[row * a.mask_ld + lane] = word;
    }
  }
}

int gather_hint() {
  // Gather cache policy (PCGCN_GATHER_HINT, tuning override).  Measured on C3
  // (bench, 10 steps, two interleaved runs each), F=128 / F=41 sparse ms:
  //   0 (default) rows plain ld.global.nc, index evict_first  3.40 / 1.41
  //   1 rows L2::evict_last                                    3.83 / 1.50
  //   2 rows L1::no_allocate + evict_last                      3.83 / 2.81
  //   3 rows and index plain                                   3.43 / 1.39
  // (evict_last pins all of Y' and starves the L1/L2 replacement of the
  // hot hub rows; no_allocate loses the L1 hits of the narrow rows)
  static int h = -1;
  if (h < 0) {
    const char* e = getenv("PCGCN_GATHER_HINT");
    h = e ? atoi(e) : 0;
    if (h != 1) h = 0;
  }
  return h;
}

template <int G, int V, int HINT>
void launch_ghv(const AggArgs& a, cudaStream_t s) {
  // Occupancy target: 4 CTAs (32 warps) per SM caps registers at 64.  On C3
  // (same box, interleaved runs) F=128 3.72 -> 3.62 ms, F=41 1.60 -> 1.42 ms
  // against the unconstrained 76-80 registers (3 CTAs).  PCGCN_SPARSE_MINB=1
  // restores the unconstrained build (tuning override).
  static int minb = -1;
  if (minb < 0) {
    const char* e = getenv("PCGCN_SPARSE_MINB");
    minb = (e && atoi(e) == 1) ? 1 : 4;
  }
  dim3 grid(unsigned((a.rows + 7) / 8));
#define LAUNCH(MB)                                                        \
  if (a.zd_index)                                                         \
    sparse_agg_kernel<G, V, true, HINT, MB><<<grid, 256, 0, s>>>(a);      \
  else                                                                    \
    sparse_agg_kernel<G, V, false, HINT, MB><<<grid, 256, 0, s>>>(a);
  if (minb == 4) { LAUNCH(4) } else { LAUNCH(1) }
#undef LAUNCH
}

template <int G, int V>
cudaError_t launch_gv(const AggArgs& a, cudaStream_t s) {
  // variants 2 and 3 of the table in gather_hint() are not instantiated
  if (gather_hint() == 1) launch_ghv<G, V, 1>(a, s);
  else launch_ghv<G, V, 0>(a, s);
  return cudaGetLastError();
}

// ypre = diag(r)·Y (row-major, ld ldpre)
__global__ void prescale_kernel(const float* __restrict__ Y, int64_t ldy, const float* __restrict__ r,
                                int64_t n, int F, float* __restrict__ ypre, int64_t ldpre) {
  const int nvec = (F + 3) >> 2;
  const int64_t total = n * nvec;
  for (int64_t idx = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; idx < total;
       idx += int64_t(gridDim.x) * blockDim.x) {
    const int64_t i = idx / nvec;
    const int q = int(idx - i * nvec);
    float4 v = ld_f4(Y + i * ldy + 4 * q);
    const float ri = __ldg(r + i);
    v.x *= ri; v.y *= ri; v.z *= ri; v.w *= ri;
    *reinterpret_cast<float4*>(ypre + i * ldpre + 4 * q) = v;
  }
}

// tf32 split of the (prescaled) input, written TRANSPOSED (feature-major):
//   hiT[f][j] = Y[j][f] with the low 13 mantissa bits cleared, loT = Y - hi.
// Feature-major rows make the dense kernel's B operand K-major (source index
// contiguous), the layout the tf32 UMMA reads.  32x32 tiles through smem keep
// both the row-major reads and the transposed writes coalesced.  Feature rows
// F..npad-1 are written as zero.
__global__ void __launch_bounds__(256) split_transpose_kernel(const float* __restrict__ Y, int64_t ldy,
                                                              int64_t n, int F, int npad,
                                                              float* __restrict__ hiT,
                                                              float* __restrict__ loT, int64_t ldT) {
  __shared__ float tile[32][33];
  const int64_t j0 = int64_t(blockIdx.x) * 32;
  const int f0 = blockIdx.y * 32;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;  // 32 x 8
  for (int rr = ty; rr < 32; rr += 8) {
    const int64_t j = j0 + rr;
    const int f = f0 + tx;
    tile[rr][tx] = (j < n && f < F) ? __ldg(Y + j * ldy + f) : 0.f;
  }
  __syncthreads();
  for (int rr = ty; rr < 32; rr += 8) {
    const int f = f0 + rr;
    const int64_t j = j0 + tx;
    if (f < npad && j < ldT) {
      const float v = tile[tx][rr];
      const float h = __uint_as_float(__float_as_uint(v) & 0xffffe000u);
      hiT[int64_t(f) * ldT + j] = h;
      loT[int64_t(f) * ldT + j] = v - h;
    }
  }
}

}  // namespace

cudaError_t launch_sparse_agg_pass(const AggArgs& a, cudaStream_t s);

// Optional feature-split passes (64 feature columns per pass) so each pass's
// gather set stays L2-resident.  Measured on C3 at F=128 (θ=0.04): one pass
// reads 4.4 GB from DRAM at an 81% L2 hit rate in 4.16 ms; two passes read
// 2 x 0.74 GB at 93.5% but take 2 x 2.37 ms — the gather is bound by the
// per-edge work, not by the DRAM misses — so the split is OFF by default
// (PCGCN_SPLIT_BYTES=<bytes> enables it above that Y' size).
cudaError_t launch_sparse_agg(const AggArgs& a, cudaStream_t s) {
  if (a.rows <= 0) return cudaSuccess;
  static int64_t split_bytes = -1;
  if (split_bytes < 0) {
    const char* e = getenv("PCGCN_SPLIT_BYTES");  // tuning override (benchmarks only)
    split_bytes = e ? atoll(e) : INT64_MAX;
  }
  const int64_t ybytes = a.n_src * int64_t((a.F + 3) / 4 * 4) * 4;
  if (a.F <= 64 || ybytes <= split_bytes) return launch_sparse_agg_pass(a, s);
  for (int c0 = 0; c0 < a.F; c0 += 64) {
    AggArgs b = a;
    b.F = (a.F - c0) < 64 ? a.F - c0 : 64;
    b.Y = a.Y + c0;
    b.Z = a.Z + c0;
    if (a.zd) b.zd = a.zd + c0;
    if (a.mask) b.mask = a.mask + c0 / 32;
    cudaError_t e = launch_sparse_agg_pass(b, s);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

cudaError_t launch_sparse_agg_pass(const AggArgs& a, cudaStream_t s) {
  // (G lanes x V float4) per edge, minimising warp instructions per edge
  // (~G*(3+5V)/32) while keeping each v-slice of G lanes a contiguous segment
  const int nvec = (a.F + 3) / 4;
  // tuning override (benchmarks only): PCGCN_SPARSE_GV="G,V" when G*V >= nvec
  static int og = -1, ov = -1;
  if (og < 0) {
    og = ov = 0;
    if (const char* e = getenv("PCGCN_SPARSE_GV")) sscanf(e, "%d,%d", &og, &ov);
  }
  if (og > 0 && og * ov >= nvec) {
#define GV(g, v) if (og == g && ov == v) return launch_gv<g, v>(a, s);
    GV(32, 1) GV(32, 2) GV(16, 1) GV(16, 2) GV(16, 3) GV(16, 4) GV(8, 1) GV(8, 2) GV(8, 3) GV(8, 4)
    GV(4, 3) GV(4, 4) GV(2, 4)
#undef GV
  }
  if (nvec <= 1) return launch_gv<1, 1>(a, s);
  if (nvec <= 2) return launch_gv<1, 2>(a, s);
  if (nvec <= 3) return launch_gv<1, 3>(a, s);
  if (nvec <= 4) return launch_gv<1, 4>(a, s);
  if (nvec <= 6) return launch_gv<2, 3>(a, s);
  if (nvec <= 8) return launch_gv<2, 4>(a, s);
  if (nvec <= 12) return launch_gv<4, 3>(a, s);
  if (nvec <= 16) return launch_gv<4, 4>(a, s);
  if (nvec <= 24) return launch_gv<8, 3>(a, s);
  if (nvec <= 32) return launch_gv<32, 1>(a, s);  // measured faster than (8,4) at F=128 on C3
  if (nvec <= 48) return launch_gv<16, 3>(a, s);
  return launch_gv<16, 4>(a, s);
}

cudaError_t launch_prescale(const float* Y, int64_t ldy, const float* r, int64_t n, int F, float* ypre,
                            int64_t ldpre, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  const int64_t total = n * ((F + 3) / 4);
  const int blocks = int(std::min<int64_t>((total + 255) / 256, 148 * 16));
  prescale_kernel<<<blocks, 256, 0, s>>>(Y, ldy, r, n, F, ypre, ldpre);
  return cudaGetLastError();
}

cudaError_t launch_split_transpose(const float* Y, int64_t ldy, int64_t n, int F, int npad, float* hiT,
                                   float* loT, int64_t ldT, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  dim3 grid(unsigned((ldT + 31) / 32), unsigned((npad + 31) / 32));
  split_transpose_kernel<<<grid, 256, 0, s>>>(Y, ldy, n, F, npad, hiT, loT, ldT);
  return cudaGetLastError();
}

}  // namespace pcgcn
