// Full-mode ("dense") aggregation on the sm_100a tensor cores.
//
// Paper: §III-B.b (L151-L153: a dense edge block is treated as fully
// connected, missing edges carry value 0, processed "sequentially instead of
// decoding the indexes"), §IV-A (L175: dense format), §IV-D (L191-L193: the
// full mode mapped onto Tensor Core MMA, with a mixed-precision policy and a
// conversion when the two modes are combined).
//
// B200 design:
//   * one CTA per 128-row destination tile (UMMA M = 128); its full-mode
//     blocks arrive as a list of 128x32 bit chunks (512 B each — 32x less HBM
//     than an fp32 dense tile);
//   * warp 0 (one lane): TMA producer — for every chunk, the 32 source rows of
//     the prescaled input's tf32 hi and lo parts (Y' = hi + lo, hi = Y' with
//     the low 13 mantissa bits cleared) land in SWIZZLE_128B/64B smem tiles
//     that are exactly the UMMA MN-major canonical layout (B operand);
//   * warps 2..5 (128 threads): expand the chunk's bits into a 128x32 tf32
//     0/1 tile in the K-major SWIZZLE_128B canonical layout (A operand);
//     A∈{0,1} is exact in tf32, so only Y is split;
//   * warp 1 (one lane): issues tcgen05.mma.kind::tf32 (M=128, N=npad, K=8)
//     4 K-steps × {hi, lo} per chunk into one fp32 TMEM accumulator and frees
//     the smem stage with tcgen05.commit -> mbarrier;
//   * after the last chunk, warps 2..5 read the accumulator with tcgen05.ld
//     and write the fp32 partial sums Zd; the selective kernel adds its sum
//     and applies r_i / ReLU (mode combine, L193).
//   Accuracy: |Y' - (hi + tf32(lo))| <= 2^-22 |Y'| per term, fp32 accumulate.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <cstdint>
#include <cstring>
#include <mutex>

#include "kernels.h"

namespace pcgcn {
namespace {

constexpr int BM = 128;      // rows per tile (UMMA M)
constexpr int BK = 32;       // source columns per chunk (4 x UMMA K=8 for tf32)
constexpr int NTHREADS = 192;

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  uint32_t addr = smem_u32(b);
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(addr),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(const CUtensorMap* map, uint64_t* bar, void* dst, int c0,
                                            int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
          smem_u32(dst)),
      "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tc_mma_tf32(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc,
                                            uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}

// UMMA shared-memory matrix descriptor (sm_100): start>>4 [0,14), LBO>>4
// [16,30), SBO>>4 [32,46), version=1 [46,48), layout type [61,64).
__device__ __forceinline__ uint64_t make_sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo,
                                               uint32_t layout) {
  uint64_t d = 0;
  d |= uint64_t((saddr >> 4) & 0x3FFFu);
  d |= uint64_t((lbo >> 4) & 0x3FFFu) << 16;
  d |= uint64_t((sbo >> 4) & 0x3FFFu) << 32;
  d |= uint64_t(1) << 46;
  d |= uint64_t(layout & 7u) << 61;
  return d;
}

// instruction descriptor, kind::tf32: D f32 [4,6), A tf32 [7,10), B tf32
// [10,13), A and B K-major (bits 15/16 = 0), N>>3 [17,23), M>>4 [24,29).
// (MN-major B reads as zeros for kind::tf32 on the B200 — measured with
// tests/cuda/tc_probe.cu — so the split input is stored feature-major.)
__host__ __device__ constexpr uint32_t make_idesc_tf32(int M, int N) {
  return (1u << 4) | (2u << 7) | (2u << 10) | (uint32_t(N >> 3) << 17) | (uint32_t(M >> 4) << 24);
}

struct SmemPlan {
  int npad, stages;
  uint32_t a_bytes, b_bytes, stage_bytes;
};

__host__ __device__ inline SmemPlan smem_plan(int npad) {
  SmemPlan s;
  s.npad = npad;
  s.a_bytes = BM * BK * 4;                       // 16 KB: 128 rows x 128 B (K-major SW128)
  s.b_bytes = npad * BK * 4;                     // per operand (hi or lo): npad rows x 128 B (K-major SW128)
  s.stage_bytes = s.a_bytes + 2 * s.b_bytes;
  int st = int((200 * 1024) / s.stage_bytes);
  s.stages = st < 2 ? 2 : (st > 6 ? 6 : st);
  return s;
}

__global__ void __launch_bounds__(NTHREADS, 1)
    dense_tc_kernel(const __grid_constant__ CUtensorMap map_hi, const __grid_constant__ CUtensorMap map_lo,
                    const int64_t* __restrict__ rt_cptr, const int32_t* __restrict__ ch_col0,
                    const uint32_t* __restrict__ bits, float* __restrict__ zd, int64_t ldzd, int npad,
                    uint32_t tmem_cols) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  const SmemPlan sp = smem_plan(npad);
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sBh = sA + sp.stages * sp.a_bytes;
  uint8_t* sBl = sBh + sp.stages * sp.b_bytes;
  uint64_t* bar = reinterpret_cast<uint64_t*>(sBl + sp.stages * sp.b_bytes);
  uint64_t* full_tma = bar;                  // [stages] TMA bytes landed
  uint64_t* full_a = bar + sp.stages;        // [stages] A tile expanded (128 arrivals)
  uint64_t* empty = bar + 2 * sp.stages;     // [stages] MMA done with the stage
  uint64_t* acc_full = bar + 3 * sp.stages;  // accumulator complete
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc_full + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t t = blockIdx.x;
  const int64_t c_begin = rt_cptr[t], c_end = rt_cptr[t + 1];
  const int nch = int(c_end - c_begin);

  if (threadIdx.x == 0) {
    for (int s = 0; s < sp.stages; ++s) {
      mbar_init(&full_tma[s], 1);
      mbar_init(&full_a[s], 128);
      mbar_init(&empty[s], 1);
    }
    mbar_init(acc_full, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(tmem_cols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // ---- TMA producer ----
      const uint32_t tx = 2u * sp.b_bytes;
      for (int i = 0; i < nch; ++i) {
        const int s = i % sp.stages;
        const uint32_t ph = uint32_t(i / sp.stages) & 1u;
        mbar_wait(&empty[s], ph ^ 1u);
        const int src0 = ch_col0[c_begin + i];
        mbar_expect_tx(&full_tma[s], tx);
        // box = 32 sources (128 B, inner) x npad features: row f of the smem
        // tile holds Y'[src0..src0+31][f] — the K-major SW128 B operand
        tma_load_2d(&map_hi, &full_tma[s], sBh + s * sp.b_bytes, src0, 0);
        tma_load_2d(&map_lo, &full_tma[s], sBl + s * sp.b_bytes, src0, 0);
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ---- MMA issuer ----
      const uint32_t idesc = make_idesc_tf32(BM, npad);
      for (int i = 0; i < nch; ++i) {
        const int s = i % sp.stages;
        const uint32_t ph = uint32_t(i / sp.stages) & 1u;
        mbar_wait(&full_tma[s], ph);
        mbar_wait(&full_a[s], ph);
        tc_fence_after();
        const uint32_t a0 = smem_u32(sA + s * sp.a_bytes);
        const uint32_t bh0 = smem_u32(sBh + s * sp.b_bytes);
        const uint32_t bl0 = smem_u32(sBl + s * sp.b_bytes);
#pragma unroll
        for (int kk = 0; kk < BK / 8; ++kk) {
          const uint64_t ad = make_sdesc(a0 + kk * 32u, 16u, 1024u, 2u);
          const uint64_t bh = make_sdesc(bh0 + kk * 32u, 16u, 1024u, 2u);
          const uint64_t bl = make_sdesc(bl0 + kk * 32u, 16u, 1024u, 2u);
          tc_mma_tf32(tmem_base, ad, bh, idesc, (i > 0 || kk > 0) ? 1u : 0u);
          tc_mma_tf32(tmem_base, ad, bl, idesc, 1u);
        }
        tc_commit(&empty[s]);
      }
      tc_commit(acc_full);
    }
  } else {
    // ---- A expander (warps 2..5), then epilogue ----
    const int m = ((warp & 3) << 5) | lane;  // tile row == TMEM lane owned by this warp
    for (int i = 0; i < nch; ++i) {
      const int s = i % sp.stages;
      const uint32_t ph = uint32_t(i / sp.stages) & 1u;
      const uint32_t w = __ldg(bits + (c_begin + i) * BM + m);
      mbar_wait(&empty[s], ph ^ 1u);
      uint8_t* rowp = sA + s * sp.a_bytes + m * 128;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        float4 v;
        v.x = (w >> (4 * j + 0)) & 1u ? 1.f : 0.f;
        v.y = (w >> (4 * j + 1)) & 1u ? 1.f : 0.f;
        v.z = (w >> (4 * j + 2)) & 1u ? 1.f : 0.f;
        v.w = (w >> (4 * j + 3)) & 1u ? 1.f : 0.f;
        *reinterpret_cast<float4*>(rowp + ((j ^ (m & 7)) << 4)) = v;
      }
      fence_proxy_async();
      mbar_arrive(&full_a[s]);
    }
    mbar_wait(acc_full, 0);
    tc_fence_after();
    float* out = zd + (t * BM + m) * ldzd;
    const uint32_t lane_addr = tmem_base + (uint32_t((warp & 3) * 32) << 16);
    for (int c0 = 0; c0 < npad; c0 += 16) {
      uint32_t r[16];
      asm volatile(
          "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
          : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
            "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]),
            "=r"(r[15])
          : "r"(lane_addr + uint32_t(c0)));
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        float4 v = make_float4(__uint_as_float(r[4 * q]), __uint_as_float(r[4 * q + 1]),
                               __uint_as_float(r[4 * q + 2]), __uint_as_float(r[4 * q + 3]));
        *reinterpret_cast<float4*>(out + c0 + 4 * q) = v;
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(tmem_cols)
                 : "memory");
  }
}

PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  return fn;
}

// feature-major split input [npad rows][ldT floats]; inner dim = n sources,
// so chunk boxes that run past n are zero-filled by the TMA unit
bool make_map(CUtensorMap* map, const float* base, int64_t n, int64_t ldT, int npad) {
  auto enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[2] = {cuuint64_t(n), cuuint64_t(npad)};
  cuuint64_t strides[1] = {cuuint64_t(ldT) * 4};
  cuuint32_t box[2] = {cuuint32_t(BK), cuuint32_t(npad)};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box,
                   estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

}  // namespace

cudaError_t launch_dense_tc(const DenseArgs& a, cudaStream_t s) {
  if (a.nrt <= 0) return cudaSuccess;
  if (a.npad % 16 != 0 || a.npad < 16 || a.npad > 256 || a.ldT % 4 != 0) return cudaErrorInvalidValue;
  const SmemPlan sp = smem_plan(a.npad);
  CUtensorMap mh, ml;
  if (!make_map(&mh, a.hiT, a.n, a.ldT, a.npad) || !make_map(&ml, a.loT, a.n, a.ldT, a.npad))
    return cudaErrorInvalidValue;
  const size_t smem = 1024 + size_t(sp.stages) * sp.stage_bytes + (3 * sp.stages + 1) * 8 + 16;
  static bool attr_done = false;
  if (!attr_done) {
    cudaError_t e = cudaFuncSetAttribute(dense_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         227 * 1024);
    if (e != cudaSuccess) return e;
    attr_done = true;
  }
  uint32_t cols = 32;
  while (cols < uint32_t(a.npad)) cols <<= 1;
  dense_tc_kernel<<<unsigned(a.nrt), NTHREADS, smem, s>>>(mh, ml, a.rt_cptr, a.ch_col0, a.bits, a.zd,
                                                          a.ldzd, a.npad, cols);
  return cudaGetLastError();
}

}  // namespace pcgcn
