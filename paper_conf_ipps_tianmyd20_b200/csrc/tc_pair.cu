// Full-mode aggregation on CTA pairs (tcgen05 cta_group::2), PAPER.md
// §III-B.b / §IV-D (L151-L153, L191-L193) — the Y'-reuse variant of the
// A_BITS path of tc_engine.cu.
//
// A 2-CTA cluster owns two destination row tiles (t0 on CTA 0, t1 on CTA 1)
// and walks the UNION of their 32-aligned source windows.  For every window
// each CTA loads only HALF of the feature columns of Y' (hi and lo, N/2 rows
// of 128 B each, K-major SWIZZLE_128B) and builds the 0/1 A tile of its own
// row tile in its own TMEM (zeros where its tile lacks the window); the
// leader CTA issues tcgen05.mma.cta_group::2 with M = 256, so one MMA covers
// both tiles and each Y' window crosses L2 once per PAIR of row tiles —
// half the L2/HBM traffic of the single-CTA kernel, which is the binding
// resource of the full mode at F = 128 (DESIGN.md §6/§7).  Each CTA's TMEM
// receives its own 128 x N accumulator; accumulation groups (<= 8 windows)
// are folded into fp32 registers by each CTA's epilogue (reading #23).
//
// Cross-CTA protocol: builders and epilogue warps of both CTAs arrive on the
// leader's a_full / acc_empty barriers (mapa + mbarrier.arrive.shared::
// cluster); the leader's commits are multicast to both CTAs' empty / acc_full
// barriers.  Used when npad is a multiple of 32 (N % 32 == 0 for 2-CTA tf32).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <cstdint>
#include <cstdlib>

#include "kernels.h"
#include "tc_common.cuh"

namespace pcgcn {
namespace {

using namespace tc;
constexpr int BM = 128;
constexpr int BK = 32;
constexpr int NTHREADS = 320;
constexpr int UMAX = 4;

__device__ __forceinline__ uint32_t cta_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t mapa_cta(uint32_t addr, uint32_t cta) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(cta));
  return r;
}
__device__ __forceinline__ void arrive_cluster(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void mma2_ts(uint32_t d, uint32_t a, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::2.kind::tf32 [%0], [%1], %2, %3, p;\n"
      "}\n" ::"r"(d),
      "r"(a), "l"(bdesc), "r"(idesc), "r"(acc)
      : "memory");
}
__device__ __forceinline__ void commit2_mc(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"(uint16_t(3))
      : "memory");
}

struct PairLayout {
  int npad, stages, U, gst;
  uint32_t bh_bytes, a_bytes, stage_bytes, tmem_cols, a_col0, a_cols;
};

PairLayout make_pair_layout(int npad) {
  PairLayout L;
  L.npad = npad;
  static int u_env = -1;  // PCGCN_PAIR_U: windows per stage (tuning override)
  if (u_env < 0) {
    const char* e = getenv("PCGCN_PAIR_U");
    u_env = e ? atoi(e) : 2;
    u_env = u_env >= 4 ? 4 : (u_env >= 2 ? 2 : 1);
  }
  L.U = u_env;
  L.a_cols = L.U * BK;
  L.bh_bytes = uint32_t(npad / 2) * BK * 4;  // half the features of one window, one operand (hi or lo)
  L.a_bytes = 2048 + 1024;                   // bits of U windows (U*512 <= 2048) + per-stage metadata
  L.stage_bytes = L.a_bytes + 2 * uint32_t(L.U) * L.bh_bytes;
  int st = int((200 * 1024) / L.stage_bytes);
  if (st > 8) st = 8;
  while (st > 2 && 2 * npad + st * L.a_cols > 512) --st;
  L.stages = st;
  const uint32_t need = uint32_t(2 * npad + L.stages * L.a_cols);
  uint32_t cols = 32;
  while (cols < need) cols <<= 1;
  L.tmem_cols = cols;
  L.a_col0 = uint32_t(2 * npad);
  L.gst = 8 / L.U > 0 ? 8 / L.U : 1;
  return L;
}

// Two-pointer walk of the union of two sorted chunk lists (by window col0).
struct UnionWalk {
  int64_t a, ae, b, be;
  __device__ void init(const int64_t* cptr, int64_t t0, int64_t t1, int64_t nrt) {
    a = cptr[t0];
    ae = cptr[t0 + 1];
    if (t1 < nrt) { b = cptr[t1]; be = cptr[t1 + 1]; } else { b = be = 0; }
  }
  __device__ bool done() const { return a >= ae && b >= be; }
  // returns col0; ia/ib = chunk index of tile 0 / tile 1 or -1
  __device__ int next(const int32_t* col0, int64_t& ia, int64_t& ib) {
    const int ca = a < ae ? col0[a] : 0x7fffffff;
    const int cb = b < be ? col0[b] : 0x7fffffff;
    const int c = ca < cb ? ca : cb;
    ia = (ca == c) ? a++ : -1;
    ib = (cb == c) ? b++ : -1;
    return c;
  }
  __device__ int64_t count(const int32_t* col0) {
    int64_t n = 0, ia, ib;
    while (!done()) { next(col0, ia, ib); ++n; }
    return n;
  }
};

template <int NPC>
__global__ void __launch_bounds__(NTHREADS, 1)
    tc_pair_kernel(const __grid_constant__ CUtensorMap map_b, const int64_t* __restrict__ rt_cptr,
                   const int32_t* __restrict__ ch_col0, const uint32_t* __restrict__ bits, int64_t nrt,
                   float* __restrict__ zd, int64_t ldzd, const PairLayout L) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + L.stages * L.stage_bytes);
  uint64_t* full = bar;                     // [stages] local: this CTA's B half + bits landed
  uint64_t* a_full = bar + L.stages;        // [stages] leader: A of both CTAs in TMEM (256 arrivals)
  uint64_t* empty = bar + 2 * L.stages;     // [stages] both: MMAs done with the stage (multicast commit)
  uint64_t* acc_full = bar + 3 * L.stages;  // [2] both: accumulator group ready (multicast commit)
  uint64_t* acc_empty = acc_full + 2;       // [2] leader: both epilogues drained it (256 arrivals)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acc_empty + 2);
  const int npad = L.npad;
  const uint32_t rank = cta_rank();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t npairs_grid = gridDim.x / 2;
  const int64_t pr = blockIdx.x / 2;
  const int64_t ntp = (nrt + 1) / 2;  // tile pairs

  if (threadIdx.x == 0) {
    for (int s = 0; s < L.stages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&a_full[s], 256);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&acc_full[b], 1);
      mbar_init(&acc_empty[b], 256);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(L.tmem_cols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // ---- producer (both CTAs): own half of B, own bits ----
      int s = 0;
      uint32_t ph = 0;
      for (int64_t q = pr; q < ntp; q += npairs_grid) {
        UnionWalk uw;
        uw.init(rt_cptr, 2 * q, 2 * q + 1, nrt);
        while (!uw.done()) {
          mbar_wait(&empty[s], ph ^ 1u);
          uint8_t* st = smem + s * L.stage_bytes;
          int32_t* meta = reinterpret_cast<int32_t*>(st + 2048);
          int nu = 0, npres = 0;
          int cols[UMAX];
          int64_t own[UMAX];
          while (nu < L.U && !uw.done()) {
            int64_t ia, ib;
            cols[nu] = uw.next(ch_col0, ia, ib);
            own[nu] = rank == 0 ? ia : ib;
            meta[nu] = own[nu] >= 0 ? 1 : 0;
            npres += own[nu] >= 0;
            ++nu;
          }
          meta[UMAX] = nu;
          mbar_expect_tx(&full[s], uint32_t(nu) * 2u * L.bh_bytes + uint32_t(npres) * BM * 4);
          for (int u = 0; u < nu; ++u) {
            if (own[u] >= 0) bulk_load(st + u * BM * 4, bits + own[u] * BM, BM * 4, &full[s]);
            uint8_t* bdst = st + L.a_bytes + u * 2 * L.bh_bytes;
            // rows [rank*N/2, +N/2) of hi and of lo (hi rows 0..N-1, lo rows N..2N-1 in map_b)
            tma_load_2d(&map_b, &full[s], bdst, cols[u], int(rank) * (npad / 2));
            tma_load_2d(&map_b, &full[s], bdst + L.bh_bytes, cols[u], npad + int(rank) * (npad / 2));
          }
          if (++s == L.stages) { s = 0; ph ^= 1u; }
        }
      }
    }
  } else if (warp == 1) {
    if (rank == 0 && lane == 0) {
      // ---- MMA issuer (leader only): M = 256 over both CTAs ----
      const uint32_t idesc = idesc_tf32(2 * BM, npad);
      int s = 0;
      uint32_t ph = 0, gc = 0;
      for (int64_t q = pr; q < ntp; q += npairs_grid) {
        UnionWalk uw;
        uw.init(rt_cptr, 2 * q, 2 * q + 1, nrt);
        const int64_t nwin = uw.count(ch_col0);
        const int64_t nst = (nwin + L.U - 1) / L.U;
        for (int64_t g0 = 0; g0 < nst; g0 += L.gst, ++gc) {
          const uint32_t ab = gc & 1u;
          mbar_wait(&acc_empty[ab], ((gc >> 1) & 1u) ^ 1u);
          tc_fence_after();
          const uint32_t d = tmem + ab * uint32_t(npad);
          uint32_t acc = 0;
          const int64_t g1 = g0 + L.gst < nst ? g0 + L.gst : nst;
          for (int64_t si = g0; si < g1; ++si) {
            const int nu = int((si + 1) * L.U <= nwin ? L.U : nwin - si * L.U);
            mbar_wait(&a_full[s], ph);
            tc_fence_after();
            const uint32_t sb = smem_u32(smem + s * L.stage_bytes + L.a_bytes);
            const uint32_t sa = tmem + L.a_col0 + uint32_t(s) * uint32_t(L.a_cols);
            for (int u = 0; u < nu; ++u) {
              const uint32_t bh0 = sb + uint32_t(u) * 2u * L.bh_bytes;
              const uint32_t bl0 = bh0 + L.bh_bytes;
#pragma unroll
              for (int kk = 0; kk < BK / 8; ++kk) {
                mma2_ts(d, sa + uint32_t(u) * BK + kk * 8u, sdesc_kmajor_sw128(bh0 + kk * 32u), idesc, acc);
                mma2_ts(d, sa + uint32_t(u) * BK + kk * 8u, sdesc_kmajor_sw128(bl0 + kk * 32u), idesc, 1u);
                acc = 1u;
              }
            }
            commit2_mc(&empty[s]);
            if (++s == L.stages) { s = 0; ph ^= 1u; }
          }
          commit2_mc(&acc_full[ab]);
        }
      }
    }
  } else if (warp < 6) {
    // ---- A builders (both CTAs): own tile's 0/1 rows into own TMEM ----
    const int m = ((warp & 3) << 5) | lane;
    const uint32_t lane_base = uint32_t((warp & 3) * 32) << 16;
    int s = 0;
    uint32_t ph = 0;
    for (int64_t q = pr; q < ntp; q += npairs_grid) {
      UnionWalk uw;
      uw.init(rt_cptr, 2 * q, 2 * q + 1, nrt);
      const int64_t nwin = uw.count(ch_col0);
      for (int64_t i = 0; i < nwin; i += L.U) {
        mbar_wait(&full[s], ph);
        const uint8_t* st = smem + s * L.stage_bytes;
        const int32_t* meta = reinterpret_cast<const int32_t*>(st + 2048);
        const int nu = meta[UMAX];
        const uint32_t taddr = tmem + lane_base + L.a_col0 + uint32_t(s) * uint32_t(L.a_cols);
        for (int u = 0; u < nu; ++u) {
          const uint32_t wd = meta[u] ? reinterpret_cast<const uint32_t*>(st + u * BM * 4)[m] : 0u;
          uint32_t v[32];
#pragma unroll
          for (int b = 0; b < 32; ++b) v[b] = ((wd >> b) & 1u) ? 0x3f800000u : 0u;
          sttm32(taddr + uint32_t(u) * BK, v);
        }
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        tc_fence_before();
        arrive_cluster(mapa_cta(smem_u32(&a_full[s]), 0));
        if (++s == L.stages) { s = 0; ph ^= 1u; }
      }
    }
  } else {
    // ---- epilogue (both CTAs): fold accumulation groups, write own tile ----
    const int m = ((warp & 3) << 5) | lane;
    const uint32_t lane_base = uint32_t((warp & 3) * 32) << 16;
    uint32_t gc = 0;
    for (int64_t q = pr; q < ntp; q += npairs_grid) {
      UnionWalk uw;
      uw.init(rt_cptr, 2 * q, 2 * q + 1, nrt);
      const int64_t nwin = uw.count(ch_col0);
      const int64_t nst = (nwin + L.U - 1) / L.U;
      const int64_t ngrp = (nst + L.gst - 1) / L.gst;
      const int64_t t = 2 * q + rank;
      float racc[NPC];
#pragma unroll
      for (int c = 0; c < NPC; ++c) racc[c] = 0.f;
      for (int64_t grp = 0; grp < ngrp; ++grp, ++gc) {
        const uint32_t ab = gc & 1u;
        mbar_wait(&acc_full[ab], (gc >> 1) & 1u);
        tc_fence_after();
        const uint32_t src = tmem + lane_base + ab * uint32_t(npad);
#pragma unroll
        for (int c0 = 0; c0 < NPC; c0 += 16) {
          if (c0 < npad) {
            uint32_t r[16];
            asm volatile(
                "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, "
                "[%16];"
                : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                  "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]),
                  "=r"(r[15])
                : "r"(src + uint32_t(c0)));
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
            for (int k = 0; k < 16; ++k) racc[(c0 + k) % NPC] += __uint_as_float(r[k]);
          }
        }
        tc_fence_before();
        arrive_cluster(mapa_cta(smem_u32(&acc_empty[ab]), 0));
      }
      if (t < nrt) {
        float* out = zd + (t * BM + m) * ldzd;
#pragma unroll
        for (int c0 = 0; c0 < NPC; c0 += 4)
          if (c0 < npad) *reinterpret_cast<float4*>(out + c0) = make_float4(racc[c0], racc[c0 + 1], racc[c0 + 2], racc[c0 + 3]);
      }
    }
  }
  tc_fence_before();
  cluster_sync();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(L.tmem_cols) : "memory");
  }
}

}  // namespace

// Opt-in (PCGCN_DENSE_PAIR=1): measured on C3 at F=128 / θ=0.028 the pair
// kernel is correct but slower than the single-CTA engine (1.32 vs 0.85 ms per
// forward; 0.41 vs 0.65 of tf32 peak) for U = 1, 2, 4 — the union of the two
// tiles' windows is only 4% larger, so the loss is in the cross-CTA pipeline
// (DESIGN.md §10 Next #1).
bool dense_pair_eligible(int npad) {
  static int mode = -1;
  if (mode < 0) {
    const char* e = getenv("PCGCN_DENSE_PAIR");
    mode = e ? atoi(e) : 0;
  }
  return mode != 0 && npad % 32 == 0 && npad >= 32 && npad <= 128;
}

cudaError_t launch_dense_pair(const DenseArgs& a, const CUtensorMap& map_b, cudaStream_t s) {
  if (a.nrt <= 0) return cudaSuccess;
  const PairLayout L = make_pair_layout(a.npad);
  const size_t smem = 1024 + size_t(L.stages) * L.stage_bytes + (3 * L.stages + 4) * 8 + 16;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  int64_t pairs = (a.nrt + 1) / 2;
  if (pairs > sms / 2) pairs = sms / 2;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(unsigned(2 * pairs));
  cfg.blockDim = dim3(NTHREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  auto go = [&](auto kernel, bool& done) -> cudaError_t {
    if (!done) {
      cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
      if (e != cudaSuccess) return e;
      done = true;
    }
    return cudaLaunchKernelEx(&cfg, kernel, map_b, a.rt_cptr, a.ch_col0, a.bits, a.nrt, a.zd, a.ldzd, L);
  };
  static bool d32 = false, d64 = false, d128 = false;
  if (a.npad <= 32) return go(tc_pair_kernel<32>, d32);
  if (a.npad <= 64) return go(tc_pair_kernel<64>, d64);
  return go(tc_pair_kernel<128>, d128);
}

}  // namespace pcgcn
