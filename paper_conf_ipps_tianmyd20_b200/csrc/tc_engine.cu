// tcgen05 engine for sm_100a: one persistent, warp-specialised kernel that
// computes   D[tile] = Σ_chunks A[tile, chunk] · B[chunk]   with fp32
// accumulators in TMEM, B tiles fed by TMA and A tiles built by threads
// directly in TMEM.  Three A sources share the pipeline:
//
//  A_BITS     full-mode ("dense") aggregation — PAPER.md §III-B.b (L151-L153:
//             a dense block is treated as fully connected, missing edges carry
//             0), §IV-A (L175 dense format) and §IV-D (L191-L193: full mode on
//             Tensor Cores, mixed precision, conversion when combining).  A is
//             the 128x32 0/1 tile of a destination row tile over a 32-aligned
//             source window, shipped as 512 B of bits and expanded to tf32 in
//             TMEM; B = the window's 32 source rows of Y' = hi + lo.
//             2 MMAs per K-step (A·B_hi, A·B_lo; A∈{0,1} is exact in tf32).
//  A_ROWMAJOR transform GEMM  Y = diag(s)·X·W  (Alg. 1 a^l = h^{l-1} w^l, L114):
//             A = 128x32 tile of row-major X (TMA, SWIZZLE_128B), split by
//             the builders into tf32 hi/lo in TMEM; B = Wᵀ split hi/lo.
//             3xTF32: A_hi·B_hi + A_lo·B_hi + A_hi·B_lo.
//  A_TRANS    weight-gradient GEMM  ∇Θ = Xᵀ·G  (backward of L114; the paper
//             is silent on the backward, reading A4): A = Xᵀ tile, loaded as a
//             32-row x 128-feature box of X and transposed by the builders;
//             B = Gᵀ split hi/lo; split-K over rows into fixed slices.
//
// Roles (320 threads): warp 0 lane 0 = TMA producer, warp 1 = TMEM allocator
// + MMA issuer (the whole warp walks the schedule, one elected lane issues), warps 2..5 = A builders (thread m owns tile row
// m = TMEM lane m), warps 6..9 = epilogue (tcgen05.ld -> global), with a
// double-buffered accumulator so a tile's epilogue overlaps the next tile's
// MMAs.  Split precision: for any fp32 v, hi = v with the low 13 mantissa
// bits cleared and lo = v - hi are exact; tf32(lo) keeps 11 more bits, so
// hi + tf32(lo) = v (1 ± 2^-22).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "kernels.h"
#include "tc_common.cuh"

namespace pcgcn {
namespace {

constexpr int BM = 128;        // rows per tile (UMMA M)
constexpr int BK = 32;         // K per chunk (4 x UMMA K=8 for tf32)
constexpr int NTHREADS = 320;  // 10 warps
enum AMode { A_BITS = 0, A_ROWMAJOR = 1, A_TRANS = 2 };

using namespace tc;
// A pipeline stage holds U chunks (U > 1 only for A_BITS, where a chunk is
// small): per-stage barrier round trips, the TMEM-store wait and the MMA
// issue bookkeeping are paid once per U chunks.
struct Layout {
  int npad, stages, nacc, U, a_cols;  // a_cols: TMEM columns of one A stage (U*32, U*16 bf16x3, or 64 for hi+lo)
  uint32_t bchunk;                    // smem bytes of ONE chunk's B (all parts)
  uint32_t out_bytes;                 // A_ROWMAJOR: epilogue staging (4 warps x 32 rows x (64+4) floats)
  uint32_t raw_bytes;                 // A_TRANS + raw B: one row-major [32 x npad] D box per stage
  int gst;                            // stages per TMEM accumulation group (<= 8 chunks)
  uint32_t a_bytes, b_bytes, stage_bytes, a_load_bytes;  // b_bytes: ONE chunk of ONE operand
  uint32_t tmem_cols, a_col0;
  int accw;                           // TMEM columns of one accumulator: npad, or 3·npad when the three
                                      // bf16 parts are stacked along N (one MMA per K-step, see below)
};

// PCGCN_TC_STACK=0 (A/B knob): bf16x3 full mode with three N=npad MMAs per
// K-step instead of one N=3·npad MMA over the stacked parts
bool tc_stack_enabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("PCGCN_TC_STACK");
    v = e ? (atoi(e) != 0) : 1;
  }
  return v != 0;
}

Layout make_layout(int mode, int npad, int max_stages, int max_u, bool b_raw = false, int bfp = 0) {
  Layout L;
  // bf16x3 with npad <= 64 (F <= 64; the NPC = 64 epilogue): the window block's three parts are
  // contiguous K-major SW64 row blocks, i.e. one B operand of 3·npad rows; one
  // MMA per K-step writes A·b0 | A·b1 | A·b2 side by side in TMEM and the
  // epilogue adds the three column blocks (a third of the MMA issues)
  L.accw = (mode == A_BITS && bfp == 3 && npad <= 64 && tc_stack_enabled()) ? 3 * npad : npad;
  L.raw_bytes = (mode == A_TRANS && b_raw) ? uint32_t(npad) * BK * 4 : 0u;
  L.npad = npad;
  L.b_bytes = uint32_t(npad) * BK * 4;
  // bf16 full modes: bfp (3: BF16X3, 1: BF16X1) K-major SW64 parts of npad rows x 64 B; else hi + lo tf32 (128 B rows)
  L.bchunk = bfp ? uint32_t(bfp) * uint32_t(npad) * 64u : 2u * L.b_bytes;
  // transform GEMM outputs (N x npad rows, HBM-bound at scale) leave through a
  // shared-memory transpose so each store instruction writes whole row pieces
  L.out_bytes = (mode == A_ROWMAJOR && npad <= 128) ? 4u * 32u * (64u + 4u) * 4u : 0u;
  for (int U = (mode == A_BITS ? max_u : 1); U >= 1; U = U > 1 ? U / 2 : 0) {
    L.U = U;
    L.a_cols = mode == A_BITS ? U * (bfp ? BK / 2 : BK) : 2 * BK;
    L.a_bytes = mode == A_BITS ? uint32_t((U * BM * 4 + 1023) / 1024 * 1024) : BM * BK * 4;
    L.a_load_bytes = mode == A_BITS ? BM * 4 : BM * BK * 4;  // per chunk
    L.stage_bytes = L.a_bytes + uint32_t(U) * L.bchunk + L.raw_bytes;
    int st = int((200 * 1024 - L.out_bytes) / L.stage_bytes);
    st = st > max_stages ? max_stages : st;
    L.nacc = 2;
    while (st >= 2 && L.nacc * L.accw + st * L.a_cols > 512) {
      if (st > 2) --st;
      else if (L.nacc == 2) L.nacc = 1;
      else st = 0;
    }
    L.stages = st;
    if (st >= 2 || U == 1) break;
  }
  if (L.stages < 2) L.stages = 2;
  const uint32_t need = uint32_t(L.nacc * L.accw + L.stages * L.a_cols);
  uint32_t cols = 32;
  while (cols < need) cols <<= 1;
  L.tmem_cols = cols;
  L.a_col0 = uint32_t(L.nacc * L.accw);
  static int group_chunks = -1;  // chunks per TMEM accumulation chain (PCGCN_TC_GROUP: tuning override)
  if (group_chunks < 0) {
    const char* e = getenv("PCGCN_TC_GROUP");
    group_chunks = e ? atoi(e) : 8;
    if (group_chunks < 1) group_chunks = 1;
  }
  L.gst = group_chunks / L.U > 0 ? group_chunks / L.U : 1;  // <= 8 chunks (64-96 MMAs) per chain by default
  return L;
}

struct Work {
  // tiles
  int64_t ntiles;
  // A_BITS
  const int64_t* rt_cptr;
  const int32_t* ch_col0;
  const uint32_t* bits;
  // GEMMs: reduction extent and split
  int64_t kdim;      // A_ROWMAJOR: K (features); A_TRANS: rows (reduction)
  int64_t kslice;    // A_TRANS: rows per split (multiple of 32)
  int64_t mdim;      // rows of the output (A_ROWMAJOR: M rows; A_TRANS: K features)
  int mtiles;        // A_TRANS: ceil(mdim / 128)
  // output
  float* out;
  int64_t ldo;
  int ncols;         // columns written per output row (<= npad, multiple of 4)
  const float* rowscale;
  const uint32_t* mask;  // A_ROWMAJOR: output column c of row r kept iff bit c of mask[r*mask_ld + c/32]
  int64_t mask_ld;
  int64_t split_stride;
  int b_fused;       // B lo rows follow the hi rows in memory: one TMA box {32, 2*npad} per chunk
  int single;        // A_BITS: B hi only (bf16-rounded input), one MMA per K-step (PCGCN_DENSE_BF16X1)
  int bf3;           // A_BITS: bf16 parts of B (kind::f16; 3: PCGCN_DENSE_BF16X3, 1: BF16X1; 0: tf32), window blocks only
  const int32_t* order;  // A_BITS: tile processed at position t (nullptr: t itself)
  int* dyn;              // A_BITS: tile ticket counter (zeroed before the launch): CTAs claim positions
                         // dynamically, in order, through a smem ring (nullptr: static round robin)
  const float* bblk;     // A_BITS: source-window blocks of B (pre-swizzled); nullptr: TMA boxes
  int64_t bblk_stride;   // floats per window block
  float* wblk;       // A_ROWMAJOR: also write the output as full-mode window blocks (fused split)
  int wmode;         // 1: tf32 hi/lo (SW128, 2·npad rows), 3: bf16x3 (three SW64 parts), 4: bf16x1 (one SW64 part)
  int64_t wblk_floats, wblk_nwin;  // floats per window block; windows in the buffer
  int b_raw;         // A_TRANS: B = row-major D box; the builders split + transpose it into the
                     // K-major SWIZZLE_128B hi/lo layout in smem (no feature-major pre-split pass)
};

template <int MODE>
__device__ __forceinline__ void tile_range(const Work& w, int64_t t, int64_t& kb, int64_t& nch, int64_t& m0,
                                           int64_t& sp) {
  if (MODE == A_BITS && w.order) t = w.order[t];
  if (MODE == A_BITS) {
    kb = w.rt_cptr[t];
    nch = w.rt_cptr[t + 1] - kb;
    m0 = t * BM;
    sp = 0;
  } else if (MODE == A_ROWMAJOR) {
    kb = 0;
    nch = (w.kdim + BK - 1) / BK;
    m0 = t * BM;
    sp = 0;
  } else {
    const int64_t mt = t % w.mtiles;
    sp = t / w.mtiles;
    m0 = mt * BM;
    kb = sp * w.kslice;
    int64_t ke = kb + w.kslice < w.kdim ? kb + w.kslice : w.kdim;
    nch = ke > kb ? (ke - kb + BK - 1) / BK : 0;
  }
}

// Tile sequence of one CTA: static round robin (t = blockIdx.x + i·gridDim.x),
// or (w.dyn) positions claimed by the producer from a global ticket counter and
// passed to the MMA issuer, the builders and the epilogue through a ring of TQ
// smem slots — every role sees the same sequence; a slot is reused once all
// three consumer roles have read it (tq_empty, 3 arrivals).
constexpr int TQ = 16;

struct TileIter {
  int64_t t;       // current position
  uint32_t qi;     // ring counter
};

// consumer side: next position, or false when the sequence ends.  `bar_id` > 0:
// the role's named barrier (all its 128 threads read the slot before one
// releases it); 0 for the single-thread MMA issuer.
__device__ __forceinline__ bool tile_next(const Work& w, TileIter& it, bool first, uint64_t* tq_full,
                                          uint64_t* tq_empty, const int64_t* tq, int bar_id, bool leader) {
  if (!w.dyn) {
    it.t = first ? int64_t(blockIdx.x) : it.t + gridDim.x;
    return it.t < w.ntiles;
  }
  const uint32_t slot = it.qi % TQ, par = (it.qi / TQ) & 1u;
  mbar_wait(&tq_full[slot], par);
  it.t = *reinterpret_cast<const volatile int64_t*>(&tq[slot]);
  if (bar_id > 0) asm volatile("bar.sync %0, 128;" ::"r"(bar_id) : "memory");
  else __syncwarp();  // the MMA warp: every lane has read the slot before lane 0 releases it
  if (leader) mbar_arrive(&tq_empty[slot]);
  ++it.qi;
  return it.t >= 0;
}

// producer side: claim the next position and publish it to the ring
__device__ __forceinline__ bool tile_claim(const Work& w, TileIter& it, bool first, uint64_t* tq_full,
                                           uint64_t* tq_empty, int64_t* tq) {
  if (!w.dyn) {
    it.t = first ? int64_t(blockIdx.x) : it.t + gridDim.x;
    return it.t < w.ntiles;
  }
  const uint32_t slot = it.qi % TQ, par = (it.qi / TQ) & 1u;
  mbar_wait(&tq_empty[slot], par ^ 1u);
  int64_t t = atomicAdd(w.dyn, 1);
  if (t >= w.ntiles) t = -1;
  *reinterpret_cast<volatile int64_t*>(&tq[slot]) = t;
  mbar_arrive(&tq_full[slot]);
  ++it.qi;
  it.t = t;
  return t >= 0;
}

// NPC: register-accumulator width of the epilogue (>= npad), 0 = accumulate in the output row
template <int MODE, int NPC>
__global__ void __launch_bounds__(NTHREADS, 1)
    tc_engine_kernel(const __grid_constant__ CUtensorMap map_bhi, const __grid_constant__ CUtensorMap map_blo,
                     const __grid_constant__ CUtensorMap map_a, const Work w, const Layout L) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  float* stage_out = reinterpret_cast<float*>(smem + L.stages * L.stage_bytes);
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + L.stages * L.stage_bytes + L.out_bytes);
  uint64_t* full = bar;                     // [stages] A + B landed
  uint64_t* a_full = bar + L.stages;        // [stages] A written to TMEM (128 arrivals)
  uint64_t* empty = bar + 2 * L.stages;     // [stages] MMAs done with the stage
  uint64_t* acc_full = bar + 3 * L.stages;  // [2]
  uint64_t* acc_empty = acc_full + 2;       // [2] (128 arrivals)
  uint64_t* tq_full = acc_empty + 2;        // [TQ] tile id written by the producer
  uint64_t* tq_empty = tq_full + TQ;        // [TQ] tile id read by the 3 consumer roles
  uint64_t* bfull = tq_empty + TQ;          // [stages] A_BITS: the stage's bit tiles landed (A can be built
                                            // while the B windows are still in flight)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bfull + L.stages);
  int64_t* tq = reinterpret_cast<int64_t*>(tmem_slot + 4);  // [TQ] tile positions (-1: done)
  const int npad = L.npad;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < L.stages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&bfull[s], 1);
      mbar_init(&a_full[s], 128);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&acc_full[b], 1);
      mbar_init(&acc_empty[b], 128);
    }
    for (int q = 0; q < TQ; ++q) {
      mbar_init(&tq_full[q], 1);
      mbar_init(&tq_empty[q], 3);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(L.tmem_cols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // ---- producer ----
      int s = 0;
      uint32_t ph = 0;
      TileIter it{0, 0};
      for (bool f = true; tile_claim(w, it, f, tq_full, tq_empty, tq); f = false) {
        const int64_t t = it.t;
        int64_t kb, nch, m0, sp;
        tile_range<MODE>(w, t, kb, nch, m0, sp);
        // A_BITS: the source windows of a stage's chunks are loaded one stage
        // ahead (independent loads, consumed after the next empty-slot wait),
        // so the single producer thread never waits on a global load between
        // two bulk copies (a load per chunk in the copy loop serialised ~1000
        // cycles per chunk: the engine's cost per chunk was independent of N)
        int c0_cur[4] = {0, 0, 0, 0}, c0_nxt[4] = {0, 0, 0, 0};
        if (MODE == A_BITS) {
#pragma unroll
          for (int u = 0; u < 4; ++u)
            if (u < L.U && u < nch) c0_nxt[u] = __ldg(w.ch_col0 + kb + u);
        }
        for (int64_t i = 0; i < nch; i += L.U) {
          const int nu = int(nch - i < L.U ? nch - i : L.U);
          if (MODE == A_BITS) {
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              c0_cur[u] = c0_nxt[u];
              if (u < L.U && i + L.U + u < nch) c0_nxt[u] = __ldg(w.ch_col0 + kb + i + L.U + u);
            }
          }
          mbar_wait(&empty[s], ph ^ 1u);
          uint8_t* st = smem + s * L.stage_bytes;
          mbar_expect_tx(&full[s], uint32_t(nu) * ((MODE == A_BITS ? 0u : L.a_load_bytes) +
                                                   (w.b_raw ? L.raw_bytes
                                                            : w.bf3 ? L.bchunk : (w.single ? 1u : 2u) * L.b_bytes)));
          // the bits of a tile's chunks are contiguous: one bulk copy per stage, on its own barrier
          if (MODE == A_BITS) {
            mbar_expect_tx(&bfull[s], uint32_t(nu) * BM * 4);
            bulk_load(st, w.bits + (kb + i) * BM, uint32_t(nu) * BM * 4, &bfull[s]);
          }
          for (int u = 0; u < nu; ++u) {
            int k0;
            if (MODE == A_BITS) {
              k0 = c0_cur[u & 3];
            } else if (MODE == A_ROWMAJOR) {
              k0 = int(i * BK);
              tma_load_2d(&map_a, &full[s], st, k0, int(m0));
            } else {
              k0 = int(kb + i * BK);
              tma_load_2d(&map_a, &full[s], st, int(m0), k0);
            }
            // chunk u's B tile in smem: [hi: npad rows][lo: npad rows] x 128 B
            uint8_t* bdst = st + L.a_bytes + u * L.bchunk;
            if (MODE == A_BITS && w.bblk) {
              // the window's hi+lo (or hi, or 3 bf16 parts) rows: one contiguous, pre-swizzled block
              bulk_load(bdst, w.bblk + int64_t(k0 >> 5) * w.bblk_stride,
                        w.bf3 ? L.bchunk : (w.single ? 1u : 2u) * L.b_bytes, &full[s]);
            } else if (MODE == A_TRANS && w.b_raw) {
              // row-major D rows [k0, k0+32) x features [0, npad) (OOB columns zero-filled)
              tma_load_2d(&map_bhi, &full[s], st + L.a_bytes + 2 * L.b_bytes, 0, k0);
            } else if (w.b_fused || w.single) {
              tma_load_2d(&map_bhi, &full[s], bdst, k0, 0);  // one box {32, 2*npad}: hi rows then lo rows
            } else {
              tma_load_2d(&map_bhi, &full[s], bdst, k0, 0);
              tma_load_2d(&map_blo, &full[s], bdst + L.b_bytes, k0, 0);
            }
          }
          if (++s == L.stages) { s = 0; ph ^= 1u; }
        }
      }
    }
  } else if (warp == 1) {
    {
      // ---- MMA issuer: the whole warp walks the schedule with warp-uniform
      // operands, one elected lane issues each tcgen05.mma / commit ----
      const bool stacked = L.accw != npad;
      const uint32_t idesc = (MODE == A_BITS && w.bf3) ? idesc_bf16(BM, L.accw) : idesc_tf32(BM, npad);
      int s = 0;
      uint32_t ph = 0, gc = 0;  // gc: accumulation-group counter (shared enumeration with the epilogue)
      TileIter it{0, 0};
      for (bool f = true; tile_next(w, it, f, tq_full, tq_empty, tq, 0, lane == 0); f = false) {
        const int64_t t = it.t;
        int64_t kb, nch, m0, sp;
        tile_range<MODE>(w, t, kb, nch, m0, sp);
        const int64_t nst = (nch + L.U - 1) / L.U;
        for (int64_t g0 = 0; g0 < nst; g0 += L.gst, ++gc) {
        // one accumulation group: at most L.gst stages accumulate in TMEM before
        // the epilogue folds the partial sum into fp32 registers
        const uint32_t ab = L.nacc == 2 ? (gc & 1u) : 0u;
        const uint32_t aph = L.nacc == 2 ? ((gc >> 1) & 1u) : (gc & 1u);
        mbar_wait(&acc_empty[ab], aph ^ 1u);
        tc_fence_after();
        const uint32_t d = tmem + ab * uint32_t(L.accw);
        uint32_t acc = 0;
        const int64_t ge = (g0 + L.gst < nst ? g0 + L.gst : nst) * L.U;
        for (int64_t i = g0 * L.U; i < (ge < nch ? ge : nch); i += L.U) {
          const int nu = int(nch - i < L.U ? nch - i : L.U);
          mbar_wait(&full[s], ph);
          mbar_wait(&a_full[s], ph);
          tc_fence_after();
          const uint32_t sb = smem_u32(smem + s * L.stage_bytes + L.a_bytes);
          const uint32_t sa = tmem + L.a_col0 + uint32_t(s) * uint32_t(L.a_cols);
          for (int u = 0; u < nu; ++u) {
            if (MODE == A_BITS && w.bf3) {
              // A (0/1 as bf16, 16 TMEM columns) against the bf16 parts of the
              // window (3, or 1 for BF16X1): 2 K=16 MMAs per part, fp32 accumulation in TMEM
              const uint32_t b0 = sb + uint32_t(u) * L.bchunk;
              const uint32_t a0 = sa + uint32_t(u) * (BK / 2);
              if (stacked) {  // one N = 3·npad MMA per K-step over the stacked parts
#pragma unroll
                for (int kk = 0; kk < 2; ++kk) {
                  mma_ts_f16_w(d, a0 + kk * 8u, sdesc_kmajor_sw64(b0 + kk * 32u), idesc, acc);
                  acc = 1u;
                }
                continue;
              }
#pragma unroll
              for (int part = 0; part < 3; ++part)
#pragma unroll
                for (int kk = 0; kk < 2; ++kk) {
                  if (part >= w.bf3) break;
                  const uint64_t bd = sdesc_kmajor_sw64(b0 + uint32_t(part) * uint32_t(npad) * 64u + kk * 32u);
                  mma_ts_f16_w(d, a0 + kk * 8u, bd, idesc, acc);
                  acc = 1u;
                }
              continue;
            }
            const uint32_t bh0 = sb + uint32_t(u) * L.bchunk;
            const uint32_t bl0 = bh0 + L.b_bytes;
            const uint32_t a0 = sa + uint32_t(u) * BK;
#pragma unroll
            for (int kk = 0; kk < BK / 8; ++kk) {
              const uint64_t bh = sdesc_kmajor_sw128(bh0 + kk * 32u);
              const uint64_t bl = sdesc_kmajor_sw128(bl0 + kk * 32u);
              mma_ts_w(d, a0 + kk * 8u, bh, idesc, acc);
              if (!w.single) mma_ts_w(d, a0 + kk * 8u, bl, idesc, 1u);
              if (MODE != A_BITS) mma_ts_w(d, a0 + BK + kk * 8u, bh, idesc, 1u);
              acc = 1u;
            }
          }
          tc_commit_w(&empty[s]);
          if (++s == L.stages) { s = 0; ph ^= 1u; }
        }
        tc_commit_w(&acc_full[ab]);
        }
      }
    }
  } else if (warp < 6) {
    // ---- A builders: thread m writes row m of the A tile into TMEM ----
    const int m = ((warp & 3) << 5) | lane;
    const uint32_t lane_base = uint32_t((warp & 3) * 32) << 16;
    int s = 0;
    uint32_t ph = 0;
    TileIter it{0, 0};
    for (bool f = true; tile_next(w, it, f, tq_full, tq_empty, tq, 1, m == 0); f = false) {
      const int64_t t = it.t;
      int64_t kb, nch, m0, sp;
      tile_range<MODE>(w, t, kb, nch, m0, sp);
      for (int64_t i = 0; i < nch; i += L.U) {
        const int nu = int(nch - i < L.U ? nch - i : L.U);
        // data landed (A_BITS: the bits only); the stage and its TMEM A buffer are free
        mbar_wait(MODE == A_BITS ? &bfull[s] : &full[s], ph);
        const uint8_t* st = smem + s * L.stage_bytes;
        const uint32_t taddr = tmem + lane_base + L.a_col0 + uint32_t(s) * uint32_t(L.a_cols);
        uint32_t v[32];
        if (MODE == A_BITS && w.bf3) {
          // bf16 A: two elements per TMEM column, element 2j in the low half
          for (int u = 0; u < nu; ++u) {
            const uint32_t wd = reinterpret_cast<const uint32_t*>(st + u * BM * 4)[m];
            uint32_t h[16];
#pragma unroll
            for (int j = 0; j < 16; ++j)
              h[j] = (((wd >> (2 * j)) & 1u) ? 0x3f80u : 0u) | (((wd >> (2 * j + 1)) & 1u) ? 0x3f800000u : 0u);
            sttm16(taddr + uint32_t(u) * (BK / 2), h);
          }
        } else if (MODE == A_BITS) {
          for (int u = 0; u < nu; ++u) {
            const uint32_t wd = reinterpret_cast<const uint32_t*>(st + u * BM * 4)[m];
#pragma unroll
            for (int b = 0; b < 32; ++b) v[b] = ((wd >> b) & 1u) ? 0x3f800000u : 0u;
            sttm32(taddr + uint32_t(u) * BK, v);
          }
        } else {
          float x[32];
          if (MODE == A_ROWMAJOR) {
            // row m of a SWIZZLE_128B tile: 16-byte chunk j lives at j ^ (m & 7)
            const float4* row = reinterpret_cast<const float4*>(st + m * 128);
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              const float4 q = row[j ^ (m & 7)];
              x[4 * j] = q.x; x[4 * j + 1] = q.y; x[4 * j + 2] = q.z; x[4 * j + 3] = q.w;
            }
          } else {
            // column m of a plain [32 rows][128 features] tile
            const float* tile = reinterpret_cast<const float*>(st);
#pragma unroll
            for (int r = 0; r < 32; ++r) x[r] = tile[r * BM + m];
          }
          uint32_t lo[32];
#pragma unroll
          for (int k = 0; k < 32; ++k) {
            const uint32_t h = __float_as_uint(x[k]) & 0xffffe000u;
            v[k] = h;
            lo[k] = __float_as_uint(x[k] - __uint_as_float(h));
          }
          sttm32(taddr, v);
          sttm32(taddr + BK, lo);
          if (MODE == A_TRANS && w.b_raw && m < npad) {
            // B: thread m owns feature m; raw[k][m] (k = 32 rows of the chunk)
            // -> hi/lo rows m of the K-major SWIZZLE_128B tiles: 16-byte chunk
            // j (k = 4j..4j+3) of row m lives at m*128 + ((j ^ (m & 7)) * 16)
            const float* raw = reinterpret_cast<const float*>(st + L.a_bytes + 2 * L.b_bytes);
            uint8_t* bh = const_cast<uint8_t*>(st) + L.a_bytes;
            uint8_t* bl = bh + L.b_bytes;
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              float4 h4, l4;
              float xv[4];
#pragma unroll
              for (int e = 0; e < 4; ++e) xv[e] = raw[(4 * j + e) * npad + m];
              float hv[4], lv[4];
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                hv[e] = __uint_as_float(__float_as_uint(xv[e]) & 0xffffe000u);
                lv[e] = xv[e] - hv[e];
              }
              h4 = make_float4(hv[0], hv[1], hv[2], hv[3]);
              l4 = make_float4(lv[0], lv[1], lv[2], lv[3]);
              const uint32_t off = uint32_t(m) * 128u + uint32_t((j ^ (m & 7)) * 16);
              *reinterpret_cast<float4*>(bh + off) = h4;
              *reinterpret_cast<float4*>(bl + off) = l4;
            }
            // generic-proxy smem writes -> visible to the tensor core (async proxy)
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          }
        }
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        tc_fence_before();
        mbar_arrive(&a_full[s]);
        if (++s == L.stages) { s = 0; ph ^= 1u; }
      }
    }
  } else {
    // ---- epilogue: TMEM accumulator -> global ----
    // The tensor core's fp32 accumulation in TMEM is biased (measured: the
    // relative error grows ~linearly with the accumulation chain, 2e-4 for
    // C3 hub rows accumulating thousands of chunks); so each accumulation
    // group (<= 8 chunks) is folded into an fp32 register accumulator here
    // (round-to-nearest adds, deterministic order), or into the output row
    // for npad > 128 (NPC == 0).
    const int m = ((warp & 3) << 5) | lane;
    const uint32_t lane_base = uint32_t((warp & 3) * 32) << 16;
    uint32_t gc = 0;
    TileIter it{0, 0};
    for (bool f = true; tile_next(w, it, f, tq_full, tq_empty, tq, 2, m == 0); f = false) {
      const int64_t t = it.t;
      int64_t kb, nch, m0, sp;
      tile_range<MODE>(w, t, kb, nch, m0, sp);
      const int64_t nst = (nch + L.U - 1) / L.U;
      const int64_t ngrp = (nst + L.gst - 1) / L.gst;
      const int64_t row = m0 + m;
      const bool live = MODE == A_BITS || row < w.mdim;
      float* out = w.out + sp * w.split_stride + row * w.ldo;
      const float sc = (MODE == A_ROWMAJOR && w.rowscale && live) ? w.rowscale[row] : 1.f;
      float racc[NPC > 0 ? NPC : 1];
#pragma unroll
      for (int c = 0; c < (NPC > 0 ? NPC : 1); ++c) racc[c] = 0.f;
      for (int64_t grp = 0; grp < ngrp; ++grp, ++gc) {
        const uint32_t ab = L.nacc == 2 ? (gc & 1u) : 0u;
        mbar_wait(&acc_full[ab], L.nacc == 2 ? ((gc >> 1) & 1u) : (gc & 1u));
        tc_fence_after();
        const uint32_t src = tmem + lane_base + ab * uint32_t(L.accw);
        const bool stacked = L.accw != npad;  // add the three part blocks (A·b0 + A·b1) + A·b2
#pragma unroll
        for (int c0 = 0; c0 < (NPC > 0 ? NPC : 256); c0 += 16) {
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
            if constexpr (MODE == A_BITS && NPC > 0 && NPC <= 64) if (stacked) {
#pragma unroll
              for (int part = 1; part < 3; ++part) {
                uint32_t r2[16];
                asm volatile(
                    "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, "
                    "[%16];"
                    : "=r"(r2[0]), "=r"(r2[1]), "=r"(r2[2]), "=r"(r2[3]), "=r"(r2[4]), "=r"(r2[5]), "=r"(r2[6]),
                      "=r"(r2[7]), "=r"(r2[8]), "=r"(r2[9]), "=r"(r2[10]), "=r"(r2[11]), "=r"(r2[12]), "=r"(r2[13]),
                      "=r"(r2[14]), "=r"(r2[15])
                    : "r"(src + uint32_t(part * npad + c0)));
                asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
                for (int q = 0; q < 16; ++q) r[q] = __float_as_uint(__uint_as_float(r[q]) + __uint_as_float(r2[q]));
              }
            }
            if (NPC > 0) {
#pragma unroll
              for (int q = 0; q < 16; ++q) racc[(c0 + q) % (NPC > 0 ? NPC : 1)] += __uint_as_float(r[q]);
            } else if (live) {
#pragma unroll
              for (int q = 0; q < 16; q += 4)
                if (c0 + q < w.ncols) {
                  float4 v = make_float4(__uint_as_float(r[q]), __uint_as_float(r[q + 1]),
                                         __uint_as_float(r[q + 2]), __uint_as_float(r[q + 3]));
                  if (grp > 0) {
                    const float4 o = *reinterpret_cast<const float4*>(out + c0 + q);
                    v.x += o.x; v.y += o.y; v.z += o.z; v.w += o.w;
                  }
                  *reinterpret_cast<float4*>(out + c0 + q) = v;
                }
            }
          }
        }
        tc_fence_before();
        mbar_arrive(&acc_empty[ab]);
      }
      // (all 32 lanes take the staged path: rows past M are written to smem
      // only, never to global)
      if (live || (NPC > 0 && MODE == A_ROWMAJOR && L.out_bytes)) {
        const uint32_t* mrow = (MODE == A_ROWMAJOR && w.mask && live) ? w.mask + row * w.mask_ld : nullptr;
        // mask words in registers (loaded once per row, not once per column)
        constexpr int NMW = NPC > 0 ? (NPC + 31) / 32 : 1;
        uint32_t mwd[NMW];
#pragma unroll
        for (int i = 0; i < NMW; ++i) mwd[i] = (mrow && (NPC > 0) && 32 * i < w.ncols) ? __ldg(mrow + i) : 0xffffffffu;
        auto mk = [&](int c) {
          if (!mrow) return sc;
          const uint32_t wd = NPC > 0 ? mwd[(c >> 5) % NMW] : __ldg(mrow + (c >> 5));
          return ((wd >> (c & 31)) & 1u) ? sc : 0.f;
        };
        if (NPC > 0 && MODE == A_ROWMAJOR && L.out_bytes) {
          // staged store: each thread holds one row; 64-column halves go
          // through this warp's [32 rows][68] smem tile and leave as two rows
          // of 16 float4 per store instruction (whole 256-byte row pieces)
          float* sb = stage_out + (warp & 3) * 32 * 68;
          const int64_t rbase = m0 + ((warp & 3) << 5);
#pragma unroll
          for (int h = 0; h < (NPC > 0 ? NPC : 1); h += 64) {
#pragma unroll
            for (int c = 0; c < 64; c += 4)
              if (h + c < (NPC > 0 ? NPC : 1))
                *reinterpret_cast<float4*>(sb + lane * 68 + c) =
                    make_float4(racc[h + c] * mk(h + c), racc[h + c + 1] * mk(h + c + 1),
                                racc[h + c + 2] * mk(h + c + 2), racc[h + c + 3] * mk(h + c + 3));
            __syncwarp();
            const int q = lane & 15;
#pragma unroll 4
            for (int r = 0; r < 32; r += 2) {
              const int rr = r + (lane >> 4);
              const int64_t grow = rbase + rr;
              if (grow < w.mdim && h + 4 * q < w.ncols)
                *reinterpret_cast<float4*>(w.out + grow * w.ldo + h + 4 * q) =
                    *reinterpret_cast<const float4*>(sb + rr * 68 + 4 * q);
            }
            if (w.wblk) {
              // fused split: this warp's 32 rows are one source
              // window and the smem tile holds them transposed-ready: lane l
              // takes features h+l and h+32+l, reads the 32 sources of each
              // from a column of the tile, and writes them in the full mode's
              // pre-swizzled window-block image — the bits split_window_kernel
              // would write, so the aggregation sees identical input
              const int64_t win = (m0 >> 5) + (warp & 3);
              if (win < w.wblk_nwin) {
                float* blk = w.wblk + win * w.wblk_floats;
#pragma unroll
                for (int fh = 0; fh < 64; fh += 32) {
                  const int f = h + fh + lane;
                  if (f >= npad) continue;
                  if (w.wmode >= 3) {
                    uint16_t* b16 = reinterpret_cast<uint16_t*>(blk);
#pragma unroll
                    for (int j = 0; j < 4; ++j) {  // sources 8j..8j+7: one 16-byte chunk per part
                      uint32_t p0[4], p1[4], p2[4];
#pragma unroll
                      for (int e = 0; e < 8; e += 2) {
                        uint32_t hh[2][3];
#pragma unroll
                        for (int t = 0; t < 2; ++t) {
                          const float v = sb[(8 * j + e + t) * 68 + fh + lane];
                          const uint32_t u0 = __float_as_uint(v);
                          const uint32_t h0 = (u0 + 0x7fffu + ((u0 >> 16) & 1u)) & 0xffff0000u;
                          const float r1 = v - __uint_as_float(h0);
                          const uint32_t u1 = __float_as_uint(r1);
                          const uint32_t h1 = (u1 + 0x7fffu + ((u1 >> 16) & 1u)) & 0xffff0000u;
                          const uint32_t u2 = __float_as_uint(r1 - __uint_as_float(h1));
                          hh[t][0] = h0 >> 16;
                          hh[t][1] = h1 >> 16;
                          hh[t][2] = ((u2 + 0x7fffu + ((u2 >> 16) & 1u)) & 0xffff0000u) >> 16;
                        }
                        p0[e / 2] = hh[0][0] | (hh[1][0] << 16);
                        p1[e / 2] = hh[0][1] | (hh[1][1] << 16);
                        p2[e / 2] = hh[0][2] | (hh[1][2] << 16);
                      }
                      const int pos = f * 32 + ((j ^ ((f >> 1) & 3)) << 3);
                      *reinterpret_cast<uint4*>(b16 + pos) = make_uint4(p0[0], p0[1], p0[2], p0[3]);
                      if (w.wmode == 3) {
                        *reinterpret_cast<uint4*>(b16 + npad * 32 + pos) = make_uint4(p1[0], p1[1], p1[2], p1[3]);
                        *reinterpret_cast<uint4*>(b16 + 2 * npad * 32 + pos) = make_uint4(p2[0], p2[1], p2[2], p2[3]);
                      }
                    }
                  } else {
#pragma unroll
                    for (int j = 0; j < 8; ++j) {  // sources 4j..4j+3: one 16-byte chunk
                      float4 hv, lv;
                      float* hp = &hv.x;
                      float* lp = &lv.x;
#pragma unroll
                      for (int e = 0; e < 4; ++e) {
                        const float v = sb[(4 * j + e) * 68 + fh + lane];
                        if (w.wmode == 1) {
                          hp[e] = __uint_as_float(__float_as_uint(v) & 0xffffe000u);
                          lp[e] = v - hp[e];
                        } else {
                          const uint32_t u = __float_as_uint(v);
                          hp[e] = __uint_as_float((u + 0x7fffu + ((u >> 16) & 1u)) & 0xffff0000u);
                        }
                      }
                      const int rh = f, rl = npad + f;
                      *reinterpret_cast<float4*>(blk + rh * 32 + ((j ^ (rh & 7)) << 2)) = hv;
                      if (w.wmode == 1) *reinterpret_cast<float4*>(blk + rl * 32 + ((j ^ (rl & 7)) << 2)) = lv;
                    }
                  }
                }
              }
            }
            __syncwarp();
          }
        } else if (NPC > 0) {
#pragma unroll
          for (int c0 = 0; c0 < (NPC > 0 ? NPC : 1); c0 += 4)
            if (c0 < w.ncols)
              *reinterpret_cast<float4*>(out + c0) =
                  make_float4(racc[c0] * mk(c0), racc[c0 + 1] * mk(c0 + 1), racc[c0 + 2] * mk(c0 + 2),
                              racc[c0 + 3] * mk(c0 + 3));
        } else {
          for (int c0 = 0; c0 < w.ncols; c0 += 4) {
            float4 v = ngrp > 0 ? *reinterpret_cast<const float4*>(out + c0) : make_float4(0.f, 0.f, 0.f, 0.f);
            v.x *= mk(c0); v.y *= mk(c0 + 1); v.z *= mk(c0 + 2); v.w *= mk(c0 + 3);
            *reinterpret_cast<float4*>(out + c0) = v;
          }
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(L.tmem_cols)
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

// 2-D fp32 tensor map: inner extent d0 (contiguous), outer d1, row pitch ld floats
bool make_map(CUtensorMap* map, const float* base, int64_t d0, int64_t d1, int64_t ld, int box0, int box1,
              bool swz128) {
  auto enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[2] = {cuuint64_t(d0), cuuint64_t(d1)};
  cuuint64_t strides[1] = {cuuint64_t(ld) * 4};
  cuuint32_t box[2] = {cuuint32_t(box0), cuuint32_t(box1)};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE,
                   swz128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

int num_sms() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
  }
  return sms;
}

int max_stages_env() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("PCGCN_TC_STAGES");  // tuning override (benchmarks only)
    v = e ? atoi(e) : 8;
    if (v < 2) v = 2;
    if (v > 12) v = 12;
  }
  return v;
}

// B operand maps over a feature-major split [npad rows hi][npad rows lo]: when
// lo directly follows hi and 2*npad fits one box, a single map/box covers both
bool make_b_maps(const float* hi, const float* lo, int64_t d0, int64_t ld, int npad, CUtensorMap* mh,
                 CUtensorMap* ml, int* fused) {
  *fused = (lo == hi + int64_t(npad) * ld && 2 * npad <= 256) ? 1 : 0;
  if (*fused) {
    *ml = CUtensorMap{};
    return make_map(mh, hi, d0, 2 * npad, ld, BK, 2 * npad, true);
  }
  return make_map(mh, hi, d0, npad, ld, BK, npad, true) && make_map(ml, lo, d0, npad, ld, BK, npad, true);
}

int max_u_env() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("PCGCN_TC_U");  // tuning override (benchmarks only)
    v = e ? atoi(e) : 4;
    v = v >= 4 ? 4 : (v >= 2 ? 2 : 1);
  }
  return v;
}

template <int MODE>
cudaError_t launch_engine(const CUtensorMap& bhi, const CUtensorMap& blo, const CUtensorMap& amap, const Work& w,
                          int npad, cudaStream_t s) {
  if (w.ntiles <= 0) return cudaSuccess;
  const Layout L = make_layout(MODE, npad, max_stages_env(), max_u_env(), w.b_raw != 0, w.bf3);
  const size_t smem = 1024 + size_t(L.stages) * L.stage_bytes + L.out_bytes + (4 * L.stages + 4 + 2 * TQ) * 8 + 16 +
                     TQ * 8;
  if (smem > 227 * 1024) return cudaErrorInvalidValue;
  static int grid_cap = -1;  // PCGCN_TC_GRID: full-mode CTAs (tuning override, benchmarks only)
  if (grid_cap < 0) {
    const char* e = getenv("PCGCN_TC_GRID");
    grid_cap = e ? atoi(e) : 0;
  }
  int64_t grid = w.ntiles < num_sms() ? w.ntiles : num_sms();
  if (MODE == A_BITS && grid_cap > 0 && grid > grid_cap) grid = grid_cap;
  auto go = [&](auto kernel, bool& attr_done) -> cudaError_t {
    if (!attr_done) {
      cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
      if (e != cudaSuccess) return e;
      attr_done = true;
    }
    kernel<<<unsigned(grid), NTHREADS, smem, s>>>(bhi, blo, amap, w, L);
    return cudaGetLastError();
  };
  static bool a32 = false, a64 = false, a128 = false, a0 = false;
  if (npad <= 32) return go(tc_engine_kernel<MODE, 32>, a32);
  if (npad <= 64) return go(tc_engine_kernel<MODE, 64>, a64);
  if (npad <= 128) return go(tc_engine_kernel<MODE, 128>, a128);
  return go(tc_engine_kernel<MODE, 0>, a0);
}

}  // namespace

// ---- full-mode aggregation ----
cudaError_t launch_dense_tc(const DenseArgs& a, cudaStream_t s) {
  if (a.nrt <= 0) return cudaSuccess;
  if (a.npad % 16 != 0 || a.npad < 16 || a.npad > 256 || a.ldT % 4 != 0) return cudaErrorInvalidValue;
  CUtensorMap mh, ml;
  if (a.blk) {
    // window blocks: B arrives by bulk copies (no tensor maps)
    Work w{};
    w.bblk = a.blk;
    w.bblk_stride = a.blk_floats;
    w.order = a.rt_order;
    w.single = (a.loT || a.bf3) ? 0 : 1;
    w.bf3 = a.bf3;
    w.dyn = a.dyn;
    w.ntiles = a.nrt;
    w.rt_cptr = a.rt_cptr;
    w.ch_col0 = a.ch_col0;
    w.bits = a.bits;
    w.out = a.zd;
    w.ldo = a.ldzd;
    w.ncols = a.npad;
    mh = CUtensorMap{};
    return launch_engine<A_BITS>(mh, mh, mh, w, a.npad, s);
  }
  if (dense_pair_eligible(a.npad) && a.loT == a.hiT + int64_t(a.npad) * a.ldT) {
    // CTA-pair kernel (tc_pair.cu): one map over [hi rows; lo rows], box = half the features
    if (!make_map(&mh, a.hiT, a.n, 2 * a.npad, a.ldT, BK, a.npad / 2, true)) return cudaErrorInvalidValue;
    return launch_dense_pair(a, mh, s);
  }
  int fused = 0;
  Work w{};
  if (a.loT) {
    if (!make_b_maps(a.hiT, a.loT, a.n, a.ldT, a.npad, &mh, &ml, &fused)) return cudaErrorInvalidValue;
  } else {  // BF16X1: hi rows only
    if (!make_map(&mh, a.hiT, a.n, a.npad, a.ldT, BK, a.npad, true)) return cudaErrorInvalidValue;
    ml = mh;
    w.single = 1;
  }
  w.b_fused = fused;
  w.ntiles = a.nrt;
  w.rt_cptr = a.rt_cptr;
  w.ch_col0 = a.ch_col0;
  w.bits = a.bits;
  w.out = a.zd;
  w.ldo = a.ldzd;
  w.ncols = a.npad;
  return launch_engine<A_BITS>(mh, ml, mh, w, a.npad, s);
}

// ---- Y = diag(s)·X·W, W pre-split feature-major (wT hi/lo [npad][ldwT]) ----
cudaError_t launch_tc_gemm_xw(const float* X, int64_t ldx, const float* wThi, const float* wTlo, int64_t ldwT,
                              const float* rs, float* Y, int64_t ldy, int64_t M, int K, int N, cudaStream_t s,
                              const uint32_t* mask, int64_t mask_ld, const WindowOut* wo) {
  const int npad = (N + 15) / 16 * 16;
  if (ldx % 4 || ldwT % 4 || ldy % 4 || npad > 256) return cudaErrorInvalidValue;
  CUtensorMap mh, ml, ma;
  int fused = 0;
  if (!make_b_maps(wThi, wTlo, K, ldwT, npad, &mh, &ml, &fused) || !make_map(&ma, X, K, M, ldx, BK, BM, true))
    return cudaErrorInvalidValue;
  Work w{};
  w.b_fused = fused;
  w.ntiles = (M + BM - 1) / BM;
  w.kdim = K;
  w.mdim = M;
  w.out = Y;
  w.ldo = ldy;
  w.ncols = int(ldy < npad ? ldy : npad);
  w.rowscale = rs;
  w.mask = mask;
  w.mask_ld = mask_ld;
  if (wo && wo->blk) {
    if (npad > 128 || ldy < N) return cudaErrorInvalidValue;  // fused split: staged epilogue path only
    w.wblk = wo->blk;
    w.wmode = wo->mode;
    w.wblk_floats = wo->blk_floats;
    w.wblk_nwin = wo->nwin;
  }
  return launch_engine<A_ROWMAJOR>(mh, ml, ma, w, npad, s);
}

// ---- partial[sp] = X[rows of slice sp]ᵀ · D, D pre-split feature-major ----
int64_t tc_xtg_slices(int64_t M, int K) {
  // split-K over rows so that (output row tiles) x (slices) fills the 148
  // SMs of a B200 in one wave (a constant, not the queried SM count: the
  // slicing fixes the summation order, which must not depend on the device),
  // with >= 1024 rows per slice
  const int64_t mt = (K + BM - 1) / BM;
  int64_t sl = 148 / mt;
  const int64_t cap = (M + 1023) / 1024;
  sl = sl < cap ? sl : cap;
  return sl < 1 ? 1 : (sl > 148 ? 148 : sl);
}
// ---- partial[sp] = X[rows of slice sp]ᵀ · D with D row-major (ld ldd, N <= 128):
//      B converted in the kernel (no split pass; D read once from HBM) ----
cudaError_t launch_tc_gemm_xtg_raw(const float* X, int64_t ldx, const float* D, int64_t ldd, float* partial,
                                   int64_t M, int K, int N, cudaStream_t s) {
  const int npad = (N + 15) / 16 * 16;
  if (ldx % 4 || ldd % 4 || npad > 128) return cudaErrorInvalidValue;
  CUtensorMap mr, ma;
  // D as a [M x N] tensor (row pitch ldd): the box {npad, 32} zero-fills columns >= N
  if (!make_map(&mr, D, N, M, ldd, npad, BK, false) || !make_map(&ma, X, K, M, ldx, BM, BK, false))
    return cudaErrorInvalidValue;
  const int64_t ns = tc_xtg_slices(M, K);
  Work w{};
  w.mtiles = (K + BM - 1) / BM;
  w.ntiles = int64_t(w.mtiles) * ns;
  w.kdim = M;
  w.kslice = ((M + ns - 1) / ns + BK - 1) / BK * BK;
  w.mdim = K;
  w.out = partial;
  w.ldo = npad;
  w.ncols = npad;
  w.split_stride = int64_t(K) * npad;
  w.b_raw = 1;
  return launch_engine<A_TRANS>(mr, mr, ma, w, npad, s);
}

cudaError_t launch_tc_gemm_xtg(const float* X, int64_t ldx, const float* dThi, const float* dTlo, int64_t lddT,
                               float* partial, int64_t M, int K, int N, cudaStream_t s) {
  const int npad = (N + 15) / 16 * 16;
  if (ldx % 4 || lddT % 4 || npad > 256) return cudaErrorInvalidValue;
  CUtensorMap mh, ml, ma;
  int fused = 0;
  if (!make_b_maps(dThi, dTlo, M, lddT, npad, &mh, &ml, &fused) || !make_map(&ma, X, K, M, ldx, BM, BK, false))
    return cudaErrorInvalidValue;
  const int64_t ns = tc_xtg_slices(M, K);
  Work w{};
  w.mtiles = (K + BM - 1) / BM;
  w.ntiles = int64_t(w.mtiles) * ns;
  w.kdim = M;
  w.kslice = ((M + ns - 1) / ns + BK - 1) / BK * BK;
  w.mdim = K;
  w.out = partial;
  w.ldo = npad;
  w.ncols = npad;
  w.split_stride = int64_t(K) * npad;
  w.b_fused = fused;
  return launch_engine<A_TRANS>(mh, ml, ma, w, npad, s);
}

}  // namespace pcgcn
