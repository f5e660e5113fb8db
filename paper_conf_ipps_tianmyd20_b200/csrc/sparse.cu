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
//   * one warp per destination row (persistent warps claim rows in plan order
//     from a ticket counter); the 32 lanes split into S = 32/G edge slots of
//     G lanes, G the narrowest power of two covering the row's lane vectors,
//     so one load instruction reads whole rows and touches the fewest
//     128-byte lines; a lane vector is 32 bytes (one 256-bit load) when the
//     row needs no extra padding for it, else 16 (F=128 -> G=16 x 32 B, two
//     rows per load; F=41 -> G=16 x 16 B, two rows per load);
//   * the warp loads 32 source indices with one coalesced load and broadcasts
//     them by shuffle; a row address is one 32x32->64 multiply-add; full
//     batches are unguarded and keep 8 float4 loads per lane in flight;
//   * rows longer than SEG_EDGES are cut into segments gathered by a
//     separate pass (balance, and bounded sequential sums: reading #22);
//   * edge values are not stored: Â_ij = r_i r_j, with r_j folded into the
//     producer (IN_PRESCALED) and r_i applied once in the epilogue;
//   * fused epilogue: + dense-mode partial sum Zd (mode combine, L193),
//     × r_i, optional second × r_i, ReLU and the bit-packed ReLU mask;
//   * fixed summation order (2 interleaved accumulators, then a butterfly over
//     slots, segments in order): bitwise reproducible run to run.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>

#include "kernels.h"

namespace pcgcn {
int knobs_mrow_sort();  // PCGCN_MROW_SORT (0: multi-row groups in plan order)
int knobs_seg_inline(); // PCGCN_SEG_INLINE (0: separate up-front segment pass)
int knobs_seg_ahead();  // PCGCN_SEG_AHEAD (segment window, in quarters of the resident warps' row tickets)
namespace {

__device__ __forceinline__ float4 ld_f4(const float* p) {
  return __ldg(reinterpret_cast<const float4*>(p));
}
__device__ __forceinline__ float4 ld_f4b(const char* p) {
  return __ldg(reinterpret_cast<const float4*>(p));
}
// base + j*stride as one 32x32->64 multiply-add (IMAD.WIDE.U32 with a 64-bit addend)
__device__ __forceinline__ const char* row_addr(const char* base, uint32_t j, uint32_t stride) {
  uint64_t r;
  asm("mad.wide.u32 %0, %1, %2, %3;" : "=l"(r) : "r"(j), "r"(stride), "l"(reinterpret_cast<uint64_t>(base)));
  return reinterpret_cast<const char*>(r);
}
// a source index as the gather uses it: the plan row (PEER = false), or (owner
// shard << 28) | row inside the owner's buffer (PEER: every index is decoded
// once, by the lane that loads it, and reaches the other lanes by shuffle)
template <bool PEER>
__device__ __forceinline__ int ld_col(const int* p, const AggArgs& a) {
  const int j = __ldg(p);
  if constexpr (!PEER) {
    return j;
  } else {
    int o = 0;
#pragma unroll
    for (int q = 1; q < 8; ++q) o += (q < a.peer_world && j >= a.peer_row0[q]) ? 1 : 0;
    return (o << 28) | int(j - a.peer_row0[o]);
  }
}
template <bool PEER>
__device__ __forceinline__ const char* src_row(const char* yb, uint32_t j, uint32_t rstride, const AggArgs& a) {
  if constexpr (!PEER) {
    return row_addr(yb, j, rstride);
  } else {  // yb holds this lane's byte offset inside a row
    return row_addr(a.peer_base[j >> 28] + reinterpret_cast<uintptr_t>(yb), j & 0x0fffffffu, rstride);
  }
}
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
// a += b as two packed fp32 adds (add.rn.f32x2 = SASS FADD2, sm_100+): the
// same two IEEE round-to-nearest adds per pair (bitwise equal to four FADDs)
// at half the issue slots — the gather's FADDs are most of its instructions
__device__ __forceinline__ void add2(float& ax, float& ay, float bx, float by) {
  asm("{\n\t.reg .b64 pa, pb;\n\tmov.b64 pa, {%0, %1};\n\tmov.b64 pb, {%2, %3};\n\t"
      "add.rn.f32x2 pa, pa, pb;\n\tmov.b64 {%0, %1}, pa;\n\t}"
      : "+f"(ax), "+f"(ay)
      : "f"(bx), "f"(by));
}
__device__ __forceinline__ void add4(float4& a, const float4& b) {
  add2(a.x, a.y, b.x, b.y);
  add2(a.z, a.w, b.z, b.w);
}
// one lane vector of H float4 (H = 2: one 32-byte LDG.E.ENL2.256, sm_100's
// widest load — half the load, shuffle and address instructions per gathered
// byte; needs 32-byte aligned rows)
template <int H>
__device__ __forceinline__ void ld_vec(const char* p, float4 (&o)[H]) {
  if constexpr (H == 1) {
    o[0] = ld_f4b(p);
  } else {
    asm("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=f"(o[0].x), "=f"(o[0].y), "=f"(o[0].z), "=f"(o[0].w), "=f"(o[1].x), "=f"(o[1].y), "=f"(o[1].z),
          "=f"(o[1].w)
        : "l"(p));
  }
}

// Lane layout for a feature row of nvec lane vectors (H float4 each): the
// warp's 32 lanes form S = 32/G edge slots of G lanes; lane l of a slot owns
// vectors l, l+G, ..., l+(V-1)G.  A slot's G lanes read one contiguous piece
// of the row per load, so each load instruction touches the fewest 128-byte
// lines (the L1TEX wavefront count is what bounds a gather of L2-resident rows).
// G need not be a power of two: the S = floor(32/G) slots then leave
// 32 - S·G lanes idle (they issue no loads), an index batch holds S·STEPS
// <= 32 edges, and the slots are combined by a fixed sequence of shuffles
// instead of the butterfly.  (F = 41 rows of 48 floats as six 32-byte
// vectors: G = 6, five rows per load instruction, 30 of 32 lanes busy — vs
// 11 of 16 lanes with 16-byte vectors.)
template <int G, int V, int H>
struct Lay {
  static constexpr bool POW2 = (G & (G - 1)) == 0;
  static constexpr int S = 32 / G;       // edges per warp step
  static constexpr int STEPS = 32 / S;   // steps per index batch
  static constexpr int BATCH = S * STEPS;  // edges per coalesced index load (<= 32)
  // steps whose loads are all issued before any is consumed: <= 8 float4 per
  // lane in flight for the power-of-two layouts (more costs occupancy than it
  // gains in MLP on C3); the partial-warp layouts hold up to 12 (they run at
  // 3 CTAs per SM, see sparse_row_kernel's launch bounds)
  static constexpr int UCAP = (POW2 ? 8 : 12) / (V * H);
  static constexpr int UNR = (UCAP >= 8 && STEPS % 8 == 0) ? 8
                           : (UCAP >= 6 && STEPS % 6 == 0) ? 6
                           : (UCAP >= 4 && STEPS % 4 == 0) ? 4
                           : (UCAP >= 3 && STEPS % 3 == 0) ? 3
                           : (UCAP >= 2 && STEPS % 2 == 0) ? 2 : 1;
  static constexpr int NACC = (V * H == 1 && UNR >= 2) ? 2 : 1;  // interleaved partial sums
  static constexpr int MINB = POW2 ? 4 : 3;  // resident 256-thread CTAs per SM
};

// tot[v][h] (valid in lanes < G; in every lane for power-of-two G) = sum over the n edges
// at cp[0..n) of Y'[cp[e]][cols of this lane].  yb = this lane's byte offset
// into row 0 of Y' (lanes past the row re-read column 0: same line, ignored;
// vectors v >= 1 past the row are not loaded: lok[v] false).
// Fixed order: per slot sequential over its edges in NACC interleaved sums,
// then a butterfly over the slots — bitwise reproducible.
// Index batches are loaded one ahead: `first` is this range's first batch
// (lane l: cp[l] if l < n), and the prefetch slot of the last batch loads the
// first batch of the NEXT range (cpn, nn), which is returned — so a warp
// walking rows never waits on a row's first index load.
template <int G, int V, int H, bool PEER = false>
__device__ __forceinline__ int gather_sum(const int* __restrict__ cp, int n, int first,
                                          const int* __restrict__ cpn, int nn, const char* __restrict__ yb,
                                          uint32_t rstride, const bool (&lok)[V], int lane,
                                          float4 (&tot)[V][H], const AggArgs& a) {
  using L = Lay<G, V, H>;
  constexpr int S = L::S, STEPS = L::STEPS, UNR = L::UNR, NACC = L::NACC, BATCH = L::BATCH;
  const int slot = lane / G;
  const bool active = L::POW2 || slot < S;  // idle lanes of a partial-warp layout load nothing
  float4 acc[NACC][V][H];
#pragma unroll
  for (int u = 0; u < NACC; ++u)
#pragma unroll
    for (int v = 0; v < V; ++v)
#pragma unroll
      for (int h = 0; h < H; ++h) acc[u][v][h] = make_float4(0.f, 0.f, 0.f, 0.f);
  int nextidx = first;
  if (n == 0) nextidx = lane < nn ? ld_col<PEER>(cpn + lane, a) : 0;
  for (int base = 0; base < n; base += BATCH) {
    const int cnt = (n - base) < BATCH ? n - base : BATCH;
    const int myidx = nextidx;
    // next batch, one ahead (past the end: the next range's first batch)
    nextidx = (base + BATCH + lane < n) ? ld_col<PEER>(cp + base + BATCH + lane, a)
            : (lane < nn ? ld_col<PEER>(cpn + lane, a) : 0);
    if (cnt == BATCH) {
      // full batch: unguarded, every lane keeps UNR*V*H 16-byte pieces in flight
#pragma unroll
      for (int k0 = 0; k0 < STEPS; k0 += UNR) {
        float4 buf[UNR][V][H];
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
          const uint32_t j = uint32_t(__shfl_sync(0xffffffffu, myidx, (k0 + u) * S + slot));
          const char* p = src_row<PEER>(yb, j, rstride, a);
#pragma unroll
          for (int v = 0; v < V; ++v) {
            if (active && (v == 0 || lok[v])) {
              ld_vec<H>(p + 16 * H * G * v, buf[u][v]);
            } else {
#pragma unroll
              for (int h = 0; h < H; ++h) buf[u][v][h] = make_float4(0.f, 0.f, 0.f, 0.f);
            }
          }
        }
#pragma unroll
        for (int u = 0; u < UNR; ++u)
#pragma unroll
          for (int v = 0; v < V; ++v)
#pragma unroll
            for (int h = 0; h < H; ++h) add4(acc[u % NACC][v][h], buf[u][v][h]);
      }
    } else {
      // last (partial) batch of the row: slots past the end add nothing
#pragma unroll
      for (int k0 = 0; k0 < STEPS; k0 += UNR) {
        float4 buf[UNR][V][H];
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
          const int e = (k0 + u) * S + slot;
          const uint32_t j = uint32_t(__shfl_sync(0xffffffffu, myidx, e));
          const char* p = src_row<PEER>(yb, j, rstride, a);
#pragma unroll
          for (int v = 0; v < V; ++v) {
            if (active && e < cnt && (v == 0 || lok[v])) {
              ld_vec<H>(p + 16 * H * G * v, buf[u][v]);
            } else {
#pragma unroll
              for (int h = 0; h < H; ++h) buf[u][v][h] = make_float4(0.f, 0.f, 0.f, 0.f);
            }
          }
        }
#pragma unroll
        for (int u = 0; u < UNR; ++u)
#pragma unroll
          for (int v = 0; v < V; ++v)
#pragma unroll
            for (int h = 0; h < H; ++h) add4(acc[u % NACC][v][h], buf[u][v][h]);
        if ((k0 + UNR) * S >= cnt) break;  // warp-uniform: rest of the batch is empty
      }
    }
  }
#pragma unroll
  for (int v = 0; v < V; ++v)
#pragma unroll
    for (int h = 0; h < H; ++h) {
      float4& t = tot[v][h];
      t = acc[0][v][h];
#pragma unroll
      for (int u = 1; u < NACC; ++u) add4(t, acc[u][v][h]);
      if constexpr (L::POW2) {
#pragma unroll
        for (int off = G; off < 32; off <<= 1) {  // fixed butterfly over the slots
          t.x += __shfl_xor_sync(0xffffffffu, t.x, off);
          t.y += __shfl_xor_sync(0xffffffffu, t.y, off);
          t.z += __shfl_xor_sync(0xffffffffu, t.z, off);
          t.w += __shfl_xor_sync(0xffffffffu, t.w, off);
        }
      } else {
        // slots 1..S-1 added to slot 0 in slot order (valid in lanes < G only)
        const float4 mine = t;
#pragma unroll
        for (int k = 1; k < S; ++k) {
          const int src = lane + k * G;
          t.x += __shfl_sync(0xffffffffu, mine.x, src);
          t.y += __shfl_sync(0xffffffffu, mine.y, src);
          t.z += __shfl_sync(0xffffffffu, mine.z, src);
          t.w += __shfl_sync(0xffffffffu, mine.w, src);
        }
      }
    }
  return nextidx;
}

// this lane's vector index q for vector v (lanes past the row: -1)
template <int G>
__device__ __forceinline__ int lane_col(int lane, int v, int nvec) {
  const int q = lane % G + G * v;
  return q < nvec ? q : -1;
}

// Segment pass: one warp per segment of a long row (<= SEG_EDGES edges),
// partial sums to seg_ws.
// 4-warp CTAs (8K registers): small enough to co-reside with a full-mode
// engine CTA (tc_engine, 320 threads) when the two run concurrently
template <int G, int V, int H, bool PEER>
__global__ void __launch_bounds__(128, 2 * Lay<G, V, H>::MINB) sparse_seg_kernel(AggArgs a) {
  const int64_t sg = int64_t(blockIdx.x) * 4 + (threadIdx.x >> 5);
  if (sg >= a.nseg) return;
  const int lane = threadIdx.x & 31;
  const int nvec = (a.F + 4 * H - 1) / (4 * H);
  const int nvec4 = (a.F + 3) >> 2;
  const int q0 = lane_col<G>(lane, 0, nvec);
  const char* yb = (PEER ? nullptr : reinterpret_cast<const char*>(a.Y)) + 16 * H * (q0 < 0 ? 0 : q0);
  const int64_t lo = a.seg_lo[sg], hi = a.seg_hi[sg];
  bool lok[V];
#pragma unroll
  for (int v = 0; v < V; ++v) lok[v] = lane_col<G>(lane, v, nvec) >= 0;
  float4 tot[V][H];
  const int n = int(hi - lo);
  const int first = lane < n ? ld_col<PEER>(a.col + lo + lane, a) : 0;
  gather_sum<G, V, H, PEER>(a.col + lo, n, first, nullptr, 0, yb, uint32_t(a.ldy * 4), lok, lane, tot, a);
  if (lane < G) {
#pragma unroll
    for (int v = 0; v < V; ++v) {
      const int q = lane_col<G>(lane, v, nvec);
#pragma unroll
      for (int h = 0; h < H; ++h)
        if (q >= 0 && H * q + h < nvec4)
          *reinterpret_cast<float4*>(a.seg_ws + sg * a.ldws + 4 * (H * q + h)) = tot[v][h];
    }
  }
}

// Inline long-row segments (a.seg_inline): instead of a separate
// up-front segment pass, the row pass's warps claim the segments of a long row
// from a second ticket counter when the row-ticket frontier comes near the
// row (segment s is taken once its row is within seg_ahead row tickets of the
// claiming warp's next block), so a hub's segments gather while its community
// is L2-resident.  A segment writes its partial sum, and the warp completing a
// row's LAST segment (an atomic count per row, threadfence pattern) adds the
// row's partials in segment order — the same fixed order as the two-pass
// scheme, so results are bitwise identical — and runs the row's epilogue.
// Block rows with segments are skipped by the block walk.
__device__ __forceinline__ int peek_ticket(const int* t) { return *reinterpret_cast<const volatile int*>(t); }

// Row pass: persistent warps claim destination rows in plan order from a
// ticket counter (dynamic balance without losing the partition order's L2
// locality); a row is gathered directly or, if long, summed from its
// segment partials in segment order.  Fused epilogue: + full-mode partial
// sum Zd (mode combine, L193), x r_i (optionally twice), ReLU, bit mask.
template <int G, int V, int H, bool HAS_ZD, bool HAS_SEG, bool PEER>
__global__ void __launch_bounds__(256, Lay<G, V, H>::MINB) sparse_row_kernel(AggArgs a) {
  const int lane = threadIdx.x & 31;
  const int slot = lane / G;
  const int nvec = (a.F + 4 * H - 1) / (4 * H);
  const int nvec4 = (a.F + 3) >> 2;
  int qv[V];
  bool lok[V];
#pragma unroll
  for (int v = 0; v < V; ++v) {
    qv[v] = lane_col<G>(lane, v, nvec);
    lok[v] = qv[v] >= 0;
  }
  const char* yb = (PEER ? nullptr : reinterpret_cast<const char*>(a.Y)) + 16 * H * (qv[0] < 0 ? 0 : qv[0]);
  const uint32_t rstride = uint32_t(a.ldy * 4);

  // epilogue of one row (totals valid in slot-0 lanes): + Zd, x r_i, mask, ReLU, store
  auto epilogue = [&](int64_t row, float4 (&tot)[V][H], int zi, float ri) {
    uint32_t bal[V][4];
    uint32_t mbyte[V];
#pragma unroll
    for (int v = 0; v < V; ++v) {
      mbyte[v] = 0;
#pragma unroll
      for (int h = 0; h < H; ++h) {
        const int q4 = H * qv[v] + h;  // float4 column index (valid iff qv >= 0 and q4 < nvec4)
        const bool own = slot == 0 && qv[v] >= 0 && q4 < nvec4;
        float4 z = tot[v][h];
        if (HAS_ZD && own && zi >= 0) add4(z, ld_f4(a.zd + int64_t(zi) * a.ldzd + 4 * q4));
        z.x *= ri; z.y *= ri; z.z *= ri; z.w *= ri;
        if (a.out_prescaled) { z.x *= ri; z.y *= ri; z.z *= ri; z.w *= ri; }
        if (a.mask) {
          const int c = 4 * q4;
          if constexpr (H == 1) {
            bal[v][0] = __ballot_sync(0xffffffffu, own && z.x > 0.f && c + 0 < a.F);
            bal[v][1] = __ballot_sync(0xffffffffu, own && z.y > 0.f && c + 1 < a.F);
            bal[v][2] = __ballot_sync(0xffffffffu, own && z.z > 0.f && c + 2 < a.F);
            bal[v][3] = __ballot_sync(0xffffffffu, own && z.w > 0.f && c + 3 < a.F);
          } else if (own) {  // 8 columns per lane vector = one byte of the mask row
            const uint32_t m = uint32_t(z.x > 0.f && c + 0 < a.F) | uint32_t(z.y > 0.f && c + 1 < a.F) << 1 |
                               uint32_t(z.z > 0.f && c + 2 < a.F) << 2 | uint32_t(z.w > 0.f && c + 3 < a.F) << 3;
            mbyte[v] |= m << (4 * h);
          }
        }
        if (a.relu) {
          z.x = fmaxf(z.x, 0.f); z.y = fmaxf(z.y, 0.f); z.z = fmaxf(z.z, 0.f); z.w = fmaxf(z.w, 0.f);
        }
        if (own) *reinterpret_cast<float4*>(a.Z + int64_t(row) * a.ldz + 4 * q4) = z;
      }
    }
    if (a.mask) {
      if constexpr (H == 1) {
        // lane w assembles mask word w: column col = 32w + 4k + c (k < 8) is
        // float4 q = 8w + k, held by lane q % G of vector v = q / G, component
        // c; bit q % G of bal[v][c].  The 8 q's of a word share one v (G >= 8,
        // or a single word when G < 8), so the word interleaves four bytes:
        // bit 4k + c = bit k of byte c.
        const int mw = (a.F + 31) >> 5;
        if (lane < mw) {
          const int vv = (8 * lane) / G, l0 = (8 * lane) % G;
          uint32_t word = 0;
#pragma unroll
          for (int c = 0; c < 4; ++c) {
            uint32_t x = 0;
#pragma unroll
            for (int v = 0; v < V; ++v)
              if (v == vv) x = (bal[v][c] >> l0) & 0xffu;
            x = (x | (x << 12)) & 0x000f000fu;  // spread bit k to bit 4k
            x = (x | (x << 6)) & 0x03030303u;
            x = (x | (x << 3)) & 0x11111111u;
            word |= x << c;
          }
          a.mask[int64_t(row) * a.mask_ld + lane] = word;
        }
      } else {
        // the mask row is a little-endian bitset: byte q holds columns
        // 8q..8q+7, i.e. lane vector q's bits; bytes past the row are zero
        uint8_t* mrow = reinterpret_cast<uint8_t*>(a.mask + int64_t(row) * a.mask_ld);
        if (slot == 0) {
#pragma unroll
          for (int v = 0; v < V; ++v)
            if (qv[v] >= 0) mrow[qv[v]] = uint8_t(mbyte[v]);
        }
        // zero this row's bytes past the last vector, up to the end of ITS mask
        // words (ceil(F/32) words: a column slice of PCGCN_SPARSE_FSPLIT owns only
        // its own words of a wider row)
        if (nvec + lane < 4 * ((a.F + 31) >> 5)) mrow[nvec + lane] = 0;
      }
    }
  };
  // one segment of a long row, gathered by this warp (inline segments)
  auto run_segment = [&](int sgi) {
    const int64_t lo = a.seg_lo[sgi], hi = a.seg_hi[sgi];
    const int n = int(hi - lo);
    const int first = lane < n ? ld_col<PEER>(a.col + lo + lane, a) : 0;
    float4 tot[V][H];
    gather_sum<G, V, H, PEER>(a.col + lo, n, first, nullptr, 0, yb, rstride, lok, lane, tot, a);
    const int64_t row = a.seg_row[sgi];
    const int s0 = a.row_seg[row];
    const int ns = int((a.rowptr[row + 1] - a.rowptr[row] + SEG_EDGES - 1) / SEG_EDGES);
    if (slot == 0) {
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int h = 0; h < H; ++h)
          if (qv[v] >= 0 && H * qv[v] + h < nvec4)
            __stcg(reinterpret_cast<float4*>(a.seg_ws + int64_t(sgi) * a.ldws + 4 * (H * qv[v] + h)), tot[v][h]);
    }
    __threadfence();
    __syncwarp();
    int last = 0;
    if (lane == 0) last = atomicAdd(a.seg_cnt + s0, 1) == ns - 1;
    if (__shfl_sync(0xffffffffu, last, 0)) {
      __threadfence();
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int h = 0; h < H; ++h) tot[v][h] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (slot == 0) {
        for (int k = 0; k < ns; ++k)
#pragma unroll
          for (int v = 0; v < V; ++v)
#pragma unroll
            for (int h = 0; h < H; ++h)
              if (qv[v] >= 0 && H * qv[v] + h < nvec4)
                add4(tot[v][h], __ldcg(reinterpret_cast<const float4*>(a.seg_ws + int64_t(s0 + k) * a.ldws +
                                                                        4 * (H * qv[v] + h))));
      }
      epilogue(row, tot, HAS_ZD ? a.zd_index[row] : -1, a.r[a.row_lo + row]);
      if (lane == 0) a.seg_cnt[s0] = 0;  // self-resetting for the next call
    }
  };
  const bool inl = HAS_SEG && a.seg_inline;
  // claim segments while the next unclaimed one belongs to a row before
  // `limit` (warp-uniform; limit < 0: drain every remaining segment)
  auto seg_loop = [&](int64_t limit) {
    while (true) {
      int sgi = 0;
      if (lane == 0) sgi = atomicAdd(a.seg_ticket, 1);
      sgi = __shfl_sync(0xffffffffu, sgi, 0);
      if (sgi >= a.nseg) return;
      run_segment(sgi);
      if (limit >= 0) {
        int go = 0;
        if (lane == 0) {
          const int pk = peek_ticket(a.seg_ticket);
          go = pk < a.nseg && a.seg_row[pk] < limit;
        }
        if (!__shfl_sync(0xffffffffu, go, 0)) return;
      }
    }
  };
  // Rows are claimed in blocks of R consecutive rows per ticket (R >= 4 from
  // the plan's mean selective degree: short rows would otherwise pay the
  // ticket -> rowptr -> index dependency chain per row).  The next block's
  // ticket is issued when a block starts and consumed three rows before its
  // end; its R+1 row pointers are then copied global -> shared with cp.async
  // (no registers held in flight) while those rows gather; and the first
  // index batch of the next row is always in flight while the current row
  // gathers: in steady state a row costs one gather round trip.
  __shared__ long long s_rp[8][2][32];  // per warp: this block's / the next block's row pointers
  const int wib = threadIdx.x >> 5;
  const int R = a.rows_per_ticket;
  const int nblk_total = int((a.rows + R - 1) / R);
  auto fetch_rp = [&](int blk, int b) {  // async copy of rowptr[blk*R .. blk*R+R] into s_rp[wib][b]
    if (blk < nblk_total && lane <= R) {
      const int64_t r = int64_t(blk) * R + lane;
      const long long* src = reinterpret_cast<const long long*>(a.rowptr + (r < a.rows ? r : a.rows));
      asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_addr(&s_rp[wib][b][lane])), "l"(src)
                   : "memory");
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  auto wait_rp = [&]() {
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncwarp();
  };
  int blk;
  {
    int t = 0;
    if (lane == 0) t = atomicAdd(a.counter, 1);
    blk = __shfl_sync(0xffffffffu, t, 0);
  }
  int b = 0;
  fetch_rp(blk, b);
  wait_rp();
  int pre = 0;
  if (blk < nblk_total) {
    const int64_t f0 = s_rp[wib][b][0], f1 = s_rp[wib][b][1];
    pre = (f0 + lane < f1) ? ld_col<PEER>(a.col + f0 + lane, a) : 0;
  }
  while (blk < nblk_total) {
    int tk = 0;
    if (lane == 0) tk = atomicAdd(a.counter, 1);  // next block's ticket, consumed later
    // inline segments: the next unclaimed segment (peeked now, its row read
    // three rows before the block's end, decided at the end)
    int speek = 0;
    if (inl && lane == 0) speek = peek_ticket(a.seg_ticket);
    int64_t srow = INT64_MAX;
    int nblk = nblk_total;
    const int nr = int(a.rows - int64_t(blk) * R < R ? a.rows - int64_t(blk) * R : R);
    const int ic = nr > 3 ? nr - 3 : 0;
    for (int i = 0; i < nr; ++i) {
    const int64_t row = int64_t(blk) * R + i;
    if (i == ic) {
      nblk = __shfl_sync(0xffffffffu, tk, 0);
      fetch_rp(nblk, b ^ 1);
      if (inl && lane == 0 && speek < a.nseg) srow = a.seg_row[speek];
    }
    if (i + 1 == nr) wait_rp();
    // edge ranges (re-read from shared memory, not kept live across the gather):
    // this row [e0, e1) and the next row [n0, n1) (this block's, or the next block's first)
    const int64_t e0 = s_rp[wib][b][i], e1 = s_rp[wib][b][i + 1];
    int64_t n0 = 0, n1 = 0;
    if (i + 1 < nr) {
      n0 = e1;
      n1 = s_rp[wib][b][i + 2];
    } else if (nblk < nblk_total) {
      n0 = s_rp[wib][b ^ 1][0];
      n1 = s_rp[wib][b ^ 1][1];
    }
    float4 tot[V][H];
    int pre_next;
    // the epilogue's per-row scalars are loaded before the gather (in flight with it)
    const float ri = a.r[a.row_lo + row];
    const int zi = HAS_ZD ? a.zd_index[row] : -1;
    const int sg = HAS_SEG ? a.row_seg[row] : -1;
    bool skip = false;
    if (HAS_SEG && sg >= 0) {
      pre_next = (n0 + lane < n1) ? ld_col<PEER>(a.col + n0 + lane, a) : 0;
      skip = inl;  // written by the warp that completes its last segment
      const int ns = int((e1 - e0 + SEG_EDGES - 1) / SEG_EDGES);
#pragma unroll
      for (int v = 0; v < V; ++v)
#pragma unroll
        for (int h = 0; h < H; ++h) tot[v][h] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (slot == 0 && !inl) {
        for (int k = 0; k < ns; ++k)
#pragma unroll
          for (int v = 0; v < V; ++v)
#pragma unroll
            for (int h = 0; h < H; ++h)
              if (qv[v] >= 0 && H * qv[v] + h < nvec4)
                add4(tot[v][h], __ldcg(reinterpret_cast<const float4*>(a.seg_ws + int64_t(sg + k) * a.ldws +
                                                                        4 * (H * qv[v] + h))));
      }
    } else {
      pre_next = gather_sum<G, V, H, PEER>(a.col + e0, int(e1 - e0), pre, a.col + n0, int(n1 - n0), yb, rstride,
                                           lok, lane, tot, a);
    }
    if (!skip) epilogue(row, tot, zi, ri);
    pre = pre_next;
    }
    if (inl) {
      const int64_t sr = __shfl_sync(0xffffffffu, srow, 0);
      const int64_t limit = (int64_t(nblk) + a.seg_ahead) * R;
      if (sr < limit) seg_loop(limit);
    }
    blk = nblk;
    b ^= 1;
  }
  if (inl) seg_loop(-1);  // the row stream is done: drain the remaining segments
}

// Multi-row pass for short rows (C5's mean selective degree
// 31): each of the warp's S = 32/G edge slots owns one destination row of a
// group of S consecutive plan rows, so a row costs no cross-slot reduction
// and the per-row work (row pointers, ticket, epilogue) is shared by S rows.
// A slot walks its row's edges in CSR order with one running sum (lane g
// holds columns [8g, 8g+8) as one 32-byte vector): the summation order is
// fixed, bitwise run to run.  The warp steps max(deg) over its S rows, so the
// layout wants rows of similar degree next to each other (degree vertex
// order, reading #24).  Index batches: lane g of a slot loads edge base+g of
// its row (G indices per slot per load), one batch ahead; the next group's
// row pointers and segment ids are loaded while the current group gathers,
// and its first index batch is issued by the current group's last step.
template <int G, bool HAS_ZD, bool HAS_SEG, bool PEER>
__global__ void __launch_bounds__(256, 4) sparse_mrow_kernel(AggArgs a) {
  constexpr int H = 2;
  constexpr int S = 32 / G;
  static_assert(G >= 4 && G <= 16, "multi-row layout: 2..8 slots");
  const int lane = threadIdx.x & 31;
  const int slot = lane / G, g = lane % G;
  const int nvec = (a.F + 7) >> 3;  // <= G
  const int nvec4 = (a.F + 3) >> 2;
  const bool lok = g < nvec;
  const char* yb = (PEER ? nullptr : reinterpret_cast<const char*>(a.Y)) + 32 * (lok ? g : 0);
  const uint32_t rstride = uint32_t(a.ldy * 4);
  // tickets of 32 consecutive plan rows, S-row groups inside a ticket
  const int GPT = 32 / S;
  const int64_t ntk = (a.rows + 31) / 32;
  auto ticket = [&]() {
    int t = 0;
    if (lane == 0) t = atomicAdd(a.counter, 1);
    return __shfl_sync(0xffffffffu, t, 0);
  };
  // ticket tt's row pointers and segment ids -> this warp's shared-memory
  // buffer b with cp.async (nothing held in registers while they travel)
  __shared__ long long s_rp[8][2][34];
  __shared__ int s_sg[8][2][32];
  const int wib = threadIdx.x >> 5;
  auto load_tk = [&](int tt, int b) {
    if (tt < ntk) {
      const int64_t r0 = int64_t(tt) * 32;
      for (int l = lane; l <= 32; l += 32) {
        const int64_t r = r0 + l < a.rows ? r0 + l : a.rows;
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_addr(&s_rp[wib][b][l])),
                     "l"(reinterpret_cast<const long long*>(a.rowptr + r))
                     : "memory");
      }
      if (HAS_SEG) {
        if (r0 + lane < a.rows)
          asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_addr(&s_sg[wib][b][lane])),
                       "l"(a.row_seg + r0 + lane)
                       : "memory");
        else
          s_sg[wib][b][lane] = -1;
      }
    } else {  // past the last ticket: empty rows (the lookahead reads this buffer)
      s_rp[wib][b][lane] = 0;
      if (lane == 0) s_rp[wib][b][32] = 0;
      if (HAS_SEG) s_sg[wib][b][lane] = -1;
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  auto wait_tk = [&]() {
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncwarp();
  };
  // the ticket's rows ordered by gathered degree (bitonic sort across the warp,
  // ties by row): each group of S rows then has rows of similar length, so a
  // group costs about its mean row instead of its longest (the plan order
  // stays as it is: only the 32-row window is reordered)
  const bool sort_rows = a.mrow_sort != 0;
  auto sort_tk = [&](int b) {
    if (!sort_rows) return lane;
    const bool sgd = HAS_SEG && s_sg[wib][b][lane] >= 0;
    int x = ((sgd ? 0 : int(s_rp[wib][b][lane + 1] - s_rp[wib][b][lane])) << 5) | lane;
#pragma unroll
    for (int kk = 2; kk <= 32; kk <<= 1)
#pragma unroll
      for (int j = kk >> 1; j > 0; j >>= 1) {
        const int o = __shfl_xor_sync(0xffffffffu, x, j);
        const bool asc = (lane & kk) == 0, low = (lane & j) == 0;
        x = (low == asc) ? min(x, o) : max(x, o);
      }
    return x & 31;
  };
  // group kq of the ticket in buffer b: this slot's row (index inside the ticket) and its range
  auto slot_row = [&](int kq, int perm, int b, int& idx, int64_t& e0, int64_t& e1, int& sgv) {
    idx = __shfl_sync(0xffffffffu, perm, kq * S + slot);
    e0 = s_rp[wib][b][idx];
    e1 = s_rp[wib][b][idx + 1];
    sgv = HAS_SEG ? s_sg[wib][b][idx] : -1;
    return (HAS_SEG && sgv >= 0) ? 0 : int(e1 - e0);
  };
  // epilogue of one row held by this lane's slot: + Zd, x r_i (twice if prescaled output), mask byte, ReLU
  auto epilogue = [&](int64_t row, float4 (&acc)[H], int zi, float ri) {
      uint32_t mbyte = 0;
#pragma unroll
      for (int h = 0; h < H; ++h) {
        const int q4 = H * g + h;
        const bool own = lok && q4 < nvec4;
        float4 z = acc[h];
        if (HAS_ZD && own && zi >= 0) add4(z, ld_f4(a.zd + int64_t(zi) * a.ldzd + 4 * q4));
        z.x *= ri; z.y *= ri; z.z *= ri; z.w *= ri;
        if (a.out_prescaled) { z.x *= ri; z.y *= ri; z.z *= ri; z.w *= ri; }
        const int c = 4 * q4;
        mbyte |= (uint32_t(z.x > 0.f && c + 0 < a.F) | uint32_t(z.y > 0.f && c + 1 < a.F) << 1 |
                  uint32_t(z.z > 0.f && c + 2 < a.F) << 2 | uint32_t(z.w > 0.f && c + 3 < a.F) << 3)
                 << (4 * h);
        if (a.relu) {
          z.x = fmaxf(z.x, 0.f); z.y = fmaxf(z.y, 0.f); z.z = fmaxf(z.z, 0.f); z.w = fmaxf(z.w, 0.f);
        }
        if (own) *reinterpret_cast<float4*>(a.Z + row * a.ldz + 4 * q4) = z;
      }
      if (a.mask) {  // byte g of the little-endian mask row = columns 8g..8g+7
        uint8_t* mrow = reinterpret_cast<uint8_t*>(a.mask + row * a.mask_ld);
        if (lok) mrow[g] = uint8_t(mbyte);
        if (nvec + g < 4 * ((a.F + 31) >> 5)) mrow[nvec + g] = 0;
      }
  };
  const bool inl = HAS_SEG && a.seg_inline;
  // inline segments (see sparse_row_kernel): one segment of a long row gathered
  // by the whole warp in the one-row layout (G lanes per edge slot, S slots);
  // the warp completing the row's last segment adds the partials in segment
  // order and runs the epilogue in slot 0
  auto run_segment = [&](int sgi) {
    const int64_t lo = a.seg_lo[sgi], hi = a.seg_hi[sgi];
    const int n = int(hi - lo);
    const int first = lane < n ? ld_col<PEER>(a.col + lo + lane, a) : 0;
    const bool lk[1] = {lok};
    float4 tot[1][H];
    gather_sum<G, 1, H, PEER>(a.col + lo, n, first, nullptr, 0, yb, rstride, lk, lane, tot, a);
    const int64_t row = a.seg_row[sgi];
    const int s0 = a.row_seg[row];
    const int ns = int((a.rowptr[row + 1] - a.rowptr[row] + SEG_EDGES - 1) / SEG_EDGES);
    if (slot == 0 && lok) {
#pragma unroll
      for (int h = 0; h < H; ++h)
        if (H * g + h < nvec4)
          __stcg(reinterpret_cast<float4*>(a.seg_ws + int64_t(sgi) * a.ldws + 4 * (H * g + h)), tot[0][h]);
    }
    __threadfence();
    __syncwarp();
    int last = 0;
    if (lane == 0) last = atomicAdd(a.seg_cnt + s0, 1) == ns - 1;
    if (__shfl_sync(0xffffffffu, last, 0)) {
      __threadfence();
      float4 acc[H];
#pragma unroll
      for (int h = 0; h < H; ++h) acc[h] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (slot == 0 && lok) {
        for (int k = 0; k < ns; ++k)
#pragma unroll
          for (int h = 0; h < H; ++h)
            if (H * g + h < nvec4)
              add4(acc[h], __ldcg(reinterpret_cast<const float4*>(a.seg_ws + int64_t(s0 + k) * a.ldws +
                                                                 4 * (H * g + h))));
      }
      if (slot == 0) epilogue(row, acc, HAS_ZD ? a.zd_index[row] : -1, a.r[a.row_lo + row]);
      if (lane == 0) a.seg_cnt[s0] = 0;
    }
  };
  auto seg_loop = [&](int64_t limit) {
    while (true) {
      int sgi = 0;
      if (lane == 0) sgi = atomicAdd(a.seg_ticket, 1);
      sgi = __shfl_sync(0xffffffffu, sgi, 0);
      if (sgi >= a.nseg) return;
      run_segment(sgi);
      if (limit >= 0) {
        int go = 0;
        if (lane == 0) {
          const int pk = peek_ticket(a.seg_ticket);
          go = pk < a.nseg && a.seg_row[pk] < limit;
        }
        if (!__shfl_sync(0xffffffffu, go, 0)) return;
      }
    }
  };
  int t = ticket();
  if (t >= ntk) { if (inl) seg_loop(-1); return; }
  int tn = ticket();  // the next ticket, consumed when this one ends
  int bt = 0;          // smem buffer of the current ticket
  load_tk(t, bt);
  wait_tk();
  int perm = sort_tk(bt), permn = 0;
  int kq = 0, ri_idx, sgv;
  int64_t e0, e1;
  int n = slot_row(0, perm, bt, ri_idx, e0, e1, sgv);
  int idx = g < n ? ld_col<PEER>(a.col + e0 + g, a) : 0;
  while (true) {
    const bool last = kq == GPT - 1;
    if (kq == GPT - 2) load_tk(tn, bt ^ 1);  // the next ticket's rows, in flight for a group
    if (last) {
      wait_tk();
      permn = sort_tk(bt ^ 1);
    }
    int speek = a.nseg;
    if (inl && last && lane == 0) speek = peek_ticket(a.seg_ticket);
    const int64_t row = int64_t(t) * 32 + ri_idx;
    const bool valid = row < a.rows;
    const float ri = valid ? __ldg(a.r + a.row_lo + row) : 0.f;
    const int zi = (HAS_ZD && valid) ? __ldg(a.zd_index + row) : -1;
    // the next group's row (this ticket, or the next one's first group)
    int idxn, sgn;
    int64_t e0n, e1n;
    const int nn = last ? slot_row(0, permn, bt ^ 1, idxn, e0n, e1n, sgn)
                        : slot_row(kq + 1, perm, bt, idxn, e0n, e1n, sgn);
    float4 acc[H];
#pragma unroll
    for (int h = 0; h < H; ++h) acc[h] = make_float4(0.f, 0.f, 0.f, 0.f);
    const int nmax = __reduce_max_sync(0xffffffffu, n);
    for (int base = 0; base < nmax; base += G) {
      const int cur = idx;
      if (base + G < nmax) {
        idx = (base + G + g < n) ? ld_col<PEER>(a.col + e0 + base + G + g, a) : 0;
      } else {  // last step: the next group's first batch
        idx = g < nn ? ld_col<PEER>(a.col + e0n + g, a) : 0;
      }
#pragma unroll
      for (int u0 = 0; u0 < G; u0 += 4) {
        float4 buf[4][H];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const uint32_t j = uint32_t(__shfl_sync(0xffffffffu, cur, slot * G + u0 + u));
          if (lok && base + u0 + u < n) {
            ld_vec<H>(src_row<PEER>(yb, j, rstride, a), buf[u]);
          } else {
#pragma unroll
            for (int h = 0; h < H; ++h) buf[u][h] = make_float4(0.f, 0.f, 0.f, 0.f);
          }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
          for (int h = 0; h < H; ++h) add4(acc[h], buf[u][h]);
        if (base + u0 + 4 >= nmax) break;  // warp-uniform: the rest of the batch is past every row
      }
    }
    if (nmax == 0) idx = g < nn ? ld_col<PEER>(a.col + e0n + g, a) : 0;
    if (HAS_SEG && !inl && sgv >= 0 && lok) {  // long row: its segment partials in segment order
      const int ns = int((e1 - e0 + SEG_EDGES - 1) / SEG_EDGES);
      for (int k = 0; k < ns; ++k)
#pragma unroll
        for (int h = 0; h < H; ++h)
          if (H * g + h < nvec4)
            add4(acc[h], __ldcg(reinterpret_cast<const float4*>(a.seg_ws + int64_t(sgv + k) * a.ldws +
                                                               4 * (H * g + h))));
    }
    if (valid && !(inl && sgv >= 0)) epilogue(row, acc, zi, ri);  // inline: a long row is written by its last segment
    if (last) {
      if (inl) {
        int64_t sr = INT64_MAX;
        if (lane == 0 && speek < a.nseg) sr = a.seg_row[speek];
        sr = __shfl_sync(0xffffffffu, sr, 0);
        const int64_t limit = (int64_t(tn) + a.seg_ahead) * 32;
        if (sr < limit) seg_loop(limit);
      }
      if (tn >= ntk) {
        if (inl) seg_loop(-1);
        break;
      }
      t = tn;
      tn = ticket();
      bt ^= 1;
      perm = permn;
      kq = 0;
    } else {
      ++kq;
    }
    ri_idx = idxn;
    e0 = e0n;
    e1 = e1n;
    sgv = sgn;
    n = nn;
  }
}

constexpr float MROW_MAX_DEG = 64.f;

template <int G, bool PEER>
cudaError_t launch_mrow(const AggArgs& a, cudaStream_t s) {
  static int slots = 0;
  if (!slots) {
    int dev = 0, sms = 148, per = 4;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, sparse_mrow_kernel<G, true, true, PEER>, 256, 0);
    slots = sms * (per > 0 ? per : 1);
  }
  const bool inl = a.nseg > 0 && a.phase == 0 && a.seg_row && knobs_seg_inline();
  if (a.nseg > 0 && a.phase != 2 && !inl) {
    sparse_seg_kernel<G, 1, 2, PEER><<<unsigned((a.nseg + 3) / 4), 128, 0, s>>>(a);
    if (a.phase == 1) return cudaGetLastError();
  }
  // row ticket counter[0] and (inline segments) segment ticket counter[8]
  cudaError_t e = cudaMemsetAsync(a.counter, 0, (inl ? 9 : 1) * sizeof(int), s);
  if (e != cudaSuccess) return e;
  AggArgs b = a;
  b.mrow_sort = knobs_mrow_sort();
  const int64_t ntk = (a.rows + 31) / 32;  // tickets of 32 rows
  const int64_t want = (ntk + 7) / 8;
  const unsigned grid = unsigned(want < slots ? want : slots);
  b.seg_inline = inl ? 1 : 0;
  b.seg_ahead = int64_t(grid) * 8 * knobs_seg_ahead() / 4;
  const bool zd = a.zd_index != nullptr, sg = a.nseg > 0;
#define LAUNCH(ZD, SG) sparse_mrow_kernel<G, ZD, SG, PEER><<<grid, 256, 0, s>>>(b)
  if (zd && sg) LAUNCH(true, true);
  else if (zd) LAUNCH(true, false);
  else if (sg) LAUNCH(false, true);
  else LAUNCH(false, false);
#undef LAUNCH
  return cudaGetLastError();
}

template <int G, int V, int H, bool PEER>
cudaError_t launch_gvp(const AggArgs& a, cudaStream_t s) {
  // persistent row pass: as many 8-warp CTAs as fit (4 per SM at 64 registers)
  static int slots = 0;
  if (!slots) {
    int dev = 0, sms = 148, per = 4;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, sparse_row_kernel<G, V, H, true, true, PEER>, 256, 0);
    slots = sms * (per > 0 ? per : 1);
  }
  const bool inl = a.nseg > 0 && a.phase == 0 && a.seg_row && knobs_seg_inline();
  if (a.nseg > 0 && a.phase != 2 && !inl) {
    sparse_seg_kernel<G, V, H, PEER><<<unsigned((a.nseg + 3) / 4), 128, 0, s>>>(a);
    if (a.phase == 1) return cudaGetLastError();
  }
  // row ticket counter[0] and (inline segments) segment ticket counter[8]
  cudaError_t e = cudaMemsetAsync(a.counter, 0, (inl ? 9 : 1) * sizeof(int), s);
  if (e != cudaSuccess) return e;
  const int64_t want = ((a.rows + a.rows_per_ticket - 1) / a.rows_per_ticket + 7) / 8;
  const unsigned grid = unsigned(want < slots ? want : slots);
  AggArgs b = a;
  b.seg_inline = inl ? 1 : 0;
  b.seg_ahead = int64_t(grid) * 8 * knobs_seg_ahead() / 4;
  const bool zd = a.zd_index != nullptr, sg = a.nseg > 0;
#define LAUNCH(ZD, SG) sparse_row_kernel<G, V, H, ZD, SG, PEER><<<grid, 256, 0, s>>>(b)
  if (zd && sg) LAUNCH(true, true);
  else if (zd) LAUNCH(true, false);
  else if (sg) LAUNCH(false, true);
  else LAUNCH(false, false);
#undef LAUNCH
  return cudaGetLastError();
}

template <int G, int V, int H>
cudaError_t launch_gv(const AggArgs& a, cudaStream_t s) {
  return a.peer_world > 0 ? launch_gvp<G, V, H, true>(a, s) : launch_gvp<G, V, H, false>(a, s);
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
      if (loT) {
        const float h = __uint_as_float(__float_as_uint(v) & 0xffffe000u);
        hiT[int64_t(f) * ldT + j] = h;
        loT[int64_t(f) * ldT + j] = v - h;
      } else {  // bf16 round-to-nearest-even (BF16X1 full mode); exact in tf32
        uint32_t u = __float_as_uint(v);
        u = (u + 0x7fffu + ((u >> 16) & 1u)) & 0xffff0000u;
        hiT[int64_t(f) * ldT + j] = __uint_as_float(u);
      }
    }
  }
}

// tf32 split of the (prescaled) input into source-window blocks for the full
// mode's B operand: window w (sources 32w..32w+31) is one contiguous block of
// R = 2*npad rows (hi rows 0..npad-1, lo rows npad..2npad-1; R = npad for the
// bf16-rounded single mode) x 32 sources, each 128-byte row stored already in
// the UMMA K-major SWIZZLE_128B image (16-byte chunk j of row r at j ^ (r & 7)),
// so the engine fetches a chunk's whole B with one contiguous bulk copy
// instead of an R-row strided TMA box.  Sources >= n and features >= F are 0.
// mode 2 (BF16X3): y = b0 + b1 + b2 with b0 = bf16(y), b1 = bf16(y - b0),
// b2 = bf16(y - b0 - b1) (round to nearest even; each residual is exact in
// fp32, |y - b0 - b1 - b2| <= 2^-24 |y|), as three parts of npad rows x 32
// bf16 = 64-byte rows in the K-major SWIZZLE_64B image (16-byte chunk j of
// row r at j ^ ((r >> 1) & 3)).
__device__ __forceinline__ uint32_t bf16_rn_bits(float v) {
  const uint32_t u = __float_as_uint(v);
  return (u + 0x7fffu + ((u >> 16) & 1u)) & 0xffff0000u;
}

__global__ void __launch_bounds__(256) split_window_kernel(const float* __restrict__ Y, int64_t ldy, int64_t n,
                                                           int F, int npad, int mode,
                                                           float* __restrict__ blk) {
  __shared__ float tile[32][33];
  const int64_t w = blockIdx.x;
  const int f0 = blockIdx.y * 32;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;  // 32 x 8
  for (int rr = ty; rr < 32; rr += 8) {
    const int64_t j = w * 32 + rr;
    const int f = f0 + tx;
    tile[rr][tx] = (j < n && f < F) ? __ldg(Y + j * ldy + f) : 0.f;
  }
  __syncthreads();
  const int k = tx;  // source within the window
  if (mode == 2 || mode == 3) {  // 3 bf16 parts (BF16X3) or the first only (BF16X1)
    const int parts = mode == 2 ? 3 : 1;
    uint16_t* out = reinterpret_cast<uint16_t*>(blk + w * int64_t(npad) * 16 * parts);  // parts x npad x 64 B
    for (int ff = ty; ff < 32; ff += 8) {
      const int f = f0 + ff;
      if (f >= npad) continue;
      const float v = tile[k][ff];
      const uint32_t h0 = bf16_rn_bits(v);
      const float r1 = v - __uint_as_float(h0);
      const uint32_t h1 = bf16_rn_bits(r1);
      const uint32_t h2 = bf16_rn_bits(r1 - __uint_as_float(h1));
      const int pos = f * 32 + ((((k >> 3) ^ ((f >> 1) & 3)) << 3) | (k & 7));  // bf16 element offset
      out[pos] = uint16_t(h0 >> 16);
      if (parts == 3) {
        out[npad * 32 + pos] = uint16_t(h1 >> 16);
        out[2 * npad * 32 + pos] = uint16_t(h2 >> 16);
      }
    }
    return;
  }
  const bool single = mode == 1;
  const int R = single ? npad : 2 * npad;
  float* out = blk + w * int64_t(R) * 32;
  for (int ff = ty; ff < 32; ff += 8) {
    const int f = f0 + ff;
    if (f >= npad) continue;
    const float v = tile[k][ff];
    if (!single) {
      const float h = __uint_as_float(__float_as_uint(v) & 0xffffe000u);
      const int rh = f, rl = npad + f;
      out[rh * 32 + ((((k >> 2) ^ (rh & 7)) << 2) | (k & 3))] = h;
      out[rl * 32 + ((((k >> 2) ^ (rl & 7)) << 2) | (k & 3))] = v - h;
    } else {  // bf16 round-to-nearest-even (BF16X1 full mode); exact in tf32
      out[f * 32 + ((((k >> 2) ^ (f & 7)) << 2) | (k & 3))] = __uint_as_float(bf16_rn_bits(v));
    }
  }
}

}  // namespace

cudaError_t launch_split_windows(const float* Y, int64_t ldy, int64_t n, int F, int npad, int mode, float* blk,
                                 int64_t nwin, cudaStream_t s) {
  if (nwin <= 0) return cudaSuccess;
  dim3 grid(unsigned(nwin), unsigned((npad + 31) / 32));
  split_window_kernel<<<grid, 256, 0, s>>>(Y, ldy, n, F, npad, mode, blk);
  return cudaGetLastError();
}

cudaError_t launch_sparse_pass(const AggArgs& a, cudaStream_t s);

// Tuning knob read once (benchmarks only): PCGCN_SPARSE_FSPLIT=<cols> runs
// the gather in column slices of that width (each slice of Y' is a smaller
// L2 working set; the index stream is re-read per slice).  (An L2
// evict_first hint on the index stream was measured and dropped: no gain.)
// PCGCN_SPARSE_V8=0 keeps 16-byte lane vectors even where rows allow the
// 32-byte ones (A/B measurement).
struct SparseKnobs {
  int fsplit = 0;
  bool v8 = true;
  bool g6 = true;  // PCGCN_SPARSE_G6=0: F = 41..48 keeps the 16-byte G = 16 layout (A/B)
  // PCGCN_SPARSE_MROW: -1 (default) multi-row warps for 17..64 features when the
  // plan's mean selective degree is <= MROW_MAX_DEG and its rows are degree-ordered;
  // 0 never; 1 wherever the layout fits
  int mrow = -1;
  int mrow_sort = 0;  // PCGCN_MROW_SORT=1: rows of a 32-row ticket grouped by degree (id-ordered plans)
  int seg_inline = 0;  // measured (B200, fixed θ, interleaved): C3 F=41 passes +5%, C5 neutral -> off
  int seg_ahead = 4;  // quarters of (grid warps) row tickets
  SparseKnobs() {
    if (const char* e = getenv("PCGCN_SEG_INLINE")) seg_inline = atoi(e);
    if (const char* e = getenv("PCGCN_SEG_AHEAD")) seg_ahead = std::max(1, atoi(e));
    if (const char* e = getenv("PCGCN_SPARSE_MROW")) mrow = atoi(e);
    if (const char* e = getenv("PCGCN_MROW_SORT")) mrow_sort = atoi(e);
    if (const char* e = getenv("PCGCN_SPARSE_FSPLIT")) fsplit = atoi(e) / 32 * 32;
    if (const char* e = getenv("PCGCN_SPARSE_V8")) v8 = atoi(e) != 0;
    if (const char* e = getenv("PCGCN_SPARSE_G6")) g6 = atoi(e) != 0;
  }
};


static SparseKnobs& knobs() {
  static SparseKnobs k;
  return k;
}
int knobs_mrow_sort() { return knobs().mrow_sort; }
int knobs_seg_inline() { return knobs().seg_inline; }

int knobs_seg_ahead() { return knobs().seg_ahead; }

bool sparse_fsplit_active(int F) { return knobs().fsplit > 0 && F > knobs().fsplit; }

cudaError_t launch_sparse_agg(const AggArgs& a0, cudaStream_t s) {
  if (a0.rows <= 0) return cudaSuccess;
  const SparseKnobs& kn = knobs();
  AggArgs a = a0;
  if (kn.fsplit <= 0 || a.F <= kn.fsplit) return launch_sparse_pass(a, s);
  for (int c0 = 0; c0 < a.F; c0 += kn.fsplit) {
    AggArgs b = a;
    b.F = (a.F - c0) < kn.fsplit ? a.F - c0 : kn.fsplit;
    b.Y = a.Y + c0;
    b.Z = a.Z + c0;
    if (a.zd) b.zd = a.zd + c0;
    if (a.mask) b.mask = a.mask + c0 / 32;
    cudaError_t e = launch_sparse_pass(b, s);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

cudaError_t launch_sparse_pass(const AggArgs& a, cudaStream_t s) {
  // G lanes x V vectors per edge slot: the narrowest power-of-two slot that
  // covers the row, so one load instruction reads whole rows (fewest lines).
  // Vectors are 32 bytes (8 floats) when the rows are 32-byte aligned and the
  // wider vector reads no padding the 16-byte one skips (F = 41: 48 vs 44
  // floats per row, measured 6% slower on C3's L2-bound F = 41 pass); else 16.
  // Measured (B200, PCGCN_SPARSE_V8=0 vs 1): C5's issue-bound row pass F = 32
  // 21.2 -> 19.2 ms, F = 128 45.4 -> 43.3 ms; C3 F = 128 unchanged.
  const bool al32 = knobs().v8 && a.ldy % 8 == 0 && (reinterpret_cast<uintptr_t>(a.Y) & 31) == 0;
  const bool v8 = al32 && (a.F + 7) / 8 * 2 == (a.F + 3) / 4;
  // 41..48 features in 32-byte aligned rows (C3's class width, ld 48): six
  // 32-byte vectors per row read the row's 192 bytes (6 sectors, as many as the
  // 44 floats of the 16-byte layout touch) with 5 rows per load instruction
  if (al32 && knobs().g6 && (a.F + 7) / 8 == 6) return launch_gv<6, 1, 2>(a, s);
  // short rows (mean selective degree <= MROW_MAX_DEG) of degree-ordered plans:
  // one row per edge slot (C5's F=32 pass: 19.6 -> 16.3 ms in degree order; in
  // id order 26.1 ms, and 23.8 ms with the per-ticket degree grouping, against
  // 20.0 ms for the warp-per-row pass — so id-ordered plans keep the latter)
  if (v8 && knobs().mrow != 0 &&
      (knobs().mrow > 0 || (a.mean_deg <= MROW_MAX_DEG && a.rows_by_degree))) {
    const int nvec = (a.F + 7) / 8;
    if (nvec >= 3 && nvec <= 4) return a.peer_world > 0 ? launch_mrow<4, true>(a, s) : launch_mrow<4, false>(a, s);
    if (nvec >= 5 && nvec <= 8) return a.peer_world > 0 ? launch_mrow<8, true>(a, s) : launch_mrow<8, false>(a, s);
  }
  if (v8) {
    const int nvec = (a.F + 7) / 8;
    if (nvec <= 1) return launch_gv<1, 1, 2>(a, s);
    if (nvec <= 2) return launch_gv<2, 1, 2>(a, s);
    if (nvec <= 4) return launch_gv<4, 1, 2>(a, s);
    if (nvec <= 8) return launch_gv<8, 1, 2>(a, s);
    if (nvec <= 16) return launch_gv<16, 1, 2>(a, s);
    if (nvec <= 32) return launch_gv<32, 1, 2>(a, s);  // F <= 256 = f_max
  }
  const int nvec = (a.F + 3) / 4;
  if (nvec <= 1) return launch_gv<1, 1, 1>(a, s);
  if (nvec <= 2) return launch_gv<2, 1, 1>(a, s);
  if (nvec <= 4) return launch_gv<4, 1, 1>(a, s);
  if (nvec <= 8) return launch_gv<8, 1, 1>(a, s);
  if (nvec <= 16) return launch_gv<16, 1, 1>(a, s);
  if (nvec <= 32) return launch_gv<32, 1, 1>(a, s);
  return launch_gv<32, 2, 1>(a, s);
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
