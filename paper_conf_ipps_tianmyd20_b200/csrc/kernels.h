// Launchers of the sm_100a kernels (internal; the ABI is include/pcgcn.h).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

namespace pcgcn {

// fused split target of a transform GEMM: the full mode's window blocks of the output
struct WindowOut {
  float* blk = nullptr;      // window blocks (DevicePlan::yhi)
  int mode = 0;              // 1 tf32 hi/lo, 2 bf16x1, 3 bf16x3
  int64_t blk_floats = 0;    // floats per window block
  int64_t nwin = 0;          // windows in the buffer
};

// ---- aggregation (sparse.cu) ----
struct AggArgs {
  const float* Y;            // prescaled input (all n rows), ld ldy
  int64_t ldy;
  float* Z;                  // shard-local output rows, ld ldz
  int64_t ldz;
  uint32_t* mask;            // shard-local [rows x ceil(F/32)] or nullptr
  const int64_t* rowptr;     // shard-local merged selective CSR
  const int32_t* col;
  const float* r;            // [n] plan order
  int64_t row_lo;            // first plan row of the shard
  int64_t rows;              // rows in the shard
  const int32_t* zd_index;   // shard-local, or nullptr if no dense tiles
  const float* zd;           // dense partial sums, ld ldzd
  int64_t ldzd;
  const float* zrow;         // >= 16 zero floats (load sentinel)
  int mask_ld;               // u32 words per mask row
  int64_t n_src;             // rows of Y (for the L2-residency decision)
  int F;
  bool relu, out_prescaled;
  // long-row segments (reading #22): rows with more than SEG_EDGES
  // selective edges are summed by a segment pass into seg_ws first; the row
  // pass then adds its row's segment partials in segment order
  const int32_t* row_seg;    // [rows] first segment id, -1 = row gathered directly (nullptr: none)
  const int64_t* seg_lo;     // [nseg] shard-local edge range [seg_lo, seg_hi) of each segment
  const int64_t* seg_hi;     // [nseg]
  int64_t nseg;
  float* seg_ws;             // [nseg x ldws] fp32 partial sums
  int64_t ldws;
  int* counter;              // dynamic row scheduler ticket (zeroed on the stream before each pass)
  // inline segments: the row pass also claims the segments
  const int32_t* seg_row = nullptr;  // [nseg] shard-local row of each segment
  int* seg_cnt = nullptr;            // [nseg] completed segments per long row (at its first segment; self-resetting)
  int* seg_ticket = nullptr;         // segment ticket (zeroed with the row ticket)
  int seg_inline = 0;                // 1: no separate segment pass
  int64_t seg_ahead = 0;             // row tickets ahead of the claiming warp within which segments are taken
  // device-initiated peer gather: sources of shard q are read from
  // shard q's own buffer (peer_base[q] = its row row0[q]; NVLink peer memory
  // on a multi-GPU node, CUDA IPC in the 1-GPU tests) instead of an exchanged copy
  int peer_world = 0;        // 0: sources come from Y
  const char* peer_base[8];
  int64_t peer_row0[9];
  int phase = 0;             // 0: segment pass + row pass; 1: segment pass only; 2: row pass only
  int rows_per_ticket = 1;   // consecutive rows per scheduler ticket, 1..16
  float mean_deg = 0.f;      // selective edges per row (layout choice: short rows -> multi-row warps)
  int rows_by_degree = 0;    // plan rows sorted by degree inside partitions (multi-row groups are balanced)
  int mrow_sort = 1;         // multi-row pass: group a ticket's 32 rows by degree
};
// selective edges per long-row segment
constexpr int SEG_EDGES = 1024;
bool sparse_fsplit_active(int F);  // benchmark knob PCGCN_SPARSE_FSPLIT splits this width
cudaError_t launch_sparse_agg(const AggArgs& a, cudaStream_t s);

// ypre = diag(r)·Y
cudaError_t launch_prescale(const float* Y, int64_t ldy, const float* r, int64_t n, int F, float* ypre,
                            int64_t ldpre, cudaStream_t s);
// tf32 hi/lo split of Y written feature-major: hiT/loT [npad x ldT]; loT == nullptr: hiT = bf16 RN-even of Y
cudaError_t launch_split_transpose(const float* Y, int64_t ldy, int64_t n, int F, int npad, float* hiT,
                                   float* loT, int64_t ldT, cudaStream_t s);

// ---- dense-mode tcgen05 tile contraction (dense_tc.cu) ----
struct DenseArgs {
  const float* hiT;          // [npad x ldT] tf32 hi part of the prescaled input, feature-major
  const float* loT;          // [npad x ldT] lo part; nullptr: single product on bf16-rounded hiT (BF16X1)
  int64_t n, ldT;
  const int32_t* rt_row0;    // shard row tiles
  const int32_t* rt_nrows;
  const int64_t* rt_cptr;
  const int32_t* ch_col0;
  const uint32_t* bits;
  int64_t nrt;
  float* zd;                 // [nrt*128 x ldzd]
  int64_t ldzd;
  int npad;                  // UMMA N (multiple of 16, >= F)
  const int32_t* rt_order = nullptr;  // engine tile order (position i of CTA b: tile rt_order[b + i*G])
  const float* blk = nullptr;  // source-window blocks (launch_split_windows); nullptr: hiT/loT maps
  int64_t blk_floats = 0;      // floats per window block
  int64_t n_src = 0;           // real source rows (vertices); rows [n_src, n) of the input are never read
  int bf3 = 0;                 // bf16 parts per window block (kind::f16 MMAs): 3 BF16X3, 1 BF16X1; 0 tf32
  int* dyn = nullptr;          // zeroed tile ticket: CTAs claim tiles dynamically in rt_order / plan order
};
// mode 0: tf32 hi/lo, 1: bf16-rounded tf32 single (unused since BF16X1 runs on kind::f16),
// 2: three bf16 parts (BF16X3), 3: one bf16 part (BF16X1)
cudaError_t launch_split_windows(const float* Y, int64_t ldy, int64_t n, int F, int npad, int mode, float* blk,
                                 int64_t nwin, cudaStream_t s);
cudaError_t launch_dense_tc(const DenseArgs& a, cudaStream_t s);
// CTA-pair (cta_group::2) variant of the full mode (tc_pair.cu); map_b covers [hi rows; lo rows]
bool dense_pair_eligible(int npad);
cudaError_t launch_dense_pair(const DenseArgs& a, const struct CUtensorMap_st& map_b, cudaStream_t s);
// CUDA-core fp32 full mode (§IV-C) on the prescaled input y
cudaError_t launch_dense_simt_y(const DenseArgs& a, const float* y, int64_t ldy, int F,
                                cudaStream_t s);

// ---- GEMMs (gemm.cu) ----
int64_t gemm_xw_work_floats(int K, int N);
cudaError_t launch_gemm_xw(const float* X, int64_t ldx, const float* W, int64_t ldw, const float* s,
                           float* Y, int64_t ldy, int64_t M, int K, int N, float* work, cudaStream_t st,
                           const WindowOut* wo = nullptr);
// tcgen05 engine GEMMs (tc_engine.cu)
cudaError_t launch_tc_gemm_xw(const float* X, int64_t ldx, const float* wThi, const float* wTlo, int64_t ldwT,
                              const float* rs, float* Y, int64_t ldy, int64_t M, int K, int N, cudaStream_t s,
                              const uint32_t* mask = nullptr, int64_t mask_ld = 0, const WindowOut* wo = nullptr);
int64_t tc_xtg_slices(int64_t M, int K);
cudaError_t launch_tc_gemm_xtg_raw(const float* X, int64_t ldx, const float* D, int64_t ldd, float* partial,
                                   int64_t M, int K, int N, cudaStream_t s);
cudaError_t launch_tc_gemm_xtg(const float* X, int64_t ldx, const float* dThi, const float* dTlo, int64_t lddT,
                               float* partial, int64_t M, int K, int N, cudaStream_t s);
int64_t gemm_xtg_work_floats(int64_t M, int K, int N);
cudaError_t launch_gemm_xtg(const float* X, int64_t ldx, const float* D, int64_t ldd, float* G,
                            int64_t M, int K, int N, float* work, cudaStream_t st);
int64_t gemm_dwt_work_floats(int K, int N);
cudaError_t launch_gemm_dwt(const float* D, int64_t ldd, const float* W, const uint32_t* mask,
                            const float* s, float* O, int64_t ldo, int64_t M, int N, int K,
                            float* work, cudaStream_t st, const WindowOut* wo = nullptr);

// ---- halo exchange of a sharded plan (halo.cu) ----
cudaError_t launch_halo_copy(bool pack, const float* src, int64_t lds, float* dst, int64_t ldd, const int32_t* idx,
                             int64_t rows, int w, cudaStream_t s);

// ---- loss / optimiser (loss_opt.cu) ----
cudaError_t launch_softmax_ce(const float* L, int64_t ld, const int32_t* labels,
                              const uint8_t* train, int64_t M, int C, float inv_nT, const float* s,
                              float* dL, float* loss, float* work, cudaStream_t st);
cudaError_t launch_adam(float* th, const float* g, float* m, float* v, int64_t n, float lr, float b1,
                        float b2, float eps, int32_t* step, cudaStream_t st);
cudaError_t launch_sgd(float* th, const float* g, int64_t n, float lr, cudaStream_t st);

}  // namespace pcgcn
