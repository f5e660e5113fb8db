/*
 * pcgcn.h — C ABI of libpcgcn.so, the B200-native hot path of PCGCN
 * (Tian, Ma, Yang, Dai, "PCGCN: Partition-Centric Processing for Accelerating
 * Graph Convolutional Network", IPDPS 2020).  Citations "L<n>" are line
 * numbers of the paper text plus the section / equation they sit in.
 *
 * The path computes the GCN propagation of Eq. (1) (L55):
 *      Z = D̃^-1/2 (A + I) D̃^-1/2 · Y,      Y = X·Θ  (Alg. 1 line a^l = h^{l-1} w^l, L114)
 * partition-centric (Alg. 1): vertices are clustered into P vertex
 * blocks V_k, the normalised adjacency is cut into P×P edge blocks E_{k,i}
 * (L95 §III-A.a), and every block runs in one of two modes chosen by the
 * density threshold θ (L155-L161 §III-B.c):
 *   selective ("sparse") — merged CSR gather over the block's edges (L137,
 *                          L149, L179 §IV-B);
 *   full ("dense")       — the block treated as a dense 0/1 matrix (L151-L153,
 *                          L175) contracted on the tcgen05 tensor cores
 *                          (the B200 analogue of §IV-D).
 *
 * Conventions (all functions):
 *   - extern "C", no C++ exceptions cross the ABI; every call returns a
 *     pcgcn_status; pcgcn_last_error() gives a thread-local message.
 *   - "HOST" pointers are read during the call only (borrowed).  "DEVICE"
 *     pointers are CUDA device memory owned by the caller, and every device
 *     call is asynchronous on the given cudaStream_t (passed as void*), never
 *     synchronises the host, allocates nothing, and is CUDA-graph capturable
 *     (one exception: the first forward/backward WITHOUT PCGCN_IN_PRESCALED
 *     allocates the plan's n x f_max prescale workspace).
 *   - Dense matrices are row-major fp32 with an explicit leading dimension
 *     (elements); ld >= roundup(F, 4) and rows 16-byte aligned.  Pad columns
 *     of inputs must be zero; pad columns of outputs are written as zero.
 *     Inputs with 32-byte aligned rows (ld % 8 == 0, 32-byte aligned base)
 *     let the selective pass read 32-byte lane vectors when roundup(F, 8) ==
 *     roundup(F, 4) (same results within tolerance; a different fixed order).
 *   - Device buffers are in PLAN ORDER: row v of Y/Z is the vertex
 *     perm[v] of the input graph (pcgcn_plan_perm).  The caller permutes its
 *     features / labels once, outside any timed region.
 *   - There is no CPU fallback: device calls on a machine without an sm_100
 *     GPU fail with PCGCN_ECUDA.
 */
#ifndef PCGCN_H
#define PCGCN_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct pcgcn_plan_s* pcgcn_plan_t;

typedef enum {
  PCGCN_OK = 0,
  PCGCN_EINVAL = 1,   /* bad argument (null pointer, size, ld, F > f_max, ...) */
  PCGCN_ENOTSYM = 2,  /* input adjacency not symmetric (needed for Âᵀ = Â) */
  PCGCN_ECUDA = 3,    /* CUDA runtime error (also: no usable GPU) */
  PCGCN_ENOMEM = 4,   /* host or device allocation failed */
  PCGCN_ENCCL = 5,    /* NCCL missing or a collective failed (pcgcn_nccl_* / pcgcn_halo_exchange) */
  PCGCN_EUNSUP = 6    /* unsupported option combination */
} pcgcn_status;

/* Input graph, HOST, borrowed.  Row v lists the in-neighbours of v — the
 * Dst/Src convention of Fig. 5(a) (L171-L173) without the Val array (edge
 * values are recomputed from degrees).  Must be symmetric (undirected graph,
 * Fig. 4 L87); duplicates collapse to one edge; input self-loops are dropped
 * and I is added (Kipf renormalisation, reading #1). */
typedef struct {
  int64_t n;              /* vertices */
  int64_t nnz;            /* entries of col (= rowptr[n]) */
  const int64_t* rowptr;  /* [n+1], rowptr[0] = 0, non-decreasing */
  const int32_t* col;     /* [nnz], 0 <= col < n, any order within a row */
} pcgcn_csr;

enum { PCGCN_NORM_SYM = 0, PCGCN_NORM_NONE = 1 };     /* Â = D̃^-½ÃD̃^-½  |  Â = Ã (integer pin) */
enum {
  PCGCN_DENSE_TF32X2 = 0,    /* full mode on tcgen05 (kind::tf32): A∈{0,1} exact, Y = hi + lo, 2 MMAs */
  PCGCN_DENSE_FP32_SIMT = 1, /* full mode on CUDA cores in fp32 (the paper's §IV-C kernel, L183-L187) */
  PCGCN_DENSE_BF16X1 = 2,    /* full mode on tcgen05 kind::f16 with the input rounded to bf16 (RN-even):
                                one bf16 part, 2 K=16 MMAs and 2·32·npad B bytes per 128x32 chunk, fp32
                                accumulation: the paper's 16-bit tensor-core policy (L191-L193, §V-E);
                                error <= 2^-9 per term, gate 2e-2 (BASELINE.json north_star) */
  PCGCN_DENSE_BF16X3 = 3     /* full mode on tcgen05 kind::f16: Y = b0 + b1 + b2, three bf16 parts
                                (round to nearest, exact fp32 residuals: |Y - Σb| <= 2^-24|Y|), A∈{0,1}
                                exact; 6 K=16 MMAs and 6·32·npad B bytes per 128x32 chunk against the
                                tf32 split's 8 K=8 MMAs (at half the bf16 rate) and 8·32·npad; gate 1e-5 */
};

typedef struct {
  int32_t norm;           /* PCGCN_NORM_*; default SYM */
  int32_t dense_prec;     /* PCGCN_DENSE_*; default TF32X2 */
  int32_t f_max;          /* largest F passed to forward/backward (workspace size); default 128, <= 256 */
  int32_t lp_sweeps;      /* label-propagation sweep cap T; default 10 */
  const int32_t* part;    /* HOST [n] optional partition override (0 <= part < P); NULL => LP + packing */
  int32_t build_device;   /* 1 (default): upload to the current CUDA device; 0: host-only plan (tests) */
  int32_t rank, world;    /* destination-partition shard of this process; default 0, 1 */
  int32_t vertex_order;   /* PCGCN_ORDER_*: order of the vertices inside a partition; default ID */
  int32_t mode_grain;     /* PCGCN_GRAIN_*: unit of the selective/full decision; default BLOCK */
} pcgcn_opts;

/* Vertex order inside a vertex block V_k (the paper fixes only the blocks, L95-L97):
 *   ID     — ascending original id (plan spec of DESIGN.md §3a);
 *   DEGREE — descending degree, ties by id: high-degree rows and sources gather at the
 *            start of every block, so the 128x32 sub-blocks of a dense region are denser
 *            (reading #24). */
enum { PCGCN_ORDER_ID = 0, PCGCN_ORDER_DEGREE = 1 };
/* Unit of the mode decision (θ rule of L161):
 *   BLOCK — the partition pair E_{k,i}: full iff nnz(E_ki)/(|V_k||V_i|) > θ (the paper);
 *   TILE  — the 128-row x 32-source sub-block the full mode executes as one chunk (a row
 *           tile of V_k against a 32-aligned source window): full iff its nnz/(rows·cols) > θ,
 *           the same rule at the granularity of the B200 kernel (reading #25). */
enum { PCGCN_GRAIN_BLOCK = 0, PCGCN_GRAIN_TILE = 1 };

/* Plan statistics (L304-style mode usage + cost model inputs). */
typedef struct {
  int64_t n, nnz;               /* vertices, nnz(Ã) including the n self-loops */
  int32_t P, lp_sweeps;         /* partitions; label-propagation sweeps run (0 if overridden) */
  int64_t clusters;             /* LP clusters before packing */
  int64_t blocks_nonempty, blocks_dense;
  int64_t nnz_sparse, nnz_dense;/* Ã entries handled by each mode */
  int64_t intra_edges;          /* Ã entries with both ends in one partition (self-loops included) */
  int64_t row_tiles, chunks;    /* dense 128-row tiles, 128x32 bit chunks */
  int64_t row_lo, row_hi;       /* this shard's plan-row range [row_lo, row_hi) */
  int64_t shard_nnz_sparse, shard_chunks;
  double theta;
  double partition_ms, plan_ms; /* host time of LP+packing, and of the whole plan */
  int64_t device_bytes;         /* device memory owned by the plan */
  int64_t shard_segments;       /* long selective rows' segments (> 1024 edges per row, reading #22) */
  int64_t src_rows_pc;          /* Σ_k |distinct sources of V_k's selective edges| (B_pc model) */
  int64_t shard_src_rows_pc;    /* the same over this shard's partitions */
  int64_t halo_recv_rows;       /* rows of other shards this shard reads (0 unsharded) */
  int64_t halo_send_rows;       /* Σ_q rows of this shard that shard q reads */
} pcgcn_stats;

void pcgcn_opts_default(pcgcn_opts* o);

/* Build a plan (host C++, deterministic, independent of thread count).
 *   theta: density threshold θ of L161; block (k,i) runs in full mode iff
 *          nnz(E_ki)/(|V_k||V_i|) > θ (strict, reading #10).
 *          θ = 0  => every non-empty block dense  ("PCGCN-full", Table III)
 *          θ >= 1 => every block sparse           ("PCGCN-sel", Table III)
 *          θ < 0  => calibrate first on the current device (pcgcn_calibrate at width
 *                    f_max, p = 0.05, blocks of the mean partition size; L161), then plan
 *                    with that θ (the value lands in pcgcn_stats.theta); needs
 *                    build_device = 1, else PCGCN_EINVAL.  NaN => PCGCN_EINVAL.
 *   P: number of vertex blocks K (Alg. 1 "Partition G -> {S_k}", L112), 1..n.
 * On success *out owns host + device memory until pcgcn_destroy. */
pcgcn_status pcgcn_plan(const pcgcn_csr* A, int32_t P, float theta, const pcgcn_opts* o,
                        pcgcn_plan_t* out);
void pcgcn_destroy(pcgcn_plan_t p);

/* flags for forward/backward */
enum {
  PCGCN_IN_PRESCALED = 1u,  /* Y already holds diag(r)·Y (r = d̃^-½ applied by the producing GEMM) */
  PCGCN_RELU = 2u,          /* Z = max(Z, 0) */
  PCGCN_MASK_OUT = 4u,      /* write mask bit [Z_pre > 0], 1 bit per element, row stride ceil(F/32) u32 */
  PCGCN_OUT_PRESCALED = 8u, /* Z = diag(r)·Z again (feeds the next aggregation directly) */
  PCGCN_PROFILE = 16u,      /* record CUDA events around each internal kernel (not graph-capturable);
                               read them with pcgcn_plan_last_timings after the stream completes */
  PCGCN_IN_SPLIT = 32u      /* with IN_PRESCALED: the plan's full-mode window blocks already hold this
                               input (written by pcgcn_gemm_xw_split / pcgcn_gemm_dwt_split with this plan
                               and F), so the split pass is skipped */
};

/* Per-kernel times (ms) of the last PCGCN_PROFILE call on this plan:
 * ms[0] prescale, ms[1] tf32 split, ms[2] full-mode (tcgen05) tiles, ms[3] selective gather
 * (0 for kernels that did not run).  Synchronises on the recorded events. */
pcgcn_status pcgcn_plan_last_timings(pcgcn_plan_t p, float ms[4]);

/* Measurement helper: streams `bytes` of device memory `iters` times with 16-byte
 * loads from all SMs and returns the read bandwidth in GB/s (an L2-resident size
 * measures the L2->SM path, a size >> 126 MB the HBM path).  Synchronises. */
pcgcn_status pcgcn_probe_read_gbs(int64_t bytes, int32_t iters, float* gbs);

/* Measurement helper: the selective kernel's access pattern (L149, L181: one source
 * feature row per edge) without its index stream — every warp slot of G = row_bytes/16
 * lanes (G the narrowest power of two covering the row, as in the kernel) reads
 * pseudo-random rows of `row_bytes` (multiple of 16, 16..512; row stride = row_bytes) from a buffer
 * of `bytes`, 8 rows in flight per lane, `steps` (>= 8) rows per slot; returns the
 * gathered GB/s.  The buffer size selects the level serving the rows (L1 ~<= 128 KB,
 * L2 << 126 MB, HBM >> 126 MB): the measured ceilings of the gather roofline
 * (DESIGN.md §6).  Allocates and frees a device buffer; synchronises. */
pcgcn_status pcgcn_probe_gather_gbs(int64_t bytes, int32_t row_bytes, int32_t steps, float* gbs);

/* Z = Â·Y  (Eq. 1 propagation; Alg. 1 inner loop h_k = Σ_i f(E_{k,i}, a_i), L118-L121).
 *   Y: DEVICE [n x F] (full plan order, all n rows even on a shard), ld ldy.
 *   Z: DEVICE [rows x F] with rows = row_hi - row_lo of this shard (n unsharded), ld ldz.
 *   mask: DEVICE u32 [rows x ceil(F/32)] written iff flags & MASK_OUT, else may be NULL.
 *   F: 1..f_max.  Dense blocks then sparse rows; each output row is reduced by
 *   one warp in a fixed order (bitwise reproducible run to run). */
pcgcn_status pcgcn_forward(pcgcn_plan_t p, const float* Y, int64_t ldy, float* Z, int64_t ldz,
                           int32_t F, uint32_t flags, uint32_t* mask, void* stream);

/* dY = Âᵀ·dZ = Â·dZ (A symmetric, reading #2): the backward of the propagation
 * reuses the forward plan.  Same argument rules as pcgcn_forward (mask unused). */
pcgcn_status pcgcn_backward(pcgcn_plan_t p, const float* dZ, int64_t ldz, float* dY, int64_t ldy,
                            int32_t F, uint32_t flags, void* stream);

/* ---- halo exchange of a sharded plan (world > 1) ----
 * Shard r owns plan rows [row0[r], row0[r+1]).  Before an aggregation it needs the
 * rows of other shards that its selective edges read and every row of the 32-source
 * windows of its full-mode chunks: the halo.  The planner lists them per peer q
 * (ascending plan rows): RECV = rows of shard q this shard reads, SEND = rows of this
 * shard that shard q reads (= q's RECV list for this rank; every rank builds the same
 * deterministic plan).  A shard's own rows are never listed; world = 1 => empty. */
pcgcn_status pcgcn_plan_shard_rows(pcgcn_plan_t p, int64_t* row0 /* HOST [world+1] */);
int64_t pcgcn_plan_halo_rows(pcgcn_plan_t p, int32_t q, int32_t send);  /* list length; -1 on bad args */
pcgcn_status pcgcn_plan_halo_export(pcgcn_plan_t p, int32_t q, int32_t send, int32_t* host_buf, int64_t cap);
/* pack: buf[i] = Y[send row i] for the concatenated SEND lists (peers in rank order),
 * unpack: Y[recv row i] = buf[i] for the concatenated RECV lists.  Y DEVICE [n x ldy]
 * (full height, plan order), buf DEVICE [rows x w] dense; w floats are copied per row
 * (multiple of 4, <= ldy: pass the activation stride to move pad columns too).
 * Bitwise copies; stream-ordered, graph-capturable.  The transport between the two
 * (NCCL grouped send/recv, or an all-to-all) is the caller's (dist.py). */
pcgcn_status pcgcn_halo_pack(pcgcn_plan_t p, const float* Y, int64_t ldy, int32_t w, float* buf, void* stream);
pcgcn_status pcgcn_halo_unpack(pcgcn_plan_t p, const float* buf, float* Y, int64_t ldy, int32_t w, void* stream);

/* In-library NCCL transport (SURVEY.md §8(b) nccl_comm): libnccl.so.2 is opened at first
 * use (no link-time dependency); PCGCN_ENCCL when it is missing or a call fails.
 *   pcgcn_nccl_unique_id: rank 0 creates the 128-byte id (HOST buffer) that the caller
 *       distributes (e.g. over the torch process group);
 *   pcgcn_nccl_comm_init: every rank joins on the current CUDA device (collective);
 *   pcgcn_halo_exchange: pack -> one NCCL group of ncclSend/ncclRecv to every peer with a
 *       non-empty list -> unpack, on `stream` (graph-capturable); sendbuf/recvbuf DEVICE
 *       [Σ send rows x w] / [Σ recv rows x w]; world = 1 => no-op. */
pcgcn_status pcgcn_nccl_unique_id(void* id128);
pcgcn_status pcgcn_nccl_comm_init(const void* id128, int32_t rank, int32_t world, void** comm_out);
void pcgcn_nccl_comm_destroy(void* comm);
pcgcn_status pcgcn_halo_exchange(pcgcn_plan_t p, float* Y, int64_t ldy, int32_t w, float* sendbuf, float* recvbuf,
                                 void* nccl_comm, void* stream);

/* Device-initiated peer gather: the selective pass of shard r reads
 * each source row straight from its owner's buffer — peer_Y[q] (DEVICE pointer valid in
 * this process: NVLink peer memory, or a CUDA IPC mapping) holds shard q's rows
 * [row0[q], row0[q+1]) (pcgcn_plan_shard_rows) with row stride ldy — so no halo copy is
 * exchanged at all.  Z: this shard's rows.  Selective-only shards (a shard with full-mode
 * chunks returns PCGCN_EUNSUP), prescaled inputs (IN_PRESCALED required), world <= 8.
 * Each row is summed in the same order as by pcgcn_forward on a full-height input:
 * bitwise the same result. */
pcgcn_status pcgcn_forward_peer(pcgcn_plan_t p, const float* const* peer_Y /* HOST [world] */, int64_t ldy,
                                float* Z, int64_t ldz, int32_t F, uint32_t flags, uint32_t* mask, void* stream);
pcgcn_status pcgcn_backward_peer(pcgcn_plan_t p, const float* const* peer_dZ /* HOST [world] */, int64_t ldz,
                                 float* dY, int64_t ldy, int32_t F, uint32_t flags, void* stream);
/* CUDA IPC plumbing for peer buffers between processes: allocate (zeroed, its own
 * allocation so the handle covers exactly it), export a 64-byte handle, open a peer's
 * handle (lazy peer access), close, free. */
pcgcn_status pcgcn_ipc_alloc(int64_t bytes, void** ptr);
void pcgcn_ipc_free(void* ptr);
pcgcn_status pcgcn_ipc_handle(void* ptr, void* handle64);
pcgcn_status pcgcn_ipc_open(const void* handle64, void** ptr);
void pcgcn_ipc_close(void* ptr);

/* ---- dense helpers of the 2-layer GCN step (Alg. 1 transform, L114) ---- */

/* Y = diag(s)·(X·W):  X DEVICE [M x K] ld ldx, W DEVICE [K x N] ld ldw, Y DEVICE [M x N] ld ldy.
 * s: DEVICE [M] row scale or NULL.  fp32 in/out.  With ldx, ldy multiples of
 * 4 and `work` (DEVICE, pcgcn_gemm_xw_work_floats(K,N) floats) it runs on the
 * tcgen05 tensor cores in 3xTF32 (A_hi·B_hi + A_lo·B_hi + A_hi·B_lo); else
 * (work NULL / unaligned) on fp32 CUDA cores. */
int64_t pcgcn_gemm_xw_work_floats(int32_t K, int32_t N);
pcgcn_status pcgcn_gemm_xw(const float* X, int64_t ldx, const float* W, int64_t ldw, const float* s,
                           float* Y, int64_t ldy, int64_t M, int32_t K, int32_t N, float* work, void* stream);

/* The same transform GEMM with the full mode's split fused into its epilogue:
 * besides Y it writes plan p's window blocks of Y (p's precision, width N) — bit-identical
 * to what the split pass of a following forward/backward would write, which then runs
 * with PCGCN_IN_SPLIT.  p unsharded, M == n, N <= min(f_max, 128), the tcgen05 path
 * (work, ld multiples of 4); a plan without full-mode chunks writes Y only. */
pcgcn_status pcgcn_gemm_xw_split(pcgcn_plan_t p, const float* X, int64_t ldx, const float* W, int64_t ldw,
                                 const float* s, float* Y, int64_t ldy, int64_t M, int32_t K, int32_t N, float* work,
                                 void* stream);

/* G = Xᵀ·D:  X DEVICE [M x K] ld ldx, D DEVICE [M x N] ld ldd, G DEVICE [K x N] (ld N), fp32.
 * Split over M into fixed slices whose partial products land in `work`
 * (DEVICE, pcgcn_gemm_xtg_work_floats(M,K,N) floats), then summed in a fixed
 * order: deterministic, no atomics.  tcgen05 3xTF32 when ldx, ldd are
 * multiples of 4, else fp32 CUDA cores. */
int64_t pcgcn_gemm_xtg_work_floats(int64_t M, int32_t K, int32_t N);
pcgcn_status pcgcn_gemm_xtg(const float* X, int64_t ldx, const float* D, int64_t ldd, float* G,
                            int64_t M, int32_t K, int32_t N, float* work, void* stream);

/* O = diag(s)·((D·Wᵀ) ⊙ mask):  D DEVICE [M x N] ld ldd, W DEVICE [K x N] (ld N),
 * mask DEVICE u32 bits [M x ceil(K/32)] (PCGCN_MASK_OUT layout) or NULL, s DEVICE [M] or NULL,
 * O DEVICE [M x K] ld ldo (pad columns [K, ldo) written as 0).  The backward of the layer-2
 * transform through the ReLU (a11; the paper is silent on the backward).  With ldd, ldo
 * multiples of 4, K <= 256 and `work` (DEVICE, pcgcn_gemm_dwt_work_floats(K,N) floats) it
 * runs on the tcgen05 engine in 3xTF32 with the mask and scale in the epilogue; else (work
 * NULL / unaligned) on fp32 CUDA cores. */
int64_t pcgcn_gemm_dwt_work_floats(int32_t K, int32_t N);
pcgcn_status pcgcn_gemm_dwt(const float* D, int64_t ldd, const float* W, const uint32_t* mask,
                            const float* s, float* O, int64_t ldo, int64_t M, int32_t N, int32_t K,
                            float* work, void* stream);
/* ... with plan p's window blocks of O written in the epilogue (as pcgcn_gemm_xw_split; width K) */
pcgcn_status pcgcn_gemm_dwt_split(pcgcn_plan_t p, const float* D, int64_t ldd, const float* W, const uint32_t* mask,
                                  const float* s, float* O, int64_t ldo, int64_t M, int32_t N, int32_t K, float* work,
                                  void* stream);

/* Softmax cross-entropy over the train mask (reading #14):
 *   loss = (1/nT) Σ_{i: train_i} [logsumexp(L_i) - L_{i,y_i}]
 *   dL_i = s_i · (softmax(L_i) - onehot(y_i)) · train_i / nT   (s = row scale or NULL)
 * L, dL DEVICE [M x C] ld ld; labels DEVICE i32 [M]; train DEVICE u8 [M];
 * loss DEVICE f32 [1] (sum of this shard's terms, divided by nT; deterministic).
 * dL has the same ld as L. */
#define PCGCN_CE_WORK_FLOATS 1024
pcgcn_status pcgcn_softmax_ce(const float* L, int64_t ld, const int32_t* labels, const uint8_t* train,
                              int64_t M, int32_t C, float inv_nT, const float* s, float* dL,
                              float* loss, float* work /* DEVICE >= PCGCN_CE_WORK_FLOATS */,
                              void* stream);

/* Adam (β1, β2, ε as given; bias-corrected) on n fp32 parameters.  The
 * update uses t = *step + 1 and then stores t into *step (DEVICE i32), so a
 * captured CUDA graph replays correctly. */
pcgcn_status pcgcn_adam(float* theta, const float* grad, float* m, float* v, int64_t n, float lr,
                        float b1, float b2, float eps, int32_t* step, void* stream);
pcgcn_status pcgcn_sgd(float* theta, const float* grad, int64_t n, float lr, void* stream);

/* ---- introspection (tests / harness) ---- */

pcgcn_status pcgcn_plan_perm(pcgcn_plan_t p, int32_t* perm /* HOST [n], new -> old id */);
pcgcn_status pcgcn_plan_stats(pcgcn_plan_t p, pcgcn_stats* s);
const float* pcgcn_plan_rowscale(pcgcn_plan_t p); /* DEVICE [n] r = fp32(d̃^-½) in plan order */

/* bit-exact export of host plan arrays (compared with the oracle/plan.py spec) */
enum {
  PCGCN_X_PART = 0,      /* i32 [n]   partition of each ORIGINAL vertex id */
  PCGCN_X_PERM = 1,      /* i32 [n]   plan row -> original id */
  PCGCN_X_PSTART = 2,    /* i64 [P+1] first plan row of each partition */
  PCGCN_X_R = 3,         /* f32 [n]   r in plan order */
  PCGCN_X_BLK_K = 4,     /* i32 [nb]  non-empty blocks, sorted by (k, i) */
  PCGCN_X_BLK_I = 5,     /* i32 [nb] */
  PCGCN_X_BLK_NNZ = 6,   /* i64 [nb] */
  PCGCN_X_BLK_DENSE = 7, /* u8  [nb]  1 = full mode */
  PCGCN_X_SP_ROWPTR = 8, /* i64 [n+1] merged selective CSR (L179), plan ids */
  PCGCN_X_SP_COL = 9,    /* i32 [nnz_sparse] sources ascending per row */
  PCGCN_X_RT_ROW0 = 10,  /* i32 [nrt] first plan row of each dense row tile */
  PCGCN_X_RT_NROWS = 11, /* i32 [nrt] rows in the tile (<= 128) */
  PCGCN_X_RT_CPTR = 12,  /* i64 [nrt+1] chunk range of each row tile */
  PCGCN_X_CH_COL0 = 13,  /* i32 [nch] first plan column of each 128x32 chunk */
  PCGCN_X_BITS = 14,     /* u32 [nch*128] word r, bit b: edge (row0+r <- col0+b) */
  PCGCN_X_ZD_INDEX = 15, /* i32 [n] row of the dense partial-sum buffer, -1 if none */
  PCGCN_X_SWEEPS = 16,   /* i32 [1] */
  PCGCN_X_COUNT = 17
};
int64_t pcgcn_plan_export_bytes(pcgcn_plan_t p, int32_t which);   /* -1 on bad args */
pcgcn_status pcgcn_plan_export(pcgcn_plan_t p, int32_t which, void* host_buf, int64_t bytes);

/* θ calibration on the device (L161): times the selective and the full kernel
 * on synthetic P-sized blocks at density p_ref and width F and returns
 * θ = T_f·p_ref/T_s in *theta_out.  Synchronises its own stream. */
pcgcn_status pcgcn_calibrate(int32_t F, int32_t block_rows, float p_ref, float* theta_out,
                             float* t_full_ms, float* t_sel_ms);
/* The same with the full mode in dense_prec (PCGCN_DENSE_*; pcgcn_calibrate = TF32X2): one point
 * (p_ref, T_f, T_s) of the calibration curve T_s(ρ), T_f over densities and widths. */
pcgcn_status pcgcn_calibrate_prec(int32_t F, int32_t block_rows, float p_ref, int32_t dense_prec,
                                  float* theta_out, float* t_full_ms, float* t_sel_ms);

/* In-situ refinement of θ for one feature width F (the L161 procedure applied
 * to the workload itself): times the plan's full-mode tiles and selective
 * gather on the caller's (prescaled) input Y with PCGCN_PROFILE (median of 5),
 * derives the cost of one 128x32 full-mode chunk (c_chunk) and of one
 * selective edge (c_edge), and returns θ_F = c_chunk / (4096·c_edge): the block
 * density at which a chunk costs as much as its edges would in selective mode.
 * Needs a plan with both modes present (else returns the plan's θ).  Z is a
 * DEVICE scratch output [rows x F] (ld ldz).  Synchronises its own stream. */
pcgcn_status pcgcn_refine_theta(pcgcn_plan_t p, const float* Y, int64_t ldy, float* Z, int64_t ldz, int32_t F,
                                float* theta_out, float* c_chunk_ns, float* c_edge_ns);

const char* pcgcn_last_error(void);
/* optional device allocator hook (e.g. PyTorch's caching allocator); NULL => cudaMalloc/cudaFree */
void pcgcn_set_allocator(void* (*alloc)(size_t bytes, void* ctx), void (*release)(void* ptr, void* ctx),
                         void* ctx);
int32_t pcgcn_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* PCGCN_H */
