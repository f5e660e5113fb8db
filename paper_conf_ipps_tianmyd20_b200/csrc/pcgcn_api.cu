// C ABI of libpcgcn.so (include/pcgcn.h): plan lifetime, device upload,
// forward/backward orchestration (prescale/split -> full-mode tiles ->
// selective rows with the combine epilogue), and the GEMM / loss / optimiser
// entry points.  No CPU fallback: every device entry fails with PCGCN_ECUDA
// when no usable GPU is present.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>

#include "kernels.h"
#include "plan_internal.h"

namespace pcgcn {

namespace {
thread_local std::string g_err;
void* (*g_alloc)(size_t, void*) = nullptr;
void (*g_free)(void*, void*) = nullptr;
void* g_ctx = nullptr;

int64_t round_up(int64_t x, int64_t m) { return (x + m - 1) / m * m; }

pcgcn_status cuda_fail(cudaError_t e, const char* where) {
  set_error(std::string(where) + ": " + cudaGetErrorString(e));
  return PCGCN_ECUDA;
}

void* dev_alloc(size_t bytes) {
  if (bytes == 0) bytes = 16;
  if (g_alloc) return g_alloc(bytes, g_ctx);
  void* p = nullptr;
  if (cudaMalloc(&p, bytes) != cudaSuccess) return nullptr;
  return p;
}
void dev_free(void* p) {
  if (!p) return;
  if (g_free) g_free(p, g_ctx);
  else cudaFree(p);
}

template <class T>
pcgcn_status upload(DevicePlan& d, T** dst, const T* src, int64_t count) {
  *dst = static_cast<T*>(dev_alloc(sizeof(T) * std::max<int64_t>(count, 1)));
  if (!*dst) { set_error("device allocation failed"); return PCGCN_ENOMEM; }
  d.owned.push_back(*dst);
  d.bytes += int64_t(sizeof(T)) * std::max<int64_t>(count, 1);
  if (count > 0 && src) {
    cudaError_t e = cudaMemcpy(*dst, src, sizeof(T) * count, cudaMemcpyHostToDevice);
    if (e != cudaSuccess) return cuda_fail(e, "upload");
  }
  return PCGCN_OK;
}

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }
}  // namespace

void set_error(const std::string& msg) { g_err = msg; }

void free_device_plan(pcgcn_plan_s* p) {
  for (void*& ev : p->d.ev)
    if (ev) cudaEventDestroy(static_cast<cudaEvent_t>(ev));
  if (p->d.ev_fork) cudaEventDestroy(static_cast<cudaEvent_t>(p->d.ev_fork));
  if (p->d.ev_join) cudaEventDestroy(static_cast<cudaEvent_t>(p->d.ev_join));
  if (p->d.side) cudaStreamDestroy(static_cast<cudaStream_t>(p->d.side));
  for (void* q : p->d.owned) dev_free(q);
  p->d = DevicePlan();
}

pcgcn_status upload_plan(pcgcn_plan_s* p) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice (no usable GPU)");
  cudaDeviceProp prop;
  e = cudaGetDeviceProperties(&prop, dev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceProperties");
  if (prop.major < 10) {
    set_error("libpcgcn requires an sm_100 (B200) device");
    return PCGCN_ECUDA;
  }
  DevicePlan& d = p->d;
  const int64_t n = p->n;
  d.rows = p->row_hi - p->row_lo;
  d.nnz_s = p->sp_rowptr[p->row_hi] - p->sp_rowptr[p->row_lo];
  d.nrt = p->rt_hi - p->rt_lo;
  const int64_t ch_lo = p->rt_cptr[p->rt_lo], ch_hi = p->rt_cptr[p->rt_hi];
  d.nch = ch_hi - ch_lo;
  d.fpad_max = int(round_up(std::max(p->opts.f_max, 1), 16));
  d.n_pad = round_up(n, 32);  // row stride of the feature-major hi/lo split (zero-filled past n)
  pcgcn_status st;
#define UP(dst, src, cnt) \
  if ((st = upload(d, dst, src, cnt)) != PCGCN_OK) return st
  UP(&d.r, p->r.data(), n);
  std::vector<int64_t> rp(d.rows + 1);
  for (int64_t v = 0; v <= d.rows; ++v) rp[v] = p->sp_rowptr[p->row_lo + v] - p->sp_rowptr[p->row_lo];
  UP(&d.sp_rowptr, rp.data(), d.rows + 1);
  UP(&d.sp_col, p->sp_col.data() + p->sp_rowptr[p->row_lo], d.nnz_s);
  if (d.nch > 0) {
    std::vector<int32_t> zi(d.rows);
    const int64_t base = p->rt_lo * TILE_M;
    for (int64_t v = 0; v < d.rows; ++v) {
      int32_t z = p->zd_index[p->row_lo + v];
      zi[v] = z < 0 ? -1 : int32_t(z - base);
    }
    UP(&d.zd_index, zi.data(), d.rows);
    UP(&d.rt_row0, p->rt_row0.data() + p->rt_lo, d.nrt);
    UP(&d.rt_nrows, p->rt_nrows.data() + p->rt_lo, d.nrt);
    std::vector<int64_t> cp(d.nrt + 1);
    for (int64_t t = 0; t <= d.nrt; ++t) cp[t] = p->rt_cptr[p->rt_lo + t] - ch_lo;
    UP(&d.rt_cptr, cp.data(), d.nrt + 1);
    {
      // engine tile order: largest tiles first, dealt to the persistent CTAs
      // in snake order (CTA b takes positions b, 2G-1-b, 2G+b, ...), so the
      // static round-robin of the engine sees balanced chunk counts (plain
      // plan order left 8-18% of the full mode in the slowest CTA on C3)
      int dev = 0, sms = 148;
      cudaGetDevice(&dev);
      cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
      const int64_t G = std::min<int64_t>(d.nrt, sms > 0 ? sms : 148);
      std::vector<int32_t> bysize(d.nrt);
      for (int64_t t = 0; t < d.nrt; ++t) bysize[t] = int32_t(t);
      std::stable_sort(bysize.begin(), bysize.end(), [&](int32_t a, int32_t b) {
        return cp[a + 1] - cp[a] > cp[b + 1] - cp[b];
      });
      std::vector<int32_t> order(d.nrt);
      for (int64_t i = 0; i < d.nrt; ++i) {
        const int64_t round = i / G, k = i % G;
        const bool full_round = (round + 1) * G <= d.nrt;  // a partial last round stays in forward order
        const int64_t b = ((round & 1) && full_round) ? G - 1 - k : k;  // CTA receiving the i-th largest tile
        order[round * G + b] = bysize[i];
      }
      // PCGCN_TC_ORDER=plan (A/B knob): tiles in plan order, so the CTAs work on
      // neighbouring row tiles at the same time and share their source windows in L2
      if (const char* e = getenv("PCGCN_TC_ORDER"))
        if (std::string(e) == "plan")
          for (int64_t i = 0; i < d.nrt; ++i) order[i] = int32_t(i);
      UP(&d.rt_order, order.data(), d.nrt);
      UP(&d.rt_bysize, bysize.data(), d.nrt);
    }
    UP(&d.ch_col0, p->ch_col0.data() + ch_lo, d.nch);
    UP(&d.bits, p->bits.data() + ch_lo * TILE_M, d.nch * TILE_M);
    UP(&d.zd, (float*)nullptr, d.nrt * TILE_M * d.fpad_max);
    // the full mode's B: window blocks (or the feature-major split) of the whole
    // input — tf32 hi + lo: 2 floats per element, bf16x3: 3 bf16 = 1.5 floats,
    // bf16x1: 1; the CUDA-core full mode reads the input directly
    const int dp = p->opts.dense_prec;
    const int64_t half_floats = dp == PCGCN_DENSE_BF16X3 ? 3 : dp == PCGCN_DENSE_BF16X1 ? 2
                              : dp == PCGCN_DENSE_FP32_SIMT ? 0 : 4;
    if (half_floats > 0) UP(&d.yhi, (float*)nullptr, half_floats * d.n_pad * d.fpad_max / 2);
  }
  // (ypre, the prescaled copy of an un-prescaled input, is allocated by the
  // first forward/backward call without PCGCN_IN_PRESCALED)
  UP(&d.zrow, (float*)nullptr, 256);
  if (p->opts.world > 1) {
    std::vector<int32_t> sl, rl;
    for (auto& l : p->halo_send) sl.insert(sl.end(), l.begin(), l.end());
    for (auto& l : p->halo_recv) rl.insert(rl.end(), l.begin(), l.end());
    d.halo_nsend = int64_t(sl.size());
    d.halo_nrecv = int64_t(rl.size());
    UP(&d.halo_send, sl.data(), d.halo_nsend);
    UP(&d.halo_recv, rl.data(), d.halo_nrecv);
  }
  UP(&d.counter, (int*)nullptr, 32);
  {
    // long selective rows -> segments of SEG_EDGES edges (reading #22)
    std::vector<int32_t> rs(d.rows, -1), srow;
    std::vector<int64_t> lo, hi;
    for (int64_t v = 0; v < d.rows; ++v) {
      if (rp[v + 1] - rp[v] <= SEG_EDGES) continue;
      rs[v] = int32_t(lo.size());
      for (int64_t e = rp[v]; e < rp[v + 1]; e += SEG_EDGES) {
        lo.push_back(e);
        hi.push_back(std::min<int64_t>(e + SEG_EDGES, rp[v + 1]));
        srow.push_back(int32_t(v));
      }
    }
    d.nseg = int64_t(lo.size());
    if (d.nseg > 0) {
      UP(&d.row_seg, rs.data(), d.rows);
      UP(&d.seg_lo, lo.data(), d.nseg);
      UP(&d.seg_hi, hi.data(), d.nseg);
      UP(&d.seg_ws, (float*)nullptr, d.nseg * d.fpad_max);
      UP(&d.seg_row, srow.data(), d.nseg);
      UP(&d.seg_cnt, (int32_t*)nullptr, d.nseg);
      if ((e = cudaMemset(d.seg_cnt, 0, d.nseg * sizeof(int32_t))) != cudaSuccess) return cuda_fail(e, "memset");
    }
  }
#undef UP
  e = cudaMemset(d.zrow, 0, 256 * sizeof(float));
  if (e != cudaSuccess) return cuda_fail(e, "memset");
  if (d.nseg > 0 && d.nch > 0) {
    // high-priority side stream for the split + full-mode tiles, which run
    // concurrently with the long-row segment pass on the caller's stream (the
    // two are independent; fork/join by events, CUDA-graph capturable); the
    // priority lets the engine's CTAs claim SMs first, segment CTAs fill in
    cudaStream_t side;
    cudaEvent_t f, j;
    int lo_pri = 0, hi_pri = 0;
    cudaDeviceGetStreamPriorityRange(&lo_pri, &hi_pri);
    if ((e = cudaStreamCreateWithPriority(&side, cudaStreamNonBlocking, hi_pri)) != cudaSuccess)
      return cuda_fail(e, "side stream");
    d.side = side;
    if ((e = cudaEventCreateWithFlags(&f, cudaEventDisableTiming)) != cudaSuccess) return cuda_fail(e, "event");
    d.ev_fork = f;
    if ((e = cudaEventCreateWithFlags(&j, cudaEventDisableTiming)) != cudaSuccess) return cuda_fail(e, "event");
    d.ev_join = j;
  }
  d.built = true;
  p->stats.device_bytes = d.bytes;
  p->stats.shard_segments = d.nseg;
  return PCGCN_OK;
}

namespace {

// PCGCN_OVERLAP=1 runs the split + full-mode tiles on a high-priority side stream
// concurrently with the segment pass (measured on C3: no gain, 9.85 vs 9.62 ms
// epoch; the engine CTAs leave too few registers for co-resident gathers)
bool overlap_enabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("PCGCN_OVERLAP");
    v = e ? (atoi(e) != 0) : 0;
  }
  return v != 0;
}

// PCGCN_DENSE_BLOCKED=0: full-mode B through strided TMA boxes of the
// feature-major split instead of window blocks (A/B knob, benchmarks only)
bool dense_blocked_enabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("PCGCN_DENSE_BLOCKED");
    v = e ? (atoi(e) != 0) : 1;
  }
  return v != 0;
}

// full-mode tiles claimed dynamically in plan order (default): the CTAs work on
// neighbouring row tiles, whose source windows then hit in L2 (C3 F=128: DRAM
// reads 610 -> 265 MB, 0.55 -> 0.45 ms); PCGCN_TC_DYN=0 restores the static
// balanced snake order (A/B knob; bitwise identical results)
bool tc_dyn_enabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("PCGCN_TC_DYN");
    v = e ? (atoi(e) != 0) : 1;
  }
  return v != 0;
}

// dynamic full-mode tile claims, largest tile first (longest-processing-time
// order: C3's largest row tile holds ~the mean CTA share of chunks, and claimed
// late in plan order it set the kernel's tail): measured C3 full mode F=128
// 0.457 -> 0.399 ms, F=41 0.250 -> 0.204 ms.  PCGCN_TC_DYN_ORDER=plan (A/B
// knob): claims in plan order (neighbouring tiles share source windows in L2)
bool tc_dyn_order_size() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("PCGCN_TC_DYN_ORDER");
    v = (e && std::string(e) == "plan") ? 0 : 1;
  }
  return v != 0;
}

// rows per scheduler ticket: enough that a ticket covers ~128 selective edges
// (C5's mean degree 31 -> 8: the next ticket and row pointers are then fetched
// while the block's rows gather; measured C5 epoch 250 -> 206 ms), 1 for long
// rows (C3's mean 348: R = 4 measured 2.5% slower there), at most 16
// (PCGCN_ROWS_PER_TICKET overrides; benchmarks only)
int rows_per_ticket(int64_t nnz_s, int64_t rows) {
  static int env = -1;
  if (env < 0) {
    const char* e = getenv("PCGCN_ROWS_PER_TICKET");
    env = e ? atoi(e) : 0;
  }
  int R = 1;
  if (env > 0) {
    R = env;
  } else if (rows > 0) {
    const double deg = double(nnz_s) / double(rows);
    while (R < 16 && deg * R < 128.0) R *= 2;
  }
  return R < 1 ? 1 : (R > 16 ? 16 : R);
}

// the plan's full-mode window-block target for a producer of width F (fused
// split); false if the plan has no chunks on this device / precision
bool window_out(pcgcn_plan_t p, int32_t F, WindowOut* wo) {
  const DevicePlan& d = p->d;
  const int dp = p->opts.dense_prec;
  if (!d.built || d.nch == 0 || !d.yhi || dp == PCGCN_DENSE_FP32_SIMT) return false;
  if (dp == PCGCN_DENSE_TF32X2 && (!dense_blocked_enabled() || dense_pair_eligible(int(round_up(F, 16)))))
    return false;
  const int64_t npad = round_up(F, 16);
  wo->blk = d.yhi;
  wo->mode = dp == PCGCN_DENSE_BF16X3 ? 3 : dp == PCGCN_DENSE_BF16X1 ? 4 : 1;
  wo->blk_floats = dp == PCGCN_DENSE_BF16X3 ? npad * 48 : dp == PCGCN_DENSE_BF16X1 ? npad * 16 : 2 * npad * 32;
  wo->nwin = d.n_pad / 32;
  return true;
}

pcgcn_status aggregate(pcgcn_plan_t p, const float* Y, int64_t ldy, float* Z, int64_t ldz, int32_t F,
                       uint32_t flags, uint32_t* mask, void* stream) {
  if (!p || !p->d.built) { set_error("plan has no device structures"); return PCGCN_EINVAL; }
  if (!Y || !Z || F < 1 || F > p->opts.f_max || ldy < round_up(F, 4) || ldz < round_up(F, 4) ||
      (ldy & 3) || (ldz & 3) || !aligned16(Y) || !aligned16(Z)) {
    set_error("forward/backward: bad Y/Z/F/ld (ld >= roundup(F,4), 16-byte aligned rows, F <= f_max)");
    return PCGCN_EINVAL;
  }
  if ((flags & PCGCN_MASK_OUT) && !mask) { set_error("MASK_OUT needs a mask buffer"); return PCGCN_EINVAL; }
  if ((flags & PCGCN_IN_SPLIT) && !(flags & PCGCN_IN_PRESCALED)) {
    set_error("IN_SPLIT requires IN_PRESCALED (the fused split writes the prescaled producer output)");
    return PCGCN_EINVAL;
  }
  DevicePlan& d = p->d;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  cudaError_t e;
  const bool dense = d.nch > 0;
  const bool prescaled = (flags & PCGCN_IN_PRESCALED) != 0;
  const int npad = int(round_up(F, 16));
  const int64_t ld4 = round_up(F, 4);
  const float* src = Y;
  int64_t ldsrc = ldy;
  const bool bf16 = p->opts.dense_prec == PCGCN_DENSE_BF16X1;
  const bool bf3 = p->opts.dense_prec == PCGCN_DENSE_BF16X3;
  const bool tc = p->opts.dense_prec == PCGCN_DENSE_TF32X2 || bf16 || bf3;
  const bool prof = (flags & PCGCN_PROFILE) != 0;
  auto mark = [&](int k) {
    if (!prof) return;
    if (!d.ev[k]) cudaEventCreate(reinterpret_cast<cudaEvent_t*>(&d.ev[k]));
    cudaEventRecord(static_cast<cudaEvent_t>(d.ev[k]), s);
  };
  if (prof) for (int k = 0; k < 4; ++k) d.ev_used[k] = false;
  mark(0);
  if (!prescaled) {
    if (!d.ypre) {
      // first un-prescaled call: the prescale workspace (n x fpad_max floats);
      // not capturable — calls inside a CUDA graph pass prescaled inputs
      d.ypre = static_cast<float*>(dev_alloc(sizeof(float) * size_t(std::max<int64_t>(p->n * d.fpad_max, 1))));
      if (!d.ypre) { set_error("device allocation of the prescale workspace failed"); return PCGCN_ENOMEM; }
      d.owned.push_back(d.ypre);
      d.bytes += int64_t(sizeof(float)) * p->n * d.fpad_max;
      p->stats.device_bytes = d.bytes;
    }
    if (prof) d.ev_used[0] = true;
    e = launch_prescale(Y, ldy, d.r, p->n, F, d.ypre, ld4, s);
    if (e != cudaSuccess) return cuda_fail(e, "prescale");
    src = d.ypre;
    ldsrc = ld4;
  }
  mark(1);
  AggArgs a;
  a.Y = src; a.ldy = ldsrc; a.Z = Z; a.ldz = ldz;
  a.mask = (flags & PCGCN_MASK_OUT) ? mask : nullptr;
  a.rowptr = d.sp_rowptr; a.col = d.sp_col; a.r = d.r;
  a.row_lo = p->row_lo; a.rows = d.rows;
  a.zd_index = dense ? d.zd_index : nullptr;
  a.zd = d.zd; a.ldzd = npad;
  a.zrow = d.zrow;
  a.mask_ld = (F + 31) / 32;
  a.n_src = p->n;
  a.F = F;
  a.relu = (flags & PCGCN_RELU) != 0;
  a.out_prescaled = (flags & PCGCN_OUT_PRESCALED) != 0;
  a.row_seg = d.row_seg; a.seg_lo = d.seg_lo; a.seg_hi = d.seg_hi; a.nseg = d.nseg;
  a.seg_row = d.seg_row; a.seg_cnt = d.seg_cnt; a.seg_ticket = d.counter + 8;
  a.seg_ws = d.seg_ws; a.ldws = d.fpad_max;
  a.counter = d.counter;
  a.rows_per_ticket = rows_per_ticket(d.nnz_s, d.rows);
  a.mean_deg = float(double(p->sp_rowptr[p->n]) / double(p->n));  // plan-global: every shard picks the same layout
  a.rows_by_degree = p->opts.vertex_order == PCGCN_ORDER_DEGREE ? 1 : 0;
  // the split + full-mode tiles run on the plan's high-priority side stream,
  // concurrently with the long-row segment pass on the caller's stream;
  // PROFILE calls stay serial so per-kernel times add up
  const bool overlap = overlap_enabled() && !prof && dense && d.nseg > 0 && d.side && d.rows > 0 &&
                       !sparse_fsplit_active(F);
  cudaStream_t ms = s;  // stream of the full-mode work
  if (overlap) {
    cudaStream_t side = static_cast<cudaStream_t>(d.side);
    cudaEvent_t ef = static_cast<cudaEvent_t>(d.ev_fork);
    if ((e = cudaEventRecord(ef, s)) != cudaSuccess) return cuda_fail(e, "fork");
    if ((e = cudaStreamWaitEvent(side, ef, 0)) != cudaSuccess) return cuda_fail(e, "fork");
    ms = side;
  }
  float* ylo = d.yhi ? d.yhi + int64_t(npad) * d.n_pad : nullptr;
  // full mode's B: source-window blocks fetched by one bulk copy per chunk
  // (default), or the feature-major split read by strided TMA boxes (the
  // CTA-pair kernel, or PCGCN_DENSE_BLOCKED=0)
  const bool blocked = bf3 || bf16 || (tc && dense_blocked_enabled() && !dense_pair_eligible(npad));
  // IN_SPLIT: the producer already wrote the window blocks (pcgcn_gemm_*_split
  // writes them exactly when the full mode uses window blocks)
  const bool presplit = (flags & PCGCN_IN_SPLIT) && blocked;
  if (dense && tc && !presplit) {
    if (prof) d.ev_used[1] = true;
    e = blocked ? launch_split_windows(src, ldsrc, p->n, F, npad, bf3 ? 2 : (bf16 ? 3 : 0), d.yhi, d.n_pad / 32, ms)
                : launch_split_transpose(src, ldsrc, p->n, F, npad, d.yhi, bf16 ? nullptr : ylo, d.n_pad, ms);
    if (e != cudaSuccess) return cuda_fail(e, "split_transpose");
  }
  mark(2);
  if (dense) {
    if (prof) d.ev_used[2] = true;
    DenseArgs da{d.yhi, bf16 ? nullptr : ylo, d.n_pad, d.n_pad, d.rt_row0, d.rt_nrows, d.rt_cptr, d.ch_col0,
                 d.bits, d.nrt, d.zd, npad, npad};
    da.rt_order = d.rt_order;
    da.n_src = p->n;
    if (blocked && tc_dyn_enabled()) {
      // tiles claimed dynamically, in plan order: neighbouring row tiles (and
      // their source windows) are in flight together, balance comes from the claims
      da.dyn = d.counter + 16;
      da.rt_order = tc_dyn_order_size() ? d.rt_bysize : nullptr;
      if ((e = cudaMemsetAsync(da.dyn, 0, sizeof(int), ms)) != cudaSuccess) return cuda_fail(e, "memset");
    }
    if (blocked) {
      da.blk = d.yhi;
      da.blk_floats = bf3 ? int64_t(npad) * 48 : bf16 ? int64_t(npad) * 16 : int64_t(2) * npad * 32;
      da.bf3 = bf3 ? 3 : (bf16 ? 1 : 0);  // bf16 parts of B (kind::f16)
    }
    e = tc ? launch_dense_tc(da, ms) : launch_dense_simt_y(da, src, ldsrc, F, ms);
    if (e != cudaSuccess) return cuda_fail(e, "dense-mode kernel");
  }
  if (overlap) {
    if ((e = cudaEventRecord(static_cast<cudaEvent_t>(d.ev_join), ms)) != cudaSuccess) return cuda_fail(e, "join");
    AggArgs sa = a;
    sa.phase = 1;
    if ((e = launch_sparse_agg(sa, s)) != cudaSuccess) return cuda_fail(e, "segment pass");
  }
  mark(3);
  if (prof) d.ev_used[3] = true;
  if (overlap) {
    if ((e = cudaStreamWaitEvent(s, static_cast<cudaEvent_t>(d.ev_join), 0)) != cudaSuccess)
      return cuda_fail(e, "join");
    a.phase = 2;
  }
  e = launch_sparse_agg(a, s);
  if (e != cudaSuccess) return cuda_fail(e, "selective-mode kernel");
  mark(4);
  return PCGCN_OK;
}

}  // namespace
}  // namespace pcgcn

using namespace pcgcn;

extern "C" {

int32_t pcgcn_abi_version(void) { return 2; }

const char* pcgcn_last_error(void) { return g_err.c_str(); }

void pcgcn_set_allocator(void* (*alloc)(size_t, void*), void (*release)(void*, void*), void* ctx) {
  g_alloc = alloc;
  g_free = release;
  g_ctx = ctx;
}

void pcgcn_opts_default(pcgcn_opts* o) {
  if (!o) return;
  std::memset(o, 0, sizeof(*o));
  o->norm = PCGCN_NORM_SYM;
  o->dense_prec = PCGCN_DENSE_TF32X2;
  o->f_max = 128;
  o->lp_sweeps = 10;
  o->part = nullptr;
  o->build_device = 1;
  o->rank = 0;
  o->world = 1;
}

pcgcn_status pcgcn_plan(const pcgcn_csr* A, int32_t P, float theta, const pcgcn_opts* o,
                        pcgcn_plan_t* out) {
  if (!A || !out) { set_error("pcgcn_plan: null argument"); return PCGCN_EINVAL; }
  *out = nullptr;
  pcgcn_opts def;
  pcgcn_opts_default(&def);
  if (!o) o = &def;
  if (o->f_max < 1 || o->f_max > 256) { set_error("f_max must be in [1, 256]"); return PCGCN_EINVAL; }
  if (o->dense_prec != PCGCN_DENSE_TF32X2 && o->dense_prec != PCGCN_DENSE_FP32_SIMT &&
      o->dense_prec != PCGCN_DENSE_BF16X1 && o->dense_prec != PCGCN_DENSE_BF16X3) {
    set_error("unknown dense_prec");
    return PCGCN_EUNSUP;
  }
  if ((o->vertex_order != PCGCN_ORDER_ID && o->vertex_order != PCGCN_ORDER_DEGREE) ||
      (o->mode_grain != PCGCN_GRAIN_BLOCK && o->mode_grain != PCGCN_GRAIN_TILE)) {
    set_error("unknown vertex_order / mode_grain");
    return PCGCN_EUNSUP;
  }
  if (!(theta >= 0.f)) {
    // θ < 0: the L161 procedure on this device first (synthetic p = 0.05 blocks
    // of the plan's mean partition size, width f_max)
    if (!o->build_device || std::isnan(theta)) {
      set_error("theta < 0 (calibrate on the device) needs build_device = 1");
      return PCGCN_EINVAL;
    }
    const int64_t rows = A->n / (P > 0 ? P : 1);
    float th = 0.f, tf = 0.f, ts = 0.f;
    pcgcn_status cs = pcgcn_calibrate(o->f_max, int32_t(std::max<int64_t>(64, std::min<int64_t>(8192, rows))),
                                      0.05f, &th, &tf, &ts);
    if (cs != PCGCN_OK) return cs;
    theta = th;
  }
  if (o->dense_prec == PCGCN_DENSE_FP32_SIMT && o->f_max > 128) {
    set_error("FP32_SIMT full mode supports F <= 128");
    return PCGCN_EUNSUP;
  }
  pcgcn_plan_s* p = new (std::nothrow) pcgcn_plan_s();
  if (!p) { set_error("out of host memory"); return PCGCN_ENOMEM; }
  pcgcn_status st;
  try {
    st = build_host_plan(A, P, theta, o, p);
  } catch (const std::bad_alloc&) {
    st = PCGCN_ENOMEM;
    set_error("out of host memory in planner");
  } catch (...) {
    st = PCGCN_EINVAL;
    set_error("planner failure");
  }
  if (st == PCGCN_OK && o->build_device) st = upload_plan(p);
  if (st != PCGCN_OK) {
    free_device_plan(p);
    delete p;
    return st;
  }
  p->opts.part = nullptr;  // borrowed pointer: do not keep
  *out = p;
  return PCGCN_OK;
}

void pcgcn_destroy(pcgcn_plan_t p) {
  if (!p) return;
  free_device_plan(p);
  delete p;
}

pcgcn_status pcgcn_forward(pcgcn_plan_t p, const float* Y, int64_t ldy, float* Z, int64_t ldz,
                           int32_t F, uint32_t flags, uint32_t* mask, void* stream) {
  return aggregate(p, Y, ldy, Z, ldz, F, flags, mask, stream);
}

pcgcn_status pcgcn_backward(pcgcn_plan_t p, const float* dZ, int64_t ldz, float* dY, int64_t ldy,
                            int32_t F, uint32_t flags, void* stream) {
  // Âᵀ = Â for a symmetric input: the forward plan serves the backward.
  return aggregate(p, dZ, ldz, dY, ldy, F, flags & ~uint32_t(PCGCN_MASK_OUT), nullptr, stream);
}

int64_t pcgcn_plan_halo_rows(pcgcn_plan_t p, int32_t q, int32_t send) {
  if (!p || q < 0 || q >= p->opts.world) return -1;
  if (p->opts.world == 1) return 0;
  return int64_t((send ? p->halo_send : p->halo_recv)[q].size());
}

pcgcn_status pcgcn_plan_halo_export(pcgcn_plan_t p, int32_t q, int32_t send, int32_t* buf, int64_t cap) {
  const int64_t n = pcgcn_plan_halo_rows(p, q, send);
  if (n < 0 || (n > 0 && (!buf || cap < n))) { set_error("plan_halo_export: bad peer / buffer"); return PCGCN_EINVAL; }
  if (n > 0) std::memcpy(buf, (send ? p->halo_send : p->halo_recv)[q].data(), sizeof(int32_t) * size_t(n));
  return PCGCN_OK;
}

pcgcn_status pcgcn_plan_shard_rows(pcgcn_plan_t p, int64_t* row0) {
  if (!p || !row0) { set_error("null argument"); return PCGCN_EINVAL; }
  if (p->shard_row0.empty()) { row0[0] = 0; row0[1] = p->n; return PCGCN_OK; }
  std::memcpy(row0, p->shard_row0.data(), sizeof(int64_t) * p->shard_row0.size());
  return PCGCN_OK;
}

static pcgcn_status halo_copy(pcgcn_plan_t p, bool pack, const float* src, int64_t lds, float* dst, int64_t ldd,
                              int32_t w, void* stream) {
  if (!p || !p->d.built) { set_error("plan has no device structures"); return PCGCN_EINVAL; }
  const int64_t rows = pack ? p->d.halo_nsend : p->d.halo_nrecv;
  if (rows == 0) return PCGCN_OK;
  if (!src || !dst || w < 4 || (w & 3) || lds < w || ldd < w || (lds & 3) || (ldd & 3) ||
      (reinterpret_cast<uintptr_t>(src) & 15) || (reinterpret_cast<uintptr_t>(dst) & 15)) {
    set_error("halo pack/unpack: bad buffers (w multiple of 4, ld >= w, 16-byte aligned rows)");
    return PCGCN_EINVAL;
  }
  cudaError_t e = launch_halo_copy(pack, src, lds, dst, ldd, pack ? p->d.halo_send : p->d.halo_recv, rows, w,
                                   static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, pack ? "halo_pack" : "halo_unpack");
}

pcgcn_status pcgcn_halo_pack(pcgcn_plan_t p, const float* Y, int64_t ldy, int32_t w, float* buf, void* stream) {
  return halo_copy(p, true, Y, ldy, buf, w, w, stream);
}

pcgcn_status pcgcn_halo_unpack(pcgcn_plan_t p, const float* buf, float* Y, int64_t ldy, int32_t w, void* stream) {
  return halo_copy(p, false, buf, w, Y, ldy, w, stream);
}

// ---- device-initiated peer gather ----
static pcgcn_status aggregate_peer(pcgcn_plan_t p, const float* const* peer, int64_t ldy, float* Z, int64_t ldz,
                                   int32_t F, uint32_t flags, uint32_t* mask, void* stream) {
  if (!p || !p->d.built) { set_error("plan has no device structures"); return PCGCN_EINVAL; }
  const int32_t W = p->opts.world;
  if (!peer || W < 1 || W > 8) { set_error("forward_peer: peer table of 1..8 shards required"); return PCGCN_EINVAL; }
  if (!(flags & PCGCN_IN_PRESCALED)) { set_error("forward_peer: inputs must be prescaled (IN_PRESCALED)"); return PCGCN_EINVAL; }
  if (p->d.nch > 0) { set_error("forward_peer: the shard has full-mode chunks (selective-only plans)"); return PCGCN_EUNSUP; }
  if (sparse_fsplit_active(F)) { set_error("forward_peer: PCGCN_SPARSE_FSPLIT not supported"); return PCGCN_EUNSUP; }
  if (!Z || F < 1 || F > p->opts.f_max || ldy < round_up(F, 4) || ldz < round_up(F, 4) || (ldy & 3) || (ldz & 3) ||
      !aligned16(Z)) {
    set_error("forward_peer: bad Z/F/ld");
    return PCGCN_EINVAL;
  }
  if ((flags & PCGCN_MASK_OUT) && !mask) { set_error("MASK_OUT needs a mask buffer"); return PCGCN_EINVAL; }
  DevicePlan& d = p->d;
  AggArgs a;
  a.Y = nullptr; a.ldy = ldy; a.Z = Z; a.ldz = ldz;
  a.mask = (flags & PCGCN_MASK_OUT) ? mask : nullptr;
  a.rowptr = d.sp_rowptr; a.col = d.sp_col; a.r = d.r;
  a.row_lo = p->row_lo; a.rows = d.rows;
  a.zd_index = nullptr; a.zd = nullptr; a.ldzd = 0; a.zrow = d.zrow;
  a.mask_ld = (F + 31) / 32;
  a.n_src = p->n;
  a.F = F;
  a.relu = (flags & PCGCN_RELU) != 0;
  a.out_prescaled = (flags & PCGCN_OUT_PRESCALED) != 0;
  a.row_seg = d.row_seg; a.seg_lo = d.seg_lo; a.seg_hi = d.seg_hi; a.nseg = d.nseg;
  a.seg_row = d.seg_row; a.seg_cnt = d.seg_cnt; a.seg_ticket = d.counter + 8;
  a.seg_ws = d.seg_ws; a.ldws = d.fpad_max;
  a.counter = d.counter;
  a.rows_per_ticket = rows_per_ticket(d.nnz_s, d.rows);
  a.mean_deg = float(double(p->sp_rowptr[p->n]) / double(p->n));  // plan-global: every shard picks the same layout
  a.rows_by_degree = p->opts.vertex_order == PCGCN_ORDER_DEGREE ? 1 : 0;
  a.peer_world = W;
  for (int q = 0; q < 8; ++q) a.peer_base[q] = q < W ? reinterpret_cast<const char*>(peer[q]) : nullptr;
  for (int q = 0; q <= 8; ++q)
    a.peer_row0[q] = W == 1 ? (q == 0 ? 0 : p->n) : p->shard_row0[std::min<int32_t>(q, W)];
  for (int q = 0; q < W; ++q)
    if (!a.peer_base[q] || (reinterpret_cast<uintptr_t>(a.peer_base[q]) & 31)) {
      set_error("forward_peer: null or not 32-byte aligned peer buffer");
      return PCGCN_EINVAL;
    }
  cudaError_t e = launch_sparse_agg(a, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "forward_peer");
}

pcgcn_status pcgcn_forward_peer(pcgcn_plan_t p, const float* const* peer_Y, int64_t ldy, float* Z, int64_t ldz,
                                int32_t F, uint32_t flags, uint32_t* mask, void* stream) {
  return aggregate_peer(p, peer_Y, ldy, Z, ldz, F, flags, mask, stream);
}

pcgcn_status pcgcn_backward_peer(pcgcn_plan_t p, const float* const* peer_dZ, int64_t ldz, float* dY, int64_t ldy,
                                 int32_t F, uint32_t flags, void* stream) {
  return aggregate_peer(p, peer_dZ, ldz, dY, ldy, F, flags & ~uint32_t(PCGCN_MASK_OUT), nullptr, stream);
}

// ---- CUDA IPC helpers (peer buffers across processes) ----
pcgcn_status pcgcn_ipc_alloc(int64_t bytes, void** ptr) {
  if (!ptr || bytes <= 0) { set_error("ipc_alloc: bad arguments"); return PCGCN_EINVAL; }
  cudaError_t e = cudaMalloc(ptr, size_t(bytes));
  if (e != cudaSuccess) return cuda_fail(e, "ipc_alloc");
  e = cudaMemset(*ptr, 0, size_t(bytes));
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "ipc_alloc memset");
}
void pcgcn_ipc_free(void* ptr) { if (ptr) cudaFree(ptr); }
pcgcn_status pcgcn_ipc_handle(void* ptr, void* handle64) {
  if (!ptr || !handle64) { set_error("ipc_handle: null argument"); return PCGCN_EINVAL; }
  cudaIpcMemHandle_t h;
  cudaError_t e = cudaIpcGetMemHandle(&h, ptr);
  if (e != cudaSuccess) return cuda_fail(e, "cudaIpcGetMemHandle");
  static_assert(sizeof(h) == 64, "cudaIpcMemHandle_t is 64 bytes");
  std::memcpy(handle64, &h, 64);
  return PCGCN_OK;
}
pcgcn_status pcgcn_ipc_open(const void* handle64, void** ptr) {
  if (!ptr || !handle64) { set_error("ipc_open: null argument"); return PCGCN_EINVAL; }
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle64, 64);
  cudaError_t e = cudaIpcOpenMemHandle(ptr, h, cudaIpcMemLazyEnablePeerAccess);
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "cudaIpcOpenMemHandle");
}
void pcgcn_ipc_close(void* ptr) { if (ptr) cudaIpcCloseMemHandle(ptr); }

pcgcn_status pcgcn_plan_perm(pcgcn_plan_t p, int32_t* perm) {
  if (!p || !perm) { set_error("null argument"); return PCGCN_EINVAL; }
  std::memcpy(perm, p->perm.data(), sizeof(int32_t) * p->n);
  return PCGCN_OK;
}

pcgcn_status pcgcn_plan_stats(pcgcn_plan_t p, pcgcn_stats* s) {
  if (!p || !s) { set_error("null argument"); return PCGCN_EINVAL; }
  *s = p->stats;
  return PCGCN_OK;
}

const float* pcgcn_plan_rowscale(pcgcn_plan_t p) { return p && p->d.built ? p->d.r : nullptr; }

pcgcn_status pcgcn_plan_last_timings(pcgcn_plan_t p, float ms[4]) {
  if (!p || !ms) { set_error("null argument"); return PCGCN_EINVAL; }
  for (int k = 0; k < 4; ++k) {
    ms[k] = 0.f;
    if (!p->d.ev_used[k] || !p->d.ev[k] || !p->d.ev[k + 1]) continue;
    cudaEvent_t a = static_cast<cudaEvent_t>(p->d.ev[k]), b = static_cast<cudaEvent_t>(p->d.ev[k + 1]);
    cudaError_t e = cudaEventSynchronize(b);
    if (e == cudaSuccess) e = cudaEventElapsedTime(&ms[k], a, b);
    if (e != cudaSuccess) return cuda_fail(e, "plan_last_timings");
  }
  return PCGCN_OK;
}

int64_t pcgcn_plan_export_bytes(pcgcn_plan_t p, int32_t which) {
  if (!p) return -1;
  switch (which) {
    case PCGCN_X_PART: return 4 * int64_t(p->part.size());
    case PCGCN_X_PERM: return 4 * int64_t(p->perm.size());
    case PCGCN_X_PSTART: return 8 * int64_t(p->pstart.size());
    case PCGCN_X_R: return 4 * int64_t(p->r.size());
    case PCGCN_X_BLK_K: return 4 * int64_t(p->blk_k.size());
    case PCGCN_X_BLK_I: return 4 * int64_t(p->blk_i.size());
    case PCGCN_X_BLK_NNZ: return 8 * int64_t(p->blk_nnz.size());
    case PCGCN_X_BLK_DENSE: return int64_t(p->blk_dense.size());
    case PCGCN_X_SP_ROWPTR: return 8 * int64_t(p->sp_rowptr.size());
    case PCGCN_X_SP_COL: return 4 * int64_t(p->sp_col.size());
    case PCGCN_X_RT_ROW0: return 4 * int64_t(p->rt_row0.size());
    case PCGCN_X_RT_NROWS: return 4 * int64_t(p->rt_nrows.size());
    case PCGCN_X_RT_CPTR: return 8 * int64_t(p->rt_cptr.size());
    case PCGCN_X_CH_COL0: return 4 * int64_t(p->ch_col0.size());
    case PCGCN_X_BITS: return 4 * int64_t(p->bits.size());
    case PCGCN_X_ZD_INDEX: return 4 * int64_t(p->zd_index.size());
    case PCGCN_X_SWEEPS: return 4;
    default: return -1;
  }
}

pcgcn_status pcgcn_plan_export(pcgcn_plan_t p, int32_t which, void* buf, int64_t bytes) {
  int64_t need = pcgcn_plan_export_bytes(p, which);
  if (need < 0 || !buf || bytes < need) { set_error("plan_export: bad which / buffer"); return PCGCN_EINVAL; }
  const void* src = nullptr;
  switch (which) {
    case PCGCN_X_PART: src = p->part.data(); break;
    case PCGCN_X_PERM: src = p->perm.data(); break;
    case PCGCN_X_PSTART: src = p->pstart.data(); break;
    case PCGCN_X_R: src = p->r.data(); break;
    case PCGCN_X_BLK_K: src = p->blk_k.data(); break;
    case PCGCN_X_BLK_I: src = p->blk_i.data(); break;
    case PCGCN_X_BLK_NNZ: src = p->blk_nnz.data(); break;
    case PCGCN_X_BLK_DENSE: src = p->blk_dense.data(); break;
    case PCGCN_X_SP_ROWPTR: src = p->sp_rowptr.data(); break;
    case PCGCN_X_SP_COL: src = p->sp_col.data(); break;
    case PCGCN_X_RT_ROW0: src = p->rt_row0.data(); break;
    case PCGCN_X_RT_NROWS: src = p->rt_nrows.data(); break;
    case PCGCN_X_RT_CPTR: src = p->rt_cptr.data(); break;
    case PCGCN_X_CH_COL0: src = p->ch_col0.data(); break;
    case PCGCN_X_BITS: src = p->bits.data(); break;
    case PCGCN_X_ZD_INDEX: src = p->zd_index.data(); break;
    case PCGCN_X_SWEEPS: src = &p->sweeps; break;
  }
  if (need > 0) std::memcpy(buf, src, size_t(need));
  return PCGCN_OK;
}

int64_t pcgcn_gemm_xw_work_floats(int32_t K, int32_t N) { return gemm_xw_work_floats(K, N); }

pcgcn_status pcgcn_gemm_xw(const float* X, int64_t ldx, const float* W, int64_t ldw, const float* s,
                           float* Y, int64_t ldy, int64_t M, int32_t K, int32_t N, float* work, void* stream) {
  if (!X || !W || !Y || M < 0 || K < 1 || N < 1 || ldx < K || ldw < N || ldy < N) {
    set_error("gemm_xw: bad arguments");
    return PCGCN_EINVAL;
  }
  cudaError_t e = launch_gemm_xw(X, ldx, W, ldw, s, Y, ldy, M, K, N, work, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "gemm_xw");
}

static pcgcn_status split_target(pcgcn_plan_t p, int64_t M, int32_t F, const float* work, int64_t ldx, int64_t ldy,
                                 WindowOut* wo, bool* any) {
  *any = false;
  if (!p || !p->d.built) { set_error("gemm *_split: plan has no device structures"); return PCGCN_EINVAL; }
  if (p->opts.world != 1 || M != p->n) {
    set_error("gemm *_split: unsharded plan and all n rows only (a sharded input is split after its exchange)");
    return PCGCN_EINVAL;
  }
  if (F > p->opts.f_max || F > 128) { set_error("gemm *_split: F > f_max or > 128"); return PCGCN_EINVAL; }
  *any = window_out(p, F, wo);
  if (*any && (!work || (ldx & 3) || (ldy & 3))) {
    set_error("gemm *_split: needs the tcgen05 path (work buffer, ld multiples of 4)");
    return PCGCN_EINVAL;
  }
  return PCGCN_OK;
}

pcgcn_status pcgcn_gemm_xw_split(pcgcn_plan_t p, const float* X, int64_t ldx, const float* W, int64_t ldw,
                                 const float* s, float* Y, int64_t ldy, int64_t M, int32_t K, int32_t N, float* work,
                                 void* stream) {
  if (!X || !W || !Y || M < 0 || K < 1 || N < 1 || ldx < K || ldw < N || ldy < N) {
    set_error("gemm_xw_split: bad arguments");
    return PCGCN_EINVAL;
  }
  WindowOut wo;
  bool any = false;
  pcgcn_status st = split_target(p, M, N, work, ldx, ldy, &wo, &any);
  if (st != PCGCN_OK) return st;
  cudaError_t e = launch_gemm_xw(X, ldx, W, ldw, s, Y, ldy, M, K, N, work, static_cast<cudaStream_t>(stream),
                                 any ? &wo : nullptr);
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "gemm_xw_split");
}

pcgcn_status pcgcn_gemm_dwt_split(pcgcn_plan_t p, const float* D, int64_t ldd, const float* W, const uint32_t* mask,
                                  const float* s, float* O, int64_t ldo, int64_t M, int32_t N, int32_t K, float* work,
                                  void* stream) {
  if (!D || !W || !O || M < 0 || K < 1 || N < 1 || ldd < N || ldo < K) {
    set_error("gemm_dwt_split: bad arguments");
    return PCGCN_EINVAL;
  }
  WindowOut wo;
  bool any = false;
  pcgcn_status st = split_target(p, M, K, work, ldd, ldo, &wo, &any);
  if (st != PCGCN_OK) return st;
  cudaError_t e = launch_gemm_dwt(D, ldd, W, mask, s, O, ldo, M, N, K, work, static_cast<cudaStream_t>(stream),
                                  any ? &wo : nullptr);
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "gemm_dwt_split");
}

int64_t pcgcn_gemm_xtg_work_floats(int64_t M, int32_t K, int32_t N) { return gemm_xtg_work_floats(M, K, N); }

pcgcn_status pcgcn_gemm_xtg(const float* X, int64_t ldx, const float* D, int64_t ldd, float* G,
                            int64_t M, int32_t K, int32_t N, float* work, void* stream) {
  if (!X || !D || !G || !work || M < 0 || K < 1 || N < 1 || ldx < K || ldd < N) {
    set_error("gemm_xtg: bad arguments");
    return PCGCN_EINVAL;
  }
  cudaError_t e = launch_gemm_xtg(X, ldx, D, ldd, G, M, K, N, work, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "gemm_xtg");
}

int64_t pcgcn_gemm_dwt_work_floats(int32_t K, int32_t N) { return gemm_dwt_work_floats(K, N); }

pcgcn_status pcgcn_gemm_dwt(const float* D, int64_t ldd, const float* W, const uint32_t* mask,
                            const float* s, float* O, int64_t ldo, int64_t M, int32_t N, int32_t K,
                            float* work, void* stream) {
  if (!D || !W || !O || M < 0 || K < 1 || N < 1 || ldd < N || ldo < K) {
    set_error("gemm_dwt: bad arguments");
    return PCGCN_EINVAL;
  }
  cudaError_t e = launch_gemm_dwt(D, ldd, W, mask, s, O, ldo, M, N, K, work, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "gemm_dwt");
}

pcgcn_status pcgcn_softmax_ce(const float* L, int64_t ld, const int32_t* labels, const uint8_t* train,
                              int64_t M, int32_t C, float inv_nT, const float* s, float* dL,
                              float* loss, float* work, void* stream) {
  if (!L || !labels || !train || !dL || !loss || !work || C < 1 || C > 256 || ld < C) {
    set_error("softmax_ce: bad arguments");
    return PCGCN_EINVAL;
  }
  cudaError_t e = launch_softmax_ce(L, ld, labels, train, M, C, inv_nT, s, dL, loss, work,
                                    static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "softmax_ce");
}

pcgcn_status pcgcn_adam(float* theta, const float* grad, float* m, float* v, int64_t n, float lr,
                        float b1, float b2, float eps, int32_t* step, void* stream) {
  if (!theta || !grad || !m || !v || !step || n < 0) { set_error("adam: bad arguments"); return PCGCN_EINVAL; }
  cudaError_t e = launch_adam(theta, grad, m, v, n, lr, b1, b2, eps, step, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "adam");
}

pcgcn_status pcgcn_sgd(float* theta, const float* grad, int64_t n, float lr, void* stream) {
  if (!theta || !grad || n < 0) { set_error("sgd: bad arguments"); return PCGCN_EINVAL; }
  cudaError_t e = launch_sgd(theta, grad, n, lr, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? PCGCN_OK : cuda_fail(e, "sgd");
}

}  // extern "C"
