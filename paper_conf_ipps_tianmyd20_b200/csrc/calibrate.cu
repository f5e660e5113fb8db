// θ calibration (row a3): the paper's procedure of L161 (§III-B.c) on the
// B200 itself.  "We profile the runtime of full and selective modes for a
// block of sparsity p, denoted by T_f and T_s ... θ = T_f·p/T_s."
//
// Synthetic workload: pairs of vertex blocks of `block_rows` vertices joined
// by random bipartite blocks of edge density p_ref (seeded splitmix64, so the
// blocks are the same on every call), plus the n self-loops of Ã.  The plan
// is built twice with an explicit partition override (θ >= 1 -> every block
// selective; θ just below p_ref -> the p-blocks full) and each mode's forward
// at width F is timed with CUDA events (median of 15 after 3 warm-ups).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <vector>

#include "plan_internal.h"

namespace {

uint64_t mix64(uint64_t x) {
  x ^= x >> 30; x *= 0xBF58476D1CE4E5B9ull;
  x ^= x >> 27; x *= 0x94D049BB133111EBull;
  x ^= x >> 31;
  return x;
}

float time_forward(pcgcn_plan_t p, const float* Y, float* Z, int F, int64_t ld, cudaStream_t s) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  std::vector<float> ts;
  for (int it = 0; it < 18; ++it) {
    cudaEventRecord(a, s);
    pcgcn_forward(p, Y, ld, Z, ld, F, PCGCN_IN_PRESCALED, nullptr, s);
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    if (it >= 3) ts.push_back(ms);
  }
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  std::sort(ts.begin(), ts.end());
  return ts[ts.size() / 2];
}

}  // namespace

extern "C" pcgcn_status pcgcn_refine_theta(pcgcn_plan_t p, const float* Y, int64_t ldy, float* Z, int64_t ldz,
                                           int32_t F, float* theta_out, float* c_chunk_ns, float* c_edge_ns) {
  if (!p || !Y || !Z || !theta_out) {
    pcgcn::set_error("refine_theta: null argument");
    return PCGCN_EINVAL;
  }
  *theta_out = p->theta;
  if (c_chunk_ns) *c_chunk_ns = 0.f;
  if (c_edge_ns) *c_edge_ns = 0.f;
  const int64_t chunks = p->stats.shard_chunks, edges = p->stats.shard_nnz_sparse;
  if (chunks == 0 || edges == 0) return PCGCN_OK;  // one mode absent: nothing to compare
  cudaStream_t s = nullptr;
  if (cudaStreamCreate(&s) != cudaSuccess) {
    pcgcn::set_error("refine_theta: stream");
    return PCGCN_ECUDA;
  }
  std::vector<float> td, ts;
  for (int it = 0; it < 7; ++it) {
    pcgcn_status st = pcgcn_forward(p, Y, ldy, Z, ldz, F, PCGCN_IN_PRESCALED | PCGCN_PROFILE, nullptr, s);
    if (st != PCGCN_OK) { cudaStreamDestroy(s); return st; }
    float ms[4];
    st = pcgcn_plan_last_timings(p, ms);
    if (st != PCGCN_OK) { cudaStreamDestroy(s); return st; }
    if (it >= 2) { td.push_back(ms[2]); ts.push_back(ms[3]); }
  }
  cudaStreamDestroy(s);
  std::sort(td.begin(), td.end());
  std::sort(ts.begin(), ts.end());
  const double cc = double(td[td.size() / 2]) * 1e6 / double(chunks);  // ns per chunk
  const double ce = double(ts[ts.size() / 2]) * 1e6 / double(edges);   // ns per selective edge
  if (c_chunk_ns) *c_chunk_ns = float(cc);
  if (c_edge_ns) *c_edge_ns = float(ce);
  if (ce > 0) *theta_out = float(cc / (4096.0 * ce));
  return PCGCN_OK;
}

extern "C" pcgcn_status pcgcn_calibrate_prec(int32_t F, int32_t block_rows, float p_ref, int32_t dense_prec,
                                             float* theta_out, float* t_full_ms, float* t_sel_ms) {
  if (F < 1 || F > 256 || block_rows < 32 || !(p_ref > 0.f && p_ref <= 1.f) || !theta_out ||
      dense_prec < PCGCN_DENSE_TF32X2 || dense_prec > PCGCN_DENSE_BF16X3) {
    pcgcn::set_error("calibrate: bad arguments");
    return PCGCN_EINVAL;
  }
  // Pc vertex blocks of B rows; blocks (2q, 2q+1) are joined by a symmetric
  // random bipartite block of density p.  Pc is chosen so the full-mode
  // kernel sees >= 2 row tiles per SM (a 2-block probe would leave most of
  // the 148 SMs idle and overstate T_f).
  const int64_t B = block_rows;
  const int64_t tiles_per_block = (B + 127) / 128;
  int64_t Pc = (8 * 148 + tiles_per_block - 1) / tiles_per_block;  // >= 8 row tiles per SM: balanced waves
  Pc = std::max<int64_t>(2, Pc + (Pc & 1));
  const int64_t n = Pc * B;
  const uint64_t thr = uint64_t(double(p_ref) * 18446744073709551615.0);
  std::vector<std::vector<int32_t>> adj(n);
  for (int64_t q = 0; q < Pc / 2; ++q) {
    const int64_t b0 = 2 * q * B, b1 = b0 + B;
    for (int64_t u = 0; u < B; ++u)
      for (int64_t v = 0; v < B; ++v)
        if (mix64(0x5eedull * 0x9E3779B97F4A7C15ull + uint64_t((q * B + u) * B + v)) < thr) {
          adj[b0 + u].push_back(int32_t(b1 + v));
          adj[b1 + v].push_back(int32_t(b0 + u));
        }
  }
  std::vector<int64_t> rowptr(n + 1, 0);
  for (int64_t v = 0; v < n; ++v) rowptr[v + 1] = rowptr[v] + int64_t(adj[v].size());
  std::vector<int32_t> col(rowptr[n]);
  for (int64_t v = 0; v < n; ++v) std::copy(adj[v].begin(), adj[v].end(), col.begin() + rowptr[v]);
  std::vector<int32_t> part(n);
  for (int64_t v = 0; v < n; ++v) part[v] = int32_t(v / B);
  pcgcn_csr A{n, rowptr[n], rowptr.data(), col.data()};
  pcgcn_opts o;
  pcgcn_opts_default(&o);
  o.part = part.data();
  o.f_max = F;
  o.dense_prec = dense_prec;
  pcgcn_plan_t ps = nullptr, pf = nullptr;
  // diagonal blocks hold only the self-loops (density 1/B): keep them selective
  // in both plans so the two timings differ only in the mode of the p-blocks
  const float theta_full = 2.0f / float(B);
  pcgcn_status st = pcgcn_plan(&A, int32_t(Pc), 2.0f, &o, &ps);
  if (st != PCGCN_OK) return st;
  st = pcgcn_plan(&A, int32_t(Pc), std::min(theta_full, 0.5f * p_ref), &o, &pf);
  if (st != PCGCN_OK) { pcgcn_destroy(ps); return st; }
  const int64_t ld = (F + 3) / 4 * 4;
  float *Y = nullptr, *Z = nullptr;
  cudaStream_t s = nullptr;
  if (cudaMalloc(&Y, sizeof(float) * n * ld) != cudaSuccess || cudaMalloc(&Z, sizeof(float) * n * ld) != cudaSuccess ||
      cudaStreamCreate(&s) != cudaSuccess) {
    pcgcn_destroy(ps);
    pcgcn_destroy(pf);
    pcgcn::set_error("calibrate: allocation failed");
    return PCGCN_ENOMEM;
  }
  cudaMemsetAsync(Y, 0, sizeof(float) * n * ld, s);
  float ts = time_forward(ps, Y, Z, F, ld, s);
  float tf = time_forward(pf, Y, Z, F, ld, s);
  cudaError_t e = cudaStreamSynchronize(s);
  cudaFree(Y);
  cudaFree(Z);
  cudaStreamDestroy(s);
  pcgcn_destroy(ps);
  pcgcn_destroy(pf);
  if (e != cudaSuccess) {
    pcgcn::set_error(std::string("calibrate: ") + cudaGetErrorString(e));
    return PCGCN_ECUDA;
  }
  *theta_out = tf * p_ref / ts;  // θ = T_f·p/T_s (L161)
  if (t_full_ms) *t_full_ms = tf;
  if (t_sel_ms) *t_sel_ms = ts;
  return PCGCN_OK;
}

extern "C" pcgcn_status pcgcn_calibrate(int32_t F, int32_t block_rows, float p_ref, float* theta_out,
                                        float* t_full_ms, float* t_sel_ms) {
  return pcgcn_calibrate_prec(F, block_rows, p_ref, PCGCN_DENSE_TF32X2, theta_out, t_full_ms, t_sel_ms);
}
