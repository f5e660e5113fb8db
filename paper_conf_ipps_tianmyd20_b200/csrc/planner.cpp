// Host planner of PCGCN (deterministic, multithreaded, result independent of
// the thread count).  Builds, for one symmetric input graph:
//   1. Ã = A + I in clean form, d̃ and r = fp32(d̃^-½)      (Eq. 1; reading #1-#4)
//   2. the vertex partition {V_k}                           (L95-L97 §III-A.a)
//      — synchronous label propagation + packing, replacing METIS (reading #8)
//   3. the plan-order permutation (vertex blocks become row ranges, so the
//      "split a^l -> a_k^l" and "concat h_k^l" of Alg. 1, L115/L123, are free)
//   4. the K×K edge-block table with densities and mode bits (θ rule, L161)
//   5. the merged selective CSR (L179) and the full-mode tiles (L175) as
//      128×32 bit chunks grouped per 128-row destination tile.
// The plan spec it implements is DESIGN.md §3a; oracle/plan.py is an
// independent re-derivation and tests/test_plan_abi.py compares them bit-exactly.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstring>
#include <numeric>
#include <thread>
#include <vector>

#include "plan_internal.h"

namespace pcgcn {
namespace {

int nthreads() {
  unsigned h = std::thread::hardware_concurrency();
  return h == 0 ? 4 : int(std::min(h, 64u));
}

template <class F>
void parallel_for(int64_t n, F f) {
  int T = nthreads();
  if (n < 4096) T = 1;
  std::vector<std::thread> th;
  for (int t = 0; t < T; ++t) {
    int64_t a = n * t / T, b = n * (t + 1) / T;
    if (T == 1) { f(t, a, b); return; }
    th.emplace_back([=, &f] { f(t, a, b); });
  }
  for (auto& x : th) x.join();
}

double ms_since(std::chrono::steady_clock::time_point t0) {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

// Clean binary A (no self-loops, no duplicates, sorted rows).
struct CleanA {
  std::vector<int64_t> ptr;
  std::vector<int32_t> col;
};

pcgcn_status clean_graph(const pcgcn_csr* A, CleanA& C) {
  const int64_t n = A->n;
  std::vector<int64_t> cnt(n, 0);
  std::vector<int32_t> tmp(A->nnz);
  bool bad = false;
  parallel_for(n, [&](int, int64_t a, int64_t b) {
    for (int64_t v = a; v < b; ++v) {
      int64_t s = A->rowptr[v], e = A->rowptr[v + 1];
      int32_t* out = tmp.data() + s;
      int64_t k = 0;
      for (int64_t i = s; i < e; ++i) {
        int32_t j = A->col[i];
        if (j < 0 || j >= n) { bad = true; continue; }
        if (j != v) out[k++] = j;
      }
      std::sort(out, out + k);
      cnt[v] = std::unique(out, out + k) - out;
    }
  });
  if (bad) { set_error("column index out of range"); return PCGCN_EINVAL; }
  C.ptr.assign(n + 1, 0);
  for (int64_t v = 0; v < n; ++v) C.ptr[v + 1] = C.ptr[v] + cnt[v];
  C.col.resize(C.ptr[n]);
  parallel_for(n, [&](int, int64_t a, int64_t b) {
    for (int64_t v = a; v < b; ++v)
      std::memcpy(C.col.data() + C.ptr[v], tmp.data() + A->rowptr[v], sizeof(int32_t) * cnt[v]);
  });
  // symmetry: every (v, j) must have (j, v)
  std::vector<uint8_t> asym(nthreads(), 0);
  parallel_for(n, [&](int t, int64_t a, int64_t b) {
    for (int64_t v = a; v < b && !asym[t]; ++v)
      for (int64_t i = C.ptr[v]; i < C.ptr[v + 1]; ++i) {
        int32_t j = C.col[i];
        if (!std::binary_search(C.col.data() + C.ptr[j], C.col.data() + C.ptr[j + 1], int32_t(v))) {
          asym[t] = 1;
          break;
        }
      }
  });
  for (auto x : asym)
    if (x) { set_error("adjacency is not symmetric (A^T != A)"); return PCGCN_ENOTSYM; }
  return PCGCN_OK;
}

// Synchronous label propagation on Ã (self vote included), ties -> smallest label.
int32_t label_propagation(const CleanA& C, int64_t n, int32_t T, std::vector<int32_t>& lab) {
  lab.resize(n);
  std::iota(lab.begin(), lab.end(), 0);
  std::vector<int32_t> nxt(n);
  int32_t it = 0;
  for (it = 1; it <= T; ++it) {
    std::vector<uint8_t> changed(nthreads(), 0);
    parallel_for(n, [&](int t, int64_t a, int64_t b) {
      std::vector<int32_t> buf;
      for (int64_t v = a; v < b; ++v) {
        int64_t s = C.ptr[v], e = C.ptr[v + 1];
        buf.resize(e - s + 1);
        for (int64_t i = s; i < e; ++i) buf[i - s] = lab[C.col[i]];
        buf[e - s] = lab[v];
        std::sort(buf.begin(), buf.end());
        int32_t best = buf[0];
        int64_t best_c = 0;
        for (size_t i = 0; i < buf.size();) {
          size_t j = i;
          while (j < buf.size() && buf[j] == buf[i]) ++j;
          if (int64_t(j - i) > best_c) { best_c = int64_t(j - i); best = buf[i]; }
          i = j;
        }
        nxt[v] = best;
        if (best != lab[v]) changed[t] = 1;
      }
    });
    bool any = false;
    for (auto c : changed) any |= c != 0;
    if (!any) return it;
    lab.swap(nxt);
  }
  return T;
}

// Clusters ordered by (size desc, smallest member asc), members by id, cut
// into P consecutive chunks (numpy array_split sizes).
int64_t pack_parts(const std::vector<int32_t>& lab, int64_t n, int32_t P, std::vector<int32_t>& part) {
  std::vector<int64_t> size(n, 0), minid(n, n);
  for (int64_t v = 0; v < n; ++v) {
    size[lab[v]]++;
    minid[lab[v]] = std::min(minid[lab[v]], v);
  }
  std::vector<int32_t> cl;
  for (int64_t l = 0; l < n; ++l)
    if (size[l] > 0) cl.push_back(int32_t(l));
  std::sort(cl.begin(), cl.end(), [&](int32_t a, int32_t b) {
    if (size[a] != size[b]) return size[a] > size[b];
    return minid[a] < minid[b];
  });
  std::vector<int64_t> off(n, 0);
  int64_t run = 0;
  for (int32_t l : cl) { off[l] = run; run += size[l]; }
  std::vector<int32_t> seq(n);
  for (int64_t v = 0; v < n; ++v) seq[off[lab[v]]++] = int32_t(v);
  part.assign(n, 0);
  const int64_t q = n / P, rem = n % P;
  int64_t pos = 0;
  for (int32_t k = 0; k < P; ++k) {
    int64_t sz = q + (k < rem ? 1 : 0);
    for (int64_t i = 0; i < sz; ++i) part[seq[pos++]] = k;
  }
  return int64_t(cl.size());
}

}  // namespace

pcgcn_status build_host_plan(const pcgcn_csr* A, int32_t P, float theta, const pcgcn_opts* o,
                             pcgcn_plan_s* p) {
  auto t0 = std::chrono::steady_clock::now();
  const int64_t n = A->n;
  if (n <= 0 || P < 1 || P > n || !A->rowptr || (A->nnz > 0 && !A->col) || A->rowptr[0] != 0 ||
      A->rowptr[n] != A->nnz) {
    set_error("pcgcn_plan: bad graph or P");
    return PCGCN_EINVAL;
  }
  for (int64_t v = 0; v < n; ++v)
    if (A->rowptr[v + 1] < A->rowptr[v]) { set_error("rowptr not monotone"); return PCGCN_EINVAL; }
  if (!(theta >= 0.f)) { set_error("theta must be >= 0 (calibrate first)"); return PCGCN_EINVAL; }
  if (o->vertex_order != PCGCN_ORDER_ID && o->vertex_order != PCGCN_ORDER_DEGREE) {
    set_error("unknown vertex_order");
    return PCGCN_EINVAL;
  }
  if (o->world < 1 || o->rank < 0 || o->rank >= o->world) { set_error("bad rank/world"); return PCGCN_EINVAL; }
  p->n = n; p->P = P; p->theta = theta; p->opts = *o;

  CleanA C;
  pcgcn_status st = clean_graph(A, C);
  if (st != PCGCN_OK) return st;
  p->nnz_t = C.ptr[n] + n;

  // r = fp32(1/sqrt(fp64 d̃)), d̃ = 1 + deg  (correctly rounded => bit-exact)
  std::vector<float> r_orig(n);
  for (int64_t v = 0; v < n; ++v) {
    double d = double(C.ptr[v + 1] - C.ptr[v] + 1);
    r_orig[v] = o->norm == PCGCN_NORM_NONE ? 1.0f : float(1.0 / std::sqrt(d));
  }

  // partition
  auto tp = std::chrono::steady_clock::now();
  if (o->part) {
    p->part.assign(o->part, o->part + n);
    for (int64_t v = 0; v < n; ++v)
      if (p->part[v] < 0 || p->part[v] >= P) { set_error("part override out of range"); return PCGCN_EINVAL; }
    p->sweeps = 0;
    p->clusters = 0;
  } else {
    std::vector<int32_t> lab;
    p->sweeps = label_propagation(C, n, o->lp_sweeps, lab);
    p->clusters = pack_parts(lab, n, P, p->part);
  }
  double part_ms = ms_since(tp);

  // permutation: sort by (part, id), or by (part, -degree, id) (vertex_order DEGREE)
  std::vector<int64_t> psize(P, 0);
  for (int64_t v = 0; v < n; ++v) psize[p->part[v]]++;
  p->pstart.assign(P + 1, 0);
  for (int32_t k = 0; k < P; ++k) p->pstart[k + 1] = p->pstart[k] + psize[k];
  p->perm.resize(n);
  std::vector<int64_t> inv(n);
  {
    std::vector<int64_t> fill(p->pstart.begin(), p->pstart.end() - 1);
    for (int64_t v = 0; v < n; ++v) p->perm[fill[p->part[v]]++] = int32_t(v);  // (part, id)
    if (o->vertex_order == PCGCN_ORDER_DEGREE) {
      parallel_for(P, [&](int, int64_t a, int64_t b) {
        for (int64_t k = a; k < b; ++k)
          std::stable_sort(p->perm.begin() + p->pstart[k], p->perm.begin() + p->pstart[k + 1],
                           [&](int32_t x, int32_t y) {
                             return C.ptr[x + 1] - C.ptr[x] > C.ptr[y + 1] - C.ptr[y];
                           });
      });
    }
    for (int64_t pos = 0; pos < n; ++pos) inv[p->perm[pos]] = pos;
  }
  p->r.resize(n);
  for (int64_t v = 0; v < n; ++v) p->r[v] = r_orig[p->perm[v]];
  std::vector<int32_t> pid(n);  // partition of each plan row
  for (int32_t k = 0; k < P; ++k)
    for (int64_t v = p->pstart[k]; v < p->pstart[k + 1]; ++v) pid[v] = k;

  // Ã in plan order, rows sorted
  std::vector<int64_t> tptr(n + 1, 0);
  for (int64_t v = 0; v < n; ++v) {
    int32_t old = p->perm[v];
    tptr[v + 1] = tptr[v] + (C.ptr[old + 1] - C.ptr[old]) + 1;
  }
  std::vector<int32_t> tcol(tptr[n]);
  parallel_for(n, [&](int, int64_t a, int64_t b) {
    for (int64_t v = a; v < b; ++v) {
      int32_t old = p->perm[v];
      int32_t* out = tcol.data() + tptr[v];
      int64_t k = 0;
      for (int64_t i = C.ptr[old]; i < C.ptr[old + 1]; ++i) out[k++] = int32_t(inv[C.col[i]]);
      out[k++] = int32_t(v);
      std::sort(out, out + k);
    }
  });
  std::vector<int64_t>().swap(C.ptr);
  std::vector<int32_t>().swap(C.col);

  // block table per destination partition k (rows contiguous)
  std::vector<std::vector<std::pair<int32_t, int64_t>>> blocks(P);  // (i, nnz) sorted by i
  parallel_for(P, [&](int, int64_t a, int64_t b) {
    std::vector<int64_t> cnt(P, 0);
    std::vector<int32_t> touched;
    for (int64_t k = a; k < b; ++k) {
      for (int64_t v = p->pstart[k]; v < p->pstart[k + 1]; ++v)
        for (int64_t e = tptr[v]; e < tptr[v + 1]; ++e) {
          int32_t i = pid[tcol[e]];
          if (cnt[i]++ == 0) touched.push_back(i);
        }
      std::sort(touched.begin(), touched.end());
      for (int32_t i : touched) { blocks[k].push_back({i, cnt[i]}); cnt[i] = 0; }
      touched.clear();
    }
  });
  std::vector<int64_t> bptr(P + 1, 0);
  for (int32_t k = 0; k < P; ++k) bptr[k + 1] = bptr[k] + int64_t(blocks[k].size());
  const int64_t nb = bptr[P];
  p->blk_k.resize(nb); p->blk_i.resize(nb); p->blk_nnz.resize(nb); p->blk_dense.resize(nb);
  const double th = double(theta);
  const bool tile_grain = o->mode_grain == PCGCN_GRAIN_TILE;
  int64_t nb_dense = 0, intra = 0;
  for (int32_t k = 0; k < P; ++k)
    for (size_t j = 0; j < blocks[k].size(); ++j) {
      int64_t b = bptr[k] + int64_t(j);
      int32_t i = blocks[k][j].first;
      int64_t z = blocks[k][j].second;
      p->blk_k[b] = k; p->blk_i[b] = i; p->blk_nnz[b] = z;
      double dens = double(z) / (double(psize[k]) * double(psize[i]));
      p->blk_dense[b] = (!tile_grain && dens > th) ? 1 : 0;
      if (i == k) intra += z;
    }

  // mode of each edge -> merged selective CSR + dense chunks, per partition.
  // A chunk is the 128-row destination tile x 32-aligned global source window
  // the full mode executes as one unit (TMA box starts must be 16-byte aligned,
  // so windows are global, not partition-relative).  BLOCK grain: the edges of
  // full-mode blocks, grouped into chunks (blocks sharing a window share its
  // chunk); TILE grain: every chunk whose own density nnz/(rows·cols) > θ.
  std::vector<int64_t> sp_cnt(n, 0);
  struct TileOut {
    int32_t row0, nrows;
    std::vector<int32_t> col0;
    std::vector<uint32_t> bits;
  };
  std::vector<std::vector<TileOut>> tiles(P);
  auto win_cols = [&](int64_t c0) { return double(std::min<int64_t>(TILE_K, n - c0)); };
  parallel_for(P, [&](int, int64_t a, int64_t b) {
    std::vector<uint8_t> dense_i(P, 0);
    std::vector<int64_t> blk_pos(P, -1);
    std::vector<int32_t> wcnt((n + TILE_K - 1) / TILE_K, 0), wslot((n + TILE_K - 1) / TILE_K, -1), touched;
    for (int64_t k = a; k < b; ++k) {
      bool any_dense = tile_grain;
      for (int64_t j = bptr[k]; j < bptr[k + 1]; ++j) {
        dense_i[p->blk_i[j]] = p->blk_dense[j];
        blk_pos[p->blk_i[j]] = j;
        any_dense |= p->blk_dense[j] != 0;
      }
      if (!tile_grain) {
        for (int64_t v = p->pstart[k]; v < p->pstart[k + 1]; ++v) {
          int64_t c = 0;
          for (int64_t e = tptr[v]; e < tptr[v + 1]; ++e) c += dense_i[pid[tcol[e]]] ? 0 : 1;
          sp_cnt[v] = c;
        }
      } else {
        for (int64_t v = p->pstart[k]; v < p->pstart[k + 1]; ++v) sp_cnt[v] = tptr[v + 1] - tptr[v];
      }
      if (any_dense) {
        for (int64_t r0 = p->pstart[k]; r0 < p->pstart[k + 1]; r0 += TILE_M) {
          const int64_t r1 = std::min<int64_t>(r0 + TILE_M, p->pstart[k + 1]);
          // count the candidate edges per 32-source window (dense per-thread
          // counters over the n/32 windows; only the touched ones are reset)
          touched.clear();
          for (int64_t v = r0; v < r1; ++v)
            for (int64_t e = tptr[v]; e < tptr[v + 1]; ++e) {
              const int32_t j = tcol[e];
              if (!tile_grain && !dense_i[pid[j]]) continue;
              const int32_t wv = j / TILE_K;
              if (wcnt[wv]++ == 0) touched.push_back(wv);
            }
          if (touched.empty()) continue;
          std::sort(touched.begin(), touched.end());
          TileOut T;
          T.row0 = int32_t(r0);
          T.nrows = int32_t(r1 - r0);
          for (int32_t wv : touched) {
            const int64_t c0 = int64_t(wv) * TILE_K;
            // block grain: every window of a full-mode block is a chunk; tile
            // grain: the chunk's own density decides (a selective chunk's edges
            // stay in the merged CSR)
            if (!tile_grain || double(wcnt[wv]) / (double(r1 - r0) * win_cols(c0)) > th) {
              wslot[wv] = int32_t(T.col0.size());
              T.col0.push_back(int32_t(c0));
            }
            wcnt[wv] = 0;
          }
          T.bits.assign(T.col0.size() * TILE_M, 0u);
          if (!T.col0.empty()) {
            for (int64_t v = r0; v < r1; ++v)
              for (int64_t e = tptr[v]; e < tptr[v + 1]; ++e) {
                const int32_t j = tcol[e];
                const int32_t sl = wslot[j / TILE_K];
                if (sl < 0 || (!tile_grain && !dense_i[pid[j]])) continue;
                const int32_t bit = j % TILE_K;
                T.bits[size_t(sl) * TILE_M + size_t(v - r0)] |= 1u << bit;
                if (tile_grain) {
                  sp_cnt[v]--;
                  p->blk_dense[blk_pos[pid[j]]] = 1;  // block holds full-mode edges
                }
              }
          }
          for (int32_t wv : touched) wslot[wv] = -1;
          if (!T.col0.empty()) tiles[k].push_back(std::move(T));
        }
      }
      for (int64_t j = bptr[k]; j < bptr[k + 1]; ++j) {
        dense_i[p->blk_i[j]] = 0;
        blk_pos[p->blk_i[j]] = -1;
      }
    }
  });
  for (int64_t b2 = 0; b2 < nb; ++b2) nb_dense += p->blk_dense[b2];
  p->sp_rowptr.assign(n + 1, 0);
  for (int64_t v = 0; v < n; ++v) p->sp_rowptr[v + 1] = p->sp_rowptr[v] + sp_cnt[v];
  p->sp_col.resize(p->sp_rowptr[n]);
  parallel_for(P, [&](int, int64_t a, int64_t b) {
    std::vector<uint8_t> dense_i(P, 0);
    for (int64_t k = a; k < b; ++k) {
      for (int64_t j = bptr[k]; j < bptr[k + 1]; ++j) dense_i[p->blk_i[j]] = p->blk_dense[j];
      const TileOut* T = tiles[k].empty() ? nullptr : tiles[k].data();
      size_t tn = tiles[k].size(), ti = 0;
      for (int64_t v = p->pstart[k]; v < p->pstart[k + 1]; ++v) {
        int64_t o2 = p->sp_rowptr[v];
        if (!tile_grain) {
          for (int64_t e = tptr[v]; e < tptr[v + 1]; ++e)
            if (!dense_i[pid[tcol[e]]]) p->sp_col[o2++] = tcol[e];
          continue;
        }
        // TILE grain: the edge is selective unless its window is a chunk of v's tile
        while (ti < tn && T[ti].row0 + T[ti].nrows <= v) ++ti;
        const bool has = ti < tn && T[ti].row0 <= v;
        const int32_t rr = has ? int32_t(v - T[ti].row0) : 0;
        for (int64_t e = tptr[v]; e < tptr[v + 1]; ++e) {
          const int32_t j = tcol[e];
          bool dense = false;
          if (has) {
            const int32_t c0 = (j / TILE_K) * TILE_K;
            auto it = std::lower_bound(T[ti].col0.begin(), T[ti].col0.end(), c0);
            dense = it != T[ti].col0.end() && *it == c0 &&
                    ((T[ti].bits[size_t(it - T[ti].col0.begin()) * TILE_M + rr] >> (j - c0)) & 1u);
          }
          if (!dense) p->sp_col[o2++] = j;
        }
      }
      for (int64_t j = bptr[k]; j < bptr[k + 1]; ++j) dense_i[p->blk_i[j]] = 0;
    }
  });
  p->rt_cptr.assign(1, 0);
  p->zd_index.assign(n, -1);
  std::vector<int64_t> part_rt(P + 1, 0);  // row-tile range of each partition
  for (int32_t k = 0; k < P; ++k) {
    part_rt[k] = int64_t(p->rt_row0.size());
    for (auto& T : tiles[k]) {
      int64_t t = int64_t(p->rt_row0.size());
      p->rt_row0.push_back(T.row0);
      p->rt_nrows.push_back(T.nrows);
      p->ch_col0.insert(p->ch_col0.end(), T.col0.begin(), T.col0.end());
      p->bits.insert(p->bits.end(), T.bits.begin(), T.bits.end());
      p->rt_cptr.push_back(int64_t(p->ch_col0.size()));
      for (int32_t rr = 0; rr < T.nrows; ++rr) p->zd_index[T.row0 + rr] = int32_t(t * TILE_M + rr);
    }
    std::vector<TileOut>().swap(tiles[k]);
  }
  part_rt[P] = int64_t(p->rt_row0.size());

  // shard: contiguous partition ranges balanced by cost_k = nnz(Ã rows of V_k)
  // + |V_k| — independent of θ, so plans of the same graph built for
  // different feature widths (per-width θ) shard identically
  {
    std::vector<double> cost(P, 0.0);
    for (int32_t k = 0; k < P; ++k)
      cost[k] = double(tptr[p->pstart[k + 1]] - tptr[p->pstart[k]]) + double(psize[k]);
    double tot = 0;
    for (double c : cost) tot += c;
    auto bound = [&](int32_t q) -> int32_t {
      if (q <= 0) return 0;
      if (q >= o->world) return P;
      double target = tot * double(q) / double(o->world), run = 0;
      for (int32_t k = 0; k < P; ++k) {
        if (run >= target) return k;
        run += cost[k];
      }
      return P;
    };
    p->k_lo = bound(o->rank);
    p->k_hi = bound(o->rank + 1);
    p->row_lo = p->pstart[p->k_lo];
    p->row_hi = p->pstart[p->k_hi];
    p->rt_lo = part_rt[p->k_lo];
    p->rt_hi = part_rt[p->k_hi];
    p->shard_row0.assign(o->world + 1, 0);
    for (int32_t q = 0; q <= o->world; ++q) p->shard_row0[q] = p->pstart[bound(q)];
    // halo lists (L99: a shard reads the source rows its
    // blocks touch): rows of shard q that shard r reads — the sources of r's
    // selective edges and every row of the 32-source windows of r's chunks —
    // for r = this rank (recv, one list per q) and q = this rank (send, one
    // list per r).  Lists are ascending; a shard's own rows are never listed.
    const int32_t W = o->world;
    if (W > 1) {
      std::vector<std::vector<uint64_t>> need(W, std::vector<uint64_t>((n + 63) / 64, 0));
      parallel_for(W, [&](int, int64_t a, int64_t b) {
        for (int64_t r = a; r < b; ++r) {
          auto& bm = need[r];
          const int32_t ka = bound(int32_t(r)), kb = bound(int32_t(r) + 1);
          for (int64_t v = p->pstart[ka]; v < p->pstart[kb]; ++v)
            for (int64_t e = p->sp_rowptr[v]; e < p->sp_rowptr[v + 1]; ++e) {
              const int64_t j = p->sp_col[e];
              bm[j >> 6] |= 1ull << (j & 63);
            }
          for (int64_t t = part_rt[ka]; t < part_rt[kb]; ++t)
            for (int64_t c = p->rt_cptr[t]; c < p->rt_cptr[t + 1]; ++c) {
              const int64_t c0 = p->ch_col0[c];
              for (int64_t j = c0; j < std::min<int64_t>(c0 + TILE_K, n); ++j) bm[j >> 6] |= 1ull << (j & 63);
            }
        }
      });
      auto rows_in = [&](const std::vector<uint64_t>& bm, int64_t lo, int64_t hi, std::vector<int32_t>& out) {
        for (int64_t j = lo; j < hi; ++j)
          if ((bm[j >> 6] >> (j & 63)) & 1ull) out.push_back(int32_t(j));
      };
      p->halo_recv.assign(W, {});
      p->halo_send.assign(W, {});
      for (int32_t q = 0; q < W; ++q) {
        if (q == o->rank) continue;
        rows_in(need[o->rank], p->shard_row0[q], p->shard_row0[q + 1], p->halo_recv[q]);
        rows_in(need[q], p->row_lo, p->row_hi, p->halo_send[q]);
      }
    }
  }

  // partition-centric source rows (SURVEY.md §8(d) B_pc): Σ_k |distinct sources
  // of V_k's selective edges| — the rows a destination partition must fetch if
  // each of its blocks' source slices were read once (L129 §III-A.b)
  {
    std::vector<int64_t> upc(P, 0);
    parallel_for(P, [&](int, int64_t a, int64_t b) {
      std::vector<int32_t> buf;
      for (int64_t k = a; k < b; ++k) {
        buf.assign(p->sp_col.begin() + p->sp_rowptr[p->pstart[k]], p->sp_col.begin() + p->sp_rowptr[p->pstart[k + 1]]);
        std::sort(buf.begin(), buf.end());
        upc[k] = std::unique(buf.begin(), buf.end()) - buf.begin();
      }
    });
    for (int32_t k = 0; k < P; ++k) {
      p->stats_src_rows_pc += upc[k];
      if (k >= p->k_lo && k < p->k_hi) p->stats_shard_src_rows_pc += upc[k];
    }
  }

  // stats
  pcgcn_stats& S = p->stats;
  std::memset(&S, 0, sizeof(S));
  S.n = n; S.nnz = p->nnz_t; S.P = P; S.lp_sweeps = p->sweeps; S.clusters = p->clusters;
  S.blocks_nonempty = nb; S.blocks_dense = nb_dense;
  S.nnz_sparse = p->sp_rowptr[n]; S.nnz_dense = p->nnz_t - p->sp_rowptr[n];
  S.intra_edges = intra;
  S.row_tiles = int64_t(p->rt_row0.size()); S.chunks = int64_t(p->ch_col0.size());
  S.row_lo = p->row_lo; S.row_hi = p->row_hi;
  S.shard_nnz_sparse = p->sp_rowptr[p->row_hi] - p->sp_rowptr[p->row_lo];
  S.shard_chunks = p->rt_cptr[p->rt_hi] - p->rt_cptr[p->rt_lo];
  S.theta = theta;
  S.src_rows_pc = p->stats_src_rows_pc;
  S.shard_src_rows_pc = p->stats_shard_src_rows_pc;
  for (auto& l : p->halo_recv) S.halo_recv_rows += int64_t(l.size());
  for (auto& l : p->halo_send) S.halo_send_rows += int64_t(l.size());
  S.partition_ms = part_ms;
  S.plan_ms = ms_since(t0);
  return PCGCN_OK;
}

}  // namespace pcgcn
