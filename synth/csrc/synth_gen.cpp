// Multithreaded twin of synth/graphs.py::sbm (input infrastructure only; no
// part of the PCGCN method).  Bit-identical to the numpy path: every edge is a
// pure function of (stream key, counter), so the thread count never matters.
#include <algorithm>
#include <atomic>
#include <cstdint>
#include <cstring>
#include <thread>
#include <utility>
#include <vector>

namespace {

const uint64_t GOLDEN = 0x9E3779B97F4A7C15ull;

inline uint64_t mix64(uint64_t x) {
  x ^= x >> 30; x *= 0xBF58476D1CE4E5B9ull;
  x ^= x >> 27; x *= 0x94D049BB133111EBull;
  x ^= x >> 31;
  return x;
}
inline uint64_t draw(uint64_t key, uint64_t ctr) { return mix64(key + (ctr + 1) * GOLDEN); }
inline double unit(uint64_t u) { return double(u >> 11) * (1.0 / 9007199254740992.0); }

// searchsorted(cdf, t, 'right') - 1
inline int64_t pick(const int64_t* cdf, int64_t n, int64_t t) {
  return int64_t(std::upper_bound(cdf, cdf + n + 1, t) - cdf) - 1;
}

int nthreads() {
  unsigned h = std::thread::hardware_concurrency();
  return h == 0 ? 4 : int(std::min(h, 64u));
}

template <class F>
void parallel_for(int64_t n, F f) {
  int T = nthreads();
  std::vector<std::thread> th;
  for (int t = 0; t < T; ++t) {
    int64_t a = n * t / T, b = n * (t + 1) / T;
    th.emplace_back([=, &f] { f(t, a, b); });
  }
  for (auto& x : th) x.join();
}

struct Model {
  int64_t n;
  const int64_t *cdf, *class_start, *sub_start, *id_of;
  const int32_t *class_of, *sub_of;
  double p_sub, p_class;
  uint64_t key;
};

// returns UINT64_MAX for a dropped self-pair
inline uint64_t edge_key(const Model& M, uint64_t e) {
  const uint64_t d0 = draw(M.key, 3 * e), d1 = draw(M.key, 3 * e + 1), d2 = draw(M.key, 3 * e + 2);
  const double lvl = unit(d0);
  const uint64_t W = uint64_t(M.cdf[M.n]);
  const int64_t gu = pick(M.cdf, M.n, int64_t(d1 % W));
  int64_t lo = 0, hi = M.n;
  if (lvl < M.p_sub) {
    lo = M.sub_start[M.sub_of[gu]]; hi = M.sub_start[M.sub_of[gu] + 1];
  } else if (lvl < M.p_sub + M.p_class) {
    lo = M.class_start[M.class_of[gu]]; hi = M.class_start[M.class_of[gu] + 1];
  }
  const int64_t base = M.cdf[lo];
  const uint64_t span = uint64_t(M.cdf[hi] - base);
  const int64_t gv = pick(M.cdf, M.n, base + int64_t(d2 % span));
  if (gu == gv) return UINT64_MAX;
  uint64_t a = uint64_t(M.id_of[gu]), b = uint64_t(M.id_of[gv]);
  if (a > b) std::swap(a, b);
  return a * uint64_t(M.n) + b;
}

// Distinct upper-triangle edges of the given keys: per-row sorted lists.
struct Upper {
  std::vector<int64_t> ptr;  // n+1
  std::vector<int32_t> nb;   // neighbours b > a, sorted, unique (compacted)
};

void gen_keys(const Model& M, int64_t c0, int64_t c1, uint64_t* out) {
  parallel_for(c1 - c0, [&](int, int64_t a, int64_t b) {
    for (int64_t e = a; e < b; ++e) out[e] = edge_key(M, uint64_t(c0 + e));
  });
}

Upper build_upper(int64_t n, const std::vector<uint64_t>& keys) {
  const int64_t m = int64_t(keys.size());
  int T = nthreads();
  std::vector<std::vector<int64_t>> cnt(T, std::vector<int64_t>(n, 0));
  parallel_for(m, [&](int t, int64_t a, int64_t b) {
    auto& c = cnt[t];
    for (int64_t e = a; e < b; ++e)
      if (keys[e] != UINT64_MAX) c[keys[e] / uint64_t(n)]++;
  });
  std::vector<int64_t> ptr(n + 1, 0);
  int64_t run = 0;
  for (int64_t r = 0; r < n; ++r) {
    ptr[r] = run;
    for (int t = 0; t < T; ++t) { int64_t c = cnt[t][r]; cnt[t][r] = run; run += c; }
  }
  ptr[n] = run;
  std::vector<int32_t> nb(run);
  parallel_for(m, [&](int t, int64_t a, int64_t b) {
    auto& o = cnt[t];
    for (int64_t e = a; e < b; ++e) {
      uint64_t k = keys[e];
      if (k != UINT64_MAX) nb[o[k / uint64_t(n)]++] = int32_t(k % uint64_t(n));
    }
  });
  std::vector<int64_t> uniq(n, 0);
  parallel_for(n, [&](int, int64_t a, int64_t b) {
    for (int64_t r = a; r < b; ++r) {
      int32_t* s = nb.data() + ptr[r];
      int32_t* e = nb.data() + ptr[r + 1];
      std::sort(s, e);
      uniq[r] = std::unique(s, e) - s;
    }
  });
  Upper U;
  U.ptr.assign(n + 1, 0);
  for (int64_t r = 0; r < n; ++r) U.ptr[r + 1] = U.ptr[r] + uniq[r];
  U.nb.resize(U.ptr[n]);
  parallel_for(n, [&](int, int64_t a, int64_t b) {
    for (int64_t r = a; r < b; ++r)
      std::memcpy(U.nb.data() + U.ptr[r], nb.data() + ptr[r], sizeof(int32_t) * uniq[r]);
  });
  return U;
}

}  // namespace

extern "C" int64_t synth_sbm_csr(int64_t n, const int64_t* cdf, const int32_t* class_of,
                                 const int64_t* class_start, const int32_t* sub_of,
                                 const int64_t* sub_start, const int64_t* id_of, double p_sub,
                                 double p_class, uint64_t key, uint64_t drop_key,
                                 int64_t m_target, int64_t* rowptr, int32_t* col) {
  Model M{n, cdf, class_start, sub_start, id_of, class_of, sub_of, p_sub, p_class, key};
  int64_t m_gen = m_target, m_done = 0;
  std::vector<uint64_t> keys;
  Upper U;
  for (;;) {
    keys.resize(m_gen);
    gen_keys(M, m_done, m_gen, keys.data() + m_done);
    m_done = m_gen;
    U = build_upper(n, keys);
    int64_t cnt = U.ptr[n];
    if (cnt >= m_target) break;
    m_gen = m_gen + ((m_target - cnt) * 5) / 4 + 64;
  }
  std::vector<uint64_t>().swap(keys);
  // keep the m_target smallest (hash, key) pairs
  std::vector<uint8_t> keep(U.ptr[n], 1);
  if (U.ptr[n] > m_target) {
    std::vector<std::pair<uint64_t, uint64_t>> hk(U.ptr[n]);
    parallel_for(n, [&](int, int64_t a, int64_t b) {
      for (int64_t r = a; r < b; ++r)
        for (int64_t i = U.ptr[r]; i < U.ptr[r + 1]; ++i) {
          uint64_t k = uint64_t(r) * uint64_t(n) + uint64_t(U.nb[i]);
          hk[i] = {mix64(k ^ drop_key), k};
        }
    });
    std::vector<std::pair<uint64_t, uint64_t>> tmp(hk);
    std::nth_element(tmp.begin(), tmp.begin() + (m_target - 1), tmp.end());
    auto thr = tmp[m_target - 1];
    for (int64_t i = 0; i < U.ptr[n]; ++i) keep[i] = hk[i] <= thr;
  }
  // symmetric CSR
  std::vector<int64_t> deg(n, 0);
  for (int64_t r = 0; r < n; ++r)
    for (int64_t i = U.ptr[r]; i < U.ptr[r + 1]; ++i)
      if (keep[i]) { deg[r]++; deg[U.nb[i]]++; }
  rowptr[0] = 0;
  for (int64_t r = 0; r < n; ++r) rowptr[r + 1] = rowptr[r] + deg[r];
  std::vector<int64_t> pos(rowptr, rowptr + n);
  for (int64_t r = 0; r < n; ++r)
    for (int64_t i = U.ptr[r]; i < U.ptr[r + 1]; ++i)
      if (keep[i]) { col[pos[r]++] = U.nb[i]; col[pos[U.nb[i]]++] = int32_t(r); }
  parallel_for(n, [&](int, int64_t a, int64_t b) {
    for (int64_t r = a; r < b; ++r) std::sort(col + rowptr[r], col + rowptr[r + 1]);
  });
  return rowptr[n] / 2;
}
