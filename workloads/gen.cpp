// workloads/gen.cpp — seeded synthetic sparse-matrix generators (input recipe only).
//
// This module holds NONE of the SpGEMM method's arithmetic: it only draws sparse
// patterns and values.  It is the one piece shared by the oracle tests, the GPU
// parity tests and bench.py (DESIGN.md §3 "input recipe").
//
//   * Chung-Lu power-law matrices with a rank-correlation knob between a vertex's
//     out-rank (row weight) and in-rank (column weight) — SURVEY.md Appendix A.
//     Row sizes follow a power law with exponent alpha, the property the paper
//     studies (Fig. 1, L183 Table I "alpha").
//   * R-MAT with the GTgraph default quadrant probabilities (the generator the
//     paper uses for its synthetic experiments, ref [3]).
//
// Every random draw is a pure function of (seed, stream, index) — a counter-based
// generator — so results do not depend on thread count or call order.
//
// Output: 0-based CSR, int32 row_ptr/col_idx, columns strictly ascending within a
// row (duplicates removed), values U[1,2) drawn per stored entry.
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <numeric>
#include <thread>
#include <vector>

namespace {

inline uint64_t mix64(uint64_t z) {  // splitmix64 finaliser
  z += 0x9e3779b97f4a7c15ULL;
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}
inline uint64_t ctr_rng(uint64_t seed, uint64_t stream, uint64_t idx) {
  uint64_t key = mix64(seed ^ mix64(stream * 0x2545F4914F6CDD1DULL + 0x1234567ULL));
  return mix64(key ^ (idx * 0xD1B54A32D192ED03ULL));
}
inline double u01(uint64_t r) { return (double)(r >> 11) * (1.0 / 9007199254740992.0); }  // [0,1)

enum : uint64_t { S_PERM_R = 1, S_PERM_C, S_NORMAL, S_ROW, S_COL, S_VAL, S_RMAT, S_RELABEL };

int nthreads() {
  unsigned n = std::thread::hardware_concurrency();
  return n == 0 ? 1 : (int)std::min(n, 64u);
}

template <class F>
void parallel_for(int64_t n, F f) {
  int T = nthreads();
  if (n < 100000) T = 1;
  std::vector<std::thread> th;
  for (int t = 0; t < T; ++t) {
    int64_t b = n * t / T, e = n * (t + 1) / T;
    th.emplace_back([=, &f] { f(b, e); });
  }
  for (auto& x : th) x.join();
}

// Fisher-Yates permutation of 0..n-1 driven by the counter RNG.
std::vector<int32_t> permutation(int64_t n, uint64_t seed, uint64_t stream) {
  std::vector<int32_t> p(n);
  std::iota(p.begin(), p.end(), 0);
  for (int64_t i = n - 1; i > 0; --i) {
    uint64_t j = ctr_rng(seed, stream, (uint64_t)i) % (uint64_t)(i + 1);
    std::swap(p[i], p[j]);
  }
  return p;
}

// Power-law weights w(i) ∝ (i+1)^(-1/(alpha-1)), total = target, clipped at cap with
// iterative rescaling of the unclipped part.
std::vector<double> powerlaw_weights(int64_t n, double alpha, double target, double cap) {
  std::vector<double> w(n);
  double ex = -1.0 / (alpha - 1.0);
  for (int64_t i = 0; i < n; ++i) w[i] = std::pow((double)(i + 1), ex);
  std::vector<char> clipped(n, 0);
  for (int it = 0; it < 200; ++it) {
    double fixed = 0, free_sum = 0;
    for (int64_t i = 0; i < n; ++i) (clipped[i] ? fixed : free_sum) += clipped[i] ? cap : w[i];
    if (free_sum <= 0) break;
    double s = (target - fixed) / free_sum;
    bool changed = false;
    for (int64_t i = 0; i < n; ++i) {
      if (clipped[i]) { w[i] = cap; continue; }
      w[i] *= s;
      if (cap > 0 && w[i] > cap) { clipped[i] = 1; changed = true; }
    }
    if (!changed) break;
  }
  for (int64_t i = 0; i < n; ++i) if (clipped[i]) w[i] = cap;
  return w;
}

struct Result {
  int32_t nrows = 0, ncols = 0;
  std::vector<int32_t> row_ptr, col;
  uint64_t val_seed = 0;
};

// Build CSR from (row, col) pairs: counting sort by row, sort + unique inside rows.
void build_csr(Result& R, std::vector<int32_t>& pr, std::vector<int32_t>& pc) {
  int64_t m = (int64_t)pr.size();
  std::vector<int64_t> cnt((size_t)R.nrows + 1, 0);
  for (int64_t e = 0; e < m; ++e) cnt[pr[e] + 1]++;
  for (int32_t i = 0; i < R.nrows; ++i) cnt[i + 1] += cnt[i];
  std::vector<int32_t> tmp(m);
  {
    std::vector<int64_t> pos(cnt.begin(), cnt.end() - 1);
    for (int64_t e = 0; e < m; ++e) tmp[pos[pr[e]]++] = pc[e];
  }
  std::vector<int32_t>().swap(pr);
  std::vector<int32_t>().swap(pc);
  std::vector<int32_t> len(R.nrows);
  parallel_for(R.nrows, [&](int64_t b, int64_t e) {
    for (int64_t i = b; i < e; ++i) {
      auto* s = tmp.data() + cnt[i];
      auto* t = tmp.data() + cnt[i + 1];
      std::sort(s, t);
      len[i] = (int32_t)(std::unique(s, t) - s);
    }
  });
  R.row_ptr.assign((size_t)R.nrows + 1, 0);
  for (int32_t i = 0; i < R.nrows; ++i) R.row_ptr[i + 1] = R.row_ptr[i] + len[i];
  R.col.resize(R.row_ptr[R.nrows]);
  parallel_for(R.nrows, [&](int64_t b, int64_t e) {
    for (int64_t i = b; i < e; ++i)
      std::memcpy(R.col.data() + R.row_ptr[i], tmp.data() + cnt[i], sizeof(int32_t) * len[i]);
  });
}

}  // namespace

extern "C" {

// Chung-Lu with rank correlation.
//   sigma < 0  : independent column ranks;   sigma >= 0 : in-rank = rank(log(1+out_rank) + sigma*N(0,1))
//   (correlation requires nrows == ncols).  m = round(m_factor * nnz_target) pairs are drawn.
void* wl_chung_lu(int32_t nrows, int32_t ncols, double alpha_r, double alpha_c, int64_t nnz_target,
                  double row_cap, double col_cap, double sigma, double m_factor, uint64_t seed) {
  auto* R = new Result;
  R->nrows = nrows;
  R->ncols = ncols;
  R->val_seed = seed;
  std::vector<double> wr = powerlaw_weights(nrows, alpha_r, (double)nnz_target, row_cap);
  std::vector<double> wc = powerlaw_weights(ncols, alpha_c, (double)nnz_target, col_cap);
  std::vector<double> cr(nrows), cc(ncols);
  std::partial_sum(wr.begin(), wr.end(), cr.begin());
  std::partial_sum(wc.begin(), wc.end(), cc.begin());
  std::vector<int32_t> perm_r = permutation(nrows, seed, S_PERM_R);  // out-rank -> vertex
  std::vector<int32_t> by_in_rank(ncols);                            // in-rank  -> vertex
  if (sigma >= 0 && nrows == ncols) {
    std::vector<int32_t> rank_of(nrows);
    for (int32_t r = 0; r < nrows; ++r) rank_of[perm_r[r]] = r;
    std::vector<double> score(ncols);
    for (int32_t v = 0; v < ncols; ++v) {
      double u1 = u01(ctr_rng(seed, S_NORMAL, 2 * (uint64_t)v));
      double u2 = u01(ctr_rng(seed, S_NORMAL, 2 * (uint64_t)v + 1));
      double z = std::sqrt(-2.0 * std::log(1.0 - u1)) * std::cos(6.283185307179586 * u2);
      score[v] = std::log(1.0 + (double)rank_of[v]) + sigma * z;
    }
    std::iota(by_in_rank.begin(), by_in_rank.end(), 0);
    std::sort(by_in_rank.begin(), by_in_rank.end(), [&](int32_t a, int32_t b) {
      return score[a] < score[b] || (score[a] == score[b] && a < b);
    });
  } else {
    by_in_rank = permutation(ncols, seed, S_PERM_C);
  }
  int64_t m = (int64_t)std::llround(m_factor * (double)nnz_target);
  std::vector<int32_t> pr(m), pc(m);
  double tr = cr.back(), tc = cc.back();
  parallel_for(m, [&](int64_t b, int64_t e) {
    for (int64_t k = b; k < e; ++k) {
      double ur = u01(ctr_rng(seed, S_ROW, (uint64_t)k)) * tr;
      double uc = u01(ctr_rng(seed, S_COL, (uint64_t)k)) * tc;
      int64_t r = std::upper_bound(cr.begin(), cr.end(), ur) - cr.begin();
      int64_t s = std::upper_bound(cc.begin(), cc.end(), uc) - cc.begin();
      if (r >= nrows) r = nrows - 1;
      if (s >= ncols) s = ncols - 1;
      pr[k] = perm_r[r];
      pc[k] = by_in_rank[s];
    }
  });
  build_csr(*R, pr, pc);
  return R;
}

// R-MAT (GTgraph defaults a,b,c,d) on 2^scale vertices, edge_factor * 2^scale edges, vertices
// randomly relabelled, duplicates removed, self-loops kept.
void* wl_rmat(int32_t scale, int32_t edge_factor, double a, double b, double c, uint64_t seed) {
  auto* R = new Result;
  int64_t n = (int64_t)1 << scale;
  R->nrows = R->ncols = (int32_t)n;
  R->val_seed = seed;
  int64_t m = n * edge_factor;
  std::vector<int32_t> relabel = permutation(n, seed, S_RELABEL);
  std::vector<int32_t> pr(m), pc(m);
  double ab = a + b, abc = a + b + c;
  parallel_for(m, [&](int64_t lo, int64_t hi) {
    for (int64_t e = lo; e < hi; ++e) {
      int64_t r = 0, s = 0;
      for (int l = 0; l < scale; ++l) {
        double u = u01(ctr_rng(seed, S_RMAT, (uint64_t)e * 64 + l));
        int rb = u >= ab, cb = (u >= a && u < ab) || u >= abc;
        r = (r << 1) | rb;
        s = (s << 1) | cb;
      }
      pr[e] = relabel[r];
      pc[e] = relabel[s];
    }
  });
  build_csr(*R, pr, pc);
  return R;
}

void wl_sizes(void* h, int32_t* nrows, int32_t* ncols, int64_t* nnz) {
  auto* R = (Result*)h;
  *nrows = R->nrows;
  *ncols = R->ncols;
  *nnz = (int64_t)R->col.size();
}

// Copies CSR out; values U[1,2) per stored entry: fp64 has 52 random mantissa bits, fp32 23
// (exactly representable, never rounds up to 2).  val_kind: 0 = fp32, 1 = fp64.
void wl_copy(void* h, int32_t* row_ptr, int32_t* col, void* val, int val_kind) {
  auto* R = (Result*)h;
  std::memcpy(row_ptr, R->row_ptr.data(), sizeof(int32_t) * R->row_ptr.size());
  std::memcpy(col, R->col.data(), sizeof(int32_t) * R->col.size());
  int64_t nnz = (int64_t)R->col.size();
  uint64_t vs = R->val_seed;
  if (val == nullptr) return;
  if (val_kind == 1) {
    double* v = (double*)val;
    parallel_for(nnz, [&](int64_t b, int64_t e) {
      for (int64_t p = b; p < e; ++p)
        v[p] = 1.0 + (double)(ctr_rng(vs, S_VAL, (uint64_t)p) >> 12) * (1.0 / 4503599627370496.0);
    });
  } else {
    float* v = (float*)val;
    parallel_for(nnz, [&](int64_t b, int64_t e) {
      for (int64_t p = b; p < e; ++p)
        v[p] = 1.0f + (float)(ctr_rng(vs, S_VAL, (uint64_t)p) >> 41) * (1.0f / 8388608.0f);
    });
  }
}

void wl_free(void* h) { delete (Result*)h; }

}  // extern "C"
