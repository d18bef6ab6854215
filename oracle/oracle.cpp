// oracle/oracle.cpp — TEST INFRASTRUCTURE ONLY.  Plain, slow, obviously-correct CPU
// reference for the SpGEMM hot path (C = A x B, CSR).  Only tests/, __graft_entry__.smoke()
// and bench.py's cpu_baseline / --impl reference legs may load this library; the product
// path (paper_conf_ipps_ramamoorthybsk15_b200/) never does and shares no code with it.
//
// What it computes follows PAPER.md directly:
//   * Row-Row (Gustavson) formulation, PAPER.md L62 (§II-A.a):
//       C(i,:) = sum_k A(i, j_k) * B(j_k, :)   over the stored entries of row i of A.
//     Every stored pair (A(i,k), B(k,j)) contributes one "intermediate product"; its count
//     per row is the row's flop count f_i.
//   * Phase IV merge semantics, PAPER.md L154-156 (§III-D): tuples <r,c,v> with identical
//     (r,c) are added ("add like-tuples"); the output holds distinct (r,c) in sorted order.
//     Nothing is dropped for being numerically zero (reading R2).
//   * Multi-GPU split points (reading R10): s_0 = 0, s_P = M,
//     s_r = min{ i : Pf[i]*P >= r*F }, Pf the exclusive prefix of f.
//   * Log2 flop bins: bin = -1 if f = 0 else ceil(log2 f).
//   * Sparse x dense (CSTMM / csrmm, the extension named in PAPER.md L289, §VI):
//       C(i,:) = sum_k A(i,k) * D(k,:) over the stored entries of row i of A — the same Row-Row
//     formulation with a dense right operand; C is dense.
//
// Values are promoted to double; for each output entry the oracle also returns
// abs = sum |a*b| so that tests can apply the per-entry bound |gpu - sum| <= rtol * abs.
//
// Parity pins (tests/test_oracle.py): Fig. 2 worked example (tests/golden/fig2.txt),
// dense triple loop + Boolean pattern product on tiny random inputs, identity and
// permutation products, C*1 = A*(B*1), c_i <= f_i, nnz(C) <= F, scipy on positive data,
// brute-force split points and closed-form bins.
#include <cstdint>
#include <cstdlib>
#include <map>
#include <thread>
#include <utility>
#include <vector>

namespace {

struct Mat {
  int32_t nrows;
  const int32_t* rp;
  const int32_t* ci;
  const void* v;
  int is_f64;
  double val(int64_t p) const {
    return is_f64 ? ((const double*)v)[p] : (double)((const float*)v)[p];
  }
};

// One row of C by the Row-Row formulation with a sorted-map accumulator
// (like-tuples are added, output in (r,c) order).
void row_product(const Mat& A, const Mat& B, int32_t i, std::map<int32_t, std::pair<double, double>>& acc) {
  acc.clear();
  for (int64_t p = A.rp[i]; p < A.rp[i + 1]; ++p) {
    int32_t k = A.ci[p];
    double a = A.val(p);
    for (int64_t q = B.rp[k]; q < B.rp[k + 1]; ++q) {
      double t = a * B.val(q);
      auto& e = acc[B.ci[q]];
      e.first += t;
      e.second += t < 0 ? -t : t;
    }
  }
}

template <class F>
void run_threads(int32_t r0, int32_t r1, int nthreads, F f) {
  if (nthreads <= 1 || r1 - r0 < 2) {
    f(r0, r1);
    return;
  }
  std::vector<std::thread> th;
  for (int t = 0; t < nthreads; ++t) {
    int32_t b = r0 + (int32_t)((int64_t)(r1 - r0) * t / nthreads);
    int32_t e = r0 + (int32_t)((int64_t)(r1 - r0) * (t + 1) / nthreads);
    th.emplace_back([=] { f(b, e); });
  }
  for (auto& x : th) x.join();
}

}  // namespace

extern "C" {

// f_i = number of intermediate products of row i = sum over stored A(i,k) of nnz(B(k,:)).
void orc_row_flops(int32_t M, const int32_t* rpA, const int32_t* colA, const int32_t* rpB, int64_t* f) {
  for (int32_t i = 0; i < M; ++i) {
    int64_t s = 0;
    for (int64_t p = rpA[i]; p < rpA[i + 1]; ++p) s += (int64_t)rpB[colA[p] + 1] - rpB[colA[p]];
    f[i] = s;
  }
}

// bin_i = -1 if f_i = 0, else the smallest b with 2^b >= f_i;  hist[b+1] counts rows.
void orc_bins(int32_t M, const int64_t* f, int32_t* bin, int64_t* hist /* [65]: bins -1..63 */) {
  for (int b = 0; b < 65; ++b) hist[b] = 0;
  for (int32_t i = 0; i < M; ++i) {
    int32_t b = -1;
    if (f[i] > 0) {
      b = 0;
      while (((int64_t)1 << b) < f[i]) ++b;
    }
    bin[i] = b;
    hist[b + 1]++;
  }
}

// s_0 = 0, s_P = M, s_r = min{ i in [0,M] : Pf[i]*P >= r*F } for 0 < r < P.
void orc_split_points(int32_t M, const int64_t* f, int32_t P, int32_t* s) {
  std::vector<int64_t> Pf((size_t)M + 1, 0);
  for (int32_t i = 0; i < M; ++i) Pf[i + 1] = Pf[i] + f[i];
  int64_t F = Pf[M];
  s[0] = 0;
  s[P] = M;
  for (int32_t r = 1; r < P; ++r) {
    int32_t i = 0;
    while (i < M && (__int128)Pf[i] * P < (__int128)r * F) ++i;
    s[r] = i;
  }
}

// Symbolic: c[i - r0] = |{ j : exists stored A(i,k), B(k,j) }| for rows [r0, r1).
void orc_spgemm_count(int32_t r0, int32_t r1, int32_t M, const int32_t* rpA, const int32_t* colA, const void* valA,
                      int32_t K, const int32_t* rpB, const int32_t* colB, const void* valB, int is_f64,
                      int64_t* c, int nthreads) {
  Mat A{M, rpA, colA, valA, is_f64}, B{K, rpB, colB, valB, is_f64};
  run_threads(r0, r1, nthreads, [&](int32_t b, int32_t e) {
    std::map<int32_t, std::pair<double, double>> acc;
    for (int32_t i = b; i < e; ++i) {
      row_product(A, B, i, acc);
      c[i - r0] = (int64_t)acc.size();
    }
  });
}

// Numeric: rows [r0, r1) written at rowptr[i - r0] (rowptr local, rowptr[0] may be != 0 only
// through the caller's choice); columns ascending; val = sum of products, absv = sum |products|.
void orc_spgemm_fill(int32_t r0, int32_t r1, int32_t M, const int32_t* rpA, const int32_t* colA, const void* valA,
                     int32_t K, const int32_t* rpB, const int32_t* colB, const void* valB, int is_f64,
                     const int64_t* rowptr, int32_t* col, double* val, double* absv, int nthreads) {
  Mat A{M, rpA, colA, valA, is_f64}, B{K, rpB, colB, valB, is_f64};
  run_threads(r0, r1, nthreads, [&](int32_t b, int32_t e) {
    std::map<int32_t, std::pair<double, double>> acc;
    for (int32_t i = b; i < e; ++i) {
      row_product(A, B, i, acc);
      int64_t o = rowptr[i - r0];
      for (auto& kv : acc) {
        col[o] = kv.first;
        val[o] = kv.second.first;
        if (absv) absv[o] = kv.second.second;
        ++o;
      }
    }
  });
}

// Sparse x dense: C (M x n, row-major, double) = A (CSR) x D (K x n, row-major, double), rows
// [0, M); absv = sum |A(i,k) * D(k,j)| per entry (tolerance bound).  Plain row loop.
void orc_csrmm(int32_t M, const int32_t* rpA, const int32_t* colA, const void* valA, int is_f64, const double* D,
               int64_t n, double* C, double* absv) {
  Mat A{M, rpA, colA, valA, is_f64};
  for (int32_t i = 0; i < M; ++i)
    for (int64_t j = 0; j < n; ++j) {
      double s = 0.0, t = 0.0;
      for (int64_t p = A.rp[i]; p < A.rp[i + 1]; ++p) {
        const double x = A.val(p) * D[(int64_t)A.ci[p] * n + j];
        s += x;
        t += x < 0 ? -x : x;
      }
      C[(int64_t)i * n + j] = s;
      absv[(int64_t)i * n + j] = t;
    }
}

}  // extern "C"
