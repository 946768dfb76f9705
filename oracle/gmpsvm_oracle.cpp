// gmpsvm_oracle.cpp -- plain FP64 CPU oracle for the GMP-SVM hot path.
//
// TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
// cpu_baseline / --impl reference legs may load this library.  It shares no code,
// header, table or helper with the CUDA path (paper_conf_icde_wenshcc19_b200/csrc),
// and neither side includes or links the other.
//
// Every function follows the paper (PAPER.md = /root/reference/PAPER.md) step by step,
// in FP64, with the readings of SURVEY.md §8(c) where the paper is silent or garbled
// (each listed in DESIGN.md "Readings").  No blocking, fusion or reordering: the
// kernel value is the direct difference formula of L75, not the norm expansion.
//
// Pins (tests/test_oracle_*.py, -m "not gpu"):
//   oracle_rbf_matrix   -> scipy.spatial.distance.cdist (library routine), K_ii = 1
//   oracle_smo          -> brute-force active-set QP (n <= 8), 2-point closed form,
//                          sklearn/LibSVM at tight tol, KKT at eps, dual monotone
//   oracle_rho          -> sklearn intercept_, 2-point closed form (b = 0)
//   oracle_sigmoid_fit  -> scipy BFGS on Eq 13, zero gradient, constant-v closed form
//   oracle_couple       -> k=2 closed form, Bradley-Terry consistent r, Eq 15 by inverse,
//                          direct minimisation of Eq 14, Example 1 ordering (L210-L216)
//   oracle_predict      -> in-sample identity v = f + y - rho (Eq 3 vs Eq 11)
// No function here is "parity unpinned".
#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <functional>
#include <limits>
#include <list>
#include <thread>
#include <vector>

namespace {

const double kTau = 1e-12;  // eta floor, SURVEY §8(c) #3

// Run fn(i) for i in [0, n) on up to nthreads threads (dynamic chunking).
void parallel_for(int64_t n, int nthreads, const std::function<void(int64_t)>& fn) {
  if (nthreads <= 1 || n <= 1) {
    for (int64_t i = 0; i < n; ++i) fn(i);
    return;
  }
  std::atomic<int64_t> next(0);
  int nt = (int)std::min<int64_t>(nthreads, n);
  std::vector<std::thread> th;
  for (int t = 0; t < nt; ++t)
    th.emplace_back([&]() {
      for (;;) {
        int64_t i = next.fetch_add(1);
        if (i >= n) break;
        fn(i);
      }
    });
  for (auto& x : th) x.join();
}

// Kernel functions: the Gaussian kernel K(x_i, x_j) = exp(-gamma ||x_i - x_j||^2)
// (direct differences) is the default; oracle_set_kernel selects the other kernels the paper lists
// (NEXT-4): linear x_i.x_j, polynomial (gamma x_i.x_j + coef0)^degree, sigmoid
// tanh(gamma x_i.x_j + coef0) -- the LibSVM definitions.  Set before a call, process-wide.
struct KernelSpec {
  int type = 0;  // 0 RBF, 1 linear, 2 polynomial, 3 sigmoid
  double coef0 = 0.0;
  int degree = 3;
};
KernelSpec g_kernel;

inline double rbf(const float* xi, const float* xj, int d, double gamma) {
  if (g_kernel.type != 0) {
    double dot = 0.0;
    for (int c = 0; c < d; ++c) dot += (double)xi[c] * (double)xj[c];
    if (g_kernel.type == 1) return dot;
    if (g_kernel.type == 2) return std::pow(gamma * dot + g_kernel.coef0, (double)g_kernel.degree);
    return std::tanh(gamma * dot + g_kernel.coef0);
  }
  double s = 0.0;
  for (int c = 0; c < d; ++c) {
    double diff = (double)xi[c] - (double)xj[c];
    s += diff * diff;
  }
  return std::exp(-gamma * s);
}

// Kernel rows of one binary problem, computed on demand, LRU-cached (memory capped).
// Caching a row does not change its arithmetic.
struct KernelRows {
  const float* const* x;  // x[i] -> row i of the problem
  int64_t n;
  int d;
  double gamma;
  size_t cap;
  std::vector<std::vector<double>> slot;
  std::vector<int64_t> slot_of, owner;
  std::list<int64_t> lru;  // front = most recent slot
  std::vector<std::list<int64_t>::iterator> where;

  KernelRows(const float* const* x_, int64_t n_, int d_, double g, size_t bytes)
      : x(x_), n(n_), d(d_), gamma(g) {
    cap = std::max<size_t>(2, bytes / (sizeof(double) * (size_t)std::max<int64_t>(n, 1)));
    cap = std::min<size_t>(cap, (size_t)n);
    slot_of.assign(n, -1);
  }
  const double* row(int64_t i) {
    int64_t s = slot_of[i];
    if (s >= 0) {
      lru.erase(where[s]);
      lru.push_front(s);
      where[s] = lru.begin();
      return slot[s].data();
    }
    if (slot.size() < cap) {
      s = (int64_t)slot.size();
      slot.emplace_back(n);
      owner.push_back(-1);
      lru.push_front(s);
      where.push_back(lru.begin());
    } else {
      s = lru.back();
      lru.pop_back();
      slot_of[owner[s]] = -1;
      lru.push_front(s);
      where[s] = lru.begin();
    }
    owner[s] = i;
    slot_of[i] = s;
    double* r = slot[s].data();
    for (int64_t j = 0; j < n; ++j) r[j] = rbf(x[i], x[j], d, gamma);
    return r;
  }
};

// I_u = I1 u I2 u I3, I_l = I1 u I4 u I5.
inline bool in_u(int y, double a, double C) { return (y > 0 && a < C) || (y < 0 && a > 0); }
inline bool in_l(int y, double a, double C) { return (y > 0 && a > 0) || (y < 0 && a < C); }

// SMO, Algorithm 1 with Eq 3-10 (L86-L138), WSS2 (Eq 5, ref [17]).
// Returns 0 on convergence, 1 if the iteration cap was hit (LibSVM-style warning).
int smo(const float* const* x, const int* y, int64_t n, int d, double C, double gamma, double eps,
        int64_t max_iter, double* alpha, double* f, int64_t* iters_out, double* dual_trace,
        int64_t trace_cap, size_t cache_bytes) {
  KernelRows K(x, n, d, gamma, cache_bytes);
  std::vector<double> Kdiag(n);  // K(x_t, x_t), needed by every eta_t of Eq 5
  for (int64_t t = 0; t < n; ++t) Kdiag[t] = rbf(x[t], x[t], d, gamma);
  for (int64_t i = 0; i < n; ++i) {  // Alg 1 lines 1-2: alpha_i <- 0, f_i <- -y_i
    alpha[i] = 0.0;
    f[i] = -(double)y[i];
  }
  if (max_iter <= 0) max_iter = std::max<int64_t>(10000000, 100 * n);
  int status = 1;
  int64_t it = 0;
  for (; it < max_iter; ++it) {
    if (dual_trace && it < trace_cap) {  // W = 1/2 sum alpha_i (1 - y_i f_i)  (Eq 2 with Eq 3)
      double w = 0.0;
      for (int64_t i = 0; i < n; ++i) w += alpha[i] * (1.0 - y[i] * f[i]);
      dual_trace[it] = 0.5 * w;
    }
    // Step 1: u = argmin_{I_u} f (Eq 4); f_max = max_{I_l} f (Eq 10). Ties: lowest index.
    int64_t u = -1;
    double fu = std::numeric_limits<double>::infinity();
    double fmax = -std::numeric_limits<double>::infinity();
    for (int64_t i = 0; i < n; ++i) {
      if (in_u(y[i], alpha[i], C) && f[i] < fu) {
        fu = f[i];
        u = i;
      }
      if (in_l(y[i], alpha[i], C) && f[i] > fmax) fmax = f[i];
    }
    // Stop (Eq 9 with tolerance eps)
    if (u < 0 || fmax == -std::numeric_limits<double>::infinity() || fmax - fu < eps) {
      status = 0;
      break;
    }
    const double* Ku = K.row(u);
    // l = argmax_{t in I_l, f_t > f_u} (f_u - f_t)^2 / eta_t (Eq 5), eta floored at tau.
    int64_t l = -1;
    double best = -std::numeric_limits<double>::infinity();
    for (int64_t t = 0; t < n; ++t) {
      if (!in_l(y[t], alpha[t], C) || !(f[t] > fu)) continue;
      double eta = Ku[u] + Kdiag[t] - 2.0 * Ku[t];
      if (eta < kTau) eta = kTau;
      double diff = fu - f[t];
      double score = diff * diff / eta;
      if (score > best) {
        best = score;
        l = t;
      }
    }
    if (l < 0) {  // cannot happen when fmax - fu >= eps > 0; treat as converged
      status = 0;
      break;
    }
    std::vector<double> Ku_copy(Ku, Ku + n);  // keep row u while row l is fetched
    const double* Kl = K.row(l);
    // Step 2: Eq 6-7 with the clipping of L123 made explicit.
    double eta = Ku_copy[u] + Kl[l] - 2.0 * Ku_copy[l];
    if (eta < kTau) eta = kTau;
    double s = (f[l] - fu) / eta;
    double Uu = y[u] > 0 ? C - alpha[u] : alpha[u];
    double Ll = y[l] > 0 ? alpha[l] : C - alpha[l];
    bool bu = false, bl = false;
    if (Uu <= s) {
      s = Uu;
      bu = true;
    }
    if (Ll <= s) {
      if (Ll < s) bu = false;
      s = Ll;
      bl = true;
    }
    alpha[u] += y[u] * s;
    alpha[l] -= y[l] * s;
    if (bu) alpha[u] = y[u] > 0 ? C : 0.0;
    if (bl) alpha[l] = y[l] > 0 ? 0.0 : C;
    // Step 3: Eq 8, f_i += (a_u' - a_u) y_u K_ui + (a_l' - a_l) y_l K_li = s (K_ui - K_li)
    for (int64_t i = 0; i < n; ++i) f[i] += s * (Ku_copy[i] - Kl[i]);
  }
  if (iters_out) *iters_out = it;
  return status;
}

// Bias (absent from the paper; Table 4 compares it, L425-L436): LibSVM's rule in f terms.
// f must be exact for alpha (caller recomputes it).
double rho_of(const double* alpha, const double* f, const int* y, int64_t n, double C) {
  double sum_free = 0.0, ub = std::numeric_limits<double>::infinity(),
         lb = -std::numeric_limits<double>::infinity();
  int64_t n_free = 0;
  for (int64_t i = 0; i < n; ++i) {
    if (alpha[i] > 0.0 && alpha[i] < C) {
      sum_free += f[i];
      ++n_free;
    } else {
      if (in_u(y[i], alpha[i], C)) ub = std::min(ub, f[i]);
      if (in_l(y[i], alpha[i], C)) lb = std::max(lb, f[i]);
    }
  }
  if (n_free > 0) return sum_free / (double)n_free;
  return 0.5 * (ub + lb);
}

// Eq 3 evaluated from scratch: f_i = sum_j alpha_j y_j K(x_i, x_j) - y_i.
void exact_f(const float* const* x, const int* y, int64_t n, int d, double gamma, const double* alpha,
             double* f, int nthreads) {
  std::vector<int64_t> sv;
  for (int64_t j = 0; j < n; ++j)
    if (alpha[j] != 0.0) sv.push_back(j);
  parallel_for(n, nthreads, [&](int64_t i) {
    double s = 0.0;
    for (int64_t j : sv) s += alpha[j] * y[j] * rbf(x[i], x[j], d, gamma);
    f[i] = s - (double)y[i];
  });
}

// Negative log likelihood of Eq 13 (read as a minimisation), stable form.
double nll(const double* v, const double* t, int64_t n, double A, double B) {
  double F = 0.0;
  for (int64_t i = 0; i < n; ++i) {
    double z = v[i] * A + B;
    if (z >= 0)
      F += t[i] * z + std::log1p(std::exp(-z));
    else
      F += (t[i] - 1.0) * z + std::log1p(std::exp(z));
  }
  return F;
}

// Platt sigmoid fit (Eq 12-13), Newton with backtracking, constants of ref [15].
int sigmoid_fit(const double* v, const int* y, int64_t n, double* A_out, double* B_out, int* iters) {
  const int max_iter = 100;
  const double min_step = 1e-10, sigma = 1e-12, geps = 1e-5;
  double Np = 0, Nm = 0;
  for (int64_t i = 0; i < n; ++i) (y[i] > 0 ? Np : Nm) += 1.0;
  const double hi = (Np + 1.0) / (Np + 2.0), lo = 1.0 / (Nm + 2.0);  // targets t_i (L183)
  std::vector<double> t(n);
  for (int64_t i = 0; i < n; ++i) t[i] = y[i] > 0 ? hi : lo;
  double A = 0.0, B = std::log((Nm + 1.0) / (Np + 1.0));
  double F = nll(v, t.data(), n, A, B);
  int it = 0, status = 0;
  for (; it < max_iter; ++it) {
    // gradient (L254-L255 with the sign of the minimisation) and Hessian
    double h11 = sigma, h22 = sigma, h21 = 0.0, g1 = 0.0, g2 = 0.0;
    for (int64_t i = 0; i < n; ++i) {
      double z = v[i] * A + B, p, q;
      if (z >= 0) {
        double e = std::exp(-z);
        p = e / (1.0 + e);
        q = 1.0 / (1.0 + e);
      } else {
        double e = std::exp(z);
        p = 1.0 / (1.0 + e);
        q = e / (1.0 + e);
      }
      double d2 = p * q;
      h11 += v[i] * v[i] * d2;
      h22 += d2;
      h21 += v[i] * d2;
      double d1 = t[i] - p;
      g1 += v[i] * d1;
      g2 += d1;
    }
    if (std::fabs(g1) < geps && std::fabs(g2) < geps) break;
    double det = h11 * h22 - h21 * h21;
    double dA = -(h22 * g1 - h21 * g2) / det;
    double dB = -(-h21 * g1 + h11 * g2) / det;
    double gd = g1 * dA + g2 * dB;
    double step = 1.0;
    while (step >= min_step) {
      double nA = A + step * dA, nB = B + step * dB;
      double nF = nll(v, t.data(), n, nA, nB);
      if (nF < F + 1e-4 * step * gd) {
        A = nA;
        B = nB;
        F = nF;
        break;
      }
      step *= 0.5;
    }
    if (step < min_step) {
      status = 2;  // line search failed (LibSVM prints a warning and stops)
      break;
    }
  }
  if (it >= max_iter) status = 1;
  *A_out = A;
  *B_out = B;
  if (iters) *iters = it;
  return status;
}

// P(y=1|v) = 1/(1+exp(A v + B)) (Eq 12), evaluated stably.
inline double sigmoid_predict(double v, double A, double B) {
  double z = v * A + B;
  if (z >= 0) return std::exp(-z) / (1.0 + std::exp(-z));
  return 1.0 / (1.0 + std::exp(z));
}

// Solve M x = rhs (dimension m) by Gaussian elimination with partial pivoting. Returns 0 or -1.
int gauss_solve(std::vector<double>& M, std::vector<double>& rhs, int m) {
  for (int c = 0; c < m; ++c) {
    int piv = c;
    for (int r = c + 1; r < m; ++r)
      if (std::fabs(M[r * m + c]) > std::fabs(M[piv * m + c])) piv = r;
    if (M[piv * m + c] == 0.0) return -1;
    if (piv != c) {
      for (int j = 0; j < m; ++j) std::swap(M[c * m + j], M[piv * m + j]);
      std::swap(rhs[c], rhs[piv]);
    }
    for (int r = c + 1; r < m; ++r) {
      double fac = M[r * m + c] / M[c * m + c];
      if (fac == 0.0) continue;
      for (int j = c; j < m; ++j) M[r * m + j] -= fac * M[c * m + j];
      rhs[r] -= fac * rhs[c];
    }
  }
  for (int r = m - 1; r >= 0; --r) {
    double s = rhs[r];
    for (int j = r + 1; j < m; ++j) s -= M[r * m + j] * rhs[j];
    rhs[r] = s / M[r * m + r];
  }
  return 0;
}

// Pairwise coupling (Eq 14; closed form Eq 15): solve the bordered
// system [Q e; e^T 0][p; mu] = [0; 1] with Q_ss = sum_{u!=s} r_us^2, Q_st = -r_st r_ts.
// r is k x k row-major, r[s*k+t] = r_st (diagonal ignored).
int couple(const double* r, int k, double* p) {
  const int m = k + 1;
  for (int attempt = 0; attempt < 2; ++attempt) {
    std::vector<double> M((size_t)m * m, 0.0), rhs(m, 0.0);
    for (int s = 0; s < k; ++s) {
      double qss = 0.0;
      for (int u = 0; u < k; ++u)
        if (u != s) qss += r[u * k + s] * r[u * k + s];
      M[s * m + s] = qss + (attempt ? 1e-12 : 0.0);  // SURVEY §8(c) #14 fallback on zero pivot
      for (int t = 0; t < k; ++t)
        if (t != s) M[s * m + t] = -r[s * k + t] * r[t * k + s];
      M[s * m + k] = 1.0;
      M[k * m + s] = 1.0;
    }
    rhs[k] = 1.0;
    if (gauss_solve(M, rhs, m) == 0) {
      for (int s = 0; s < k; ++s) p[s] = rhs[s];
      return 0;
    }
  }
  return -1;
}

inline int pair_index(int s, int t, int k) { return s * k - s * (s + 1) / 2 + (t - s - 1); }

}  // namespace

extern "C" {

// ---------------------------------------------------------------------------------------
// Kernel values.  out[i*m + j] = K(X_i, Y_j), FP64.
void oracle_rbf_matrix(const float* X, int64_t n, const float* Y, int64_t m, int d, double gamma,
                       double* out, int nthreads) {
  parallel_for(n, nthreads, [&](int64_t i) {
    for (int64_t j = 0; j < m; ++j) out[i * m + j] = rbf(X + i * d, Y + j * d, d, gamma);
  });
}

// Binary SMO (Algorithm 1).  y in {+1,-1}.  Returns 0 converged, 1 iteration cap reached.
int oracle_smo(const float* X, const int32_t* y, int64_t n, int d, double C, double gamma, double eps,
               int64_t max_iter, double* alpha, double* f, int64_t* iters, double* dual_trace,
               int64_t trace_cap) {
  std::vector<const float*> rows(n);
  for (int64_t i = 0; i < n; ++i) rows[i] = X + i * d;
  return smo(rows.data(), y, n, d, C, gamma, eps, max_iter, alpha, f, iters, dual_trace, trace_cap,
             (size_t)1 << 30);
}

// f of Eq 3 recomputed exactly in FP64 for a given alpha (KKT audits of any solver's alpha).
void oracle_exact_f(const float* X, const int32_t* y, int64_t n, int d, double gamma, const double* alpha,
                    double* f, int nthreads) {
  std::vector<const float*> rows(n);
  for (int64_t i = 0; i < n; ++i) rows[i] = X + i * d;
  exact_f(rows.data(), y, n, d, gamma, alpha, f, nthreads);
}

// rho of the LibSVM rule (b = -rho); f must be exact for alpha.
double oracle_rho(const double* alpha, const double* f, const int32_t* y, int64_t n, double C) {
  return rho_of(alpha, f, y, n, C);
}

int oracle_sigmoid_fit(const double* v, const int32_t* y, int64_t n, double* A, double* B, int* iters) {
  return sigmoid_fit(v, y, n, A, B, iters);
}

int oracle_couple(const double* r, int k, double* p) { return couple(r, k, p); }

// Kernel of every following call (NEXT-4; type 0 = the paper's RBF, the default).
int oracle_set_kernel(int type, double coef0, int degree) {
  if (type < 0 || type > 3 || degree < 1) return -1;
  g_kernel.type = type;
  g_kernel.coef0 = coef0;
  g_kernel.degree = degree;
  return 0;
}

// ---------------------------------------------------------------------------------------
// Multi-class training (Algorithm 2; pairs L191-L195).
// labels in [0,k); pair p=(s,t), s<t, holds the instances of class s then class t, each in
// original index order; class s is +1.  Outputs (sized by the caller):
//   alpha_out [sum_p n_p]  pairs in order p, pair-local order
//   f_out     [sum_p n_p]  exact f (Eq 3) at the returned alpha (may be NULL)
//   b_out, A_out, B_out [P]; iters_out [P]; status_out [P] (0 ok, 1 cap)
// Pairs run concurrently (largest first) on nthreads threads.
int oracle_train(const float* X, const int32_t* labels, int64_t n, int d, int k, double C, double gamma,
                 double eps, int nthreads, double* alpha_out, double* f_out, double* b_out, double* A_out,
                 double* B_out, int64_t* iters_out, int32_t* status_out) {
  const int P = k * (k - 1) / 2;
  std::vector<std::vector<int64_t>> members(k);
  for (int64_t i = 0; i < n; ++i) {
    if (labels[i] < 0 || labels[i] >= k) return -1;
    members[labels[i]].push_back(i);
  }
  for (int c = 0; c < k; ++c)
    if (members[c].empty()) return -1;
  std::vector<int> ps(P), pt(P);
  std::vector<int64_t> off(P + 1, 0);
  for (int s = 0; s < k; ++s)
    for (int t = s + 1; t < k; ++t) {
      int p = pair_index(s, t, k);
      ps[p] = s;
      pt[p] = t;
    }
  for (int p = 0; p < P; ++p) off[p + 1] = off[p] + (int64_t)(members[ps[p]].size() + members[pt[p]].size());
  std::vector<int> order(P);
  for (int p = 0; p < P; ++p) order[p] = p;
  std::stable_sort(order.begin(), order.end(),
                   [&](int a, int b) { return off[a + 1] - off[a] > off[b + 1] - off[b]; });
  int inner_threads = std::max(1, nthreads / std::max(1, P));
  int outer_threads = std::max(1, std::min(nthreads, P));
  size_t cache_bytes = std::max<size_t>((size_t)64 << 20, ((size_t)8 << 30) / (size_t)outer_threads);
  parallel_for(P, outer_threads, [&](int64_t oi) {
    int p = order[oi];
    const auto& ms = members[ps[p]];
    const auto& mt = members[pt[p]];
    int64_t np = (int64_t)(ms.size() + mt.size());
    std::vector<const float*> rows(np);
    std::vector<int> y(np);
    for (size_t i = 0; i < ms.size(); ++i) {
      rows[i] = X + ms[i] * d;
      y[i] = +1;
    }
    for (size_t i = 0; i < mt.size(); ++i) {
      rows[ms.size() + i] = X + mt[i] * d;
      y[ms.size() + i] = -1;
    }
    double* alpha = alpha_out + off[p];
    std::vector<double> f(np);
    int64_t it = 0;
    int st = smo(rows.data(), y.data(), np, d, C, gamma, eps, 0, alpha, f.data(), &it, nullptr, 0, cache_bytes);
    exact_f(rows.data(), y.data(), np, d, gamma, alpha, f.data(), inner_threads);
    double rho = rho_of(alpha, f.data(), y.data(), np, C);
    b_out[p] = -rho;
    // In-sample decision values v_i = f_i + y_i - rho (Eq 3 + Eq 11), then Eq 13 fit.
    std::vector<double> v(np);
    for (int64_t i = 0; i < np; ++i) v[i] = f[i] + y[i] - rho;
    sigmoid_fit(v.data(), y.data(), np, &A_out[p], &B_out[p], nullptr);
    if (f_out) std::memcpy(f_out + off[p], f.data(), sizeof(double) * np);
    if (iters_out) iters_out[p] = it;
    if (status_out) status_out[p] = st;
  });
  return 0;
}

// Multi-class probability estimation (L259-L273, Eq 11, 12, 14, 15).
// Model = the outputs of oracle_train on (X, labels).  dec_out [m*P], r not returned,
// prob_out [m*k] (either may be NULL).  min_prob clamp 1e-7.
int oracle_predict(const float* X, const int32_t* labels, int64_t n, int d, int k, double gamma,
                   const double* alpha, const double* b, const double* A, const double* B, const float* Xt,
                   int64_t m, double* dec_out, double* prob_out, int nthreads) {
  const int P = k * (k - 1) / 2;
  std::vector<std::vector<int64_t>> members(k);
  for (int64_t i = 0; i < n; ++i) members[labels[i]].push_back(i);
  std::vector<int64_t> off(P + 1, 0);
  std::vector<int> ps(P), pt(P);
  for (int s = 0; s < k; ++s)
    for (int t = s + 1; t < k; ++t) {
      int p = pair_index(s, t, k);
      ps[p] = s;
      pt[p] = t;
    }
  for (int p = 0; p < P; ++p) off[p + 1] = off[p] + (int64_t)(members[ps[p]].size() + members[pt[p]].size());
  // Instances with a nonzero alpha in some pair (only those contribute to Eq 11).
  std::vector<char> is_sv(n, 0);
  for (int p = 0; p < P; ++p) {
    const auto& ms = members[ps[p]];
    const auto& mt = members[pt[p]];
    for (size_t i = 0; i < ms.size(); ++i)
      if (alpha[off[p] + i] != 0.0) is_sv[ms[i]] = 1;
    for (size_t i = 0; i < mt.size(); ++i)
      if (alpha[off[p] + ms.size() + i] != 0.0) is_sv[mt[i]] = 1;
  }
  int status = 0;
  std::atomic<int> bad(0);
  parallel_for(m, nthreads, [&](int64_t q) {
    const float* x = Xt + q * d;
    std::vector<double> kx(n, 0.0);
    for (int64_t j = 0; j < n; ++j)
      if (is_sv[j]) kx[j] = rbf(X + j * d, x, d, gamma);
    std::vector<double> r((size_t)k * k, 0.0);
    for (int p = 0; p < P; ++p) {
      const auto& ms = members[ps[p]];
      const auto& mt = members[pt[p]];
      double dec = 0.0;  // Eq 11: v = sum_j y_j alpha_j K(x_j, x) + b
      for (size_t i = 0; i < ms.size(); ++i) {
        double a = alpha[off[p] + i];
        if (a != 0.0) dec += a * kx[ms[i]];
      }
      for (size_t i = 0; i < mt.size(); ++i) {
        double a = alpha[off[p] + ms.size() + i];
        if (a != 0.0) dec -= a * kx[mt[i]];
      }
      dec += b[p];
      if (dec_out) dec_out[q * P + p] = dec;
      double rst = sigmoid_predict(dec, A[p], B[p]);
      rst = std::min(std::max(rst, 1e-7), 1.0 - 1e-7);
      r[ps[p] * k + pt[p]] = rst;
      r[pt[p] * k + ps[p]] = 1.0 - rst;
    }
    if (prob_out) {
      if (couple(r.data(), k, prob_out + q * k) != 0) bad.store(1);
    }
  });
  if (bad.load()) status = -1;
  return status;
}

}  // extern "C"
