// model.h -- the library-owned model object (opaque gmpsvm_model in the ABI).
#pragma once

#include <memory>
#include <mutex>
#include <vector>

#include "kernels.h"

namespace gmpsvm {

// Device-resident prediction structures (support-vector sharing):
// the SV union in class-pure 128-column tiles, stored feature-major (SvT[c][slot]),
// its norms, the LibSVM-style coefficient matrix coef[slot][k-1] (= y * alpha of the SV in
// each of the k-1 pairs of its class), and the per-class runs of tiles ("items").
struct DevModel {
  int device = -1;
  int d_pad = 0, km1 = 0, km1_pad = 0, n_items = 0;
  int64_t nsv_pad = 0;
  float* SvT = nullptr;     // [d_pad][nsv_pad]
  float* nsv = nullptr;     // [nsv_pad]
  float* coef = nullptr;    // [nsv_pad][km1_pad]
  DecItem* items = nullptr; // [n_items]
  int32_t* item_begin = nullptr;  // [k]
  int32_t* item_end = nullptr;    // [k]
  double* b = nullptr;      // [P]
  double* A = nullptr;      // [P]
  double* B = nullptr;      // [P]
  // tensor-core decision values (dec_tc): SV rows centred by mu, TF32 hi/lo split, row-major
  // [nsv_pad][dpt], their centred squared norms; test rows are split with the same mu
  bool tc = false;
  int dpt = 0;
  float* SvHi = nullptr;
  float* SvLo = nullptr;
  float* nsvc = nullptr;    // [nsv_pad]
  float* mu = nullptr;      // [d]
  float sc = 1.f;           // split scale (exact power of two; 1 for TF32)
  std::vector<DecItem> h_items;  // host copy of the items (work-unit lists of dec_tc)
  std::vector<int64_t> slot_sv;  // slot -> index into the model's SV list, -1 = padding
  // training output kept on the device: alpha of every trained pair in the solver's pair order;
  // alpha_dev_off[p] = offset of model pair p (-1: untrained).  The host copy Model::alpha is
  // materialised from it only when asked for (introspection, serialisation, merge).
  double* alpha_dev = nullptr;
  // Decision-value path (DESIGN.md §3 "decision-value routing"): the fastest path whose
  // worst-case probability error 2 * max_p |A_p|/4 * sum_j |alpha_pj| * E_K (E_K: that path's
  // bound on |K~ - K|; 2: the coupling's measured amplification) is <= kDecProbBound.
  //   kDecI8  dec_i8.cu: exact int8-digit dot products on tcgen05, FP64 kernel values (RBF)
  //   kDecF64 predict.cu: FP64 SIMT (any kernel; the fallback)
  //   kDecF16 krow_tc.cu dec_tc: FP16 hi/lo split, FP32 kernel values (forced: GMPSVM_DEC=f16)
  int path = 0;
  bool f64 = false;             // path == kDecF64
  double wsum = 0.0;            // max_p |A_p| * sum_j |alpha_pj|
  std::vector<double> abs_sum;  // [P] sum_j |alpha_pj|
  double cond_i8 = 0.0, cond_f16 = 0.0;
  double* coef64 = nullptr;  // [nsv_pad][km1_pad]
  double* nsv64 = nullptr;   // [nsv_pad] FP64 squared norms of the SV rows
  // int8-digit SV planes [5][nsv_pad][round_up(d, 32)], per-row exponents and FP64 norms of the
  // fixed-point rows, max |x| over the SV rows
  int8_t* SvI8 = nullptr;
  int32_t* sv_e = nullptr;
  double* sv_n64 = nullptr;
  float amax_sv = 0.f;
  std::vector<int64_t> alpha_dev_off;
  cudaEvent_t last_use = nullptr;  // recorded on the caller's stream after every use
  // stream-ordered allocation: freed on the library stream after last_use (no device sync)
  ~DevModel();
};

struct Model {
  int32_t k = 0, d = 0;
  double C = 0, gamma = 0, eps = 0;
  int32_t kernel = 0;  // GMPSVM_KERNEL_* (0 = RBF)
  double coef0 = 0;
  int32_t degree = 3;
  int64_t n = 0;
  std::vector<int64_t> class_count;  // [k]
  std::vector<int64_t> perm;         // class-sorted position -> original index [n]
  std::vector<uint8_t> trained;      // [P]
  std::vector<double> b, A, B;       // [P]
  std::vector<int32_t> status;       // [P] solver status (0 ok, 2 outer cap) | sigmoid status << 8
  // [P] telemetry of the training run (0 for models built from alpha / deserialised): outer
  // iterations, inner SMO steps, kernel rows computed (ROW_CACHE regime; 0 in FULL_K)
  std::vector<int64_t> pair_outer, pair_inner, pair_rows;
  std::vector<double> alpha;         // [sum_p n_p] pair-local order, all pairs (0 for untrained)
  bool alpha_ready = true;           // false: alpha still only on the device (ensure_host_alpha)
  std::vector<int64_t> sv_pos;       // class-sorted positions of the SV union, ascending
  std::vector<float> sv_X;           // [n_sv][d] host copy (materialised lazily from the device)
  bool sv_X_ready = false;
  gmpsvm_train_stats stats{};
  mutable std::mutex mu;
  // shared: a prediction holds its own reference for the whole call, so a concurrent call that
  // moves the model to another device (ensure_dev_model) cannot free structures still in use
  mutable std::shared_ptr<DevModel> dev;

  int P() const { return k * (k - 1) / 2; }
  std::vector<int64_t> class_off() const;
  std::vector<int64_t> pair_offsets() const;  // [P+1] offsets of each pair into alpha
  int n_trained() const;
};

// engine.cu
int engine_train(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C, double gamma, double eps,
                 const gmpsvm_options& opt, Model** out);
int engine_model_from_alpha(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C, double gamma,
                            const double* alpha, const double* b, const double* A, const double* B,
                            const int32_t* status, const gmpsvm_options& opt, Model** out);
int engine_train_csr(const int64_t* indptr, const int32_t* indices, const float* values, const int32_t* y, int64_t n,
                     int32_t d, int32_t k, double C, double gamma, double eps, const gmpsvm_options& opt, Model** out);
int engine_predict_csr(const Model& mdl, const int64_t* indptr, const int32_t* indices, const float* values, int64_t m,
                       double* prob_out, const gmpsvm_options& opt);
int engine_predict(const Model& mdl, const float* Xt, int64_t m, double* prob_out, double* dec_out,
                   const gmpsvm_options& opt);
int engine_rbf_kernel(const float* X, int64_t n, const float* Y, int64_t m, int32_t d, double gamma, float* K_out,
                      const gmpsvm_options& opt);
int engine_couple(const double* dec, int64_t m, int32_t k, const double* A, const double* B, double* prob_out,
                  const gmpsvm_options& opt);
void ensure_host_sv(const Model& mdl);     // materialise sv_X on the host
void ensure_host_alpha(const Model& mdl);  // materialise alpha on the host
gmpsvm_predict_stats& tls_predict_stats();

// shard.cu (NEXT-1)
struct Shard;
Shard* shard_create(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, int32_t s, int32_t t, double C,
                    double gamma, double eps, int32_t rank, int32_t world, const gmpsvm_options& opt);
void shard_free(Shard* S);
int shard_cand_doubles(const Shard* S);
void shard_slice(const Shard* S, int64_t* lo, int64_t* hi, int64_t* np, int32_t* ws_size);
void shard_candidates(Shard* S, double* out);
int shard_select(Shard* S, const double* all, int32_t* stop, double* fws_out);
void shard_fws(Shard* S, double* out);
void shard_step(Shard* S, const double* fws_sum, double* cand_out);
void shard_f(Shard* S, double* out);
int shard_finish(Shard* S, const double* f_full, double* alpha_out, double* b, double* A, double* Bsig, int32_t* status,
                 int64_t* outer, int64_t* inner);
double shard_merge(const double* all, int world, int cand_doubles, int need, int need_u, std::vector<int32_t>& picks);

}  // namespace gmpsvm

struct gmpsvm_model {
  std::unique_ptr<gmpsvm::Model> m;
};
