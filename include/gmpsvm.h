/* gmpsvm.h -- C ABI of libgmpsvm.so, the B200 (sm_100a) hot path of GMP-SVM.
 *
 * Paper: Wen, Shi, He, Chen, Chen, "Efficient Multi-Class Probabilistic SVMs on GPUs",
 * ICDE 2019 (PAPER.md = /root/reference/PAPER.md; citations are PAPER.md line numbers).
 *
 * Problem statement (L191-L208): train the k(k-1)/2 one-vs-one binary SVMs of a k-class
 * problem (dual QP Eq 2, RBF kernel L75), fit one Platt sigmoid per pair
 * (Eq 12-13), and turn the pairwise probabilities of a test instance into
 * k-class probabilities by pairwise coupling (Eq 14-15).
 *
 * Conventions (all entry points):
 *   - X, Xtest: FP32, row-major, n x d (resp. m x d).  Labels y: int32 in [0, k); every
 *     class must be non-empty.  Classes are ordered by label value.
 *   - Pair p = (s, t), s < t, has index p = s*k - s(s+1)/2 + (t - s - 1).  Class s is the
 *     +1 side (L195), r_st = P(class s | pair p); its instances are those of class s then
 *     those of class t, each in original index order ("pair-local order").
 *   - Pointers are HOST pointers unless gmpsvm_options.inputs_on_device = 1, in which case
 *     X / y / Xtest / out are DEVICE pointers on gmpsvm_options.device (e.g. torch CUDA
 *     tensors).  Inputs are borrowed read-only and never retained after return.
 *   - Errors: return codes only; nothing aborts and no C++ exception crosses the ABI.
 *     Negative = error (message in gmpsvm_last_error()), 0 = OK, positive = warning with a
 *     valid result (GMPSVM_WARN_MAXITER, as LibSVM does on its iteration cap).
 *   - Models are library-owned, immutable after train, and safe to use for concurrent
 *     predictions; free with gmpsvm_model_free().
 *   - Precision: X and kernel values FP32; solver state (alpha, f), b, A, B, decision
 *     values and probabilities FP64.
 */
#ifndef GMPSVM_H_
#define GMPSVM_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GMPSVM_ABI_VERSION 1

#if defined(__GNUC__)
#define GMPSVM_API __attribute__((visibility("default")))
#else
#define GMPSVM_API
#endif

typedef struct gmpsvm_model gmpsvm_model; /* opaque; owned by the library */

enum {
  GMPSVM_OK = 0,
  GMPSVM_WARN_MAXITER = 1, /* an iteration cap was reached; the model is valid          */
  GMPSVM_EINVAL = -1,      /* bad argument (sizes, labels, non-finite values, options)   */
  GMPSVM_ENOMEM = -2,      /* device or host allocation failed                           */
  GMPSVM_ECUDA = -3,       /* CUDA runtime / kernel error (message kept)                 */
  GMPSVM_ENOTIMPL = -4,    /* configuration not supported by this build                  */
  GMPSVM_EFORMAT = -5      /* malformed or incompatible serialized model                 */
};

/* Options; zero-initialised (or gmpsvm_options_init) = defaults. */
typedef struct {
  int32_t struct_size;      /* sizeof(gmpsvm_options); 0 is accepted as "current"           */
  int32_t ws_size;          /* B: working-set = kernel-buffer rows per pair (L299-L303, L377);
                               default 192 (K_ws,ws then lives in shared memory; the paper's
                               1024 is a tuning point); must be even, 2..1024     */
  int32_t q;                /* new violators per outer iteration (L289, L297); default B/2;
                               the newest B-q rows of the previous working set are kept     */
  int32_t device;           /* CUDA device ordinal                                           */
  int64_t cache_bytes;      /* kernel-value cache budget in bytes; 0 = 85% of device memory.
                               n*round_up(n,4)*4 <= budget: FULL_K (whole matrix resident);
                               else ROW_CACHE: per pair a B x round_up(n_p,4) row buffer, the
                               rows of each outer iteration's new working-set entries computed
                               on demand (L297-L303); GMPSVM_ENOTIMPL if even the
                               row buffers exceed 85% of device memory                       */
  void* stream;             /* cudaStream_t to run on (NULL = a library-owned stream)       */
  const int32_t* pair_ids;  /* train only these pair indices (multi-GPU sharding); NULL = all */
  int32_t n_pair_ids;       /* >= 1 when pair_ids != NULL (else GMPSVM_EINVAL)               */
  int32_t inputs_on_device; /* 1: X/y/Xtest/out are device pointers on `device`             */
  int64_t max_outer_iter;   /* cap on outer (working-set) iterations per pair; 0 = 1,000,000 */
  int32_t inner_iter_cap;   /* cap on inner SMO steps per working set; 0 = B / 2 for the RBF */
                            /* kernel on the shared-memory solver (B <= 224), else 100 * B  */
  int32_t kernel;           /* GMPSVM_KERNEL_*: the paper's RBF (L75, default) or one of the
                               other kernels it lists (L76-L78; LibSVM definitions, gamma the
                               train call's): training needs the FULL_K regime on the tensor
                               cores (else GMPSVM_ENOTIMPL); prediction runs in FP64         */
  double coef0;             /* polynomial / sigmoid offset (LibSVM coef0); default 0         */
  int32_t degree;           /* polynomial degree; 0 = 3                                      */
  int32_t prob_folds;       /* 0: sigmoids fitted on the pairs' in-sample decision values (the
                               paper, L193-L195; reading R10).  F >= 2: LibSVM's practice
                               (NEXT-2): F-fold cross-validated decision values -- F extra
                               trainings on the other folds (fold of an instance = its rank
                               within its class mod F), the sigmoid of each pair fitted on the
                               out-of-fold values; every class needs >= F instances         */
  int32_t reserved[2];
} gmpsvm_options;

enum { GMPSVM_KERNEL_RBF = 0,      /* exp(-gamma |x - y|^2)                 */
       GMPSVM_KERNEL_LINEAR = 1,   /* x . y                                 */
       GMPSVM_KERNEL_POLY = 2,     /* (gamma x . y + coef0)^degree          */
       GMPSVM_KERNEL_SIGMOID = 3   /* tanh(gamma x . y + coef0)             */ };

/* Per-phase CUDA-event times of the last training run (mirrors the paper's Fig 11
 * breakdown, L483-L497) and counters. */
typedef struct {
  double t_total_ms;        /* whole gmpsvm_train_ex call (host clock)                       */
  double t_stage_ms;        /* a1: H2D (if host input), class sort, transpose, norms         */
  double t_kernel_ms;       /* a2: kernel-value contraction (krow_contract launches)         */
  double t_select_ms;       /* a4: working-set selection + stop test                         */
  double t_subproblem_ms;   /* a5: K_ws,ws gather + local SMO                                 */
  double t_fupdate_ms;      /* a6: f update                                                   */
  double t_finalize_ms;     /* a7-a9: bias, decision values, sigmoid fit, model assembly    */
  double kernel_flops;      /* flops executed by krow_contract (2d+3 per computed value)     */
  double kernel_values;     /* kernel values computed (FULL_K: distinct, symmetric half +
                               diagonal; ROW_CACHE: rows computed x n_p, summed over pairs)   */
  int64_t krow_launches;    /* launches of the kernel-value contraction (FULL_K: 1;
                               ROW_CACHE: one per issued outer iteration per pair group)      */
  int64_t outer_iters_max;  /* max over pairs of outer iterations                             */
  int64_t outer_iters_sum;  /* sum over pairs                                                 */
  int64_t inner_iters_sum;  /* sum over pairs and working sets of inner SMO steps            */
  int64_t n_sv;             /* |SV union| over the trained pairs                              */
  int32_t cache_regime;     /* 0 = FULL_K (whole kernel matrix resident), 1 = ROW_CACHE       */
  int32_t n_pairs_trained;
  int64_t launches;         /* kernels launched by this call                                  */
  int64_t smo_cycles_sum;   /* SM clock cycles spent in the local SMO, summed over pairs      */
  double t_solver_ms;       /* a3-a6 as a whole: pairs run on concurrent streams, so select,  */
                            /* subproblem and f-update overlap (their own fields then stay 0)  */
  int32_t n_streams;        /* concurrent branches of the solver graph (pairs packed into them) */
  int32_t kernel_path;      /* kernel values from: 0 dense rows on tcgen05, 1 dense rows on the FP32
                               SIMT contraction, 2 CSR rows (sparse x dense, NEXT-3, L299 / L513) */
} gmpsvm_train_stats;

typedef struct {
  double t_total_ms;        /* whole call (host clock)                                        */
  double t_stage_ms;        /* H2D of Xtest (if host), transpose, norms                       */
  double t_decision_ms;     /* a10: decision-value contraction + reduction                    */
  double t_couple_ms;       /* a11-a12: sigmoid + coupling                                    */
  double t_d2h_ms;          /* D2H of the probabilities (host output)                         */
  double dec_flops;         /* (2d + 3 + 2(k-1)) per (test, SV) pair                           */
  int64_t dec_launches;     /* decision-value contractions (one per <= 32768-row chunk)       */
  int64_t launches;         /* kernels launched by this call                                  */
  int32_t dec_path;         /* decision-value path taken (DESIGN.md §3 routing): 0 FP64 SIMT,
                               1 int8-digit tensor cores (exact dot products, FP64 K),
                               2 FP16-split tensor cores (FP32 K; GMPSVM_DEC=f16 only)        */
  int32_t pad0;
} gmpsvm_predict_stats;

GMPSVM_API void gmpsvm_options_init(gmpsvm_options* opt);

/* Training (Algorithm 2).  X [n x d] FP32, y [n] int32 in [0,k); C > 0,
 * gamma > 0, eps > 0 (stop when max_{I_l} f - min_{I_u} f < eps, Eq 9 with tolerance:
 * DESIGN.md reading R1).  On success *out receives a new model. */
GMPSVM_API int gmpsvm_train(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C,
                 double gamma, double eps, gmpsvm_model** out);
GMPSVM_API int gmpsvm_train_ex(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C,
                    double gamma, double eps, const gmpsvm_options* opt, gmpsvm_model** out);

/* Probability estimation (L259-L273, L331-L363): out [m x k] FP64 row-major, caller-
 * allocated; each row sums to 1.  Requires a model with every pair trained. */
/* CSR input (NEXT-3; the sparse format of the paper's datasets, L385): row i's nonzeros are
 * values[indptr[i] .. indptr[i+1]) at columns indices[.] (each in [0, d), else EINVAL).  The rows
 * are densified on the device and take the dense path (the kernel-value contraction runs on the
 * dense rows).  indptr: n+1 int64; indices: nnz int32; values: nnz float; host or device pointers
 * per opt->inputs_on_device.  y, model, out, errors as gmpsvm_train_ex / gmpsvm_predict_proba. */
GMPSVM_API int gmpsvm_train_csr(const int64_t* indptr, const int32_t* indices, const float* values, const int32_t* y,
                                int64_t n, int32_t d, int32_t k, double C, double gamma, double eps,
                                const gmpsvm_options* opt, gmpsvm_model** out);
GMPSVM_API int gmpsvm_predict_proba_csr(const gmpsvm_model* model, const int64_t* indptr, const int32_t* indices,
                                        const float* values, int64_t m, double* out, const gmpsvm_options* opt);
GMPSVM_API int gmpsvm_predict_proba(const gmpsvm_model* model, const float* Xtest, int64_t m, double* out);
GMPSVM_API int gmpsvm_predict_proba_ex(const gmpsvm_model* model, const float* Xtest, int64_t m, double* out,
                            const gmpsvm_options* opt);

/* Decision values only (Eq 11): dec_out [m x P] FP64 row-major (includes b). */
GMPSVM_API int gmpsvm_predict_decision(const gmpsvm_model* model, const float* Xtest, int64_t m, double* dec_out,
                            const gmpsvm_options* opt);

GMPSVM_API void gmpsvm_model_free(gmpsvm_model* model);
GMPSVM_API const char* gmpsvm_last_error(void); /* thread-local message of the last non-OK return */

/* ---- introspection (parity tests) ---- */
GMPSVM_API int gmpsvm_model_dims(const gmpsvm_model* model, int32_t* k, int32_t* d, int64_t* n_sv,
                      int32_t* n_pairs_trained);
/* Pair (s,t), s<t: b (= -rho), Platt A, B, and alpha [n_s + n_t] in pair-local order
 * (alpha_out may be NULL).  EINVAL if the pair was not trained by this model. */
GMPSVM_API int gmpsvm_model_pair(const gmpsvm_model* model, int32_t s, int32_t t, double* b, double* A, double* B,
                      double* alpha_out);
/* Original training indices of the SV union, ascending in (class, original index). */
/* Telemetry of pair (s, t) from its training run (SURVEY §8(d) "report outer/inner iterations
 * and rows computed"): outer iterations (Alg 2 l.5-12), inner SMO steps, kernel rows computed
 * (ROW_CACHE regime; 0 in FULL_K, where every row is computed once for all pairs).  0 for models
 * rebuilt from alpha or deserialised.  Any pointer may be NULL. */
GMPSVM_API int gmpsvm_model_pair_iters(const gmpsvm_model* model, int32_t s, int32_t t, int64_t* outer, int64_t* inner,
                                       int64_t* rows);
GMPSVM_API int gmpsvm_model_sv_index(const gmpsvm_model* model, int64_t* idx_out);
GMPSVM_API int gmpsvm_model_train_stats(const gmpsvm_model* model, gmpsvm_train_stats* stats);
GMPSVM_API void gmpsvm_last_predict_stats(gmpsvm_predict_stats* stats); /* thread-local, last predict call */

/* ---- multi-GPU plumbing (pairs sharded across ranks, models gathered with NCCL) ---- */
/* Flat little-endian blob.  *len: in = capacity of buf (buf may be NULL to query),
 * out = bytes needed.  Returns EINVAL if the capacity is too small. */
GMPSVM_API int gmpsvm_model_serialize(const gmpsvm_model* model, void* buf, size_t* len);
GMPSVM_API int gmpsvm_model_deserialize(const void* buf, size_t len, gmpsvm_model** out);
/* Union of partial models trained on disjoint pair subsets of the same (X, y, C, gamma). */
GMPSVM_API int gmpsvm_model_merge(const gmpsvm_model* const* parts, int32_t n_parts, gmpsvm_model** out);
/* The complete model from every pair's solution computed elsewhere -- the multi-GPU path's
 * gather: each rank trains a pair subset (pair_ids), the ranks all-reduce the disjoint per-pair
 * alpha / b / A / B (O(sum n_p) doubles over NCCL) and every rank rebuilds the model from its
 * own replicated X (SV union, coefficients, Alg 2 l.16, L331-L333, L363).  X, y: as in
 * gmpsvm_train_ex (device pointers if opt->inputs_on_device); alpha: sum_p n_p doubles, pairs
 * in index order, each in pair-local order (the layout of gmpsvm_model_pair's alpha_out), every
 * value in [0, C] (else EINVAL); b, A, B: P doubles; status: P int32 or NULL -- host pointers. */
GMPSVM_API int gmpsvm_model_from_alpha(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C,
                                       double gamma, const double* alpha, const double* b, const double* A,
                                       const double* B, const int32_t* status, const gmpsvm_options* opt,
                                       gmpsvm_model** out);

/* ---- NEXT-1: one pair's binary SVM trained by several ranks, its instances sharded ----------
 * (the paper's instance-level parallelism; kernel rows
 * as a product of the working-set rows with the rest, L299; Algorithm 2 lines 5-13.)  Each rank
 * holds X (replicated) and owns the slice [lo, hi) of the pair's instances (pair-local order:
 * class s, then class t).  Per outer iteration the caller runs, on every rank, with its own
 * collectives (torch.distributed; paper_conf_icde_wenshcc19_b200/dist.py train_pair_sharded):
 *   gmpsvm_shard_candidates(sh, c)          once before the loop; c: this rank's block of
 *                                           gmpsvm_shard_cand_doubles
 *   all_gather(c) -> all [world x cand_doubles], rank order
 *   gmpsvm_shard_select(sh, all, &stop, fws)  identical merge on every rank; stop = 1: converged
 *                                           (Eq 9 with tolerance eps) or the outer cap; fws (B
 *                                           doubles, may be NULL): f of the members this rank owns
 *   all_reduce_sum(fws)
 *   gmpsvm_shard_step(sh, fws, c)           local SMO (same on every rank) + f update of the slice;
 *                                           c (may be NULL): the next iteration's candidates
 * (one device round trip per collective; gmpsvm_shard_fws gives fws separately.)
 * then gathers every rank's f slice (gmpsvm_shard_f, rank order) and calls gmpsvm_shard_finish
 * for alpha (n_p, pair-local order), b, A, B and the status word of gmpsvm_model_pair.  All
 * buffers are host pointers.  world = 1 is a complete single-rank solver; any world gives
 * bitwise the same alpha.  RBF kernel only (else ENOTIMPL); opt: ws_size, q, device, stream,
 * max_outer_iter, inputs_on_device (X, y device pointers). */
typedef struct gmpsvm_shard gmpsvm_shard;
GMPSVM_API int gmpsvm_shard_create(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, int32_t s,
                                   int32_t t, double C, double gamma, double eps, int32_t rank, int32_t world,
                                   const gmpsvm_options* opt, gmpsvm_shard** out);
GMPSVM_API int32_t gmpsvm_shard_cand_doubles(const gmpsvm_shard* sh);
GMPSVM_API int gmpsvm_shard_slice(const gmpsvm_shard* sh, int64_t* lo, int64_t* hi, int64_t* n_p, int32_t* ws_size);
GMPSVM_API int gmpsvm_shard_candidates(gmpsvm_shard* sh, double* out);
GMPSVM_API int gmpsvm_shard_select(gmpsvm_shard* sh, const double* all, int32_t* stop, double* fws_out);
GMPSVM_API int gmpsvm_shard_fws(gmpsvm_shard* sh, double* fws);
GMPSVM_API int gmpsvm_shard_step(gmpsvm_shard* sh, const double* fws_sum, double* cand_out);
GMPSVM_API int gmpsvm_shard_f(gmpsvm_shard* sh, double* f_slice);
GMPSVM_API int gmpsvm_shard_finish(gmpsvm_shard* sh, const double* f_full, double* alpha, double* b, double* A,
                                   double* B, int32_t* status, int64_t* outer_iters, int64_t* inner_iters);
GMPSVM_API void gmpsvm_shard_free(gmpsvm_shard* sh);
/* The candidate merge alone (host arithmetic, no GPU): all = world blocks of cand_doubles
 * [fmin, fmax, nU, nL, U keys (order-preserving bits of f, as doubles) x m, U indices x m, L keys
 * (~bits) x m, L indices x m], m = (cand_doubles - 4) / 4; need picks, need_u of them from I_u
 * first (R19).  picks_out: need int32 (selection order), *n_picks; *gap = max_{I_l} f - min_{I_u} f
 * (-DBL_MAX if a side is empty). */
GMPSVM_API int gmpsvm_shard_merge(const double* all, int32_t world, int32_t cand_doubles, int32_t need, int32_t need_u,
                                  int32_t* picks_out, int32_t* n_picks, double* gap);

/* ---- component entry points (steps of the path, exposed for parity tests and bench) ---- */
/* a2 alone (K1, L287-L299, RBF L75): K_out[i*m + j] = exp(-gamma ||X_i - Y_j||^2) in FP32 via
 * the norm expansion ||x||^2 + ||y||^2 - 2 x.y (distance clamped at 0).  K_out [n x m].
 * If X == Y (same pointer) and n == m, the symmetric FULL_K launch used by training runs
 * (upper-triangular tiles mirrored, K_ii = 1). */
GMPSVM_API int gmpsvm_rbf_kernel(const float* X, int64_t n, const float* Y, int64_t m, int32_t d, double gamma,
                      float* K_out, const gmpsvm_options* opt);
/* a11 + a12 alone (Eq 12, 14, 15): dec [m x P] FP64, A/B [P] -> prob [m x k] FP64. */
GMPSVM_API int gmpsvm_couple(const double* dec, int64_t m, int32_t k, const double* A, const double* B,
                  double* prob_out, const gmpsvm_options* opt);

/* Kernels launched by this library in this process (monotone counter). */
GMPSVM_API uint64_t gmpsvm_launch_count(void);
GMPSVM_API int32_t gmpsvm_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* GMPSVM_H_ */
