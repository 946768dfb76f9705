// kernels.h -- launchers of the sm_100a kernels (internal to libgmpsvm).
#pragma once

#include <vector>

#include "common.cuh"

namespace gmpsvm {

// CUDA_DEVICE_MAX_CONNECTIONS actually in effect for this process (api.cpp, at library load)
int connections_in_effect();
// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) for the CURRENT device (the attribute is
// per device context): set once per (kernel, device) and raised when a launch needs more
void set_max_dyn_smem(const void* func, size_t bytes);
template <typename F>
inline void set_max_dyn_smem(F* func, size_t bytes) {
  set_max_dyn_smem(reinterpret_cast<const void*>(func), bytes);
}


// ---------------- a1 staging (stage.cu)
void launch_class_sort(const int32_t* y, int64_t n, int k, int32_t* blk_counts, int32_t* blk_off,
                       int64_t* class_count, int64_t* class_off, cudaStream_t st);
void launch_class_rank(const int32_t* y, int64_t n, int k, const int32_t* blk_off, const int64_t* class_off,
                       int64_t* perm, cudaStream_t st);
// XT[c][j] = X[src(j)][c] (src = perm[j], or j if perm == NULL; src < 0 = zero padding slot),
// norms[j] = ||X[src(j)]||^2; *bad (may be NULL) set to 1 if a row is non-finite.
void launch_stage_features(const float* X, int64_t n, int d, const int64_t* perm, float* XT, int64_t ldx, int d_pad,
                           int64_t n_pad, float* norms, int32_t* bad, cudaStream_t st);
void launch_gather_rows(const float* X, int d, const int64_t* idx, int64_t nr, float* dst, cudaStream_t st);

// ---------------- a2 kernel values (krow.cu)
void launch_krow_full_sym(const float* XT, int64_t ldx, const float* norms, int64_t n, int kdim, double gamma,
                          float* K, int64_t ldk, cudaStream_t st);
void launch_krow_rect(const float* AT, int64_t lda, const float* na, int64_t n, const float* BT, int64_t ldb,
                      const float* nb, int64_t m, int kdim, double gamma, float* K, int64_t ldk, cudaStream_t st);

// ---------------- a2 on tcgen05 (krow_tc.cu): 2-part split (FP16 default, TF32 with
// GMPSVM_SPLIT=tf32), TMEM split accumulators, TMA staging.  hi / lo buffers are row-major
// n_pad x d_pad elements of the split type (krow_tc_buf_floats floats of storage).
int64_t krow_tc_rows_pad(int64_t n);  // row padding the tile grid needs (multiple of 128)
bool krow_split_f16();
int krow_tc_d_pad(int d);             // feature padding in elements (one 128-byte atom: 64 FP16 / 32 TF32)
size_t krow_tc_buf_floats(int64_t n_pad, int d_pad);
float krow_split_scale(float maxabs);  // exact power-of-two scale of the FP16 split (1 for TF32)
// centre by the column means (mean of the original rows; perm only reorders), scale, split into
// hi/lo rows and compute the squared norms (scaled units); returns the scale
size_t krow_tc_scratch_bytes(int64_t n, int d);
const float* krow_tc_scratch_mu(const void* scratch, int64_t n, int d);
float launch_split_hilo(const float* X, int64_t n, int d, const int64_t* perm, void* hi, void* lo, float* norms,
                        int64_t n_pad, int d_pad, void* scratch, cudaStream_t st, bool center = true);
// the paper's other kernels (L76-L78): type 1 linear, 2 polynomial, 3 sigmoid (inv_s2 set by the launch)
struct KrowKernel {
  int type;
  float gamma, coef0, inv_s2;
  int degree;
  unsigned long long* resident;  // optional: each CTA adds 1 when it starts (persistent solver's lead group)
};
// max over the rows (perm[j] >= 0, or all) of |x - mu| (synchronises the stream)
float launch_maxabs(const float* X, int64_t n, int d, const int64_t* perm, const float* mu, cudaStream_t st);
bool krow_tc_2cta();
void launch_csr_densify(const int64_t* indptr, const int32_t* indices, const float* values, int64_t n, int d, float* X,
                        int32_t* bad, cudaStream_t st);
void launch_scatter_oof(const double* dec, int64_t m, int P, const int32_t* cls, const int64_t* rnk,
                        const PairDesc* pairs, double* v, cudaStream_t st);
void launch_sigmoid_fit_on(const PairDesc* pairs, int P, const double* v, double* A, double* B, int32_t* status,
                           cudaStream_t st);
void launch_build_coef(const double* alpha, const int64_t* aoff, const int64_t* slot_g, const int64_t* off,
                       const int64_t* cc, int k, int64_t nsv_pad, int km1_pad, float* coef, double* coef64,
                       cudaStream_t st);
void launch_alpha_abs_sum(const double* alpha, const int64_t* aoff, const int64_t* np, int P, double* out,
                          cudaStream_t st);
std::vector<int2> krow_tc_tiles(int64_t n, bool two_cta);
constexpr int kKrowTileRows = 128;  // krow_tc tile edge (rows = columns)
// per-class means of the staged hi rows (class c = rows [coff[c], coff[c+1])): mu[k][d_pad]
void launch_class_means(const void* hi, int d_pad, const int64_t* coff, int k, float* mu, float* m2, cudaStream_t st);
// split with a given centre mu[d] and scale sc (prediction: the test rows take the SVs' mu, sc)
void launch_split_hilo_mu(const float* X, int64_t n, int d, const int64_t* perm, const float* mu, float sc, void* hi,
                          void* lo, float* norms, int64_t n_pad, int d_pad, cudaStream_t st);
// mu[c] = mean over the rows idx[i] >= 0 (cnt of them) of X[., c]
void launch_gather_col_mean(const float* X, int d, const int64_t* idx, int64_t n, int64_t cnt, float* mu,
                            cudaStream_t st);
// a10 with exact dot products (dec_i8.cu): rows -> 5 int8 digit planes [5][rows_pad][round_up(d, 32)]
// (src: row index per output row, < 0 = zero row; nullptr = identity), per-row exponent and FP64
// norm of the fixed-point row; amax (optional): max |x| over the rows as float bits (atomicMax)
int dec_i8_max_km1();
size_t dec_i8_plane_bytes(int64_t rows_pad, int d);
double dec_i8_kernel_err(double ax, double ay, int d, double gamma);  // bound on |K~ - K| (RBF)
void launch_stage_i8(const float* X, int64_t n, int d, const int64_t* src, int8_t* planes, int64_t rows_pad,
                     int32_t* ex, double* nrm, unsigned* amax, cudaStream_t st);
void launch_dec_i8(const int8_t* tplanes, int64_t m_pad, const int32_t* et, const double* nt, const int8_t* splanes,
                   int64_t nsv_pad, const int32_t* es, const double* ns, int d, const int2* tiles,
                   const int32_t* unit_off, const int32_t* unit_item, int n_units, const double* coef64, int km1,
                   int km1_pad, double gamma, double* part, cudaStream_t st);
// a10 on tcgen05 (krow_tc.cu): tiles = (test tile, SV tile) grouped in units [unit_off[u],
// unit_off[u+1]), unit u writes part[unit_item[u]][row][0..km1_pad) (as launch_dec_contract)
int dec_tc_max_km1();
void launch_dec_tc(const void* thi, const void* tlo, int64_t m_pad, const void* shi, const void* slo, int64_t nsv_pad,
                   int d_pad, const int2* tiles, const int32_t* unit_off, const int32_t* unit_item, int n_units,
                   const float* nt, const float* nsv, const float* coef, int km1, int km1_pad, double gamma, float sc,
                   float* part, cudaStream_t st,
                   const KrowKernel* dk = nullptr);
void launch_krow_tc(const void* hi, const void* lo, int64_t n_pad, int d_pad, const int2* tiles, int n_tiles,
                    const float* norms, int64_t n, double gamma, float sc, float* K, int64_t ldk, cudaStream_t st,
                    bool two_cta = false, const KrowKernel* dk = nullptr, int reserve_sms = 0,
                    unsigned long long* resident = nullptr, bool mc = false, int d_real = 0);
int krow_tc_grid(int n_tiles, int reserve_sms, bool mc = false);  // CTAs of that launch
// 2-CTA clusters with the shared row operand multicast (default; GMPSVM_KROW_MC=0 off): the tile
// list must be cluster pairs (krow_tc_mc_pairs) and the launch passes mc = true
bool krow_tc_mc();
std::vector<int2> krow_tc_mc_pairs(const std::vector<int2>& tiles);
void launch_row_norms(const float* X, int64_t n, int d, const int64_t* perm, float* norms, int64_t n_pad, int32_t* bad,
                      cudaStream_t st);
bool krow_use_tc();  // GMPSVM_KROW=simt selects the FP32 SIMT kernel

// ---------------- a4-a9 solver (solver.cu, wsolve.cu)
struct SolverArgs {
  const PairDesc* pairs;
  const float* K;
  int64_t ldk;
  double* alpha;        // [sum n_p]
  double* f;            // [sum n_p]
  double* v;            // [sum n_p] in-sample decision values (finalize)
  uint32_t* stamp;      // [sum n_p] selection stamps
  int32_t* ws;          // [P][B] working set (pair-local indices), oldest first
  int32_t* ws_n;        // [P]
  int32_t* ws_tmp;      // [P][B]
  float* Kws;           // [P][B][B] gathered K_ws,ws
  double* dcoef;        // [P][B] delta-alpha * y of the last local solve
  int32_t* status;      // [P] 0 active, 1 converged, 2 outer cap
  double* gap;          // [P] global gap at the last selection
  int64_t* inner_iters; // [P]
  int64_t* smo_cycles;  // [P] SM clock cycles spent in local_smo (diagnostic)
  int64_t* smo_phase;   // [P][5] optional per-phase cycles (GMPSVM_SMO_PHASES=1), else NULL
  int64_t* body_iters;  // [P] executions of the graph loop body (device-driven solver)
  int64_t* trace;       // optional kernel timeline of one pair (GMPSVM_TRACE=<pair position>): [cap][3]
  int32_t* trace_n;
  int32_t trace_pair, trace_cap;
  int32_t fu_chunks = 1;  // 128-column chunks per f-update CTA (ws_fupdate_kernel)
  int32_t smo_f32 = 0;    // local SMO with FP32 working-set f (wsolve.cu ws_smo_body)
  uint8_t* ulf = nullptr;  // per instance: bit0 in I_u, bit1 in I_l (wsolve.cu: written by the local SMO,
                           // read by the selection instead of alpha; null: alpha is read)
  int64_t* sel_phase;   // [P][5] optional select_ws phase cycles (GMPSVM_SMO_PHASES=1), else NULL
  int32_t* outer_iters; // [P]
  double* b;            // [P]
  double* A;            // [P]
  double* Bs;           // [P] (sigmoid B)
  int32_t* sig_status;  // [P]
  int B, q, inner_cap;
  int pair_base;        // first local pair of this launch (grid.x pairs from here)
  double C, eps;
  double local_ratio;  // local solve stops at gap < max(eps, local_ratio * delta0) (reading R20: 0.1)
  // ---- ROW_CACHE regime (kernel matrix does not fit): R != NULL, K == NULL
  float* R;             // per pair B x ldr rows K(x_ws, x_pair) in pair-local column order (the paper's buffer)
  int32_t* ws_slot;     // [P][B] R row slot of each working-set position
  int32_t* ws_slot_tmp; // [P][B]
  int32_t* ws_keep;     // [P] retained positions of the last selection (rows to compute start there)
  const float* XT;      // class-sorted feature-major X, d_pad x ldx (zero padded)
  int64_t ldx;
  const float* norms;   // [ldx] squared norms (class-sorted)
  float* ATnew;         // [P][d_pad][B] gathered new working-set rows (feature-major)
  int d_pad;
  int64_t* rows_done;  // [P] kernel rows computed (ROW_CACHE statistics)
  int ldat;            // leading dimension of ATnew (round_up(B, 128))
  double gamma;
  // ---- ROW_CACHE rows on tcgen05 (krow_tc.cu rows_tc_kernel): the class-sorted FP16 hi/lo split
  // of X (row-major, dpt halfs per row; norms above are then its centred, scaled norms) and the
  // gathered new rows of every pair [P][ldat][dpt]; exp2 scale of the split (-gamma log2 e / s^2)
  const void* Xhi;
  const void* Xlo;
  void* Ahi;
  void* Alo;
  int dpt;
  int64_t n_pad;
  float kscale;
};
constexpr int kWsMaxNp = 16384;  // pair size limit of the default path (keys + flags in shared memory)

void launch_init_pairs(const SolverArgs& a, int P, int64_t tot, cudaStream_t st);
void launch_select_ws(const SolverArgs& a, int P, uint32_t stampv, int first, cudaStream_t st);
void launch_gather_kws(const SolverArgs& a, int P, int first, cudaStream_t st);
void launch_local_smo(const SolverArgs& a, int P, cudaStream_t st);
bool local_smo_uses_smem(int B);  // K_ws,ws gathered in-kernel (no gather_kws launch, no Kws buffer)
void launch_f_update(const SolverArgs& a, int P, int64_t np_max, cudaStream_t st);
// ROW_CACHE: kernel rows of the new working-set entries of every pair of the launch
void launch_f_update_loop(const SolverArgs& a, int P, int64_t np_max, cudaGraphConditionalHandle h, int64_t max_outer,
                          cudaStream_t st);
void launch_rows_compute(const SolverArgs& a, int P, int64_t np_max, cudaStream_t st);
// the same rows on tcgen05: tiles = (local pair, 128-row tile of its new rows, column tile of its
// two class segments) for the pairs of the launch (krow_tc.cu); n_pairs_all = Pl (rows of A)
std::vector<int4> rows_tc_tiles(const std::vector<PairDesc>& pairs, int first, int count, int B);
void launch_rows_compute_tc(const SolverArgs& a, int P, const int4* tiles, int n_tiles, int n_pairs_all,
                            cudaStream_t st);
// a3-a5 default kernels (wsolve.cu): fast selection, multi-CTA K_ws,ws gather into an
// L2-resident tile, single-warp local SMO (FULL_K regime, B <= 224, n_p <= 16384;
// GMPSVM_WSOLVE=0 selects the select_ws / gather_kws / local_smo kernels of solver.cu)
bool ws_solve_supported(int B, int64_t np_max);
void launch_ws_smo(const SolverArgs& a, int P, cudaStream_t st);  // single-warp local SMO alone (B <= ws_smo_max_b)
int ws_smo_max_b();
int ws_tile_ld_of(int B);  // row stride of the K_ws,ws tile of the single-warp solver
size_t ws_tile_floats(int B);  // per-pair floats of the Kws buffer (tile + SMO state)
// Per-pair stride (floats) of the Kws buffer, the same for both solver paths: one graph may run
// wsolve.cu pairs (tile with row stride round_up(B, 4) + alpha/f/index state) next to solver.cu
// pairs (B x B tile), so every pair's slot must use this stride.
__host__ __device__ inline size_t kws_pair_stride(int B) {
  const size_t ld = (size_t)((B + 3) & ~3);
  return (size_t)B * ld + 4 * (size_t)B + ld;
}
// one outer iteration: selection (+ stop test), K_ws,ws gather, single-warp local SMO, f-update
// (with set_cond it sets the graph loop condition); programmatic dependent launches inside the
// iteration, and across iterations when chained (the previous iteration is in the same stream)
void launch_ws_iteration(const SolverArgs& a, int P, int64_t np_max, cudaGraphConditionalHandle h, int set_cond,
                         int64_t max_outer, cudaStream_t st, bool chained = false);
// Persistent solver (wsolve.cu): the outer loops of pairs [pair_base, pair_base + P) as P leader
// CTAs (one per SM) and `nworkers` worker CTAs (ws_persist_workers_per_sm() per SM beside them),
// launched together on st; ring: ws_persist_ring_bytes(), ctr: ws_persist_ctr_words(P) words,
// both zeroed before the launch; ctr[3] != 0 after the run: a wait timed out (the solve is invalid).
bool ws_persist_supported(int B, int64_t np_max);
size_t ws_persist_smem(int B);
size_t ws_persist_ctr_words(int P);
size_t ws_persist_ring_bytes();
int ws_persist_workers_per_sm();
// wait_resident > 0: the leaders trigger the workers only once *res_ctr (the kernel-value launch's
// started-CTA count, KrowKernel::resident) reaches it, so the workers land beside that launch.
void launch_ws_persist(const SolverArgs& a, int P, int nworkers, int64_t max_outer, void* ring, unsigned long long* ctr,
                       cudaStream_t st, const unsigned long long* res_ctr = nullptr, int wait_resident = 0);
// ---------------- NEXT-3: CSR kernel values (csr.cu)
// device CSR rows of X: indptr [n+1], indices [nnz] (columns in [0, d)), values [nnz]
struct CsrSrc {
  const int64_t* indptr;
  const int32_t* indices;
  const float* values;
  int64_t nnz;
};
// class-sorted copy: row i of the sorted order = input row perm[i], sptr its row pointers;
// norms[i] = |x_i|^2 (FP64-accumulated); *bad = 1 on a column outside [0, d) or a non-finite value
void launch_csr_stage(const int64_t* indptr, const int32_t* indices, const float* values, const int64_t* perm, int64_t n,
                      int32_t d, const int64_t* sptr, int32_t* sidx, float* sval, float* norms, int32_t* bad,
                      cudaStream_t st);
int krow_csr_rows_per_cta(int32_t d);  // dense rows per CTA in shared memory (0: d too large)
// FULL_K (n x ldk, symmetric, K_ii = 1) from the sorted CSR rows: sparse x dense, one warp per column row
void launch_krow_csr(const int64_t* sptr, const int32_t* sidx, const float* sval, const float* norms, int64_t n,
                     int32_t d, double gamma, float* K, int64_t ldk, cudaStream_t st);
void launch_csr_densify_rows(const int64_t* indptr, const int32_t* indices, const float* values, const int64_t* rows,
                             int64_t nr, int32_t d, float* out, cudaStream_t st);
void launch_finalize(const SolverArgs& a, int P, cudaStream_t st);
void launch_sigmoid_fit(const SolverArgs& a, int P, cudaStream_t st);
void launch_sv_flags(const SolverArgs& a, int P, int64_t np_max, uint8_t* flags, cudaStream_t st);

// ---------------- a10-a12 prediction (predict.cu)
struct DecItem {
  int32_t cls, tile_begin, tile_end, pad;
};
void launch_dec_contract(const float* XtT, int64_t ldt, const float* nt, int64_t m, int64_t m_pad, const float* SvT,
                         int64_t lds, const float* nsv, const float* coef, int km1, int km1_pad, const DecItem* items,
                         int n_items, int kdim, double gamma, float* part, cudaStream_t st);
void launch_col_norms64(const float* XT, int64_t ld, int64_t n, int d_pad, double* out, cudaStream_t st);
void launch_dec_f64(const float* XtT, int64_t ldt, const double* nt64, int64_t m_pad, const float* SvT, int64_t lds,
                    const double* nsv64, const double* coef64, int km1, int km1_pad, const DecItem* items, int n_items,
                    int d_pad, double gamma, double* part, cudaStream_t st, int ktype = 0, double coef0 = 0.0,
                    int degree = 3);
void launch_dec_reduce64(const double* part, int64_t m, int64_t m_pad, int k, int km1_pad, const int32_t* item_begin,
                         const int32_t* item_end, const double* b, double* dec, cudaStream_t st);
void launch_dec_reduce(const float* part, int64_t m, int64_t m_pad, int k, int km1_pad, const int32_t* item_begin,
                       const int32_t* item_end, const double* b, double* dec, cudaStream_t st);
void launch_couple(const double* dec, int64_t m, int k, const double* A, const double* B, double* prob,
                   cudaStream_t st);

}  // namespace gmpsvm
