// shard.cu -- NEXT-1: one binary SVM of a pair trained by several ranks at
// once, its instances sharded (the paper's instance-level parallelism inside a pair, PAPER.md
// L250; a row batch is "a matrix multiplication between the q instances and the rest", L299).
//
// Every rank holds X (replicated, as in the pair-sharded path) and owns a contiguous slice
// [lo, hi) of the pair's instances (pair-local order: class s, then class t): it keeps f for its
// slice and the kernel rows K(x_ws, x_slice) of the working set.  alpha is replicated.  Per outer
// iteration (Algorithm 2 lines 6-11, readings R19 / R20):
//   candidates  each rank: min_{I_u} f / max_{I_l} f of its slice (Eq 9-10) and its `need`
//               smallest (key, index) per side among the non-retained I_u / I_l members
//   [all_gather of the candidate blocks: the caller's collective]
//   select      every rank: the same exact merge (R19 semantics; ties -> lowest index) -> the
//               new working set; kernel rows of its new members against the slice (SIMT FP32,
//               the ROW_CACHE contraction) and K_ws,ws (B x B, identical on every rank)
//   fws         each rank: f of the working-set members it owns (0 elsewhere)
//   [all_reduce (sum) of fws: the caller's collective]
//   step        every rank: the same local SMO on K_ws,ws (solver.cu's local_smo, deterministic,
//               so alpha stays replicated), then the f update of its slice (Eq 8)
// The collectives move O(world * B) doubles per outer iteration; rows, f update and candidate
// selection are split world-ways.  finish: the caller gathers f; bias (R7), in-sample decision
// values and the sigmoid (Eq 12-13) run on the full vectors.  With world = 1 this is a complete
// single-rank solver; world > 1 gives bitwise the same alpha (every per-column quantity is
// computed by the same arithmetic regardless of the slicing).
#include <algorithm>
#include <cfloat>
#include <climits>
#include <cstring>
#include <vector>

#include "kernels.h"
#include "model.h"
#include "solver_dev.cuh"

namespace gmpsvm {

namespace {

constexpr int kCandChunk = 16384;  // slice elements per candidate CTA

// candidate source over the slice [lo, lo + len) of the pair (alpha / f full pair-local vectors)
struct SliceSrc {
  const double* al;
  const double* fl;
  const uint8_t* ret;  // [len] retained by the next working set
  uint32_t* st;        // [len] taken stamps
  uint32_t stampv;
  int64_t lo;
  int n_s;
  double C;
  template <bool SIDE_U>
  __device__ __forceinline__ bool cand(int i, uint64_t& key) const {
    const int64_t j = lo + i;
    const int y = j < n_s ? 1 : -1;
    const double a = al[j];
    const bool ok = SIDE_U ? in_u(y, a, C) : in_l(y, a, C);
    if (!ok || ret[i] || st[i] == stampv) return false;
    key = ord_key(fl[j]);
    if (!SIDE_U) key = ~key;
    return true;
  }
  __device__ __forceinline__ void take(int i) const { st[i] = stampv; }
};

// out (doubles): [fmin, fmax, nU, nL, U key bits x need, U index x need, L key bits x need, L index x need]
// grid: one CTA per chunk of the slice (chunk elements each), CTA c writing sub-block c
__global__ void __launch_bounds__(1024) shard_cand_kernel(const double* al, const double* fl, const uint8_t* ret_all,
                                                          uint32_t* st_all, uint32_t stamp0, int64_t lo_all, int len_all,
                                                          int chunk, int n_s, double C, int need, int stride,
                                                          int32_t* tmp_all, double* out_all) {
  __shared__ SelSmem sm;
  __shared__ double red[32];
  const int c0 = blockIdx.x * chunk;
  const int len = max(0, min(chunk, len_all - c0));
  const int64_t lo = lo_all + c0;
  const uint8_t* ret = ret_all + c0;
  uint32_t* st = st_all + c0;
  int32_t* tmp = tmp_all + (int64_t)blockIdx.x * 2 * need;
  double* out = out_all + (int64_t)blockIdx.x * (4 + 4 * stride);
  double fmin = DBL_MAX, fmax = -DBL_MAX;
  for (int i = threadIdx.x; i < len; i += blockDim.x) {
    const int64_t j = lo + i;
    const int y = j < n_s ? 1 : -1;
    const double a = al[j], f = fl[j];
    if (in_u(y, a, C)) fmin = fmin < f ? fmin : f;
    if (in_l(y, a, C)) fmax = fmax > f ? fmax : f;
  }
  fmin = block_reduce(fmin, [](double x, double y2) { return x < y2 ? x : y2; }, red);
  fmax = block_reduce(fmax, [](double x, double y2) { return x > y2 ? x : y2; }, red);
  // each side independently (the merge decides which ones the other side may not take)
  const SliceSrc su{al, fl, ret, st, stamp0, lo, n_s, C};
  const int nu = radix_pick<true>(su, len, need, tmp, sm);
  const SliceSrc sl{al, fl, ret, st, stamp0 + 1, lo, n_s, C};
  const int nl = radix_pick<false>(sl, len, need, tmp + need, sm);
  double* uk = out + 4;
  double* ui = uk + stride;
  double* lk = ui + stride;
  double* li = lk + stride;
  for (int e = threadIdx.x; e < need; e += blockDim.x) {
    if (e < nu) {
      const int64_t j = lo + tmp[e];
      uk[e] = __longlong_as_double((long long)ord_key(fl[j]));
      ui[e] = (double)j;
    }
    if (e < nl) {
      const int64_t j = lo + tmp[need + e];
      lk[e] = __longlong_as_double((long long)~ord_key(fl[j]));
      li[e] = (double)j;
    }
  }
  if (threadIdx.x == 0) {
    out[0] = fmin;
    out[1] = fmax;
    out[2] = nu;
    out[3] = nl;
  }
}

// feature-major gather of working-set rows: AT[c][e] = XT[c][idx[e]], norms
__global__ void shard_gather_kernel(const float* XT, int64_t ldx, const float* nx, const int32_t* idx, int cnt,
                                    int d_pad, float* AT, int64_t lda, float* na) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= lda) return;
  const int64_t j = e < cnt ? idx[e] : -1;
  for (int c = blockIdx.y; c < d_pad; c += gridDim.y) AT[(int64_t)c * lda + e] = j >= 0 ? XT[(int64_t)c * ldx + j] : 0.f;
  if (blockIdx.y == 0) na[e] = j >= 0 ? nx[j] : 0.f;
}

// new kernel rows (tmp row r) -> their slots of R
__global__ void shard_place_rows_kernel(const float* tmp, int64_t ldt, const int32_t* slot, int cnt, int64_t len,
                                        float* R, int64_t ldr) {
  const int r = blockIdx.y;
  if (r >= cnt) return;
  const float* src = tmp + (int64_t)r * ldt;
  float* dst = R + (int64_t)slot[r] * ldr;
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < len; j += (int64_t)gridDim.x * blockDim.x)
    dst[j] = src[j];
}

// the rows with dalpha != 0, in position order: nzl = [count, (coef, slot) ...]
__global__ void shard_nz_kernel(const double* dcoef, const int32_t* slot, int wn, double* nzc, int32_t* nzs, int* nzn) {
  if (threadIdx.x == 0) {
    int c = 0;
    for (int e = 0; e < wn; ++e)
      if (dcoef[e] != 0.0) {
        nzc[c] = dcoef[e];
        nzs[c] = slot[e];
        ++c;
      }
    *nzn = c;
  }
}
// f_j += sum_{e : dcoef_e != 0} dcoef_e R[slot_e][j - lo] over the slice, FP64, rows in position order
__global__ void shard_fupdate_kernel(const double* nzc, const int32_t* nzs, const int* nzn, const float* R, int64_t ldr,
                                     int64_t lo, int64_t len, double* f) {
  __shared__ double cf[1024];
  __shared__ int32_t sl[1024];
  const int nz = *nzn;
  for (int r = threadIdx.x; r < nz; r += blockDim.x) {
    cf[r] = nzc[r];
    sl[r] = nzs[r];
  }
  __syncthreads();
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= len) return;
  double acc = 0.0;
  for (int r = 0; r < nz; ++r) acc = fma(cf[r], (double)R[(int64_t)sl[r] * ldr + j], acc);
  f[lo + j] += acc;
}

__global__ void shard_fws_kernel(const double* f, const int32_t* ws, int wn, int64_t lo, int64_t hi, double* out) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= wn) return;
  const int32_t j = ws[e];
  out[e] = (j >= lo && j < hi) ? f[j] : 0.0;
}
__global__ void shard_scatter_fws_kernel(const double* fws, const int32_t* ws, int wn, double* f) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e < wn) f[ws[e]] = fws[e];
}
// the single-warp solver's state behind the tile: alpha, f, index of the working set (sorted order)
__global__ void shard_state_kernel(const double* alpha, const double* fws, const int32_t* ws, int wn, float* buf,
                                   size_t state_off, int B) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= wn) return;
  double* st_al = reinterpret_cast<double*>(buf + state_off);
  double* st_f = st_al + B;
  int32_t* st_ix = reinterpret_cast<int32_t*>(st_f + B);
  st_al[e] = alpha[ws[e]];
  st_f[e] = fws[e];
  st_ix[e] = ws[e];
}
__global__ void shard_init_kernel(double* alpha, double* f, int64_t np, int n_s) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < np) {
    alpha[j] = 0.0;
    f[j] = j < n_s ? -1.0 : 1.0;  // f = -y (Alg 1 lines 1-2)
  }
}

}  // namespace

struct Shard {
  int device = 0;
  cudaStream_t st = nullptr;
  bool own_stream = false;
  int k = 0, s = 0, t = 0, rank = 0, world = 1;
  double C = 0, gamma = 0, eps = 0;
  int64_t n_s = 0, n_t = 0, np = 0, lo = 0, hi = 0, len = 0, ldr = 0;
  int d = 0, d_pad = 0, B = 0, q = 0, need_max = 0;
  int64_t ldx = 0;
  int64_t max_outer = 0, outer = 0, inner = 0;
  int status = 0;       // 0 running, 1 converged, 2 outer cap
  double gap = 0.0;
  std::vector<int32_t> ws_age;   // working set, age order (oldest first)
  std::vector<int32_t> ws;       // sorted by index
  std::vector<int32_t> slot_of;  // slot of each ws position (sorted order)
  std::vector<int32_t> prev_slot_by_idx_keys, prev_slot_by_idx_vals;
  // device
  DevBuf<float> XT, nx, AT, na, Rtmp, R, Kws;
  DevBuf<double> alpha, f, cand, v, dcoef, fws, bb, AA, BB, gapv;
  DevBuf<uint8_t> ret;
  DevBuf<uint32_t> stamp;
  DevBuf<int32_t> tmp, d_ws, d_slot, d_status, d_wsn, d_inner, d_outer, d_sig, nzs, nzn;
  DevBuf<double> nzc;
  DevBuf<int64_t> d_inner64, d_cyc;
  DevBuf<PairDesc> d_pair;
  uint32_t stampv = 1;
  int chunks = 1;  // candidate CTAs (sub-blocks) per rank: the same count on every rank
  bool warp_smo() const { return B <= ws_smo_max_b(); }  // wsolve.cu's single-warp solver, tile in smem
  int tile_ld() const { return warp_smo() ? ws_tile_ld_of(B) : B; }
  int cand_doubles() const { return chunks * (4 + 4 * need_max); }
};

static SolverArgs shard_args(Shard& S) {
  SolverArgs a{};
  a.pairs = S.d_pair.get();
  a.alpha = S.alpha.get();
  a.f = S.f.get();
  a.v = S.v.get();
  a.ws = S.d_ws.get();
  a.ws_n = S.d_wsn.get();
  a.Kws = S.Kws.get();
  a.dcoef = S.dcoef.get();
  a.status = S.d_status.get();
  a.gap = S.gapv.get();
  a.inner_iters = S.d_inner64.get();
  a.smo_cycles = S.d_cyc.get();
  a.outer_iters = S.d_outer.get();
  a.b = S.bb.get();
  a.A = S.AA.get();
  a.Bs = S.BB.get();
  a.sig_status = S.d_sig.get();
  a.B = S.B;
  a.q = S.q;
  // FP32 working-set f in the local solve (R29, as the single-GPU solver for the Gaussian kernel);
  // no B/2 step cap here: a sharded pair is a large one, where each outer iteration costs a full
  // selection over the pair (measured, MNIST8M-shaped 1M rows, pair (0,8): 4,234 -> 14,028 outer
  // iterations with the cap)
  a.inner_cap = 100 * S.B;
  a.smo_f32 = 1;
  a.pair_base = 0;
  a.C = S.C;
  a.eps = S.eps;
  a.local_ratio = 0.1;
  a.gamma = S.gamma;
  return a;
}

Shard* shard_create(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, int32_t s, int32_t t, double C,
                    double gamma, double eps, int32_t rank, int32_t world, const gmpsvm_options& opt) {
  if (!X || !y || n < 2 || d < 1 || k < 2 || s < 0 || t <= s || t >= k || !(C > 0) || !(gamma > 0) || !(eps > 0) ||
      world < 1 || rank < 0 || rank >= world)
    throw Error(GMPSVM_EINVAL, "bad shard arguments");
  if (opt.kernel != 0) throw Error(GMPSVM_ENOTIMPL, "the sharded pair solver runs the Gaussian kernel");
  auto S = std::make_unique<Shard>();
  S->device = opt.device;
  GM_CUDA(cudaSetDevice(opt.device));
  S->st = opt.stream ? static_cast<cudaStream_t>(opt.stream) : nullptr;
  if (!S->st) {
    GM_CUDA(cudaStreamCreateWithFlags(&S->st, cudaStreamNonBlocking));
    S->own_stream = true;
  }
  cudaStream_t st = S->st;
  S->k = k;
  S->s = s;
  S->t = t;
  S->rank = rank;
  S->world = world;
  S->C = C;
  S->gamma = gamma;
  S->eps = eps;
  S->d = d;
  std::vector<int32_t> hy(n);
  if (opt.inputs_on_device) GM_CUDA(cudaMemcpy(hy.data(), y, (size_t)n * 4, cudaMemcpyDeviceToHost));
  else std::memcpy(hy.data(), y, (size_t)n * 4);
  std::vector<int64_t> perm;  // pair-local order -> original row
  for (int64_t i = 0; i < n; ++i)
    if (hy[i] == s) perm.push_back(i);
  S->n_s = (int64_t)perm.size();
  for (int64_t i = 0; i < n; ++i)
    if (hy[i] == t) perm.push_back(i);
  S->np = (int64_t)perm.size();
  S->n_t = S->np - S->n_s;
  if (S->n_s == 0 || S->n_t == 0) throw Error(GMPSVM_EINVAL, "both classes of the pair need instances");
  if (S->np > INT32_MAX / 2) throw Error(GMPSVM_ENOTIMPL, "pair too large");
  S->B = opt.ws_size > 0 ? opt.ws_size : 192;
  if (S->B < 2 || (S->B & 1) || S->B > 1024) throw Error(GMPSVM_EINVAL, "ws_size must be even, 2..1024");
  S->B = (int)std::min<int64_t>(S->B, S->np + (S->np & 1));
  S->q = opt.q > 0 ? std::min(opt.q, S->B) : S->B / 2;
  S->need_max = S->B;
  S->max_outer = opt.max_outer_iter > 0 ? opt.max_outer_iter : 1000000;
  // slice: contiguous, boundaries on multiples of 128 (aligned float4 column access)
  const int64_t per = round_up(ceil_div(S->np, world), kTile);
  S->lo = std::min(S->np, per * rank);
  S->hi = std::min(S->np, S->lo + per);
  S->len = S->hi - S->lo;
  S->chunks = (int)std::max<int64_t>(1, ceil_div(per, kCandChunk));
  S->ldr = round_up(std::max<int64_t>(S->len, 1), 4);
  S->d_pad = (int)round_up(d, kBK);
  S->ldx = round_up(S->np, kTile) + kTile;  // + a tile: column tiles starting at lo stay in bounds
  // stage the pair's rows feature-major (pair-local order), with norms
  DevBuf<int64_t> d_perm(S->np, st);
  GM_CUDA(cudaMemcpyAsync(d_perm.get(), perm.data(), (size_t)S->np * 8, cudaMemcpyHostToDevice, st));
  DevBuf<float> xin(opt.inputs_on_device ? 0 : (size_t)n * d, st);
  const float* dX = X;
  if (!opt.inputs_on_device) {
    GM_CUDA(cudaMemcpyAsync(xin.get(), X, (size_t)n * d * 4, cudaMemcpyHostToDevice, st));
    dX = xin.get();
  }
  new (&S->XT) DevBuf<float>((size_t)S->d_pad * S->ldx, st);
  new (&S->nx) DevBuf<float>(S->ldx, st);
  GM_CUDA(cudaMemsetAsync(S->XT.get(), 0, (size_t)S->d_pad * S->ldx * 4, st));
  GM_CUDA(cudaMemsetAsync(S->nx.get(), 0, (size_t)S->ldx * 4, st));
  launch_stage_features(dX, S->np, d, d_perm.get(), S->XT.get(), S->ldx, S->d_pad, S->ldx, S->nx.get(), nullptr, st);
  const int ldat = (int)round_up(S->B, kTile);
  new (&S->AT) DevBuf<float>((size_t)S->d_pad * ldat, st);
  new (&S->na) DevBuf<float>(ldat, st);
  new (&S->Rtmp) DevBuf<float>((size_t)S->B * S->ldr, st);
  new (&S->R) DevBuf<float>((size_t)S->B * S->ldr, st);
  new (&S->Kws) DevBuf<float>(kws_pair_stride(S->B), st);
  new (&S->alpha) DevBuf<double>(S->np, st);
  new (&S->f) DevBuf<double>(S->np, st);
  new (&S->v) DevBuf<double>(S->np, st);
  new (&S->cand) DevBuf<double>(S->cand_doubles(), st);
  new (&S->dcoef) DevBuf<double>(S->B, st);
  new (&S->fws) DevBuf<double>(S->B, st);
  new (&S->bb) DevBuf<double>(1, st);
  new (&S->AA) DevBuf<double>(1, st);
  new (&S->BB) DevBuf<double>(1, st);
  new (&S->gapv) DevBuf<double>(1, st);
  new (&S->ret) DevBuf<uint8_t>(std::max<int64_t>(S->len, 1), st);
  new (&S->stamp) DevBuf<uint32_t>(std::max<int64_t>(S->len, 1), st);
  new (&S->tmp) DevBuf<int32_t>((size_t)2 * S->B * S->chunks, st);
  new (&S->nzs) DevBuf<int32_t>(S->B, st);
  new (&S->nzn) DevBuf<int32_t>(1, st);
  new (&S->nzc) DevBuf<double>(S->B, st);
  new (&S->d_ws) DevBuf<int32_t>(S->B, st);
  new (&S->d_slot) DevBuf<int32_t>(S->B, st);
  new (&S->d_status) DevBuf<int32_t>(1, st);
  new (&S->d_wsn) DevBuf<int32_t>(1, st);
  new (&S->d_outer) DevBuf<int32_t>(1, st);
  new (&S->d_sig) DevBuf<int32_t>(1, st);
  new (&S->d_inner64) DevBuf<int64_t>(1, st);
  new (&S->d_cyc) DevBuf<int64_t>(1, st);
  new (&S->d_pair) DevBuf<PairDesc>(1, st);
  PairDesc pd{};
  pd.s = s;
  pd.t = t;
  pd.n_s = (int32_t)S->n_s;
  pd.n_t = (int32_t)S->n_t;
  pd.off_s = 0;
  pd.off_t = S->n_s;
  pd.a_off = 0;
  pd.pid = pair_index(s, t, k);
  GM_CUDA(cudaMemcpyAsync(S->d_pair.get(), &pd, sizeof(pd), cudaMemcpyHostToDevice, st));
  GM_LAUNCH(shard_init_kernel, dim3((unsigned)ceil_div(S->np, 256)), dim3(256), 0, st, S->alpha.get(), S->f.get(), S->np,
            (int)S->n_s);
  GM_CUDA(cudaMemsetAsync(S->stamp.get(), 0, (size_t)std::max<int64_t>(S->len, 1) * 4, st));
  GM_CUDA(cudaMemsetAsync(S->d_status.get(), 0, 4, st));
  GM_CUDA(cudaMemsetAsync(S->d_inner64.get(), 0, 8, st));
  GM_CUDA(cudaMemsetAsync(S->d_cyc.get(), 0, 8, st));
  GM_CUDA(cudaStreamSynchronize(st));
  return S.release();
}

void shard_free(Shard* S) {
  if (!S) return;
  cudaSetDevice(S->device);
  cudaStreamSynchronize(S->st);
  cudaStream_t st = S->own_stream ? S->st : nullptr;
  delete S;  // device buffers are freed stream-ordered on S->st
  if (st) {
    cudaStreamSynchronize(st);
    cudaStreamDestroy(st);
  }
}

int shard_cand_doubles(const Shard* S) { return S->cand_doubles(); }

// retained rows of the next selection: the newest B - q of the current working set (R19)
static std::vector<int32_t> retained(const Shard& S) {
  if (S.np <= S.B || S.ws_age.empty()) return {};
  const int keep = std::min<int>((int)S.ws_age.size(), S.B - S.q);
  return std::vector<int32_t>(S.ws_age.end() - keep, S.ws_age.end());
}

static void cand_launch(Shard* S, double* out) {
  cudaStream_t st = S->st;
  const std::vector<int32_t> kept = retained(*S);
  std::vector<uint8_t> r(std::max<int64_t>(S->len, 1), 0);
  for (int32_t j : kept)
    if (j >= S->lo && j < S->hi) r[j - S->lo] = 1;
  GM_CUDA(cudaMemcpyAsync(S->ret.get(), r.data(), r.size(), cudaMemcpyHostToDevice, st));
  const int need = S->np <= S->B ? 0 : S->B - (int)kept.size();
  GM_CUDA(cudaMemsetAsync(S->cand.get(), 0, (size_t)S->cand_doubles() * 8, st));
  GM_LAUNCH(shard_cand_kernel, dim3((unsigned)S->chunks), dim3(1024), 0, st, S->alpha.get(), S->f.get(), S->ret.get(),
            S->stamp.get(), S->stampv, S->lo, (int)S->len, kCandChunk, (int)S->n_s, S->C, need, S->need_max,
            S->tmp.get(), S->cand.get());
  S->stampv += 2;
  GM_CUDA(cudaMemcpyAsync(out, S->cand.get(), (size_t)S->cand_doubles() * 8, cudaMemcpyDeviceToHost, st));
}

void shard_candidates(Shard* S, double* out) {
  GM_CUDA(cudaSetDevice(S->device));
  cand_launch(S, out);
  GM_CUDA(cudaStreamSynchronize(S->st));
}

// The exact merge of every rank's candidate block (host, deterministic).  need / need_u: picks
// wanted in total / from I_u first.  picks: selection order (U by (key, index), then L skipping
// U's picks, then U again if L ran short).  Returns the global gap max_{I_l} f - min_{I_u} f.
double shard_merge(const double* all, int world, int cand_doubles, int need, int need_u, std::vector<int32_t>& picks) {
  const int nmax = (cand_doubles - 4) / 4;
  double fmin = DBL_MAX, fmax = -DBL_MAX;
  struct E {
    uint64_t k;
    int32_t i;
  };
  std::vector<E> U, L;
  for (int r = 0; r < world; ++r) {
    const double* c = all + (size_t)r * cand_doubles;
    fmin = std::min(fmin, c[0]);
    fmax = std::max(fmax, c[1]);
    const int nu = (int)c[2], nl = (int)c[3];
    const double* uk = c + 4;
    const double* ui = uk + nmax;
    const double* lk = ui + nmax;
    const double* li = lk + nmax;
    for (int e = 0; e < nu; ++e) {
      uint64_t key;
      std::memcpy(&key, &uk[e], 8);
      U.push_back(E{key, (int32_t)ui[e]});
    }
    for (int e = 0; e < nl; ++e) {
      uint64_t key;
      std::memcpy(&key, &lk[e], 8);
      L.push_back(E{key, (int32_t)li[e]});
    }
  }
  auto lt = [](const E& a, const E& b) { return a.k < b.k || (a.k == b.k && a.i < b.i); };
  std::sort(U.begin(), U.end(), lt);
  std::sort(L.begin(), L.end(), lt);
  picks.clear();
  std::vector<int32_t> taken;
  auto is_taken = [&](int32_t i) { return std::find(taken.begin(), taken.end(), i) != taken.end(); };
  size_t ue = 0;
  for (; ue < U.size() && (int)picks.size() < need_u; ++ue) {
    picks.push_back(U[ue].i);
    taken.push_back(U[ue].i);
  }
  for (size_t e = 0; e < L.size() && (int)picks.size() < need; ++e)
    if (!is_taken(L[e].i)) {
      picks.push_back(L[e].i);
      taken.push_back(L[e].i);
    }
  for (; ue < U.size() && (int)picks.size() < need; ++ue)
    if (!is_taken(U[ue].i)) {
      picks.push_back(U[ue].i);
      taken.push_back(U[ue].i);
    }
  if (fmin == DBL_MAX || fmax == -DBL_MAX) return -DBL_MAX;  // a side is empty: converged
  return fmax - fmin;
}

static void fws_launch(Shard* S, double* out);

int shard_select(Shard* S, const double* all, int32_t* stop, double* fws_out) {
  GM_CUDA(cudaSetDevice(S->device));
  cudaStream_t st = S->st;
  const std::vector<int32_t> kept = retained(*S);
  const int need = S->np <= S->B ? 0 : S->B - (int)kept.size();
  std::vector<int32_t> picks;
  const double gap = shard_merge(all, S->world * S->chunks, 4 + 4 * S->need_max, need, need / 2, picks);
  S->gap = gap;
  if (!(gap >= S->eps)) {
    S->status = 1;
    *stop = 1;
    return GMPSVM_OK;
  }
  if (S->outer >= S->max_outer) {
    S->status = 2;
    *stop = 1;
    return GMPSVM_WARN_MAXITER;
  }
  *stop = 0;
  ++S->outer;
  // the new working set: retained (age order) + picks; the whole pair when it fits
  std::vector<int32_t> age;
  if (S->np <= S->B) {
    for (int32_t j = 0; j < (int32_t)S->np; ++j) age.push_back(j);
  } else {
    age = kept;
    age.insert(age.end(), picks.begin(), picks.end());
  }
  // row slots: retained rows keep theirs, new rows take free ones
  std::vector<int32_t> old_idx = S->ws, old_slot = S->slot_of;
  std::vector<int32_t> sorted = age;
  std::sort(sorted.begin(), sorted.end());
  const int wn = (int)sorted.size();
  std::vector<int32_t> slot(wn, -1);
  std::vector<uint8_t> used(S->B, 0);
  std::vector<int32_t> new_pos;  // positions (sorted order) whose rows must be computed
  for (int e = 0; e < wn; ++e) {
    const auto it = std::lower_bound(old_idx.begin(), old_idx.end(), sorted[e]);
    if (it != old_idx.end() && *it == sorted[e]) {
      slot[e] = old_slot[it - old_idx.begin()];
      used[slot[e]] = 1;
    }
  }
  int nxt = 0;
  for (int e = 0; e < wn; ++e)
    if (slot[e] < 0) {
      while (used[nxt]) ++nxt;
      slot[e] = nxt;
      used[nxt] = 1;
      new_pos.push_back(e);
    }
  S->ws_age = age;
  S->ws = sorted;
  S->slot_of = slot;
  GM_CUDA(cudaMemcpyAsync(S->d_ws.get(), sorted.data(), (size_t)wn * 4, cudaMemcpyHostToDevice, st));
  GM_CUDA(cudaMemcpyAsync(S->d_wsn.get(), &wn, 4, cudaMemcpyHostToDevice, st));
  const int ldat = (int)round_up(S->B, kTile);
  // kernel rows of the new members against the slice: gather their features, contract
  if (!new_pos.empty() && S->len > 0) {
    std::vector<int32_t> nidx, nslot;
    for (int e : new_pos) {
      nidx.push_back(sorted[e]);
      nslot.push_back(slot[e]);
    }
    DevBuf<int32_t> d_nidx(nidx.size(), st), d_nslot(nslot.size(), st);
    GM_CUDA(cudaMemcpyAsync(d_nidx.get(), nidx.data(), nidx.size() * 4, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(d_nslot.get(), nslot.data(), nslot.size() * 4, cudaMemcpyHostToDevice, st));
    GM_LAUNCH(shard_gather_kernel, dim3((unsigned)ceil_div(ldat, 128), 64), dim3(128), 0, st, S->XT.get(), S->ldx,
              S->nx.get(), d_nidx.get(), (int)nidx.size(), S->d_pad, S->AT.get(), (int64_t)ldat, S->na.get());
    launch_krow_rect(S->AT.get(), ldat, S->na.get(), (int64_t)nidx.size(), S->XT.get() + S->lo, S->ldx,
                     S->nx.get() + S->lo, S->len, S->d_pad, S->gamma, S->Rtmp.get(), S->ldr, st);
    GM_LAUNCH(shard_place_rows_kernel, dim3((unsigned)std::min<int64_t>(ceil_div(S->len, 256), 64), (unsigned)nidx.size()),
              dim3(256), 0, st, S->Rtmp.get(), S->ldr, d_nslot.get(), (int)nidx.size(), S->len, S->R.get(), S->ldr);
  }
  // K_ws,ws (B x B, row stride B) of the whole working set, sorted order: identical on every rank
  GM_LAUNCH(shard_gather_kernel, dim3((unsigned)ceil_div(ldat, 128), 64), dim3(128), 0, st, S->XT.get(), S->ldx,
            S->nx.get(), S->d_ws.get(), wn, S->d_pad, S->AT.get(), (int64_t)ldat, S->na.get());
  launch_krow_rect(S->AT.get(), ldat, S->na.get(), wn, S->AT.get(), ldat, S->na.get(), wn, S->d_pad, S->gamma,
                   S->Kws.get(), S->tile_ld(), st);
  GM_CUDA(cudaMemcpyAsync(S->d_slot.get(), slot.data(), (size_t)wn * 4, cudaMemcpyHostToDevice, st));
  if (fws_out) fws_launch(S, fws_out);  // this rank's f of the new working set, same round trip
  GM_CUDA(cudaStreamSynchronize(st));
  return GMPSVM_OK;
}

static void fws_launch(Shard* S, double* out) {
  const int wn = (int)S->ws.size();
  GM_LAUNCH(shard_fws_kernel, dim3((unsigned)ceil_div(std::max(wn, 1), 256)), dim3(256), 0, S->st, S->f.get(),
            S->d_ws.get(), wn, S->lo, S->hi, S->fws.get());
  std::memset(out, 0, (size_t)S->B * 8);
  if (wn) GM_CUDA(cudaMemcpyAsync(out, S->fws.get(), (size_t)wn * 8, cudaMemcpyDeviceToHost, S->st));
}

void shard_fws(Shard* S, double* out) {
  GM_CUDA(cudaSetDevice(S->device));
  fws_launch(S, out);
  GM_CUDA(cudaStreamSynchronize(S->st));
}

void shard_step(Shard* S, const double* fws_sum, double* cand_out) {
  GM_CUDA(cudaSetDevice(S->device));
  cudaStream_t st = S->st;
  const int wn = (int)S->ws.size();
  GM_CUDA(cudaMemcpyAsync(S->fws.get(), fws_sum, (size_t)wn * 8, cudaMemcpyHostToDevice, st));
  GM_LAUNCH(shard_scatter_fws_kernel, dim3((unsigned)ceil_div(std::max(wn, 1), 256)), dim3(256), 0, st, S->fws.get(),
            S->d_ws.get(), wn, S->f.get());
  SolverArgs a = shard_args(*S);
  // the same local solve on every rank (alpha stays replicated)
  if (S->warp_smo()) {
    GM_LAUNCH(shard_state_kernel, dim3((unsigned)ceil_div(std::max(wn, 1), 256)), dim3(256), 0, st, S->alpha.get(),
              S->fws.get(), S->d_ws.get(), wn, S->Kws.get(), (size_t)S->B * S->tile_ld(), S->B);
    launch_ws_smo(a, 1, st);
  } else {
    launch_local_smo(a, 1, st);
  }
  if (S->len > 0) {
    GM_LAUNCH(shard_nz_kernel, dim3(1), dim3(32), 0, st, S->dcoef.get(), S->d_slot.get(), wn, S->nzc.get(), S->nzs.get(),
              S->nzn.get());
    GM_LAUNCH(shard_fupdate_kernel, dim3((unsigned)ceil_div(S->len, 256)), dim3(256), 0, st, S->nzc.get(), S->nzs.get(),
              S->nzn.get(), S->R.get(), S->ldr, S->lo, S->len, S->f.get());
  }
  if (cand_out) cand_launch(S, cand_out);  // the next iteration's candidates, same round trip
  GM_CUDA(cudaStreamSynchronize(st));
}

void shard_slice(const Shard* S, int64_t* lo, int64_t* hi, int64_t* np, int32_t* ws_size) {
  if (lo) *lo = S->lo;
  if (hi) *hi = S->hi;
  if (np) *np = S->np;
  if (ws_size) *ws_size = S->B;
}

void shard_f(Shard* S, double* out) {
  GM_CUDA(cudaSetDevice(S->device));
  if (S->len) GM_CUDA(cudaMemcpy(out, S->f.get() + S->lo, (size_t)S->len * 8, cudaMemcpyDeviceToHost));
}

int shard_finish(Shard* S, const double* f_full, double* alpha_out, double* b, double* A, double* Bsig, int32_t* status,
                 int64_t* outer, int64_t* inner) {
  GM_CUDA(cudaSetDevice(S->device));
  cudaStream_t st = S->st;
  GM_CUDA(cudaMemcpyAsync(S->f.get(), f_full, (size_t)S->np * 8, cudaMemcpyHostToDevice, st));
  SolverArgs a = shard_args(*S);
  launch_finalize(a, 1, st);  // bias (R7) and in-sample decision values (Eq 3 + 11)
  launch_sigmoid_fit(a, 1, st);
  int32_t sig = 0;
  int64_t in = 0;
  GM_CUDA(cudaMemcpyAsync(alpha_out, S->alpha.get(), (size_t)S->np * 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaMemcpyAsync(b, S->bb.get(), 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaMemcpyAsync(A, S->AA.get(), 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaMemcpyAsync(Bsig, S->BB.get(), 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaMemcpyAsync(&sig, S->d_sig.get(), 4, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaMemcpyAsync(&in, S->d_inner64.get(), 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaStreamSynchronize(st));
  // status word as in gmpsvm_model_pair: solver status (0 ok, 2 outer cap) | sigmoid status << 8
  if (status) *status = (S->status == 2 ? 2 : 0) | (sig << 8);
  if (outer) *outer = S->outer;
  if (inner) *inner = in;
  return (S->status == 2 || sig == 1) ? GMPSVM_WARN_MAXITER : GMPSVM_OK;
}

}  // namespace gmpsvm
