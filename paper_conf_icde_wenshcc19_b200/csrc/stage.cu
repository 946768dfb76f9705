// stage.cu -- a1: staging / class grouping (Alg 2 line 3 "getIns", L342).
//
// A stable counting sort of the instances by class on the device, so that pair (s,t) is
// two contiguous class blocks of one class-sorted copy of X (kernel rows shared across
// pairs, L313-L325).  The sorted copy is stored feature-major (XT[c][j]) and zero-padded
// to (d_pad x n_pad) for the tile contraction; squared norms are accumulated in FP64.
#include <cstdlib>
#include <string>

#include "kernels.h"

namespace gmpsvm {

// Per-block class histogram of 1024 labels; slot k counts invalid labels.
__global__ void label_block_count_kernel(const int32_t* __restrict__ y, int64_t n, int k, int32_t* blk_counts) {
  extern __shared__ int32_t cnt[];
  for (int c = threadIdx.x; c <= k; c += blockDim.x) cnt[c] = 0;
  __syncthreads();
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) {
    const int32_t c = y[i];
    atomicAdd(&cnt[(c >= 0 && c < k) ? c : k], 1);
  }
  __syncthreads();
  for (int c = threadIdx.x; c <= k; c += blockDim.x) blk_counts[(int64_t)blockIdx.x * (k + 1) + c] = cnt[c];
}

// Exclusive scan of the per-block histograms per class; class sizes and class offsets.
__global__ void label_scan_kernel(const int32_t* __restrict__ blk_counts, int nb, int k, int32_t* blk_off,
                                  int64_t* class_count, int64_t* class_off) {
  for (int c = threadIdx.x; c <= k; c += blockDim.x) {
    int64_t run = 0;
    for (int b = 0; b < nb; ++b) {
      if (c < k) blk_off[(int64_t)b * k + c] = (int32_t)run;
      run += blk_counts[(int64_t)b * (k + 1) + c];
    }
    class_count[c] = run;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int64_t run = 0;
    for (int c = 0; c < k; ++c) {
      class_off[c] = run;
      run += class_count[c];
    }
    class_off[k] = run;
  }
}

// Stable position of every instance: class_off[c] + (# earlier instances of class c).
// Labels are validated before this launch.  perm[pos] = original index.
__global__ void __launch_bounds__(1024) label_rank_kernel(const int32_t* __restrict__ y, int64_t n, int k,
                                                          const int32_t* __restrict__ blk_off,
                                                          const int64_t* __restrict__ class_off, int64_t* perm) {
  extern __shared__ int32_t wcnt[];  // [32][k]
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int i = threadIdx.x; i < 32 * k; i += blockDim.x) wcnt[i] = 0;
  __syncthreads();
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int c = (i < n) ? y[i] : -1;
  const unsigned mask = __match_any_sync(0xffffffffu, c);
  const int rank = __popc(mask & ((1u << lane) - 1u));
  if (c >= 0 && rank == 0) wcnt[warp * k + c] = __popc(mask);
  __syncthreads();
  if (c >= 0) {
    int before = 0;
    for (int w = 0; w < warp; ++w) before += wcnt[w * k + c];
    const int64_t pos = class_off[c] + blk_off[(int64_t)blockIdx.x * k + c] + before + rank;
    perm[pos] = i;
  }
}

// XT[c][j] = X[src(j)][c] for c < d, j < n; zero in the padding.  src(j) = perm ? perm[j] : j.
__global__ void gather_transpose_kernel(const float* __restrict__ X, int64_t n, int d, const int64_t* __restrict__ perm,
                                        float* __restrict__ XT, int64_t ldx, int d_pad, int64_t n_pad) {
  __shared__ float tile[32][33];
  const int64_t j0 = (int64_t)blockIdx.x * 32;
  const int c0 = blockIdx.y * 32;
  const int tx = threadIdx.x, ty = threadIdx.y;
  for (int jj = ty; jj < 32; jj += 8) {
    const int64_t j = j0 + jj;
    const int c = c0 + tx;
    float v = 0.f;
    if (j < n && c < d) {
      const int64_t src = perm ? perm[j] : j;  // src < 0: padding slot
      if (src >= 0) v = X[src * d + c];
    }
    tile[jj][tx] = v;
  }
  __syncthreads();
  for (int cc = ty; cc < 32; cc += 8) {
    const int c = c0 + cc;
    const int64_t j = j0 + tx;
    if (c < d_pad && j < n_pad) XT[(int64_t)c * ldx + j] = tile[tx][cc];
  }
}

// norms[j] = ||X[src(j)]||^2 accumulated in FP64, rounded once to FP32; 0 in the padding.
// Sets *bad if a row holds a non-finite value (input validation, EINVAL).
__global__ void row_norms_kernel(const float* __restrict__ X, int64_t n, int d, const int64_t* __restrict__ perm,
                                 float* __restrict__ norms, int64_t n_pad, int32_t* bad) {
  const int64_t j = (int64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (j >= n_pad) return;
  double s = 0.0;
  const int64_t src = (j < n) ? (perm ? perm[j] : j) : -1;
  if (src >= 0) {
    const float* x = X + src * d;
    for (int c = lane; c < d; c += 32) {
      const double v = x[c];
      s = fma(v, v, s);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) {
    norms[j] = (float)s;
    if (bad && !isfinite(s)) atomicExch(bad, 1);
  }
}

// Gather rows: dst[r][:] = X[idx[r]][:]  (SV rows of the model, original feature layout)
__global__ void gather_rows_kernel(const float* __restrict__ X, int d, const int64_t* __restrict__ idx, int64_t nr,
                                   float* __restrict__ dst) {
  const int64_t r = blockIdx.x;
  if (r >= nr) return;
  const float* s = X + idx[r] * d;
  float* o = dst + r * d;
  for (int c = threadIdx.x; c < d; c += blockDim.x) o[c] = s[c];
}

void launch_class_sort(const int32_t* y, int64_t n, int k, int32_t* blk_counts, int32_t* blk_off,
                       int64_t* class_count, int64_t* class_off, cudaStream_t st) {
  const int nb = (int)ceil_div(n, 1024);
  GM_LAUNCH(label_block_count_kernel, dim3(nb), dim3(1024), (size_t)(k + 1) * sizeof(int32_t), st, y, n, k,
            blk_counts);
  GM_LAUNCH(label_scan_kernel, dim3(1), dim3(std::min(1024, k + 1)), 0, st, blk_counts, nb, k, blk_off, class_count,
            class_off);
}

void launch_class_rank(const int32_t* y, int64_t n, int k, const int32_t* blk_off, const int64_t* class_off,
                       int64_t* perm, cudaStream_t st) {
  const int nb = (int)ceil_div(n, 1024);
  GM_LAUNCH(label_rank_kernel, dim3(nb), dim3(1024), (size_t)32 * k * sizeof(int32_t), st, y, n, k, blk_off,
            class_off, perm);
}

void launch_stage_features(const float* X, int64_t n, int d, const int64_t* perm, float* XT, int64_t ldx, int d_pad,
                           int64_t n_pad, float* norms, int32_t* bad, cudaStream_t st) {
  GM_LAUNCH(gather_transpose_kernel, dim3((unsigned)ceil_div(n_pad, 32), (unsigned)ceil_div(d_pad, 32)), dim3(32, 8), 0,
            st, X, n, d, perm, XT, ldx, d_pad, n_pad);
  GM_LAUNCH(row_norms_kernel, dim3((unsigned)ceil_div(n_pad, 8)), dim3(256), 0, st, X, n, d, perm, norms, n_pad, bad);
}

void launch_row_norms(const float* X, int64_t n, int d, const int64_t* perm, float* norms, int64_t n_pad, int32_t* bad,
                      cudaStream_t st) {
  GM_LAUNCH(row_norms_kernel, dim3((unsigned)ceil_div(n_pad, 8)), dim3(256), 0, st, X, n, d, perm, norms, n_pad, bad);
}

bool krow_use_tc() {
  static const bool simt = getenv("GMPSVM_KROW") && std::string(getenv("GMPSVM_KROW")) == "simt";
  return !simt;
}

void launch_gather_rows(const float* X, int d, const int64_t* idx, int64_t nr, float* dst, cudaStream_t st) {
  if (nr <= 0) return;
  GM_LAUNCH(gather_rows_kernel, dim3((unsigned)nr), dim3(128), 0, st, X, d, idx, nr, dst);
}

// a9: LibSVM-style coefficients of the SV slots, coef[slot][col] = y * alpha of the SV in each of
// the k - 1 pairs of its class, read from the training call's device
// alpha (aoff[p] = offset of pair p's alpha, -1: untrained -> 0).  One thread per slot.
__global__ void build_coef_kernel(const double* __restrict__ alpha, const int64_t* __restrict__ aoff,
                                  const int64_t* __restrict__ slot_g, const int64_t* __restrict__ off,
                                  const int64_t* __restrict__ cc, int k, int64_t nsv_pad, int km1_pad,
                                  float* __restrict__ coef, double* __restrict__ coef64) {
  const int64_t slot = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (slot >= nsv_pad) return;
  float* out = coef + slot * km1_pad;
  double* out64 = coef64 ? coef64 + slot * km1_pad : nullptr;
  for (int col = 0; col < km1_pad; ++col) {
    out[col] = 0.f;
    if (out64) out64[col] = 0.0;
  }
  const int64_t g = slot_g[slot];
  if (g < 0) return;  // padding slot
  int c = 0;
  while (c + 1 < k && off[c + 1] <= g) ++c;
  for (int u = 0; u < k; ++u) {
    if (u == c) continue;
    const int s = c < u ? c : u, t = c < u ? u : c;
    const int p = pair_index(s, t, k);
    const int64_t j = (c == s) ? (g - off[s]) : (cc[s] + (g - off[t]));
    const double a = aoff[p] >= 0 ? alpha[aoff[p] + j] : 0.0;
    out[u < c ? u : u - 1] = (float)((c == s) ? a : -a);
    if (out64) out64[u < c ? u : u - 1] = (c == s) ? a : -a;
  }
}

// sum_j |alpha_j| per trained pair (conditioning of the decision values)
__global__ void alpha_abs_sum_kernel(const double* __restrict__ alpha, const int64_t* __restrict__ aoff,
                                     const int64_t* __restrict__ np, double* __restrict__ out) {
  const int p = blockIdx.x;
  __shared__ double red[32];
  double s = 0.0;
  if (aoff[p] >= 0)
    for (int64_t j = threadIdx.x; j < np[p]; j += blockDim.x) s += fabs(alpha[aoff[p] + j]);
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += red[w];
    out[p] = t;
  }
}

void launch_alpha_abs_sum(const double* alpha, const int64_t* aoff, const int64_t* np, int P, double* out,
                          cudaStream_t st) {
  GM_LAUNCH(alpha_abs_sum_kernel, dim3((unsigned)P), dim3(256), 0, st, alpha, aoff, np, out);
}

void launch_build_coef(const double* alpha, const int64_t* aoff, const int64_t* slot_g, const int64_t* off,
                       const int64_t* cc, int k, int64_t nsv_pad, int km1_pad, float* coef, double* coef64,
                       cudaStream_t st) {
  GM_LAUNCH(build_coef_kernel, dim3((unsigned)ceil_div(nsv_pad, 256)), dim3(256), 0, st, alpha, aoff, slot_g, off, cc, k,
            nsv_pad, km1_pad, coef, coef64);
}

// CSR input (the paper's / LibSVM's sparse format, NEXT-3): row i's nonzeros
// values[indptr[i] .. indptr[i+1]) at columns indices[.] scattered into a zeroed dense row-major
// n x d matrix; one warp per row.  Out-of-range columns set *bad.
__global__ void csr_densify_kernel(const int64_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                   const float* __restrict__ values, int64_t n, int d, float* __restrict__ X,
                                   int32_t* __restrict__ bad) {
  const int64_t row = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= n) return;
  const int64_t b = indptr[row], e = indptr[row + 1];
  for (int64_t j = b + lane; j < e; j += 32) {
    const int32_t c = indices[j];
    if (c < 0 || c >= d) {
      *bad = 1;
      continue;
    }
    X[row * d + c] = values[j];
  }
}

void launch_csr_densify(const int64_t* indptr, const int32_t* indices, const float* values, int64_t n, int d, float* X,
                        int32_t* bad, cudaStream_t st) {
  GM_CUDA(cudaMemsetAsync(X, 0, (size_t)n * d * sizeof(float), st));
  if (n > 0)
    GM_LAUNCH(csr_densify_kernel, dim3((unsigned)ceil_div(n, 8)), dim3(256), 0, st, indptr, indices, values, n, d, X, bad);
}

}  // namespace gmpsvm
