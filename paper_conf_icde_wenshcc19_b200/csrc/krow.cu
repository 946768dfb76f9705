// krow.cu -- a2: the kernel-value contraction (K1, RBF L75).
//
//   K[i][j] = exp(-gamma * max(0, ||x_i||^2 + ||x_j||^2 - 2 x_i . x_j)),   K[i][i] = 1
//
// FULL_K regime: one launch computes the whole class-sorted n x n matrix, so every kernel
// row is computed once and shared by all k-1 pairs that contain its class (the paper's
// kernel-value sharing, L313-L325, taken to its limit because 180 GB of HBM holds it:
// MNIST-shaped n = 60k -> 14.4 GB).  Symmetry: only tiles (bi <= bj) are computed; each
// off-diagonal tile is also stored transposed.  FP32 SIMT.
#include "gemm_simt.cuh"
#include "kernels.h"

namespace gmpsvm {

// Upper-triangular tile enumeration: L -> (bi, bj), bi <= bj, row-major over the triangle.
__device__ __forceinline__ void tri_tile(int64_t L, int T, int& bi, int& bj) {
  // rows before bi: S(bi) = bi*T - bi*(bi-1)/2
  double tt = 2.0 * T + 1.0;
  int r = (int)floor((tt - sqrt(tt * tt - 8.0 * (double)L)) * 0.5);
  if (r < 0) r = 0;
  if (r > T - 1) r = T - 1;
  auto S = [&](int b) { return (int64_t)b * T - (int64_t)b * (b - 1) / 2; };
  while (r > 0 && S(r) > L) --r;
  while (r + 1 < T && S(r + 1) <= L) ++r;
  bi = r;
  bj = r + (int)(L - S(r));
}

template <bool SYM>
__global__ void __launch_bounds__(kGemmThreads, 2)
    krow_contract_kernel(const float* __restrict__ AT, int64_t lda, const float* __restrict__ na, int64_t n,
                         const float* __restrict__ BT, int64_t ldb, const float* __restrict__ nb, int64_t m,
                         int kdim, float scale /* -gamma*log2(e) */, float* __restrict__ K, int64_t ldk,
                         int T /* tiles per side (SYM) or row tiles */) {
  __shared__ __align__(16) GemmSmem sm;
  int bi, bj;
  if (SYM) {
    tri_tile((int64_t)blockIdx.x, T, bi, bj);
  } else {
    bi = blockIdx.y;
    bj = blockIdx.x;
  }
  const int64_t r0 = (int64_t)bi * kTile, c0 = (int64_t)bj * kTile;
  float acc[8][8];
  gemm_tile_128(AT, lda, r0, BT, ldb, c0, kdim, sm, acc);

  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  float nr[8], nc[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) nr[i] = na[r0 + tile_row(ty, i)];  // norms are zero-padded to the tile
#pragma unroll
  for (int j = 0; j < 8; ++j) nc[j] = nb[c0 + tile_col(tx, j)];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      float d2 = fmaf(-2.f, acc[i][j], nr[i] + nc[j]);
      acc[i][j] = fast_exp2(fmaxf(d2, 0.f) * scale);
    }
  if (SYM && bi == bj) {
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int j = 0; j < 8; ++j)
        if (tile_row(ty, i) == tile_col(tx, j)) acc[i][j] = 1.f;
  }
  // direct store K[r][c]: two float4 per row
  const bool vec_ok = (ldk % 4) == 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int64_t r = r0 + tile_row(ty, i);
    if (r >= n) continue;
    float* dst = K + r * ldk;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int64_t c = c0 + h * 64 + tx * 4;
      const float4 v = make_float4(acc[i][h * 4 + 0], acc[i][h * 4 + 1], acc[i][h * 4 + 2], acc[i][h * 4 + 3]);
      if (vec_ok && c + 3 < m) {
        *reinterpret_cast<float4*>(dst + c) = v;
      } else {
        if (c + 0 < m) dst[c + 0] = v.x;
        if (c + 1 < m) dst[c + 1] = v.y;
        if (c + 2 < m) dst[c + 2] = v.z;
        if (c + 3 < m) dst[c + 3] = v.w;
      }
    }
  }
  if (SYM && bi != bj) {
    // transposed store K[c][r]: for each owned column, 4 consecutive rows per half
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int64_t c = c0 + tile_col(tx, j);
      if (c >= n) continue;
      float* dst = K + c * ldk;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int64_t r = r0 + h * 64 + ty * 4;
        const float4 v = make_float4(acc[h * 4 + 0][j], acc[h * 4 + 1][j], acc[h * 4 + 2][j], acc[h * 4 + 3][j]);
        if (vec_ok && r + 3 < n) {
          *reinterpret_cast<float4*>(dst + r) = v;
        } else {
          if (r + 0 < n) dst[r + 0] = v.x;
          if (r + 1 < n) dst[r + 1] = v.y;
          if (r + 2 < n) dst[r + 2] = v.z;
          if (r + 3 < n) dst[r + 3] = v.w;
        }
      }
    }
  }
}

void launch_krow_full_sym(const float* XT, int64_t ldx, const float* norms, int64_t n, int kdim, double gamma,
                          float* K, int64_t ldk, cudaStream_t st) {
  const int T = (int)ceil_div(n, kTile);
  const int64_t tiles = (int64_t)T * (T + 1) / 2;
  const float scale = (float)(-gamma * 1.4426950408889634);
  GM_LAUNCH(krow_contract_kernel<true>, dim3((unsigned)tiles), dim3(kGemmThreads), 0, st, XT, ldx, norms, n, XT, ldx,
            norms, n, kdim, scale, K, ldk, T);
}

void launch_krow_rect(const float* AT, int64_t lda, const float* na, int64_t n, const float* BT, int64_t ldb,
                      const float* nb, int64_t m, int kdim, double gamma, float* K, int64_t ldk, cudaStream_t st) {
  const int Tr = (int)ceil_div(n, kTile), Tc = (int)ceil_div(m, kTile);
  const float scale = (float)(-gamma * 1.4426950408889634);
  GM_LAUNCH(krow_contract_kernel<false>, dim3(Tc, Tr), dim3(kGemmThreads), 0, st, AT, lda, na, n, BT, ldb, nb, m, kdim,
            scale, K, ldk, Tr);
}

}  // namespace gmpsvm
