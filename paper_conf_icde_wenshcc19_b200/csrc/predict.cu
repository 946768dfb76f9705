// predict.cu -- a10..a12: probability estimation.
//
//   dec_contract  a10  shared-SV decision values (Eq 11 with support-vector and kernel-value
//                      sharing, L333, L363): one CTA = one 128-row test tile x a run of
//                      class-pure 128-SV tiles of one class c.  dot -> exp -> x coef tile:
//                      each SV of class c contributes to exactly the k-1 pairs (c, u), so the
//                      CTA accumulates a 128 x (k-1) block in shared memory.  K never hits HBM.
//   dec_reduce         fixed-order FP64 sum of the per-run partials + b (deterministic).
//   couple        a11  r_st = clamp(1/(1+exp(A dec + B)), 1e-7, 1-1e-7) (Eq 12, reading R15)
//                 a12  one warp per test instance: bordered (k+1)x(k+2) system of Eq 14/15
//                      solved by Gaussian elimination with partial pivoting in FP64 (L206, R13).
#include <cfloat>

#include "gemm_simt.cuh"
#include "kernels.h"

namespace gmpsvm {

// dynamic smem: GemmSmem | coefS[128][km1_pad] | decS[128][km1_pad]
__global__ void __launch_bounds__(kGemmThreads, 2)
    dec_contract_kernel(const float* __restrict__ XtT, int64_t ldt, const float* __restrict__ nt, int64_t m,
                        int64_t m_pad, const float* __restrict__ SvT, int64_t lds, const float* __restrict__ nsv,
                        const float* __restrict__ coef, int km1, int km1_pad, const DecItem* __restrict__ items,
                        int kdim, float scale, float* __restrict__ part) {
  extern __shared__ __align__(16) unsigned char dsm[];
  GemmSmem& sm = *reinterpret_cast<GemmSmem*>(dsm);
  float* coefS = reinterpret_cast<float*>(dsm + sizeof(GemmSmem));
  float* decS = coefS + kTile * km1_pad;
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int64_t r0 = (int64_t)blockIdx.x * kTile;
  const DecItem it = items[blockIdx.y];
  for (int i = tid; i < kTile * km1_pad; i += kGemmThreads) decS[i] = 0.f;
  float nr[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) nr[i] = nt[r0 + tile_row(ty, i)];
  for (int tile = it.tile_begin; tile < it.tile_end; ++tile) {
    const int64_t c0 = (int64_t)tile * kTile;
    __syncthreads();  // previous tile done with coefS / decS updates
    for (int i = tid; i < kTile * km1_pad; i += kGemmThreads) coefS[i] = coef[c0 * km1_pad + i];
    float acc[8][8];
    gemm_tile_128(XtT, ldt, r0, SvT, lds, c0, kdim, sm, acc);
    float nc[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) nc[j] = nsv[c0 + tile_col(tx, j)];
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const float d2 = fmaf(-2.f, acc[i][j], nr[i] + nc[j]);
        acc[i][j] = fast_exp2(fmaxf(d2, 0.f) * scale);
      }
    __syncthreads();  // coefS visible
    // contraction with the coefficient tile, 4 pair-columns at a time
    for (int u0 = 0; u0 < km1; u0 += 4) {
      float p[8][4];
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int uu = 0; uu < 4; ++uu) p[i][uu] = 0.f;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const float4 cv = *reinterpret_cast<const float4*>(&coefS[tile_col(tx, j) * km1_pad + u0]);
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          p[i][0] = fmaf(acc[i][j], cv.x, p[i][0]);
          p[i][1] = fmaf(acc[i][j], cv.y, p[i][1]);
          p[i][2] = fmaf(acc[i][j], cv.z, p[i][2]);
          p[i][3] = fmaf(acc[i][j], cv.w, p[i][3]);
        }
      }
      // sum over the 16 threads (tx) sharing these rows: lanes 0-15 / 16-31 of the warp
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int uu = 0; uu < 4; ++uu) {
          float v = p[i][uu];
          v += __shfl_xor_sync(0xffffffffu, v, 1);
          v += __shfl_xor_sync(0xffffffffu, v, 2);
          v += __shfl_xor_sync(0xffffffffu, v, 4);
          v += __shfl_xor_sync(0xffffffffu, v, 8);
          p[i][uu] = v;
        }
      if (tx == ((u0 >> 2) & 15)) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          float* d = &decS[tile_row(ty, i) * km1_pad + u0];
          d[0] += p[i][0];
          d[1] += p[i][1];
          d[2] += p[i][2];
          d[3] += p[i][3];
        }
      }
    }
  }
  __syncthreads();
  float* out = part + ((int64_t)blockIdx.y * m_pad + r0) * km1_pad;
  for (int i = tid; i < kTile * km1_pad; i += kGemmThreads) out[i] = decS[i];
}

// dec[i][p] = b[p] + sum_{runs of class s} part[.][i][col_s(t)] + sum_{runs of class t} part[.][i][col_t(s)]
__global__ void dec_reduce_kernel(const float* __restrict__ part, int64_t m, int64_t m_pad, int k, int km1_pad,
                                  const int32_t* __restrict__ item_begin, const int32_t* __restrict__ item_end,
                                  const double* __restrict__ b, double* __restrict__ dec) {
  const int P = k * (k - 1) / 2;
  const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= m * P) return;
  const int64_t i = gid / P;
  const int p = (int)(gid % P);
  // pair p -> (s, t)
  int s = 0, rem = p;
  while (rem >= k - 1 - s) {
    rem -= k - 1 - s;
    ++s;
  }
  const int t = s + 1 + rem;
  double acc = b[p];
  const int cs = t - 1;  // column of partner t for an SV of class s (t > s)
  const int ct = s;      // column of partner s for an SV of class t (s < t)
  for (int q = item_begin[s]; q < item_end[s]; ++q) acc += (double)part[((int64_t)q * m_pad + i) * km1_pad + cs];
  for (int q = item_begin[t]; q < item_end[t]; ++q) acc += (double)part[((int64_t)q * m_pad + i) * km1_pad + ct];
  dec[gid] = acc;
}

// One warp per test instance; M is (k+1) x (k+2) (bordered Q | rhs) in shared memory.
constexpr int kCoupleWarps = 4;

__global__ void __launch_bounds__(32 * kCoupleWarps) couple_kernel(const double* __restrict__ dec, int64_t m, int k,
                                                                   const double* __restrict__ A,
                                                                   const double* __restrict__ Bv,
                                                                   double* __restrict__ prob) {
  extern __shared__ double csm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t inst = (int64_t)blockIdx.x * kCoupleWarps + warp;
  if (inst >= m) return;
  const int P = k * (k - 1) / 2, n = k + 1, ld = k + 2;
  double* r = csm + (int64_t)warp * ((int64_t)k * k + (int64_t)n * ld);
  double* M = r + k * k;
  // Eq 12 + clamp: r_st for each pair, r_ts = 1 - r_st
  for (int p = lane; p < P; p += 32) {
    int s = 0, rem = p;
    while (rem >= k - 1 - s) {
      rem -= k - 1 - s;
      ++s;
    }
    const int t = s + 1 + rem;
    const double z = dec[inst * P + p] * A[p] + Bv[p];
    double rst = z >= 0.0 ? exp(-z) / (1.0 + exp(-z)) : 1.0 / (1.0 + exp(z));
    rst = fmin(fmax(rst, 1e-7), 1.0 - 1e-7);
    r[s * k + t] = rst;
    r[t * k + s] = 1.0 - rst;
  }
  __syncwarp();
  for (int attempt = 0; attempt < 2; ++attempt) {
    // bordered system [Q e; e^T 0 | rhs]: Q_ss = sum_{u != s} r_us^2, Q_st = -r_st r_ts (Eq 15)
    for (int e = lane; e < n * ld; e += 32) {
      const int row = e / ld, col = e % ld;
      double val = 0.0;
      if (row < k && col < k) {
        if (row == col) {
          for (int u = 0; u < k; ++u)
            if (u != row) val += r[u * k + row] * r[u * k + row];
          if (attempt) val += 1e-12;
        } else {
          val = -r[row * k + col] * r[col * k + row];
        }
      } else if (row < k && col == k) {
        val = 1.0;
      } else if (row == k && col < k) {
        val = 1.0;
      } else if (row == k && col == k + 1) {
        val = 1.0;  // rhs = [0 ... 0 1]
      }
      M[row * ld + col] = val;
    }
    __syncwarp();
    bool singular = false;
    for (int c = 0; c < n && !singular; ++c) {
      // partial pivot: first row with the largest |M[r][c]|, r >= c
      double best = -1.0;
      int piv = n;
      for (int rr = c + lane; rr < n; rr += 32) {
        const double v = fabs(M[rr * ld + c]);
        if (v > best) {
          best = v;
          piv = rr;
        }
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        const double ob = __shfl_xor_sync(0xffffffffu, best, o);
        const int op = __shfl_xor_sync(0xffffffffu, piv, o);
        if (ob > best || (ob == best && op < piv)) {
          best = ob;
          piv = op;
        }
      }
      if (!(best > 0.0)) {
        singular = true;
        break;
      }
      if (piv != c)
        for (int j = lane; j < ld; j += 32) {
          const double tmp = M[c * ld + j];
          M[c * ld + j] = M[piv * ld + j];
          M[piv * ld + j] = tmp;
        }
      __syncwarp();
      const double diag = M[c * ld + c];
      for (int rr = c + 1; rr < n; ++rr) {
        const double fac = M[rr * ld + c] / diag;
        __syncwarp();
        if (fac != 0.0)
          for (int j = c + lane; j < ld; j += 32) M[rr * ld + j] -= fac * M[c * ld + j];
        __syncwarp();
      }
    }
    if (singular) continue;
    if (lane == 0) {  // back substitution (rhs column k+1)
      for (int rr = n - 1; rr >= 0; --rr) {
        double s = M[rr * ld + k + 1];
        for (int j = rr + 1; j < n; ++j) s -= M[rr * ld + j] * M[j * ld + k + 1];
        M[rr * ld + k + 1] = s / M[rr * ld + rr];
      }
    }
    __syncwarp();
    for (int s = lane; s < k; s += 32) prob[inst * k + s] = M[s * ld + k + 1];
    return;
  }
  for (int s = lane; s < k; s += 32) prob[inst * k + s] = nan("");
}

void launch_dec_contract(const float* XtT, int64_t ldt, const float* nt, int64_t m, int64_t m_pad, const float* SvT,
                         int64_t lds, const float* nsv, const float* coef, int km1, int km1_pad, const DecItem* items,
                         int n_items, int kdim, double gamma, float* part, cudaStream_t st) {
  const size_t smem = sizeof(GemmSmem) + 2 * (size_t)kTile * km1_pad * sizeof(float);
  if (smem > 48 * 1024) set_max_dyn_smem(dec_contract_kernel, smem);
  const float scale = (float)(-gamma * 1.4426950408889634);
  GM_LAUNCH(dec_contract_kernel, dim3((unsigned)(m_pad / kTile), (unsigned)n_items), dim3(kGemmThreads), smem, st, XtT,
            ldt, nt, m, m_pad, SvT, lds, nsv, coef, km1, km1_pad, items, kdim, scale, part);
}

// ------------------------------------------------------------------------------------------
// a10 in FP64 (ill-conditioned models): when sum_j |coef_j| K_ij is so large that
// FP32 kernel values alone would move probabilities beyond the 1e-4 contract (e.g. C = 1000),
// the decision values are computed in FP64 end to end -- FP64 norms and dot products of the
// FP32 inputs, exp in FP64, FP64 coefficient contraction -- the oracle's arithmetic up to
// summation order.  Same work decomposition as dec_contract (one CTA = a test tile x a class-pure
// run of SV tiles); FP64 tiles of 64 x 64, thread (ty, tx) owns rows 4 ty.. and columns 4 tx...
constexpr int kF64Tile = 64, kF64BK = 16;

__global__ void __launch_bounds__(256) dec_f64_kernel(const float* __restrict__ XtT, int64_t ldt,
                                                      const double* __restrict__ nt64, const float* __restrict__ SvT,
                                                      int64_t lds, const double* __restrict__ nsv64,
                                                      const double* __restrict__ coef64, int km1, int km1_pad,
                                                      const DecItem* __restrict__ items, int kdim, double gamma,
                                                      int64_t m_pad, double* __restrict__ part, int ktype,
                                                      double coef0, int degree) {
  extern __shared__ __align__(16) unsigned char dsm[];
  double* as = reinterpret_cast<double*>(dsm);        // [kF64BK][64]
  double* bs = as + kF64BK * kF64Tile;                // [kF64BK][64]
  double* coefS = bs + kF64BK * kF64Tile;             // [64][km1_pad]
  double* decS = coefS + kF64Tile * km1_pad;          // [64][km1_pad]
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int64_t r0 = (int64_t)blockIdx.x * kF64Tile;
  const DecItem it = items[blockIdx.y];
  for (int i = tid; i < kF64Tile * km1_pad; i += 256) decS[i] = 0.0;
  double nr[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) nr[i] = nt64[r0 + ty * 4 + i];
  const int64_t c_begin = (int64_t)it.tile_begin * kTile, c_end = (int64_t)it.tile_end * kTile;
  for (int64_t c0 = c_begin; c0 < c_end; c0 += kF64Tile) {
    double acc[4][4] = {};
    for (int k0 = 0; k0 < kdim; k0 += kF64BK) {
      __syncthreads();  // previous chunk / tile done with as, bs, coefS
      for (int e = tid; e < kF64BK * kF64Tile; e += 256) {
        const int kk = e / kF64Tile, c = e % kF64Tile;
        as[e] = (double)XtT[(int64_t)(k0 + kk) * ldt + r0 + c];
        bs[e] = (double)SvT[(int64_t)(k0 + kk) * lds + c0 + c];
      }
      __syncthreads();
#pragma unroll
      for (int kk = 0; kk < kF64BK; ++kk) {
        double a[4], b[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) a[i] = as[kk * kF64Tile + ty * 4 + i];
#pragma unroll
        for (int j = 0; j < 4; ++j) b[j] = bs[kk * kF64Tile + tx * 4 + j];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) acc[i][j] = fma(a[i], b[j], acc[i][j]);
      }
    }
    for (int e = tid; e < kF64Tile * km1_pad; e += 256) coefS[e] = coef64[c0 * km1_pad + e];
    __syncthreads();
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const double nc = nsv64[c0 + tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        if (ktype == 0) {
          const double d2 = nr[i] + nc - 2.0 * acc[i][j];
          acc[i][j] = exp(-gamma * (d2 > 0.0 ? d2 : 0.0));  // K in FP64
        } else if (ktype == 1) {  // linear: x . y (L76-L78)
        } else if (ktype == 2) {  // polynomial
          const double z = fma(gamma, acc[i][j], coef0);
          double v = 1.0;
          for (int e = 0; e < degree; ++e) v *= z;
          acc[i][j] = v;
        } else {  // sigmoid
          acc[i][j] = tanh(fma(gamma, acc[i][j], coef0));
        }
      }
    }
    for (int u = 0; u < km1; ++u) {
      double p[4] = {0.0, 0.0, 0.0, 0.0};
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const double cv = coefS[(tx * 4 + j) * km1_pad + u];
#pragma unroll
        for (int i = 0; i < 4; ++i) p[i] = fma(acc[i][j], cv, p[i]);
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) {  // sum over the 16 threads sharing these rows (fixed order)
        double v = p[i];
        v += __shfl_xor_sync(0xffffffffu, v, 1);
        v += __shfl_xor_sync(0xffffffffu, v, 2);
        v += __shfl_xor_sync(0xffffffffu, v, 4);
        v += __shfl_xor_sync(0xffffffffu, v, 8);
        p[i] = v;
      }
      if (tx == 0)
#pragma unroll
        for (int i = 0; i < 4; ++i) decS[(ty * 4 + i) * km1_pad + u] += p[i];
    }
  }
  __syncthreads();
  double* out = part + ((int64_t)blockIdx.y * m_pad + r0) * km1_pad;
  for (int i = tid; i < kF64Tile * km1_pad; i += 256) out[i] = decS[i];
}

// FP64 squared norms of the columns of a feature-major matrix XT[d_pad][ld] (n columns)
__global__ void col_norms64_kernel(const float* __restrict__ XT, int64_t ld, int64_t n, int d_pad,
                                   double* __restrict__ out) {
  const int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= n) return;
  double s = 0.0;
  for (int f = 0; f < d_pad; ++f) {
    const double x = (double)XT[(int64_t)f * ld + c];
    s = fma(x, x, s);
  }
  out[c] = s;
}

__global__ void dec_reduce64_kernel(const double* __restrict__ part, int64_t m, int64_t m_pad, int k, int km1_pad,
                                    const int32_t* __restrict__ item_begin, const int32_t* __restrict__ item_end,
                                    const double* __restrict__ b, double* __restrict__ dec) {
  const int P = k * (k - 1) / 2;
  const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= m * P) return;
  const int64_t i = gid / P;
  const int p = (int)(gid % P);
  int s = 0, rem = p;
  while (rem >= k - 1 - s) {
    rem -= k - 1 - s;
    ++s;
  }
  const int t = s + 1 + rem;
  double acc = b[p];
  for (int q = item_begin[s]; q < item_end[s]; ++q) acc += part[((int64_t)q * m_pad + i) * km1_pad + (t - 1)];
  for (int q = item_begin[t]; q < item_end[t]; ++q) acc += part[((int64_t)q * m_pad + i) * km1_pad + s];
  dec[gid] = acc;
}

void launch_col_norms64(const float* XT, int64_t ld, int64_t n, int d_pad, double* out, cudaStream_t st) {
  GM_LAUNCH(col_norms64_kernel, dim3((unsigned)ceil_div(n, 256)), dim3(256), 0, st, XT, ld, n, d_pad, out);
}

void launch_dec_f64(const float* XtT, int64_t ldt, const double* nt64, int64_t m_pad, const float* SvT, int64_t lds,
                    const double* nsv64, const double* coef64, int km1, int km1_pad, const DecItem* items, int n_items,
                    int d_pad, double gamma, double* part, cudaStream_t st, int ktype, double coef0, int degree) {
  const size_t smem = (size_t)(2 * kF64BK * kF64Tile + 2 * kF64Tile * km1_pad) * sizeof(double);
  set_max_dyn_smem(dec_f64_kernel, 96 * 1024);
  GM_LAUNCH(dec_f64_kernel, dim3((unsigned)(m_pad / kF64Tile), (unsigned)n_items), dim3(256), smem, st, XtT, ldt, nt64,
            SvT, lds, nsv64, coef64, km1, km1_pad, items, d_pad, gamma, m_pad, part, ktype, coef0, degree);
}

void launch_dec_reduce64(const double* part, int64_t m, int64_t m_pad, int k, int km1_pad, const int32_t* item_begin,
                         const int32_t* item_end, const double* b, double* dec, cudaStream_t st) {
  const int64_t tot = m * (int64_t)(k * (k - 1) / 2);
  GM_LAUNCH(dec_reduce64_kernel, dim3((unsigned)ceil_div(tot, 256)), dim3(256), 0, st, part, m, m_pad, k, km1_pad,
            item_begin, item_end, b, dec);
}

void launch_dec_reduce(const float* part, int64_t m, int64_t m_pad, int k, int km1_pad, const int32_t* item_begin,
                       const int32_t* item_end, const double* b, double* dec, cudaStream_t st) {
  const int64_t tot = m * (int64_t)(k * (k - 1) / 2);
  GM_LAUNCH(dec_reduce_kernel, dim3((unsigned)ceil_div(tot, 256)), dim3(256), 0, st, part, m, m_pad, k, km1_pad,
            item_begin, item_end, b, dec);
}

void launch_couple(const double* dec, int64_t m, int k, const double* A, const double* B, double* prob,
                   cudaStream_t st) {
  const size_t per = (size_t)k * k + (size_t)(k + 1) * (k + 2);
  const size_t smem = per * kCoupleWarps * sizeof(double);
  if (smem > 48 * 1024) set_max_dyn_smem(couple_kernel, smem);
  GM_LAUNCH(couple_kernel, dim3((unsigned)ceil_div(m, kCoupleWarps)), dim3(32 * kCoupleWarps), smem, st, dec, m, k, A,
            B, prob);
}

}  // namespace gmpsvm
