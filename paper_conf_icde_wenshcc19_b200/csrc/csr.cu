// csr.cu -- NEXT-3: kernel values from CSR rows without densifying X (the q rows
// against the rest "by a matrix multiplication", done there with cuSPARSE on CSR data, L513).
//
//   csr_stage_kernel      class-sorted CSR (row i of the sorted order = input row perm[i]): the
//                         row's segment copied, columns range-checked, values checked finite,
//                         squared norm accumulated in FP64 (stored FP32, like the dense staging).
//   krow_csr_kernel       FULL_K from the sorted CSR: a CTA densifies R consecutive rows into
//                         shared memory (R = rows whose d floats fit, <= kCsrMaxR) and one thread per
//                         column row j >= the block's first row streams j's non-zeros once,
//                         gathering the R dense rows -> R dot products per pass over j (the sparse
//                         x dense contraction of the paper's design); d^2 = |x_i|^2 + |x_j|^2 - 2 x_i.x_j
//                         clamped at 0, K = exp2(-gamma log2(e) d^2) (ex2.approx, as krow.cu),
//                         K_ii = 1, written with its mirror (the resident matrix is symmetric).
//   csr_densify_rows      dense rows of a row subset (the model's support vectors).
// Work: sum over row blocks of the non-zeros of the rows j >= the block -- about n * nnz / 2
// multiply-adds, against n^2 d / 2 for the dense contraction (density times fewer flops).
#include <algorithm>
#include <cstdint>

#include "kernels.h"

namespace gmpsvm {

namespace {

constexpr int kCsrThreads = 1024;
constexpr int kCsrMaxR = 16;  // rows densified per CTA (one accumulator register per row per thread)

__global__ void csr_stage_kernel(const int64_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                 const float* __restrict__ values, const int64_t* __restrict__ perm, int64_t n,
                                 int32_t d, const int64_t* __restrict__ sptr, int32_t* __restrict__ sidx,
                                 float* __restrict__ sval, float* __restrict__ norms, int32_t* __restrict__ bad) {
  const int lane = threadIdx.x & 31;
  const int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;  // one warp per sorted row
  if (i >= n) return;
  const int64_t src = perm[i];
  const int64_t b = indptr[src], e = indptr[src + 1], o = sptr[i];
  double acc = 0.0;
  for (int64_t t = b + lane; t < e; t += 32) {
    const int32_t c = indices[t];
    const float v = values[t];
    if (c < 0 || c >= d || !isfinite(v)) atomicExch(bad, 1);
    sidx[o + (t - b)] = c;
    sval[o + (t - b)] = v;
    acc = fma((double)v, (double)v, acc);
  }
#pragma unroll
  for (int s = 16; s > 0; s >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, s);
  if (lane == 0) norms[i] = (float)acc;
}

// R rows [r0, r0 + R) densified in shared memory ([R][d] FP32); one THREAD per column row j >= r0:
// it streams j's non-zeros and gathers the R dense rows at their columns (R dot products, no
// cross-lane reduction), then stores K[r0 + r][j] (coalesced across the warp's consecutive j) and
// the mirror K[j][r0 + r].  1024 threads: the row streams of many j are in flight per SM.
template <int R>
__global__ void __launch_bounds__(kCsrThreads) krow_csr_kernel(const int64_t* __restrict__ sptr,
                                                               const int32_t* __restrict__ sidx,
                                                               const float* __restrict__ sval,
                                                               const float* __restrict__ norms, int64_t n, int32_t d,
                                                               float scale, float* __restrict__ K, int64_t ldk) {
  extern __shared__ float dense[];  // [R][d]
  __shared__ float nrm[R];
  const int64_t r0 = (int64_t)blockIdx.x * R;
  const int nr = (int)(n - r0 < R ? n - r0 : R);
  for (int64_t t = threadIdx.x; t < (int64_t)R * d; t += blockDim.x) dense[t] = 0.f;
  if (threadIdx.x < R) nrm[threadIdx.x] = threadIdx.x < nr ? norms[r0 + threadIdx.x] : 0.f;
  __syncthreads();
  for (int r = 0; r < nr; ++r) {
    const int64_t b = sptr[r0 + r], e = sptr[r0 + r + 1];
    for (int64_t t = b + threadIdx.x; t < e; t += blockDim.x) dense[(size_t)r * d + sidx[t]] = sval[t];
  }
  __syncthreads();
  for (int64_t j = r0 + threadIdx.x; j < n; j += blockDim.x) {
    const int64_t b = sptr[j], e = sptr[j + 1];
    float acc[R];
#pragma unroll
    for (int r = 0; r < R; ++r) acc[r] = 0.f;
    int64_t t = b;
    for (; t + 1 < e; t += 2) {  // two non-zeros per pass: their loads in flight together
      const int32_t c0 = sidx[t], c1 = sidx[t + 1];
      const float v0 = sval[t], v1 = sval[t + 1];
#pragma unroll
      for (int r = 0; r < R; ++r) acc[r] = fmaf(v1, dense[(size_t)r * d + c1], fmaf(v0, dense[(size_t)r * d + c0], acc[r]));
    }
    if (t < e) {
      const int32_t c0 = sidx[t];
      const float v0 = sval[t];
#pragma unroll
      for (int r = 0; r < R; ++r) acc[r] = fmaf(v0, dense[(size_t)r * d + c0], acc[r]);
    }
    const float nj = norms[j];
    if ((R % 4) == 0 && nr == R && j >= r0 + R) {  // every i < j: the mirror row segment as float4 stores
      float kv[R];
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const float d2 = fmaxf(fmaf(-2.f, acc[r], nrm[r] + nj), 0.f);
        asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(kv[r]) : "f"(d2 * scale));
        K[(r0 + r) * ldk + j] = kv[r];
      }
      float4* dst = reinterpret_cast<float4*>(K + j * ldk + r0);  // ldk and r0 multiples of 4
#pragma unroll
      for (int r = 0; r < R; r += 4) dst[r / 4] = make_float4(kv[r], kv[r + 1], kv[r + 2], kv[r + 3]);
      continue;
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int64_t i = r0 + r;
      if (r < nr && j >= i) {
        float kv;
        if (j == i) {
          kv = 1.f;
        } else {
          const float d2 = fmaxf(fmaf(-2.f, acc[r], nrm[r] + nj), 0.f);
          asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(kv) : "f"(d2 * scale));
        }
        K[i * ldk + j] = kv;
        K[j * ldk + i] = kv;
      }
    }
  }
}

__global__ void csr_densify_rows_kernel(const int64_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                                        const float* __restrict__ values, const int64_t* __restrict__ rows, int64_t nr,
                                        int32_t d, float* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;  // one warp per output row
  if (i >= nr) return;
  float* o = out + i * (int64_t)d;
  for (int c = lane; c < d; c += 32) o[c] = 0.f;
  __syncwarp();
  const int64_t src = rows[i];
  for (int64_t t = indptr[src] + lane; t < indptr[src + 1]; t += 32) o[indices[t]] = values[t];
}

template <int R>
void launch_r(const int64_t* sptr, const int32_t* sidx, const float* sval, const float* norms, int64_t n, int32_t d,
              float scale, float* K, int64_t ldk, cudaStream_t st) {
  const size_t smem = (size_t)R * d * sizeof(float);
  set_max_dyn_smem(krow_csr_kernel<R>, smem);
  GM_LAUNCH(krow_csr_kernel<R>, dim3((unsigned)ceil_div(n, R)), dim3(kCsrThreads), smem, st, sptr, sidx, sval, norms,
            n, d, scale, K, ldk);
}

}  // namespace

void launch_csr_stage(const int64_t* indptr, const int32_t* indices, const float* values, const int64_t* perm, int64_t n,
                      int32_t d, const int64_t* sptr, int32_t* sidx, float* sval, float* norms, int32_t* bad,
                      cudaStream_t st) {
  GM_LAUNCH(csr_stage_kernel, dim3((unsigned)ceil_div(n * 32, 256)), dim3(256), 0, st, indptr, indices, values, perm, n,
            d, sptr, sidx, sval, norms, bad);
}

int krow_csr_rows_per_cta(int32_t d) {
  int dev = 0, optin = 0;
  GM_CUDA(cudaGetDevice(&dev));
  GM_CUDA(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  const int64_t r = (int64_t)optin / ((int64_t)d * 4);
  return (int)std::min<int64_t>(kCsrMaxR, r);  // 0: one dense row does not fit shared memory
}

void launch_krow_csr(const int64_t* sptr, const int32_t* sidx, const float* sval, const float* norms, int64_t n,
                     int32_t d, double gamma, float* K, int64_t ldk, cudaStream_t st) {
  const float scale = (float)(-gamma * 1.4426950408889634);
  const int r = krow_csr_rows_per_cta(d);
  if (r >= 16) launch_r<16>(sptr, sidx, sval, norms, n, d, scale, K, ldk, st);
  else if (r >= 12) launch_r<12>(sptr, sidx, sval, norms, n, d, scale, K, ldk, st);
  else if (r >= 8) launch_r<8>(sptr, sidx, sval, norms, n, d, scale, K, ldk, st);
  else if (r >= 4) launch_r<4>(sptr, sidx, sval, norms, n, d, scale, K, ldk, st);
  else if (r >= 2) launch_r<2>(sptr, sidx, sval, norms, n, d, scale, K, ldk, st);
  else if (r >= 1) launch_r<1>(sptr, sidx, sval, norms, n, d, scale, K, ldk, st);
  else throw Error(GMPSVM_ENOTIMPL, "CSR kernel values: one dense row of d floats must fit shared memory");
}

void launch_csr_densify_rows(const int64_t* indptr, const int32_t* indices, const float* values, const int64_t* rows,
                             int64_t nr, int32_t d, float* out, cudaStream_t st) {
  if (nr <= 0) return;
  GM_LAUNCH(csr_densify_rows_kernel, dim3((unsigned)ceil_div(nr * 32, 256)), dim3(256), 0, st, indptr, indices, values,
            rows, nr, d, out);
}

}  // namespace gmpsvm
