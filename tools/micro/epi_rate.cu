// The int8 decision-value epilogue's FP64 arithmetic on its own (dec_i8.cu): per (test row, SV)
// element x~.y~ scaling, d2, 2^(tsc d2) by the degree-10 series and the k - 1 = 9 coefficient
// FMAs, 8 elements in flight per thread, 8 math warps per SM (as the kernel) -- how many SM
// cycles per element does the FP64 pipe need, without the tensor core or TMEM beside it?
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o epi_rate epi_rate.cu && ./epi_rate
#include <cstdio>
#include <cuda_runtime.h>

constexpr int KM = 9;
constexpr double kShift52 = 6755399441055744.0;
__device__ __constant__ const double kC[11] = {7.054911620801123e-09, 1.01780860092397e-07, 1.321548679014431e-06,
                                               1.5252733804059841e-05, 0.0001540353039338161, 0.0013333558146428443,
                                               0.009618129107628477, 0.05550410866482158, 0.24022650695910072,
                                               0.6931471805599453, 1.0};
__device__ __forceinline__ double pow2(int k) { return __hiloint2double((k + 1023) << 20, 0); }

template <int MODE>  // 0: full element math; 1: no coefficient FMAs; 2: no series (kv = t)
__global__ void __launch_bounds__(320, 1) epi_k(const double* es_in, double* out, int halves, long long* cyc) {
  __shared__ double cs[64 * KM];
  for (int i = threadIdx.x; i < 64 * KM; i += blockDim.x) cs[i] = 1e-3 * (i % 17);
  __syncthreads();
  const int warp = threadIdx.x >> 5;
  if (warp < 2) return;  // producer / MMA warps idle
  const int part = (warp - 2) >> 2, lane = threadIdx.x & 31;
  double acc[KM];
  for (int v = 0; v < KM; ++v) acc[v] = 0.0;
  const double tsc = -0.125 * 1.4426950408889634, nr = 1.0 + lane * 1e-3;
  double dot[32];
  for (int j = 0; j < 32; ++j) dot[j] = 1e6 * (j + lane);
  const long long t0 = clock64();
  for (int h = 0; h < halves; ++h) {
#pragma unroll
    for (int jb = 0; jb < 32; jb += 8) {
      double tt[8], ff[8], pp[8];
      int nn[8];
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const int c = part * 32 + jb + e;
        const double xy = dot[jb + e] * pow2(-40 - (h & 3));
        const double d2 = fmax(fma(-2.0, xy, nr + __ldg(es_in + c)), 0.0);
        tt[e] = fmax(tsc * d2, -1020.0);
      }
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const double big = tt[e] + kShift52;
        const double n = big - kShift52;
        ff[e] = tt[e] - n;
        nn[e] = __double2loint(big);
        pp[e] = kC[0];
      }
      if (MODE != 2) {
#pragma unroll
        for (int k = 1; k < 11; ++k)
#pragma unroll
          for (int e = 0; e < 8; ++e) pp[e] = fma(pp[e], ff[e], kC[k]);
      }
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const double kv = pp[e] * pow2(nn[e]);
        if (MODE == 1) {
          acc[e & 7] += kv;
        } else {
          const double* cj = cs + (part * 32 + jb + e) * KM;
#pragma unroll
          for (int v = 0; v < KM; ++v) acc[v] = fma(kv, cj[v], acc[v]);
        }
      }
    }
  }
  const long long t1 = clock64();
  double s = 0;
  for (int v = 0; v < KM; ++v) s += acc[v];
  if (s == 1.2345) out[0] = s;
  if (blockIdx.x == 0 && threadIdx.x == 64) cyc[0] = t1 - t0;
}

int main() {
  double *es, *out;
  long long* cyc;
  cudaMalloc(&es, 64 * 8);
  cudaMemset(es, 0, 64 * 8);
  cudaMalloc(&out, 8);
  cudaMalloc(&cyc, 8);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int halves = 200;
  auto run = [&](const char* name, auto kern) {
    kern<<<sms, 320>>>(es, out, 4, cyc);
    cudaDeviceSynchronize();
    kern<<<sms, 320>>>(es, out, halves, cyc);
    cudaError_t e = cudaDeviceSynchronize();
    long long c = 0;
    cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
    // per SM per half: 8 warps x 32 threads x 32 elements = 8192 elements
    printf("{\"epilogue\": \"%s\", \"err\": \"%s\", \"cycles_per_half\": %.0f, \"sm_cycles_per_element\": %.3f}\n", name,
           cudaGetErrorString(e), (double)c / halves, (double)c / halves / 8192.0);
  };
  run("full (series + 9 coefficient FMAs)", epi_k<0>);
  run("no coefficient FMAs", epi_k<1>);
  run("no series", epi_k<2>);
  return 0;
}
