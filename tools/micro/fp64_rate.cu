// FP64 pipe microbenchmark (B200): DFMA throughput with ILP chains per thread, and the rate of
// the conversions the int8 decision-value epilogue uses (I2F.F64.S64, F2I, FRND.F64).
#include <cstdio>
#include <cuda_runtime.h>
template <int CH>
__global__ void dfma_k(double* out, int iters) {
  double a[CH];
  for (int c = 0; c < CH; ++c) a[c] = threadIdx.x * 1e-3 + c;
  const double b = 0.999999, d = 1e-7;
  for (int i = 0; i < iters; ++i)
#pragma unroll
    for (int c = 0; c < CH; ++c) a[c] = fma(a[c], b, d);
  double s = 0;
  for (int c = 0; c < CH; ++c) s += a[c];
  if (s == 123.456) out[0] = s;
}
__global__ void i2f_k(double* out, int iters) {
  long long x = threadIdx.x * 12345ll;
  double s = 0;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) s += (double)(x + c * 77 + i);
  }
  if (s == 123.456) out[0] = s;
}
__global__ void frnd_k(double* out, int iters) {
  double x[8];
  for (int c = 0; c < 8; ++c) x[c] = threadIdx.x * 0.37 + c;
  for (int i = 0; i < iters; ++i)
#pragma unroll
    for (int c = 0; c < 8; ++c) x[c] = rint(x[c] * 1.0000001) + 0.25;
  double s = 0;
  for (int c = 0; c < 8; ++c) s += x[c];
  if (s == 123.456) out[0] = s;
}
int main() {
  double* out;
  cudaMalloc(&out, 8);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int iters = 4096;
  auto run = [&](const char* name, auto kern, int blocks, int threads, double ops_per_thread_iter) {
    kern<<<blocks, threads>>>(out, 16);
    cudaEventRecord(e0);
    kern<<<blocks, threads>>>(out, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double ops = (double)blocks * threads * iters * ops_per_thread_iter;
    int clk = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    printf("{\"kernel\": \"%s\", \"blocks\": %d, \"threads\": %d, \"ms\": %.3f, \"Gop_s\": %.1f, \"per_sm_per_cycle\": %.2f}\n", name,
           blocks, threads, ms, ops / ms / 1e6, ops / (ms * 1e-3) / sms / (clk * 1e3));
  };
  run("dfma_chains1", dfma_k<1>, sms * 4, 256, 1);
  run("dfma_chains4", dfma_k<4>, sms * 4, 256, 4);
  run("dfma_chains8", dfma_k<8>, sms * 4, 256, 8);
  run("dfma_chains8_1warp_per_smsp", dfma_k<8>, sms, 128, 8);
  run("dfma_chains8_2warps_per_smsp", dfma_k<8>, sms, 256, 8);
  run("i2f_s64_f64", i2f_k, sms * 4, 256, 8);
  run("frnd_f64", frnd_k, sms * 4, 256, 8);
  return 0;
}
