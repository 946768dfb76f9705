// Latency microbenchmarks of the primitives on the local-SMO critical chain (one warp or one
// 7-warp CTA, dependent chains of N ops, clock64 around them).  nvcc -arch=sm_100a lat.cu
#include <cstdio>
#include <cstdint>
#define N 256
__global__ void k(long long* out, unsigned seed, double dseed, float fseed) {
  __shared__ unsigned sm[1024];
  __shared__ double smd[1024];
  const int t = threadIdx.x;
  sm[t] = t * seed;
  smd[t] = t * dseed;
  __syncthreads();
  unsigned v = t * seed + 1;
  long long c0, c1;
  // redux.sync min
  c0 = clock64();
  for (int i = 0; i < N; ++i) v = __reduce_min_sync(0xffffffffu, v) + t;
  c1 = clock64();
  if (t == 0) out[0] = (c1 - c0) / N;
  // shfl idx
  c0 = clock64();
  for (int i = 0; i < N; ++i) v = __shfl_sync(0xffffffffu, v, (v + t) & 31) + 1;
  c1 = clock64();
  if (t == 0) out[1] = (c1 - c0) / N;
  // ballot + ffs
  c0 = clock64();
  for (int i = 0; i < N; ++i) v = __ffs(__ballot_sync(0xffffffffu, (v >> (t & 7)) & 1)) + v;
  c1 = clock64();
  if (t == 0) out[2] = (c1 - c0) / N;
  // LDS dependent
  c0 = clock64();
  for (int i = 0; i < N; ++i) v = sm[(v + t) & 1023];
  c1 = clock64();
  if (t == 0) out[3] = (c1 - c0) / N;
  // DADD dependent
  double d = dseed * t;
  c0 = clock64();
  for (int i = 0; i < N; ++i) d = d + dseed;
  c1 = clock64();
  if (t == 0) out[4] = (c1 - c0) / N;
  // DFMA dependent
  c0 = clock64();
  for (int i = 0; i < N; ++i) d = fma(d, dseed, dseed);
  c1 = clock64();
  if (t == 0) out[5] = (c1 - c0) / N;
  // F2F f64->f32->f64
  c0 = clock64();
  for (int i = 0; i < N; ++i) d = (double)((float)d) + dseed;
  c1 = clock64();
  if (t == 0) out[6] = (c1 - c0) / N;
  // MUFU rcp approx f32
  float f = fseed + t;
  c0 = clock64();
  for (int i = 0; i < N; ++i) { float r; asm volatile("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(f)); f = r + fseed; }
  c1 = clock64();
  if (t == 0) out[7] = (c1 - c0) / N;
  // bar.sync among all threads of the CTA
  c0 = clock64();
  for (int i = 0; i < N; ++i) { __syncthreads(); v += sm[(v + i) & 1023]; }
  c1 = clock64();
  if (t == 0) out[8] = (c1 - c0) / N;
  // STS + bar + LDS (cross-warp exchange round trip)
  c0 = clock64();
  for (int i = 0; i < N; ++i) { if ((t & 31) == 0) sm[t >> 5] = v; __syncthreads(); v = sm[(v + i) & 7] + 1; }
  c1 = clock64();
  if (t == 0) out[9] = (c1 - c0) / N;
  // double division
  c0 = clock64();
  for (int i = 0; i < N; ++i) d = dseed / d + 1.0;
  c1 = clock64();
  if (t == 0) out[10] = (c1 - c0) / N;
  // shfl of a double
  c0 = clock64();
  for (int i = 0; i < N; ++i) d = __shfl_sync(0xffffffffu, d, (int)(v + i) & 31) + 1.0;
  c1 = clock64();
  if (t == 0) out[11] = (c1 - c0) / N;
  // DSETP + select
  c0 = clock64();
  for (int i = 0; i < N; ++i) d = d > dseed ? d - dseed : d + 1.0;
  c1 = clock64();
  if (t == 0) out[12] = (c1 - c0) / N;
  out[20 + (t & 3)] = v + (long long)d + (long long)f + smd[t & 7];
}
int main() {
  long long* o;
  cudaMallocManaged(&o, 64 * 8);
  const char* names[] = {"redux.min", "shfl.idx", "ballot+ffs", "LDS dep", "DADD", "DFMA", "F2F rt+DADD", "MUFU.RCP+FADD",
                         "bar.sync+LDS", "STS+bar+LDS", "DDIV", "shfl f64", "DSETP+sel"};
  for (int nt : {32, 224, 1024}) {
    k<<<1, nt>>>(o, 3u, 1.0000001, 1.5f);
    cudaDeviceSynchronize();
    k<<<1, nt>>>(o, 3u, 1.0000001, 1.5f);
    cudaDeviceSynchronize();
    printf("threads %d:", nt);
    for (int i = 0; i < 13; ++i) printf(" %s=%lld", names[i], o[i]);
    printf("\n");
  }
}
