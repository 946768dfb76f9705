// tcgen05.mma kind::i8 / kind::f16 issue-rate microbenchmark: one CTA per SM, one thread issues
// `iters` MMAs (M = 128, N = 64 / 128 / 256) from shared memory into TMEM back to back; time per
// MMA from clock64 around the loop + the final commit's mbarrier.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(const void* p, int sw) {  // sw: 2 = 128B, 4 = 64B
  uint64_t d = (su32(p) >> 4) & 0x3FFF;
  d |= 1ull << 16;
  d |= (uint64_t)((sw == 2 ? 1024 : 512) >> 4) << 32;
  d |= 1ull << 46;
  d |= (uint64_t)sw << 61;
  return d;
}
template <int KIND, int N>  // KIND 0: i8 (K = 32), 1: f16 (K = 16)
__global__ void k(int iters, long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint32_t tbase;
  __shared__ __align__(8) uint64_t bar;
  const int warp = threadIdx.x >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(&tbase)), "r"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 32) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (threadIdx.x == 32) {
    const uint32_t tm = tbase;
    const int sw = 2;
    const uint64_t a = desc(sm, sw), b = desc(sm + 32768, sw);
    constexpr uint32_t idesc = KIND == 0 ? ((2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | (8u << 24))
                                         : ((1u << 4) | ((uint32_t)(N >> 3) << 17) | (8u << 24));
    const long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const uint32_t d = tm + (uint32_t)((i & 1) * N) % 512;
      if (KIND == 0)
        asm volatile("{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
                     "l"(a + (uint64_t)((i & 3) * 2)), "l"(b + (uint64_t)((i & 3) * 2)), "r"(idesc), "r"(1));
      else
        asm volatile("{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
                     "l"(a + (uint64_t)((i & 3) * 2)), "l"(b + (uint64_t)((i & 3) * 2)), "r"(idesc), "r"(1));
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)) : "memory");
    uint32_t done = 0;
    do {
      asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n selp.u32 %0, 1, 0, p;\n}\n"
                   : "=r"(done) : "r"(su32(&bar)) : "memory");
    } while (!done);
    const long long t1 = clock64();
    if (blockIdx.x == 0) out[0] = t1 - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase), "r"(512));
  }
}

// The int8 decision-value kernel's issue pattern (dec_i8.cu): per 32-wide k step, A plane i
// (i = 0..4) times B planes j with i + j <= 5 into accumulator i + j (N = 64 each, 6 x 64 TMEM
// columns), optionally with the A-operand collector (fill / use / lastuse), one commit per
// 64-wide k block.  Cycles per MMA for the whole sequence.
template <bool COLLECT, int NN, bool SYNC = false>
__global__ void pattern_k(int kblocks, long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint32_t tbase;
  __shared__ __align__(8) uint64_t bar;
  __shared__ __align__(8) uint64_t bar2;
  const int warp = threadIdx.x >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(&tbase)), "r"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 32) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar2)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (threadIdx.x == 32) {
    const uint32_t tm = tbase;
    constexpr uint32_t idesc = (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(NN >> 3) << 17) | (8u << 24);
    const long long t0 = clock64();
    for (int kb = 0; kb < kblocks; ++kb) {
      if (SYNC) {  // as in the kernel: wait on a (completed) stage barrier, fence, ..., commit
        uint32_t done = 0;
        do {
          asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 1;\n selp.u32 %0, 1, 0, p;\n}\n"
                       : "=r"(done) : "r"(su32(&bar)) : "memory");
        } while (!done);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      }
      for (int kk = 0; kk < 2; ++kk) {
        for (int i = 0; i < 5; ++i) {
          const uint64_t a = desc(sm + i * 8192, 4) + (uint64_t)(kk * 2);
          const int jn = 6 - i < 5 ? 6 - i : 5;
          for (int j = 0; j < jn; ++j) {
            const uint64_t b = desc(sm + 40960 + j * (NN * 64), 4) + (uint64_t)(kk * 2);
            const uint32_t d = tm + (uint32_t)((i + j) * NN);
            if (COLLECT && j == 0)
              asm volatile("{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::i8.collector::a::fill [%0], %1, %2, %3, p;\n}\n" ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(1));
            else if (COLLECT && j == jn - 1)
              asm volatile("{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::i8.collector::a::lastuse [%0], %1, %2, %3, p;\n}\n" ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(1));
            else if (COLLECT)
              asm volatile("{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::i8.collector::a::use [%0], %1, %2, %3, p;\n}\n" ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(1));
            else
              asm volatile("{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n}\n" ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(1));
          }
        }
      }
      if (SYNC) asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar2)) : "memory");
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)) : "memory");
    uint32_t done = 0;
    do {
      asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n selp.u32 %0, 1, 0, p;\n}\n"
                   : "=r"(done) : "r"(su32(&bar)) : "memory");
    } while (!done);
    const long long t1 = clock64();
    if (blockIdx.x == 0) out[0] = t1 - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase), "r"(512));
  }
}

int main() {
  long long* out;
  cudaMalloc(&out, 8);
  const int iters = 20000;
  auto run = [&](const char* name, auto kern, double macs) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 98304);
    kern<<<148, 64, 98304>>>(100, out);
    cudaDeviceSynchronize();
    kern<<<148, 64, 98304>>>(iters, out);
    cudaError_t e = cudaDeviceSynchronize();
    long long cyc = 0;
    cudaMemcpy(&cyc, out, 8, cudaMemcpyDeviceToHost);
    printf("{\"mma\": \"%s\", \"err\": \"%s\", \"cycles_per_mma\": %.2f, \"macs_per_cycle_per_sm\": %.0f}\n", name,
           cudaGetErrorString(e), (double)cyc / iters, macs / ((double)cyc / iters));
  };
  run("i8 M128 N64 K32", k<0, 64>, 128.0 * 64 * 32);
  run("i8 M128 N128 K32", k<0, 128>, 128.0 * 128 * 32);
  run("i8 M128 N256 K32", k<0, 256>, 128.0 * 256 * 32);
  run("f16 M128 N64 K16", k<1, 64>, 128.0 * 64 * 16);
  run("f16 M128 N128 K16", k<1, 128>, 128.0 * 128 * 16);
  run("f16 M128 N256 K16", k<1, 256>, 128.0 * 256 * 16);
  auto runp = [&](const char* name, auto kern, int nn) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 120 * 1024);
    kern<<<148, 64, 120 * 1024>>>(2, out);
    cudaDeviceSynchronize();
    const int kb = 2000;
    kern<<<148, 64, 120 * 1024>>>(kb, out);
    cudaError_t e = cudaDeviceSynchronize();
    long long cyc = 0;
    cudaMemcpy(&cyc, out, 8, cudaMemcpyDeviceToHost);
    const double mmas = (double)kb * 2 * 19;
    printf("{\"pattern\": \"%s\", \"err\": \"%s\", \"cycles_per_mma\": %.2f, \"macs_per_cycle_per_sm\": %.0f}\n", name,
           cudaGetErrorString(e), (double)cyc / mmas, 128.0 * nn * 32 / ((double)cyc / mmas));
  };
  runp("dec_i8 19-product pattern N64, collector", pattern_k<true, 64>, 64);
  runp("dec_i8 19-product pattern N64, no collector", pattern_k<false, 64>, 64);
  runp("dec_i8 19-product pattern N80, collector", pattern_k<true, 80>, 80);
  runp("dec_i8 19-product pattern N64, collector, per-k-block wait+fence+commit", pattern_k<true, 64, true>, 64);
  return 0;
}
