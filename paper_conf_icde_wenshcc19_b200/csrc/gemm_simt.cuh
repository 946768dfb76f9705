// gemm_simt.cuh -- FP32 SIMT 128x128 tile contraction shared by krow_contract (a2) and
// dec_contract (a10).  Both operands are stored "feature-major" (transposed): AT[k][i] with
// the instance index contiguous, so every k-slice of a tile is one contiguous 512-byte row
// and lands in shared memory with 16-byte cp.async copies (no register transpose).
//
// 256 threads; thread (ty, tx) = (tid / 16, tid % 16) owns rows {ty*4 + 0..3, 64 + ty*4 + 0..3}
// and columns {tx*4 + 0..3, 64 + tx*4 + 0..3} of the tile: 64 FP32 accumulators, 4 LDS.128
// per 64 FFMA.  kStages-deep cp.async ring over k-steps of kBK.
#pragma once

#include "common.cuh"

namespace gmpsvm {

constexpr int kGemmThreads = 256;
constexpr int kStages = 3;

struct GemmSmem {
  float a[kStages][kBK][kTile];
  float b[kStages][kBK][kTile];
};  // 48 KB

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;\n" ::"n"(N));
}

__device__ __forceinline__ float fast_exp2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// Row / column of accumulator element (i, j) inside the tile.
__device__ __forceinline__ int tile_row(int ty, int i) { return (i < 4) ? ty * 4 + i : 64 + ty * 4 + (i - 4); }
__device__ __forceinline__ int tile_col(int tx, int j) { return (j < 4) ? tx * 4 + j : 64 + tx * 4 + (j - 4); }

// acc[i][j] = sum_k AT[k][a0 + row(i)] * BT[k][b0 + col(j)] over k in [0, kdim).
// Requires: kdim % kBK == 0, lda/ldb % 4 == 0, a0/b0 % 4 == 0, columns [a0, a0+128) and
// [b0, b0+128) inside the (zero-padded) operands.  Caller syncs before reusing `sm`.
__device__ __forceinline__ void gemm_tile_128(const float* __restrict__ AT, int64_t lda, int64_t a0,
                                              const float* __restrict__ BT, int64_t ldb, int64_t b0, int kdim,
                                              GemmSmem& sm, float acc[8][8]) {
  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
  const int nk = kdim / kBK;
  // per thread: 2 x 16B of A and 2 x 16B of B per stage
  const int kk0 = tid >> 5, c40 = (tid & 31) * 4;  // lin = tid        -> (kk0, c40)
  const int kk1 = kk0 + 8;                         // lin = tid + 256  -> (kk0 + 8, c40)
  const float* pa = AT + a0 + c40;
  const float* pb = BT + b0 + c40;
  auto load_stage = [&](int stage, int kb) {
    const int64_t k0 = (int64_t)kb * kBK;
    cp_async16(&sm.a[stage][kk0][c40], pa + (k0 + kk0) * lda);
    cp_async16(&sm.a[stage][kk1][c40], pa + (k0 + kk1) * lda);
    cp_async16(&sm.b[stage][kk0][c40], pb + (k0 + kk0) * ldb);
    cp_async16(&sm.b[stage][kk1][c40], pb + (k0 + kk1) * ldb);
  };
#pragma unroll
  for (int s = 0; s < kStages - 1; ++s) {
    if (s < nk) load_stage(s, s);
    cp_async_commit();
  }
  for (int kb = 0; kb < nk; ++kb) {
    cp_async_wait<kStages - 2>();
    __syncthreads();
    const int nxt = kb + kStages - 1;
    if (nxt < nk) load_stage(nxt % kStages, nxt);
    cp_async_commit();
    const int st = kb % kStages;
#pragma unroll
    for (int kk = 0; kk < kBK; ++kk) {
      const float4 a0v = *reinterpret_cast<const float4*>(&sm.a[st][kk][ty * 4]);
      const float4 a1v = *reinterpret_cast<const float4*>(&sm.a[st][kk][64 + ty * 4]);
      const float4 b0v = *reinterpret_cast<const float4*>(&sm.b[st][kk][tx * 4]);
      const float4 b1v = *reinterpret_cast<const float4*>(&sm.b[st][kk][64 + tx * 4]);
      const float av[8] = {a0v.x, a0v.y, a0v.z, a0v.w, a1v.x, a1v.y, a1v.z, a1v.w};
      const float bv[8] = {b0v.x, b0v.y, b0v.z, b0v.w, b1v.x, b1v.y, b1v.z, b1v.w};
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
  }
  cp_async_wait<0>();
}

}  // namespace gmpsvm
