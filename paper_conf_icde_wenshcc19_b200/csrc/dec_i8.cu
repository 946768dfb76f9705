// dec_i8.cu -- a10 (decision values, Eq 11, PAPER.md L142 / L261-L263) with FP64-accurate kernel
// values on the int8 tensor cores (tcgen05.mma kind::i8, exact int32 accumulation in TMEM).
//
// Why: a probability's sensitivity to a decision value is |A_p|/4 (dP/d dec = A P (1-P), Eq 12),
// and a decision value sums sum_j |alpha_j| K_j of kernel values (Eq 11).  Any path that holds K
// in FP32 has a worst-case error of sum_j |alpha_j| * 2^-24 and more -- MNIST-shaped C = 10 models
// (sum |alpha| ~ 10^3, |A| ~ 6) then cannot be bounded below the 1e-4 probability contract.
// Here the dot products are EXACT integers and K is formed in FP64:
//
//   staging (one warp per row): e_r = 37 - ilogb(max_c |x_rc|), X_int = rint(x * 2^e_r) with
//     |X_int| < 2^38 (exact for every element >= max|x| 2^-14, else off by <= max|x| 2^-38), written
//     as 5 balanced base-256 digits D_0..D_4 in [-128, 127] (D_0 most significant), one int8 plane
//     each; ||x~||^2 in FP64 from the integers.
//   contraction: X_int . Y_int = sum_{i,j} 256^(8-i-j) P_ij, P_ij = D_i(x) . D_j(y) computed by
//     kind::i8 MMAs into int32 TMEM accumulators (|P| <= 5 * 800 * 2^14 < 2^31: exact); products
//     with the same i + j = g share accumulator g; g <= 5 kept (19 of 25 products), the dropped
//     g >= 6 terms are below 2^-44 d max|x| max|y|.
//   epilogue (FP64): x~.y~ = 2^-(e_x+e_y) sum_g 256^(8-g) G_g, d2 = ||x~||^2 + ||y~||^2 - 2 x~.y~
//     (clamped at 0), K = exp(-gamma d2) (CUDA's FP64 exp), contracted with the SV tile's FP64
//     coefficients (k - 1 pair columns) into FP64 per-row accumulators.  K never leaves the SM.
//
// CTA: warp 0 = TMA producer, warp 1 = MMA issuer (+ TMEM allocation), warps 2..5 = epilogue
// (one TMEM lane quarter each, one test row per thread).  Tile = 128 test rows x 64 SVs (half of a
// class-pure 128-slot SV tile); k-block = 64 int8 (one 64-byte swizzle atom); 3-stage ring of
// 60 KB (5 A planes of 128 x 64 B + 5 B planes of 64 x 64 B); TMEM 6 groups x 64 columns.
// Persistent CTAs take the work units of launch_dec_tc (one test tile x a run of SV tiles of one
// class) round-robin and write part[unit_item[u]][row][0..km1_pad) in FP64.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <string>

#include "kernels.h"
#include "tc_util.cuh"

namespace gmpsvm {

namespace {

constexpr int kND = 5;                     // digit planes per operand (40-bit fixed point)
constexpr int kNG = 6;                     // digit-product groups kept: g = i + j <= 5
constexpr int kIM = 128, kIN = 64, kIK = 64;  // test rows, SVs per tile, int8 per k-block (64 B atom)
constexpr int kIStages = 3;
constexpr uint32_t kIAPlane = kIM * kIK;  // 8 KB
constexpr uint32_t kIBPlane = kIN * kIK;  // 4 KB
constexpr uint32_t kIStageBytes = kND * (kIAPlane + kIBPlane);  // 60 KB
constexpr uint32_t kITmemCols = 512;      // 6 x 64 used (power-of-two allocation)
// epilogue warps: 16 (4 per TMEM lane quarter, 16 of a tile's 64 SV columns each) while the per-row
// sums fit the register budget of 576 threads (k - 1 <= 12), else 8 (two per quarter, 32 columns)
template <int KM>
constexpr int i8_epi_warps() { return 8; }
template <int KM>
constexpr int i8_threads() { return 64 + 32 * i8_epi_warps<KM>(); }  // producer, MMA issuer, epilogue
constexpr int kIExp = 37;                 // max |x| 2^e in [2^37, 2^38)
// kind::i8, D S32 (2), A S8 (1), B S8 (1), K-major, N = 64, M = 128
constexpr uint32_t kIdescI8 =
    (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(kIN >> 3) << 17) | ((uint32_t)(kIM >> 4) << 24);

template <int KM>
constexpr int i8_stages() { return KM > 12 ? 2 : kIStages; }  // large k: the coefficient tiles need the room
template <int KM>
constexpr int i8_row() { return (KM + 3) & ~1; }  // doubles per staged SV column (even: 16-byte pairs)
template <int KM>
struct DecI8Smem {
  alignas(1024) uint8_t stage[i8_stages<KM>()][kIStageBytes];
  alignas(16) double coefS[2][kIN][i8_row<KM>()];  // per SV column: 2^(24 - e_c), ||y~||^2, coefficients
  double red[kIM][KM];  // reduction of the column parts' per-row sums
  alignas(8) uint64_t full[i8_stages<KM>()];
  uint64_t empty[i8_stages<KM>()];
  uint64_t tmem_full;
  uint64_t tmem_empty;
  uint32_t tmem_base;
};

// K-major operand, 64-byte swizzle: 8-row groups 512 B apart (SBO), LBO unused, version 1
__device__ __forceinline__ uint64_t umma_desc_sw64_addr(uint32_t addr32) {
  const uint64_t addr = addr32;
  uint64_t d = 0;
  d |= (addr >> 4) & 0x3FFFull;
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)(512 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)4 << 61;  // SWIZZLE_64B
  return d;
}
// collector: 0 none, 1 fill (keep A for the next MMA), 2 use (reuse and keep), 3 lastuse
template <int COL>
__device__ __forceinline__ void umma_i8(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t accum) {
  if (COL == 1)
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::i8.collector::a::fill [%0], %1, %2, %3, "
        "p;\n}\n" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(kIdescI8), "r"(accum));
  else if (COL == 2)
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::i8.collector::a::use [%0], %1, %2, %3, "
        "p;\n}\n" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(kIdescI8), "r"(accum));
  else if (COL == 3)
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::i8.collector::a::lastuse [%0], %1, %2, "
        "%3, p;\n}\n" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(kIdescI8), "r"(accum));
  else
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n}\n" ::"r"(
            tmem_d),
        "l"(a), "l"(b), "r"(kIdescI8), "r"(accum));
}
__device__ __forceinline__ double pow2(int k) { return __hiloint2double((k + 1023) << 20, 0); }  // 2^k, |k| < 1023

// Exact int64 -> double for |w| < 2^51 without the quarter-rate I2F.F64.S64: the bit pattern of
// 1.5 2^52 plus w is the double 1.5 2^52 + w.  kShift52 also rounds a double to an integer (RNE).
constexpr double kShift52 = 6755399441055744.0;  // 1.5 * 2^52
__device__ __forceinline__ double i2d_small(long long w) {
  return __longlong_as_double(w + 0x4338000000000000ll) - kShift52;
}

// c_k = ln(2)^k / k!, k = 10 .. 0: the Taylor coefficients of 2^f (exp2_neg, the epilogue)
__device__ __constant__ const double kExp2C[11] = {7.054911620801123e-09, 1.01780860092397e-07, 1.321548679014431e-06,
                                                   1.5252733804059841e-05, 0.0001540353039338161, 0.0013333558146428443,
                                                   0.009618129107628477, 0.05550410866482158, 0.24022650695910072,
                                                   0.6931471805599453, 1.0};

// 2^t for t <= 0 in FP64: t = n + f, n = rint(t), |f| <= 1/2; 2^f by its Taylor series in
// f ln 2 to degree 10 (remainder <= (ln2 / 2)^11 / 11! e^(ln2 / 2) < 3.2e-13 relative) evaluated by
// Horner in FP64; 2^n exactly.  Below 2^-1020 the result is 0 (absolute error < 1e-307).
__device__ __forceinline__ double exp2_neg(double t) {
  if (t < -1020.0) return 0.0;
  const double n = rint(t);
  const double f = t - n;  // exact
  // c_k = ln(2)^k / k!, k = 10 .. 0
  constexpr double c[11] = {
    7.054911620801123e-09,
    1.01780860092397e-07,
    1.321548679014431e-06,
    1.5252733804059841e-05,
    0.0001540353039338161,
    0.0013333558146428443,
    0.009618129107628477,
    0.05550410866482158,
    0.24022650695910072,
    0.6931471805599453,
    1.0};
  double p = c[0];
#pragma unroll
  for (int k = 1; k < 11; ++k) p = fma(p, f, c[k]);
  return p * pow2((int)n);
}

// rows [0, n_pad) of X (row src[j], or j; < 0 / >= n: zero row) -> planes[p][j][0..d8), e[j], nrm[j];
// amax_out (optional): max over the rows of max |x| as float bits (atomicMax, non-negative floats)
__global__ void stage_i8_kernel(const float* __restrict__ X, int64_t n, int d, const int64_t* __restrict__ src,
                                int8_t* __restrict__ planes, int64_t rows_pad, int d8, int32_t* __restrict__ ex,
                                double* __restrict__ nrm, unsigned* __restrict__ amax_out) {
  const int64_t j = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (j >= rows_pad) return;
  const int64_t r = (j < n) ? (src ? src[j] : j) : -1;
  const float* row = r >= 0 ? X + r * d : nullptr;
  float a = 0.f;
  if (row)
    for (int c = lane; c < d; c += 32) a = fmaxf(a, fabsf(row[c]));
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) a = fmaxf(a, __shfl_xor_sync(0xffffffffu, a, o));
  const int e = a > 0.f ? kIExp - ilogbf(a) : 0;
  double s = 0.0;
  for (int c = lane; c < d8; c += 32) {
    long long xi = 0;
    if (row && c < d) xi = llrint(ldexp((double)row[c], e));
    const double xd = (double)xi;
    s = fma(xd, xd, s);
#pragma unroll
    for (int p = kND - 1; p >= 0; --p) {  // least significant digit first
      const int dg = (int)((xi + 128) & 255) - 128;
      planes[((int64_t)p * rows_pad + j) * d8 + c] = (int8_t)dg;
      xi = (xi - dg) >> 8;  // exact
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) {
    ex[j] = e;
    nrm[j] = s * pow2(-2 * e);
    if (amax_out && row) atomicMax(amax_out, __float_as_uint(a));
  }
}

template <int KM>
__global__ void __launch_bounds__(i8_threads<KM>(), 1)
    dec_i8_kernel(const __grid_constant__ CUtensorMap map_t, const __grid_constant__ CUtensorMap map_s,
                  const int2* __restrict__ tiles, const int32_t* __restrict__ unit_off,
                  const int32_t* __restrict__ unit_item, int n_units, const int32_t* __restrict__ et,
                  const double* __restrict__ nt, const int32_t* __restrict__ es, const double* __restrict__ ns,
                  const double* __restrict__ coef, int km1, int km1_pad, int d8, int64_t m_pad, int64_t nsv_pad,
                  double gamma, double* __restrict__ part_out, int diag) {
  extern __shared__ __align__(1024) uint8_t dsmem[];
  DecI8Smem<KM>& sm =
      *reinterpret_cast<DecI8Smem<KM>*>((reinterpret_cast<uintptr_t>(dsmem) + 1023) & ~uintptr_t(1023));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  constexpr int NS = i8_stages<KM>();
  const int nk = (d8 + kIK - 1) / kIK;
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < NS; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], 1);
    }
    mbar_init(&sm.tmem_full, 1);
    mbar_init(&sm.tmem_empty, i8_epi_warps<KM>());
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map_t)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map_s)) : "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&sm.tmem_base)),
                 "r"(kITmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = sm.tmem_base;

  if (warp == 0) {
    if (lane == 0) {  // ---- TMA producer: per (tile, half, k-block) the 5 + 5 digit planes
      int g = 0;
      const uint64_t pol = policy_evict_last();
      for (int u = blockIdx.x; u < n_units; u += gridDim.x)
        for (int t = unit_off[u]; t < unit_off[u + 1]; ++t) {
          const int2 tile = tiles[t];
          const int r0 = tile.x * kIM;
          for (int h = 0; h < 2; ++h) {
            const int c0 = tile.y * 2 * kIN + h * kIN;
            for (int kb = 0; kb < nk; ++kb, ++g) {
              const int s = g % NS;
              if (g >= NS) mbar_wait(&sm.empty[s], ((g / NS) + 1) & 1);
              uint8_t* st = sm.stage[s];
              if (diag & 4) {  // GMPSVM_I8_DIAG bit 2 (timing experiments): no operand loads
                asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.full[s])) : "memory");
                continue;
              }
              mbar_expect_tx(&sm.full[s], kIStageBytes);
#pragma unroll
              for (int p = 0; p < kND; ++p) {
                tma_load_2d(st + p * kIAPlane, &map_t, kb * kIK, (int)(p * m_pad + r0), &sm.full[s], pol);
                tma_load_2d(st + kND * kIAPlane + p * kIBPlane, &map_s, kb * kIK, (int)(p * nsv_pad + c0), &sm.full[s],
                            pol);
              }
            }
          }
        }
    }
  } else if (warp == 1) {
    // ---- MMA issuer: group g = i + j of the digit products into accumulator g.  The whole warp
    // runs the loop (warp-uniform control flow, so the descriptors and TMEM addresses live in
    // uniform registers) and one elected lane issues: issued from a lone `lane == 0` thread, every
    // MMA went through an ELECT / R2UR.BROADCAST / BRA.U.ANY sequence and the issue loop, not the
    // tensor pipe, set the pace (69 cycles per MMA against 44.6 in tools/micro/i8_mma_rate.cu;
    // measured with clock64 around the waits: 6.1M of CTA 0's 6.5M cycles were spent issuing).
    int g = 0, it = 0;
    for (int u = blockIdx.x; u < n_units; u += gridDim.x)
      for (int t = unit_off[u]; t < unit_off[u + 1]; ++t)
        for (int h = 0; h < 2; ++h, ++it) {
          if (it > 0) mbar_wait(&sm.tmem_empty, (it - 1) & 1);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          for (int kb = 0; kb < nk; ++kb, ++g) {
            const int s = g % NS;
            mbar_wait(&sm.full[s], (g / NS) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint32_t st_a = smem_u32(sm.stage[s]);
            const int nsub = (diag & 2) ? 0 : min(2, (d8 - kb * kIK + 31) / 32);  // valid 32-wide k steps
            if (elect_one()) {
              for (int kk = 0; kk < nsub; ++kk) {
                const uint64_t adv = (uint64_t)(kk * 32) >> 4;
                // A plane i stays in the tensor core's collector across its products with every B
                // plane j (i + j <= 5): the A operand is read from shared memory once per (i, kk)
#pragma unroll
                for (int i = 0; i < kND; ++i) {
                  const uint64_t ad = umma_desc_sw64_addr(st_a + i * kIAPlane) + adv;
                  const int jn = min(kND, kNG - i);  // j = 0 .. jn - 1
#pragma unroll
                  for (int j = 0; j < jn; ++j) {
                    const int gg = i + j;
                    const bool first = kb == 0 && kk == 0 && i == (gg < kND ? 0 : gg - kND + 1);
                    const uint64_t bd = umma_desc_sw64_addr(st_a + kND * kIAPlane + j * kIBPlane) + adv;
                    const uint32_t acc = first ? 0u : 1u;
                    if (j == 0) umma_i8<1>(tmem + gg * kIN, ad, bd, acc);
                    else if (j == jn - 1) umma_i8<3>(tmem + gg * kIN, ad, bd, acc);
                    else umma_i8<2>(tmem + gg * kIN, ad, bd, acc);
                  }
                }
              }
              umma_commit(&sm.empty[s]);
            }
            __syncwarp();
          }
          if (elect_one()) umma_commit(&sm.tmem_full);
          __syncwarp();
        }
  } else {  // ---- epilogue: EW warps; TMEM lane quarter warp % 4, column part (warp - 2) / 4;
            //      thread = one test row x CW of the tile's 64 SVs
    constexpr int EW = i8_epi_warps<KM>(), NP = EW / 4, CW = kIN / NP, ET = 32 * EW;
    const int q = warp & 3, part = (warp - 2) >> 2, et_id = threadIdx.x - 64;  // et_id 0 .. ET - 1
    int it = 0;
    const double tsc = -gamma * 1.4426950408889634074;  // exp(-gamma d2) = 2^(tsc d2)
    for (int u = blockIdx.x; u < n_units; u += gridDim.x) {
      double acc[KM];
#pragma unroll
      for (int v = 0; v < KM; ++v) acc[v] = 0.0;
      int64_t r = 0;
      for (int t = unit_off[u]; t < unit_off[u + 1]; ++t) {
        const int2 tile = tiles[t];
        r = (int64_t)tile.x * kIM + q * 32 + lane;
        const double pr = pow2(-et[r]);  // 2^-e_x
        const double nr = nt[r];
        for (int h = 0; h < 2; ++h, ++it) {
          const int64_t c0 = (int64_t)tile.y * 2 * kIN + h * kIN;
          // this half-tile's SV columns (double buffer): scale, norm and coefficients, staged with
          // shared-memory stores and read back with 16-byte shared loads
          constexpr int ROW = i8_row<KM>();
          const uint32_t cs = smem_u32(&sm.coefS[it & 1][0][0]);
          for (int idx = et_id; idx < kIN * ROW; idx += ET) {
            const int jj = idx / ROW, v = idx - jj * ROW;
            const int64_t c = c0 + jj;
            const double val = v == 0 ? pow2(24 - es[c]) : v == 1 ? ns[c] : (v - 2 < km1 ? coef[c * km1_pad + v - 2] : 0.0);
            asm volatile("st.shared.f64 [%0], %1;" ::"r"(cs + (uint32_t)idx * 8), "d"(val) : "memory");
          }
          asm volatile("bar.sync 1, %0;" ::"r"(ET) : "memory");
          mbar_wait(&sm.tmem_full, it & 1);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          // sum_g 256^(5-g) G_g by 16-column chunks: groups 0-2 and 3-5 combined exactly in int64
          // (|G| < 2^26: |hi|, |lo| < 2^43, exact in FP64), then hi 2^24 + lo in FP64
          const uint32_t taddr = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(part * CW);
          double dot[CW];
          if (diag & 16) {  // GMPSVM_I8_DIAG bit 4 (timing experiments): no TMEM drain
            __syncwarp();
            if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.tmem_empty)) : "memory");
            continue;
          }
#pragma unroll
          for (int ch = 0; ch < CW / 16; ++ch) {
#pragma unroll
            for (int part3 = 0; part3 < 2; ++part3) {
              long long w[16];
              uint32_t v0[16], v1[16], v2[16];  // the three groups' loads in flight together, one wait
              tmem_ld16(taddr + (uint32_t)((part3 * 3 + 0) * kIN + ch * 16), v0);
              tmem_ld16(taddr + (uint32_t)((part3 * 3 + 1) * kIN + ch * 16), v1);
              tmem_ld16(taddr + (uint32_t)((part3 * 3 + 2) * kIN + ch * 16), v2);
              asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
              for (int jj = 0; jj < 16; ++jj)
                w[jj] = ((long long)(int32_t)v0[jj] * 65536 + (long long)(int32_t)v1[jj] * 256) + (int32_t)v2[jj];
#pragma unroll
              for (int jj = 0; jj < 16; ++jj)
                dot[ch * 16 + jj] = part3 == 0 ? i2d_small(w[jj]) : fma(dot[ch * 16 + jj], 16777216.0, i2d_small(w[jj]));
            }
          }
          asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
          __syncwarp();
          if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.tmem_empty)) : "memory");
          // x~.y~ = 2^-(e_x+e_y) 256^3 (hi 2^24 + lo): the 256^3 = 2^24 folds into the exponent
          if (diag & 1) {  // GMPSVM_I8_DIAG bit 0 (timing experiments): no epilogue arithmetic
            acc[0] += dot[0] + dot[CW - 1];
            continue;
          }
          // blocks of BE columns, each step over the BE independent elements (BE chains in flight;
          // 4 when the per-row sums take the registers)
          constexpr int BE = KM > 12 ? 4 : 8;
#pragma unroll
          for (int jb = 0; jb < CW; jb += BE) {
            double tt[BE], ff[BE], pp[BE];
            int nn[BE];
#pragma unroll
            for (int e = 0; e < BE; ++e) {
              double sc, nc;
              asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(sc), "=d"(nc)
                           : "r"(cs + (uint32_t)((part * CW + jb + e) * ROW) * 8));
              const double xy = (dot[jb + e] * pr) * sc;  // powers of two: exact
              const double d2 = fmax(fma(-2.0, xy, nr + nc), 0.0);
              tt[e] = fmax(tsc * d2, -1020.0);  // below 2^-1020 the kernel value is < 1e-307 (not 0)
            }
#pragma unroll
            for (int e = 0; e < BE; ++e) {  // n = rint(t) (round to nearest even) by the 1.5 2^52 shift
              const double big = tt[e] + kShift52;
              const double n = big - kShift52;
              ff[e] = tt[e] - n;  // exact, |f| <= 1/2
              nn[e] = __double2loint(big);
              pp[e] = kExp2C[0];
            }
#pragma unroll
            for (int k = 1; k < 11; ++k)
#pragma unroll
              for (int e = 0; e < BE; ++e) pp[e] = fma(pp[e], ff[e], kExp2C[k]);
#pragma unroll
            for (int e = 0; e < BE; ++e) {
              const double kv = pp[e] * pow2(nn[e]);
              const uint32_t cj = cs + (uint32_t)((part * CW + jb + e) * ROW + 2) * 8;
#pragma unroll
              for (int v = 0; v < KM; v += 2) {
                double c0v, c1v;
                asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(c0v), "=d"(c1v) : "r"(cj + (uint32_t)v * 8));
                acc[v] = fma(kv, c0v, acc[v]);
                if (v + 1 < KM) acc[v + 1] = fma(kv, c1v, acc[v + 1]);
              }
            }
          }
        }
      }
      // the column parts of a row: parts 1 .. NP-1 hand their sums to part 0 in turn (fixed order)
      double* red = &sm.red[0][0];
      for (int p = 1; p < NP; ++p) {
        asm volatile("bar.sync 1, %0;" ::"r"(ET) : "memory");
        if (part == p)
#pragma unroll
          for (int v = 0; v < KM; ++v) red[(q * 32 + lane) * KM + v] = acc[v];
        asm volatile("bar.sync 1, %0;" ::"r"(ET) : "memory");
        if (part == 0)
#pragma unroll
          for (int v = 0; v < KM; ++v) acc[v] += red[(q * 32 + lane) * KM + v];
      }
      if (part == 0) {
        double* out = part_out + ((int64_t)unit_item[u] * m_pad + r) * km1_pad;
#pragma unroll
        for (int v = 0; v < KM; ++v)
          if (v < km1) out[v] = acc[v];
        for (int v = km1; v < km1_pad; ++v) out[v] = 0.0;
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kITmemCols));
  }
}

// planes [kND][rows_pad][d8] int8 as a 2-D tensor (d8 x kND rows_pad), 64-byte swizzle, box 64 x box_rows
CUtensorMap make_map_i8(const void* base, int64_t rows_total, int d8, int box_rows) {
  auto enc = get_encode();
  if (!enc) throw Error(GMPSVM_ECUDA, "cuTensorMapEncodeTiled unavailable");
  CUtensorMap m;
  const cuuint64_t dims[2] = {(cuuint64_t)d8, (cuuint64_t)rows_total};
  const cuuint64_t strides[1] = {(cuuint64_t)d8};
  const cuuint32_t box[2] = {(cuuint32_t)kIK, (cuuint32_t)box_rows};
  const cuuint32_t estr[2] = {1, 1};
  const CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, const_cast<void*>(base), dims, strides, box, estr,
                         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(GMPSVM_ECUDA, "cuTensorMapEncodeTiled (int8) failed: " + std::to_string((int)r));
  return m;
}

}  // namespace

int dec_i8_d8(int d) { return (int)round_up(d, 32); }
size_t dec_i8_plane_bytes(int64_t rows_pad, int d) { return (size_t)kND * rows_pad * dec_i8_d8(d); }
int dec_i8_max_km1() { return 32; }

// Worst-case |K~ - K| of this path for rows of max |x| <= ax, ay (d features, RBF gamma): the
// representation error Delta = ||dx|| + ||dy|| <= sqrt(d) 2^-38 (ax + ay) moves d2 by at most
// 2 r Delta + Delta^2 (r = ||x - y||), and K e^(-gamma r^2) 2 gamma r Delta peaks at
// Delta sqrt(2 gamma) e^(-1/2); the dropped digit groups add <= 2 (3 d 2^-44 ax ay), FP64 rounding
// of the norm combine <= 2^-49 (||x||^2 + ||y||^2) <= 2^-49 d (ax^2 + ay^2), the exp series
// remainder 3.2e-13 and rounding.  (DESIGN.md §3 "decision-value routing".)
double dec_i8_kernel_err(double ax, double ay, int d, double gamma) {
  const double sd = std::sqrt((double)d);
  const double delta = sd * std::ldexp(1.0, -38) * (ax + ay);
  const double ed2 = delta * delta + 6.0 * d * std::ldexp(1.0, -44) * ax * ay +
                     std::ldexp(1.0, -49) * d * (ax * ax + ay * ay);
  // + exp2_neg's series remainder (< 3.2e-13 relative, K <= 1) and rounding
  return delta * std::sqrt(2.0 * gamma) * std::exp(-0.5) + gamma * ed2 + 5e-13;
}

void launch_stage_i8(const float* X, int64_t n, int d, const int64_t* src, int8_t* planes, int64_t rows_pad,
                     int32_t* ex, double* nrm, unsigned* amax, cudaStream_t st) {
  GM_LAUNCH(stage_i8_kernel, dim3((unsigned)ceil_div(rows_pad, 8)), dim3(256), 0, st, X, n, d, src, planes, rows_pad,
            dec_i8_d8(d), ex, nrm, amax);
}

void launch_dec_i8(const int8_t* tplanes, int64_t m_pad, const int32_t* et, const double* nt, const int8_t* splanes,
                   int64_t nsv_pad, const int32_t* es, const double* ns, int d, const int2* tiles,
                   const int32_t* unit_off, const int32_t* unit_item, int n_units, const double* coef64, int km1,
                   int km1_pad, double gamma, double* part, cudaStream_t st) {
  const int d8 = dec_i8_d8(d);
  const CUtensorMap mt = make_map_i8(tplanes, (int64_t)kND * m_pad, d8, kIM);
  const CUtensorMap ms = make_map_i8(splanes, (int64_t)kND * nsv_pad, d8, kIN);
  int dev = 0, sms = 148;
  GM_CUDA(cudaGetDevice(&dev));
  GM_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  const int grid = n_units < sms ? n_units : sms;
  static const int diag = getenv("GMPSVM_I8_DIAG") ? atoi(getenv("GMPSVM_I8_DIAG")) : 0;
  auto go = [&](auto kern, size_t smem, int threads) {
    set_max_dyn_smem(kern, smem);
    GM_LAUNCH(kern, dim3(grid), dim3(threads), smem, st, mt, ms, tiles, unit_off, unit_item, n_units, et, nt, es, ns,
              coef64, km1, km1_pad, d8, m_pad, nsv_pad, gamma, part, diag);
  };
  // KM: pair columns contracted per SV, the smallest instantiation >= k - 1
  if (km1 <= 2) go(dec_i8_kernel<2>, sizeof(DecI8Smem<2>) + 1024, i8_threads<2>());
  else if (km1 <= 4) go(dec_i8_kernel<4>, sizeof(DecI8Smem<4>) + 1024, i8_threads<4>());
  else if (km1 <= 9) go(dec_i8_kernel<9>, sizeof(DecI8Smem<9>) + 1024, i8_threads<9>());
  else if (km1 <= 12) go(dec_i8_kernel<12>, sizeof(DecI8Smem<12>) + 1024, i8_threads<12>());
  else if (km1 <= 25) go(dec_i8_kernel<25>, sizeof(DecI8Smem<25>) + 1024, i8_threads<25>());
  else if (km1 <= 32) go(dec_i8_kernel<32>, sizeof(DecI8Smem<32>) + 1024, i8_threads<32>());
  else throw Error(GMPSVM_ENOTIMPL, "int8 decision values support k <= 33");
}

}  // namespace gmpsvm
