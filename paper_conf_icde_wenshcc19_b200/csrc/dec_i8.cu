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
constexpr int kIThreads = 192;
constexpr int kIExp = 37;                 // max |x| 2^e in [2^37, 2^38)
// kind::i8, D S32 (2), A S8 (1), B S8 (1), K-major, N = 64, M = 128
constexpr uint32_t kIdescI8 =
    (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(kIN >> 3) << 17) | ((uint32_t)(kIM >> 4) << 24);

template <int KM>
struct DecI8Smem {
  alignas(1024) uint8_t stage[kIStages][kIStageBytes];
  alignas(16) double coefS[2][kIN][KM];
  alignas(8) uint64_t full[kIStages];
  uint64_t empty[kIStages];
  uint64_t tmem_full;
  uint64_t tmem_empty;
  uint32_t tmem_base;
};

// K-major operand, 64-byte swizzle: 8-row groups 512 B apart (SBO), LBO unused, version 1
__device__ __forceinline__ uint64_t umma_desc_sw64(const void* p) {
  const uint64_t addr = smem_u32(p);
  uint64_t d = 0;
  d |= (addr >> 4) & 0x3FFFull;
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)(512 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)4 << 61;  // SWIZZLE_64B
  return d;
}
__device__ __forceinline__ void umma_i8(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t accum) {
  asm volatile(
      "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n}\n" ::"r"(
          tmem_d),
      "l"(a), "l"(b), "r"(kIdescI8), "r"(accum));
}
__device__ __forceinline__ double pow2(int k) { return __hiloint2double((k + 1023) << 20, 0); }  // 2^k, |k| < 1023

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
__global__ void __launch_bounds__(kIThreads, 1)
    dec_i8_kernel(const __grid_constant__ CUtensorMap map_t, const __grid_constant__ CUtensorMap map_s,
                  const int2* __restrict__ tiles, const int32_t* __restrict__ unit_off,
                  const int32_t* __restrict__ unit_item, int n_units, const int32_t* __restrict__ et,
                  const double* __restrict__ nt, const int32_t* __restrict__ es, const double* __restrict__ ns,
                  const double* __restrict__ coef, int km1, int km1_pad, int d8, int64_t m_pad, int64_t nsv_pad,
                  double gamma, double* __restrict__ part) {
  extern __shared__ __align__(1024) uint8_t dsmem[];
  DecI8Smem<KM>& sm =
      *reinterpret_cast<DecI8Smem<KM>*>((reinterpret_cast<uintptr_t>(dsmem) + 1023) & ~uintptr_t(1023));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nk = (d8 + kIK - 1) / kIK;
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < kIStages; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], 1);
    }
    mbar_init(&sm.tmem_full, 1);
    mbar_init(&sm.tmem_empty, 4);
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
              const int s = g % kIStages;
              if (g >= kIStages) mbar_wait(&sm.empty[s], ((g / kIStages) + 1) & 1);
              uint8_t* st = sm.stage[s];
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
    if (lane == 0) {  // ---- MMA issuer: group g = i + j of the digit products into accumulator g
      int g = 0, it = 0;
      for (int u = blockIdx.x; u < n_units; u += gridDim.x)
        for (int t = unit_off[u]; t < unit_off[u + 1]; ++t)
          for (int h = 0; h < 2; ++h, ++it) {
            if (it > 0) mbar_wait(&sm.tmem_empty, (it - 1) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            for (int kb = 0; kb < nk; ++kb, ++g) {
              const int s = g % kIStages;
              mbar_wait(&sm.full[s], (g / kIStages) & 1);
              asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
              uint8_t* st = sm.stage[s];
              const int nsub = min(2, (d8 - kb * kIK + 31) / 32);  // valid 32-wide k steps (d8 % 32 == 0)
              for (int kk = 0; kk < nsub; ++kk) {
                const uint64_t adv = (uint64_t)(kk * 32) >> 4;
#pragma unroll
                for (int gg = 0; gg < kNG; ++gg) {
#pragma unroll
                  for (int i = 0; i < kND; ++i) {
                    const int j = gg - i;
                    if (j < 0 || j >= kND) continue;
                    const bool first = kb == 0 && kk == 0 && i == (gg < kND ? 0 : gg - kND + 1);
                    umma_i8(tmem + gg * kIN, umma_desc_sw64(st + i * kIAPlane) + adv,
                            umma_desc_sw64(st + kND * kIAPlane + j * kIBPlane) + adv, first ? 0u : 1u);
                  }
                }
              }
              umma_commit(&sm.empty[s]);
            }
            umma_commit(&sm.tmem_full);
          }
    }
  } else {  // ---- epilogue: warps 2..5 (TMEM lane quarter warp % 4), thread = one test row
    const int q = warp & 3, et_id = threadIdx.x - 64;  // 0..127
    int it = 0;
    const double ng = -gamma;
    for (int u = blockIdx.x; u < n_units; u += gridDim.x) {
      double acc[KM];
#pragma unroll
      for (int v = 0; v < KM; ++v) acc[v] = 0.0;
      int64_t r = 0;
      for (int t = unit_off[u]; t < unit_off[u + 1]; ++t) {
        const int2 tile = tiles[t];
        r = (int64_t)tile.x * kIM + q * 32 + lane;
        const int ex_r = et[r];
        const double nr = nt[r];
        for (int h = 0; h < 2; ++h, ++it) {
          const int64_t c0 = (int64_t)tile.y * 2 * kIN + h * kIN;
          double* cs = &sm.coefS[it & 1][0][0];  // this half-tile's coefficients (double buffer)
          for (int idx = et_id; idx < kIN * KM; idx += 128) {
            const int jj = idx / KM, v = idx - jj * KM;
            cs[idx] = v < km1_pad ? coef[(c0 + jj) * km1_pad + v] : 0.0;
          }
          asm volatile("bar.sync 1, 128;" ::: "memory");
          mbar_wait(&sm.tmem_full, it & 1);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          double dot[kIN];  // sum_g 256^(5-g) G_g (exact integers up to rounding in the last adds)
#pragma unroll
          for (int ch = 0; ch < kIN / 32; ++ch) {
            const uint32_t taddr = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(ch * 32);
#pragma unroll
            for (int gg = 0; gg < kNG; ++gg) {
              uint32_t v[32];
              tmem_ld32(taddr + gg * kIN, v);
              asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
              const double w = pow2(8 * (kNG - 1 - gg));
#pragma unroll
              for (int jj = 0; jj < 32; ++jj) {
                const double gv = (double)(int32_t)v[jj];
                dot[ch * 32 + jj] = gg == 0 ? gv * w : fma(gv, w, dot[ch * 32 + jj]);
              }
            }
          }
          asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
          __syncwarp();
          if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.tmem_empty)) : "memory");
          // x~.y~ = 2^-(e_x+e_y) 256^3 dot: the 256^3 = 2^24 folds into the exponent
#pragma unroll
          for (int jj = 0; jj < kIN; ++jj) {
            const int64_t c = c0 + jj;
            const double xy = dot[jj] * pow2(24 - ex_r - __ldg(es + c));
            const double d2 = fmax(nr + __ldg(ns + c) - 2.0 * xy, 0.0);
            const double kv = exp(ng * d2);
            const double* cj = cs + jj * KM;
#pragma unroll
            for (int v = 0; v < KM; ++v) acc[v] = fma(kv, cj[v], acc[v]);
          }
        }
      }
      double* out = part + ((int64_t)unit_item[u] * m_pad + r) * km1_pad;
#pragma unroll
      for (int v = 0; v < KM; ++v)
        if (v < km1_pad) out[v] = v < km1 ? acc[v] : 0.0;
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
// of the norm combine <= 2^-49 (||x||^2 + ||y||^2) <= 2^-49 d (ax^2 + ay^2), exp and the products
// a few ulps.  (DESIGN.md §3 "decision-value routing".)
double dec_i8_kernel_err(double ax, double ay, int d, double gamma) {
  const double sd = std::sqrt((double)d);
  const double delta = sd * std::ldexp(1.0, -38) * (ax + ay);
  const double ed2 = delta * delta + 6.0 * d * std::ldexp(1.0, -44) * ax * ay +
                     std::ldexp(1.0, -49) * d * (ax * ax + ay * ay);
  return delta * std::sqrt(2.0 * gamma) * std::exp(-0.5) + gamma * ed2 + std::ldexp(1.0, -48);
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
  auto go = [&](auto kern, size_t smem) {
    set_max_dyn_smem(kern, smem);
    GM_LAUNCH(kern, dim3(grid), dim3(kIThreads), smem, st, mt, ms, tiles, unit_off, unit_item, n_units, et, nt, es, ns,
              coef64, km1, km1_pad, d8, m_pad, nsv_pad, gamma, part);
  };
  if (km1_pad <= 4) go(dec_i8_kernel<4>, sizeof(DecI8Smem<4>) + 1024);
  else if (km1_pad <= 12) go(dec_i8_kernel<12>, sizeof(DecI8Smem<12>) + 1024);
  else if (km1_pad <= 32) go(dec_i8_kernel<32>, sizeof(DecI8Smem<32>) + 1024);
  else throw Error(GMPSVM_ENOTIMPL, "int8 decision values support k <= 33");
}

}  // namespace gmpsvm
