// krow_tc.cu -- a2 (and the a10 decision values) on the 5th-generation tensor cores: the
// kernel-value contraction with a hi/lo split of every operand, x = hi + lo, so that
//   x.y ~= hi.hi + hi.lo + lo.hi   (the lo.lo term is below FP32 rounding)
// is accumulated in FP32 in TMEM by tcgen05.mma, operands staged by TMA into 128-byte-swizzled
// shared memory.  The epilogue (norm combine, clamp, ex2, K_ii = 1, symmetric mirrored store) is
// the same arithmetic as krow.cu's SIMT kernel.
//
// Default split: FP16 (kind::f16).  The rows are centred by the column means and scaled by an
// exact power of two s (max |x - mu| s <= 2^12, inside FP16's range and away from its
// subnormals); hi = half(x'), lo = half(x' - hi), both round-to-nearest: 11 significant bits
// per part, so hi + lo carries x' to ~2^-22.  Distances are computed in scaled units and the exp
// argument is divided by s^2 (exact).  GMPSVM_SPLIT=tf32 selects the TF32 split (kind::tf32, the
// same precision at half the MMA rate).
//
// CTA tile 128 x 128, persistent CTAs walking the tiles (bi, bj) of the upper triangle; warp 0 =
// TMA producer, warp 1 = MMA issuer (+ TMEM allocation), warps 2..5 = epilogue (one TMEM lane
// quarter each); 3-stage smem ring of 64 KB (A hi/lo and B hi/lo, 128 rows x one 128-byte
// swizzle atom along K each: 64 FP16 or 32 TF32 elements).  TMEM holds four 128-column FP32
// accumulators: hi.hi over each third of the k range, and hi.lo + lo.hi.
// Entry (r, c) is written, with its mirror (c, r), only by the tile that holds it with r <= c.
#include <cuda.h>
#include <cuda_fp16.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "kernels.h"
#include "solver_dev.cuh"
#include "tc_util.cuh"

namespace gmpsvm {

namespace {

constexpr int kTM = 128, kTN = 128, kTK = 32;  // tile rows, columns, k-step (one 128 B swizzle atom)
constexpr int kTcStages = 3;
constexpr int kMainAcc = 3;  // hi.hi accumulators (k range split in thirds)
constexpr int kTcThreads = 192;
constexpr uint32_t kABytes = kTM * kTK * 4;            // 16 KB
constexpr uint32_t kBBytes = kTN * kTK * 4;            // 16 KB
constexpr uint32_t kStageBytes = 2 * kABytes + 2 * kBBytes;  // 64 KB
constexpr uint32_t kTmemCols = 512;  // 3 x 128 hi.hi (k thirds) + 128 hi.lo + lo.hi
constexpr int kDecMaxKm1 = 32;       // dec_tc: pair columns per SV (k - 1, padded), k <= 33

constexpr int kEpiWarps = 4;
struct TcSmem {
  // each operand tile 1024-byte aligned (128B swizzle atoms)
  alignas(1024) uint8_t stage[kTcStages][kStageBytes];
  // epilogue staging for the TMA stores, per epilogue warp: [0] its 32 x 32 block of K (rows r,
  // columns c, 128-byte swizzled), [1] the mirrored block (rows c, columns r)
  alignas(1024) float epi[kEpiWarps][2][32 * 32];
  alignas(8) uint64_t full[kTcStages];
  uint64_t empty[kTcStages];
  uint64_t tmem_full;
  uint64_t tmem_empty;
  uint64_t tmem_empty2;
  uint32_t tmem_base;
};

// kind::tf32 / kind::f16, A/B K-major, D F32, M = 128, N = 128 (a/b format 2 = TF32, 0 = F16)
constexpr uint32_t kIdesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(kTN >> 3) << 17) | ((uint32_t)(kTM >> 4) << 24);
constexpr uint32_t kIdescF16 = (1u << 4) | ((uint32_t)(kTN >> 3) << 17) | ((uint32_t)(kTM >> 4) << 24);

// COL: A-operand collector (kind::f16 only): 0 none, 1 fill (keep A for the next MMA), 3 lastuse.
// hi.hi and hi.lo share the A tile (hi): issued back to back, the second reuses the collector and
// the tensor core reads A from shared memory once for both
template <bool F16, int COL = 0>
__device__ __forceinline__ void umma_hilo(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t accum) {
  if (F16 && COL == 1)
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::f16.collector::a::fill [%0], %1, %2, "
        "%3, p;\n}\n" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(kIdescF16), "r"(accum));
  else if (F16 && COL == 3)
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::f16.collector::a::lastuse [%0], %1, "
        "%2, %3, p;\n}\n" ::"r"(tmem_d),
        "l"(a), "l"(b), "r"(kIdescF16), "r"(accum));
  else if (F16)
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(
            tmem_d),
        "l"(a), "l"(b), "r"(kIdescF16), "r"(accum));
  else
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(
            tmem_d),
        "l"(a), "l"(b), "r"(kIdesc), "r"(accum));
}
// the three products of one k step: hi.hi into accumulator j, hi.lo + lo.hi into the corrections
template <bool F16, bool COLLECT>
__device__ __forceinline__ void umma_split3(uint32_t dj, uint32_t dc, uint64_t ahi, uint64_t alo, uint64_t bhi,
                                            uint64_t blo, uint32_t acc_j, uint32_t acc_c) {
  if (F16 && COLLECT) {
    umma_hilo<true, 1>(dj, ahi, bhi, acc_j);
    umma_hilo<true, 3>(dc, ahi, blo, acc_c);
  } else {
    umma_hilo<F16>(dj, ahi, bhi, acc_j);
    umma_hilo<F16>(dc, ahi, blo, acc_c);
  }
  umma_hilo<F16>(dc, alo, bhi, 1u);
}
// The paper's other kernels (L76-L78, NEXT-4) on the same contraction: with uncentred rows the
// tensor cores deliver s^2 x . y; K = x.y, (gamma x.y + coef0)^degree or tanh(gamma x.y + coef0).
template <int KT>  // 1 linear, 2 polynomial, 3 sigmoid
__device__ __forceinline__ float dot_kernel_value(float xy, const KrowKernel& kp) {
  if (KT == 1) return xy;
  const float z = fmaf(kp.gamma, xy, kp.coef0);
  if (KT == 3) return tanhf(z);
  float v = 1.f, b = z;  // z^degree by squaring, degree <= 16: no data-dependent loop in the epilogue
  int e = kp.degree;
#pragma unroll
  for (int i = 0; i < 5; ++i) {
    if (e & 1) v *= b;
    b *= b;
    e >>= 1;
  }
  return v;
}

// Persistent: one CTA per SM walks the tile list (tile = blockIdx.x + i * gridDim.x).  The TMA
// producer runs ahead across tile boundaries through the smem ring; the epilogue drains the four
// TMEM accumulators into registers and releases TMEM at once (tmem_empty), so the MMAs of the
// next tile overlap the exp + stores of the current one.
//
// MC (2-CTA cluster, krow_tc_mc): the tile list holds pairs of tiles of the same row block --
// entries 2p and 2p + 1 go to cluster p's CTA 0 and 1 (a second entry with y < 0 is a dummy: its
// CTA runs the pipeline on valid rows and stores nothing).  Each CTA loads half of the shared A
// rows (hi and lo) and multicasts it to both CTAs, and its own B rows: 48 instead of 64 KB per
// k-step leave L2 for each SM.  The MMA commits free a ring stage in both CTAs (empty barriers
// count two arrivals), so neither producer overwrites a stage its peer still reads.
// kk_last: MMAs (K = 16) of the last k-step that touch real columns -- the rest multiply the zero
// padding of d (784 -> 832 for MNIST-shaped rows) and are skipped (same sums, bit for bit).
template <bool F16, int KT, bool MC = false>  // KT: 0 the Gaussian, else a dot-product kernel (kp): 1 linear, 2 poly, 3 sigmoid
__global__ void __launch_bounds__(kTcThreads, 1)
    krow_tc_kernel(const __grid_constant__ CUtensorMap map_hi, const __grid_constant__ CUtensorMap map_lo,
                   const __grid_constant__ CUtensorMap map_ksw, const __grid_constant__ CUtensorMap map_kns,
                   const int2* __restrict__ tiles, int n_tiles, const float* __restrict__ norms, int64_t n, int nk,
                   float scale, float* __restrict__ K, int64_t ldk, int tma_store, KrowKernel kp,
                   const __grid_constant__ CUtensorMap map_hi64, const __grid_constant__ CUtensorMap map_lo64, int kk_last) {
  extern __shared__ __align__(1024) uint8_t dsmem[];
  TcSmem& sm = *reinterpret_cast<TcSmem*>((reinterpret_cast<uintptr_t>(dsmem) + 1023) & ~uintptr_t(1023));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // the CTA's tiles: entry t0, t0 + tstep, ... of the list
  const int crank = MC ? (int)cluster_ctarank() : 0;
  const int t0 = MC ? 2 * (int)(blockIdx.x >> 1) + crank : (int)blockIdx.x;
  const int tstep = (int)gridDim.x;  // MC: gridDim.x / 2 clusters x 2 entries

  if (warp == 0 && lane == 0) {
    if (kp.resident) atomicAdd(kp.resident, 1ull);  // this CTA holds its SM (engine.cu lead mode)
    for (int s = 0; s < kTcStages; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], MC ? 2 : 1);
    }
    mbar_init(&sm.tmem_full, 1);
    mbar_init(&sm.tmem_empty, 4);   // one arrive per epilogue warp: accumulators 0 and 3 drained
    mbar_init(&sm.tmem_empty2, 4);  // accumulators 1 and 2 drained
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map_hi)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map_lo)) : "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&sm.tmem_base)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  if (MC) cluster_sync();  // both CTAs' barriers initialised before any multicast or remote arrive
  const uint32_t tmem = sm.tmem_base;
  const int jn = nk < kMainAcc ? nk : kMainAcc;  // hi.hi accumulators in use (short k ranges)

  if (warp == 0) {
    if (lane == 0) {  // ---- TMA producer (runs ahead across tiles)
      int g = 0;
      const uint64_t pol = policy_evict_last();
      for (int t = t0; t < n_tiles; t += tstep) {
        const int2 tile = tiles[t];
        const int r0 = tile.x * kTM, c0 = (tile.y < 0 ? tile.x : tile.y) * kTN;  // dummy: valid rows, no stores
        for (int kb = 0; kb < nk; ++kb, ++g) {
          const int s = g % kTcStages;
          if (g >= kTcStages) mbar_wait(&sm.empty[s], ((g / kTcStages) + 1) & 1);
          uint8_t* st = sm.stage[s];
          mbar_expect_tx(&sm.full[s], kStageBytes);
          const int kx = kb * (F16 ? 2 * kTK : kTK);
          if (MC) {  // half of the A rows from each CTA, to both
            const uint32_t ho = (uint32_t)crank * (kABytes / 2);
            tma_load_2d_mc(st + ho, &map_hi64, kx, r0 + crank * (kTM / 2), &sm.full[s], (uint16_t)3, pol);
            tma_load_2d_mc(st + kABytes + ho, &map_lo64, kx, r0 + crank * (kTM / 2), &sm.full[s], (uint16_t)3, pol);
          } else {
            tma_load_2d(st, &map_hi, kx, r0, &sm.full[s], pol);
            tma_load_2d(st + kABytes, &map_lo, kx, r0, &sm.full[s], pol);
          }
          tma_load_2d(st + 2 * kABytes, &map_hi, kx, c0, &sm.full[s], pol);
          tma_load_2d(st + 2 * kABytes + kBBytes, &map_lo, kx, c0, &sm.full[s], pol);
        }
      }
    }
  } else if (warp == 1) {
    // ---- MMA issuer: the whole warp runs the loop (warp-uniform: descriptors and TMEM addresses
    // in uniform registers) and one elected lane issues -- from a lone lane-0 thread every MMA went
    // through an ELECT / R2UR.BROADCAST / BRA.U.ANY sequence (dec_i8.cu)
    int g = 0, it = 0;
    for (int t = t0; t < n_tiles; t += tstep, ++it) {
      if (it > 0) mbar_wait(&sm.tmem_empty, (it - 1) & 1);  // epilogue drained the previous tile
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      for (int kb = 0; kb < nk; ++kb, ++g) {
        const int s = g % kTcStages;
        mbar_wait(&sm.full[s], (g / kTcStages) & 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        uint8_t* st = sm.stage[s];
        const uint64_t ahi = umma_desc_sw128(st), alo = umma_desc_sw128(st + kABytes);
        const uint64_t bhi = umma_desc_sw128(st + 2 * kABytes), blo = umma_desc_sw128(st + 2 * kABytes + kBBytes);
        // the FP32 accumulation error of the tensor-core adds grows with the number of MMAs into
        // an accumulator times its magnitude: the hi.hi
        // products of each k third and the small corrections get accumulators of their own
        const int j = (kb * jn) / nk;
        const int kb_first = (j * nk + jn - 1) / jn;
        // the epilogue releases accumulators 0 + 3 first (the next tile starts with them) and 1 + 2
        // after: the second half of its drain overlaps this tile's first k third
        if (it > 0 && j == 1 && kb == kb_first) {
          mbar_wait(&sm.tmem_empty2, (it - 1) & 1);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        }
        if (elect_one()) {
          const int nkk = kb == nk - 1 ? kk_last : kTK / 8;
#pragma unroll
          for (int kk = 0; kk < kTK / 8; ++kk) {
            const uint64_t adv = (uint64_t)(kk * 32) >> 4;  // 8 TF32 = 32 bytes along K inside the atom
            if (kk < nkk)
              umma_split3<F16, true>(tmem + j * kTN, tmem + kMainAcc * kTN, ahi + adv, alo + adv, bhi + adv,
                                     blo + adv, (kb == kb_first && kk == 0) ? 0u : 1u, (kb | kk) ? 1u : 0u);
          }
          if (MC) umma_commit_mc(&sm.empty[s], (uint16_t)3);  // the stage is free in both CTAs
          else umma_commit(&sm.empty[s]);
        }
        __syncwarp();
      }
      if (elect_one()) umma_commit(&sm.tmem_full);
      __syncwarp();
    }
  } else {  // ---- epilogue: warps 2..5, TMEM lane quarter (warp % 4)
    const int q = warp & 3;
    const uint64_t spol = policy_evict_first();
    int it = 0;
    for (int t = t0; t < n_tiles; t += tstep, ++it) {
      const int2 tile = tiles[t];
      if (MC && tile.y < 0) {  // dummy partner tile: release the accumulators, store nothing
        mbar_wait(&sm.tmem_full, it & 1);
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncwarp();
        if (lane == 0) {
          asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.tmem_empty)) : "memory");
          asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.tmem_empty2)) : "memory");
        }
        continue;
      }
      const int64_t r0 = (int64_t)tile.x * kTM, c0 = (int64_t)tile.y * kTN;
      const int64_t r = r0 + q * 32 + lane;
      const float nr = (r < n) ? norms[r] : 0.f;
      float cnv[kTN / 32];  // column norms of the tile (lane holds column c0 + 32 ch + lane), loaded early
#pragma unroll
      for (int ch = 0; ch < kTN / 32; ++ch) cnv[ch] = norms[c0 + ch * 32 + lane];  // n_pad >= c0 + 128 (zero padded)
      mbar_wait(&sm.tmem_full, it & 1);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      float dot[kTN];
      const uint32_t trow = tmem + ((uint32_t)(q * 32) << 16);
#pragma unroll
      for (int ch = 0; ch < kTN / 32; ++ch) {  // accumulators 0 (first k third) and 3 (corrections)
        uint32_t v0[32], w[32];
        tmem_ld32(trow + (uint32_t)(ch * 32), v0);
        tmem_ld32(trow + (uint32_t)(ch * 32) + kMainAcc * kTN, w);
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
        for (int j = 0; j < 32; ++j) dot[ch * 32 + j] = __uint_as_float(v0[j]) + __uint_as_float(w[j]);
      }
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.tmem_empty)) : "memory");
      if (nk > 1) {
#pragma unroll
        for (int ch = 0; ch < kTN / 32; ++ch) {  // accumulators 1 and 2 (second and third k thirds)
          uint32_t v1[32], v2[32];
          tmem_ld32(trow + (uint32_t)(ch * 32) + kTN, v1);
          tmem_ld32(trow + (uint32_t)(ch * 32) + 2 * kTN, v2);
          asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            float x = dot[ch * 32 + j] + __uint_as_float(v1[j]);
            if (nk > 2) x += __uint_as_float(v2[j]);
            dot[ch * 32 + j] = x;
          }
        }
      }
      // TMEM may be overwritten by the next tile's MMAs from here on
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.tmem_empty2)) : "memory");
      if (tma_store && tile.x != tile.y) {
        // off-diagonal tile (every r < c): the 128 x 128 block and its mirror leave through shared
        // memory as full-line TMA stores (one 32 x 32 block pair per warp and column chunk; rows /
        // columns >= n are clipped by the tensor maps)
        float* eb = sm.epi[q][0];
        float* em = sm.epi[q][1];
#pragma unroll
        for (int ch = 0; ch < kTN / 32; ++ch) {
          const int64_t cb = c0 + ch * 32;
          const float cn = cnv[ch];
          float kv[32];
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            if (KT != 0) {
              kv[j] = dot_kernel_value<KT>(dot[ch * 32 + j] * kp.inv_s2, kp);
            } else {
              const float d2 = fmaf(-2.f, dot[ch * 32 + j], nr + __shfl_sync(0xffffffffu, cn, j));
              asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(kv[j]) : "f"(fmaxf(d2, 0.f) * scale));
            }
          }
          if (lane == 0) bulk_wait_read0();  // the previous chunk's stores have read the staging
          __syncwarp();
#pragma unroll
          for (int jj = 0; jj < 8; ++jj)  // row `lane`, 16-byte chunk jj at jj ^ (row % 8) (128B swizzle)
            *reinterpret_cast<float4*>(eb + lane * 32 + ((jj ^ (lane & 7)) << 2)) =
                make_float4(kv[4 * jj], kv[4 * jj + 1], kv[4 * jj + 2], kv[4 * jj + 3]);
#pragma unroll
          for (int j = 0; j < 32; ++j) em[j * 32 + lane] = kv[j];
          fence_proxy_async_smem();
          __syncwarp();
          if (lane == 0) {
            tma_store_2d_hint(&map_ksw, eb, (int)cb, (int)(r0 + q * 32), spol);
            tma_store_2d_hint(&map_kns, em, (int)(r0 + q * 32), (int)cb, spol);
            bulk_commit();
          }
        }
        continue;
      }
#pragma unroll
      for (int ch = 0; ch < kTN / 32; ++ch) {
        const int64_t cb = c0 + ch * 32;
        float kv[32];
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          if (KT != 0) {
            kv[j] = dot_kernel_value<KT>(dot[ch * 32 + j] * kp.inv_s2, kp);  // K_ii computed (not 1)
          } else {
            const float d2 = fmaf(-2.f, dot[ch * 32 + j], nr + __shfl_sync(0xffffffffu, cnv[ch], j));
            float val;
            asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(val) : "f"(fmaxf(d2, 0.f) * scale));
            kv[j] = (r == cb + j) ? 1.f : val;
          }
        }
        // direct store K[r][c] for r <= c (row segment of 32 contiguous floats)
        if (r < n) {
          float* dst = K + r * ldk + cb;
          const bool full = (cb >= r) && (cb + 31 < n) && ((ldk & 3) == 0);
          if (full) {
#pragma unroll
            for (int j = 0; j < 32; j += 4)
              *reinterpret_cast<float4*>(dst + j) = make_float4(kv[j], kv[j + 1], kv[j + 2], kv[j + 3]);
          } else {
#pragma unroll
            for (int j = 0; j < 32; ++j)
              if (cb + j >= r && cb + j < n) dst[j] = kv[j];
          }
        }
        // mirrored store K[c][r] for r < c (warp-coalesced: lanes hold consecutive rows)
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          const int64_t c = cb + j;
          if (r < c && c < n) K[c * ldk + r] = kv[j];
        }
      }
    }
    if (lane == 0) bulk_wait0();  // every TMA store of this warp complete before the CTA exits
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (MC) cluster_sync();  // the peer's multicasts and commit arrivals into this CTA are done
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
  }
}

// ------------------------------------------------------------------------------------------
// The same contraction on CTA pairs (cluster of 2, tcgen05 cta_group::2): one MMA computes a
// 256 x 128 tile; CTA r holds rows 128 r .. 128 r + 127 of A (its own 128 rows, hi and lo) and
// rows 64 r .. 64 r + 63 of B, so per SM an MMA reads 4 KB of A + 2 KB of B from shared memory
// instead of 4 + 4 KB, and each SM's TMA fills 12 instead of 16 KB per k step: the shared-memory
// operand bandwidth that bounds the single-CTA kernel drops by a quarter.  The leader (rank 0)
// issues the MMAs; its full barriers count both CTAs' TMA bytes, its MMA commits arrive on both
// CTAs' empty / tmem_full barriers (multicast), and both CTAs' epilogue warps release TMEM on the
// leader's tmem_empty barriers.  Accumulators: CTA r's TMEM lanes hold its 128 rows (same layout
// as the single-CTA kernel), so the epilogue is unchanged per CTA.  Tile (I, J) covers rows
// 256 I .. 256 I + 255 and columns 128 J .. 128 J + 127; CTA r's 128 x 128 half is the
// single-CTA tile (2 I + r, J): stored by TMA when off-diagonal, per thread on the diagonal,
// not at all when below it (computed, discarded: one half-tile per diagonal).
constexpr int kTc2Stages = 4;
constexpr uint32_t kBHalfBytes = (kTN / 2) * 128;              // 64 rows x 128 B = 8 KB
constexpr uint32_t kStage2Bytes = 2 * kABytes + 2 * kBHalfBytes;  // 48 KB
constexpr uint32_t kIdescF16M256 = (1u << 4) | ((uint32_t)(kTN >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
constexpr uint32_t kPeerMask = 0xFEFFFFFFu;  // shared::cluster address of the same offset in CTA rank 0

struct Tc2Smem {
  alignas(1024) uint8_t stage[kTc2Stages][kStage2Bytes];
  alignas(1024) float epi[kEpiWarps][2][32 * 32];
  alignas(8) uint64_t full[kTc2Stages];  // leader: TMA bytes of both CTAs
  uint64_t empty[kTc2Stages];            // both: MMA commit (multicast)
  uint64_t acc_ready[2];                 // both: MMA commit after the first / second k third (multicast)
  uint64_t tmem_full;                    // both: MMA commit after the last MMA of the tile (multicast)
  uint64_t free03;                       // leader: 8 epilogue warps (both CTAs) drained accumulators 0 and 3
  uint64_t free1;                        // leader: accumulator 1 drained
  uint64_t free2;                        // leader: accumulator 2 drained
  uint32_t tmem_base;
};

__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t mapa_rank(uint32_t addr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
  return r;
}
__device__ __forceinline__ void tma_load_2d_2sm(void* dst, const CUtensorMap* map, int x, int y, uint64_t* bar,
                                                uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], "
      "[%1, {%2, %3}], [%4], %5;" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(smem_u32(bar) & kPeerMask), "l"(policy)
      : "memory");
}
__device__ __forceinline__ void umma_f16_2sm(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t accum) {
  asm volatile(
      "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(
          tmem_d),
      "l"(a), "l"(b), "r"(kIdescF16M256), "r"(accum));
}
__device__ __forceinline__ void umma_commit_2sm(uint64_t* bar) {  // arrive on the barrier at this offset in both CTAs
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"((uint16_t)3)
      : "memory");
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kTcThreads, 1)
    krow_tc2_kernel(const __grid_constant__ CUtensorMap map_hi, const __grid_constant__ CUtensorMap map_lo,
                    const __grid_constant__ CUtensorMap map_bhi, const __grid_constant__ CUtensorMap map_blo,
                    const __grid_constant__ CUtensorMap map_ksw, const __grid_constant__ CUtensorMap map_kns,
                    const int2* __restrict__ tiles, int n_tiles, const float* __restrict__ norms, int64_t n, int nk,
                    float scale, float* __restrict__ K, int64_t ldk, int diag) {
  // diag (GMPSVM_KROW_DIAG, timing experiments only): 1 = no stores, 2 = no MMAs, 4 = drain every
  // accumulator at the tile's end
  const bool late = (diag & 4) != 0;
  extern __shared__ __align__(1024) uint8_t dsmem[];
  Tc2Smem& sm = *reinterpret_cast<Tc2Smem*>((reinterpret_cast<uintptr_t>(dsmem) + 1023) & ~uintptr_t(1023));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_rank();
  const bool leader = rank == 0;
  const int cl = blockIdx.x >> 1, ncl = gridDim.x >> 1;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < kTc2Stages; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], 1);
    }
    mbar_init(&sm.acc_ready[0], 1);
    mbar_init(&sm.acc_ready[1], 1);
    mbar_init(&sm.tmem_full, 1);
    mbar_init(&sm.free03, 2 * kEpiWarps);
    mbar_init(&sm.free1, 2 * kEpiWarps);
    mbar_init(&sm.free2, 2 * kEpiWarps);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map_hi)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map_lo)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map_bhi)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map_blo)) : "memory");
  }
  if (warp == 1) {  // same warp in both CTAs, same destination offset (cta_group::2 allocation)
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&sm.tmem_base)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  cluster_sync_all();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = sm.tmem_base;
  int jn = nk < kMainAcc ? nk : kMainAcc;
  if ((diag & 16) && jn > 1) jn = 1;  // precision experiments: one or two hi.hi accumulators
  if ((diag & 32) && jn > 2) jn = 2;

  if (warp == 0) {
    if (lane == 0) {  // ---- TMA producer (both CTAs): own A rows, own half of the B rows
      int g = 0;
      const uint64_t pol = (diag & 8) ? policy_evict_normal() : policy_evict_last();
      for (int t = cl; t < n_tiles; t += ncl) {
        const int2 tile = tiles[t];
        const int ra = tile.x * 2 * kTM + (int)rank * kTM, cbh = tile.y * kTN + (int)rank * (kTN / 2);
        for (int kb = 0; kb < nk; ++kb, ++g) {
          const int s = g % kTc2Stages;
          if (g >= kTc2Stages) mbar_wait(&sm.empty[s], ((g / kTc2Stages) + 1) & 1);
          uint8_t* st = sm.stage[s];
          if (leader) mbar_expect_tx(&sm.full[s], 2 * kStage2Bytes);
          const int kx = kb * 2 * kTK;
          tma_load_2d_2sm(st, &map_hi, kx, ra, &sm.full[s], pol);
          tma_load_2d_2sm(st + kABytes, &map_lo, kx, ra, &sm.full[s], pol);
          tma_load_2d_2sm(st + 2 * kABytes, &map_bhi, kx, cbh, &sm.full[s], pol);
          tma_load_2d_2sm(st + 2 * kABytes + kBHalfBytes, &map_blo, kx, cbh, &sm.full[s], pol);
        }
      }
    }
  } else if (warp == 1) {
    if (leader && lane == 0) {  // ---- MMA issuer (leader only)
      int g = 0, it = 0;
      for (int t = cl; t < n_tiles; t += ncl, ++it) {
        // accumulators are drained per k third: 0 during the tile (after its first third), 3 and
        // the last third's at the end; the next tile needs only 0 and 3 to start (free03)
        if (it > 0) mbar_wait(&sm.free03, (it - 1) & 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        for (int kb = 0; kb < nk; ++kb, ++g) {
          const int s = g % kTc2Stages;
          const int j = (kb * jn) / nk;
          const int kb_first = (j * nk + jn - 1) / jn;
          if (it > 0 && j > 0 && kb == kb_first && !late) {
            mbar_wait(j == 1 ? &sm.free1 : &sm.free2, (it - 1) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          }
          mbar_wait(&sm.full[s], (g / kTc2Stages) & 1);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          uint8_t* st = sm.stage[s];
          const uint64_t ahi = umma_desc_sw128(st), alo = umma_desc_sw128(st + kABytes);
          const uint64_t bhi = umma_desc_sw128(st + 2 * kABytes), blo = umma_desc_sw128(st + 2 * kABytes + kBHalfBytes);
#pragma unroll
          for (int kk = 0; kk < kTK / 8; ++kk) {
            if (diag & 2) break;
            const uint64_t adv = (uint64_t)(kk * 32) >> 4;  // 16 FP16 = 32 bytes along K inside the atom
            umma_f16_2sm(tmem + j * kTN, ahi + adv, bhi + adv, (kb == kb_first && kk == 0) ? 0u : 1u);
            if (diag & 64) continue;  // timing experiment: hi.hi only
            umma_f16_2sm(tmem + kMainAcc * kTN, ahi + adv, blo + adv, (kb | kk) ? 1u : 0u);
            umma_f16_2sm(tmem + kMainAcc * kTN, alo + adv, bhi + adv, 1u);
          }
          umma_commit_2sm(&sm.empty[s]);
          // the last k block of a third that is not the tile's last: that accumulator is complete
          if (!late && j < jn - 1 && kb + 1 == (((j + 1) * nk + jn - 1) / jn)) umma_commit_2sm(&sm.acc_ready[j]);
        }
        umma_commit_2sm(&sm.tmem_full);
      }
    }
  } else {  // ---- epilogue: warps 2..5 of both CTAs, TMEM lane quarter (warp % 4) of this CTA's rows
    const int q = warp & 3;
    const uint32_t f03 = mapa_rank(smem_u32(&sm.free03), 0), f1 = mapa_rank(smem_u32(&sm.free1), 0),
                   f2 = mapa_rank(smem_u32(&sm.free2), 0);
    auto release = [&](uint32_t bar) {  // this warp's TMEM reads are done: arrive on the leader's barrier
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(bar) : "memory");
    };
    const uint64_t spol = policy_evict_first();
    int it = 0;
    for (int t = cl; t < n_tiles; t += ncl, ++it) {
      const int2 tile = tiles[t];
      const int bi = tile.x * 2 + (int)rank;
      const int64_t r0 = (int64_t)bi * kTM, c0 = (int64_t)tile.y * kTN;
      const int64_t r = r0 + q * 32 + lane;
      const float nr = (r < n) ? norms[r] : 0.f;
      float cnv[kTN / 32];
#pragma unroll
      for (int ch = 0; ch < kTN / 32; ++ch) cnv[ch] = norms[c0 + ch * 32 + lane];
      float dot[kTN];
      const uint32_t trow = tmem + ((uint32_t)(q * 32) << 16);
      // accumulator acc of this warp's rows, added into dot (first = assign)
      auto drain = [&](int acc, bool first) {
#pragma unroll
        for (int ch = 0; ch < kTN / 32; ++ch) {
          uint32_t v[32];
          tmem_ld32(trow + (uint32_t)(ch * 32 + acc * kTN), v);
          asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
          for (int j = 0; j < 32; ++j)
            dot[ch * 32 + j] = first ? __uint_as_float(v[j]) : dot[ch * 32 + j] + __uint_as_float(v[j]);
        }
      };
      // thirds completed during the tile (all but the last): drained as soon as they are ready
      for (int j = 0; j < (late ? 0 : jn - 1); ++j) {
        mbar_wait(&sm.acc_ready[j], it & 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        drain(j, j == 0);
        if (j == 1) release(f1);
      }
      mbar_wait(&sm.tmem_full, it & 1);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      if (late) {  // all accumulators at the end: 0 + 3, release, then 1 + 2
        drain(0, true);
        drain(kMainAcc, false);
        release(f03);
        for (int j = 1; j < jn; ++j) drain(j, false);
        release(f1);
        release(f2);
      } else {
        drain(kMainAcc, jn == 1);  // corrections
        if (jn == 1) drain(0, false);
        release(f03);  // the next tile may start (accumulators 0 and 3 are free)
        if (jn >= 2) {
          drain(jn - 1, false);
          release(jn - 1 == 1 ? f1 : f2);
        }
      }
      if (diag & 1) continue;
      if (bi > tile.y) continue;  // entirely below the diagonal: nothing to store
      if (bi < tile.y) {          // off-diagonal: TMA stores of the block and its mirror
        float* eb = sm.epi[q][0];
        float* em = sm.epi[q][1];
#pragma unroll
        for (int ch = 0; ch < kTN / 32; ++ch) {
          const int64_t cb = c0 + ch * 32;
          const float cn = cnv[ch];
          float kv[32];
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            const float d2 = fmaf(-2.f, dot[ch * 32 + j], nr + __shfl_sync(0xffffffffu, cn, j));
            asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(kv[j]) : "f"(fmaxf(d2, 0.f) * scale));
          }
          if (lane == 0) bulk_wait_read0();
          __syncwarp();
#pragma unroll
          for (int jj = 0; jj < 8; ++jj)
            *reinterpret_cast<float4*>(eb + lane * 32 + ((jj ^ (lane & 7)) << 2)) =
                make_float4(kv[4 * jj], kv[4 * jj + 1], kv[4 * jj + 2], kv[4 * jj + 3]);
#pragma unroll
          for (int j = 0; j < 32; ++j) em[j * 32 + lane] = kv[j];
          fence_proxy_async_smem();
          __syncwarp();
          if (lane == 0) {
            tma_store_2d_hint(&map_ksw, eb, (int)cb, (int)(r0 + q * 32), spol);
            tma_store_2d_hint(&map_kns, em, (int)(r0 + q * 32), (int)cb, spol);
            bulk_commit();
          }
        }
        continue;
      }
#pragma unroll
      for (int ch = 0; ch < kTN / 32; ++ch) {  // diagonal tile: K[r][c] for r <= c and the mirror for r < c
        const int64_t cb = c0 + ch * 32;
        float kv[32];
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          const float d2 = fmaf(-2.f, dot[ch * 32 + j], nr + __shfl_sync(0xffffffffu, cnv[ch], j));
          float val;
          asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(val) : "f"(fmaxf(d2, 0.f) * scale));
          kv[j] = (r == cb + j) ? 1.f : val;
        }
        if (r < n) {
          float* dst = K + r * ldk + cb;
#pragma unroll
          for (int j = 0; j < 32; ++j)
            if (cb + j >= r && cb + j < n) dst[j] = kv[j];
        }
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          const int64_t c = cb + j;
          if (r < c && c < n) K[c * ldk + r] = kv[j];
        }
      }
    }
    if (lane == 0) bulk_wait0();
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  cluster_sync_all();  // the peer's MMAs / arrivals are done before TMEM is released
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
  }
}

// ------------------------------------------------------------------------------------------
// a10 on the tensor cores: decision values dec[x][p] = sum_j coef_{j,p} K(x, sv_j) (+ b_p later)
// with the same 3xTF32 split / split accumulators as the kernel-value contraction.  A = a 128-row
// test tile, B = a class-pure 128-SV tile; the epilogue turns the 128 x 128 dot products into
// kernel values and contracts them with the SV tile's coefficients (each SV of class c feeds the
// k-1 pairs of c) into per-row FP32 accumulators that live across the SV tiles of a work unit
// (one test tile x one run of SV tiles of one class); K never leaves the SM.  Persistent CTAs
// take the units round-robin; unit u covers tiles [unit_off[u], unit_off[u + 1]) of the list.
template <int KM>
struct DecTcSmem {
  alignas(1024) uint8_t stage[kTcStages][kStageBytes];
  alignas(16) float coefS[2][kTN][KM];
  alignas(8) uint64_t full[kTcStages];
  uint64_t empty[kTcStages];
  uint64_t tmem_full;
  uint64_t tmem_empty;
  uint32_t tmem_base;
};

// KM: compile-time bound of the pair columns (k - 1 <= KM, KM % 4 == 0); KT: 0 the Gaussian, else
// a dot-product kernel of L76-L78 (uncentred rows, kp), as krow_tc_kernel
template <int KM, bool F16, int KT = 0>
__global__ void __launch_bounds__(kTcThreads, 1)
    dec_tc_kernel(const __grid_constant__ CUtensorMap map_thi, const __grid_constant__ CUtensorMap map_tlo,
                  const __grid_constant__ CUtensorMap map_shi, const __grid_constant__ CUtensorMap map_slo,
                  const int2* __restrict__ tiles, const int32_t* __restrict__ unit_off,
                  const int32_t* __restrict__ unit_item, int n_units, const float* __restrict__ nt,
                  const float* __restrict__ nsv, const float* __restrict__ coef, int km1, int km1_pad, int nk,
                  float scale, int64_t m_pad, float* __restrict__ part, KrowKernel kp) {
  extern __shared__ __align__(1024) uint8_t dsmem[];
  DecTcSmem<KM>& sm =
      *reinterpret_cast<DecTcSmem<KM>*>((reinterpret_cast<uintptr_t>(dsmem) + 1023) & ~uintptr_t(1023));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < kTcStages; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], 1);
    }
    mbar_init(&sm.tmem_full, 1);
    mbar_init(&sm.tmem_empty, 4);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&sm.tmem_base)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = sm.tmem_base;
  const int jn = nk < kMainAcc ? nk : kMainAcc;

  if (warp == 0) {
    if (lane == 0) {  // ---- TMA producer
      int g = 0;
      for (int u = blockIdx.x; u < n_units; u += gridDim.x)
        for (int t = unit_off[u]; t < unit_off[u + 1]; ++t) {
          const int2 tile = tiles[t];
          const int r0 = tile.x * kTM, c0 = tile.y * kTN;
          for (int kb = 0; kb < nk; ++kb, ++g) {
            const int s = g % kTcStages;
            if (g >= kTcStages) mbar_wait(&sm.empty[s], ((g / kTcStages) + 1) & 1);
            uint8_t* st = sm.stage[s];
            mbar_expect_tx(&sm.full[s], kStageBytes);
            const int kx = kb * (F16 ? 2 * kTK : kTK);
            tma_load_2d(st, &map_thi, kx, r0, &sm.full[s]);
            tma_load_2d(st + kABytes, &map_tlo, kx, r0, &sm.full[s]);
            tma_load_2d(st + 2 * kABytes, &map_shi, kx, c0, &sm.full[s]);
            tma_load_2d(st + 2 * kABytes + kBBytes, &map_slo, kx, c0, &sm.full[s]);
          }
        }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ---- MMA issuer
      int g = 0, it = 0;
      for (int u = blockIdx.x; u < n_units; u += gridDim.x)
        for (int t = unit_off[u]; t < unit_off[u + 1]; ++t, ++it) {
          if (it > 0) mbar_wait(&sm.tmem_empty, (it - 1) & 1);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          for (int kb = 0; kb < nk; ++kb, ++g) {
            const int s = g % kTcStages;
            mbar_wait(&sm.full[s], (g / kTcStages) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            uint8_t* st = sm.stage[s];
            const uint64_t ahi = umma_desc_sw128(st), alo = umma_desc_sw128(st + kABytes);
            const uint64_t bhi = umma_desc_sw128(st + 2 * kABytes), blo = umma_desc_sw128(st + 2 * kABytes + kBBytes);
            const int j = (kb * jn) / nk;
            const int kb_first = (j * nk + jn - 1) / jn;
#pragma unroll
            for (int kk = 0; kk < kTK / 8; ++kk) {
              const uint64_t adv = (uint64_t)(kk * 32) >> 4;
              umma_split3<F16, true>(tmem + j * kTN, tmem + kMainAcc * kTN, ahi + adv, alo + adv, bhi + adv, blo + adv,
                                     (kb == kb_first && kk == 0) ? 0u : 1u, (kb | kk) ? 1u : 0u);
            }
            umma_commit(&sm.empty[s]);
          }
          umma_commit(&sm.tmem_full);
        }
    }
  } else {  // ---- epilogue: warps 2..5 (TMEM lane quarter warp % 4), thread = one test row
    const int q = warp & 3, et = threadIdx.x - 64;  // et: 0..127
    int it = 0;
    for (int u = blockIdx.x; u < n_units; u += gridDim.x) {
      float acc[KM];
#pragma unroll
      for (int v = 0; v < KM; ++v) acc[v] = 0.f;
      int64_t r = 0;
      for (int t = unit_off[u]; t < unit_off[u + 1]; ++t, ++it) {
        const int2 tile = tiles[t];
        const int64_t r0 = (int64_t)tile.x * kTM, c0 = (int64_t)tile.y * kTN;
        r = r0 + q * 32 + lane;
        // this SV tile's coefficients (double buffer: one barrier per tile)
        float* cs = &sm.coefS[it & 1][0][0];
#pragma unroll
        for (int v = 0; v < KM; ++v) cs[et * KM + v] = v < km1_pad ? coef[(c0 + et) * km1_pad + v] : 0.f;
        asm volatile("bar.sync 1, 128;" ::: "memory");
        mbar_wait(&sm.tmem_full, it & 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        float dot[kTN];
#pragma unroll
        for (int ch = 0; ch < kTN / 32; ++ch) {  // one 32-column accumulator slice at a time (registers)
          const uint32_t taddr = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(ch * 32);
          uint32_t v[32];
          tmem_ld32(taddr + kMainAcc * kTN, v);
          asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
          for (int jj = 0; jj < 32; ++jj) dot[ch * 32 + jj] = __uint_as_float(v[jj]);
#pragma unroll
          for (int a = 0; a < kMainAcc; ++a) {
            if (a >= nk) break;
            tmem_ld32(taddr + a * kTN, v);
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
            for (int jj = 0; jj < 32; ++jj) dot[ch * 32 + jj] += __uint_as_float(v[jj]);
          }
        }
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncwarp();
        if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.tmem_empty)) : "memory");
        const float nr = nt[r];
#pragma unroll
        for (int j = 0; j < kTN; ++j) {
          float kv;
          if (KT != 0) {
            kv = dot_kernel_value<KT>(dot[j] * kp.inv_s2, kp);
          } else {
            const float d2 = fmaf(-2.f, dot[j], nr + __ldg(nsv + c0 + j));
            asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(kv) : "f"(fmaxf(d2, 0.f) * scale));
          }
          const float4* cj = reinterpret_cast<const float4*>(cs + j * KM);
#pragma unroll
          for (int v4 = 0; v4 < KM / 4; ++v4) {
            const float4 cv = cj[v4];
            acc[4 * v4 + 0] = fmaf(kv, cv.x, acc[4 * v4 + 0]);
            acc[4 * v4 + 1] = fmaf(kv, cv.y, acc[4 * v4 + 1]);
            acc[4 * v4 + 2] = fmaf(kv, cv.z, acc[4 * v4 + 2]);
            acc[4 * v4 + 3] = fmaf(kv, cv.w, acc[4 * v4 + 3]);
          }
        }
      }
      // the unit's partial decision values: part[item][row][col]
      float* out = part + ((int64_t)unit_item[u] * m_pad + r) * km1_pad;
#pragma unroll
      for (int v = 0; v < KM; ++v)
        if (v < km1_pad) out[v] = v < km1 ? acc[v] : 0.f;
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
  }
}


// ------------------------------------------------------------------------------------------
// ROW_CACHE rows on tcgen05 (a2 + a3 when K does not fit): per outer
// iteration, the kernel rows of every pair's NEW working-set entries against the pair's
// instances, K(x_new, x_pair) with the same FP16 hi/lo split and split accumulators as the FULL_K
// contraction.  A = the new rows gathered per pair ([pair][ldat] rows of the Ahi / Alo buffers,
// rows_gather_tc_kernel), B = the class-sorted split X; column tiles walk the pair's two class
// segments; the epilogue writes row r's values at R[r_off + slot * ldr + pair-local column]
// (per-thread stores, K_ii = 1).  Tiles whose rows do not exist this iteration (fewer new rows,
// pair converged) are skipped by all three roles from the same global state.
struct RowsTcArgs {
  const PairDesc* pairs;
  const int32_t* status;
  const int32_t* ws;
  const int32_t* ws_n;
  const int32_t* ws_keep;
  const int32_t* ws_slot;
  const float* norms;
  float* R;
  int B, ldat;
  float scale;
};

__device__ __forceinline__ bool rows_tile_live(const RowsTcArgs& ra, const int4 tl, int& nnew) {
  const int lp = tl.x;
  if (ra.status[lp] != 0) return false;
  nnew = ra.ws_n[lp] - ra.ws_keep[lp];
  return tl.y * kTM < nnew;
}

__global__ void __launch_bounds__(kTcThreads, 1)
    rows_tc_kernel(const __grid_constant__ CUtensorMap map_ahi, const __grid_constant__ CUtensorMap map_alo,
                   const __grid_constant__ CUtensorMap map_xhi, const __grid_constant__ CUtensorMap map_xlo,
                   const int4* __restrict__ tiles, int n_tiles, int nk, RowsTcArgs ra) {
  extern __shared__ __align__(1024) uint8_t dsmem[];
  TcSmem& sm = *reinterpret_cast<TcSmem*>((reinterpret_cast<uintptr_t>(dsmem) + 1023) & ~uintptr_t(1023));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < kTcStages; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], 1);
    }
    mbar_init(&sm.tmem_full, 1);
    mbar_init(&sm.tmem_empty, 4);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&sm.tmem_base)),
                 "r"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = sm.tmem_base;
  const int jn = nk < kMainAcc ? nk : kMainAcc;
  auto col0 = [&](const int4 tl, int64_t& c0, int64_t& hi, int64_t& loc0) {
    const PairDesc pd = ra.pairs[tl.x];
    const int ts = (pd.n_s + kTN - 1) / kTN;
    const bool seg_s = tl.z < ts;
    c0 = seg_s ? pd.off_s + (int64_t)tl.z * kTN : pd.off_t + (int64_t)(tl.z - ts) * kTN;
    hi = seg_s ? pd.off_s + pd.n_s : pd.off_t + pd.n_t;
    loc0 = seg_s ? -pd.off_s : pd.n_s - pd.off_t;  // pair-local column = g + loc0
  };
  if (warp == 0) {
    if (lane == 0) {  // ---- TMA producer
      int g = 0, nnew = 0;
      const uint64_t pol = policy_evict_last();
      for (int t = blockIdx.x; t < n_tiles; t += gridDim.x) {
        const int4 tl = tiles[t];
        if (!rows_tile_live(ra, tl, nnew)) continue;
        int64_t c0, hi, loc0;
        col0(tl, c0, hi, loc0);
        const int r0 = tl.x * ra.ldat + tl.y * kTM;
        for (int kb = 0; kb < nk; ++kb, ++g) {
          const int s = g % kTcStages;
          if (g >= kTcStages) mbar_wait(&sm.empty[s], ((g / kTcStages) + 1) & 1);
          uint8_t* st = sm.stage[s];
          mbar_expect_tx(&sm.full[s], kStageBytes);
          const int kx = kb * 2 * kTK;
          tma_load_2d(st, &map_ahi, kx, r0, &sm.full[s], pol);
          tma_load_2d(st + kABytes, &map_alo, kx, r0, &sm.full[s], pol);
          tma_load_2d(st + 2 * kABytes, &map_xhi, kx, (int)c0, &sm.full[s], pol);
          tma_load_2d(st + 2 * kABytes + kBBytes, &map_xlo, kx, (int)c0, &sm.full[s], pol);
        }
      }
    }
  } else if (warp == 1) {  // ---- MMA issuer (whole warp, one elected lane issues; see krow_tc_kernel)
    int g = 0, it = 0, nnew = 0;
    for (int t = blockIdx.x; t < n_tiles; t += gridDim.x) {
      const int4 tl = tiles[t];
      if (!rows_tile_live(ra, tl, nnew)) continue;
      if (it > 0) mbar_wait(&sm.tmem_empty, (it - 1) & 1);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      for (int kb = 0; kb < nk; ++kb, ++g) {
        const int s = g % kTcStages;
        mbar_wait(&sm.full[s], (g / kTcStages) & 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        uint8_t* st = sm.stage[s];
        const uint64_t ahi = umma_desc_sw128(st), alo = umma_desc_sw128(st + kABytes);
        const uint64_t bhi = umma_desc_sw128(st + 2 * kABytes), blo = umma_desc_sw128(st + 2 * kABytes + kBBytes);
        const int j = (kb * jn) / nk;
        const int kb_first = (j * nk + jn - 1) / jn;
        if (elect_one()) {
#pragma unroll
          for (int kk = 0; kk < kTK / 8; ++kk) {
            const uint64_t adv = (uint64_t)(kk * 32) >> 4;
            umma_split3<true, true>(tmem + j * kTN, tmem + kMainAcc * kTN, ahi + adv, alo + adv, bhi + adv, blo + adv,
                                    (kb == kb_first && kk == 0) ? 0u : 1u, (kb | kk) ? 1u : 0u);
          }
          umma_commit(&sm.empty[s]);
        }
        __syncwarp();
      }
      if (elect_one()) umma_commit(&sm.tmem_full);
      __syncwarp();
      ++it;
    }
  } else {  // ---- epilogue: warps 2..5 (TMEM lane quarter warp % 4), thread = one new row
    const int q = warp & 3;
    int it = 0, nnew = 0;
    for (int t = blockIdx.x; t < n_tiles; t += gridDim.x) {
      const int4 tl = tiles[t];
      if (!rows_tile_live(ra, tl, nnew)) continue;
      const PairDesc pd = ra.pairs[tl.x];
      int64_t c0, hi, loc0;
      col0(tl, c0, hi, loc0);
      const int r = tl.y * kTM + q * 32 + lane;  // index among the pair's new rows
      const bool live = r < nnew;
      const int keep = ra.ws_keep[tl.x];
      const int64_t gr = live ? gpos(pd, ra.ws[(int64_t)tl.x * ra.B + keep + r]) : -1;
      const float nr = live ? ra.norms[gr] : 0.f;
      const int64_t ldr = (pd.n_s + pd.n_t + 3) & ~3;
      float* dst = live ? ra.R + pd.r_off + (int64_t)ra.ws_slot[(int64_t)tl.x * ra.B + keep + r] * ldr : nullptr;
      float cnv[kTN / 32];
#pragma unroll
      for (int ch = 0; ch < kTN / 32; ++ch) cnv[ch] = ra.norms[c0 + ch * 32 + lane];  // norms zero-padded past n
      mbar_wait(&sm.tmem_full, it & 1);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      float dot[kTN];
      const uint32_t trow = tmem + ((uint32_t)(q * 32) << 16);
#pragma unroll
      for (int ch = 0; ch < kTN / 32; ++ch) {
        uint32_t v0[32], w[32];
        tmem_ld32(trow + (uint32_t)(ch * 32), v0);
        tmem_ld32(trow + (uint32_t)(ch * 32) + kMainAcc * kTN, w);
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
        for (int j = 0; j < 32; ++j) dot[ch * 32 + j] = __uint_as_float(v0[j]) + __uint_as_float(w[j]);
        if (nk > 1) {
          tmem_ld32(trow + (uint32_t)(ch * 32) + kTN, v0);
          tmem_ld32(trow + (uint32_t)(ch * 32) + 2 * kTN, w);
          asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            float x = dot[ch * 32 + j] + __uint_as_float(v0[j]);
            if (nk > 2) x += __uint_as_float(w[j]);
            dot[ch * 32 + j] = x;
          }
        }
      }
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&sm.tmem_empty)) : "memory");
      ++it;
#pragma unroll
      for (int ch = 0; ch < kTN / 32; ++ch) {
        const int64_t cb = c0 + ch * 32;
        float kv[32];
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          const float d2 = fmaf(-2.f, dot[ch * 32 + j], nr + __shfl_sync(0xffffffffu, cnv[ch], j));
          float val;
          asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(val) : "f"(fmaxf(d2, 0.f) * ra.scale));
          kv[j] = (cb + j == gr) ? 1.f : val;
        }
        if (!live || cb >= hi) continue;
        float* o = dst + cb + loc0;
        if (cb + 31 < hi && (reinterpret_cast<uintptr_t>(o) & 15) == 0) {
#pragma unroll
          for (int j = 0; j < 32; j += 4) *reinterpret_cast<float4*>(o + j) = make_float4(kv[j], kv[j + 1], kv[j + 2], kv[j + 3]);
        } else {
#pragma unroll
          for (int j = 0; j < 32; ++j)
            if (cb + j < hi) o[j] = kv[j];
        }
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols));
  }
}

// the new rows' hi / lo split rows into A (row lp * ldat + r), FP16 halfs, dpt per row
__global__ void rows_gather_tc_kernel(const PairDesc* pairs, const int32_t* status, const int32_t* ws,
                                      const int32_t* ws_n, const int32_t* ws_keep, int B, int ldat, int pair_base,
                                      const __half* xhi, const __half* xlo, __half* ahi, __half* alo, int dpt,
                                      int64_t* rows_done) {
  const int lp = blockIdx.x + pair_base;
  if (status[lp] != 0) return;
  const PairDesc pd = pairs[lp];
  const int keep = ws_keep[lp], nnew = ws_n[lp] - keep;
  if (nnew <= 0) return;
  if (blockIdx.y == 0 && threadIdx.x == 0) rows_done[lp] += nnew;
  const int vq = dpt / 8;  // 16-byte vectors per row
  for (int r = blockIdx.y; r < nnew; r += gridDim.y) {
    const int64_t g = gpos(pd, ws[(int64_t)lp * B + keep + r]);
    const uint4* sh = reinterpret_cast<const uint4*>(xhi + g * dpt);
    const uint4* sl = reinterpret_cast<const uint4*>(xlo + g * dpt);
    uint4* dh = reinterpret_cast<uint4*>(ahi + ((int64_t)lp * ldat + r) * dpt);
    uint4* dl = reinterpret_cast<uint4*>(alo + ((int64_t)lp * ldat + r) * dpt);
    for (int v = threadIdx.x; v < vq; v += blockDim.x) {
      dh[v] = sh[v];
      dl[v] = sl[v];
    }
  }
}

// column means of the rows idx[0..n) of X (idx < 0: skipped): per-chunk FP64 partials, then a
// fixed-order sum over the chunks (deterministic)
constexpr int kGatherMeanRows = 256;  // rows per partial
constexpr int kGatherBatch = 32;     // loads in flight per thread
__global__ void gather_col_partial_kernel(const float* __restrict__ X, int d, const int64_t* __restrict__ idx,
                                          int64_t n, double* __restrict__ part) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= d) return;
  const int64_t i0 = (int64_t)blockIdx.y * kGatherMeanRows;
  const int64_t i1 = (n < i0 + kGatherMeanRows) ? n : i0 + kGatherMeanRows;
  double s = 0.0;
  for (int64_t b = i0; b < i1; b += kGatherBatch) {
    float v[kGatherBatch];  // a batch of loads in flight before its (fixed-order) sum
#pragma unroll
    for (int j = 0; j < kGatherBatch; ++j) {
      const int64_t r = b + j < i1 ? idx[b + j] : -1;
      v[j] = r >= 0 ? X[r * d + c] : 0.f;
    }
#pragma unroll
    for (int j = 0; j < kGatherBatch; ++j) s += v[j];
  }
  part[(int64_t)blockIdx.y * d + c] = s;
}
__global__ void gather_col_mean_kernel(const double* __restrict__ part, int nch, int d, int64_t cnt,
                                       float* __restrict__ mu) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= d) return;
  double s = 0.0;
  for (int q = 0; q < nch; ++q) s += part[(int64_t)q * d + c];
  mu[c] = (float)(cnt > 0 ? s / (double)cnt : 0.0);
}

// Column means (deterministic two-level FP64 reduction): RBF distances are translation
// invariant, and centring shrinks the dot products whose tensor-core accumulation error
// limits the 3xTF32 contraction.
constexpr int kMeanRows = 1024;
__global__ void col_partial_kernel(const float* __restrict__ X, int64_t n, int d, double* __restrict__ part) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= d) return;
  const int64_t r0 = (int64_t)blockIdx.y * kMeanRows;
  const int64_t r1 = (n < r0 + kMeanRows) ? n : r0 + kMeanRows;
  double s = 0.0;
  for (int64_t r = r0; r < r1; ++r) s += X[r * d + c];
  part[(int64_t)blockIdx.y * d + c] = s;
}
__global__ void col_mean_kernel(const double* __restrict__ part, int nchunks, int64_t n, int d, float* __restrict__ mu) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= d) return;
  double s = 0.0;
  for (int q = 0; q < nchunks; ++q) s += part[(int64_t)q * d + c];
  mu[c] = (float)(s / (double)n);
}

// x' = (x - mu) s (FP32; s = 1 for TF32); TF32: hi = TF32(x'), lo = TF32(x' - hi) (round to
// nearest); FP16: hi = half(x'), lo = half(x' - hi); norms[j] = ||x'_j||^2 accumulated in FP64
// (one warp per row); zero padding.  hi / lo rows are d_pad elements (4 or 2 bytes).
template <bool F16>
__global__ void split_hilo_kernel(const float* __restrict__ X, int64_t n, int d, const int64_t* __restrict__ perm,
                                  const float* __restrict__ mu, float sc, void* __restrict__ hi_, void* __restrict__ lo_,
                                  float* __restrict__ norms, int64_t n_pad, int d_pad) {
  const int64_t j = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (j >= n_pad) return;
  const int64_t src = (j < n) ? (perm ? perm[j] : j) : -1;
  double s = 0.0;
  for (int c = lane; c < d_pad; c += 32) {
    float x = 0.f;
    if (src >= 0 && c < d) x = (X[src * d + c] - mu[c]) * sc;
    if (F16) {
      const __half h = __float2half_rn(x);
      const float r = x - __half2float(h);
      static_cast<__half*>(hi_)[j * d_pad + c] = h;
      static_cast<__half*>(lo_)[j * d_pad + c] = __float2half_rn(r);
    } else {
      // round-to-nearest TF32 for both parts, so the tensor core sees exact TF32 values (it would
      // otherwise drop the low 13 bits of lo) and the dropped lo.lo / lo-rounding terms are unbiased
      const float h = __uint_as_float((__float_as_uint(x) + 0x1000u) & 0xFFFFE000u);
      const float r = x - h;
      static_cast<float*>(hi_)[j * d_pad + c] = h;
      static_cast<float*>(lo_)[j * d_pad + c] = __uint_as_float((__float_as_uint(r) + 0x1000u) & 0xFFFFE000u);
    }
    s = fma((double)x, (double)x, s);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) norms[j] = (float)s;
}

// max over the rows of |x - mu| (non-negative floats order as their bit patterns: atomicMax);
// one warp per row (grid-stride), lanes over the columns: no per-element index division
__global__ void maxabs_kernel(const float* __restrict__ X, int64_t n, int d, const int64_t* __restrict__ perm,
                              const float* __restrict__ mu, unsigned* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t w0 = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  float m = 0.f;
  for (int64_t j = w0; j < n; j += nw) {
    const int64_t src = perm ? perm[j] : j;
    if (src < 0) continue;
    const float* row = X + src * d;
    for (int c = lane; c < d; c += 32) m = fmaxf(m, fabsf(row[c] - mu[c]));
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  if (lane == 0) atomicMax(out, __float_as_uint(m));
}

CUtensorMap make_map(const void* base, int64_t rows, int d_pad, bool f16, int box_rows = kTM) {
  auto enc = get_encode();
  if (!enc) throw Error(GMPSVM_ECUDA, "cuTensorMapEncodeTiled unavailable");
  CUtensorMap m;
  const size_t eb = f16 ? 2 : 4;
  const cuuint64_t dims[2] = {(cuuint64_t)d_pad, (cuuint64_t)rows};
  const cuuint64_t strides[1] = {(cuuint64_t)d_pad * eb};
  const cuuint32_t box[2] = {(cuuint32_t)(128 / eb), (cuuint32_t)box_rows};  // one 128-byte swizzle atom along K
  const cuuint32_t estr[2] = {1, 1};
  const CUresult r = enc(&m, f16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2,
                         const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(GMPSVM_ECUDA, "cuTensorMapEncodeTiled failed: " + std::to_string((int)r));
  return m;
}

}  // namespace

int64_t krow_tc_rows_pad(int64_t n) { return round_up(n, kTN > kTM ? kTN : kTM); }
bool krow_split_f16() {
  static const bool tf32 = getenv("GMPSVM_SPLIT") && std::string(getenv("GMPSVM_SPLIT")) == "tf32";
  return !tf32;
}
int krow_tc_d_pad(int d) { return (int)round_up(d, krow_split_f16() ? 2 * kTK : kTK); }
size_t krow_tc_buf_floats(int64_t n_pad, int d_pad) {
  return (size_t)n_pad * d_pad * (krow_split_f16() ? 2 : 4) / 4;
}
float krow_split_scale(float maxabs) {  // power of two with maxabs * s <= 2^12 (FP16 split); 1 for TF32
  if (!krow_split_f16() || !(maxabs > 0.f) || !std::isfinite(maxabs)) return 1.f;
  int e = 0;
  std::frexp(4096.0 / (double)maxabs, &e);  // 4096 / maxabs = f * 2^e, f in [0.5, 1)
  e = std::max(-60, std::min(60, e - 1));
  return (float)std::ldexp(1.0, e);
}

const float* krow_tc_scratch_mu(const void* scratch, int64_t n, int d) {  // the column means launch_split_hilo left
  return reinterpret_cast<const float*>(static_cast<const double*>(scratch) + (size_t)ceil_div(n, kMeanRows) * d);
}
size_t krow_tc_scratch_bytes(int64_t n, int d) {
  return (size_t)ceil_div(n, kMeanRows) * d * sizeof(double) + (size_t)d * sizeof(float) + 16;
}

float launch_maxabs(const float* X, int64_t n, int d, const int64_t* perm, const float* mu, cudaStream_t st) {
  unsigned* dm = nullptr;
  GM_CUDA(cudaMallocAsync(&dm, sizeof(unsigned), st));
  GM_CUDA(cudaMemsetAsync(dm, 0, sizeof(unsigned), st));
  GM_LAUNCH(maxabs_kernel, dim3(1184), dim3(256), 0, st, X, n, d, perm, mu, dm);
  unsigned h = 0;
  GM_CUDA(cudaMemcpyAsync(&h, dm, sizeof(unsigned), cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaFreeAsync(dm, st));
  GM_CUDA(cudaStreamSynchronize(st));
  float v;
  std::memcpy(&v, &h, 4);
  return v;
}

void launch_split_hilo_mu(const float* X, int64_t n, int d, const int64_t* perm, const float* mu, float sc, void* hi,
                          void* lo, float* norms, int64_t n_pad, int d_pad, cudaStream_t st) {
  if (krow_split_f16())
    GM_LAUNCH(split_hilo_kernel<true>, dim3((unsigned)ceil_div(n_pad, 8)), dim3(256), 0, st, X, n, d, perm, mu, sc, hi,
              lo, norms, n_pad, d_pad);
  else
    GM_LAUNCH(split_hilo_kernel<false>, dim3((unsigned)ceil_div(n_pad, 8)), dim3(256), 0, st, X, n, d, perm, mu, 1.f,
              hi, lo, norms, n_pad, d_pad);
}

float launch_split_hilo(const float* X, int64_t n, int d, const int64_t* perm, void* hi, void* lo, float* norms,
                        int64_t n_pad, int d_pad, void* scratch, cudaStream_t st, bool center) {
  const int nch = (int)ceil_div(n, kMeanRows);
  double* part = static_cast<double*>(scratch);
  float* mu = reinterpret_cast<float*>(part + (size_t)nch * d);
  if (center) {  // RBF: translation invariant, centring shrinks the dot products
    GM_LAUNCH(col_partial_kernel, dim3((unsigned)ceil_div(d, 128), (unsigned)nch), dim3(128), 0, st, X, n, d, part);
    GM_LAUNCH(col_mean_kernel, dim3((unsigned)ceil_div(d, 128)), dim3(128), 0, st, part, nch, n, d, mu);
  } else {  // dot-product kernels need x . y itself
    GM_CUDA(cudaMemsetAsync(mu, 0, (size_t)d * sizeof(float), st));
  }
  const float sc = krow_split_f16() ? krow_split_scale(launch_maxabs(X, n, d, nullptr, mu, st)) : 1.f;
  launch_split_hilo_mu(X, n, d, perm, mu, sc, hi, lo, norms, n_pad, d_pad, st);
  return sc;
}

// Per-class means and second moments (per feature) of the staged (centred, class-sorted) rows,
// from the hi part: used only to order the pairs (engine.cu).
template <typename T>
__global__ void class_means_kernel(const T* hi, int d_pad, const int64_t* coff, float* mu, float* m2) {
  const int c = blockIdx.y, f = blockIdx.x * 32 + threadIdx.x;
  const int64_t r0 = coff[c], r1 = coff[c + 1];
  float s = 0.f, s2 = 0.f;
  if (f < d_pad)
    for (int64_t r = r0 + threadIdx.y; r < r1; r += 8) {
      const float v = (float)hi[r * d_pad + f];
      s += v;
      s2 = fmaf(v, v, s2);
    }
  __shared__ float red[2][8][33];
  red[0][threadIdx.y][threadIdx.x] = s;
  red[1][threadIdx.y][threadIdx.x] = s2;
  __syncthreads();
  if (threadIdx.y == 0 && f < d_pad) {
    float t = 0.f, t2 = 0.f;
#pragma unroll
    for (int y = 0; y < 8; ++y) {
      t += red[0][y][threadIdx.x];
      t2 += red[1][y][threadIdx.x];
    }
    const float inv = r1 > r0 ? 1.f / (float)(r1 - r0) : 0.f;
    mu[(int64_t)c * d_pad + f] = t * inv;
    m2[(int64_t)c * d_pad + f] = t2 * inv;
  }
}

// FP16 split: the rows of a class in kCmChunks slices (more loads in flight than one CTA per 32
// features and class; the sequential loop of class_means_kernel took ~170 us for MNIST-shaped X,
// on the path to the first kernel-value wave), each thread two features (half2), partial sums
// reduced over the slices in a fixed order (deterministic).
constexpr int kCmChunks = 16;
__global__ void class_means_part_kernel(const __half* hi, int d_pad, const int64_t* coff, float* part) {
  const int c = blockIdx.y, ch = blockIdx.z, f = blockIdx.x * 64 + 2 * threadIdx.x;
  const int64_t r0 = coff[c], r1 = coff[c + 1], len = r1 - r0;
  const int64_t a = r0 + len * ch / kCmChunks, b = r0 + len * (ch + 1) / kCmChunks;
  float s0 = 0.f, s1 = 0.f, q0 = 0.f, q1 = 0.f;
  if (f < d_pad)
    for (int64_t r = a + threadIdx.y; r < b; r += 8) {
      const float2 v = __half22float2(*reinterpret_cast<const __half2*>(hi + r * d_pad + f));
      s0 += v.x;
      s1 += v.y;
      q0 = fmaf(v.x, v.x, q0);
      q1 = fmaf(v.y, v.y, q1);
    }
  __shared__ float red[4][8][33];
  red[0][threadIdx.y][threadIdx.x] = s0;
  red[1][threadIdx.y][threadIdx.x] = s1;
  red[2][threadIdx.y][threadIdx.x] = q0;
  red[3][threadIdx.y][threadIdx.x] = q1;
  __syncthreads();
  if (threadIdx.y < 4) {  // y = 0, 1: sums of features f, f + 1; y = 2, 3: their squares
    float t = 0.f;
#pragma unroll
    for (int y = 0; y < 8; ++y) t += red[threadIdx.y][y][threadIdx.x];
    const int ff = f + (threadIdx.y & 1);
    if (ff < d_pad) part[(((int64_t)ch * 2 + (threadIdx.y >> 1)) * gridDim.y + c) * d_pad + ff] = t;
  }
}
__global__ void class_means_reduce_kernel(const float* part, int d_pad, int k, const int64_t* coff, float* mu,
                                          float* m2) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;  // c * d_pad + f
  if (i >= (int64_t)k * d_pad) return;
  const int c = (int)(i / d_pad);
  float t = 0.f, t2 = 0.f;
  for (int ch = 0; ch < kCmChunks; ++ch) {
    t += part[((int64_t)ch * 2 + 0) * k * d_pad + i];
    t2 += part[((int64_t)ch * 2 + 1) * k * d_pad + i];
  }
  const int64_t cnt = coff[c + 1] - coff[c];
  const float inv = cnt > 0 ? 1.f / (float)cnt : 0.f;
  mu[i] = t * inv;
  m2[i] = t2 * inv;
}

void launch_class_means(const void* hi, int d_pad, const int64_t* coff, int k, float* mu, float* m2, cudaStream_t st) {
  if (krow_split_f16()) {  // d_pad is a multiple of 64 (krow_tc_d_pad): half2 loads stay aligned
    DevBuf<float> part((size_t)kCmChunks * 2 * k * d_pad, st);
    GM_LAUNCH(class_means_part_kernel, dim3((unsigned)ceil_div(d_pad, 64), (unsigned)k, kCmChunks), dim3(32, 8), 0, st,
              static_cast<const __half*>(hi), d_pad, coff, part.get());
    GM_LAUNCH(class_means_reduce_kernel, dim3((unsigned)ceil_div((int64_t)k * d_pad, 256)), dim3(256), 0, st, part.get(),
              d_pad, k, coff, mu, m2);
  } else
    GM_LAUNCH(class_means_kernel<float>, dim3((unsigned)ceil_div(d_pad, 32), (unsigned)k), dim3(32, 8), 0, st,
              static_cast<const float*>(hi), d_pad, coff, mu, m2);
}

// Tiles (bi, bj) of 128 x 128 with at least one entry r <= c, in blocked order (16 x 16 tiles)
// so a wave of CTAs reuses its operand tiles from L2.
// CTA-pair kernel (FP16 split only), opt-in with GMPSVM_KROW_CTA=2: measured on B200 (MNIST-shaped
// n = 60,000) at 8.0-10.6 ms against 7.7 ms for the single-CTA kernel -- halving the B operand's
// shared-memory reads and L2 traffic did not help; the contraction is bound by the TMA operand
// stream's latency x bytes in flight (TMA alone: 4.0 ms; MMA alone ~3.8 ms), DESIGN.md §6.1.
bool krow_tc_2cta() {
  static const bool two = getenv("GMPSVM_KROW_CTA") && std::string(getenv("GMPSVM_KROW_CTA")) == "2";
  return two && krow_split_f16();
}

std::vector<int2> krow_tc_tiles(int64_t n, bool two_cta) {
  const int Tc = (int)ceil_div(n, kTN);
  std::vector<int2> t;
  if (two_cta) {  // tiles (I, J) of 256 x 128 whose first 128-row half has an entry r <= c
    const int Tr2 = (int)ceil_div(n, 2 * kTM);
    for (int I = 0; I < Tr2; I += 8)
      for (int J = 0; J < Tc; J += 16)
        for (int bi = I; bi < std::min(Tr2, I + 8); ++bi)
          for (int bj = J; bj < std::min(Tc, J + 16); ++bj)
            if ((int64_t)(bj + 1) * kTN - 1 >= (int64_t)bi * 2 * kTM) t.push_back(make_int2(bi, bj));
    return t;
  }
  const int Tr = (int)ceil_div(n, kTM);
  for (int I = 0; I < Tr; I += 16)
    for (int J = 0; J < Tc; J += 16)
      for (int bi = I; bi < std::min(Tr, I + 16); ++bi)
        for (int bj = J; bj < std::min(Tc, J + 16); ++bj)
          if ((int64_t)(bj + 1) * kTN - 1 >= (int64_t)bi * kTM) t.push_back(make_int2(bi, bj));
  return t;
}

static int num_sms() {
  int sms = 148, dev = 0;
  GM_CUDA(cudaGetDevice(&dev));
  GM_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  return sms;
}

// K (n x n FP32, row stride ldk) as the target of the epilogue's 32 x 32 TMA stores
CUtensorMap make_kmap(float* K, int64_t n, int64_t ldk, bool swizzle) {
  auto enc = get_encode();
  if (!enc) throw Error(GMPSVM_ECUDA, "cuTensorMapEncodeTiled unavailable");
  CUtensorMap m;
  const cuuint64_t dims[2] = {(cuuint64_t)n, (cuuint64_t)n};
  const cuuint64_t strides[1] = {(cuuint64_t)ldk * 4};
  const cuuint32_t box[2] = {32, 32};
  const cuuint32_t estr[2] = {1, 1};
  const CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, K, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         swizzle ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                         CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(GMPSVM_ECUDA, "cuTensorMapEncodeTiled (K) failed: " + std::to_string((int)r));
  return m;
}

int krow_tc_grid(int n_tiles, int reserve_sms, bool mc) {
  const int cap = std::max(1, num_sms() - std::max(0, reserve_sms));
  if (mc) return 2 * std::min(n_tiles / 2, cap / 2);  // clusters of two CTAs, one tile pair each
  return n_tiles < cap ? n_tiles : cap;
}

void launch_krow_tc(const void* hi, const void* lo, int64_t n_pad, int d_pad, const int2* tiles, int n_tiles,
                    const float* norms, int64_t n, double gamma, float sc, float* K, int64_t ldk, cudaStream_t st,
                    bool two_cta, const KrowKernel* dk, int reserve_sms, unsigned long long* resident, bool mc,
                    int d_real) {
  const bool f16 = krow_split_f16();
  const CUtensorMap mhi = make_map(hi, n_pad, d_pad, f16), mlo = make_map(lo, n_pad, d_pad, f16);
  // TMA stores need a 16-byte aligned base and row stride; otherwise every tile takes the
  // per-thread store path
  static const bool no_tma_env = getenv("GMPSVM_KROW_STORE") && std::string(getenv("GMPSVM_KROW_STORE")) == "st";
  const int tma = !no_tma_env && (ldk % 4) == 0 && (reinterpret_cast<uintptr_t>(K) & 15) == 0 && n < (int64_t)INT32_MAX;
  const CUtensorMap mksw = make_kmap(K, tma ? n : 1, tma ? ldk : 4, true), mkns = make_kmap(K, tma ? n : 1, tma ? ldk : 4, false);
  const size_t smem = sizeof(TcSmem) + 1024;
  set_max_dyn_smem(krow_tc_kernel<true, 0>, smem);
  set_max_dyn_smem(krow_tc_kernel<false, 0>, smem);
  set_max_dyn_smem(krow_tc_kernel<true, 1>, smem);
  set_max_dyn_smem(krow_tc_kernel<true, 2>, smem);
  set_max_dyn_smem(krow_tc_kernel<true, 3>, smem);
  // distances are in units scaled by sc: exp(-gamma d2 / sc^2) = exp2(d2 * scale)
  const float scale = (float)(-gamma * 1.4426950408889634 / ((double)sc * (double)sc));
  const int sms = num_sms();
  const int nk = d_pad / (f16 ? 2 * kTK : kTK);
  if (two_cta) {
    if (!f16 || !tma) throw Error(GMPSVM_EINVAL, "CTA-pair kernel-value launch needs the FP16 split and TMA stores");
    const size_t smem2 = sizeof(Tc2Smem) + 1024;
    set_max_dyn_smem(krow_tc2_kernel, smem2);
    // B operand: 64-row boxes (each CTA of the pair loads its half of the 128 columns' rows)
    const CUtensorMap mbhi = make_map(hi, n_pad, d_pad, f16, kTN / 2), mblo = make_map(lo, n_pad, d_pad, f16, kTN / 2);
    const int clusters = std::min(n_tiles, sms / 2);
    static const int diag = getenv("GMPSVM_KROW_DIAG") ? atoi(getenv("GMPSVM_KROW_DIAG")) : 0;
    GM_LAUNCH(krow_tc2_kernel, dim3(2 * clusters), dim3(kTcThreads), smem2, st, mhi, mlo, mbhi, mblo, mksw, mkns, tiles,
              n_tiles, norms, n, nk, scale, K, ldk, diag);
    return;
  }
  // reserve_sms: SMs left free (the lead pairs' solver chains run beside the kernel values, engine.cu)
  const int grid = krow_tc_grid(n_tiles, reserve_sms, mc);
  // MMAs of the last k-step over real columns (K = 16 FP16 / 8 TF32 per MMA)
  const int kper = f16 ? 16 : 8, kblk = f16 ? 2 * kTK : kTK;
  const int dr = d_real > 0 ? std::min(d_real, d_pad) : d_pad;
  const int kk_last = std::max(1, (int)ceil_div(dr - (nk - 1) * kblk, kper));
  const CUtensorMap mhi64 = mc ? make_map(hi, n_pad, d_pad, f16, kTM / 2) : mhi;
  const CUtensorMap mlo64 = mc ? make_map(lo, n_pad, d_pad, f16, kTM / 2) : mlo;
  KrowKernel kp{};
  if (dk) {
    if (!f16 || two_cta) throw Error(GMPSVM_ENOTIMPL, "dot-product kernels need the FP16-split single-CTA launch");
    if (mc) throw Error(GMPSVM_EINVAL, "cluster tile pairs are built for the Gaussian kernel only");
    kp = *dk;
    kp.resident = nullptr;
    kp.inv_s2 = (float)(1.0 / ((double)sc * (double)sc));
    auto go = [&](auto kern) {
      GM_LAUNCH(kern, dim3(grid), dim3(kTcThreads), smem, st, mhi, mlo, mksw, mkns, tiles, n_tiles, norms, n, nk, scale,
                K, ldk, tma, kp, mhi, mlo, kk_last);
    };
    if (kp.type == 1) go(krow_tc_kernel<true, 1>);
    else if (kp.type == 2) go(krow_tc_kernel<true, 2>);
    else go(krow_tc_kernel<true, 3>);
    return;
  }
  kp.resident = resident;
  if (mc) {
    if (!f16 || (n_tiles & 1)) throw Error(GMPSVM_EINVAL, "cluster launch: FP16 split and tile pairs required");
    set_max_dyn_smem(krow_tc_kernel<true, 0, true>, smem);
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(kTcThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    GM_CUDA(cudaLaunchKernelEx(&cfg, krow_tc_kernel<true, 0, true>, mhi, mlo, mksw, mkns, tiles, n_tiles, norms, n, nk,
                               scale, K, ldk, tma, kp, mhi64, mlo64, kk_last));
    g_launches.fetch_add(1, std::memory_order_relaxed);
  } else if (f16) {
    GM_LAUNCH((krow_tc_kernel<true, 0>), dim3(grid), dim3(kTcThreads), smem, st, mhi, mlo, mksw, mkns, tiles,
              n_tiles, norms, n, nk, scale, K, ldk, tma, kp, mhi, mlo, kk_last);
  } else {
    GM_LAUNCH((krow_tc_kernel<false, 0>), dim3(grid), dim3(kTcThreads), smem, st, mhi, mlo, mksw, mkns, tiles,
              n_tiles, norms, n, nk, scale, K, ldk, tma, kp, mhi, mlo, kk_last);
  }
}

bool krow_tc_mc() {
  static const bool off = getenv("GMPSVM_KROW_MC") && std::string(getenv("GMPSVM_KROW_MC")) == "0";
  return !off && krow_split_f16();
}

// Cluster tile pairs (krow_tc_kernel MC): tiles of the same row block, in list order as far as the
// pairing allows (a tile waits for the next one of its row); an unmatched tile gets a dummy partner.
std::vector<int2> krow_tc_mc_pairs(const std::vector<int2>& t) {
  std::vector<int2> out;
  out.reserve(t.size() + 64);
  std::vector<int> pend;  // per row block: index into t of the unpaired tile, or -1
  for (size_t i = 0; i < t.size(); ++i) {
    const int r = t[i].x;
    if ((int)pend.size() <= r) pend.resize(r + 1, -1);
    if (pend[r] < 0) {
      pend[r] = (int)i;
    } else {
      out.push_back(t[pend[r]]);
      out.push_back(t[i]);
      pend[r] = -1;
    }
  }
  for (size_t r = 0; r < pend.size(); ++r)
    if (pend[r] >= 0) {
      out.push_back(t[pend[r]]);
      out.push_back(make_int2((int)r, -1));
    }
  return out;
}

std::vector<int4> rows_tc_tiles(const std::vector<PairDesc>& pairs, int first, int count, int B) {
  std::vector<int4> t;
  const int at = (int)ceil_div(B, kTM);
  for (int lp = first; lp < first + count; ++lp) {
    const PairDesc& pd = pairs[lp];
    const int ct = (int)(ceil_div(pd.n_s, kTN) + ceil_div(pd.n_t, kTN));
    for (int a = 0; a < at; ++a)
      for (int c = 0; c < ct; ++c) t.push_back(make_int4(lp, a, c, 0));
  }
  return t;
}

void launch_rows_compute_tc(const SolverArgs& a, int P, const int4* tiles, int n_tiles, int n_pairs_all,
                            cudaStream_t st) {
  GM_LAUNCH(rows_gather_tc_kernel, dim3(P, 64), dim3(128), 0, st, a.pairs, a.status, a.ws, a.ws_n, a.ws_keep, a.B,
            a.ldat, a.pair_base, static_cast<const __half*>(a.Xhi), static_cast<const __half*>(a.Xlo),
            static_cast<__half*>(a.Ahi), static_cast<__half*>(a.Alo), a.dpt, a.rows_done);
  const CUtensorMap mahi = make_map(a.Ahi, (int64_t)n_pairs_all * a.ldat, a.dpt, true);
  const CUtensorMap malo = make_map(a.Alo, (int64_t)n_pairs_all * a.ldat, a.dpt, true);
  const CUtensorMap mxhi = make_map(a.Xhi, a.n_pad, a.dpt, true), mxlo = make_map(a.Xlo, a.n_pad, a.dpt, true);
  const size_t smem = sizeof(TcSmem) + 1024;
  set_max_dyn_smem(rows_tc_kernel, smem);
  RowsTcArgs ra{a.pairs, a.status, a.ws, a.ws_n, a.ws_keep, a.ws_slot, a.norms, a.R, a.B, a.ldat, a.kscale};
  const int grid = std::min(n_tiles, num_sms());
  GM_LAUNCH(rows_tc_kernel, dim3(grid), dim3(kTcThreads), smem, st, mahi, malo, mxhi, mxlo, tiles, n_tiles,
            a.dpt / (2 * kTK), ra);
}

void launch_gather_col_mean(const float* X, int d, const int64_t* idx, int64_t n, int64_t cnt, float* mu,
                            cudaStream_t st) {
  const int nch = (int)ceil_div(n, kGatherMeanRows);
  double* part = nullptr;
  GM_CUDA(cudaMallocAsync(&part, (size_t)nch * d * sizeof(double), st));
  GM_LAUNCH(gather_col_partial_kernel, dim3((unsigned)ceil_div(d, 128), (unsigned)nch), dim3(128), 0, st, X, d, idx, n,
            part);
  GM_LAUNCH(gather_col_mean_kernel, dim3((unsigned)ceil_div(d, 128)), dim3(128), 0, st, part, nch, d, cnt, mu);
  GM_CUDA(cudaFreeAsync(part, st));
}

int dec_tc_max_km1() { return kDecMaxKm1; }

void launch_dec_tc(const void* thi, const void* tlo, int64_t m_pad, const void* shi, const void* slo, int64_t nsv_pad,
                   int d_pad, const int2* tiles, const int32_t* unit_off, const int32_t* unit_item, int n_units,
                   const float* nt, const float* nsv, const float* coef, int km1, int km1_pad, double gamma, float sc,
                   float* part, cudaStream_t st, const KrowKernel* dk) {
  const bool f16 = krow_split_f16();
  const CUtensorMap mthi = make_map(thi, m_pad, d_pad, f16), mtlo = make_map(tlo, m_pad, d_pad, f16);
  const CUtensorMap mshi = make_map(shi, nsv_pad, d_pad, f16), mslo = make_map(slo, nsv_pad, d_pad, f16);
  const float scale = (float)(-gamma * 1.4426950408889634 / ((double)sc * (double)sc));
  const int sms = num_sms();
  const int grid = n_units < sms ? n_units : sms;
  const int nk = d_pad / (f16 ? 2 * kTK : kTK);
  KrowKernel kp{};
  if (dk) {
    kp = *dk;
    kp.inv_s2 = (float)(1.0 / ((double)sc * (double)sc));
  }
  auto go = [&](auto kern, size_t smem) {
    set_max_dyn_smem(kern, smem);
    GM_LAUNCH(kern, dim3(grid), dim3(kTcThreads), smem, st, mthi, mtlo, mshi, mslo, tiles, unit_off, unit_item, n_units,
              nt, nsv, coef, km1, km1_pad, nk, scale, m_pad, part, kp);
  };
  if (dk) {  // the other kernels: FP16 split, k - 1 <= 12 (engine.cu routes the rest to the FP64 path)
    if (!f16 || km1_pad > 12) throw Error(GMPSVM_ENOTIMPL, "tensor-core decision values of this kernel need k <= 13");
    if (kp.type == 1) go(dec_tc_kernel<12, true, 1>, sizeof(DecTcSmem<12>) + 1024);
    else if (kp.type == 2) go(dec_tc_kernel<12, true, 2>, sizeof(DecTcSmem<12>) + 1024);
    else go(dec_tc_kernel<12, true, 3>, sizeof(DecTcSmem<12>) + 1024);
  } else if (km1_pad <= 12) {
    if (f16) go(dec_tc_kernel<12, true>, sizeof(DecTcSmem<12>) + 1024);
    else go(dec_tc_kernel<12, false>, sizeof(DecTcSmem<12>) + 1024);
  } else {
    if (f16) go(dec_tc_kernel<kDecMaxKm1, true>, sizeof(DecTcSmem<kDecMaxKm1>) + 1024);
    else go(dec_tc_kernel<kDecMaxKm1, false>, sizeof(DecTcSmem<kDecMaxKm1>) + 1024);
  }
}

}  // namespace gmpsvm
