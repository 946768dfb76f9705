// solver.cu -- a4..a9: the batched working-set SMO solver of every active pair, run
// concurrently (one CTA per pair per step; Alg 2), plus the
// bias, in-sample decision values, Platt fit and SV flags.
//
//   select_ws   a4  q/2 smallest f in I_u + q/2 largest f in I_l, newest B-q kept
//                   (L293-L297, Alg 2 lines 6-7; radix select on order-preserving keys)
//                   and the global stop test max_{I_l} f - min_{I_u} f < eps (Eq 9-10)
//   gather_kws  a3  K_ws,ws gathered from the resident kernel matrix (the "GPU buffer", L299-L303)
//   local_smo   a5  WSS2 SMO restricted to the working set (ImproveSVM, L301-L305, Eq 4-8),
//                   early stop at local gap < max(eps, 0.1 delta0) (L305, reading R20)
//   f_update    a6  f_j += sum_ws dalpha_i y_i K_ij over the whole pair (Alg 2 line 11, Eq 8)
//   finalize    a7  rho (LibSVM rule, reading R7), b = -rho, v_i = f_i + y_i - rho (Eq 3 + 11)
//   sigmoid_fit a8  Newton + backtracking on Eq 13, 4 step sizes evaluated per pass (L327)
//   sv_flags    a9  SV union membership over pairs (support-vector sharing, L363)
#include <cfloat>
#include <climits>
#include <cstdlib>
#include <string>

#include "gemm_simt.cuh"
#include <cstring>

#include "kernels.h"
#include "solver_dev.cuh"

namespace gmpsvm {

__global__ void init_pairs_kernel(SolverArgs a, const int64_t tot, int P) {
  // alpha = 0, f = -y (Alg 1 lines 1-2 / Alg 2 line 4), stamps 0
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < tot) {
    // find pair by binary search over a_off
    int lo = 0, hi = P - 1;
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (a.pairs[mid].a_off <= i) lo = mid;
      else hi = mid - 1;
    }
    const PairDesc pd = a.pairs[lo];
    const int64_t j = i - pd.a_off;
    a.alpha[i] = 0.0;
    a.f[i] = (j < pd.n_s) ? -1.0 : 1.0;
    a.stamp[i] = 0u;
    if (a.ulf) a.ulf[i] = (j < pd.n_s) ? 1 : 2;  // alpha = 0: y = +1 in I_u only, y = -1 in I_l only
  }
  if (i < P) {
    a.status[i] = 0;
    a.ws_n[i] = 0;
    a.inner_iters[i] = 0;
    a.smo_cycles[i] = 0;
    a.outer_iters[i] = 0;
    a.gap[i] = 0.0;
  }
}


// Fast path of the selection for shared-memory-staged pairs: one histogram pass (2048 bins,
// linear in key over each side's [kmin, kmax]) finds the threshold bin of each side, one
// compaction pass collects the candidates at or below it (typically ~q/2 + a few), and an
// exact (key, index) bitonic sort of those short lists picks the working set.  Returns -1 (and
// leaves the flags untouched) when a list would overflow; the caller then runs radix_pick.
constexpr int kSelBins = 2048;
constexpr int kSelListCap = 2048;

struct SelLists {
  int32_t hist[2][kSelBins];
  uint64_t key[2][kSelListCap];
  int32_t idx[2][kSelListCap];
  int32_t cnt[2];
  int32_t bin[2];
  int32_t tot[2];
};

// bins linear in f over each side's range (monotone: f1 <= f2 => bin1 <= bin2)
struct FBins {
  double lo, scale;  // bin = (f - lo) * scale (U side) or (lo - f) * scale (L side, lo = max f)
  __device__ __forceinline__ int up(double f) const { return (int)fmin((f - lo) * scale, (double)(kSelBins - 1)); }
  __device__ __forceinline__ int down(double f) const { return (int)fmin((lo - f) * scale, (double)(kSelBins - 1)); }
};
__device__ __forceinline__ double fbin_scale(double span) { return span > 0.0 ? (kSelBins - 1) / span : 0.0; }

// bitonic sort of (key, idx) pairs, n2 a power of two, ascending
__device__ void bitonic_pairs(uint64_t* key, int32_t* idx, int n2) {
  for (int k = 2; k <= n2; k <<= 1)
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = threadIdx.x; i < n2; i += blockDim.x) {
        const int p = i ^ j;
        if (p > i) {
          const bool up = (i & k) == 0;
          const uint64_t ka = key[i], kb = key[p];
          const int32_t ia = idx[i], ib = idx[p];
          const bool gt = ka > kb || (ka == kb && ia > ib);
          if (gt == up) {
            key[i] = kb;
            key[p] = ka;
            idx[i] = ib;
            idx[p] = ia;
          }
        }
      }
      __syncthreads();
    }
}

__device__ int fast_select_sides(const uint64_t* keys, uint8_t* flags, int np, int need, int32_t* out,
                                 uint64_t ku0, uint64_t ku1, uint64_t kl0, uint64_t kl1, SelLists& L, SelSmem& sm,
                                 int64_t* tacc = nullptr) {
  long long tq = clock64();
  auto tmark = [&](int k) {
    if (tacc && threadIdx.x == 0) {
      const long long t = clock64();
      atomicAdd((unsigned long long*)&tacc[k], (unsigned long long)(t - tq));
      tq = t;
    }
  };
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const double fu0 = key_double(ku0), fu1 = key_double(ku1);    // U: smallest .. largest f over I_u
  const double fl1 = key_double(~kl0), fl0 = key_double(~kl1);  // L: largest .. smallest f over I_l
  const FBins bu_{fu0, fbin_scale(fu1 - fu0)}, bl_{fl1, fbin_scale(fl1 - fl0)};
  for (int i = tid; i < 2 * kSelBins; i += blockDim.x) (&L.hist[0][0])[i] = 0;
  if (tid < 2) L.cnt[tid] = 0;
  __syncthreads();
  for (int base = 0; base < np; base += blockDim.x) {
    const int i = base + tid;
    const uint8_t f = i < np ? flags[i] : 4;
    const uint64_t k = i < np ? keys[i] : 0;
    // warp-aggregated histogram updates (clustered f values hit the same bin)
    const bool cu = (f & 5) == 1, cl = (f & 6) == 2;
    const double fv = key_double(k);
    const int b0 = cu ? bu_.up(fv) : -1;
    const int b1 = cl ? bl_.down(fv) : -1;
    const unsigned m0 = __match_any_sync(FULLMASK, b0), m1 = __match_any_sync(FULLMASK, b1);
    if (cu && lane == __ffs(m0) - 1) atomicAdd(&L.hist[0][b0], __popc(m0));
    if (cl && lane == __ffs(m1) - 1) atomicAdd(&L.hist[1][b1], __popc(m1));
  }
  __syncthreads();
  tmark(0);
  // warps 0 / 1: threshold bin of the U / L side (cumulative count reaches the wanted number)
  if (warp < 2) {
    const int side = warp;
    int loc = 0;
    for (int b = lane * 64; b < lane * 64 + 64; ++b) loc += L.hist[side][b];
    int incl = loc;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(FULLMASK, incl, o);
      if (lane >= o) incl += y;
    }
    const int total = __shfl_sync(FULLMASK, incl, 31);
    const int totU = __shfl_sync(FULLMASK, incl, 31);  // this warp's own side total
    (void)totU;
    if (lane == 0) L.tot[side] = total;
    // U wants need/2 (or all it has); L wants the rest (estimate; exact counts are handled below)
    const int want = side == 0 ? min(need / 2, total) : min(need, total);
    const int excl = incl - loc;
    if (want == 0) {
      if (lane == 0) L.bin[side] = -1;
    } else if (excl < want && want <= incl) {
      int cum = excl, b = lane * 64;
      for (; b < lane * 64 + 64; ++b) {
        cum += L.hist[side][b];
        if (cum >= want) break;
      }
      L.bin[side] = b;
    }
  }
  __syncthreads();
  tmark(1);
  const int bu = L.bin[0], bl = L.bin[1];
  // compaction of the candidates at or below the threshold bins
  for (int base = 0; base < np; base += blockDim.x) {
    const int i = base + tid;
    const uint8_t f = i < np ? flags[i] : 4;
    const uint64_t k = i < np ? keys[i] : 0;
    const double fv = key_double(k);
    const bool tu = (f & 5) == 1 && bu_.up(fv) <= bu;
    const bool tl = (f & 6) == 2 && bl_.down(fv) <= bl;
    const unsigned mu = __ballot_sync(FULLMASK, tu), ml = __ballot_sync(FULLMASK, tl);
    int pu = 0, pl = 0;
    if (lane == 0) {
      if (mu) pu = atomicAdd(&L.cnt[0], __popc(mu));
      if (ml) pl = atomicAdd(&L.cnt[1], __popc(ml));
    }
    pu = __shfl_sync(FULLMASK, pu, 0) + __popc(mu & ((1u << lane) - 1u));
    pl = __shfl_sync(FULLMASK, pl, 0) + __popc(ml & ((1u << lane) - 1u));
    if (tu && pu < kSelListCap) {
      L.key[0][pu] = k;
      L.idx[0][pu] = i;
    }
    if (tl && pl < kSelListCap) {
      L.key[1][pl] = ~k;
      L.idx[1][pl] = i;
    }
  }
  __syncthreads();
  tmark(2);
  const int nu = L.cnt[0], nl = L.cnt[1];
  if (tacc && threadIdx.x == 0) atomicAdd((unsigned long long*)&tacc[4], (unsigned long long)(nu + nl));
  if (nu > kSelListCap || nl > kSelListCap) return -1;
  // U side: exact (key, index) order of the short list, take the first need/2
  int n2 = 1;
  while (n2 < nu) n2 <<= 1;
  for (int i = nu + tid; i < n2; i += blockDim.x) {
    L.key[0][i] = ~0ull;
    L.idx[0][i] = INT_MAX;
  }
  __syncthreads();
  bitonic_pairs(L.key[0], L.idx[0], n2);
  const int take_u = min(need / 2, L.tot[0]);
  for (int i = tid; i < take_u; i += blockDim.x) {
    out[i] = L.idx[0][i];
    flags[L.idx[0][i]] |= 4;
  }
  __syncthreads();
  // L side: drop the ones U took, order, take what is still needed
  n2 = 1;
  while (n2 < nl) n2 <<= 1;
  for (int i = tid; i < n2; i += blockDim.x) {
    if (i >= nl || (flags[L.idx[1][i]] & 4)) {
      L.key[1][i] = ~0ull;
      L.idx[1][i] = INT_MAX;
    }
  }
  __syncthreads();
  bitonic_pairs(L.key[1], L.idx[1], n2);
  int valid = 0;
  for (int i = tid; i < n2; i += blockDim.x) valid += L.idx[1][i] != INT_MAX;
  valid = block_reduce(valid, [](int x, int y) { return x + y; }, sm.scan);
  const int need_l = need - take_u;
  // the list holds every L candidate below the threshold bin; if U took some of them the list
  // may be short of need_l while more candidates sit in higher bins: radix_pick completes it
  const int take_l = min(need_l, valid);
  for (int i = tid; i < take_l; i += blockDim.x) {
    out[take_u + i] = L.idx[1][i];
    flags[L.idx[1][i]] |= 4;
  }
  __syncthreads();
  tmark(3);
  return take_u + take_l;
}

constexpr int kSelSmemMax = 16384;  // n_p up to which keys + flags are staged in shared memory

// Selection of one pair by the whole CTA (1024 threads); sel_dyn: >= kSelDynBytes of smem.
__device__ void select_body(const SolverArgs& a, int lp, uint32_t stampv, int first, SelSmem& sm,
                            unsigned char* sel_dyn) {
  const long long t0 = clock64();
  if (a.status[lp] != 0) return;
  long long tp = t0;
  auto mark = [&](int k) {
    if (a.sel_phase && threadIdx.x == 0) {
      const long long t = clock64();
      a.sel_phase[lp * 5 + k] += t - tp;
      tp = t;
    }
  };
  const PairDesc pd = a.pairs[lp];
  const int np = pd.n_s + pd.n_t;
  const double* al = a.alpha + pd.a_off;
  const double* fl = a.f + pd.a_off;
  const double C = a.C;
  const bool use_smem = np <= kSelSmemMax && np > a.B;
  uint64_t* keys = reinterpret_cast<uint64_t*>(sel_dyn);
  uint8_t* flags = sel_dyn + (size_t)kSelSmemMax * 8;
  // global stop test (Eq 9-10 with tolerance eps); stage keys/flags on the way
  double fmin = DBL_MAX, fmax = -DBL_MAX, umax = -DBL_MAX, lmin = DBL_MAX;
  for (int i = threadIdx.x; i < np; i += blockDim.x) {
    const int y = i < pd.n_s ? 1 : -1;
    const double av = al[i], fv = fl[i];
    const bool u = in_u(y, av, C), l = in_l(y, av, C);
    if (u) {
      fmin = fmin < fv ? fmin : fv;
      umax = umax > fv ? umax : fv;
    }
    if (l) {
      fmax = fmax > fv ? fmax : fv;
      lmin = lmin < fv ? lmin : fv;
    }
    if (use_smem) {
      keys[i] = ord_key(fv);
      flags[i] = (u ? 1 : 0) | (l ? 2 : 0);
    }
  }
  mark(0);
  {  // the four extremes in one block reduction: warp shuffles, then warp 0 over the warp partials
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      fmin = ::fmin(fmin, __shfl_xor_sync(FULLMASK, fmin, o));
      fmax = ::fmax(fmax, __shfl_xor_sync(FULLMASK, fmax, o));
      umax = ::fmax(umax, __shfl_xor_sync(FULLMASK, umax, o));
      lmin = ::fmin(lmin, __shfl_xor_sync(FULLMASK, lmin, o));
    }
    double* red4 = sm.red4;
    if (lane == 0) {
      red4[warp] = fmin;
      red4[32 + warp] = fmax;
      red4[64 + warp] = umax;
      red4[96 + warp] = lmin;
    }
    __syncthreads();
    if (warp == 0) {
      double a0 = lane < nw ? red4[lane] : DBL_MAX, a1 = lane < nw ? red4[32 + lane] : -DBL_MAX;
      double a2 = lane < nw ? red4[64 + lane] : -DBL_MAX, a3 = lane < nw ? red4[96 + lane] : DBL_MAX;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        a0 = ::fmin(a0, __shfl_xor_sync(FULLMASK, a0, o));
        a1 = ::fmax(a1, __shfl_xor_sync(FULLMASK, a1, o));
        a2 = ::fmax(a2, __shfl_xor_sync(FULLMASK, a2, o));
        a3 = ::fmin(a3, __shfl_xor_sync(FULLMASK, a3, o));
      }
      if (lane == 0) {
        red4[128] = a0;
        red4[129] = a1;
        red4[130] = a2;
        red4[131] = a3;
      }
    }
    __syncthreads();
    fmin = red4[128];
    fmax = red4[129];
    umax = red4[130];
    lmin = red4[131];
  }
  // key bounds of the two sides: U keys = ord(f) over I_u, L keys = ~ord(f) over I_l
  mark(1);
  const double gap = fmax - fmin;
  const bool done = (fmin == DBL_MAX) || (fmax == -DBL_MAX) || !(gap >= a.eps);
  if (threadIdx.x == 0) {
    a.gap[lp] = gap;
    if (done) a.status[lp] = 1;
    else a.outer_iters[lp] += 1;
  }
  if (done) return;
  const int B = a.B;
  int32_t* ws = a.ws + (int64_t)lp * B;
  if (np <= B) {  // the whole pair is the working set
    if (first) {
      for (int i = threadIdx.x; i < np; i += blockDim.x) {
        ws[i] = i;
        if (a.R) a.ws_slot[(int64_t)lp * B + i] = i;
      }
      if (threadIdx.x == 0) a.ws_n[lp] = np;
    }
    if (a.R && threadIdx.x == 0) a.ws_keep[lp] = first ? 0 : np;  // rows computed once
    return;
  }
  int32_t* nxt = a.ws_tmp + (int64_t)lp * B;
  uint32_t* stp = a.stamp + pd.a_off;
  const int prev_n = first ? 0 : a.ws_n[lp];
  const int keep = min(prev_n, B - a.q);
  for (int e = threadIdx.x; e < keep; e += blockDim.x) {
    const int idx = ws[prev_n - keep + e];
    nxt[e] = idx;
    if (use_smem) flags[idx] |= 4;
    else stp[idx] = stampv;
  }
  __syncthreads();
  mark(2);
  int cnt = keep;
  const uint64_t ku0 = ord_key(fmin), ku1 = ord_key(umax), kl0 = ~ord_key(fmax), kl1 = ~ord_key(lmin);
  if (use_smem) {
    SmemSrc src{keys, flags};
    SelLists& lists = *reinterpret_cast<SelLists*>(sel_dyn + (size_t)kSelSmemMax * 9 + 16);
    const int need = B - keep;
    const int got = fast_select_sides(keys, flags, np, need, nxt + cnt, ku0, ku1, kl0, kl1, lists, sm,
                                      a.sel_phase ? a.sel_phase + (size_t)gridDim.x * 0 + 5 * 64 * 0 + a.pair_base * 0 +
                                                        (int64_t)5 * (lp + 4096) : nullptr);
    if (got < 0) {
      cnt += select_sides(src, np, need, nxt + cnt, sm, ku0, ku1, kl0, kl1);
    } else {
      cnt += got;
      // L side short (its candidates overlapped U's picks): complete from the full arrays
      if (got < need) cnt += radix_pick<false>(src, np, need - got, nxt + cnt, sm, kl0, kl1);
      if (cnt - keep < need) cnt += radix_pick<true>(src, np, keep + need - cnt, nxt + cnt, sm, ku0, ku1);
    }
  } else {
    GlobalSrc src{al, fl, stp, stampv, pd.n_s, C};
    cnt += select_sides(src, np, B - keep, nxt + cnt, sm, ku0, ku1, kl0, kl1);
  }
  mark(3);
  if (a.R) {
    // ROW_CACHE: retained positions keep their row slots; new positions take the free slots in
    // increasing order (deterministic)
    int32_t* slot = a.ws_slot + (int64_t)lp * B;
    int32_t* snx = a.ws_slot_tmp + (int64_t)lp * B;
    uint8_t* used = reinterpret_cast<uint8_t*>(sm.hist);  // B <= 1024 flags
    __syncthreads();
    for (int i = threadIdx.x; i < B; i += blockDim.x) used[i] = 0;
    __syncthreads();
    for (int e = threadIdx.x; e < keep; e += blockDim.x) {
      const int sl = slot[prev_n - keep + e];
      snx[e] = sl;
      used[sl] = 1;
    }
    __syncthreads();
    int base = 0;
    for (int i0 = 0; i0 < B; i0 += blockDim.x) {
      const int i = i0 + threadIdx.x;
      const bool fr = i < B && !used[i];
      int tot = 0;
      const int pos = block_excl_scan(fr, tot, sm.scan);
      if (fr && keep + base + pos < cnt) snx[keep + base + pos] = i;
      base += tot;
    }
    __syncthreads();
    for (int e = threadIdx.x; e < cnt; e += blockDim.x) slot[e] = snx[e];
    if (threadIdx.x == 0) a.ws_keep[lp] = keep;
  }
  for (int e = threadIdx.x; e < cnt; e += blockDim.x) ws[e] = nxt[e];
  if (threadIdx.x == 0) a.ws_n[lp] = cnt;
  mark(4);
}

constexpr size_t kSelDynBytes = (size_t)kSelSmemMax * 9 + 16 + sizeof(SelLists);

__global__ void __launch_bounds__(1024) select_ws_kernel(SolverArgs a, uint32_t stampv, int first) {
  TraceScope ts_(a, blockIdx.x + a.pair_base, 0);
  __shared__ SelSmem sm;
  extern __shared__ __align__(16) unsigned char sel_dyn[];
  if (stampv == 0) {  // device-driven loop (graph): iteration from the pair's own counter
    const int32_t oi = a.outer_iters[blockIdx.x + a.pair_base];  // read before select_body increments it
    first = oi == 0;
    stampv = (uint32_t)oi + 1u;
  }
  select_body(a, blockIdx.x + a.pair_base, stampv, first, sm, sel_dyn);
}

// ------------------------------------------------------------------------------------------
// a3: K_ws,ws gathered into a dense B x B tile per pair (L2-resident during local_smo)
constexpr int kGatherRows = 16;

// rows [r0, r1) of the pair's K_ws,ws tile (g: >= wn int64 of scratch, filled here)
__device__ void gather_rows_body(const SolverArgs& a, int lp, int r0, int r1, int64_t* g) {
  const PairDesc pd = a.pairs[lp];
  const int wn = a.ws_n[lp];
  const int32_t* ws = a.ws + (int64_t)lp * a.B;
  // FULL_K: global class-sorted columns of the resident matrix; ROW_CACHE: pair-local columns
  for (int e = threadIdx.x; e < wn; e += blockDim.x) g[e] = a.R ? (int64_t)ws[e] : gpos(pd, ws[e]);
  __syncthreads();
  r1 = min(wn, r1);
  const int64_t ldr = (pd.n_s + pd.n_t + 3) & ~3;
  for (int r = r0; r < r1; ++r) {
    const float* row = a.R ? a.R + pd.r_off + (int64_t)a.ws_slot[(int64_t)lp * a.B + r] * ldr : a.K + g[r] * a.ldk;
    float* dst = a.Kws + (int64_t)lp * kws_pair_stride(a.B) + (int64_t)r * a.B;
    for (int e = threadIdx.x; e < wn; e += blockDim.x) dst[e] = __ldg(row + g[e]);
  }
}

__global__ void __launch_bounds__(256) gather_kws_kernel(SolverArgs a, int first) {
  TraceScope ts_(a, blockIdx.x + a.pair_base, 1);
  const int lp = blockIdx.x + a.pair_base;
  if (a.status[lp] != 0) return;
  const PairDesc pd = a.pairs[lp];
  const int np = pd.n_s + pd.n_t;
  if (first < 0) first = a.outer_iters[lp] == 1;  // device-driven loop: after the first selection
  if (np <= a.B && !first) return;  // working set unchanged
  const int r0 = blockIdx.y * kGatherRows;
  if (r0 >= a.ws_n[lp]) return;
  __shared__ int64_t g[1024];
  gather_rows_body(a, lp, r0, r0 + kGatherRows, g);
}

// ------------------------------------------------------------------------------------------
// a5: local SMO on the working set (ImproveSVM, Alg 2 line 10).  One CTA per pair, one
// thread per working-set row (blockDim = B rounded up to a warp multiple, <= 1024).  Per
// inner step: block argmin (u, Eq 4) -> row u of K_ws,ws -> block argmax (l, Eq 5) fused
// with max_{I_l} f -> clipped step (Eq 6-7) -> row l -> f update (Eq 8) on the ws.  The two
// block reductions use redux.sync on 32-bit key words; the winner's alpha, f, K_ii and K_ui
// travel in the reduction payload, so the only dependent global loads are the two K rows,
// and a row already held in registers (u or l of the previous step) is reused.
struct RedSlot {
  uint32_t k0, k1;
  int32_t idx, e;
  double alpha, f;
  uint32_t m0, m1;  // running max key (f_max over I_l)
  float kd, ku;     // K_ee and K_ue of the candidate
};

// lexicographic min of (k0, k1, idx) over the warp; returns the winning lane (lowest on ties)
__device__ __forceinline__ int warp_argmin(uint32_t& k0, uint32_t& k1, int32_t& idx) {
  const uint32_t m0 = __reduce_min_sync(FULLMASK, k0);
  const uint32_t t1 = (k0 == m0) ? k1 : 0xffffffffu;
  const uint32_t m1 = __reduce_min_sync(FULLMASK, t1);
  const bool tie = (k0 == m0) && (k1 == m1);
  const uint32_t t2 = tie ? (uint32_t)idx : 0xffffffffu;
  const uint32_t m2 = __reduce_min_sync(FULLMASK, t2);
  const unsigned b = __ballot_sync(FULLMASK, tie && t2 == m2);
  k0 = m0;
  k1 = m1;
  idx = (int32_t)m2;
  return __ffs(b) - 1;
}
__device__ __forceinline__ void warp_max64(uint32_t& h, uint32_t& l) {
  const uint32_t mh = __reduce_max_sync(FULLMASK, h);
  const uint32_t tl = (h == mh) ? l : 0u;
  l = __reduce_max_sync(FULLMASK, tl);
  h = mh;
}

// Block argmin of (k0,k1,idx) carrying the payload and (WITH_MAX) a running max key (m0,m1).
// barrier over the first nt threads of the CTA (id 0 with nt == blockDim.x is __syncthreads)
__device__ __forceinline__ void bar_sync(int id, int nt) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nt) : "memory");
}

template <bool WITH_MAX>
__device__ __forceinline__ RedSlot block_argmin(const RedSlot& c, RedSlot* slots, int nt, int bar_id) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = nt >> 5;
  uint32_t k0 = c.k0, k1 = c.k1, mh = c.m0, ml = c.m1;
  int32_t idx = c.idx;
  const int wl = warp_argmin(k0, k1, idx);
  if (WITH_MAX) warp_max64(mh, ml);
  if (lane == wl) {
    RedSlot s = c;
    s.m0 = mh;
    s.m1 = ml;
    slots[warp] = s;
  }
  bar_sync(bar_id, nt);
  if (lane < nw) {
    k0 = slots[lane].k0;
    k1 = slots[lane].k1;
    idx = slots[lane].idx;
    mh = slots[lane].m0;
    ml = slots[lane].m1;
  } else {
    k0 = k1 = 0xffffffffu;
    idx = INT_MAX;
    mh = ml = 0u;
  }
  const int w2 = warp_argmin(k0, k1, idx);
  if (WITH_MAX) warp_max64(mh, ml);
  RedSlot out = slots[w2 < nw ? w2 : 0];
  out.m0 = mh;
  out.m1 = ml;
  if (idx == INT_MAX) out.idx = INT_MAX;
  return out;
}

__device__ __forceinline__ RedSlot empty_slot() {
  RedSlot s;
  s.k0 = s.k1 = 0xffffffffu;
  s.idx = INT_MAX;
  s.e = -1;
  s.alpha = s.f = 0.0;
  s.m0 = s.m1 = 0u;
  s.kd = s.ku = 0.f;
  return s;
}

__device__ __forceinline__ bool key_less(uint32_t h, uint32_t l, int32_t i, const RedSlot& c) {
  return h < c.k0 || (h == c.k0 && (l < c.k1 || (l == c.k1 && i < c.idx)));
}

// E working-set rows per thread (thread t owns rows t, t + nt, ...; nt = blockDim.x).
// SMEM: K_ws,ws (B <= kSmemMaxB, built by gather_kws) is copied into shared memory at kernel
// start, so the two row reads of every inner step are LDS instead of L2/HBM loads; otherwise
// rows are read from the global K_ws,ws buffer.
constexpr int kSmemMaxB = 224;

// Run by threads [0, nt) of a CTA; bar_id/nt name the barrier those threads share.
template <int E, bool SMEM>
__device__ void smo_body(const SolverArgs& a, int lp, int nt, int bar_id, RedSlot (*slots)[32], float* kw_smem) {
  const long long t_entry = clock64();
  if (a.status[lp] != 0) return;
  const PairDesc pd = a.pairs[lp];
  const int B = a.B, wn = a.ws_n[lp];
  const double C = a.C;
  const float* Kw;
  if (SMEM) {
    // copy this pair's K_ws,ws tile (built by gather_kws, L2-resident) into shared memory
    const float4* src = reinterpret_cast<const float4*>(a.Kws + (int64_t)lp * kws_pair_stride(B));
    float4* dst = reinterpret_cast<float4*>(kw_smem);
    const int nv = (B * B) / 4;  // B is even and B*B % 4 == 0
    for (int i = threadIdx.x; i < nv; i += nt) dst[i] = __ldg(src + i);
    bar_sync(bar_id, nt);
    Kw = kw_smem;
  } else {
    Kw = a.Kws + (int64_t)lp * kws_pair_stride(B);
  }
  bool valid[E], iu[E], il[E];
  int32_t idx[E];
  int y[E];
  double al[E], a0[E], fv[E];
  float kd[E], va[E], vb[E], ku[E];
#pragma unroll
  for (int q = 0; q < E; ++q) {
    const int e = threadIdx.x + q * nt;
    valid[q] = e < wn;
    idx[q] = valid[q] ? a.ws[(int64_t)lp * B + e] : INT_MAX;
    y[q] = (valid[q] && idx[q] < pd.n_s) ? 1 : -1;
    al[q] = valid[q] ? a.alpha[pd.a_off + idx[q]] : 0.0;
    a0[q] = al[q];
    fv[q] = valid[q] ? a.f[pd.a_off + idx[q]] : 0.0;
    kd[q] = valid[q] ? Kw[(int64_t)e * B + e] : 1.f;
    iu[q] = valid[q] && in_u(y[q], al[q], C);
    il[q] = valid[q] && in_l(y[q], al[q], C);
    va[q] = vb[q] = 0.f;
  }
  // two cached K_ws,ws rows (this thread's entries of them): rows ra / rb
  int ra = -1, rb = -1;
  const int cap = a.inner_cap;
  int it = 0, par = 0;
  double delta0 = 0.0;
  const long long t_begin = clock64();
  long long ph[5] = {0, 0, 0, 0, 0}, tp = t_begin;
  const bool prof = a.smo_phase != nullptr;
  for (;;) {
    // Step 1 (Eq 4): u = argmin_{I_u} f, ties -> lowest pair-local index
    RedSlot c = empty_slot();
#pragma unroll
    for (int q = 0; q < E; ++q) {
      if (iu[q]) {
        const uint64_t key = ord_key(fv[q]);
        const uint32_t h = (uint32_t)(key >> 32), l = (uint32_t)key;
        if (key_less(h, l, idx[q], c)) {
          c.k0 = h;
          c.k1 = l;
          c.idx = idx[q];
          c.e = threadIdx.x + q * nt;
          c.alpha = al[q];
          c.f = fv[q];
          c.kd = kd[q];
        }
      }
    }
    const RedSlot ru = block_argmin<false>(c, slots[par], nt, bar_id);
    par ^= 1;
    if (prof) {
      const long long t = clock64();
      ph[0] += t - tp;
      tp = t;
    }
    if (ru.idx == INT_MAX) break;
    const int ue = ru.e;
    const double fu = ru.f, au = ru.alpha;
    const float kuu = ru.kd;
    const int yu = ru.idx < pd.n_s ? 1 : -1;
    if (ue == ra) {
#pragma unroll
      for (int q = 0; q < E; ++q) ku[q] = va[q];
    } else if (ue == rb) {
#pragma unroll
      for (int q = 0; q < E; ++q) ku[q] = vb[q];
    } else {
      const float* row = Kw + (int64_t)ue * B;
#pragma unroll
      for (int q = 0; q < E; ++q) ku[q] = valid[q] ? row[threadIdx.x + q * nt] : 0.f;
    }
    if (prof) {
      float sum = 0.f;
#pragma unroll
      for (int q = 0; q < E; ++q) sum += ku[q];
      if (sum == -1.f) ph[3] += 1;  // force the loads to complete before reading the clock
      const long long t = clock64();
      ph[1] += t - tp;
      tp = t;
    }
    // Eq 5: l = argmax_{t in I_l, f_t > f_u} (f_u - f_t)^2 / eta_t, and f_max over I_l (Eq 10)
    c = empty_slot();
#pragma unroll
    for (int q = 0; q < E; ++q) {
      if (il[q]) {
        const uint64_t fk = ord_key(fv[q]);
        const uint32_t h = (uint32_t)(fk >> 32), l = (uint32_t)fk;
        if (h > c.m0 || (h == c.m0 && l > c.m1)) {
          c.m0 = h;
          c.m1 = l;
        }
        if (fv[q] > fu) {
          const float eta = fmaxf(kuu + kd[q] - 2.f * ku[q], 1e-12f);
          const float df = (float)(fv[q] - fu);
          const uint32_t sk = ~__float_as_uint(df * df * __frcp_rn(eta));
          if (key_less(sk, 0u, idx[q], c)) {
            c.k0 = sk;
            c.k1 = 0u;
            c.idx = idx[q];
            c.e = threadIdx.x + q * nt;
            c.alpha = al[q];
            c.f = fv[q];
            c.kd = kd[q];
            c.ku = ku[q];
          }
        }
      }
    }
    const RedSlot rl = block_argmin<true>(c, slots[par], nt, bar_id);
    par ^= 1;
    if (prof) {
      const long long t = clock64();
      ph[2] += t - tp;
      tp = t;
    }
    const double fmax = (rl.m0 == 0u && rl.m1 == 0u) ? -DBL_MAX : key_double(((uint64_t)rl.m0 << 32) | rl.m1);
    const double gap = fmax - fu;
    if (it == 0) delta0 = gap;
    const double tol = a.eps > a.local_ratio * delta0 ? a.eps : a.local_ratio * delta0;
    if (!(gap >= tol) || rl.idx == INT_MAX || it >= cap) break;
    const int le = rl.e;
    const double fl = rl.f, alv = rl.alpha;
    const int yl = rl.idx < pd.n_s ? 1 : -1;
    // Step 2 (Eq 6-7) with explicit clipping (reading R4): common step s (FP64)
    double eta = (double)kuu + (double)rl.kd - 2.0 * (double)rl.ku;
    eta = eta > kTau ? eta : kTau;
    double s = (fl - fu) / eta;
    const double Uu = yu > 0 ? C - au : au;
    const double Ll = yl > 0 ? alv : C - alv;
    bool bu = false, bl = false;
    if (Uu <= s) {
      s = Uu;
      bu = true;
    }
    if (Ll <= s) {
      if (Ll < s) bu = false;
      s = Ll;
      bl = true;
    }
    double nau = au + yu * s, nal = alv - yl * s;
    if (bu) nau = yu > 0 ? C : 0.0;
    if (bl) nal = yl > 0 ? 0.0 : C;
    // Step 3 (Eq 8) on the working set: f_i += s (K_ui - K_li)
    float kl[E];
    if (le == ra) {
#pragma unroll
      for (int q = 0; q < E; ++q) kl[q] = va[q];
    } else if (le == rb) {
#pragma unroll
      for (int q = 0; q < E; ++q) kl[q] = vb[q];
    } else {
      const float* row = Kw + (int64_t)le * B;
#pragma unroll
      for (int q = 0; q < E; ++q) kl[q] = valid[q] ? row[threadIdx.x + q * nt] : 0.f;
    }
#pragma unroll
    for (int q = 0; q < E; ++q) {
      const int e = threadIdx.x + q * nt;
      fv[q] += s * ((double)ku[q] - (double)kl[q]);
      if (e == ue || e == le) {
        al[q] = (e == ue) ? nau : nal;
        iu[q] = in_u(y[q], al[q], C);
        il[q] = in_l(y[q], al[q], C);
      }
      va[q] = ku[q];
      vb[q] = kl[q];
    }
    ra = ue;
    rb = le;
    ++it;
    if (prof) {
      const long long t = clock64();
      ph[3] += t - tp;
      tp = t;
    }
  }
#pragma unroll
  for (int q = 0; q < E; ++q) {
    const int e = threadIdx.x + q * nt;
    if (valid[q]) {
      a.alpha[pd.a_off + idx[q]] = al[q];
      a.dcoef[(int64_t)lp * B + e] = (al[q] - a0[q]) * (double)y[q];
    }
  }
  if (threadIdx.x == 0) {
    a.inner_iters[lp] += it;
    a.smo_cycles[lp] += clock64() - t_begin;
    if (prof)
      for (int k = 0; k < 4; ++k) a.smo_phase[lp * 5 + k] += ph[k];
    if (prof) a.smo_phase[lp * 5 + 4] += t_begin - t_entry;
  }
}

template <int E, bool SMEM>
__global__ void __launch_bounds__(SMEM ? kSmemMaxB : 1024 / E) local_smo_kernel(SolverArgs a) {
  TraceScope ts_(a, blockIdx.x + a.pair_base, 2);
  __shared__ RedSlot slots[2][32];
  extern __shared__ float kw_smem[];
  smo_body<E, SMEM>(a, blockIdx.x + a.pair_base, blockDim.x, 0, slots, kw_smem);
}

// ------------------------------------------------------------------------------------------
// a6: f update, f_j += sum_{i in ws, dalpha_i != 0} dalpha_i y_i K_ij for all j in the pair.
// HBM-bound GEMV over the rows with dalpha != 0: each thread owns kFQ 16-byte column quads of
// the pair's two class segments (aligned to the kernel matrix rows, ldk % 4 == 0) and streams
// the rows 2 at a time (kFQ x 2 float4 loads in flight), accumulating in FP64.
constexpr int kFQ = 1;                       // quads per thread
constexpr int kFThreads = 128;
constexpr int kFCols = kFThreads * kFQ * 4;  // columns per CTA (512: many CTAs per pair, short latency)

struct FupSmem {
  double coef[1024];
  const float4* rowp[1024];
  int scan[33];
};

// Quad range [q0, q1) of the pair's concatenated class segments, any blockDim (kFQ quads per
// thread per sweep).  Returns early (uniformly) when no alpha changed.
__device__ void fupdate_body(const SolverArgs& a, int lp, int64_t q0, int64_t q1, FupSmem& fs) {
  const PairDesc pd = a.pairs[lp];
  const bool rc = a.R != nullptr;  // ROW_CACHE: rows are pair-local, columns 0..n_p contiguous
  const int64_t q1b = rc ? 0 : pd.off_s >> 2;
  const int64_t q1e = rc ? (pd.n_s + pd.n_t + 3) >> 2 : (pd.off_s + pd.n_s + 3) >> 2;  // quads of class s
  const int64_t q2b = rc ? 0 : pd.off_t >> 2, q2e = rc ? 0 : (pd.off_t + pd.n_t + 3) >> 2;  // quads of class t
  const int64_t nq1 = q1e - q1b, nq = nq1 + (q2e - q2b);
  const int64_t ldr = (pd.n_s + pd.n_t + 3) & ~3;
  q1 = q1 < nq ? q1 : nq;
  if (q0 >= q1) return;
  const int B = a.B, wn = a.ws_n[lp];
  const int32_t* ws = a.ws + (int64_t)lp * B;
  const double* dc = a.dcoef + (int64_t)lp * B;
  int nnz = 0;
  for (int base = 0; base < wn; base += blockDim.x) {
    const int e = base + threadIdx.x;
    const double c = (e < wn) ? dc[e] : 0.0;
    const bool nz = c != 0.0;
    int tot = 0;
    const int pos = block_excl_scan(nz, tot, fs.scan);
    if (nz) {
      fs.coef[nnz + pos] = c;
      fs.rowp[nnz + pos] = reinterpret_cast<const float4*>(
          rc ? a.R + pd.r_off + (int64_t)a.ws_slot[(int64_t)lp * B + e] * ldr : a.K + gpos(pd, ws[e]) * a.ldk);
    }
    nnz += tot;
  }
  __syncthreads();
  if (nnz == 0) return;
  double* f = a.f + pd.a_off;
  for (int64_t qs = q0; qs < q1; qs += (int64_t)blockDim.x * kFQ) {
    int64_t gq[kFQ];
    bool okq[kFQ], seg1[kFQ];
    double acc[kFQ][4];
#pragma unroll
    for (int u = 0; u < kFQ; ++u) {
      const int64_t qi = qs + threadIdx.x + (int64_t)u * blockDim.x;
      okq[u] = qi < q1;
      seg1[u] = qi < nq1;  // a boundary quad shared by adjacent classes is owned once per segment
      gq[u] = !okq[u] ? 0 : (qi < nq1 ? q1b + qi : q2b + (qi - nq1));
#pragma unroll
      for (int c = 0; c < 4; ++c) acc[u][c] = 0.0;
    }
    // rows 8 at a time: kFQ x 8 independent 16-byte loads in flight per thread (Little's law at
    // ~1.5 us loaded-DRAM latency needs ~10 MB in flight chip-wide for 6.5 TB/s)
    int r = 0;
    for (; r + 8 <= nnz; r += 8) {
      float4 v[8][kFQ];
#pragma unroll
      for (int rr = 0; rr < 8; ++rr)
#pragma unroll
        for (int u = 0; u < kFQ; ++u)
          v[rr][u] = okq[u] ? __ldg(fs.rowp[r + rr] + gq[u]) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int rr = 0; rr < 8; ++rr) {
        const double cv = fs.coef[r + rr];
#pragma unroll
        for (int u = 0; u < kFQ; ++u) {
          acc[u][0] = fma(cv, (double)v[rr][u].x, acc[u][0]);
          acc[u][1] = fma(cv, (double)v[rr][u].y, acc[u][1]);
          acc[u][2] = fma(cv, (double)v[rr][u].z, acc[u][2]);
          acc[u][3] = fma(cv, (double)v[rr][u].w, acc[u][3]);
        }
      }
    }
    for (; r < nnz; ++r) {
      const float4* p0 = fs.rowp[r];
      const double c0v = fs.coef[r];
#pragma unroll
      for (int u = 0; u < kFQ; ++u) {
        const float4 v0 = okq[u] ? __ldg(p0 + gq[u]) : make_float4(0.f, 0.f, 0.f, 0.f);
        acc[u][0] = fma(c0v, (double)v0.x, acc[u][0]);
        acc[u][1] = fma(c0v, (double)v0.y, acc[u][1]);
        acc[u][2] = fma(c0v, (double)v0.z, acc[u][2]);
        acc[u][3] = fma(c0v, (double)v0.w, acc[u][3]);
      }
    }
#pragma unroll
    for (int u = 0; u < kFQ; ++u) {
      if (!okq[u]) continue;
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const int64_t g = gq[u] * 4 + c;  // global (class-sorted) column, or pair-local (ROW_CACHE)
        if (rc) {
          if (g < pd.n_s + pd.n_t) f[g] += acc[u][c];
        } else if (seg1[u]) {
          if (g >= pd.off_s && g < pd.off_s + pd.n_s) f[g - pd.off_s] += acc[u][c];
        } else if (g >= pd.off_t && g < pd.off_t + pd.n_t) {
          f[pd.n_s + (g - pd.off_t)] += acc[u][c];
        }
      }
    }
  }
}

// Row-split f update (the launched kernels): a CTA of kFSWarps warps owns 32 column quads (128
// columns); warp w streams rows w, w + kFSWarps, ... (8 float4 loads in flight per thread), so
// a pair's update has ~n_p/128 CTAs x 256 threads of loads in flight instead of one thread
// walking all rows of its quad; the kFSWarps partial sums are combined in a fixed order
// (deterministic).  FP64 accumulation as in fupdate_body.
constexpr int kFSWarps = 8;
constexpr int kFSThreads = kFSWarps * 32;
constexpr int kFSCols = 128;
struct FupSplitSmem {
  double coef[1024];
  const float4* rowp[1024];
  int scan[33];
  double red[kFSWarps][32][4];
};

__device__ void fupdate_split(const SolverArgs& a, int lp, int64_t q0, FupSplitSmem& fs) {
  const PairDesc pd = a.pairs[lp];
  const bool rc = a.R != nullptr;
  const int64_t q1b = rc ? 0 : pd.off_s >> 2;
  const int64_t q1e = rc ? (pd.n_s + pd.n_t + 3) >> 2 : (pd.off_s + pd.n_s + 3) >> 2;
  const int64_t q2b = rc ? 0 : pd.off_t >> 2, q2e = rc ? 0 : (pd.off_t + pd.n_t + 3) >> 2;
  const int64_t nq1 = q1e - q1b, nq = nq1 + (q2e - q2b);
  const int64_t ldr = (pd.n_s + pd.n_t + 3) & ~3;
  if (q0 >= nq) return;
  const int B = a.B, wn = a.ws_n[lp];
  const int32_t* ws = a.ws + (int64_t)lp * B;
  const double* dc = a.dcoef + (int64_t)lp * B;
  int nnz = 0;
  for (int base = 0; base < wn; base += blockDim.x) {
    const int e = base + threadIdx.x;
    const double c = (e < wn) ? dc[e] : 0.0;
    const bool nz = c != 0.0;
    int tot = 0;
    const int pos = block_excl_scan(nz, tot, fs.scan);
    if (nz) {
      fs.coef[nnz + pos] = c;
      fs.rowp[nnz + pos] = reinterpret_cast<const float4*>(
          rc ? a.R + pd.r_off + (int64_t)a.ws_slot[(int64_t)lp * B + e] * ldr : a.K + gpos(pd, ws[e]) * a.ldk);
    }
    nnz += tot;
  }
  __syncthreads();
  if (nnz == 0) return;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t qi = q0 + lane;
  const bool okq = qi < nq;
  const int64_t gq = !okq ? 0 : (qi < nq1 ? q1b + qi : q2b + (qi - nq1));
  double acc[4] = {0.0, 0.0, 0.0, 0.0};
  int r = warp;
  for (; r + 7 * kFSWarps < nnz; r += 8 * kFSWarps) {
    float4 v[8];
#pragma unroll
    for (int rr = 0; rr < 8; ++rr)
      v[rr] = okq ? __ldg(fs.rowp[r + rr * kFSWarps] + gq) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int rr = 0; rr < 8; ++rr) {
      const double cv = fs.coef[r + rr * kFSWarps];
      acc[0] = fma(cv, (double)v[rr].x, acc[0]);
      acc[1] = fma(cv, (double)v[rr].y, acc[1]);
      acc[2] = fma(cv, (double)v[rr].z, acc[2]);
      acc[3] = fma(cv, (double)v[rr].w, acc[3]);
    }
  }
  for (; r < nnz; r += kFSWarps) {
    const float4 v0 = okq ? __ldg(fs.rowp[r] + gq) : make_float4(0.f, 0.f, 0.f, 0.f);
    const double cv = fs.coef[r];
    acc[0] = fma(cv, (double)v0.x, acc[0]);
    acc[1] = fma(cv, (double)v0.y, acc[1]);
    acc[2] = fma(cv, (double)v0.z, acc[2]);
    acc[3] = fma(cv, (double)v0.w, acc[3]);
  }
#pragma unroll
  for (int c = 0; c < 4; ++c) fs.red[warp][lane][c] = acc[c];
  __syncthreads();
  if (threadIdx.x < 128) {
    const int l = threadIdx.x >> 2, c = threadIdx.x & 3;
    const int64_t qj = q0 + l;
    if (qj < nq) {
      double sum = 0.0;
#pragma unroll
      for (int w = 0; w < kFSWarps; ++w) sum += fs.red[w][l][c];
      const bool seg1 = qj < nq1;  // a boundary quad shared by adjacent classes is owned once per segment
      const int64_t g = (seg1 ? q1b + qj : q2b + (qj - nq1)) * 4 + c;
      double* f = a.f + pd.a_off;
      if (rc) {
        if (g < pd.n_s + pd.n_t) f[g] += sum;
      } else if (seg1) {
        if (g >= pd.off_s && g < pd.off_s + pd.n_s) f[g - pd.off_s] += sum;
      } else if (g >= pd.off_t && g < pd.off_t + pd.n_t) {
        f[pd.n_s + (g - pd.off_t)] += sum;
      }
    }
  }
}

// f update + loop condition of the device-driven (graph) outer loop of one pair: continue while
// the pair is active and below the outer-iteration cap.
__global__ void __launch_bounds__(kFSThreads) f_update_loop_kernel(SolverArgs a, cudaGraphConditionalHandle h,
                                                                   int64_t max_outer) {
  TraceScope ts_(a, blockIdx.x + a.pair_base, 3);
  const int lp = blockIdx.x + a.pair_base;
  if (blockIdx.x == 0 && blockIdx.y == 0 && threadIdx.x == 0) {
    // the branch's pairs run in lockstep: continue while any of them is active
    bool more = false;
    for (int i = 0; i < (int)gridDim.x; ++i) {
      const int p = a.pair_base + i;
      more = more || (a.status[p] == 0 && (int64_t)a.outer_iters[p] < max_outer);
    }
    cudaGraphSetConditional(h, more ? 1u : 0u);
    a.body_iters[a.pair_base] += 1;
  }
  if (a.status[lp] != 0) return;
  __shared__ FupSplitSmem fs;
  fupdate_split(a, lp, (int64_t)blockIdx.y * 32, fs);
}

__global__ void __launch_bounds__(kFSThreads) f_update_kernel(SolverArgs a) {
  TraceScope ts_(a, blockIdx.x + a.pair_base, 3);
  const int lp = blockIdx.x + a.pair_base;
  if (a.status[lp] != 0) return;
  __shared__ FupSplitSmem fs;
  fupdate_split(a, lp, (int64_t)blockIdx.y * 32, fs);
}


// ------------------------------------------------------------------------------------------
// ROW_CACHE regime (a2 + a3 when the n x n kernel matrix does not fit): per outer iteration the
// kernel rows of each pair's NEW working-set entries (positions ws_keep..ws_n) are computed
// against the pair's instances into the pair's B-row buffer R (the paper's GPU buffer,
// L299-L303; retained rows are reused, L297), in pair-local column order.
__global__ void rows_gather_kernel(SolverArgs a) {
  TraceScope ts_(a, blockIdx.x + a.pair_base, 4);
  const int lp = blockIdx.x + a.pair_base;
  if (a.status[lp] != 0) return;
  const PairDesc pd = a.pairs[lp];
  const int keep = a.ws_keep[lp], wn = a.ws_n[lp], nnew = wn - keep;
  if (nnew <= 0) return;
  const int B = a.B;
  if (blockIdx.y == 0 && threadIdx.x == 0) a.rows_done[lp] += nnew;
  float* at = a.ATnew + (int64_t)lp * a.d_pad * a.ldat;
  const int32_t* ws = a.ws + (int64_t)lp * B;
  for (int c = blockIdx.y; c < a.d_pad; c += gridDim.y)
    for (int i = threadIdx.x; i < a.ldat; i += blockDim.x)
      at[(int64_t)c * a.ldat + i] = i < nnew ? a.XT[(int64_t)c * a.ldx + gpos(pd, ws[keep + i])] : 0.f;
}

__global__ void __launch_bounds__(kGemmThreads, 2) rows_contract_kernel(SolverArgs a, float scale) {
  TraceScope ts_(a, blockIdx.x + a.pair_base, 5);
  __shared__ __align__(16) GemmSmem sm;
  const int lp = blockIdx.x + a.pair_base;
  if (a.status[lp] != 0) return;
  const PairDesc pd = a.pairs[lp];
  const int keep = a.ws_keep[lp], wn = a.ws_n[lp], nnew = wn - keep;
  const int rt = blockIdx.z;  // 128-row tile of the new rows
  if (rt * kTile >= nnew) return;
  // column tile -> (segment, first global column); segments start at 4-aligned global columns
  const int64_t sb = pd.off_s & ~3ll, tb = pd.off_t & ~3ll;
  const int ts = (int)((pd.off_s + pd.n_s - sb + kTile - 1) / kTile);
  const int tt = (int)((pd.off_t + pd.n_t - tb + kTile - 1) / kTile);
  const int ct = blockIdx.y;
  if (ct >= ts + tt) return;
  const bool seg_s = ct < ts;
  const int64_t c0 = seg_s ? sb + (int64_t)ct * kTile : tb + (int64_t)(ct - ts) * kTile;
  const int64_t lo = seg_s ? pd.off_s : pd.off_t, hi = seg_s ? pd.off_s + pd.n_s : pd.off_t + pd.n_t;
  const int64_t loc0 = seg_s ? -pd.off_s : pd.n_s - pd.off_t;  // pair-local column = g + loc0
  float acc[8][8];
  gemm_tile_128(a.ATnew + (int64_t)lp * a.d_pad * a.ldat, a.ldat, (int64_t)rt * kTile, a.XT, a.ldx, c0, a.d_pad, sm, acc);
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int32_t* ws = a.ws + (int64_t)lp * a.B;
  const int32_t* slot = a.ws_slot + (int64_t)lp * a.B;
  const int64_t ldr = (pd.n_s + pd.n_t + 3) & ~3;
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = rt * kTile + tile_row(ty, i);  // index among the new rows
    if (r >= nnew) continue;
    const int64_t gr = gpos(pd, ws[keep + r]);
    const float nr = a.norms[gr];
    float* dst = a.R + pd.r_off + (int64_t)slot[keep + r] * ldr;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int64_t g = c0 + tile_col(tx, j);
      if (g < lo || g >= hi) continue;
      const float d2 = fmaf(-2.f, acc[i][j], nr + a.norms[g]);
      dst[g + loc0] = (g == gr) ? 1.f : fast_exp2(fmaxf(d2, 0.f) * scale);
    }
  }
}

void launch_rows_compute(const SolverArgs& a, int P, int64_t np_max, cudaStream_t st) {
  GM_LAUNCH(rows_gather_kernel, dim3(P, 32), dim3(256), 0, st, a);
  const int ctiles = (int)ceil_div(np_max + 8, kTile) + 2;
  const float scale = (float)(-a.gamma * 1.4426950408889634);
  GM_LAUNCH(rows_contract_kernel, dim3(P, ctiles, (unsigned)ceil_div(a.B, kTile)), dim3(kGemmThreads), 0, st, a, scale);
}

// ------------------------------------------------------------------------------------------
// a7: bias and in-sample decision values
__global__ void __launch_bounds__(1024) finalize_kernel(SolverArgs a) {
  __shared__ double red[32];
  const int lp = blockIdx.x + a.pair_base;
  const PairDesc pd = a.pairs[lp];
  const int np = pd.n_s + pd.n_t;
  const double* al = a.alpha + pd.a_off;
  const double* fl = a.f + pd.a_off;
  const double C = a.C;
  double sum_free = 0.0, n_free = 0.0, ub = DBL_MAX, lb = -DBL_MAX;
  for (int i = threadIdx.x; i < np; i += blockDim.x) {
    const int y = i < pd.n_s ? 1 : -1;
    const double av = al[i], fv = fl[i];
    if (av > 0.0 && av < C) {
      sum_free += fv;
      n_free += 1.0;
    } else {
      if (in_u(y, av, C)) ub = ub < fv ? ub : fv;
      if (in_l(y, av, C)) lb = lb > fv ? lb : fv;
    }
  }
  auto add = [](double x, double y) { return x + y; };
  sum_free = block_reduce(sum_free, add, red);
  n_free = block_reduce(n_free, add, red);
  ub = block_reduce(ub, [](double x, double y) { return x < y ? x : y; }, red);
  lb = block_reduce(lb, [](double x, double y) { return x > y ? x : y; }, red);
  const double rho = n_free > 0.0 ? sum_free / n_free : 0.5 * (ub + lb);
  if (threadIdx.x == 0) a.b[lp] = -rho;
  for (int i = threadIdx.x; i < np; i += blockDim.x) {
    const int y = i < pd.n_s ? 1 : -1;
    a.v[pd.a_off + i] = fl[i] + (double)y - rho;
  }
}

// ------------------------------------------------------------------------------------------
// a8: Platt sigmoid fit (Eq 12-13), Newton + backtracking with the constants of ref [15]
// (reading R12); 4 candidate step sizes evaluated per pass over the data (L327).
template <int N>
__device__ void block_sum_n(double (&v)[N], double* sm /* 32*N */) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
#pragma unroll
  for (int q = 0; q < N; ++q)
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v[q] += __shfl_xor_sync(FULLMASK, v[q], o);
  __syncthreads();
  if (lane == 0)
#pragma unroll
    for (int q = 0; q < N; ++q) sm[q * 32 + warp] = v[q];
  __syncthreads();
#pragma unroll
  for (int q = 0; q < N; ++q) {
    double s = 0.0;
    for (int w = 0; w < nw; ++w) s += sm[q * 32 + w];
    v[q] = s;
  }
}

__device__ __forceinline__ double nll_term(double v, double t, double A, double B) {
  const double z = v * A + B;
  return z >= 0.0 ? t * z + log1p(exp(-z)) : (t - 1.0) * z + log1p(exp(z));
}

__global__ void __launch_bounds__(512) sigmoid_fit_kernel(SolverArgs a) {
  __shared__ double sm[32 * 5];
  const int lp = blockIdx.x + a.pair_base;
  const PairDesc pd = a.pairs[lp];
  const int np = pd.n_s + pd.n_t;
  const double* v = a.v + pd.a_off;
  const double Np = pd.n_s, Nm = pd.n_t;
  const double hi = (Np + 1.0) / (Np + 2.0), lo = 1.0 / (Nm + 2.0);
  const int max_iter = 100;
  const double min_step = 1e-10, sigma = 1e-12, geps = 1e-5;
  double A = 0.0, B = log((Nm + 1.0) / (Np + 1.0));
  double F;
  {
    double s[1] = {0.0};
    for (int i = threadIdx.x; i < np; i += blockDim.x) s[0] += nll_term(v[i], i < pd.n_s ? hi : lo, A, B);
    block_sum_n<1>(s, sm);
    F = s[0];
  }
  int status = 0, it = 0;
  for (; it < max_iter; ++it) {
    double h[5] = {0.0, 0.0, 0.0, 0.0, 0.0};  // h11, h22, h21, g1, g2
    for (int i = threadIdx.x; i < np; i += blockDim.x) {
      const double vi = v[i], t = i < pd.n_s ? hi : lo;
      const double z = vi * A + B;
      double p, q;
      if (z >= 0.0) {
        const double e = exp(-z);
        p = e / (1.0 + e);
        q = 1.0 / (1.0 + e);
      } else {
        const double e = exp(z);
        p = 1.0 / (1.0 + e);
        q = e / (1.0 + e);
      }
      const double d2 = p * q;
      h[0] += vi * vi * d2;
      h[1] += d2;
      h[2] += vi * d2;
      const double d1 = t - p;
      h[3] += vi * d1;
      h[4] += d1;
    }
    block_sum_n<5>(h, sm);
    const double h11 = h[0] + sigma, h22 = h[1] + sigma, h21 = h[2], g1 = h[3], g2 = h[4];
    if (fabs(g1) < geps && fabs(g2) < geps) break;
    const double det = h11 * h22 - h21 * h21;
    const double dA = -(h22 * g1 - h21 * g2) / det;
    const double dB = -(-h21 * g1 + h11 * g2) / det;
    const double gd = g1 * dA + g2 * dB;
    double step = 1.0;
    bool found = false;
    int ncand = 1;  // the full Newton step first (accepted in most iterations), then 4 halvings per pass
    while (step >= min_step && !found) {
      double fs[4] = {0.0, 0.0, 0.0, 0.0};
      for (int i = threadIdx.x; i < np; i += blockDim.x) {
        const double vi = v[i], t = i < pd.n_s ? hi : lo;
        double st = step;
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          if (c < ncand) fs[c] += nll_term(vi, t, A + st * dA, B + st * dB);
          st *= 0.5;
        }
      }
      block_sum_n<4>(fs, sm);
      double st = step;
      for (int c = 0; c < ncand && st >= min_step; ++c) {
        if (fs[c] < F + 1e-4 * st * gd) {
          A += st * dA;
          B += st * dB;
          F = fs[c];
          found = true;
          break;
        }
        st *= 0.5;
      }
      step = st;  // if none accepted: continue with the next halvings
      ncand = 4;
    }
    if (!found) {
      status = 2;
      break;
    }
  }
  if (it >= max_iter) status = 1;
  if (threadIdx.x == 0) {
    a.A[lp] = A;
    a.Bs[lp] = B;
    a.sig_status[lp] = status;
  }
}

// ------------------------------------------------------------------------------------------
// a9: SV union flags over class-sorted positions
__global__ void sv_flags_kernel(SolverArgs a, uint8_t* flags) {
  const int lp = blockIdx.x + a.pair_base;
  const PairDesc pd = a.pairs[lp];
  const int np = pd.n_s + pd.n_t;
  const int64_t j = (int64_t)blockIdx.y * blockDim.x + threadIdx.x;
  if (j < np && a.alpha[pd.a_off + j] > 0.0) flags[gpos(pd, j)] = 1;
}

// ------------------------------------------------------------------------------------------
void launch_init_pairs(const SolverArgs& a, int P, int64_t tot, cudaStream_t st) {
  const int64_t nthr = tot > P ? tot : P;
  GM_LAUNCH(init_pairs_kernel, dim3((unsigned)ceil_div(nthr, 256)), dim3(256), 0, st, a, tot, P);
}
void launch_select_ws(const SolverArgs& a, int P, uint32_t stampv, int first, cudaStream_t st) {
  const size_t dyn = (size_t)kSelSmemMax * 9 + 16 + sizeof(SelLists);  // keys (8 B) + flags (1 B) + lists
  set_max_dyn_smem(select_ws_kernel, dyn);
  GM_LAUNCH(select_ws_kernel, dim3(P), dim3(1024), dyn, st, a, stampv, first);
}
void launch_gather_kws(const SolverArgs& a, int P, int first, cudaStream_t st) {
  GM_LAUNCH(gather_kws_kernel, dim3(P, (unsigned)ceil_div(a.B, kGatherRows)), dim3(256), 0, st, a, first);
}
bool local_smo_uses_smem(int B) { return B <= kSmemMaxB; }

void launch_local_smo(const SolverArgs& a, int P, cudaStream_t st) {
  if (local_smo_uses_smem(a.B)) {
    const size_t dyn = (size_t)a.B * a.B * sizeof(float);
    set_max_dyn_smem(local_smo_kernel<1, true>, (size_t)kSmemMaxB * kSmemMaxB * 4 + kSmemMaxB * 4);
    GM_LAUNCH((local_smo_kernel<1, true>), dim3(P), dim3((unsigned)round_up(a.B, 32)), dyn, st, a);
    return;
  }
  // E working-set rows per thread (B <= 1024 with at most 512 threads)
  const int E = a.B > 256 ? 2 : 1;
  const int nt = (int)round_up(ceil_div(a.B, E), 32);
  if (E == 1) GM_LAUNCH((local_smo_kernel<1, false>), dim3(P), dim3(nt), 0, st, a);
  else GM_LAUNCH((local_smo_kernel<2, false>), dim3(P), dim3(nt), 0, st, a);
}
void launch_f_update(const SolverArgs& a, int P, int64_t np_max, cudaStream_t st) {
  // +8 columns: each class segment may add a partial quad at either end
  GM_LAUNCH(f_update_kernel, dim3(P, (unsigned)ceil_div(np_max + 8, kFSCols)), dim3(kFSThreads), 0, st, a);
}
void launch_f_update_loop(const SolverArgs& a, int P, int64_t np_max, cudaGraphConditionalHandle h, int64_t max_outer,
                          cudaStream_t st) {
  GM_LAUNCH(f_update_loop_kernel, dim3(P, (unsigned)ceil_div(np_max + 8, kFSCols)), dim3(kFSThreads), 0, st, a, h,
            max_outer);
}
void launch_finalize(const SolverArgs& a, int P, cudaStream_t st) {
  GM_LAUNCH(finalize_kernel, dim3(P), dim3(1024), 0, st, a);
}
// NEXT-2: out-of-fold decision values of held-out rows into the pairs' pair-local layout.
// Row h (class cls[h], rank rnk[h] within its class) of a fold's held-out set feeds every pair
// (s, t) containing its class: v[a_off(p) + (cls == s ? rnk : n_s + rnk)] = dec[h][p].
__global__ void scatter_oof_kernel(const double* __restrict__ dec, int64_t m, int P, const int32_t* __restrict__ cls,
                                   const int64_t* __restrict__ rnk, const PairDesc* __restrict__ pairs,
                                   double* __restrict__ v) {
  const int64_t gid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (gid >= m * P) return;
  const int64_t h = gid / P;
  const int p = (int)(gid % P);
  const PairDesc pd = pairs[p];
  const int c = cls[h];
  if (c != pd.s && c != pd.t) return;
  v[pd.a_off + (c == pd.s ? rnk[h] : pd.n_s + rnk[h])] = dec[gid];
}

void launch_scatter_oof(const double* dec, int64_t m, int P, const int32_t* cls, const int64_t* rnk,
                        const PairDesc* pairs, double* v, cudaStream_t st) {
  const int64_t tot = m * (int64_t)P;
  if (tot > 0) GM_LAUNCH(scatter_oof_kernel, dim3((unsigned)ceil_div(tot, 256)), dim3(256), 0, st, dec, m, P, cls, rnk, pairs, v);
}

// the Platt fit (Eq 12-13) of every pair on given decision values v (pair-local layout, a_off)
void launch_sigmoid_fit_on(const PairDesc* pairs, int P, const double* v, double* A, double* B, int32_t* status,
                           cudaStream_t st) {
  SolverArgs a;
  std::memset(&a, 0, sizeof(a));
  a.pairs = pairs;
  a.v = const_cast<double*>(v);
  a.A = A;
  a.Bs = B;
  a.sig_status = status;
  a.pair_base = 0;
  GM_LAUNCH(sigmoid_fit_kernel, dim3(P), dim3(512), 0, st, a);
}

void launch_sigmoid_fit(const SolverArgs& a, int P, cudaStream_t st) {
  GM_LAUNCH(sigmoid_fit_kernel, dim3(P), dim3(512), 0, st, a);
}
void launch_sv_flags(const SolverArgs& a, int P, int64_t np_max, uint8_t* flags, cudaStream_t st) {
  GM_LAUNCH(sv_flags_kernel, dim3(P, (unsigned)ceil_div(np_max, 256)), dim3(256), 0, st, a, flags);
}

}  // namespace gmpsvm
