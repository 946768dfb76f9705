// wsolve.cu -- the default solver kernels of one outer iteration (FULL_K regime, B <= 224,
// n_p <= 16384), Algorithm 2 lines 6-10 (L293-L305):
//
//   ws_select_kernel   a4  one 1024-thread CTA per pair.  Stages every instance's key ord(f) and
//                          I_u / I_l flags in shared memory together with the global stop test
//                          (Eq 9-10).  Sort-free selection: the r-th smallest of the warps' four
//                          smallest per-thread minima is a threshold T with at least r candidates
//                          <= T; one compaction pass collects the (few) candidates <= T and their
//                          exact (key, index) ranks are counted -- O(list^2) compares on a list of
//                          ~r entries.  Same semantics as select_body (reading R19): the newest
//                          B - q rows retained, q/2 smallest f in I_u, the rest largest f in I_l.
//                          The working set is written twice: in age order (retention) and sorted
//                          by pair-local index (everything else), so "lowest position" == "lowest
//                          index" for the tie rule R5 in the local solver.
//   ws_gather_kernel   a3  K_ws,ws from the resident class-sorted kernel matrix, rows spread over
//                          many CTAs (the gather is scattered 4-byte loads: one SM's outstanding
//                          misses bound it at ~80 us, measured), into an L2-resident tile.
//   ws_smo_kernel      a5  ONE warp per pair: the tile is bulk-copied (cp.async.bulk) into shared
//                          memory; lane l owns working-set rows l, l+32, ...  Per inner step
//                          (Eq 4-8, WSS2, local stop R20): per-lane min/max over its rows,
//                          redux.sync over the warp -- no CTA barrier, no shared reduction slots.
#include <algorithm>
#include <cfloat>
#include <climits>
#include <cstdlib>
#include <string>

#include <math_constants.h>

#include "kernels.h"
#include "solver_dev.cuh"

namespace gmpsvm {

constexpr int kWT = 1024;        // select threads per CTA
constexpr int kWMaxNp = kWsMaxNp;  // pair size up to which keys and flags fit in shared memory
constexpr int kWMaxB = 224;      // working-set rows (tile in the SMO kernel's shared memory)
constexpr int kBufW = 16;        // per-warp candidate buffer (per side)
constexpr int kFlat = 512;       // flattened candidate list capacity (per side)
constexpr int kWRank = 128;      // threshold samples per side (4 per warp)
#ifndef GMPSVM_STAGE_UNROLL
#define GMPSVM_STAGE_UNROLL 4
#endif
constexpr int kStageUnroll = GMPSVM_STAGE_UNROLL;  // staging: elements (alpha + f loads) in flight per thread

__host__ __device__ inline int ws_tile_ld(int B) { return (B + 3) & ~3; }

// Programmatic dependent launch: each kernel of an outer iteration lets the next one be scheduled
// at once (its CTAs become resident and wait), and waits for its predecessor's completion and
// memory before touching shared state -- the launch latency leaves the per-iteration chain.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_enter() {
  pdl_wait();
  pdl_trigger();
}

struct WSelSmall {
  uint32_t retained[kWMaxNp / 32];  // retained rows; then the write-out bitmap
  double red[2][32];
  uint64_t sk[2][kWRank];  // the warps' 4 smallest per-thread minima (candidate keys, below)
  uint64_t bk[2][32][kBufW];  // per-warp candidates <= threshold
  int32_t bcnt[2][32];
  int32_t boff[2][33];
  uint64_t fk[2][kFlat];  // flattened candidate lists
  int32_t pick[1024];  // new working set in age order
  int32_t wpre[kWMaxNp / 32];  // prefix popcounts of the picked-index bitmap
  uint64_t thr_k[2];
  int32_t overflow;
  SelSmem sel;  // radix_pick fallback
};

// Candidate keys: the order-preserving key of f (I_u side) or of -f (I_l side) with its low 14 bits
// replaced by the pair-local index (n_p <= kWMaxNp = 2^14), so one 64-bit compare orders the
// candidates by value and then by index (R19 / R5: smallest f first, lowest index on ties).
// Values closer than 2^-38 relative count as equal and go by index.
constexpr uint64_t kIdxBits = 14, kIdxMask = (1ull << kIdxBits) - 1;
static_assert(kWMaxNp <= (1 << kIdxBits), "the index must fit the key's low bits");
__device__ __forceinline__ uint64_t ckey_u(double f, int i) { return (ord_key(f) & ~kIdxMask) | (uint64_t)i; }
__device__ __forceinline__ uint64_t ckey_l_of_u(uint64_t ku) { return (~ku & ~kIdxMask) | (ku & kIdxMask); }
__device__ __forceinline__ int ckey_idx(uint64_t k) { return (int)(k & kIdxMask); }

// warp min of distinct keys (~0: none); all lanes get it; returns the winner's lane (-1: none)
__device__ __forceinline__ int warp_min_k(uint64_t& k) {
  const uint32_t h = (uint32_t)(k >> 32), l = (uint32_t)k;
  const uint32_t m0 = __reduce_min_sync(FULLMASK, h);
  const uint32_t m1 = __reduce_min_sync(FULLMASK, h == m0 ? l : 0xffffffffu);
  const uint64_t m = ((uint64_t)m0 << 32) | m1;
  const unsigned b = __ballot_sync(FULLMASK, k == m && m != ~0ull);
  k = m;
  return __ffs(b) - 1;
}

// radix_pick's view of the combined keys (its `~key` for the I_l side inverts only the value bits)
struct SmemSrcCK {
  const uint64_t* keys;
  uint8_t* flags;  // bit0 in I_u, bit1 in I_l, bit2 taken / retained
  template <bool SIDE_U>
  __device__ __forceinline__ bool cand(int i, uint64_t& key) const {
    const uint8_t fl = flags[i];
    if (!(fl & (SIDE_U ? 1 : 2)) || (fl & 4)) return false;
    key = SIDE_U ? keys[i] : ckey_l_of_u(keys[i]);
    return true;
  }
  __device__ __forceinline__ void take(int i) const { flags[i] |= 4; }
};

// Threads per list entry for a rank count over n entries by the whole CTA: the largest power of
// two g <= 32 with n * g <= kWT (g lanes of one warp share an entry and split its comparisons).
__device__ __forceinline__ int rank_group(int n) {
  int g = 32;
  while (g > 1 && n * g > kWT) g >>= 1;
  return g;
}
__device__ __forceinline__ int group_sum(int v, int g) {  // sum over the g-lane group (g | 32)
#pragma unroll
  for (int o = 16; o > 0; o >>= 1)
    if (o < g) v += __shfl_xor_sync(FULLMASK, v, o);
  return v;
}

// exclusive prefix over the block of one value per thread (block order = thread order)
__device__ __forceinline__ int block_excl_scan_count_thread(int v, int& total, int* sm /* 33 */) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(FULLMASK, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) sm[warp] = x;
  __syncthreads();
  if (warp == 0) {
    const int w = lane < nw ? sm[lane] : 0;
    int z = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(FULLMASK, z, o);
      if (lane >= o) z += y;
    }
    if (lane < nw) sm[lane] = z - w;
    if (lane == 31) sm[32] = z;
  }
  __syncthreads();
  total = sm[32];
  return sm[warp] + x - v;
}

// ------------------------------------------------------------------------------------------
// Kws buffer of a pair: the K_ws,ws tile (B rows, stride ld) followed by the local solver's
// state in sorted order: alpha[B] (FP64), f[B] (FP64), index[round_up(B, 4)] (int32).
__host__ __device__ inline size_t ws_state_off(int B) { return (size_t)B * ws_tile_ld(B); }  // in floats
__host__ __device__ inline size_t ws_buf_floats(int B) { return kws_pair_stride(B); }  // tile + state

// exclusive prefix of the popcounts of nwords bitmap words (any blockDim); sm: 33 ints
__device__ void bitmap_prefix(const uint32_t* bm, int nwords, int32_t* wpre, int* sm) {
  int carry = 0;
  for (int base = 0; base < nwords; base += blockDim.x) {
    const int w = base + threadIdx.x;
    const int v = w < nwords ? __popc(bm[w]) : 0;
    int tot = 0;
    const int pre = block_excl_scan_count_thread(v, tot, sm);
    if (w < nwords) wpre[w] = carry + pre;
    carry += tot;
    __syncthreads();
  }
}

// Publishes the new working set of pair lp (pick[0..cnt) in age order, oldest first): a.ws_tmp
// (age order, for the next retention), a.ws (sorted by pair-local index), a.ws_n, and the SMO
// state (alpha, f, index in sorted order) behind the pair's tile.  All threads; bm:
// kWsMaxNp/32 words, wpre: kWsMaxNp/32, sm: 33 ints of shared scratch.
__device__ void ws_write_out(const SolverArgs& a, int lp, const int32_t* pick, int cnt, uint32_t* bm, int32_t* wpre,
                             int* sm) {
  const int t = threadIdx.x;
  long long tq = clock64();
  auto mark = [&](int k) {  // GMPSVM_SMO_PHASES: write-out sub-phase cycles (thread 0)
    if (a.sel_phase && t == 0) {
      const long long tc = clock64();
      a.sel_phase[(int64_t)(lp + 8192) * 5 + k] += tc - tq;
      tq = tc;
    }
  };
  const PairDesc pd = a.pairs[lp];
  const int np = pd.n_s + pd.n_t, B = a.B, nwords = (np + 31) / 32;
  for (int w = t; w < nwords; w += blockDim.x) bm[w] = 0u;
  __syncthreads();
  for (int e = t; e < cnt; e += blockDim.x) atomicOr(&bm[pick[e] >> 5], 1u << (pick[e] & 31));
  __syncthreads();
  mark(0);
  bitmap_prefix(bm, nwords, wpre, sm);
  mark(1);
  float* buf = a.Kws + (int64_t)lp * ws_buf_floats(B);
  double* st_al = reinterpret_cast<double*>(buf + ws_state_off(B));
  double* st_f = st_al + B;
  int32_t* st_ix = reinterpret_cast<int32_t*>(st_f + B);
  for (int e = t; e < cnt; e += blockDim.x) {
    const int32_t x = pick[e];
    const int rank = wpre[x >> 5] + __popc(bm[x >> 5] & ((1u << (x & 31)) - 1u));
    a.ws_tmp[(int64_t)lp * B + e] = x;
    a.ws[(int64_t)lp * B + rank] = x;
    st_al[rank] = __ldcg(a.alpha + pd.a_off + x);  // L2 loads: written by other CTAs of a persistent solver
    st_f[rank] = __ldcg(a.f + pd.a_off + x);
    st_ix[rank] = x;
  }
  mark(2);
  if (t == 0) a.ws_n[lp] = cnt;
}

// ------------------------------------------------------------------------------------------
// a4 selection
// The selection of pair lp by the whole (kWT-thread) CTA: sdyn holds kWMaxNp * 9 bytes (keys,
// flags), W the rest.  pdl: called from ws_select_kernel (programmatic dependent launch); the
// persistent solver (ws_persist_kernel) calls it with its own ordering.
__device__ __forceinline__ void ws_select_body(const SolverArgs& a, const int lp, const int64_t max_outer,
                                               unsigned char* sdyn, WSelSmall& W, const bool pdl) {
  uint64_t* keys = reinterpret_cast<uint64_t*>(sdyn);
  uint8_t* flags = sdyn + (size_t)kWMaxNp * 8;
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  const PairDesc pd = a.pairs[lp];
  const int np = pd.n_s + pd.n_t, B = a.B;
  const double C = a.C;
  const double* al = a.alpha + pd.a_off;
  const double* fl = a.f + pd.a_off;
  const uint8_t* ulf = a.ulf ? a.ulf + pd.a_off : nullptr;
  // Before the dependency wait: the retained rows come from the previous selection's output
  // (ws_tmp, ws_n, outer_iters), which completed before this launch's predecessor (the f-update)
  // was released, so building their bitmap overlaps the f-update's tail.  L2 loads (.cg).
  const int first = __ldcg(a.outer_iters + lp) == 0;
  int32_t* ws_age = a.ws_tmp + (int64_t)lp * B;  // age order (oldest first)
  long long tq = clock64();
  auto mark = [&](int k) {  // GMPSVM_SMO_PHASES: selection sub-phase cycles (thread 0)
    if (a.sel_phase && t == 0) {
      const long long tc = clock64();
      a.sel_phase[(int64_t)(lp + 4096) * 5 + k] += tc - tq;
      tq = tc;
    }
  };
  // retained rows: the newest B - q of the previous working set (reading R19)
  const int prev_n = first ? 0 : __ldcg(a.ws_n + lp);
  const int keep = np <= B ? 0 : min(prev_n, B - a.q);
  for (int w = t; w < (np + 31) / 32; w += kWT) W.retained[w] = 0u;
  if (t == 0) W.overflow = 0;
  __syncthreads();
  for (int e = t; e < keep; e += kWT) {
    const int idx = __ldcg(ws_age + prev_n - keep + e);
    W.pick[e] = idx;
    atomicOr(&W.retained[idx >> 5], 1u << (idx & 31));
  }
  const int64_t t_res = (a.trace && lp == a.trace_pair && t == 0) ? (int64_t)gtimer() : 0;
  if (pdl) pdl_enter();  // alpha (local SMO), f (f-update) and status are read after the wait
  if (t_res) {  // GMPSVM_TRACE: f-update grid end -> selection released; selection resident -> released
    const int64_t t_go = (int64_t)gtimer();
    const int64_t fe = (int64_t)*trace_fu_end(a);
    if (fe) trace_rec(a, 7, fe, t_go);
    trace_rec(a, 8, t_res, t_go);
  }
  TraceScope ts_(a, lp, 0);
  if (a.status[lp] != 0) return;
  tq = clock64();
  __syncthreads();
  // stage keys / flags, stop test (Eq 9-10), per-thread minima of the candidates of both sides
  double fmin = DBL_MAX, fmax = -DBL_MAX;
  uint64_t mk[2] = {~0ull, ~0ull};
  for (int base = 0; base < np; base += kStageUnroll * kWT) {
    double av[kStageUnroll], fv[kStageUnroll];
    uint8_t uf[kStageUnroll];
#pragma unroll
    for (int m = 0; m < kStageUnroll; ++m) {
      const int i = base + m * kWT + t;
      if (ulf) uf[m] = i < np ? __ldcg(ulf + i) : (uint8_t)0;  // membership bits (1 B) instead of alpha (8 B)
      else av[m] = i < np ? __ldcg(al + i) : 0.0;  // L2 loads (see ws_write_out)
      fv[m] = i < np ? __ldcg(fl + i) : 0.0;
    }
#pragma unroll
    for (int m = 0; m < kStageUnroll; ++m) {
      const int i = base + m * kWT + t;
      if (i < np) {
        const int y = i < pd.n_s ? 1 : -1;
        const bool u = ulf ? (uf[m] & 1) != 0 : in_u(y, av[m], C), l = ulf ? (uf[m] & 2) != 0 : in_l(y, av[m], C);
        const bool ret = (W.retained[i >> 5] >> (i & 31)) & 1u;
        if (u) fmin = fmin < fv[m] ? fmin : fv[m];
        if (l) fmax = fmax > fv[m] ? fmax : fv[m];
        const uint64_t key = ckey_u(fv[m], i), lkey = ckey_l_of_u(key);
        keys[i] = key;
        flags[i] = (uint8_t)((u ? 1 : 0) | (l ? 2 : 0) | (ret ? 4 : 0));
        if (u && !ret && key < mk[0]) mk[0] = key;
        if (l && !ret && lkey < mk[1]) mk[1] = lkey;
      }
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    fmin = ::fmin(fmin, __shfl_xor_sync(FULLMASK, fmin, o));
    fmax = ::fmax(fmax, __shfl_xor_sync(FULLMASK, fmax, o));
  }
  if (lane == 0) {
    W.red[0][warp] = fmin;
    W.red[1][warp] = fmax;
  }
  __syncthreads();
  fmin = W.red[0][lane];
  fmax = W.red[1][lane];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    fmin = ::fmin(fmin, __shfl_xor_sync(FULLMASK, fmin, o));
    fmax = ::fmax(fmax, __shfl_xor_sync(FULLMASK, fmax, o));
  }
  const double gap = fmax - fmin;
  const bool done = (fmin == DBL_MAX) || (fmax == -DBL_MAX) || !(gap >= a.eps);
  const bool capped = !done && (int64_t)a.outer_iters[lp] >= max_outer;
  if (t == 0) {
    a.gap[lp] = gap;
    if (done) a.status[lp] = 1;
    else if (capped) a.status[lp] = 2;  // outer-iteration cap (GMPSVM_WARN_MAXITER)
    else a.outer_iters[lp] += 1;
  }
  mark(0);
  if (done || capped) return;
  if (np <= B) {  // the whole pair is the working set (unchanged from here on)
    for (int e = t; e < np; e += kWT) W.pick[e] = e;
    __syncthreads();
    ws_write_out(a, lp, W.pick, np, W.retained, W.wpre, W.boff[0]);
    return;
  }
  const int need = B - keep, need_u = need / 2;
  // the four smallest per-thread minima of each warp (both sides), for the thresholds
#pragma unroll 1
  for (int j = 0; j < 4; ++j) {
#pragma unroll
    for (int s = 0; s < 2; ++s) {
      uint64_t k = mk[s];
      const int wl = warp_min_k(k);
      if (lane == 0) W.sk[s][warp * 4 + j] = k;
      if (lane == wl) mk[s] = ~0ull;
    }
  }
  if (t < 2) W.thr_k[t] = ~0ull;  // fewer samples than the rank: every candidate qualifies
  __syncthreads();
  // thresholds by counting ranks: U at rank need_u - 1, L at rank need - 1 (so the L list
  // still holds need - (U picks) candidates after removing the U picks it shares); 4 threads per
  // sample split its comparisons
  {
    constexpr int G = kWT / (2 * kWRank);
    const int e = t / G, sub = t % G;
    const int s = e / kWRank, j = e % kWRank;
    const int r = s == 0 ? need_u : need;
    const uint64_t k = W.sk[s][j];
    int rank = 0;
    for (int q = sub; q < kWRank; q += G) rank += W.sk[s][q] < k ? 1 : 0;
    rank = group_sum(rank, G);
    if (sub == 0) {
      if (k != ~0ull && r >= 1 && r <= kWRank && rank == r - 1) W.thr_k[s] = k;
      if (s == 0 && j == 0 && r == 0) W.thr_k[0] = 0ull;  // nothing wanted from U (no key is 0)
    }
  }
  __syncthreads();
  mark(1);
  // compaction of the candidates at or below the thresholds into per-warp buffers
  {
    const uint64_t tk0 = W.thr_k[0], tk1 = W.thr_k[1];
    int c0 = 0, c1 = 0;
    for (int base = 0; base < np; base += kWT) {
      const int i = base + t;
      bool cu = false, cl = false;
      uint64_t kk = 0, lk = 0;
      if (i < np) {
        const uint8_t fg = flags[i];
        kk = keys[i];
        lk = ckey_l_of_u(kk);
        cu = (fg & 5) == 1 && kk <= tk0;
        cl = (fg & 6) == 2 && lk <= tk1;
      }
      const unsigned bu = __ballot_sync(FULLMASK, cu), bl = __ballot_sync(FULLMASK, cl);
      const int ou = c0 + __popc(bu & ((1u << lane) - 1u)), ol = c1 + __popc(bl & ((1u << lane) - 1u));
      if (cu && ou < kBufW) W.bk[0][warp][ou] = kk;
      if (cl && ol < kBufW) W.bk[1][warp][ol] = lk;
      c0 += __popc(bu);
      c1 += __popc(bl);
    }
    if (lane == 0) {
      W.bcnt[0][warp] = c0;
      W.bcnt[1][warp] = c1;
      if (c0 > kBufW || c1 > kBufW) W.overflow = 1;
    }
  }
  __syncthreads();
  if (warp < 2) {  // prefix offsets of the per-warp buffers (warp s: side s)
    const int v = W.bcnt[warp][lane];
    int x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(FULLMASK, x, o);
      if (lane >= o) x += y;
    }
    W.boff[warp][lane] = x - v;
    if (lane == 31) {
      W.boff[warp][32] = x;
      if (x > kFlat) W.overflow = 1;
    }
  }
  __syncthreads();
  int got = 0;
  mark(2);
  if (!W.overflow) {
    {  // flatten: thread (warp w, lane j) copies slot j of warp w's U (j < 16) or L (j >= 16) buffer
      const int s = lane >> 4, j = lane & 15;
      if (j < W.bcnt[s][warp]) W.fk[s][W.boff[s][warp] + j] = W.bk[s][warp][j];
    }
    __syncthreads();
    const int nu = W.boff[0][32], nl = W.boff[1][32];
    // U: exact (key, index) rank by counting (g threads per entry); the need_u smallest in rank order
    const int got_u = min(need_u, nu);
    {
      const int g = rank_group(nu), e = t / g, sub = t % g;
      uint64_t k = 0;
      int rank = 0;
      if (e < nu) {
        k = W.fk[0][e];
        for (int q = sub; q < nu; q += g) rank += W.fk[0][q] < k ? 1 : 0;
      }
      rank = group_sum(rank, g);
      if (e < nu && sub == 0 && rank < got_u) {
        const int x = ckey_idx(k);
        W.pick[keep + rank] = x;
        flags[x] |= 4;
      }
    }
    __syncthreads();
    // L: rank among the entries U did not take
    const int need_l = need - got_u;
    bool free_l = false;
    {
      const int g = rank_group(nl), e = t / g, sub = t % g;
      int rank = 0;
      int32_t x = 0;
      if (e < nl) {
        const uint64_t k = W.fk[1][e];
        x = ckey_idx(k);
        free_l = !(flags[x] & 4);
        if (free_l)
          for (int q = sub; q < nl; q += g) {
            const uint64_t kq = W.fk[1][q];
            rank += (kq < k && !(flags[ckey_idx(kq)] & 4)) ? 1 : 0;
          }
      }
      rank = group_sum(rank, g);
      free_l = free_l && sub == 0;
      if (free_l && rank < need_l) W.pick[keep + got_u + rank] = x;
    }
    const int nfree = __syncthreads_count(free_l);
    got = got_u + min(need_l, nfree);
    for (int e = keep + got_u + t; e < keep + got; e += kWT) flags[W.pick[e]] |= 4;
    __syncthreads();
    // L ran short (every L candidate is in the list): U again, as select_sides does
    if (got < need) got += radix_pick<true>(SmemSrcCK{keys, flags}, np, need - got, W.pick + keep + got, W.sel);
  } else {  // a buffer overflowed (heavily tied or clustered keys): exact radix selection
    got = select_sides(SmemSrcCK{keys, flags}, np, need, W.pick + keep, W.sel);
    if (a.sel_phase && t == 0) a.sel_phase[(int64_t)(lp + 4096) * 5 + 4] += 1000000;  // fallbacks (diagnostic)
  }
  __syncthreads();
  mark(3);
  const int cnt = keep + got;
  ws_write_out(a, lp, W.pick, cnt, W.retained, W.wpre, W.boff[0]);
  mark(4);
}

__global__ void __launch_bounds__(kWT, 1) ws_select_kernel(SolverArgs a, int64_t max_outer) {
  extern __shared__ __align__(16) unsigned char sdyn[];
  __shared__ WSelSmall W;
  ws_select_body(a, blockIdx.x + a.pair_base, max_outer, sdyn, W, true);
}

// ------------------------------------------------------------------------------------------
// a3: K_ws,ws tile (row stride ws_tile_ld(B)) from the resident kernel matrix
constexpr int kGR = 8;  // tile rows per CTA

// rows [by * kGR, +kGR) of pair lp's tile by one 256-thread CTA (g: kWMaxB shared slots).  The
// working set is read from L2: the persistent solver's workers run beside the selection's CTA.
__device__ __forceinline__ void ws_gather_body(const SolverArgs& a, const int lp, const int by, int64_t* g) {
  const PairDesc pd = a.pairs[lp];
  const int wn = __ldcg(a.ws_n + lp);
  // rows of the CTA: kGR / 2 from the top of the triangle and their mirrors from the bottom
  // (row r has wn - r entries c >= r, so each pair of rows has wn + 1: every CTA the same work)
  constexpr int kH = kGR / 2;
  const int half = (wn + 1) / 2;
  const int t0 = by * kH;
  if (t0 >= half) return;
  const int32_t* ws = a.ws + (int64_t)lp * a.B;
  for (int e = threadIdx.x; e < wn; e += blockDim.x) g[e] = gpos(pd, __ldcg(ws + e));
  __syncthreads();
  const int ld = ws_tile_ld(a.B);
  float* tile = a.Kws + (int64_t)lp * ws_buf_floats(a.B);
  auto row_of = [&](int k) -> int {  // CTA row k in [0, kGR): -1 if none
    const int tt = t0 + (k < kH ? k : k - kH);
    if (tt >= half) return -1;
    if (k < kH) return tt;
    const int rb = wn - 1 - tt;
    return rb > tt ? rb : -1;  // the middle row of an odd wn belongs to the top half only
  };
  // K is stored symmetric (both triangles, the same values): the tile's upper triangle is loaded
  // and written to both positions -- half the scattered loads (each one a DRAM burst of its own)
  constexpr int M = (kGR * kWMaxB + 255) / 256;  // loads per thread, all in flight
  float v[M];
#pragma unroll
  for (int m = 0; m < M; ++m) {
    const int q = threadIdx.x + m * 256;
    const int k = q / wn, c = q % wn;
    const int r = k < kGR ? row_of(k) : -1;
    v[m] = (r >= 0 && c >= r) ? __ldg(a.K + g[r] * a.ldk + g[c]) : 0.f;
  }
#pragma unroll
  for (int m = 0; m < M; ++m) {
    const int q = threadIdx.x + m * 256;
    const int k = q / wn, c = q % wn;
    const int r = k < kGR ? row_of(k) : -1;
    if (r >= 0 && c >= r) {
      tile[(int64_t)r * ld + c] = v[m];
      tile[(int64_t)c * ld + r] = v[m];
    }
  }
}

__global__ void __launch_bounds__(256) ws_gather_kernel(SolverArgs a) {
  const int lp = blockIdx.x + a.pair_base;
  const PairDesc pd = a.pairs[lp];  // constant for the solve: loaded before the dependency wait
  pdl_enter();
  TraceScope ts_(a, lp, 1);
  if (a.status[lp] != 0) return;
  const int np = pd.n_s + pd.n_t;
  if (np <= a.B && a.outer_iters[lp] != 1) return;  // working set (and tile) unchanged
  __shared__ int64_t g[kWMaxB];
  ws_gather_body(a, lp, blockIdx.y, g);
}

// ------------------------------------------------------------------------------------------
// a5: single-warp local SMO

__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

size_t ws_smo_smem(int B) { return ws_buf_floats(B) * 4 + (size_t)B * 8 + 256; }

__device__ __forceinline__ float lds_f32(uint32_t addr) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr));
  return v;
}
__device__ __forceinline__ double lds_f64(uint32_t addr) {
  double v;
  asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(addr));
  return v;
}
__device__ __forceinline__ void sts_f64(uint32_t addr, double v) {
  asm volatile("st.shared.f64 [%0], %1;" ::"r"(addr), "d"(v) : "memory");
}

// in-place pairwise (tree) reductions over a lane's rows; the lower row wins ties
template <int E>
__device__ __forceinline__ void tree_min_u64(uint64_t (&k)[E], int (&q)[E]) {
#pragma unroll
  for (int w = 1; w < E; w <<= 1)
#pragma unroll
    for (int i = 0; i + w < E; i += 2 * w)
      if (k[i + w] < k[i]) {
        k[i] = k[i + w];
        q[i] = q[i + w];
      }
}
template <int E>
__device__ __forceinline__ void tree_max_u32(uint32_t (&k)[E], int (&q)[E]) {
#pragma unroll
  for (int w = 1; w < E; w <<= 1)
#pragma unroll
    for (int i = 0; i + w < E; i += 2 * w)
      if (k[i + w] > k[i]) {
        k[i] = k[i + w];
        q[i] = q[i + w];
      }
}
template <int E>
__device__ __forceinline__ void tree_min_f64(double (&k)[E], int (&q)[E]) {
#pragma unroll
  for (int w = 1; w < E; w <<= 1)
#pragma unroll
    for (int i = 0; i + w < E; i += 2 * w)
      if (k[i + w] < k[i]) {
        k[i] = k[i + w];
        q[i] = q[i + w];
      }
}
template <int E>
__device__ __forceinline__ void tree_max_f64(double (&k)[E]) {
#pragma unroll
  for (int w = 1; w < E; w <<= 1)
#pragma unroll
    for (int i = 0; i + w < E; i += 2 * w) k[i] = k[i + w] > k[i] ? k[i + w] : k[i];
}
template <int E>
__device__ __forceinline__ void tree_min_f32(float (&k)[E], int (&q)[E]) {
#pragma unroll
  for (int w = 1; w < E; w <<= 1)
#pragma unroll
    for (int i = 0; i + w < E; i += 2 * w)
      if (k[i + w] < k[i]) {
        k[i] = k[i + w];
        q[i] = q[i + w];
      }
}
template <int E>
__device__ __forceinline__ void tree_max_f32(float (&k)[E]) {
#pragma unroll
  for (int w = 1; w < E; w <<= 1)
#pragma unroll
    for (int i = 0; i + w < E; i += 2 * w) k[i] = k[i + w] > k[i] ? k[i + w] : k[i];
}
__device__ __forceinline__ uint32_t ord_key_f32(float x) {  // order-preserving bits of a finite float
  const uint32_t u = __float_as_uint(x);
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ __forceinline__ float key_f32(uint32_t k) {
  return __uint_as_float((k & 0x80000000u) ? (k & 0x7fffffffu) : ~k);
}
template <int E>
__device__ __forceinline__ void tree_max_u64(uint64_t (&k)[E]) {
#pragma unroll
  for (int w = 1; w < E; w <<= 1)
#pragma unroll
    for (int i = 0; i + w < E; i += 2 * w) k[i] = k[i + w] > k[i] ? k[i + w] : k[i];
}

// The local solve of pair lp by one warp (threadIdx.x < 32); mdyn: ws_smo_smem(B) bytes.
// FT: the working set's f in the local solve -- float (a.smo_f32: the Gaussian kernel, default) or
// double.  In FP32 the lane minima / maxima are 32-bit keys (u: two reductions instead of three,
// f_max: one instead of two) and the f update of the working set is an FFMA; the step s was FP32
// already (reading R29), and the global f, alpha and the clipping stay FP64, so the local solve
// is the same heuristic subproblem solver with a rounding of f that the next outer iteration's
// exact f replaces.  The dot-product kernels keep FP64 (the sigmoid kernel is not positive
// semi-definite: its QP has several solutions and the iterate path decides which one is reached).
// GMPSVM_SMO_F32=0 forces FP64 everywhere.
template <int E, bool PROF, typename FT = double>  // PROF: GMPSVM_SMO_PHASES per-phase cycle counters
__device__ __forceinline__ void ws_smo_body(const SolverArgs& a, const int lp, unsigned char* mdyn, const bool pdl) {
  constexpr bool F32 = sizeof(FT) == 4;
  const PairDesc pd = a.pairs[lp];  // constant for the solve: loaded before the dependency wait
  if (pdl) pdl_wait();  // the f-update is released when the local solve ends (below)
  TraceScope ts_(a, lp, 2);
  if (a.status[lp] != 0) return;
  const int lane = threadIdx.x;
  const int B = a.B, wn = a.ws_n[lp], ld = ws_tile_ld(B);
  uint32_t kws;  // K_ws,ws tile, row stride ld (opaque: keeps the shared window base out of the loop)
  asm volatile("mov.u32 %0, %1;" : "=r"(kws) : "r"(smem_addr(mdyn)));
  const uint32_t als = kws + (uint32_t)ws_state_off(B) * 4;     // alpha of the working set (state)
  const uint32_t fst = als + (uint32_t)B * 8;                     // f (state)
  const uint32_t ixs = fst + (uint32_t)B * 8;                     // index (state)
  const uint32_t a0s = ixs + (uint32_t)((B + 3) & ~3) * 4;        // alpha at entry
  const uint32_t bar = a0s + (uint32_t)B * 8;                     // mbarrier of the bulk copies
  const long long t_entry = clock64();
  // bulk copies: tile rows [0, wn) and the state block (alpha, f, index) written by the selection
  const uint32_t tbytes = (uint32_t)wn * ld * 4;  // ld % 4 == 0: multiples of 16
  const uint32_t sbytes = (uint32_t)B * 16 + (uint32_t)((B + 3) & ~3) * 4;
  if (lane == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(tbytes + sbytes) : "memory");
    const char* src = reinterpret_cast<const char*>(a.Kws + (int64_t)lp * ws_buf_floats(B));
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(als),
                 "l"(src + ws_state_off(B) * 4), "r"(sbytes), "r"(bar)
                 : "memory");
    constexpr uint32_t kChunk = 32768;
    for (uint32_t o = 0; o < tbytes; o += kChunk) {
      const uint32_t n = tbytes - o < kChunk ? tbytes - o : kChunk;
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       kws + o),
                   "l"(src + o), "r"(n), "r"(bar)
                   : "memory");
    }
  }
  const double C = a.C, eps = a.eps, ratio = a.local_ratio;
  {
    uint32_t done = 0;
    do {
      asm volatile(
          "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n selp.u32 %0, 1, 0, p;\n}\n"
          : "=r"(done)
          : "r"(bar)
          : "memory");
    } while (!done);
  }
  const long long t_state = clock64();
  // per-row state: lane owns positions lane + 32 q (the working set sorted by index)
  int32_t idx[E];
  FT f[E];
  uint32_t umask = 0u, lmask = 0u, ypos = 0u, vmask = 0u;
#pragma unroll
  for (int q = 0; q < E; ++q) {
    const int e = lane + 32 * q;
    const bool valid = e < wn;
    int32_t ix = INT_MAX;
    if (valid) asm volatile("ld.shared.s32 %0, [%1];" : "=r"(ix) : "r"(ixs + e * 4));
    idx[q] = ix;
    const int y = (valid && ix < pd.n_s) ? 1 : -1;
    const double al = valid ? lds_f64(als + e * 8) : 0.0;
    f[q] = valid ? (FT)lds_f64(fst + e * 8) : (FT)0;
    if (valid) {
      sts_f64(a0s + e * 8, al);
      vmask |= 1u << q;
      if (y > 0) ypos |= 1u << q;
      if (in_u(y, al, C)) umask |= 1u << q;
      if (in_l(y, al, C)) lmask |= 1u << q;
    }
  }
  float kd[E];
#pragma unroll
  for (int q = 0; q < E; ++q) {
    const int e = lane + 32 * q;
    kd[q] = e < wn ? lds_f32(kws + (uint32_t)(e * ld + e) * 4) : 1.f;
  }
  __syncwarp();
  const int cap = a.inner_cap;
  int it = 0;
  double delta0 = 0.0;
  const long long t_begin = clock64();
  constexpr bool prof = PROF;  // GMPSVM_SMO_PHASES: per-phase SM cycles (a.smo_phase != NULL)
  long long ph[4] = {0, 0, 0, 0}, tp = t_begin;
  auto markp = [&](int k) {
    if (prof) {
      const long long tc = clock64();
      ph[k] += tc - tp;
      tp = tc;
    }
  };
  for (;;) {
    // Eq 4: u = argmin_{I_u} f; ties -> lowest position (== lowest pair-local index, R5)
    // the lane's minimum in FP64 compares (ties: lower row), one ord_key for the warp reduction
    FT uv[E];
    int uq[E];
#pragma unroll
    for (int q = 0; q < E; ++q) {
      uv[q] = ((umask >> q) & 1u) ? f[q] : (FT)CUDART_INF;
      uq[q] = q;
    }
    uint32_t ue32;
    FT fu;
    if constexpr (F32) {
      tree_min_f32<E>(uv, uq);
      const bool uempty = uv[0] == CUDART_INF_F;
      const uint32_t k32 = uempty ? 0xffffffffu : ord_key_f32(uv[0]);
      const uint32_t pos = uempty ? 0xffffffffu : (uint32_t)(lane + 32 * uq[0]);
      const uint32_t m0 = __reduce_min_sync(FULLMASK, k32);
      ue32 = __reduce_min_sync(FULLMASK, k32 == m0 ? pos : 0xffffffffu);
      fu = key_f32(m0);
    } else {
      tree_min_f64<E>(uv, uq);
      const bool uempty = uv[0] == CUDART_INF;  // f is finite: +inf marks "no I_u row in this lane"
      const uint64_t uk0 = uempty ? ~0ull : ord_key(uv[0]);
      const uint32_t h = (uint32_t)(uk0 >> 32), l = (uint32_t)uk0;
      const uint32_t pos = uempty ? 0xffffffffu : (uint32_t)(lane + 32 * uq[0]);
      const uint32_t m0 = __reduce_min_sync(FULLMASK, h);
      const uint32_t m1 = __reduce_min_sync(FULLMASK, h == m0 ? l : 0xffffffffu);
      ue32 = __reduce_min_sync(FULLMASK, (h == m0 && l == m1) ? pos : 0xffffffffu);
      fu = (FT)key_double(((uint64_t)m0 << 32) | m1);
    }
    if (ue32 == 0xffffffffu) break;  // I_u empty
    const int ue = (int)ue32;
    const int uq0 = ue >> 5, ul = ue & 31;
    const int yu = ((__shfl_sync(FULLMASK, ypos, ul) >> uq0) & 1u) ? 1 : -1;
    const uint32_t urow = kws + (uint32_t)(ue * ld) * 4;
    const double au = lds_f64(als + ue * 8);
    const float kuu = lds_f32(urow + ue * 4);
    float ku[E];
#pragma unroll
    for (int q = 0; q < E; ++q) ku[q] = lds_f32(urow + (lane + 32 * q) * 4);
    markp(0);
    // Eq 5: l = argmax_{t in I_l, f_t > f_u} (f_t - f_u)^2 / eta_t (FP32, reading R29); the
    // winner's (f_t - f_u) / eta_t is the unclipped step; Eq 10: f_max over I_l
    uint32_t sb[E];
    int sq[E];
    float st[E];
    FT lv[E];
#pragma unroll
    for (int q = 0; q < E; ++q) {
      const bool il = (lmask >> q) & 1u;
      const float eta = fmaxf(fmaf(-2.f, ku[q], kuu + kd[q]), 1e-12f);
      const float df = (float)(f[q] - fu);
      float r;
      asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(eta));
      st[q] = df * r;
      sb[q] = (il && f[q] > fu) ? __float_as_uint(df * st[q]) : 0u;  // scores >= 0: bits order as values
      sq[q] = q;
      lv[q] = il ? f[q] : (FT)-CUDART_INF;
    }
    tree_max_u32<E>(sb, sq);
    double fmax;
    uint32_t smax, le32;
    if constexpr (F32) {
      tree_max_f32<E>(lv);
      const uint32_t lk = lv[0] == -CUDART_INF_F ? 0u : ord_key_f32(lv[0]);  // 0: no I_l row in this lane
      const uint32_t xm = __reduce_max_sync(FULLMASK, lk);
      smax = __reduce_max_sync(FULLMASK, sb[0]);
      const uint32_t lpos = (sb[0] != 0u && sb[0] == smax) ? (uint32_t)(lane + 32 * sq[0]) : 0xffffffffu;
      le32 = __reduce_min_sync(FULLMASK, lpos);
      fmax = xm == 0u ? -DBL_MAX : (double)key_f32(xm);
    } else {
      tree_max_f64<E>(lv);
      const uint64_t lk0 = lv[0] == -CUDART_INF ? 0ull : ord_key(lv[0]);  // 0: no I_l row in this lane
      const uint32_t xh = __reduce_max_sync(FULLMASK, (uint32_t)(lk0 >> 32));
      const uint32_t xl = __reduce_max_sync(FULLMASK, (uint32_t)(lk0 >> 32) == xh ? (uint32_t)lk0 : 0u);
      smax = __reduce_max_sync(FULLMASK, sb[0]);
      const uint32_t lpos = (sb[0] != 0u && sb[0] == smax) ? (uint32_t)(lane + 32 * sq[0]) : 0xffffffffu;
      le32 = __reduce_min_sync(FULLMASK, lpos);
      fmax = (xh == 0u && xl == 0u) ? -DBL_MAX : key_double(((uint64_t)xh << 32) | xl);
    }
    markp(1);
    const double gap = fmax - (double)fu;
    if (it == 0) delta0 = gap;
    const double tol = eps > ratio * delta0 ? eps : ratio * delta0;
    if (!(gap >= tol) || le32 == 0xffffffffu || it >= cap) break;
    const int le = (int)le32;
    const int ll = le & 31, lq = le >> 5;
    float stl = st[0];
#pragma unroll
    for (int q = 1; q < E; ++q)
      if (q == lq) stl = st[q];
    double s = (double)__shfl_sync(FULLMASK, stl, ll);
    const int yl = ((__shfl_sync(FULLMASK, ypos, ll) >> lq) & 1u) ? 1 : -1;
    const uint32_t lrow = kws + (uint32_t)(le * ld) * 4;
    const double alv = lds_f64(als + le * 8);
    float kl[E];
#pragma unroll
    for (int q = 0; q < E; ++q) kl[q] = lds_f32(lrow + (lane + 32 * q) * 4);
    markp(2);
    // Eq 6-7 with explicit clipping (reading R4): common step s, bounds assigned exactly
    const double Uu = yu > 0 ? C - au : au;
    const double Ll = yl > 0 ? alv : C - alv;
    bool bnu = false, bnl = false;
    if (Uu <= s) {
      s = Uu;
      bnu = true;
    }
    if (Ll <= s) {
      if (Ll < s) bnu = false;
      s = Ll;
      bnl = true;
    }
    const double nau = bnu ? (yu > 0 ? C : 0.0) : au + yu * s;
    const double nal = bnl ? (yl > 0 ? 0.0 : C) : alv - yl * s;
    // Eq 8 on the working set: f_i += s (K_ui - K_li)
#pragma unroll
    for (int q = 0; q < E; ++q) {
      if constexpr (F32) f[q] = fmaf((float)s, ku[q] - kl[q], f[q]);
      else f[q] = fma(s, (double)(ku[q] - kl[q]), f[q]);
    }
    // membership of u and l after the step (owners update their bits; alpha in shared memory)
    const uint32_t uin = in_u(yu, nau, C) ? 1u : 0u, uil = in_l(yu, nau, C) ? 1u : 0u;
    const uint32_t lin = in_u(yl, nal, C) ? 1u : 0u, lil = in_l(yl, nal, C) ? 1u : 0u;
    if (lane == ul) {
      umask = (umask & ~(1u << uq0)) | (uin << uq0);
      lmask = (lmask & ~(1u << uq0)) | (uil << uq0);
    }
    if (lane == ll) {
      umask = (umask & ~(1u << lq)) | (lin << lq);
      lmask = (lmask & ~(1u << lq)) | (lil << lq);
    }
    if (lane == 0) {
      sts_f64(als + ue * 8, nau);
      sts_f64(als + le * 8, nal);
    }
    __syncwarp();
    ++it;
    if (prof && f[0] == -1.2345e300) ph[3] += 1;  // keep the f update ahead of the clock read
    markp(3);
  }
  __syncwarp();
  if (pdl) pdl_trigger();
#pragma unroll
  for (int q = 0; q < E; ++q) {
    const int e = lane + 32 * q;
    if ((vmask >> q) & 1u) {
      const double al = lds_f64(als + e * 8);
      const double a0 = lds_f64(a0s + e * 8);
      const int y = ((ypos >> q) & 1u) ? 1 : -1;
      a.dcoef[(int64_t)lp * B + e] = (al - a0) * (double)y;
      a.alpha[pd.a_off + idx[q]] = al;
      if (a.ulf) a.ulf[pd.a_off + idx[q]] = (uint8_t)((in_u(y, al, C) ? 1 : 0) | (in_l(y, al, C) ? 2 : 0));
    }
  }
  if (lane == 0) {
    a.inner_iters[lp] += it;
    a.smo_cycles[lp] += clock64() - t_begin;
    if (prof) {
      for (int k = 0; k < 4; ++k) a.smo_phase[lp * 5 + k] += ph[k];
      a.smo_phase[lp * 5 + 4] += t_begin - t_entry;
      a.sel_phase[lp * 5 + 2] += t_state - t_entry;  // prologue split: state loads | tile wait
      a.sel_phase[lp * 5 + 3] += t_begin - t_state;
    }
  }
}

template <int E, bool PROF, typename FT = double>
__global__ void __launch_bounds__(32, 1) ws_smo_kernel(SolverArgs a) {
  extern __shared__ __align__(16) unsigned char mdyn[];
  ws_smo_body<E, PROF, FT>(a, blockIdx.x + a.pair_base, mdyn, true);
}

// ------------------------------------------------------------------------------------------
// a6: f update, f_j += sum_{i in ws, dalpha_i != 0} dalpha_i y_i K_ij over the pair (Alg 2 line 11,
// Eq 8).  HBM-bound GEMV over the kernel-matrix rows of the working set: a CTA owns 32 column
// quads (128 columns) of the pair's two class segments, its 8 warps split the rows (8 float4
// loads in flight per thread), FP64 accumulation, partial sums combined in a fixed order.  With
// set_cond, block (0,0) sets the graph loop condition: continue while a pair of the launch is
// active (the selection of this iteration has set the status).
constexpr int kFW = 8;         // warps per f-update CTA
constexpr int kFT = kFW * 32;  // threads

struct WFup {
  double coef[kWMaxB];
  const float4* rowp[kWMaxB];
  double red[kFW][32][4];
  int scan[33];
};

// columns [by * 128, +128) of pair lp's f-update by one kFT-thread CTA.  The working set, its
// coefficients and f are read through L2 (the persistent solver's workers run beside the CTA that
// wrote them); f of a column is updated by exactly one CTA.
__device__ __forceinline__ void ws_fupdate_body(const SolverArgs& a, const int lp, const int by, WFup& F) {
  const PairDesc pd = a.pairs[lp];
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  const int64_t q1b = pd.off_s >> 2, q1e = (pd.off_s + pd.n_s + 3) >> 2;
  const int64_t q2b = pd.off_t >> 2, q2e = (pd.off_t + pd.n_t + 3) >> 2;
  const int64_t nq1 = q1e - q1b, nq = nq1 + (q2e - q2b);
  const int64_t q0 = (int64_t)by * 32;
  if (q0 >= nq) return;
  const int B = a.B, wn = __ldcg(a.ws_n + lp);
  const int32_t* ws = a.ws + (int64_t)lp * B;
  const double* dc = a.dcoef + (int64_t)lp * B;
  int nnz = 0;
  {
    const double c = t < wn ? __ldcg(dc + t) : 0.0;
    const bool nz = c != 0.0;
    int tot = 0;
    const int pos = block_excl_scan(nz, tot, F.scan);
    if (nz) {
      F.coef[pos] = c;
      F.rowp[pos] = reinterpret_cast<const float4*>(a.K + gpos(pd, __ldcg(ws + t)) * a.ldk);
    }
    nnz = tot;
  }
  __syncthreads();
  if (nnz == 0) return;
  const int64_t qi = q0 + lane;
  const bool okq = qi < nq;
  const int64_t gq = !okq ? 0 : (qi < nq1 ? q1b + qi : q2b + (qi - nq1));
  double acc[4] = {0.0, 0.0, 0.0, 0.0};
  int r = warp;
  for (; r + 7 * kFW < nnz; r += 8 * kFW) {
    float4 v[8];
#pragma unroll
    for (int rr = 0; rr < 8; ++rr) v[rr] = okq ? __ldg(F.rowp[r + rr * kFW] + gq) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int rr = 0; rr < 8; ++rr) {
      const double cv = F.coef[r + rr * kFW];
      acc[0] = fma(cv, (double)v[rr].x, acc[0]);
      acc[1] = fma(cv, (double)v[rr].y, acc[1]);
      acc[2] = fma(cv, (double)v[rr].z, acc[2]);
      acc[3] = fma(cv, (double)v[rr].w, acc[3]);
    }
  }
  for (; r < nnz; r += kFW) {
    const float4 v0 = okq ? __ldg(F.rowp[r] + gq) : make_float4(0.f, 0.f, 0.f, 0.f);
    const double cv = F.coef[r];
    acc[0] = fma(cv, (double)v0.x, acc[0]);
    acc[1] = fma(cv, (double)v0.y, acc[1]);
    acc[2] = fma(cv, (double)v0.z, acc[2]);
    acc[3] = fma(cv, (double)v0.w, acc[3]);
  }
#pragma unroll
  for (int c = 0; c < 4; ++c) F.red[warp][lane][c] = acc[c];
  __syncthreads();
  if (t < 128) {  // column: component t & 3 of quad t >> 2
    const int l = t >> 2, c = t & 3;
    const int64_t qj = q0 + l;
    if (qj < nq) {
      const bool seg1 = qj < nq1;  // a boundary quad shared by adjacent classes is owned once per segment
      const int64_t g = (seg1 ? q1b + qj : q2b + (qj - nq1)) * 4 + c;
      int64_t j = -1;
      if (seg1) j = (g >= pd.off_s && g < pd.off_s + pd.n_s) ? g - pd.off_s : -1;
      else j = (g >= pd.off_t && g < pd.off_t + pd.n_t) ? pd.n_s + (g - pd.off_t) : -1;
      if (j >= 0) {
        double sum = 0.0;
#pragma unroll
        for (int w = 0; w < kFW; ++w) sum += F.red[w][l][c];
        double* fp = a.f + pd.a_off + j;
        __stcg(fp, __ldcg(fp) + sum);
      }
    }
  }
}

__global__ void __launch_bounds__(kFT) ws_fupdate_kernel(SolverArgs a, cudaGraphConditionalHandle h, int set_cond) {
  const int lp = blockIdx.x + a.pair_base;
  pdl_enter();
  TraceScope ts_(a, lp, 3);
  const int t = threadIdx.x;
  if (blockIdx.x == 0 && blockIdx.y == 0 && t == 0) {
    bool more = false;
    for (int i = 0; i < (int)gridDim.x; ++i) more = more || a.status[a.pair_base + i] == 0;
    if (set_cond) {
      cudaGraphSetConditional(h, more ? 1u : 0u);
      a.body_iters[a.pair_base] += 1;
    }
  }
  if (a.status[lp] != 0) return;
  __shared__ WFup F;
  for (int ch = 0; ch < a.fu_chunks; ++ch) {  // GMPSVM_FU_CHUNKS (measured: 1 best)
    if (ch > 0) __syncthreads();
    ws_fupdate_body(a, lp, blockIdx.y * a.fu_chunks + ch, F);
  }
  if (a.trace && lp == a.trace_pair && t == 0) {  // GMPSVM_TRACE: latest CTA exit of the f-update
    __threadfence();
    atomicMax(trace_fu_end(a), (unsigned long long)gtimer());
  }
}

// ------------------------------------------------------------------------------------------
// Persistent solver: the outer loops of a group of pairs in two concurrent launches (Alg 2 lines
// 6-11, the same four steps).  ws_lead_kernel: one CTA per pair runs the selection (whole CTA) and
// the local SMO (warp 0) in its shared memory.  ws_work_kernel: small CTAs that take the gather
// rows and f-update columns of every leader's iterations from a device task queue -- each task is
// exactly one ws_gather_kernel / ws_fupdate_kernel CTA (same bodies, same summation order), so both
// paths give bitwise the same alpha.  A leader publishes a phase's tasks and waits on its pair's
// completion counter: each handoff is an L2 flag round trip instead of a kernel-grid completion
// (~5 us each, four per outer iteration, measured with GMPSVM_TRACE fu_end_to_select).
//
// Residency: the worker grid is a programmatic dependent of the leader grid and every leader CTA
// triggers it first thing, so the workers launch only once every leader is resident (one per SM
// by its shared memory) and fill the SMs around them.  Every wait is bounded (kPTimeoutNs): a
// stuck solve sets ctr[3] and the call fails with GMPSVM_ECUDA instead of hanging the GPU.
struct PTask {  // one queue entry
  int32_t kind, lp, chunk, pad;
  unsigned long long seq;  // slot index + 1 once the entry is published
  unsigned long long pad2;
};
enum { kTaskExit = 0, kTaskGather = 1, kTaskFup = 2 };
constexpr int kPQueueCap = 1 << 15;
constexpr unsigned long long kPTimeoutNs = 20000000000ull;  // 20 s per wait
// ctr words: [0] head (next slot a worker takes), [1] tail (next slot a leader fills),
// [2] leaders finished, [3] error, [8 + i] tasks completed for leader i
constexpr int kPCtrPairs = 8;

__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.global;" ::: "memory"); }

// thread 0 of a leader: n tasks of one kind for leader slot li
__device__ void p_push(PTask* ring, unsigned long long* ctr, int kind, int li, int n) {
  const unsigned long long base = atomicAdd(&ctr[1], (unsigned long long)n);
  for (int i = 0; i < n; ++i) {
    PTask* e = ring + ((base + i) & (kPQueueCap - 1));
    e->kind = kind;
    e->lp = li;
    e->chunk = i;
    st_release_u64(&e->seq, base + i + 1);  // orders the fields before the sequence number
  }
}

// whole leader CTA: publish n tasks, wait until the workers completed them (target: running count)
__device__ bool p_run(const SolverArgs& a, int lp, PTask* ring, unsigned long long* ctr, int kind, int li, int n,
                      unsigned long long& target, int* s_ok) {
  __syncthreads();  // the CTA's global writes (selection output, local-solve result) precede the publish
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned long long t0 = gtimer();
    target += (unsigned long long)n;
    p_push(ring, ctr, kind, li, n);
    int ok = 1;
    while (ld_acquire_u64(&ctr[kPCtrPairs + li]) < target) {
      if (gtimer() - t0 > kPTimeoutNs || ld_acquire_u64(&ctr[3]) != 0) {
        atomicExch(&ctr[3], 1ull);
        ok = 0;
        break;
      }
    }
    __threadfence();
    fence_proxy_async();  // the workers' tile rows are read by the local solve's bulk copy
    *s_ok = ok;
    if (a.trace && lp == a.trace_pair)  // GMPSVM_TRACE: the phase from publish to completion
      trace_rec(a, kind == kTaskGather ? 1 : 3, (int64_t)t0, (int64_t)gtimer());
  }
  __syncthreads();
  return *s_ok != 0;
}

__host__ __device__ inline size_t ws_lead_w_off(int B) {
  const size_t sel = (size_t)kWMaxNp * 9, smo = ws_buf_floats(B) * 4 + (size_t)B * 8 + 256;
  return ((sel > smo ? sel : smo) + 127) & ~(size_t)127;
}

template <int E>
__global__ void __launch_bounds__(kWT, 1)
    ws_lead_kernel(SolverArgs a, int P, int nworkers, int64_t max_outer, PTask* ring, unsigned long long* ctr,
                   const unsigned long long* res_ctr, int wait_resident) {
  if (wait_resident > 0 && threadIdx.x == 0) {  // the kernel-value launch beside us holds its SMs first
    const unsigned long long t0 = gtimer();
    while (ld_acquire_u64(res_ctr) < (unsigned long long)wait_resident && gtimer() - t0 < kPTimeoutNs) __nanosleep(256);
  }
  __syncthreads();
  pdl_trigger();  // the worker grid launches once every leader is resident
  extern __shared__ __align__(128) unsigned char pdyn[];
  WSelSmall& W = *reinterpret_cast<WSelSmall*>(pdyn + ws_lead_w_off(a.B));
  __shared__ int s_ok;
  const int t = threadIdx.x;
  const int li = blockIdx.x, lp = a.pair_base + li;
  const PairDesc pd = a.pairs[lp];
  const int np = pd.n_s + pd.n_t;
  const int64_t nq = ((pd.off_s + pd.n_s + 3) >> 2) - (pd.off_s >> 2) + ((pd.off_t + pd.n_t + 3) >> 2) - (pd.off_t >> 2);
  const int n_fup = (int)((nq + 31) / 32);  // ws_fupdate_kernel CTAs with columns
  unsigned long long target = 0;
  for (;;) {
    ws_select_body(a, lp, max_outer, pdyn, W, false);
    fence_proxy_async();  // the working set's state is read by the local solve's bulk copy
    __syncthreads();
    if (a.status[lp] != 0) break;
    if (!(np <= a.B && a.outer_iters[lp] != 1)) {  // the tile changed (ws_gather_kernel's test)
      const int n_g = (a.ws_n[lp] + kGR - 1) / kGR;
      if (!p_run(a, lp, ring, ctr, kTaskGather, li, n_g, target, &s_ok)) break;
    }
    if (t < 32) {
      if (a.smo_f32) ws_smo_body<E, false, float>(a, lp, pdyn, false);
      else ws_smo_body<E, false>(a, lp, pdyn, false);
    }
    if (!p_run(a, lp, ring, ctr, kTaskFup, li, n_fup, target, &s_ok)) break;
  }
  if (t == 0) {
    __threadfence();
    if (atomicAdd(&ctr[2], 1ull) == (unsigned long long)(P - 1)) p_push(ring, ctr, kTaskExit, 0, nworkers);
  }
}

union PWork {  // worker shared memory
  WFup F;
  int64_t g[kWMaxB];
};

__global__ void __launch_bounds__(kFT) ws_work_kernel(SolverArgs a, PTask* ring, unsigned long long* ctr) {
  __shared__ PWork w;
  __shared__ int task[3];
  const int t = threadIdx.x;
  for (;;) {
    if (t == 0) {
      const unsigned long long idx = atomicAdd(&ctr[0], 1ull);
      PTask* e = ring + (idx & (kPQueueCap - 1));
      const unsigned long long t0 = gtimer();
      int kind = kTaskExit, li = 0, ch = 0;
      for (;;) {
        if (ld_acquire_u64(&e->seq) == idx + 1) {
          kind = e->kind;
          li = e->lp;
          ch = e->chunk;
          break;
        }
        if (gtimer() - t0 > kPTimeoutNs) {
          atomicExch(&ctr[3], 1ull);
          break;
        }
        __nanosleep(32);
      }
      task[0] = kind;
      task[1] = li;
      task[2] = ch;
    }
    __syncthreads();
    const int kind = task[0], li = task[1], ch = task[2];
    if (kind == kTaskExit) return;
    const bool tr = a.trace && a.pair_base + li == a.trace_pair && t == 0;
    const int64_t tt0 = tr ? (int64_t)gtimer() : 0;
    if (kind == kTaskGather) {
      ws_gather_body(a, a.pair_base + li, ch, w.g);
      fence_proxy_async();  // read by the leader's bulk copy (async proxy)
    } else {
      ws_fupdate_body(a, a.pair_base + li, ch, w.F);
    }
    __syncthreads();
    if (t == 0) {
      __threadfence();
      atomicAdd(&ctr[kPCtrPairs + li], 1ull);
    }
    if (tr) trace_rec(a, kind == kTaskGather ? 9 : 10, tt0, (int64_t)gtimer());  // GMPSVM_TRACE: one task
  }
}

size_t ws_persist_smem(int B) { return ws_lead_w_off(B) + sizeof(WSelSmall); }
size_t ws_persist_ctr_words(int P) { return (size_t)kPCtrPairs + P; }
size_t ws_persist_ring_bytes() { return sizeof(PTask) * kPQueueCap; }

bool ws_persist_supported(int B, int64_t np_max) {
  // opt-in (GMPSVM_PERSIST=1: every group; =lead: the lead group only, the others on the graphs):
  // measured slower on MNIST-shaped data
  static const char* e = getenv("GMPSVM_PERSIST");
  static const bool off = !(e && (std::string(e) == "1" || std::string(e) == "lead"));
  int dev = 0, optin = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  return !off && ws_solve_supported(B, np_max) && ws_persist_smem(B) <= (size_t)optin;
}

int ws_persist_workers_per_sm() {
  int nb = 0;
  GM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, ws_work_kernel, kFT, 0));
  return nb;
}

template <int E>
static void launch_lead(const SolverArgs& a, int P, int nworkers, int64_t max_outer, PTask* ring,
                        unsigned long long* ctr, cudaStream_t st, const unsigned long long* res_ctr, int wait_resident) {
  const size_t smem = ws_persist_smem(a.B);
  set_max_dyn_smem(ws_lead_kernel<E>, smem);
  GM_LAUNCH(ws_lead_kernel<E>, dim3(P), dim3(kWT), smem, st, a, P, nworkers, max_outer, ring, ctr, res_ctr,
            wait_resident);
}

void launch_ws_persist(const SolverArgs& a, int P, int nworkers, int64_t max_outer, void* ring_v,
                       unsigned long long* ctr, cudaStream_t st, const unsigned long long* res_ctr, int wait_resident) {
  PTask* ring = static_cast<PTask*>(ring_v);
  switch ((a.B + 31) / 32) {
    case 1: launch_lead<1>(a, P, nworkers, max_outer, ring, ctr, st, res_ctr, wait_resident); break;
    case 2: launch_lead<2>(a, P, nworkers, max_outer, ring, ctr, st, res_ctr, wait_resident); break;
    case 3: launch_lead<3>(a, P, nworkers, max_outer, ring, ctr, st, res_ctr, wait_resident); break;
    case 4: launch_lead<4>(a, P, nworkers, max_outer, ring, ctr, st, res_ctr, wait_resident); break;
    case 5: launch_lead<5>(a, P, nworkers, max_outer, ring, ctr, st, res_ctr, wait_resident); break;
    case 6: launch_lead<6>(a, P, nworkers, max_outer, ring, ctr, st, res_ctr, wait_resident); break;
    default: launch_lead<7>(a, P, nworkers, max_outer, ring, ctr, st, res_ctr, wait_resident); break;
  }
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(nworkers);
  cfg.blockDim = dim3(kFT);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  GM_CUDA(cudaLaunchKernelEx(&cfg, ws_work_kernel, a, ring, ctr));
  g_launches.fetch_add(1, std::memory_order_relaxed);
}

// ------------------------------------------------------------------------------------------
bool ws_solve_supported(int B, int64_t np_max) {
  static const bool off = getenv("GMPSVM_WSOLVE") && std::string(getenv("GMPSVM_WSOLVE")) == "0";
  // GMPSVM_WS_MAXNP lowers the pair-size limit (tests: one graph mixing both solver paths)
  static const int64_t lim =
      getenv("GMPSVM_WS_MAXNP") ? std::min<int64_t>(kWMaxNp, atoll(getenv("GMPSVM_WS_MAXNP"))) : kWMaxNp;
  return !off && B >= 2 && B <= kWMaxB && np_max <= lim;
}

size_t ws_tile_floats(int B) { return ws_buf_floats(B); }



static bool pdl_enabled() {
  static const bool on = !(getenv("GMPSVM_PDL") && std::string(getenv("GMPSVM_PDL")) == "0");
  return on;
}

template <typename... KArgs, typename... Args>
static void launch_pdl(void (*kern)(KArgs...), dim3 g, dim3 b, size_t smem, cudaStream_t st, Args... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = g;
  cfg.blockDim = b;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  GM_CUDA(cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...));
  g_launches.fetch_add(1, std::memory_order_relaxed);
}

template <int E>
static void smo_configure(int smem) {
  set_max_dyn_smem(ws_smo_kernel<E, false>, smem);
  set_max_dyn_smem(ws_smo_kernel<E, true>, smem);
  set_max_dyn_smem(ws_smo_kernel<E, false, float>, smem);
  set_max_dyn_smem(ws_smo_kernel<E, true, float>, smem);
}
template <int E>
static void launch_smo(const SolverArgs& a, int P, size_t smem, cudaStream_t st) {
  if (a.smo_f32) {
    if (a.smo_phase) launch_pdl(ws_smo_kernel<E, true, float>, dim3(P), dim3(32), smem, st, a);
    else launch_pdl(ws_smo_kernel<E, false, float>, dim3(P), dim3(32), smem, st, a);
  } else {
    if (a.smo_phase) launch_pdl(ws_smo_kernel<E, true>, dim3(P), dim3(32), smem, st, a);
    else launch_pdl(ws_smo_kernel<E, false>, dim3(P), dim3(32), smem, st, a);
  }
}

static void ws_configure() {
  set_max_dyn_smem(ws_select_kernel, (size_t)kWMaxNp * 9);
  const int mx = (int)ws_smo_smem(kWMaxB);
  smo_configure<1>(mx);
  smo_configure<2>(mx);
  smo_configure<3>(mx);
  smo_configure<4>(mx);
  smo_configure<5>(mx);
  smo_configure<6>(mx);
  smo_configure<7>(mx);
}

// The single-warp local SMO alone (the sharded pair solver, shard.cu): each pair's K_ws,ws tile
// (row stride ws_tile_ld(B)) and state (alpha, f, index; sorted order) in the ws_write_out layout.
void launch_ws_smo(const SolverArgs& a, int P, cudaStream_t st) {
  ws_configure();
  const size_t smo_dyn = ws_smo_smem(a.B);
  switch ((a.B + 31) / 32) {
    case 1: launch_smo<1>(a, P, smo_dyn, st); break;
    case 2: launch_smo<2>(a, P, smo_dyn, st); break;
    case 3: launch_smo<3>(a, P, smo_dyn, st); break;
    case 4: launch_smo<4>(a, P, smo_dyn, st); break;
    case 5: launch_smo<5>(a, P, smo_dyn, st); break;
    case 6: launch_smo<6>(a, P, smo_dyn, st); break;
    default: launch_smo<7>(a, P, smo_dyn, st); break;
  }
}
int ws_smo_max_b() { return kWMaxB; }
int ws_tile_ld_of(int B) { return ws_tile_ld(B); }

void launch_ws_iteration(const SolverArgs& a, int P, int64_t np_max, cudaGraphConditionalHandle h, int set_cond,
                         int64_t max_outer, cudaStream_t st, bool chained) {
  ws_configure();
  const size_t sel_dyn = (size_t)kWMaxNp * 9, smo_dyn = ws_smo_smem(a.B);
  if (chained) launch_pdl(ws_select_kernel, dim3(P), dim3(kWT), sel_dyn, st, a, max_outer);
  else GM_LAUNCH(ws_select_kernel, dim3(P), dim3(kWT), sel_dyn, st, a, max_outer);
  launch_pdl(ws_gather_kernel, dim3(P, (unsigned)ceil_div(a.B, kGR)), dim3(256), 0, st, a);
  switch ((a.B + 31) / 32) {
    case 1: launch_smo<1>(a, P, smo_dyn, st); break;
    case 2: launch_smo<2>(a, P, smo_dyn, st); break;
    case 3: launch_smo<3>(a, P, smo_dyn, st); break;
    case 4: launch_smo<4>(a, P, smo_dyn, st); break;
    case 5: launch_smo<5>(a, P, smo_dyn, st); break;
    case 6: launch_smo<6>(a, P, smo_dyn, st); break;
    default: launch_smo<7>(a, P, smo_dyn, st); break;
  }
  launch_pdl(ws_fupdate_kernel, dim3(P, (unsigned)ceil_div(np_max + 8, 128 * a.fu_chunks)), dim3(kFT), 0, st, a, h,
             set_cond);
}

}  // namespace gmpsvm
