// solver_dev.cuh -- device helpers shared by the solver kernels (solver.cu, wsolve.cu):
// order-preserving keys, block reductions / scans, the optional kernel timeline, and the
// exact radix selection of working-set candidates (a4).
#pragma once

#include <cfloat>
#include <climits>

#include "kernels.h"

namespace gmpsvm {

#define FULLMASK 0xffffffffu

__device__ __forceinline__ uint64_t ord_key(double x) {
  const uint64_t u = (uint64_t)__double_as_longlong(x);
  return (u & 0x8000000000000000ull) ? ~u : (u | 0x8000000000000000ull);
}
__device__ __forceinline__ double key_double(uint64_t k) {
  const uint64_t u = (k & 0x8000000000000000ull) ? (k & 0x7fffffffffffffffull) : ~k;
  return __longlong_as_double((long long)u);
}
__device__ __forceinline__ bool in_u(int y, double a, double C) { return (y > 0 && a < C) || (y < 0 && a > 0.0); }
__device__ __forceinline__ bool in_l(int y, double a, double C) { return (y > 0 && a > 0.0) || (y < 0 && a < C); }
__device__ __forceinline__ int64_t gpos(const PairDesc& pd, int64_t j) {
  return j < pd.n_s ? pd.off_s + j : pd.off_t + (j - pd.n_s);
}

// ------------------------------------------------------------------------------------------
// block helpers (blockDim.x multiple of 32, <= 1024)
template <typename T, typename Op>
__device__ __forceinline__ T block_reduce(T v, Op op, T* sm /* >= 32 */) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = op(v, __shfl_xor_sync(FULLMASK, v, o));
  __syncthreads();
  if (lane == 0) sm[warp] = v;
  __syncthreads();
  T r = sm[0];
  for (int w = 1; w < nw; ++w) r = op(r, sm[w]);
  return r;
}

// exclusive prefix over the block of a flag (block order = thread order); returns rank
__device__ __forceinline__ int block_excl_scan(bool flag, int& total, int* sm /* 33 */) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const unsigned b = __ballot_sync(FULLMASK, flag);
  const int pre = __popc(b & ((1u << lane) - 1u));
  __syncthreads();
  if (lane == 0) sm[warp] = __popc(b);
  __syncthreads();
  if (warp == 0) {
    const int v = lane < nw ? sm[lane] : 0;
    int x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(FULLMASK, x, o);
      if (lane >= o) x += y;
    }
    if (lane < nw) sm[lane] = x - v;
    if (lane == 31) sm[32] = x;
  }
  __syncthreads();
  total = sm[32];
  return sm[warp] + pre;
}

// exclusive prefix over the warps of a per-warp count (all lanes pass the same value); returns
// this warp's offset and the block total
__device__ __forceinline__ int block_excl_scan_count(int count, int& total, int* sm /* 33 */) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  __syncthreads();
  if (lane == 0) sm[warp] = count;
  __syncthreads();
  if (warp == 0) {
    const int v = lane < nw ? sm[lane] : 0;
    int x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(FULLMASK, x, o);
      if (lane >= o) x += y;
    }
    if (lane < nw) sm[lane] = x - v;
    if (lane == 31) sm[32] = x;
  }
  __syncthreads();
  total = sm[32];
  return sm[warp];
}

// ------------------------------------------------------------------------------------------

// Optional timeline of one pair's solver kernels (GMPSVM_TRACE): thread (0,0,0) of the CTA that
// serves the traced pair records (kernel id, %globaltimer at entry, at exit).
__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// one extra record (kind, t0, t1) of the traced pair
__device__ __forceinline__ void trace_rec(const SolverArgs& a, int kid, int64_t t0, int64_t t1) {
  const int s = atomicAdd(a.trace_n, 1);
  if (s < a.trace_cap) {
    a.trace[3 * s] = kid;
    a.trace[3 * s + 1] = t0;
    a.trace[3 * s + 2] = t1;
  }
}
// latest exit of any f-update CTA of the traced pair (trace_n[2..3], 8-byte aligned)
__device__ __forceinline__ unsigned long long* trace_fu_end(const SolverArgs& a) {
  return reinterpret_cast<unsigned long long*>(a.trace_n + 2);
}
struct TraceScope {
  int64_t* buf;
  int32_t* n;
  int cap, kid;
  uint64_t t0;
  __device__ TraceScope(const SolverArgs& a, int lp, int k) : buf(nullptr), kid(k) {
    if (a.trace && threadIdx.x == 0 && blockIdx.y == 0 && blockIdx.z == 0 && a.status[lp] == 0) {
      // per-pair activity window: first entry, last entry (kernels of active pairs only)
      int64_t* w = a.trace + 3 * (int64_t)a.trace_cap + 2 * lp;
      const int64_t now = (int64_t)gtimer();
      if (w[0] == 0) w[0] = now;
      w[1] = now;
    }
    if (a.trace && lp == a.trace_pair && threadIdx.x == 0 && blockIdx.y == 0 && blockIdx.z == 0) {
      buf = a.trace;
      n = a.trace_n;
      cap = a.trace_cap;
      t0 = gtimer();
    }
  }
  __device__ ~TraceScope() {
    if (buf) {
      const int s = atomicAdd(n, 1);
      if (s < cap) {
        buf[3 * s] = kid;
        buf[3 * s + 1] = (int64_t)t0;
        buf[3 * s + 2] = (int64_t)gtimer();
      }
    }
  }
};

// ------------------------------------------------------------------------------------------
// a4: working-set selection
struct SelSmem {
  int32_t hist[256];
  int32_t scan[33];
  double red[32];
  double red4[132];
  int32_t sel_digit, sel_below, sel_count, take_all;
};

// Candidate sources: the global arrays (any n_p) or a shared-memory copy of the keys and
// I_u / I_l / taken flags (n_p <= kSelSmemMax), both with the same selection semantics.
struct GlobalSrc {
  const double* al;
  const double* fl;
  uint32_t* st;
  uint32_t stampv;
  int n_s;
  double C;
  template <bool SIDE_U>
  __device__ __forceinline__ bool cand(int i, uint64_t& key) const {
    const int y = i < n_s ? 1 : -1;
    const double a = al[i];
    const bool ok = SIDE_U ? in_u(y, a, C) : in_l(y, a, C);
    if (!ok || st[i] == stampv) return false;
    key = ord_key(fl[i]);
    if (!SIDE_U) key = ~key;  // ord_key(-f) == ~ord_key(f): largest f first
    return true;
  }
  __device__ __forceinline__ void take(int i) const { st[i] = stampv; }
};
struct SmemSrc {
  const uint64_t* keys;
  uint8_t* flags;  // bit0 in I_u, bit1 in I_l, bit2 taken / retained
  template <bool SIDE_U>
  __device__ __forceinline__ bool cand(int i, uint64_t& key) const {
    const uint8_t fl = flags[i];
    if (!(fl & (SIDE_U ? 1 : 2)) || (fl & 4)) return false;
    key = SIDE_U ? keys[i] : ~keys[i];
    return true;
  }
  __device__ __forceinline__ void take(int i) const { flags[i] |= 4; }
};

// Select the `want` smallest keys among the candidates of one side (ties: lowest index),
// append them to out[] in index order and mark them taken.  Radix select on 8-bit digits
// from the top; stops as soon as the threshold bucket holds exactly the missing count.
// kmin / kmax bound the candidates' keys: the bytes above their highest differing bit are
// common to every candidate and are not scanned.
template <bool SIDE_U, class Src>
__device__ int radix_pick(const Src& src, int np, int want, int32_t* out, SelSmem& sm, uint64_t kmin = 0,
                          uint64_t kmax = ~0ull) {
  if (want <= 0) return 0;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  uint64_t prefix = 0, pmask = 0;
  int remaining = want;
  bool take_all = false, bucket_all = false;
  int shift0 = 56;
  if (kmin <= kmax) {
    const uint64_t diff = kmin ^ kmax;
    shift0 = diff ? ((63 - __clzll((long long)diff)) / 8) * 8 : -8;
    pmask = shift0 >= 56 ? 0ull : ~((1ull << (shift0 + 8)) - 1ull);
    if (shift0 < 0) pmask = ~0ull;
    prefix = kmin & pmask;
  }
  for (int shift = shift0; shift >= 0; shift -= 8) {
    for (int b = tid; b < 256; b += blockDim.x) sm.hist[b] = 0;
    __syncthreads();
    for (int base = 0; base < np; base += blockDim.x) {
      const int i = base + tid;
      uint64_t key = 0;
      const bool m = (i < np) && src.template cand<SIDE_U>(i, key) && ((key & pmask) == prefix);
      const unsigned am = __ballot_sync(FULLMASK, m);
      if (m) {
        const int digit = (int)((key >> shift) & 255u);
        const unsigned peers = __match_any_sync(am, digit);
        if (lane == __ffs(peers) - 1) atomicAdd(&sm.hist[digit], __popc(peers));
      }
    }
    __syncthreads();
    if (warp == 0) {
      int loc[8], s = 0;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        loc[q] = sm.hist[lane * 8 + q];
        s += loc[q];
      }
      int incl = s;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(FULLMASK, incl, o);
        if (lane >= o) incl += y;
      }
      const int excl = incl - s;
      const int total = __shfl_sync(FULLMASK, incl, 31);
      if (lane == 0) sm.take_all = (shift == shift0 && total <= remaining) ? 1 : 0;
      if (excl < remaining && remaining <= incl) {
        int below = excl, dg = lane * 8, cnt = 0;
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          if (below + loc[q] >= remaining) {
            dg = lane * 8 + q;
            cnt = loc[q];
            break;
          }
          below += loc[q];
        }
        sm.sel_digit = dg;
        sm.sel_below = below;
        sm.sel_count = cnt;
      }
    }
    __syncthreads();
    if (sm.take_all) {
      take_all = true;
      break;
    }
    remaining -= sm.sel_below;
    prefix |= (uint64_t)sm.sel_digit << shift;
    pmask |= (uint64_t)0xffu << shift;
    const bool exact = sm.sel_count == remaining;  // the whole bucket is needed
    __syncthreads();
    if (exact) {
      bucket_all = true;
      break;
    }
  }
  // Collect in index order: keys below the bucket, then bucket keys (all of them, or the
  // first `remaining` by index when equal full keys tie).  Each warp owns a contiguous index
  // range: pass 1 counts per warp, one block scan gives each warp its output offset (and its
  // rank among tied keys), pass 2 writes.
  const int nw = blockDim.x >> 5;
  const int per = (np + nw - 1) / nw;
  const int lo = min(np, warp * per), hi = min(np, lo + per);
  auto classify = [&](int i, bool& lt, bool& eq) {
    uint64_t key = 0;
    const bool c = (i < hi) && src.template cand<SIDE_U>(i, key);
    const uint64_t mk = key & pmask;
    lt = c && (take_all || mk < prefix);
    eq = c && !take_all && mk == prefix;
  };
  int n_lt = 0, n_eq = 0;
  for (int base = lo; base < hi; base += 32) {
    bool lt, eq;
    classify(base + lane, lt, eq);
    n_lt += __popc(__ballot_sync(FULLMASK, lt));
    n_eq += __popc(__ballot_sync(FULLMASK, eq));
  }
  int eq_tot = 0;
  int eq_base = 0;
  if (!bucket_all) {
    eq_base = block_excl_scan_count(n_eq, eq_tot, sm.scan);
  }
  // this warp takes all its lt keys and the eq keys whose global rank is < remaining
  const int eq_mine = bucket_all ? n_eq : max(0, min(n_eq, remaining - eq_base));
  int tk_tot = 0;
  int out_base = block_excl_scan_count(n_lt + eq_mine, tk_tot, sm.scan);
  int eq_seen = 0;
  for (int base = lo; base < hi; base += 32) {
    bool lt, eq;
    classify(base + lane, lt, eq);
    const unsigned eb = __ballot_sync(FULLMASK, eq);
    const int erank = eq_seen + __popc(eb & ((1u << lane) - 1u));
    const bool take = lt || (eq && erank < eq_mine);
    const unsigned tb = __ballot_sync(FULLMASK, take);
    if (take) {
      const int i = base + lane;
      out[out_base + __popc(tb & ((1u << lane) - 1u))] = i;
      src.take(i);
    }
    out_base += __popc(tb);
    eq_seen += __popc(eb);
  }
  __syncthreads();
  return tk_tot;
}

template <class Src>
__device__ int select_sides(const Src& src, int np, int need, int32_t* out, SelSmem& sm, uint64_t umin = 0,
                            uint64_t umax = ~0ull, uint64_t lmin = 0, uint64_t lmax = ~0ull) {
  int cnt = radix_pick<true>(src, np, need / 2, out, sm, umin, umax);
  cnt += radix_pick<false>(src, np, need - cnt, out + cnt, sm, lmin, lmax);
  if (cnt < need) cnt += radix_pick<true>(src, np, need - cnt, out + cnt, sm, umin, umax);
  return cnt;
}

}  // namespace gmpsvm
