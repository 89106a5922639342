// finish.cuh — single-CTA selection over a small candidate set held in shared memory.
//
// The last step of a row once its candidates fit one CTA (the batched engine's per-row finish, the
// resident-cluster engine's small finish): among n (code, index) entries, the Kr smallest composite
// keys (code : R bits || index : IB bits — the lowest-index tie rule, reading 1) are
// emitted. It is the paper's radix select (Alg1 L15-28) on shared memory: per pass a
// histogram of one <= 11-bit digit, the inclusive scan and the target digit j with
// psum[j-1] < K <= psum[j], the filter (digit < j -> result, == j -> candidate), early stop when
// K == C. Passes start at the highest code bit where the entries differ (the digits above
// are common to all of them, their histograms would be single bins); a digit never straddles the
// code / index boundary. Code is compact (rolled loops): it runs once per row on a cold
// instruction cache.
#pragma once

#include "device.cuh"

namespace airtopk {

template <typename W, int NW>
struct SelScratch {
  unsigned hist[kMaxBins];
  unsigned long long tmp[NW];
  ScanResult res;
  W wmin[NW], wmax[NW];
  W cw[32];          // <= 32 live entries compacted for warp 0's rank count
  unsigned ci[32];
  unsigned cn;
};

// Entry e = tid + t * BLOCK (t < tcnt, block-uniform) is live iff bit t of `valid`. C = number of
// live entries (block-wide), Kr <= C. emit(pred, code, idx) is called by every thread (warp
// collective) for each of its slots; it must place the selected entries.
template <int KIND, int BLOCK, typename Emit>
__device__ void block_select_smem(const typename KT<KIND>::U* stc, const unsigned* sti, int tcnt, unsigned valid,
                                  unsigned long long Kr, unsigned long long C, int IB, bool early_stop,
                                  SelScratch<std::conditional_t<sizeof(typename KT<KIND>::U) == 8, unsigned long long,
                                                                unsigned>, BLOCK / 32>& sh,
                                  Emit emit) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  constexpr int WB = 8 * (int)sizeof(W);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (C <= 32 && tcnt == 1 && __syncthreads_and(tid < 32 || !(valid & 1u))) {
    // at most 32 live entries, all held by warp 0: rank them by counting (one shuffle round) — the
    // K smallest composite keys are the ranks < K (keys are unique)
    if (warp == 0) {
      const bool v = valid & 1u;
      const U c = v ? stc[tid] : (U)0;
      const unsigned ix = v ? sti[tid] : 0u;
      // rank by counting over the live lanes' entries, read as shared-memory broadcasts (independent
      // loads: no serial shuffle chain)
      const unsigned vm = __ballot_sync(kFull, v);
      unsigned rank = 0;
#pragma unroll 8
      for (int o = 0; o < 32; ++o) {
        const W co = (W)stc[o];
        const unsigned io = sti[o];
        rank += ((vm >> o) & 1u) && (co < (W)c || (co == (W)c && io < ix));
      }
      emit(v && rank < Kr, c, ix);
    }
    return;
  }
  // extremes of the live codes: the digits above their highest differing bit are common
  W mmin = ~(W)0, mmax = 0;
#pragma unroll 1
  for (int t = 0, e = tid; t < tcnt; ++t, e += BLOCK) {
    if ((valid >> t) & 1u) {
      const W c = (W)stc[e];
      mmin = c < mmin ? c : mmin;
      mmax = c > mmax ? c : mmax;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const W a = shfl(mmin, lane ^ o), b = shfl(mmax, lane ^ o);
    mmin = a < mmin ? a : mmin;
    mmax = b > mmax ? b : mmax;
  }
  if (lane == 0) {
    sh.wmin[warp] = mmin;
    sh.wmax[warp] = mmax;
  }
  __syncthreads();
  mmin = lane < BLOCK / 32 ? sh.wmin[lane] : ~(W)0;
  mmax = lane < BLOCK / 32 ? sh.wmax[lane] : (W)0;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const W a = shfl(mmin, lane ^ o), b = shfl(mmax, lane ^ o);
    mmin = a < mmin ? a : mmin;
    mmax = b > mmax ? b : mmax;
  }
  const W diff = mmin ^ mmax;
  int pos = IB + (diff ? (WB - (sizeof(W) == 8 ? __clzll((long long)diff) : __clz((int)diff))) : 0);
#pragma unroll 1
  while (pos > 0 && !(Kr == C && early_stop)) {
    const bool is_idx = pos <= IB;
    const int top = is_idx ? pos : pos - IB;
    const int w = top < kDigitBits ? top : kDigitBits, shf = top - w;
    const unsigned dm = (1u << w) - 1u;
    for (int i = tid; i < (1 << w); i += BLOCK) sh.hist[i] = 0;
    __syncthreads();
#pragma unroll 1
    for (int t = 0, e = tid; t < tcnt; ++t, e += BLOCK) {
      if ((valid >> t) & 1u) {
        const unsigned d = is_idx ? (sti[e] >> shf) & dm : (unsigned)((W)stc[e] >> shf) & dm;
        atomicAdd(&sh.hist[d], 1u);
      }
    }
    __syncthreads();
    const ScanResult r = scan_choose<BLOCK>([&](int b) { return (unsigned long long)sh.hist[b]; }, 1 << w, Kr,
                                           sh.tmp, &sh.res);
#pragma unroll 1
    for (int t = 0, e = tid; t < tcnt; ++t, e += BLOCK) {
      const bool v = (valid >> t) & 1u;
      const U c = v ? stc[e] : (U)0;
      const unsigned ix = v ? sti[e] : 0u;
      const unsigned d = is_idx ? (ix >> shf) & dm : (unsigned)((W)c >> shf) & dm;
      emit(v && d < r.j, c, ix);
      if (!(v && d == r.j)) valid &= ~(1u << t);
    }
    Kr -= r.before;
    C = r.cnt;
    pos -= w;
    if (C <= 32 && pos > 0 && !(Kr == C && early_stop)) {
      // at most 32 live entries left: compact them into shared memory and let warp 0 rank them by
      // counting (one shuffle round) instead of running the remaining histogram passes
      if (tid == 0) sh.cn = 0;
      __syncthreads();
#pragma unroll 1
      for (int t = 0, e = tid; t < tcnt; ++t, e += BLOCK) {
        if ((valid >> t) & 1u) {
          const unsigned slot = atomicAdd(&sh.cn, 1u);
          sh.cw[slot] = (W)stc[e];
          sh.ci[slot] = sti[e];
        }
      }
      __syncthreads();
      if (warp == 0) {
        const bool v = lane < (int)C;
        const W c = v ? sh.cw[lane] : (W)0;
        const unsigned ix = v ? sh.ci[lane] : 0u;
        unsigned rank = 0;
#pragma unroll 8
        for (int o = 0; o < 32; ++o) {
          const W co = sh.cw[o];
          const unsigned io = sh.ci[o];
          rank += (o < (int)C) && (co < c || (co == c && io < ix));
        }
        emit(v && rank < Kr, (U)c, ix);
      }
      return;
    }
  }
  // early stop (K == C) or the last digit: every remaining candidate is a result
#pragma unroll 1
  for (int t = 0, e = tid; t < tcnt; ++t, e += BLOCK) {
    const bool v = (valid >> t) & 1u;
    emit(v, v ? stc[e] : (U)0, v ? sti[e] : 0u);
  }
}

// Sample order statistic of rank `rank` among s[0..ns) (shared memory), all BLOCK threads: MSD
// digits of up to 11 bits below the bits on which every sample agrees; once at most kRankBrute
// samples share the prefix they are compacted and ranked by counting. SH provides hist[kMaxBins],
// brute[kRankBrute], tmp[BLOCK / 32], res, result, cnt (shared memory).
constexpr int kRankBrute = 1024;

// Sample order statistic of rank `rank` among the samples s[0..ns) (shared memory), all threads.
// MSD digits of up to 11 bits below the bits on which every sample agrees (prefix); once at most
// kRankBrute samples share the prefix they are compacted and ranked by counting.
template <typename W, int BLOCK, typename SH, typename Stamp = NoStamp>
__device__ W sample_rank(const W* s, int ns, int rank, W smin, W smax, SH& sh, Stamp stamp = Stamp()) {
  constexpr int WB = 8 * (int)sizeof(W);
  const W diff = smin ^ smax;
  int hb = diff ? (WB - (sizeof(W) == 8 ? __clzll((long long)diff) : __clz((int)diff))) : 0;
  W mask = (hb >= WB) ? (W)0 : (W)(~(W)0 << hb);
  W prefix = smin & mask;
  int cnt = ns;
  while (true) {
    if (hb == 0) return prefix;
    if (cnt <= kRankBrute) {
      if (threadIdx.x == 0) sh.cnt = 0;
      __syncthreads();
#pragma unroll 1
      for (int i = threadIdx.x; i < ns; i += BLOCK) {
        const W x = s[i];
        const bool m = (x & mask) == prefix;
        const unsigned b = __ballot_sync(kFull, m);
        unsigned base = 0;
        if ((threadIdx.x & 31) == 0 && b) base = atomicAdd(&sh.cnt, (unsigned)__popc(b));
        base = __shfl_sync(kFull, base, 0);
        if (m) sh.brute[base + __popc(b & lanemask_lt())] = x;
      }
      __syncthreads();
      stamp(3);
      if ((int)threadIdx.x < cnt) {
        const W x = sh.brute[threadIdx.x];
        int less = 0, eq = 0;
#pragma unroll 4
        for (int j = 0; j < cnt; ++j) {
          const W y = sh.brute[j];
          less += y < x;
          eq += y == x;
        }
        if (less <= rank && rank < less + eq) sh.result = x;
      }
      __syncthreads();
      stamp(4);
      const W r = sh.result;
      __syncthreads();
      return r;
    }
    const int shf = hb > kDigitBits ? hb - kDigitBits : 0, w = hb - shf;
    const unsigned dm = (1u << w) - 1u;
    for (int i = threadIdx.x; i < (1 << w); i += BLOCK) sh.hist[i] = 0;
    __syncthreads();
    stamp(0);
#pragma unroll 1
    for (int i = threadIdx.x; i < ns; i += BLOCK) {
      const W x = s[i];
      if ((x & mask) == prefix) atomicAdd(&sh.hist[(unsigned)(x >> shf) & dm], 1u);
    }
    __syncthreads();
    stamp(1);
    const ScanResult r = scan_choose<BLOCK>([&](int b) { return (unsigned long long)sh.hist[b]; }, 1 << w,
                                             (unsigned long long)rank + 1, sh.tmp, &sh.res);
    stamp(2);
    rank -= (int)r.before;
    cnt = (int)r.cnt;
    prefix |= (W)r.j << shf;
    mask |= (W)dm << shf;
    hb = shf;
  }
}

// Phase A for one row (all threads): window [lo, hi] from the sample order statistics.
}  // namespace airtopk
