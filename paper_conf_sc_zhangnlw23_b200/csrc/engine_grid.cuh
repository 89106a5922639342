// engine_grid.cuh — the iteration-fused multi-CTA engine (one launch per radix pass).
//
// Algorithm 1 of the paper, as reconstructed in SURVEY.md §8(c)-0, mapped to B200:
//   host (Alg1 L1-5): memset the per-row state, then enqueue P+1 launches of pass_kernel
//     (q = 0..P-1: "iteration_fused_kernel", q = P: "last_filter_kernel"); no host sync, no copy
//     (P:50). P = ceil(r/11) key digits (+ index digits, see below).
//   kernel q (Alg1 L6-29):
//     L7-8   source = input L if C' >= N/alpha, else the candidate buffer written by kernel q-1;
//     L11-13 q == 0: histogram of digit 0 of every element;
//     L15-22 q >= 1: classify digit q-1 against the target digit: smaller -> result (V, I);
//            equal -> candidate: appended to the buffer iff C < N/alpha and counted in the
//            histogram of digit q (iteration fusion: ONE load serves filter(q-1) and hist(q));
//     L23-28 the last CTA of the row to finish (atomic ticket) scans the histogram, picks j
//            with psum[j-1] < K <= psum[j], and updates C' <- C, C <- hist[j], K <- K - psum[j-1];
//     early stop: when K == C after a scan, kernel q+1 emits every candidate
//            (digit <= j) and all later kernels return immediately.
//   The last filter is kernel q = P, always in "emit all" mode: after the index digits the
//   composite key (code, index) is unique, so the final scan always ends with K == C = 1.
//
// Lowest-index tie-break (reading 1): the key is extended by the row index bits
// (code : R || index : IB). The index digits only ever run when ties at the K-th code straddle K
// (otherwise the early stop fires after the last code digit), and they follow the same adaptive
// rule, so for radix-adversarial data the first index pass reads L once and buffers the ties.
//
// B200 mapping:
//   * grid = batch x cpr CTAs of 512 threads, 2 CTAs/SM (296 CTAs fill the 148 SMs; measured
//     faster than 3-4/SM), tile t of a row -> CTA t mod cpr (grid-stride: the CTAs of a row read one
//     compact advancing region), or for a few long rows 1 CTA/SM streaming through a bulk-copy ring;
//   * 4 x 128-bit ld.global.nc.L1::no_allocate loads in flight per thread (32 KiB per CTA tile);
//   * odd passes walk their tiles backwards so the tail the previous pass left in the 126 MB L2 is
//     consumed first;
//   * 2048-bin shared histogram with plain shared atomics (measured at HBM speed on B200 even with
//     32-way same-bin conflicts), merged with global red.add of the nonzero bins only;
//   * a thread's 16 elements are classified with 3 integer ops each; only if any lane of the warp
//     holds a result/candidate does the warp take the slow path: per-warp shared-memory queues
//     (64 entries) that flush with ONE global atomic per 64 entries and coalesced stores;
//   * kernel variants are compile-time specialised on the kind of digit filtered (DF) and
//     histogrammed (DH): 0 none, 1 key digit, 2 index digit.
#pragma once

#include <algorithm>
#include <cstdlib>
#include <type_traits>

#include <cooperative_groups.h>

#include "device.cuh"
#include "engine.h"
#include "finish.cuh"
#include "passes.cuh"

namespace airtopk {

struct GridParams {
  const void* keys;
  const int64_t* in_idx;
  int64_t batch, len, k;
  int sel_min;
  int P, IB;
  void* out_vals;
  int64_t* out_idx;
  RowState* st;
  void* ghist;
  void* bcode;
  void* bidx;
  int64_t cap_rule, cap_alloc;
  int cpr;
  int cpr_buf;  // passes q >= 1 after a bulk-copy window pass (they read the window buffer)
  int64_t* trace;
  void* samp;  // sample-guided window: [batch][nsamp] sampled codes
  int nsms;    // SMs of the device
  int small_finish;  // a buffer-source pass over <= this many entries finishes the row in one CTA
  int early_stop;   // 0 on, -1 off (ablation)
  int64_t idx_off;  // added to every output index (airtopk_select_shard)
  int64_t* tstamp;  // fused tail debug: per pass [run_pass done, barrier passed, scan done] (CTA 0)
  void* thist;      // fused tail (batch 1): 3 rotating global histograms
  unsigned long long* tcnt;  // fused tail: candidates stored by pass q (zeroed with the state)
};

constexpr int kBlock = 512;
#ifndef AIRTOPK_GRID_BU
#define AIRTOPK_GRID_BU 4
#endif
constexpr int kGridBU = AIRTOPK_GRID_BU;  // buffer entries per thread per iteration of a buffer pass
constexpr int kSmallFinish = 1024;  // max buffer entries of the single-CTA finish (shared memory)

constexpr int kWarps = kBlock / 32;
#ifndef AIRTOPK_TMA_FILTER_HC
#define AIRTOPK_TMA_FILTER_HC 2  // measured (c3, paper passes): pass 2 741 -> 722 us (6 instead of 5 ring stages); c4 unchanged
#endif
// Histogram copies of a grid pass. Bulk-copy (TMA) filter passes may use fewer copies than the
// register path (AIRTOPK_TMA_FILTER_HC > 0): the shared memory saved becomes ring stages.
template <int KIND, typename IdxT, int DF, bool TMA>
__host__ __device__ constexpr int pass_hc() {
  return (TMA && (DF == 1 || DF == 2) && AIRTOPK_TMA_FILTER_HC > 0) ? AIRTOPK_TMA_FILTER_HC
                                                                      : hist_copies<KIND, IdxT, DF>();
}
#ifndef AIRTOPK_WINDOW_L2PRE
#define AIRTOPK_WINDOW_L2PRE 0
#endif
constexpr int kWindowL2Pre = AIRTOPK_WINDOW_L2PRE;  // chunks per CTA prefetched into L2 before the PDL wait
#ifndef AIRTOPK_WINDOW_EARLY
#define AIRTOPK_WINDOW_EARLY 1
#endif
constexpr bool kWindowEarly = AIRTOPK_WINDOW_EARLY != 0;  // window pass: ring stages issued before the PDL wait
#ifndef AIRTOPK_TAIL_IDENT
#define AIRTOPK_TAIL_IDENT 1
#endif
constexpr bool kTailIdent = AIRTOPK_TAIL_IDENT != 0;  // fused tail: identity-filter elision

#ifndef AIRTOPK_MINB
#define AIRTOPK_MINB 2
#endif
constexpr int kMinBlocks = AIRTOPK_MINB;
constexpr int kMinBlocksFilter = AIRTOPK_SLOW_REG ? 2 : AIRTOPK_MINB;

// Kernel q of the select. DF/DH: digit filtered / histogrammed (passes.cuh). DF == 3 is the
// sample-guided window pass (q = 0); `redo` = the pass-0 histogram re-run over the window buffer.
// TMA: the input row is streamed through per-warp shared rings by the bulk-copy engine (1 CTA/SM,
// DESIGN.md "Kernels"); otherwise 4 x 16-byte register loads per thread (2 CTAs/SM).
// Debug timing of pass q (trace mode only; trace slot 7 + q of the row, zero-initialised):
// [0] ~min CTA start, [1] max run_pass end, [2] max ticket arrival, [3] last CTA: scan done,
// [4] CTA 0 start, [5] CTA 0 run_pass end
__device__ __forceinline__ void dbg_stamp(int64_t* trace, int64_t row, int q, int f, int mode, int P) {
  // only slots no pass record uses (passes 0..P fill slots 0..P; slot 15: sample_kernel)
  if (trace == nullptr || threadIdx.x != 0 || 7 + q >= kTraceMaxPasses - 1 || 7 + q <= P) return;
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  unsigned long long* a = (unsigned long long*)(trace + ((size_t)row * kTraceMaxPasses + 7 + q) * kTraceFields + f);
  if (mode == 0) atomicMax(a, ~t);
  else if (mode == 1) atomicMax(a, t);
  else *a = t;
}

template <int KIND, typename IdxT, int DF, int DH, bool HASIDX, bool TMA = false>
__global__ void __launch_bounds__(kBlock, TMA ? 1 : (DF == 0 ? kMinBlocks : kMinBlocksFilter))
    pass_kernel(const GridParams p, const int q, const int redo) {
  using U = typename KT<KIND>::U;
  using CountT = std::conditional_t<sizeof(IdxT) == 8, unsigned long long, unsigned>;
  constexpr bool HAS_Q = DF != 0;
  constexpr bool FILTER = (DF == 1 || DF == 2);  // Alg1 L15-22 filter of digit q-1
  constexpr int HC = pass_hc<KIND, IdxT, DF, TMA>();

  extern __shared__ unsigned sh_hist[];  // kHistSlots * HC counters (dynamic: may exceed 48 KB)
  __shared__ WarpQ<U, IdxT> sh_wq[HAS_Q ? kWarps : 1];  // per-warp tagged result / candidate queues
  __shared__ unsigned long long sh_tmp[kWarps];
  __shared__ ScanResult sh_res;
  __shared__ int sh_last;

  const int64_t row = blockIdx.x / p.cpr;
  const int cta = blockIdx.x % p.cpr;
  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  RowState* st = p.st + row;
  // Window pass over bulk copies: the ring's first stages (input keys only: nothing the sample kernel
  // writes) are requested BEFORE the PDL wait, so they stream in while the sample kernel finishes.
  // (The keys' producer completed before the sample kernel passed its own wait and triggered us.)
  int pre_issued = 0;
  if constexpr (DF == 3 && TMA && kWindowEarly) {
    const typename KT<KIND>::U* rp = (const typename KT<KIND>::U*)p.keys + row * p.len;
    pre_issued = tma_prologue<typename KT<KIND>::U, HC, kBlock>(rp, p.len, cta, p.cpr, false,
                                                                smem_addr(sh_hist) + (unsigned)tma_ring_offset<HC>());
    tma_prefetch_l2<typename KT<KIND>::U, kBlock>(rp, p.len, cta, p.cpr, tma_stages<HC>(), kWindowL2Pre);
  }
  pdl_wait();     // the previous pass's scan (row state, buffers) is complete and visible
  pdl_trigger();  // the next pass may be scheduled as our CTAs retire (hides launch latency)

  // ---- row state after scan q-1 ----
  const int stop1 = FILTER ? st->stop1 : 0;
  if (FILTER && stop1 != 0 && stop1 - 1 < q - 1) return;  // finished by an earlier early stop
  if (FILTER && q < st->npass) return;                     // digit done by the window pass (digit skip)
  const int win_state = (DF == 3 || (DF == 0 && redo)) ? st->win_state : 0;
  if (DF == 3 && win_state != 1) {                         // no window: pass 0 will read L
    if constexpr (TMA) {  // the pre-issued copies must land before the CTA's shared memory is released
      const unsigned fullb = smem_addr(sh_hist) + (unsigned)tma_ring_offset<HC>() + tma_stages<HC>() * kTmaChunk;
      for (int i = 0; i < pre_issued; ++i) mbar_wait(fullb + 8u * i, 0);
    }
    return;
  }
  if (DF == 0 && redo && win_state == 1) return;           // pass 0 was done by the window pass
  const int src1 = FILTER ? st->src1 : 0;    // Alg1 L7-8 (reading 6)
  const int sslot = (src1 == 1) ? 1 : 0;                   // candidate buffer this pass writes
  PassCtx<U, IdxT> c;
  c.q = q;
  c.emit_all = FILTER && ((stop1 != 0 && stop1 - 1 == q - 1) || DH == 0);
  c.do_hist = (DH != 0) && !c.emit_all;
  const unsigned long long Cprev = FILTER ? st->C : (unsigned long long)p.len;  // C_{q-1}
  c.srcL = (src1 == 0);
  if (DF == 3) c.store = (win_state == 1);
  else c.store = c.do_hist && FILTER && (Cprev <= (unsigned long long)p.cap_rule);  // Alg1 L17
  c.sel_min = p.sel_min != 0;
  c.reverse = (q & 1) != 0;  // walk back over what the previous pass left in L2
  // Window digit skip: every window member lies in [lo, hi], so the leading key digits on which lo
  // and hi agree are common to all members (their histograms would be single bins). The window pass
  // histograms the first digit where they may differ (qs); launches 1..qs then have nothing to do.
  int qs = q;
  if (DF == 3) {
    const int pc = code_passes(KT<KIND>::R);
    qs = 0;
    while (qs < pc - 1) {
      const Digit d = digit_of(qs, KT<KIND>::R, p.IB);
      if ((st->win_lo >> d.shift) != (st->win_hi >> d.shift)) break;
      ++qs;
    }
  }
  c.dh = digit_of(qs, KT<KIND>::R, p.IB);
  // window pass: the members' histogram of the next digit too (used when all members turn out to
  // share digit qs; only key digits: qs + 1 < code passes, else a copy of dh that is never used)
  const bool two = (DF == 3) && (qs + 1 < code_passes(KT<KIND>::R));
  c.dh2 = digit_of(two ? qs + 1 : qs, KT<KIND>::R, p.IB);
  c.df = digit_of(FILTER ? q - 1 : 0, KT<KIND>::R, p.IB);
  c.tcode = FILTER ? st->tcode : 0ull;
  c.tidx = FILTER ? st->tidx : 0ull;
  c.wnmin = &st->win_nmin;
  c.wmax = &st->win_max;
  c.lo = (win_state == 1) ? st->win_lo : 0ull;
  c.span1 = (win_state == 1) ? st->win_hi - st->win_lo + 1ull : 0ull;
  c.rowp = (const U*)p.keys + row * p.len;
  c.rowi = HASIDX ? p.in_idx + row * p.len : nullptr;
  c.len = p.len;
  c.slice = cta;
  c.nslices = p.cpr;
  const int islot = src1 > 0 ? src1 - 1 : 0;
  c.bcin = (const U*)p.bcode + ((size_t)islot * p.batch + row) * p.cap_alloc;
  c.biin = (const IdxT*)p.bidx + ((size_t)islot * p.batch + row) * p.cap_alloc;
  c.nbuf = (src1 > 0) ? st->buf_count[islot] : 0ull;
  c.ov = (U*)p.out_vals + row * p.k;
  c.oi = p.out_idx + row * p.k;
  c.ioff = p.idx_off;
  c.outc = &st->out_count;
  c.kk = (unsigned long long)p.k;
  c.bco = (U*)p.bcode + ((size_t)sslot * p.batch + row) * p.cap_alloc;
  c.bio = (IdxT*)p.bidx + ((size_t)sslot * p.batch + row) * p.cap_alloc;
  c.bufc = &st->buf_count[sslot];
  c.capa = (unsigned long long)p.cap_alloc;
  c.err = &st->error;
  c.hist = sh_hist;
  c.ring = smem_addr(sh_hist) + (unsigned)tma_ring_offset<HC>();
  c.pre = (DF == 3 && TMA && kWindowEarly);
  c.wq = &sh_wq[HAS_Q ? warp : 0];

  if constexpr (FILTER && DH != 0) {
    if (!c.emit_all && !c.srcL && c.nbuf <= (unsigned long long)p.small_finish && p.trace == nullptr) {
      if (cta == 0) {
        small_finish<KIND, IdxT, kBlock>(c, st->K, (U*)sh_hist,
                                         (IdxT*)((unsigned char*)sh_hist + kSmallFinish * sizeof(U)));
        if (tid == 0) st->stop1 = c.q;  // later launches (q' > q) return at once
      }
      return;
    }
  }
  dbg_stamp(p.trace, row, q, 0, 0, p.P);
  if (cta == 0) dbg_stamp(p.trace, row, q, 4, 2, p.P);
  const bool hist_on = c.do_hist || DF == 0 || DF == 3;
  if (hist_on) {
    for (int i = tid; i < kHistSlots * HC; i += kBlock) sh_hist[i] = 0;
    __syncthreads();
  }

  const unsigned long long nread = run_pass<KIND, IdxT, DF, DH, HASIDX, kBlock, HC, TMA, kGridBU>(c);
  dbg_stamp(p.trace, row, q, 1, 1, p.P);
  if (cta == 0) dbg_stamp(p.trace, row, q, 5, 2, p.P);

  if (!hist_on) return;

  // ---- merge into the row histogram; the last CTA scans ----
  __syncthreads();
  Digit dh = c.dh;
  CountT* gh = (CountT*)p.ghist + ((size_t)row * 2 + (q & 1)) * kMaxBins;
  int nb = 1 << dh.width;
  if constexpr (DF == 3) {  // two member histograms: digit qs -> slot 0, digit qs + 1 -> slot 1
    CountT* gh1 = (CountT*)p.ghist + ((size_t)row * 2 + 1) * kMaxBins;
    const int nb2 = 1 << c.dh2.width;
    for (int i = tid; i < nb; i += kBlock)
      if (sh_hist[i]) atomicAdd(&gh[i], (CountT)sh_hist[i]);
    if (two)
      for (int i = tid; i < nb2; i += kBlock)
        if (sh_hist[kHistSlots + i]) atomicAdd(&gh1[i], (CountT)sh_hist[kHistSlots + i]);
  } else {
    for (int i = tid; i < nb; i += kBlock) {
      unsigned v = 0;
#pragma unroll
      for (int h = 0; h < HC; ++h) v += sh_hist[i * HC + h];
      if (v) atomicAdd(&gh[i], (CountT)v);
    }
  }
  __syncthreads();  // the CTA's histogram merge / queue flushes precede thread 0's release
  dbg_stamp(p.trace, row, q, 2, 1, p.P);
  if (tid == 0) sh_last = (ticket_arrive(&st->ticket) == (unsigned)(p.cpr - 1));
  __syncthreads();
  if (!sh_last) return;

  const unsigned long long kk = (unsigned long long)p.k;
  unsigned long long Kin = FILTER ? st->K : kk;
  unsigned long long Cin = Cprev;  // elements counted by this histogram
  bool window_ok = false;
  if constexpr (DF == 3) {
    // ---- window pass: R results below lo, Wn members inside; the K-th key lies in the window iff
    // R < K <= R + Wn (and the buffer did not overflow). Then the histogram just merged is pass 1's
    // over the window buffer: a fresh select of K - R among the Wn members continues from it. ----
    const unsigned long long R = __ldcg(c.outc), Wn = __ldcg(c.bufc);
    window_ok = (__ldcg(&st->error) & 2u) == 0 && R < kk && kk <= R + Wn;
    Kin = kk - R;
    Cin = Wn;
    if (!window_ok) {  // miss: discard, the redo launch re-runs the paper's pass 1 over L
      for (int i = tid; i < kMaxBins; i += kBlock) gh[i] = 0;  // (slot 1 is zeroed by the redo's scan)
      if (tid == 0) {
        st->win_state = 2;
        st->out_count = 0;
        st->buf_count[sslot] = 0;
        st->error &= ~2u;
        st->ticket = 0;
      }
      return;
    }
    // every member shares digit qs as well (their extremes agree on it): digit qs's histogram is a
    // single bin, so continue from digit qs + 1's (slot 1) — launch qs + 1 then has nothing to do
    if (two) {
      const unsigned long long wmin = ~__ldcg(&st->win_nmin), wmax = __ldcg(&st->win_max);
      if (Wn > 0 && (wmin >> dh.shift) == (wmax >> dh.shift)) {
        qs += 1;
        dh = c.dh2;
        nb = 1 << dh.width;
        gh = (CountT*)p.ghist + ((size_t)row * 2 + 1) * kMaxBins;
      }
    }
  }
  const ScanResult r = scan_choose<kBlock>(
      [&](int b) { return (unsigned long long)__ldcg(&gh[b]); }, nb, Kin, sh_tmp, &sh_res);
  __syncthreads();  // (after a window digit skip the next pass may use the slot just scanned)
  CountT* gh2 = (CountT*)p.ghist + ((size_t)row * 2 + ((qs + 1) & 1)) * kMaxBins;
  for (int i = tid; i < kMaxBins; i += kBlock) gh2[i] = 0;
  if (tid == 0) {
    int next_src1 = (c.store) ? sslot + 1 : src1;  // the buffer this pass wrote feeds the next one
    if (DF == 3) st->Cp = Cin;
    {
      const unsigned long long newK = Kin - r.before, newC = r.cnt;   // Alg1 L26-28
      st->Cp = Cin;
      st->C = newC;
      st->K = newK;
      if (DF == 3 && qs > 0) {  // the digits above dh: common to every member (lo/hi, or their extremes)
        const unsigned long long ref = (gh == (CountT*)p.ghist + ((size_t)row * 2 + 1) * kMaxBins)
                                           ? ~__ldcg(&st->win_nmin) : st->win_lo;
        st->tcode = ref >> (dh.shift + dh.width) << (dh.shift + dh.width);
      }
      if (!dh.is_idx) st->tcode |= (unsigned long long)r.j << dh.shift;
      else st->tidx |= (unsigned long long)r.j << dh.shift;
      st->j = r.j;
      st->npass = qs + 1;
      if (newK == newC && p.early_stop == 0) st->stop1 = qs + 1;  // early stop; qs = the digit scanned (window skip)
      st->src1 = next_src1;
      st->buf_count[next_src1 == 1 ? 1 : 0] = 0;                        // next pass's output buffer
      if (r.total != Cin) st->error |= 4u;
      if (p.trace && q < kTraceMaxPasses) {
        int64_t* t = p.trace + ((size_t)row * kTraceMaxPasses + q) * kTraceFields;
        t[0] = dh.width; t[1] = c.srcL; t[2] = c.store; t[3] = r.j; t[4] = (int64_t)newK; t[5] = (int64_t)newC;
        t[6] = (int64_t)Cin; t[7] = (int64_t)__ldcg(c.outc); t[8] = (newK == newC); t[9] = (int64_t)nread;
      }
    }
    st->ticket = 0;
  }
  dbg_stamp(p.trace, row, q, 3, 2, p.P);
}

// Sample-guided window: one CTA per row reads S
// stratified samples, selects the sample order statistics at ranks r -/+ margin around the expected
// rank of the K-th key, and stores them as the window [lo, hi]. Exactness never depends on it: the
// window pass validates the window and falls back to the paper's passes when it misses.
constexpr int kSampleBlock = 1024;
constexpr int kMaxSamples = 16384;

// Radix rank select over a[0..n) in shared memory, 8-bit MSD digits for bits [lo_bits, hi_bits):
// elements outside (v & mask) == prefix are ignored; prefix / mask / rank are updated in place (every
// thread holds the same values). The 256-bin scan is done by warp 0 (8 bins per lane + shuffles).
template <typename W>
__device__ void select_digits(const W* a, int n, int& rank, W& prefix, W& mask, int hi_bits, int lo_bits,
                              unsigned* hist /* 256 */, W* shw) {
  const int lane = threadIdx.x & 31;
  for (int hi = hi_bits; hi > lo_bits; hi -= 8) {
    const int w = (hi - lo_bits) < 8 ? (hi - lo_bits) : 8, sh = hi - w;
    for (int i = threadIdx.x; i < 256; i += blockDim.x) hist[i] = 0;
    __syncthreads();
    for (int i = threadIdx.x; i < n; i += blockDim.x) {
      const W v = a[i];
      if ((v & mask) == prefix) atomicAdd(&hist[(unsigned)(v >> sh) & ((1u << w) - 1u)], 1u);
    }
    __syncthreads();
    if (threadIdx.x < 32) {
      unsigned c[8], tot = 0;
#pragma unroll
      for (int t = 0; t < 8; ++t) { c[t] = hist[lane * 8 + t]; tot += c[t]; }
      unsigned incl = tot;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned y = __shfl_up_sync(kFull, incl, o);
        if (lane >= o) incl += y;
      }
      unsigned run = incl - tot;
      if (run <= (unsigned)rank && (unsigned)rank < incl) {
#pragma unroll
        for (int t = 0; t < 8; ++t) {
          if (run <= (unsigned)rank && (unsigned)rank < run + c[t]) {
            shw[0] = (W)(lane * 8 + t);
            shw[1] = (W)run;
          }
          run += c[t];
        }
      }
    }
    __syncthreads();
    prefix |= shw[0] << sh;
    rank -= (int)shw[1];
    mask |= (W)((1u << w) - 1u) << sh;
    __syncthreads();
  }
}

// Sample order statistics at ranks rlo (skipped when < 0) and rhi in one sweep over the samples
// held in registers (v[t] = sample t * blockDim + tid, valid for t < tv): one 11-bit digit below the
// common prefix (bits [hb-11, hb)), block-wide scan of 2048 bins (2 per thread), compaction of the
// one or two chosen bins into `scratch`, then the exact rank inside each bin by counting (bins of
// <= kBrute samples) or, for concentrated samples, 8-bit digits over the bin (select_digits).
// Written for a short critical path: no loop carries a shared-memory load-atomic chain.
constexpr int kBrute = 128;
constexpr int kSampleHistCopies = 4;
static_assert(kSampleBlock / 8 >= kBrute, "8 threads per bin member in the brute-force rank");

template <typename W, int PER, typename Stamp = NoStamp>
__device__ void block_select_two(const W (&v)[PER], int tv, W* scratch, int rlo, int rhi, W pmin, int hb,
                                 unsigned* hist /* 2048 x copies */, unsigned* wsum /* 32 */, W* shw, int* cnt,
                                 W& lo, W& hi, Stamp stamp = Stamp()) {
  constexpr int WB = 8 * (int)sizeof(W);
  if (hb <= 0) {  // all samples equal
    lo = hi = pmin;
    return;
  }
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int w = hb < 11 ? hb : 11, sh = hb - w;
  const unsigned dmask = (1u << w) - 1u;
  const W mask = (hb >= WB) ? (W)0 : (W)(~(W)0 << hb);
  const W prefix = pmin & mask;
  // kSampleHistCopies interleaved copies of each bin (lane % copies): uniform samples crowd a few
  // bins (e.g. half of (0, 1] lies in one octave), and the copies cut the same-address serialisation
  for (int i = threadIdx.x; i < 2048 * kSampleHistCopies; i += blockDim.x) hist[i] = 0;
  if (threadIdx.x < 2) cnt[threadIdx.x] = 0;
  __syncthreads();
  const unsigned hcopy = (unsigned)(lane % kSampleHistCopies);
#pragma unroll
  for (int t = 0; t < PER; ++t)
    if (t < tv) atomicAdd(&hist[((unsigned)(v[t] >> sh) & dmask) * kSampleHistCopies + hcopy], 1u);
  __syncthreads();
  stamp(0);
  auto binc = [&](unsigned b) {
    unsigned x = 0;
#pragma unroll
    for (int h = 0; h < kSampleHistCopies; ++h) x += hist[b * kSampleHistCopies + h];
    return x;
  };
  // block scan: thread t owns bins 2t, 2t+1 (1024 threads)
  const unsigned c0 = binc(2 * threadIdx.x), c1 = binc(2 * threadIdx.x + 1), tot = c0 + c1;
  unsigned incl = tot;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned y = __shfl_up_sync(kFull, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) wsum[warp] = incl;
  __syncthreads();
  unsigned wi = wsum[lane];
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned y = __shfl_up_sync(kFull, wi, o);
    if (lane >= o) wi += y;
  }
  const unsigned wex = warp ? __shfl_sync(kFull, wi, warp - 1) : 0u;
  const unsigned s0 = wex + incl - tot, s1 = s0 + c0;
  // shw[0..1]: chosen bin of rank lo / hi, shw[2..3]: samples before it (one writer each)
  if (rlo >= 0) {
    if (s0 <= (unsigned)rlo && (unsigned)rlo < s1) { shw[0] = 2 * threadIdx.x; shw[2] = s0; }
    if (s1 <= (unsigned)rlo && (unsigned)rlo < s1 + c1) { shw[0] = 2 * threadIdx.x + 1; shw[2] = s1; }
  }
  if (s0 <= (unsigned)rhi && (unsigned)rhi < s1) { shw[1] = 2 * threadIdx.x; shw[3] = s0; }
  if (s1 <= (unsigned)rhi && (unsigned)rhi < s1 + c1) { shw[1] = 2 * threadIdx.x + 1; shw[3] = s1; }
  __syncthreads();
  const unsigned blo = (rlo >= 0) ? (unsigned)shw[0] : 0xffffffffu, bhi = (unsigned)shw[1];
  const int rk_lo = rlo - (int)shw[2], rk_hi = rhi - (int)shw[3];
  const int m_lo = (rlo >= 0) ? (int)binc(blo) : 0, m_hi = (int)binc(bhi);
  stamp(1);
  const W plo = prefix | ((W)blo << sh), phi = prefix | ((W)bhi << sh);
  if (sh == 0) {
    lo = plo;
    hi = phi;
    return;
  }
  // compaction from registers: per-thread counts, one warp scan, one shared atomic per warp and bin
  const bool same = (blo == bhi);
  W* reg_lo = scratch;
  W* reg_hi = same ? scratch : scratch + m_lo;
  unsigned cl = 0, ch = 0;
#pragma unroll
  for (int t = 0; t < PER; ++t) {
    const unsigned d = (unsigned)(v[t] >> sh) & dmask;
    cl += (t < tv) && d == blo;
    ch += (t < tv) && !same && d == bhi;
  }
  unsigned pk = cl | (ch << 16), pki = pk;  // <= 16 per thread, <= 512 per warp: 16-bit fields
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned y = __shfl_up_sync(kFull, pki, o);
    if (lane >= o) pki += y;
  }
  unsigned base = 0;
  if (lane == 31 && pki) {
    const unsigned bl = (pki & 0xffffu) ? (unsigned)atomicAdd(&cnt[0], (int)(pki & 0xffffu)) : 0u;
    const unsigned bh = (pki >> 16) ? (unsigned)atomicAdd(&cnt[1], (int)(pki >> 16)) : 0u;
    base = bl | (bh << 16);
  }
  base = __shfl_sync(kFull, base, 31);
  if (pk) {
    unsigned ol = (base & 0xffffu) + ((pki - pk) & 0xffffu), oh = (base >> 16) + ((pki - pk) >> 16);
#pragma unroll
    for (int t = 0; t < PER; ++t) {
      const unsigned d = (unsigned)(v[t] >> sh) & dmask;
      if (t < tv && d == blo) reg_lo[ol++] = v[t];
      else if (t < tv && !same && d == bhi) reg_hi[oh++] = v[t];
    }
  }
  __syncthreads();
  stamp(2);
  // exact rank inside a bin
  const W sub = (W)dmask << sh;
  W res[2] = {plo, phi};
  for (int q = (rlo >= 0 ? 0 : 1); q < 2; ++q) {
    const W* reg = q ? reg_hi : reg_lo;
    const int m = q ? m_hi : m_lo;
    int rk = q ? rk_hi : rk_lo;
    if (m <= kBrute) {
      // rank of each of the m <= 128 bin members by counting: 8 threads per member, each over every
      // 8th member, summed over the 8-lane group (m / 8 loads per thread instead of m)
      const int e = (int)threadIdx.x >> 3, part = (int)threadIdx.x & 7;
      const W x = (e < m) ? reg[e] : (W)0;
      int less = 0, eq = 0;
      if (e < m) {
        for (int j = part; j < m; j += 8) {
          const W u = reg[j];
          less += u < x;
          eq += u == x;
        }
      }
#pragma unroll
      for (int o = 1; o < 8; o <<= 1) {
        less += __shfl_xor_sync(kFull, less, o);
        eq += __shfl_xor_sync(kFull, eq, o);
      }
      if (e < m && part == 0 && less <= rk && rk < less + eq) shw[4 + q] = x;
      __syncthreads();
      res[q] = shw[4 + q];
    } else {
      W pre = res[q], msk = mask | sub;
      select_digits<W>(reg, m, rk, pre, msk, sh, 0, hist, shw + 6);
      res[q] = pre;
    }
    stamp(3 + q);
  }
  lo = res[0];
  hi = res[1];
}

#ifndef AIRTOPK_SAMPLE_LEAN
#define AIRTOPK_SAMPLE_LEAN 1
#endif
// shared scratch of sample_rank (aliases the sample kernel's histogram array)
template <typename W>
struct SampleRankShared {
  unsigned hist[kMaxBins];
  W brute[kRankBrute];
  unsigned long long tmp[32];
  ScanResult res;
  W result;
  unsigned cnt;
};

constexpr int kSampleCTAs = 16;  // max CTAs per row issuing the scattered sample loads (one SM cannot
                                 // keep 16K independent DRAM loads in flight)

// ONE: one CTA per row (cps == 1; batches) — the samples stay in registers between the phases (a
// separate instantiation: keeping them live in the multi-CTA variant costs it register spills)
template <int KIND, bool ONE>
__global__ void __launch_bounds__(kSampleBlock) sample_kernel(const GridParams p, int nsamp, int cps) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  extern __shared__ __align__(16) unsigned char sample_smem[];
  W* scratch = (W*)sample_smem;  // nsamp entries: compacted bins of the rank selection (last CTA)
  __shared__ __align__(16) unsigned hist[2048 * kSampleHistCopies];
  __shared__ unsigned wsum[32];
  __shared__ W shw[8];
  __shared__ int sh_cnt[4];
  __shared__ W sh_red[64];
  __shared__ int sh_last;
  const int64_t row = blockIdx.x / cps;
  const int part = blockIdx.x % cps;
  RowState* st = p.st + row;
  // debug timing (trace slot 15 of the row): t0 start, t1 after pdl_wait, t2 ticket won, t3 codes in
  // smem, t4 selection done
  auto stamp = [&](int f) {
    if (p.trace && threadIdx.x == 0) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      p.trace[((size_t)row * kTraceMaxPasses + (kTraceMaxPasses - 1)) * kTraceFields + f] = (int64_t)t;
    }
  };
  if (part == 0) stamp(0);
  pdl_wait();
  if (part == 0) stamp(1);
  pdl_trigger();
  const U* rowp = (const U*)p.keys + row * p.len;
  W* samp = (W*)p.samp + row * (int64_t)nsamp;
  const U xmask = p.sel_min ? (U)0 : (U)~(U)0;
  // Samples come in runs of kRun consecutive elements (one 128-byte line for f32) at nsamp/kRun
  // stratified positions: a DRAM line is fetched whole anyway, so this costs nsamp*4 bytes of traffic
  // instead of nsamp*128. (Runs are independent draws for i.i.d. data; a row whose order defeats the
  // estimate only triggers the fallback.)
#ifndef AIRTOPK_SAMPLE_RUN
#define AIRTOPK_SAMPLE_RUN 32
#endif
  constexpr int kRun = AIRTOPK_SAMPLE_RUN;  // (A/B: longer runs touch fewer pages of a long row)
  const int nruns = nsamp / kRun;
  const int64_t stride = p.len / nruns;
  // phase 1: this CTA's runs part, part + cps, ... (all loads in flight at once)
  constexpr int PER = kMaxSamples / kSampleBlock;
  W v[PER];  // phase 2: sample t * kSampleBlock + tid (valid for t < tv)
  {
    const int runs_here = (nruns - part + cps - 1) / cps;  // runs part, part + cps, ...
    const int tmax = (runs_here * kRun + kSampleBlock - 1) / kSampleBlock;
    U x[PER];
#pragma unroll
    for (int t = 0; t < PER; ++t) {
      const int slot = t * kSampleBlock + threadIdx.x;  // (run-in-part, lane)
      const int run = (slot / kRun) * cps + part, e = slot % kRun;
      const int64_t pos = (int64_t)run * stride + (stride - kRun) / 2 + e;
      if (t < tmax && run < nruns && pos < p.len) x[t] = __ldg(rowp + pos);
    }
#pragma unroll
    for (int t = 0; t < PER; ++t) {
      const int slot = t * kSampleBlock + threadIdx.x;
      const int run = (slot / kRun) * cps + part, e = slot % kRun;
      const int64_t pos = (int64_t)run * stride + (stride - kRun) / 2 + e;
      const bool ok = t < tmax && run < nruns && pos < p.len;
      const W code = ok ? (W)to_code_x<KIND>(x[t], xmask) : (W)0;
      if (ONE) v[t] = code;  // one CTA per row: sample slot == run * kRun + e, kept in registers
      else if (ok) samp[run * kRun + e] = code;
    }
  }
  if (!ONE) {
    __syncthreads();
    if (threadIdx.x == 0) sh_last = (ticket_arrive(&st->ticket) == (unsigned)(cps - 1));
    __syncthreads();
    if (!sh_last) return;
  }
  stamp(2);
  // phase 2 (last CTA of the row): the window from the sample order statistics; the samples stay
  // in registers (16 per thread)
  const int tv = (nsamp - (int)threadIdx.x + kSampleBlock - 1) / kSampleBlock;  // valid v[t]: t < tv
  if (!ONE) {
#pragma unroll
    for (int t = 0; t < PER; ++t) v[t] = (t < tv) ? __ldcg(samp + t * kSampleBlock + threadIdx.x) : (W)0;
  }
  {
    W lmin = ~(W)0, lmax = 0;
#pragma unroll
    for (int t = 0; t < PER; ++t) {
      if (t < tv) {
        lmin = v[t] < lmin ? v[t] : lmin;
        lmax = v[t] > lmax ? v[t] : lmax;
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const W x = shfl(lmin, (threadIdx.x + o) & 31), y = shfl(lmax, (threadIdx.x + o) & 31);
      lmin = x < lmin ? x : lmin;
      lmax = y > lmax ? y : lmax;
    }
    if ((threadIdx.x & 31) == 0) {
      sh_red[threadIdx.x >> 5] = lmin;
      sh_red[32 + (threadIdx.x >> 5)] = lmax;
    }
    if (threadIdx.x == 0) sh_cnt[2] = 0;
  }
  __syncthreads();
  stamp(3);
  if (threadIdx.x == 0) st->ticket = 0;
  // expected sample rank of the K-th key and a 4-sigma (+8) margin of the binomial sample count
  // (measured sample counts are somewhat over-dispersed): a miss only costs the fallback, never
  // exactness
  const double f = (double)p.k / (double)p.len;
  const double r = f * nsamp;
  const double m = 4.0 * sqrt(r * (1.0 - f)) + 8.0;
  const int rlo = (int)floor(r - m), rhi = (int)ceil(r + m);
  if (rhi >= nsamp - 1) {  // the window would hold most of the row: keep the paper's passes
    if (threadIdx.x == 0) st->win_state = 0;
    return;
  }
  W smin = sh_red[0], smax = sh_red[32];
#pragma unroll 8
  for (int i = 1; i < kSampleBlock / 32; ++i) {
    smin = sh_red[i] < smin ? sh_red[i] : smin;
    smax = sh_red[32 + i] > smax ? sh_red[32 + i] : smax;
  }
  const W diff = smin ^ smax;
  const int hb = diff ? (8 * (int)sizeof(W) - (sizeof(W) == 8 ? __clzll((long long)diff) : __clz((int)diff))) : 0;
  stamp(5);
  // no results below the window when rlo <= 0: everything up to hi is a candidate
  W lo, hi;
#if AIRTOPK_SAMPLE_LEAN
  // the samples into shared memory, then the lean rank selection (finish.cuh: MSD digit histograms,
  // counting rank once <= 1024 samples share the prefix; measured ~2x faster than the register
  // version below, whose unrolled code runs once per select on a cold instruction cache)
  (void)hb;
#pragma unroll
  for (int t = 0; t < PER; ++t)
    if (t < tv) scratch[t * kSampleBlock + threadIdx.x] = v[t];
  __syncthreads();
  hi = sample_rank<W, kSampleBlock>(scratch, nsamp, rhi, smin, smax, *(SampleRankShared<W>*)hist);
  lo = rlo > 0 ? sample_rank<W, kSampleBlock>(scratch, nsamp, rlo, smin, smax, *(SampleRankShared<W>*)hist) : (W)0;
#else
  block_select_two<W, PER>(v, tv, scratch, rlo <= 0 ? -1 : rlo, rhi, smin, hb, hist, wsum, shw, sh_cnt, lo, hi);
  if (rlo <= 0) lo = 0;
#endif
  stamp(6);
  // Estimated window size from the sample (ties at hi included): a window that would overflow the
  // candidate buffer (e.g. a row of equal keys) is not tried — the paper's passes run instead.
  {
    unsigned le = 0;
#pragma unroll
    for (int t = 0; t < PER; ++t) le += (t < tv) && v[t] <= hi && v[t] >= lo;
    le = __reduce_add_sync(kFull, le);
    if ((threadIdx.x & 31) == 0 && le) atomicAdd(&sh_cnt[2], (int)le);
    __syncthreads();
    const double est = (double)sh_cnt[2] / nsamp * (double)p.len;
    if (est > 0.5 * (double)p.cap_rule) {
      if (threadIdx.x == 0) st->win_state = 0;
      return;
    }
  }
  stamp(4);
  if (threadIdx.x == 0) {
    st->win_lo = lo;
    st->win_hi = hi;
    st->win_state = 1;
  }
}

// Launch with programmatic stream serialisation (PDL): the kernel may start while the previous one
// drains; it synchronises with pdl_wait() before touching anything the previous kernel wrote.
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, args...);
}

struct Events {
  void* const* ev;
  int n;
  void record(int i, cudaStream_t s) const {
    if (ev && i < n) cudaEventRecord((cudaEvent_t)ev[i], s);
  }
};

template <int KIND, typename IdxT, int DF, int DH, bool TMA = false>
constexpr size_t hist_smem_bytes() {
  static_assert(!(DF == 1 || DF == 2) || DH == 0 || (size_t)kHistSlots * 4 * pass_hc<KIND, IdxT, DF, TMA>() >=
                    (size_t)kSmallFinish * (sizeof(typename KT<KIND>::U) + sizeof(IdxT)), "small finish smem");
  constexpr int HC = pass_hc<KIND, IdxT, DF, TMA>();
  return TMA ? tma_smem_bytes<HC>() : (size_t)kHistSlots * 4 * HC;
}

template <int KIND, typename IdxT, int DF, int DH, bool HASIDX, bool TMA>
cudaError_t launch_one(const GridParams& gp, unsigned grid, int q, int redo, cudaStream_t s) {
  constexpr size_t smem = hist_smem_bytes<KIND, IdxT, DF, DH, TMA>();
  const cudaError_t attr = func_attr(pass_kernel<KIND, IdxT, DF, DH, HASIDX, TMA>,
                                     cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (attr != cudaSuccess) return attr;
  return launch_pdl(pass_kernel<KIND, IdxT, DF, DH, HASIDX, TMA>, dim3(grid), dim3(kBlock), smem, s, gp, q, redo);
}

// one filter pass q >= 1 of variant v = DF * 3 + DH
template <int KIND, typename IdxT, bool HASIDX, bool TMA>
cudaError_t launch_grid_pass(const GridParams& gp, unsigned grid, int q, int v, cudaStream_t s) {
  switch (v) {
    case 1 * 3 + 1: return launch_one<KIND, IdxT, 1, 1, HASIDX, TMA>(gp, grid, q, 0, s);
    case 1 * 3 + 2: return launch_one<KIND, IdxT, 1, 2, HASIDX, TMA>(gp, grid, q, 0, s);
    case 2 * 3 + 2: return launch_one<KIND, IdxT, 2, 2, HASIDX, TMA>(gp, grid, q, 0, s);
    case 2 * 3 + 0: return launch_one<KIND, IdxT, 2, 0, HASIDX, TMA>(gp, grid, q, 0, s);
    default: return cudaErrorInvalidValue;
  }
}

template <int KIND, typename IdxT, bool HASIDX, bool TMA = false>
cudaError_t launch_grid_passes(const GridParams& gp, int64_t batch, int nsamp, const Events& ev, cudaStream_t s,
                               int upto = 1 << 30) {
  const unsigned grid = (unsigned)((long long)batch * gp.cpr);
  int ie = 0;
  ev.record(ie++, s);
  if (nsamp > 0) {  // sample-guided window: sample, window pass (= pass 0 + filter), pass 0 over the window
    using W = std::conditional_t<sizeof(typename KT<KIND>::U) == 8, unsigned long long, unsigned>;
    const size_t smem = (size_t)kMaxSamples * 4;  // 8-byte keys: nsamp <= kMaxSamples / 2
    const cudaError_t attr =
        func_attr(sample_kernel<KIND, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const cudaError_t attr1 =
        func_attr(sample_kernel<KIND, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (attr != cudaSuccess) return attr;
    if (attr1 != cudaSuccess) return attr1;
    // CTAs per row: enough to spread a few rows' scattered loads over the SMs; one per row for
    // batches (each CTA then keeps up to 16 loads per thread in flight)
    const int cps = (int)std::max<int64_t>(1, std::min<int64_t>(kSampleCTAs, gp.nsms / batch));
    cudaError_t es = (cps == 1)
        ? launch_pdl(sample_kernel<KIND, true>, dim3((unsigned)batch), dim3(kSampleBlock), (size_t)nsamp * sizeof(W),
                     s, gp, nsamp, cps)
        : launch_pdl(sample_kernel<KIND, false>, dim3((unsigned)(batch * cps)), dim3(kSampleBlock),
                     (size_t)nsamp * sizeof(W), s, gp, nsamp, cps);
    if (es != cudaSuccess) return es;
    ev.record(ie++, s);
    cudaError_t e = launch_one<KIND, IdxT, 3, 0, HASIDX, TMA>(gp, grid, 0, 0, s);
    if (e != cudaSuccess) return e;
    ev.record(ie++, s);
  }
  for (int q = 0; q <= gp.P && q < upto; ++q) {
    const int DF = q == 0 ? 0 : (digit_of(q - 1, KT<KIND>::R, gp.IB).is_idx ? 2 : 1);
    const int DH = q == gp.P ? 0 : (digit_of(q, KT<KIND>::R, gp.IB).is_idx ? 2 : 1);
    const int v = DF * 3 + DH;
    cudaError_t e;
    const int redo = (q == 0 && nsamp > 0) ? 1 : 0;
    if (TMA && nsamp > 0 && q >= 1) {  // window mode: the passes after it read the window buffer
      GridParams gb = gp;
      gb.cpr = gp.cpr_buf;
      e = launch_grid_pass<KIND, IdxT, HASIDX, false>(gb, (unsigned)((long long)batch * gb.cpr), q, v, s);
      if (e != cudaSuccess) return e;
      ev.record(ie++, s);
      continue;
    }
    switch (v) {
      case 0 * 3 + 1: e = launch_one<KIND, IdxT, 0, 1, HASIDX, TMA>(gp, grid, q, redo, s); break;
      case 1 * 3 + 1: e = launch_one<KIND, IdxT, 1, 1, HASIDX, TMA>(gp, grid, q, 0, s); break;
      case 1 * 3 + 2: e = launch_one<KIND, IdxT, 1, 2, HASIDX, TMA>(gp, grid, q, 0, s); break;
      case 2 * 3 + 2: e = launch_one<KIND, IdxT, 2, 2, HASIDX, TMA>(gp, grid, q, 0, s); break;
      case 2 * 3 + 0: e = launch_one<KIND, IdxT, 2, 0, HASIDX, TMA>(gp, grid, q, 0, s); break;
      default: return cudaErrorInvalidValue;
    }
    if (e != cudaSuccess) return e;
    ev.record(ie++, s);
  }
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------------------------
// Fused tail (batch 1): every pass after the window pass — or, when the window missed or there was
// none, every pass of the paper from L — in ONE cooperative launch. The per-pass kernel boundary of
// Algorithm 1 and its last-CTA scan become a grid-wide barrier after which EVERY
// CTA scans the merged histogram itself (identical j, K, C everywhere; no second barrier), so a
// pass over a small candidate buffer costs a barrier instead of a launch (measured: the passes
// after the c4 window pass took ~58 us as 6 launches). Histograms rotate over 3 global slots (slot
// (q+2) % 3 is zeroed during pass q: every CTA finished scanning it before the barrier of pass q);
// the buffer counts are per pass (zeroed with the row state).
struct TailState {
  unsigned long long K, C, tcode, tidx, nbuf;
  int src1;   // 0 = input row L, s + 1 = candidate buffer slot s
  int stop1;  // 1 + digit after whose scan K == C (early stop); 0 = none
  int ident;  // the last scan put every candidate into the target bin (C unchanged): the next filter
              // is the identity, so a buffer-source pass only histograms its next digit (no copy)
};

template <int KIND, typename IdxT, int DF, int DH>
__device__ __forceinline__ bool tail_pass(const GridParams& p, int q, TailState& S, unsigned* sh_hist,
                                          WarpQ<typename KT<KIND>::U, IdxT>* wq, unsigned long long* sh_tmp,
                                          ScanResult* sh_res) {
  namespace cg = cooperative_groups;
  using U = typename KT<KIND>::U;
  using CountT = std::conditional_t<sizeof(IdxT) == 8, unsigned long long, unsigned>;
  constexpr bool FILTER = (DF == 1 || DF == 2);
  const int tid = threadIdx.x;
  RowState* st = p.st;
  PassCtx<U, IdxT> c;
  c.q = q;
  c.emit_all = FILTER && ((S.stop1 != 0 && S.stop1 - 1 == q - 1) || DH == 0);
  c.do_hist = (DH != 0) && !c.emit_all;
  // DF == 0 over a candidate buffer: identity-filter elision (S.ident) — histogram digit q of the
  // buffer as it stands; nothing is emitted or stored
  const unsigned long long Cin = (FILTER || S.src1 > 0) ? S.C : (unsigned long long)p.len;
  c.srcL = (S.src1 == 0);
  c.store = c.do_hist && FILTER && (Cin <= (unsigned long long)p.cap_rule);  // Alg1 L17
  c.sel_min = p.sel_min != 0;
  c.reverse = (q & 1) != 0;
  c.dh = digit_of(q, KT<KIND>::R, p.IB);
  c.dh2 = c.dh;
  c.df = digit_of(FILTER ? q - 1 : 0, KT<KIND>::R, p.IB);
  c.tcode = S.tcode;
  c.tidx = S.tidx;
  c.wnmin = nullptr;
  c.wmax = nullptr;
  c.lo = 0;
  c.span1 = 0;
  c.rowp = (const U*)p.keys;
  c.rowi = nullptr;
  c.len = p.len;
  c.slice = blockIdx.x;
  c.nslices = gridDim.x;
  const int islot = S.src1 > 0 ? S.src1 - 1 : 0;
  const int sslot = (S.src1 == 1) ? 1 : 0;  // the buffer this pass writes
  c.bcin = (const U*)p.bcode + (size_t)islot * p.cap_alloc;
  c.biin = (const IdxT*)p.bidx + (size_t)islot * p.cap_alloc;
  c.nbuf = S.src1 > 0 ? S.nbuf : 0ull;
  c.ov = (U*)p.out_vals;
  c.oi = p.out_idx;
  c.ioff = p.idx_off;
  c.outc = &st->out_count;
  c.kk = (unsigned long long)p.k;
  c.bco = (U*)p.bcode + (size_t)sslot * p.cap_alloc;
  c.bio = (IdxT*)p.bidx + (size_t)sslot * p.cap_alloc;
  c.bufc = p.tcnt + q;
  c.capa = (unsigned long long)p.cap_alloc;
  c.err = &st->error;
  c.hist = sh_hist;
  c.ring = 0;
  c.wq = &wq[tid >> 5];
  c.dbg = (p.tstamp && q < 16) ? p.tstamp + 64 + q * 4 : nullptr;  // debug: run_pass internals
  if constexpr (FILTER && DH != 0) {
    // small finish: one CTA ends the row; the decision is grid-uniform
    if (!c.emit_all && !c.srcL && c.nbuf <= (unsigned long long)p.small_finish) {
      if (blockIdx.x == 0)
        small_finish<KIND, IdxT, kBlock>(c, S.K, (U*)sh_hist, (IdxT*)((unsigned char*)sh_hist + kSmallFinish * sizeof(U)));
      return true;
    }
  }
  constexpr int HC = hist_copies<KIND, IdxT, DF>();
  if (c.do_hist || DF == 0) {
    for (int i = tid; i < kHistSlots * HC; i += kBlock) sh_hist[i] = 0;
    __syncthreads();
  }
  auto tst = [&](int f) {
    if (p.tstamp && blockIdx.x == 0 && tid == 0 && q < 16) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      p.tstamp[q * 4 + f] = (int64_t)t;
    }
  };
  tst(0);
  run_pass<KIND, IdxT, DF, DH, false, kBlock, 0, false, kGridBU>(c);
  tst(1);
  if (!(c.do_hist || DF == 0)) return true;  // emit-all pass: the row is complete
  __syncthreads();
  CountT* gh = (CountT*)p.thist + (size_t)(q % 3) * kMaxBins;
  const int nb = 1 << c.dh.width;
  for (int i = tid; i < nb; i += kBlock) {
    unsigned v = 0;
#pragma unroll
    for (int h = 0; h < HC; ++h) v += sh_hist[i * HC + h];
    if (v) atomicAdd(&gh[i], (CountT)v);
  }
  cg::this_grid().sync();  // every CTA's histogram, results and candidates of pass q are published
  tst(2);
  const ScanResult r = scan_choose<kBlock>([&](int b) { return (unsigned long long)__ldcg(&gh[b]); }, nb, S.K, sh_tmp,
                                           sh_res);
  tst(3);
  if (blockIdx.x == 0) {
    CountT* gz = (CountT*)p.thist + (size_t)((q + 2) % 3) * kMaxBins;
    for (int i = tid; i < kMaxBins; i += kBlock) gz[i] = 0;
  }
  const unsigned long long newK = S.K - r.before, newC = r.cnt;  // Alg1 L26-28
  if (c.store) {
    S.src1 = sslot + 1;
    S.nbuf = Cin;  // every candidate of the filter was stored: hist[j] of the previous scan (no L2 read)
  }
  S.ident = (newC == Cin) ? 1 : 0;
  S.C = newC;
  S.K = newK;
  if (!c.dh.is_idx) S.tcode |= (unsigned long long)r.j << c.dh.shift;
  else S.tidx |= (unsigned long long)r.j << c.dh.shift;
  if (newK == newC && p.early_stop == 0) S.stop1 = q + 1;  // early stop
  if (blockIdx.x == 0 && tid == 0) {
    st->K = newK;
    st->C = newC;
    st->Cp = Cin;
    st->tcode = S.tcode;
    st->tidx = S.tidx;
    st->j = r.j;
    st->npass = q + 1;
    st->stop1 = S.stop1;
    st->src1 = S.src1;
    if (r.total != Cin) st->error |= 4u;
  }
  return false;
}

template <int KIND, typename IdxT>
__global__ void __launch_bounds__(kBlock, kMinBlocksFilter) tail_kernel(const GridParams p) {
  using U = typename KT<KIND>::U;
  extern __shared__ unsigned sh_hist[];
  __shared__ WarpQ<U, IdxT> sh_wq[kWarps];
  __shared__ unsigned long long sh_tmp[kWarps];
  __shared__ ScanResult sh_res;
  pdl_wait();     // the window pass (previous launch) is complete
  pdl_trigger();  // the next select's first launch may be scheduled (it waits for our completion)
  const RowState* st = p.st;
  TailState S;
  int q;
  if (st->win_state == 1) {  // continue after the window pass (its scan fixed digits < npass)
    q = st->npass;
    S.K = st->K;
    S.C = st->C;
    S.tcode = st->tcode;
    S.tidx = st->tidx;
    S.src1 = st->src1;
    S.stop1 = st->stop1;
    S.nbuf = S.src1 > 0 ? st->buf_count[S.src1 - 1] : 0ull;
    S.ident = (st->C == st->Cp) ? 1 : 0;  // the window scan kept every member (e.g. c4: digit 1 is one bin)
  } else {  // no window / the window missed: the paper's passes from L
    q = 0;
    S.K = (unsigned long long)p.k;
    S.C = (unsigned long long)p.len;
    S.tcode = S.tidx = 0;
    S.src1 = 0;
    S.stop1 = 0;
    S.nbuf = 0;
    S.ident = 0;
  }
#pragma unroll 1
  for (; q <= p.P; ++q) {
    if (S.stop1 != 0 && S.stop1 - 1 < q - 1) break;
    const int DF = q == 0 ? 0 : (digit_of(q - 1, KT<KIND>::R, p.IB).is_idx ? 2 : 1);
    const int DH = q == p.P ? 0 : (digit_of(q, KT<KIND>::R, p.IB).is_idx ? 2 : 1);
    bool done;
    // identity-filter elision: after a scan that kept every candidate (S.ident), a pass over a buffer
    // that would filter a key digit and histogram the next key digit only histograms (no emit, no copy)
    const bool ident = kTailIdent && S.ident && S.src1 > 0 && DF == 1 && DH == 1 &&
                       !(S.stop1 != 0 && S.stop1 - 1 == q - 1);
    switch (ident ? 0 * 3 + 1 : DF * 3 + DH) {
      case 0 * 3 + 1: done = tail_pass<KIND, IdxT, 0, 1>(p, q, S, sh_hist, sh_wq, sh_tmp, &sh_res); break;
      case 1 * 3 + 1: done = tail_pass<KIND, IdxT, 1, 1>(p, q, S, sh_hist, sh_wq, sh_tmp, &sh_res); break;
      case 1 * 3 + 2: done = tail_pass<KIND, IdxT, 1, 2>(p, q, S, sh_hist, sh_wq, sh_tmp, &sh_res); break;
      case 2 * 3 + 2: done = tail_pass<KIND, IdxT, 2, 2>(p, q, S, sh_hist, sh_wq, sh_tmp, &sh_res); break;
      default: done = tail_pass<KIND, IdxT, 2, 0>(p, q, S, sh_hist, sh_wq, sh_tmp, &sh_res); break;
    }
    if (done) break;
  }
}

template <int KIND, typename IdxT>
cudaError_t launch_tail(const GridParams& gp, cudaStream_t s) {
  auto kern = tail_kernel<KIND, IdxT>;
  constexpr size_t smem = (size_t)kHistSlots * 4 * kHistCopies;
  static_assert((size_t)kHistSlots * 4 * kHistCopies >= (size_t)kSmallFinish * (sizeof(typename KT<KIND>::U) + sizeof(IdxT)),
                "small finish smem");
  cudaError_t e = func_attr(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int occ = 0;
  if (!occ_cache_get((const void*)kern, 0, &occ)) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBlock, smem);
    if (e != cudaSuccess) return e;
    occ_cache_put((const void*)kern, 0, occ);
  }
  if (occ < 1) return cudaErrorInvalidConfiguration;
  cudaLaunchConfig_t cfg = {};
  int G = gp.nsms * std::min(occ, kMinBlocksFilter);
  if (const char* env = getenv("AIRTOPK_TAIL_CTAS")) G = std::min(G, std::max(1, atoi(env)));  // A/B knob
  cfg.gridDim = dim3((unsigned)G);
  cfg.blockDim = dim3(kBlock);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, gp);
}

template <int KIND>
cudaError_t launch_cluster_kind(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s, int tail);

// Grid engine. With pl.tail the rows are finished after the window pass by ONE cluster-engine launch
// over the (small) window buffers instead of P+1 grid launches.
template <int KIND>
cudaError_t launch_grid_kind(const SelectArgs& a, const Plan& pl, const GridParams& gp, void* ws, cudaStream_t s) {
  const Events ev{a.events, a.n_events};
  if (a.in_idx) return launch_grid_passes<KIND, uint64_t, true>(gp, a.batch, 0, ev, s);
  cudaError_t e;
  if (pl.fused) {  // sample + window pass, then ONE cooperative launch for every remaining pass
    e = pl.idx64 ? launch_grid_passes<KIND, uint64_t, false>(gp, a.batch, pl.nsamp, ev, s, 0)
        : pl.tma ? launch_grid_passes<KIND, uint32_t, false, true>(gp, a.batch, pl.nsamp, ev, s, 0)
                 : launch_grid_passes<KIND, uint32_t, false>(gp, a.batch, pl.nsamp, ev, s, 0);
    if (e != cudaSuccess) return e;
    e = pl.idx64 ? launch_tail<KIND, uint64_t>(gp, s) : launch_tail<KIND, uint32_t>(gp, s);
    ev.record(pl.nsamp > 0 ? 3 : 1, s);
    return e;
  }
  const int upto = pl.tail ? pl.tail_q : (1 << 30);
  if (pl.idx64) e = launch_grid_passes<KIND, uint64_t, false>(gp, a.batch, pl.nsamp, ev, s, upto);
  else if (pl.tma) e = launch_grid_passes<KIND, uint32_t, false, true>(gp, a.batch, pl.nsamp, ev, s, upto);
  else e = launch_grid_passes<KIND, uint32_t, false>(gp, a.batch, pl.nsamp, ev, s, upto);
  if (e != cudaSuccess || !pl.tail) return e;
  e = launch_cluster_kind<KIND>(a, pl, ws, s, 1);
  ev.record(3 + pl.tail_q, s);
  return e;
}

#define AIRTOPK_INSTANTIATE_GRID(KIND) \
  template cudaError_t launch_grid_kind<KIND>(const SelectArgs&, const Plan&, const GridParams&, void*, cudaStream_t);

}  // namespace airtopk
