// engine_batch.cuh — the batched engine: a whole batch of rows in ONE persistent cooperative launch.
//
// SURVEY §8(a) a8 ("batched / small-row path", P:235 batches of rows with the same N and K; P:250-252
// batch 100 gave the largest speedups) combined with the sample-guided window (§8(f) NEXT #1
// SampleSelect-style pivots) so every row is read from HBM exactly once. The grid engine runs a
// batch as sample kernel + window pass + a cluster tail: three launches, the window pass quantised
// into ~2.7 waves of row-sized CTA groups (c2: 0.50 of the roofline). Here one CTA per
// SM (1024 threads) loops over three phases separated by grid-wide barriers (cooperative launch):
//
//   A  sample: CTA r (rows r, r + G, ...) draws S stratified runs of 32 keys of its row, selects the
//      sample order statistics around the expected rank of the K-th key and stores the window
//      [lo, hi] (the same estimator and 4-sigma+8 margin as sample_kernel) by MSD digit histograms
//      of the samples and a counting rank once <= 1024 candidates remain.
//   B  stream: the batch is cut into 32 KiB chunks, chunk c -> CTA c mod G (grid-stride over the
//      flattened batch: no wave quantisation, every SM streams ~equal bytes; the CTAs stream one
//      compact advancing region of HBM). Each CTA pulls its chunks through a ring of 6 bulk-copy
//      stages (cp.async.bulk, TMA engine, mbarrier full/empty handshake: 192 KiB in flight per SM,
//      the first 4 issued before phase A). Per element ONE compare of the raw key bits against the
//      transformed threshold hi (exact); the rare flagged keys (code <= hi) are written by their
//      warp to the FIXED slot of the chunk at an offset from ONE shared atomic per flagged warp —
//      no global atomics, no queues, no block barriers in the streaming loop — and the group
//      leader stores the slot's count once the group released the stage.
//   C  finish: CTA r gathers its row's slots (prefix sum over the slot counts) into shared memory
//      and registers, checks that the window holds the K-th key (R < K <= R + W, R = #codes < lo,
//      W = #members), emits the R results, then selects the K - R smallest members by radix passes
//      over the composite key (code || row index: lowest-index ties, reading 1) on the
//      register-resident entries: per pass a 2048-bin shared histogram, the inclusive scan and the
//      target digit j with psum[j-1] < K <= psum[j] (Alg1 L24-28), filter (digit < j ->
//      result, == j -> candidate), early stop when K == C.
//
// Code size matters here: phases A and C run once per row on a cold instruction cache (measured:
// fully unrolled register-array versions spent ~10 us per phase fetching straight-line code), so
// their loops stay rolled and their data lives in shared memory.
//
// Exactness never depends on the sample: a row whose window misses (or overflows a slot or the
// finish capacity, or had no usable window) is marked win_state = 3 and the next, already enqueued,
// launch (the cluster engine in fallback mode, PDL) selects it from L with the paper's passes.
#pragma once

#include <cooperative_groups.h>

#include "device.cuh"
#include "engine.h"
#include "engine_grid.cuh"
#include "finish.cuh"
#include "tma.cuh"

namespace airtopk {

constexpr int kBBlock = kBatchBlock;          // threads per CTA (1 CTA per SM)
constexpr int kBWarps = kBBlock / 32;
static_assert(kBWarps == kBatchWarps, "host/device slot geometry");
constexpr unsigned kBStage = kBatchStage;     // bytes per bulk-copy ring stage = one chunk of a row
#ifndef AIRTOPK_BATCH_STAGES
#define AIRTOPK_BATCH_STAGES 8
#endif
constexpr int kBStages = AIRTOPK_BATCH_STAGES;
#ifndef AIRTOPK_BATCH_PDL
#define AIRTOPK_BATCH_PDL 0  // measured: no gain on c2 (the fallback launch already overlaps); off
#endif  // ring depth: 8 x 24 KiB = 192 KiB in flight per SM
constexpr int kBPre = 4;                      // stages issued before the sampling phase
#ifndef AIRTOPK_BATCH_L2PRE
#define AIRTOPK_BATCH_L2PRE 0  // measured: L2 prefetches during phase A slow the sampling, stream unchanged
#endif
constexpr int kBL2Pre = AIRTOPK_BATCH_L2PRE;  // further chunks per CTA prefetched into L2 during phase A
// Phase B consumers: four groups of 8 warps take the stages in turn, 6 vectors per thread each (a
// warp's per-stage overhead — barrier wait, count store, loop — is amortised over 3 KiB; measured on
// c2: 4 x 8 warps on 8 x 24 KiB stages stream at 6.6 TB/s, 2 x 16 on 6 x 32 KiB at 6.1, 1 x 32 on
// 6 x 32 KiB at 5.3).
constexpr int kBGroups = AIRTOPK_BATCH_GROUPS;
constexpr int kBGWarps = kBWarps / kBGroups;
constexpr int kBGThreads = kBGWarps * 32;
constexpr int kBVT = (int)(kBStage / 16 / kBGThreads);  // 16-byte vectors per thread per stage
static_assert(kBVT * 16 * kBGThreads == (int)kBStage, "stage = group threads x kBVT vectors");
static_assert(kBStages % kBGroups == 0, "a stage always belongs to the same group");
constexpr int kBFcap = kBatchFcap;            // entries (results + members) one row may stage in the finish
constexpr size_t kBRingBytes = (size_t)kBStages * kBStage;
static_assert((size_t)kMaxSamples * 4 <= (size_t)(kBStages - kBPre) * kBStage, "samples fit the unused stages");

struct BatchParams {
  const void* keys;
  int64_t batch, len, k;
  int sel_min;
  int IB;                 // index bits (lowest-index tie digits)
  void* out_vals;
  int64_t* out_idx;
  int64_t idx_off;
  RowState* st;
  unsigned short* cnt;    // [batch][nwc] entries written per chunk slot (cap + 1 = overflow)
  void* scode;            // [batch][nwc][scap] codes
  unsigned* sidx;         // [batch][nwc][scap] row indices
  int nwc;                // slots per row = chunks per row
  int scap;               // entries per slot
  int cpc;                // chunks per row
  int nsamp;              // samples per row
  int early_stop;         // 0 on, -1 off
  unsigned* fail;         // [0] = number of rows for the fallback launch, [1 + i] = those rows
  int64_t* timing;        // optional (trace buffer): per CTA globaltimer stamps of the phases
  int64_t timing_n;       // int64 entries of `timing`
};

// debug timing (trace buffer): per CTA 32 %globaltimer stamps (tools/batch_timing.py)
__device__ __forceinline__ void bstamp(const BatchParams& p, int f) {
  if (p.timing && threadIdx.x == 0 && (int64_t)blockIdx.x * 32 + f < p.timing_n) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    p.timing[(int64_t)blockIdx.x * 32 + f] = (int64_t)t;
  }
}

// Shared scratch of the sampling and finish phases (static; the big arrays live in the ring).
template <typename W>
struct BatchShared {
  unsigned hist[kMaxBins];
  W brute[kRankBrute];          // compacted candidates of the rank selection
  unsigned long long tmp[kBWarps];
  ScanResult res;
  W wmin[kBWarps], wmax[kBWarps];
  SelScratch<W, kBWarps> sel;   // finish: shared-memory radix select
  W result;
  unsigned long long tot;
  unsigned cnt, out;
  int bad;
};

// ---------------------------------------------------------------------------------- phase A
template <typename U>
__device__ __forceinline__ void batch_issue(const BatchParams& p, int64_t ch, unsigned ring, int stage);
template <typename U>
__device__ __forceinline__ void batch_prefetch_l2(const BatchParams& p, int64_t ch);

template <int KIND>
__device__ void batch_sample_row(const BatchParams& p, int64_t row, void* samp_v,
                                 BatchShared<std::conditional_t<sizeof(typename KT<KIND>::U) == 8, unsigned long long,
                                                                unsigned>>& sh,
                                 int64_t issue_mine, unsigned ring) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  W* s = (W*)samp_v;
  RowState* st = p.st + row;
  const int ns = p.nsamp;
  const U* rowp = (const U*)p.keys + row * p.len;
  const U xmask = p.sel_min ? (U)0 : (U)~(U)0;
  constexpr int kRun = 32;  // samples come in runs of 32 consecutive keys (one 128-byte line for f32)
  const int64_t stride = p.len / (ns / kRun);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  W lmin = ~(W)0, lmax = 0;
  // all of a thread's sample loads are issued before any is stored: `s` is a generic pointer the
  // compiler cannot prove disjoint from the row, so interleaved store / load pairs would serialise
  // one DRAM latency per sample (measured)
  constexpr int kSPT = kMaxSamples / kBBlock;  // samples per thread (<= 16)
  {
    U x[kSPT];
#pragma unroll
    for (int t = 0; t < kSPT; ++t) {
      const int i = threadIdx.x + t * kBBlock;
      x[t] = (i < ns) ? __ldg(rowp + (int64_t)(i / kRun) * stride + (stride - kRun) / 2 + (i % kRun)) : (U)0;
    }
#pragma unroll
    for (int t = 0; t < kSPT; ++t) {
      const int i = threadIdx.x + t * kBBlock;
      if (i < ns) {
        const W c = (W)to_code_x<KIND>(x[t], xmask);
        s[i] = c;
        lmin = c < lmin ? c : lmin;
        lmax = c > lmax ? c : lmax;
      }
    }
  }
  bstamp(p, 1);
  if (threadIdx.x == 0) {  // (the loads above have returned: their values are in lmin / lmax)
    for (int i = 0; i < kBPre && i < issue_mine; ++i) batch_issue<U>(p, blockIdx.x + (int64_t)i * gridDim.x, ring, i);
    for (int i = kBPre; i < kBPre + kBL2Pre && i < issue_mine; ++i)
      batch_prefetch_l2<U>(p, blockIdx.x + (int64_t)i * gridDim.x);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const W a = shfl(lmin, lane ^ o), b = shfl(lmax, lane ^ o);
    lmin = a < lmin ? a : lmin;
    lmax = b > lmax ? b : lmax;
  }
  if (lane == 0) {
    sh.wmin[warp] = lmin;
    sh.wmax[warp] = lmax;
  }
  __syncthreads();
  W smin = sh.wmin[lane], smax = sh.wmax[lane];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const W a = shfl(smin, lane ^ o), b = shfl(smax, lane ^ o);
    smin = a < smin ? a : smin;
    smax = b > smax ? b : smax;
  }
  // expected sample rank of the K-th key and a 4-sigma (+8) binomial margin (as sample_kernel):
  // a miss only costs the fallback, never exactness
  const double f = (double)p.k / (double)p.len;
  const double r = f * ns;
  const double m = 4.0 * sqrt(r * (1.0 - f)) + 8.0;
  const int rlo = (int)floor(r - m), rhi = (int)ceil(r + m);
  int state = 1;
  W lo = 0, hi = 0;
  if (rhi >= ns - 1) {
    state = 3;
  } else {
    hi = sample_rank<W, kBBlock>(s, ns, rhi, smin, smax, sh, [&](int f) { bstamp(p, 16 + f); });
    lo = rlo > 0 ? sample_rank<W, kBBlock>(s, ns, rlo, smin, smax, sh) : (W)0;  // none below the window if rlo <= 0
    bstamp(p, 2);
    // estimated entries (results + members: every code <= hi) vs the finish capacity
    unsigned le = 0;
#pragma unroll 4
    for (int i = threadIdx.x; i < ns; i += kBBlock) le += s[i] <= hi;
    le = __reduce_add_sync(kFull, le);
    if (threadIdx.x == 0) sh.cnt = 0;
    __syncthreads();
    if (lane == 0 && le) atomicAdd(&sh.cnt, le);
    __syncthreads();
    if ((double)sh.cnt / ns * (double)p.len > 0.6 * (double)kBFcap) state = 3;
  }
  if (threadIdx.x == 0) {
    st->win_lo = lo;
    st->win_hi = hi;
    st->win_state = state;
    st->out_count = 0;
    st->error = 0;
  }
  __syncthreads();
}

// ---------------------------------------------------------------------------------- phase B
// Threshold of the raw-bit test: code(b) <= hi  <=>  (b ^ wx) <= hi (see run_pass, DF == 3).
template <int KIND>
__device__ __forceinline__ std::conditional_t<sizeof(typename KT<KIND>::U) == 8, unsigned long long, unsigned>
raw_xor_for(unsigned long long hi, bool sel_min) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  constexpr W S = (W)((W)1 << (KT<KIND>::R - 1));
  constexpr W ones = (W)(U)~(U)0;  // (U) again: ~ promotes 16-bit keys to int
  const W whi = (W)hi;
  if constexpr (KT<KIND>::IEEE) {
    if (sel_min) return (whi >= S) ? S : ones;
    return (whi < S) ? (W)(ones ^ S) : (W)0;
  } else {
    return sel_min ? (W)0 : ones;
  }
}

// Chunk ch of the flattened batch into ring stage `stage` (thread 0).
// L2 prefetch of chunk ch (no shared memory involved): phase A lasts several microseconds during
// which HBM would idle; the chunks a CTA streams right after the ring's first stages are pulled
// into L2 meanwhile.
template <typename U>
__device__ __forceinline__ void batch_prefetch_l2(const BatchParams& p, int64_t ch) {
  const int64_t row = ch / p.cpc, ci = ch - row * p.cpc;
  const int64_t rb = p.len * (int64_t)sizeof(U);
  const unsigned bytes = (unsigned)min((int64_t)kBStage, rb - ci * (int64_t)kBStage);
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"((const char*)p.keys + row * rb + ci * (int64_t)kBStage),
               "r"(bytes)
               : "memory");
}

// The input is read exactly once: its L2 lines are marked evict-first so the chunk slots
// written meanwhile stay in L2 for the finish.
template <typename U>
__device__ __forceinline__ void batch_issue(const BatchParams& p, int64_t ch, unsigned ring, int stage) {
  const int64_t row = ch / p.cpc, ci = ch - row * p.cpc;
  const int64_t rb = p.len * (int64_t)sizeof(U);
  const unsigned bytes = (unsigned)min((int64_t)kBStage, rb - ci * (int64_t)kBStage);
  const unsigned fullb = ring + (unsigned)kBRingBytes + 8u * stage;
  mbar_arrive_expect_tx(fullb, bytes);
#ifndef AIRTOPK_BATCH_EVICT_FIRST
#define AIRTOPK_BATCH_EVICT_FIRST 1  // measured: without the hint the stream ends ~4 us later (c2)
#endif
  if (AIRTOPK_BATCH_EVICT_FIRST)
    bulk_g2s_hint(ring + stage * kBStage, (const char*)p.keys + row * rb + ci * (int64_t)kBStage, bytes, fullb,
                  l2_policy_evict_first());
  else
    bulk_g2s(ring + stage * kBStage, (const char*)p.keys + row * rb + ci * (int64_t)kBStage, bytes, fullb);
}

// Flag code <= hi among this thread's vectors of a stage (gt = thread index in its group, gw =
// warp in its group), write the warp's flagged keys to its slot. Fast path per element: one xor and
// one min of the raw bits; the flags are only built when the minimum hits (a few lanes per stage).
template <int KIND, bool FULL>
__device__ __forceinline__ void batch_classify(const BatchParams& p, int64_t row, int ci, unsigned long long hi,
                                               unsigned sbase, int nv, int gt, unsigned* scnt) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  constexpr int VEC = 16 / sizeof(U);
  using FlagT = std::conditional_t<(kBVT * VEC > 32), unsigned long long, unsigned>;
  const int lane = gt & 31;
  const bool sel_min = p.sel_min != 0;
  const W whi = (W)hi;
  const W wx = raw_xor_for<KIND>(hi, sel_min);
  uint4 r[kBVT];
#pragma unroll
  for (int u = 0; u < kBVT; ++u) r[u] = lds128(sbase + (unsigned)((gt + u * kBGThreads) * 16));
  W m = ~(W)0;
#pragma unroll
  for (int u = 0; u < kBVT; ++u) {
    const bool valid = FULL || gt + u * kBGThreads < nv;
#pragma unroll
    for (int e = 0; e < VEC; ++e) {
      const W t = (W)((W)vec_elem<U>(r[u], e) ^ wx);
      m = (valid && t < m) ? t : m;
    }
  }
  const size_t slot = (size_t)row * p.nwc + (size_t)ci;  // the chunk's slot (shared by the group's warps)
  if (__any_sync(kFull, m <= whi)) {
    FlagT fl = 0;
#pragma unroll
    for (int u = 0; u < kBVT; ++u) {
      const bool valid = FULL || gt + u * kBGThreads < nv;
#pragma unroll
      for (int e = 0; e < VEC; ++e)
        if (valid && (W)((W)vec_elem<U>(r[u], e) ^ wx) <= whi) fl |= (FlagT)1 << (u * VEC + e);
    }
    const int n = (sizeof(FlagT) == 8) ? __popcll((unsigned long long)fl) : __popc((unsigned)fl);
    int incl = n;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(kFull, incl, o);
      if (lane >= o) incl += y;
    }
    const int total = __shfl_sync(kFull, incl, 31);
    // the warp's range of the chunk slot: ONE shared atomic on the stage's counter (the group
    // leader stores the slot count once every warp of the group has released the stage)
    unsigned wb = 0;
    if (lane == 31) wb = atomicAdd(scnt, (unsigned)total);
    int pos = (int)__shfl_sync(kFull, wb, 31) + incl - n;
    U* sc = (U*)p.scode + slot * p.scap;
    unsigned* si = p.sidx + slot * p.scap;
    const U xmask = sel_min ? (U)0 : (U)~(U)0;
    const unsigned long long keep = l2_policy_evict_last();
#pragma unroll 1
    while (fl) {
      const int b = ((sizeof(FlagT) == 8) ? __ffsll((long long)fl) : __ffs((int)fl)) - 1;
      fl &= fl - 1;
      if (pos < p.scap) {
        const int u = b / VEC, e = b % VEC;
        const unsigned a = sbase + (unsigned)((gt + u * kBGThreads) * 16 + e * (int)sizeof(U));
        U raw;
        if constexpr (sizeof(U) == 2) { unsigned short t; asm volatile("ld.shared.u16 %0, [%1];" : "=h"(t) : "r"(a)); raw = t; }
        else if constexpr (sizeof(U) == 4) { unsigned t; asm volatile("ld.shared.u32 %0, [%1];" : "=r"(t) : "r"(a)); raw = t; }
        else { unsigned long long t; asm volatile("ld.shared.u64 %0, [%1];" : "=l"(t) : "r"(a)); raw = t; }
        st_keep(sc + pos, to_code_x<KIND>(raw, xmask), keep);
        st_keep(si + pos, (unsigned)((int64_t)ci * (kBStage / sizeof(U)) + (int64_t)(gt + u * kBGThreads) * VEC + e), keep);
      }
      ++pos;
    }
  }
}

// Group leader, after every warp of its group released the stage: store the chunk slot's count
// (cap + 1 = overflow) and pad the written entries to whole 32-byte sectors (a partially written
// L2 sector would have to be filled from DRAM when the finish reads it; measured ~7 us), then
// reset the stage's counter for its next chunk.
template <typename U>
__device__ __forceinline__ void batch_slot_done(const BatchParams& p, int64_t row, int ci, unsigned* scnt) {
  const unsigned c = *(volatile unsigned*)scnt;
  *scnt = 0;
  const size_t slot = (size_t)row * p.nwc + (size_t)ci;
  const unsigned long long keep = l2_policy_evict_last();
  constexpr int kSec = 32 / (sizeof(U) < 4 ? sizeof(U) : 4);
  const int padded = min(p.scap, ((int)c + kSec - 1) / kSec * kSec);
  U* sc = (U*)p.scode + slot * p.scap;
  unsigned* si = p.sidx + slot * p.scap;
  for (int q = (int)c; q < padded; ++q) {
    st_keep(sc + q, (U)0, keep);
    st_keep(si + q, 0u, keep);
  }
  st_keep(p.cnt + slot, (unsigned short)((int)c > p.scap ? p.scap + 1 : (int)c), keep);
}

// ---------------------------------------------------------------------------------- phase C
// One row (all threads): gather, check the window, emit results, select the members.
template <int KIND>
__device__ void batch_finish_row(const BatchParams& p, int64_t row, void* stage,
                                 BatchShared<std::conditional_t<sizeof(typename KT<KIND>::U) == 8, unsigned long long,
                                                                unsigned>>& sh, bool dry = false) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  constexpr int WB = 8 * (int)sizeof(W);
  constexpr int PER = kBFcap / kBBlock;
  static_assert(PER <= 32, "valid bits per thread");
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  RowState* st = p.st + row;
  auto fail = [&]() {  // the fallback launch selects the row from L (nothing was emitted)
    if (tid == 0) {
      st->win_state = 3;
      p.fail[1 + atomicAdd(p.fail, 1u)] = (unsigned)row;
    }
    __syncthreads();
  };
  if (st->win_state != 1) {  // (uniform) no usable window
    fail();
    return;
  }
  const W lo = (W)st->win_lo;
  bstamp(p, 20);
  U* stc = (U*)stage;
  unsigned* sti = (unsigned*)((char*)stage + (size_t)kBFcap * sizeof(U));
  // --- gather: warp w takes the contiguous slot range [w*spw, (w+1)*spw) (one chunk slot per
  // lane, coalesced counts), a warp scan places its slots' entries, ONE shared atomic per warp
  // reserves staging room (the order of entries is irrelevant to the selection), then the warp's
  // entries are loaded lane-parallel (entry e -> slot lane by a shuffle binary search over the
  // inclusive slot prefix): consecutive lanes read consecutive entries of a slot, and every load
  // of a batch is in flight before its stores (the staging pointer is generic: interleaved
  // stores would serialise the loads) ---
  const int nwc = p.nwc;
  const unsigned short* cnt = p.cnt + (size_t)row * nwc;
  if (tid == 0) {
    sh.cnt = 0;
    sh.bad = 0;
  }
  __syncthreads();
  bstamp(p, 21);
  constexpr int kGJ = 4;  // entries per lane per batch
  const int spw = (nwc + kBWarps - 1) / kBWarps;
  const int s_end = min(nwc, (warp + 1) * spw);
#pragma unroll 1
  for (int s0 = warp * spw; s0 < s_end; s0 += 32) {
    const int sl = s0 + lane;
    int cc = sl < s_end ? (int)__ldcg(cnt + sl) : 0;
    if (cc > p.scap) sh.bad = 1;
    cc = min(cc, p.scap);
    int incl = cc;
#pragma unroll
    for (int q = 1; q < 32; q <<= 1) {
      const int y = __shfl_up_sync(kFull, incl, q);
      if (lane >= q) incl += y;
    }
    const int all = __shfl_sync(kFull, incl, 31);
    unsigned b = 0;
    if (lane == 0 && all) b = atomicAdd(&sh.cnt, (unsigned)all);
    b = __shfl_sync(kFull, b, 0);
    bstamp(p, 22);
#pragma unroll 1
    for (int e0 = 0; e0 < all; e0 += 32 * kGJ) {
      U vc[kGJ];
      unsigned vi[kGJ];
#pragma unroll
      for (int t = 0; t < kGJ; ++t) {
        const int e = e0 + t * 32 + lane;
        int L = 0;  // number of slot lanes whose inclusive prefix is <= e: e's slot
#pragma unroll
        for (int h = 16; h > 0; h >>= 1)
          if (__shfl_sync(kFull, incl, L + h - 1) <= e) L += h;
        const int ex = __shfl_sync(kFull, incl - cc, L);
        if (e < all) {
          const size_t src = ((size_t)row * nwc + s0 + L) * p.scap + (e - ex);
          vc[t] = __ldcg((const U*)p.scode + src);
          vi[t] = __ldcg(p.sidx + src);
        }
      }
#pragma unroll
      for (int t = 0; t < kGJ; ++t) {
        const unsigned d = b + (unsigned)(e0 + t * 32 + lane);
        if (e0 + t * 32 + lane < all && d < (unsigned)kBFcap) {
          stc[d] = vc[t];
          sti[d] = vi[t];
        }
      }
    }
    bstamp(p, 23);
  }
  __syncthreads();
  bstamp(p, 7);
  if (dry) return;  // (debug: gather only)
  const int n = (int)sh.cnt;
  if (sh.bad || n > kBFcap || n < (int)p.k) {
    fail();  // slot overflow / too many entries / fewer than K keys up to hi
    return;
  }
  bstamp(p, 8);
  const int tcnt = (n + kBBlock - 1) / kBBlock;  // entry rounds (block-uniform)
  // --- window check: R < K <= R + W = n, R = #codes below lo ---
  unsigned nres = 0;
#pragma unroll 1
  for (int e = tid; e < n; e += kBBlock) nres += (W)stc[e] < lo;
  nres = __reduce_add_sync(kFull, nres);
  if (tid == 0) {
    sh.tot = 0;
    sh.out = 0;
  }
  __syncthreads();
  if (lane == 0 && nres) atomicAdd(&sh.tot, (unsigned long long)nres);
  __syncthreads();
  const unsigned long long R = sh.tot;
  const unsigned long long kk = (unsigned long long)p.k;
  bstamp(p, 9);
  if (!(R < kk && kk <= (unsigned long long)n)) {
    fail();
    return;
  }
  U* ov = (U*)p.out_vals + row * p.k;
  int64_t* oi = p.out_idx + row * p.k;
  const bool sel_min = p.sel_min != 0;
  auto emit = [&](bool pred, U code, unsigned idx) {  // warp-aggregated output slots
    const unsigned m = __ballot_sync(kFull, pred);
    if (!m) return;
    unsigned b = 0;
    if (lane == 0) b = atomicAdd(&sh.out, (unsigned)__popc(m));
    b = __shfl_sync(kFull, b, 0);
    if (pred) {
      const unsigned pos = b + __popc(m & lanemask_lt());
      ov[pos] = from_code<KIND>(code, sel_min);
      oi[pos] = (int64_t)idx + p.idx_off;
    }
  };
  // results (every code below the window) leave now; members stay live
  unsigned valid = 0;
#pragma unroll 1
  for (int t = 0, e = tid; t < tcnt; ++t, e += kBBlock) {
    const bool in = e < n;
    const U c = in ? stc[e] : (U)0;
    const bool isr = in && (W)c < lo;
    emit(isr, c, in ? sti[e] : 0u);
    if (in && !isr) valid |= 1u << t;
  }
  bstamp(p, 10);
  // members: the K - R smallest composite keys (code || index), radix passes in shared memory
  block_select_smem<KIND, kBBlock>(stc, sti, tcnt, valid, kk - R, (unsigned long long)n - R, p.IB,
                                   p.early_stop == 0, sh.sel, emit);
  __syncthreads();
  bstamp(p, 14);
  if (tid == 0) {
    st->out_count = sh.out;
    st->win_state = 4;  // done
    if (sh.out != (unsigned)kk) st->error |= 4u;
  }
  __syncthreads();
}

template <int KIND>
__global__ void __launch_bounds__(kBBlock, 1) batch_kernel(const BatchParams p) {
  namespace cg = cooperative_groups;
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  extern __shared__ __align__(128) unsigned char batch_smem[];
  __shared__ BatchShared<W> sh;
  __shared__ unsigned sh_scnt[kBStages];  // entries of the chunk in each ring stage (its chunk slot)
  cg::grid_group grid = cg::this_grid();
  const int G = (int)gridDim.x, cta = (int)blockIdx.x, tid = threadIdx.x;
  const unsigned ring = smem_addr(batch_smem);
  const unsigned fullb = ring + (unsigned)kBRingBytes, emptyb = fullb + 8u * kBStages;
  const int64_t nch = p.batch * (int64_t)p.cpc;
  const int64_t mine = cta < nch ? (nch - 1 - cta) / G + 1 : 0;  // chunks cta, cta + G, ...
#if AIRTOPK_BATCH_PDL
  // PDL: launched while the previous kernel of the stream (e.g. the previous select's fallback
  // launch) runs; nothing global is touched before its writes are visible
  pdl_wait();
  pdl_trigger();
#endif
  bstamp(p, 0);
  // the first kBPre chunks this CTA streams start landing in the ring while the rows are sampled
  if (tid < kBStages) sh_scnt[tid] = 0;
  if (tid == 0) {
    if (cta == 0) *p.fail = 0;  // (appends happen after the first grid barrier)
    for (int i = 0; i < kBStages; ++i) {
      mbar_init(fullb + 8u * i, 1);
      mbar_init(emptyb + 8u * i, kBGWarps);
    }
    fence_mbar_init();
    if (cta >= p.batch) {  // no row to sample: start streaming into the ring (and L2) at once
      for (int i = 0; i < kBPre && i < mine; ++i) batch_issue<U>(p, cta + (int64_t)i * G, ring, i);
      for (int i = kBPre; i < kBPre + kBL2Pre && i < mine; ++i) batch_prefetch_l2<U>(p, cta + (int64_t)i * G);
    }
  }
  __syncthreads();
  // ---- A: windows (samples in the ring stages not yet in use); a sampling CTA issues its first
  // bulk copies once its scattered sample loads have returned (they must not queue behind them) ----
  for (int64_t row = cta; row < p.batch; row += G)
    batch_sample_row<KIND>(p, row, batch_smem + kBPre * kBStage, sh, row == cta ? mine : 0, ring);
#ifdef AIRTOPK_BATCH_TWICE  // debug: a second (warm instruction cache) sampling pass, stamps overwritten
  for (int64_t row = cta; row < p.batch; row += G)
    batch_sample_row<KIND>(p, row, batch_smem + kBPre * kBStage, sh, 0, ring);
#endif
  bstamp(p, 3);
  grid.sync();
  bstamp(p, 4);
  // ---- B: stream every chunk once through the ring; group g consumes iterations i = g (mod 2) ----
  if (tid == 0) {
    fence_proxy_async_smem();  // the sample writes precede the bulk copies into the same stages
    for (int i = kBPre; i < kBStages && i < mine; ++i) batch_issue<U>(p, cta + (int64_t)i * G, ring, i);
  }
  {
    const int grp = (tid >> 5) / kBGWarps, gt = tid & (kBGThreads - 1);
    const int64_t rb = p.len * (int64_t)sizeof(U);
    // chunk cta + i*G = (row, ci), advanced incrementally by 2 iterations; the next chunk's window is
    // loaded one iteration ahead (its L2 latency must not sit in front of every chunk)
    const int64_t step = (int64_t)kBGroups * G;
    const int64_t drow = step / p.cpc;
    const int dci = (int)(step - drow * p.cpc);
    const int64_t ch0 = cta + (int64_t)grp * G;
    int64_t row = ch0 / p.cpc;
    int ci = (int)(ch0 - row * p.cpc);
    int ws = 0;
    unsigned long long hi = 0;
    if (grp < mine) {
      ws = p.st[row].win_state;
      hi = p.st[row].win_hi;
    }
    int st = grp;
    unsigned ph = 0;
#pragma unroll 1
    for (int64_t i = grp; i < mine; i += kBGroups) {
      int64_t nrow = row + drow;
      int nci = ci + dci;
      if (nci >= p.cpc) {
        nci -= p.cpc;
        ++nrow;
      }
      int nws = 0;
      unsigned long long nhi = 0;
      if (i + kBGroups < mine) {
        nws = p.st[nrow].win_state;
        nhi = p.st[nrow].win_hi;
      }
      const int64_t left = rb - ci * (int64_t)kBStage;
      mbar_wait_sleep(fullb + 8u * st, ph);
      if (ws == 1) {
        if (left >= (int64_t)kBStage) batch_classify<KIND, true>(p, row, ci, hi, ring + st * kBStage, 0, gt, &sh_scnt[st]);
        else batch_classify<KIND, false>(p, row, ci, hi, ring + st * kBStage, (int)(left / 16), gt, &sh_scnt[st]);
      }
      __syncwarp();
      if ((tid & 31) == 0) mbar_arrive(emptyb + 8u * st);
      // the group leader, once every warp of the group released the stage: the chunk slot's count,
      // then the refill with the chunk kBStages iterations ahead
      if (gt == 0) {
        mbar_wait_sleep(emptyb + 8u * st, ph);
        batch_slot_done<U>(p, row, ci, &sh_scnt[st]);
        if (i + kBStages < mine) {
          fence_proxy_async_smem();
          batch_issue<U>(p, cta + (i + kBStages) * G, ring, st);
        }
      }
      st += kBGroups;
      if (st >= kBStages) {
        st -= kBStages;
        ph ^= 1u;
      }
      row = nrow;
      ci = nci;
      ws = nws;
      hi = nhi;
    }
  }
  bstamp(p, 5);
  // touch the pages phase C reads first (slot counts and entries of this CTA's first row): their
  // address translations are then cached before the barrier instead of after it
  if (tid < 3 && cta < p.batch) {
    const char* a = tid == 0 ? (const char*)(p.cnt + (size_t)cta * p.nwc)
                  : tid == 1 ? (const char*)p.scode + (size_t)cta * p.nwc * p.scap * sizeof(U)
                             : (const char*)(p.sidx + (size_t)cta * p.nwc * p.scap);
    asm volatile("prefetch.global.L2 [%0];" ::"l"(a) : "memory");
  }
  grid.sync();
  bstamp(p, 6);
  // ---- C: finish every row (staging in the ring: every bulk copy has been consumed) ----
#ifdef AIRTOPK_BATCH_FINISH_TWICE  // debug: a first gather-only run (warm instruction cache), stamps overwritten
  for (int64_t row = cta; row < p.batch; row += G) batch_finish_row<KIND>(p, row, batch_smem, sh, true);
  __syncthreads();
#endif
  for (int64_t row = cta; row < p.batch; row += G) batch_finish_row<KIND>(p, row, batch_smem, sh);
  bstamp(p, 15);
}

template <int KIND>
constexpr size_t batch_smem_bytes() {
  static_assert((size_t)kBFcap * (sizeof(typename KT<KIND>::U) + 4) <= kBRingBytes, "finish staging fits the ring");
  return kBRingBytes + 16 * kBStages;
}

template <int KIND>
cudaError_t launch_cluster_kind(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s, int tail);

// Batched engine: the cooperative batch kernel + the fallback launch (cluster engine, rows whose
// window failed; returns at once when there are none).
template <int KIND>
cudaError_t launch_batch_kind(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s) {
  auto kern = batch_kernel<KIND>;
  constexpr size_t smem = batch_smem_bytes<KIND>();
  cudaError_t e = func_attr(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int occ = 0;
  if (!occ_cache_get((const void*)kern, 0, &occ)) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBBlock, smem);
    if (e != cudaSuccess) return e;
    occ_cache_put((const void*)kern, 0, occ);
  }
  if (occ < 1) return cudaErrorInvalidConfiguration;
  char* base = (char*)ws;
  BatchParams p;
  p.keys = a.keys;
  p.batch = a.batch;
  p.len = a.len;
  p.k = a.k;
  p.sel_min = a.sel_min;
  p.IB = pl.IB;
  p.out_vals = a.out_vals;
  p.out_idx = a.out_idx;
  p.idx_off = a.idx_off;
  p.st = (RowState*)(base + pl.off_state);
  p.cnt = (unsigned short*)(base + pl.off_bcnt);
  p.scode = base + pl.off_bslot;
  p.sidx = (unsigned*)(base + pl.off_bsidx);
  p.fail = (unsigned*)(base + pl.off_bfail);
  p.nwc = pl.nwc;
  p.scap = pl.scap;
  p.cpc = pl.cpc;
  p.nsamp = pl.nsamp;
  p.early_stop = a.early_stop;
  p.timing = a.trace;
  p.timing_n = a.trace_len > 0 ? a.trace_len : a.batch * kTraceMaxPasses * kTraceFields;
  const int G = num_sms() * std::min(occ, 1);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)G);
  cfg.blockDim = dim3(kBBlock);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = AIRTOPK_BATCH_PDL ? 2 : 1;
  if (a.events && a.n_events > 0) cudaEventRecord((cudaEvent_t)a.events[0], s);
  e = cudaLaunchKernelEx(&cfg, kern, p);
  if (e != cudaSuccess) return e;
  if (a.events && a.n_events > 1) cudaEventRecord((cudaEvent_t)a.events[1], s);
  e = launch_cluster_kind<KIND>(a, pl, ws, s, 2);  // fallback mode
  if (a.events && a.n_events > 2) cudaEventRecord((cudaEvent_t)a.events[2], s);
  return e;
}

#define AIRTOPK_INSTANTIATE_BATCH(KIND) \
  template cudaError_t launch_batch_kind<KIND>(const SelectArgs&, const Plan&, void*, cudaStream_t);

}  // namespace airtopk
