// passes.cuh — the streaming body of one AIR Top-K pass, shared by both engines.
//
// One call processes this CTA's slice of the pass source (Alg1 L7-8: the input row L or the
// candidate buffer of the previous pass) and performs, per element,
//   DF (digit filtered, Alg1 L15-22): results (digit < target) -> output V/I; candidates
//       (digit == target) -> candidate buffer if C < N/alpha (L17-18);
//   DH (digit histogrammed, L12-13 / L19-20): candidates counted in the shared histogram.
// DF/DH: 0 none, 1 key digit, 2 index digit (the lowest-index tie-break digits);
// DF == 3 is the sample-guided window pass.
//
// B200 choices (measured, tools/microbench_stream.cu):
//   * input streaming either by 4 x 128-bit ld.global.nc.L1::no_allocate per thread (register
//     path) or through a per-CTA ring of 16 KiB bulk copies (cp.async.bulk, TMA engine) filled by
//     one thread and consumed by all warps (full / empty mbarriers). Few large bulk copies keep
//     ~190 KiB per SM in flight; many small per-warp copies measured 7-50 % slower;
//   * per element, the fast path is a few integer ops: the histogram passes add a predicated
//     shared atomic (hardware-aggregated for equal addresses), the window pass ONE compare of the
//     raw key bits against a transformed threshold (exact, no key transform needed);
//   * flagged elements (results / candidates; ~1 per warp tile in the window pass of c3) leave
//     through ONE tagged queue per warp: a warp scan of the per-lane flag counts places every
//     lane's flagged elements at once, the tag (result / candidate / drop) is set on the way in,
//     and a full queue is flushed with one global atomic per destination and coalesced stores.
#pragma once

#include <algorithm>
#include <type_traits>

#include "device.cuh"
#include "tma.cuh"

namespace airtopk {

#ifndef AIRTOPK_SLOW_REG
#define AIRTOPK_SLOW_REG 1  // register path: flagged elements re-read from the tile registers (1) or L2 (0)
#endif
#ifndef AIRTOPK_PREFETCH
#define AIRTOPK_PREFETCH 0  // register path: issue the next tile's loads before classifying this one
#endif
#ifndef AIRTOPK_UNROLL
#define AIRTOPK_UNROLL 4
#endif
#ifndef AIRTOPK_TMA_STAGES
#define AIRTOPK_TMA_STAGES 12
#endif
#ifndef AIRTOPK_TMA_CHUNK
#define AIRTOPK_TMA_CHUNK 32768
#endif
constexpr int kUnroll = AIRTOPK_UNROLL;
constexpr int kTmaStages = AIRTOPK_TMA_STAGES;       // max ring depth of the bulk-copy streaming loop
constexpr unsigned kTmaChunk = AIRTOPK_TMA_CHUNK;    // bytes per bulk copy (one ring stage)
// dynamic + static shared memory per CTA is capped at 227 KiB; the static part (queues, scan
// scratch) of the grid pass kernel stays below 20 KiB
constexpr size_t kSmemCap = 232448;
constexpr size_t kStaticSmemReserve = 19072;  // >= the largest static smem of a TMA pass kernel (ptxas: 18976)
// Copies of the shared histogram in the filter passes: lane l counts into copy l % kHistCopies
// (interleaved bin-major so copies of one bin sit in different banks); cuts the same-address
// serialisation of shared atomics when many lanes hit a few bins (radix-adversarial passes).
constexpr int kHistCopies = 4;
// Extra histogram slot that absorbs the atomics of non-candidates / invalid lanes (never scanned).
constexpr int kDummyBin = kMaxBins;
constexpr int kHistSlots = kMaxBins + 32;  // per copy; the dummy bin + padding

template <int HC>
constexpr size_t tma_ring_offset() { return ((size_t)kHistSlots * 4 * HC + 127) / 128 * 128; }
template <int HC>
constexpr int tma_stages() {
  const size_t avail = kSmemCap - kStaticSmemReserve - tma_ring_offset<HC>();
  const size_t s = avail / (kTmaChunk + 16);  // stage + its two mbarriers
  return (int)(s < (size_t)kTmaStages ? s : (size_t)kTmaStages);
}
// dynamic shared memory of a TMA pass: [histogram copies][ring stages][full bars][empty bars]
template <int HC>
constexpr size_t tma_smem_bytes() { return tma_ring_offset<HC>() + (size_t)tma_stages<HC>() * (kTmaChunk + 16); }

// +1 on a shared-window address (no return value): red.shared.add, which the hardware aggregates
// over lanes hitting the same address.
__device__ __forceinline__ void shared_inc(unsigned addr) {
  asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(addr) : "memory");
}

// Per-warp queue of flagged elements. tag: 0 result (-> V, I), 1 candidate (-> buffer), 2 dropped.
template <typename U, typename IdxT>
struct WarpQ {
  static constexpr int kCap = (sizeof(U) + sizeof(IdxT) <= 8) ? 128 : 64;
  U code[kCap];
  IdxT idx[kCap];
  unsigned char tag[kCap];
};

template <int KIND, typename IdxT, int DF>
__host__ __device__ constexpr int hist_copies() {
  using U = typename KT<KIND>::U;
  // DF == 3 (window pass): two separate histograms of the window members, digits qs and qs + 1
  return DF == 0 ? 1 : DF == 3 ? 2 : (sizeof(U) + sizeof(IdxT) <= 8 ? kHistCopies : 2);
}

// Store the n queued entries of a warp: results at out[br ...], candidates at buf[bc ...], in queue
// order (coalesced). Entries beyond a destination's limit set the error flag instead.
template <int KIND, typename IdxT>
__device__ __noinline__ void wq_write(const WarpQ<typename KT<KIND>::U, IdxT>* wq, int n, unsigned long long br,
                                      unsigned long long bc, typename KT<KIND>::U* ov, int64_t* oi,
                                      unsigned long long kk, typename KT<KIND>::U* bco, IdxT* bio,
                                      unsigned long long capa, bool sel_min, unsigned* err, int64_t ioff) {
  const int lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt();
  for (int j0 = 0; j0 < n; j0 += 32) {
    const int j = j0 + lane;
    const int tg = (j < n) ? (int)wq->tag[j] : 2;
    const unsigned mr = __ballot_sync(kFull, tg == 0), mc = __ballot_sync(kFull, tg == 1);
    if (tg == 0) {
      const unsigned long long pos = br + __popc(mr & lt);
      if (pos < kk) {
        ov[pos] = from_code<KIND>(wq->code[j], sel_min);
        oi[pos] = (int64_t)wq->idx[j] + ioff;
      } else {
        *err |= 1u;
      }
    } else if (tg == 1) {
      const unsigned long long pos = bc + __popc(mc & lt);
      if (pos < capa) {
        bco[pos] = wq->code[j];
        bio[pos] = wq->idx[j];
      } else {
        *err |= 2u;
      }
    }
    br += __popc(mr);
    bc += __popc(mc);
  }
}

// Counts of results (low 16 bits) and candidates (high 16 bits) among a warp's n queued entries.
template <typename U, typename IdxT>
__device__ __forceinline__ unsigned wq_counts(const WarpQ<U, IdxT>* wq, int n) {
  const int lane = threadIdx.x & 31;
  unsigned nr = 0, nc = 0;
  for (int j0 = 0; j0 < n; j0 += 32) {
    const int j = j0 + lane;
    const int tg = (j < n) ? (int)wq->tag[j] : 2;
    nr += __popc(__ballot_sync(kFull, tg == 0));
    nc += __popc(__ballot_sync(kFull, tg == 1));
  }
  return nr | (nc << 16);
}

// Flush a full warp queue: ONE global atomic per destination reserves the slots, then coalesced
// stores (wq_write stays out of line: I-cache; inlining this part avoids call-clobber spills).
template <int KIND, typename IdxT>
__device__ __forceinline__ void wq_flush(const WarpQ<typename KT<KIND>::U, IdxT>* wq, int n, unsigned long long* outc,
                                      unsigned long long* bufc, typename KT<KIND>::U* ov, int64_t* oi,
                                      unsigned long long kk, typename KT<KIND>::U* bco, IdxT* bio,
                                      unsigned long long capa, bool sel_min, unsigned* err, int64_t ioff) {
  const int lane = threadIdx.x & 31;
  const unsigned cnt = wq_counts(wq, n);
  unsigned long long b = 0;
  if (lane == 0 && (cnt & 0xffffu)) b = atomicAdd(outc, (unsigned long long)(cnt & 0xffffu));
  if (lane == 1 && (cnt >> 16)) b = atomicAdd(bufc, (unsigned long long)(cnt >> 16));
  const unsigned long long br = __shfl_sync(kFull, b, 0), bc = __shfl_sync(kFull, b, 1);
  wq_write<KIND, IdxT>(wq, n, br, bc, ov, oi, kk, bco, bio, capa, sel_min, err, ioff);
}

// Everything one pass of one row needs (built by the engine from its copy of the row state).
template <typename U, typename IdxT>
struct PassCtx {
  int q;
  bool emit_all, do_hist, srcL, store, sel_min, reverse;
  bool pre = false;  // TMA: the ring's first stages were issued before the PDL wait (window pass)
  Digit dh, df;
  Digit dh2;        // DF == 3: the digit after dh (its member histogram at counter offset kHistSlots)
  unsigned long long tcode, tidx;  // fixed prefix bits after scan q-1
  // source: row L (slice `slice` of `nslices`) or the previous candidate buffer
  const U* rowp;
  const int64_t* rowi;  // HASIDX: caller-given index values of the row
  int64_t len;
  int slice, nslices;
  const U* bcin;
  const IdxT* biin;
  unsigned long long nbuf;
  // results
  U* ov;
  int64_t* oi;
  int64_t ioff;     // added to every output index (multi-GPU shard: global index = local + offset)
  unsigned long long* outc;
  unsigned long long kk;
  // candidates
  U* bco;
  IdxT* bio;
  unsigned long long* bufc;
  unsigned long long capa;
  unsigned* err;
  unsigned long long lo, span1;  // DF == 3 window: candidates lo <= code < lo + span1, results code < lo
  unsigned long long* wnmin;     // DF == 3: atomicMax of ~code / code over the window members
  unsigned long long* wmax;
  unsigned* hist;  // shared, kMaxBins * hist_copies() counters, zeroed by the caller
  unsigned ring;   // TMA streaming: shared-window address of the ring (after the histogram copies)
  WarpQ<U, IdxT>* wq;
  int64_t* dbg = nullptr;  // debug (fused tail stamps): CTA 0's %globaltimer at points of the pass
};

__device__ __forceinline__ void pass_dbg(int64_t* d, int i) {
  if (d != nullptr && blockIdx.x == 0 && threadIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    d[i] = (int64_t)t;
  }
}

// First stages of the bulk-copy ring of a TMA pass over the input row (thread 0: barrier init + up to
// NST copies). Returns the number of stages issued (thread 0).
template <typename U, int HC, int BLOCK>
__device__ __forceinline__ int tma_prologue(const U* rowp, int64_t len, int slice, int nslices, bool reverse,
                                            unsigned ring) {
  constexpr int VEC = 16 / sizeof(U);
  constexpr int NST = tma_stages<HC>();
  constexpr int NVT = (int)(kTmaChunk / 16 / BLOCK);
  constexpr int64_t CV = (int64_t)BLOCK * NVT;
  constexpr int NW = BLOCK / 32;
  if (threadIdx.x != 0) return 0;
  const uintptr_t mis = (uintptr_t)rowp & 15u;
  const int64_t head = mis ? std::min<int64_t>(len, (int64_t)((16u - mis) / sizeof(U))) : 0;
  const int64_t nvec = (len - head) / VEC;
  const uint4* vp = (const uint4*)(rowp + head);
  const unsigned fullb = ring + NST * kTmaChunk, emptyb = fullb + 8u * NST;
  const int64_t nch = nvec / CV;
  const int64_t mine = (nch > slice) ? (nch - 1 - slice) / nslices + 1 : 0;
  const int64_t c0 = reverse ? (int64_t)slice + (mine - 1) * nslices : (int64_t)slice;
  const int64_t sstep = (reverse ? -(int64_t)nslices : (int64_t)nslices) * CV;
  const uint4* const src0 = vp + c0 * CV;
  for (int st = 0; st < NST; ++st) {
    mbar_init(fullb + 8u * st, 1);
    mbar_init(emptyb + 8u * st, NW);
  }
  fence_mbar_init();
  int st = 0;
  for (; st < NST && st < mine; ++st) {
    mbar_arrive_expect_tx(fullb + 8u * st, kTmaChunk);
    bulk_g2s(ring + st * kTmaChunk, src0 + st * sstep, kTmaChunk, fullb + 8u * st);
  }
  return st;
}

// L2 prefetch (cp.async.bulk.prefetch.L2) of this CTA's chunks [from, from + count) of a forward TMA
// pass (thread 0): the window pass issues it before its PDL wait, so HBM keeps streaming while the
// sample kernel finishes (the ring alone holds only its first NST chunks).
template <typename U, int BLOCK>
__device__ __forceinline__ void tma_prefetch_l2(const U* rowp, int64_t len, int slice, int nslices, int from,
                                                int count) {
  constexpr int VEC = 16 / sizeof(U);
  constexpr int NVT = (int)(kTmaChunk / 16 / BLOCK);
  constexpr int64_t CV = (int64_t)BLOCK * NVT;
  if (threadIdx.x != 0 || count <= 0) return;
  const uintptr_t mis = (uintptr_t)rowp & 15u;
  const int64_t head = mis ? std::min<int64_t>(len, (int64_t)((16u - mis) / sizeof(U))) : 0;
  const int64_t nvec = (len - head) / VEC;
  const uint4* vp = (const uint4*)(rowp + head);
  const int64_t nch = nvec / CV;
  const int64_t mine = (nch > slice) ? (nch - 1 - slice) / nslices + 1 : 0;
  for (int64_t i = from; i < mine && i < (int64_t)from + count; ++i)
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(vp + ((int64_t)slice + i * nslices) * CV),
                 "r"(kTmaChunk)
                 : "memory");
}

// Runs the pass over this CTA's slice; the queues are flushed on return. Returns the number of
// elements of the whole source (for the trace).
template <int KIND, typename IdxT, int DF, int DH, bool HASIDX, int BLOCK, int HCOPIES = 0, bool TMA = false,
          int BU = 4>
__device__ __forceinline__ unsigned long long run_pass(const PassCtx<typename KT<KIND>::U, IdxT>& c) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;  // shifted-key width
  using Q = WarpQ<U, IdxT>;
  constexpr int VEC = 16 / sizeof(U);
  constexpr int HC = HCOPIES > 0 ? HCOPIES : hist_copies<KIND, IdxT, DF>();  // histogram copies
  constexpr int NW = BLOCK / 32;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

  const int shh = c.dh.shift;
  const unsigned hmask = (1u << c.dh.width) - 1u;
  const int sf = c.df.shift;
  const bool emit_all = c.emit_all, do_hist = c.do_hist, store = c.store, sel_min = c.sel_min;

  W tc = 0, bc = 0;
  U fc = 0;
  IdxT ti = 0, bi = 0;
  if (DF == 1) {
    tc = (W)(c.tcode >> sf);
    bc = tc & ~(W)((1u << c.df.width) - 1u);
  } else if (DF == 2) {
    fc = (U)c.tcode;
    ti = (IdxT)(c.tidx >> sf);
    bi = ti & ~(IdxT)((1u << c.df.width) - 1u);
  }
  // Fast classification for adjacent key digits (DF == 1, DH == 1, sf == shh + w): with
  // t = code >> shh and B = bc << w, y = t - B lies in [0, S) for results (higher digits == prefix,
  // digit q-1 < j), in [S, S + nb) for candidates (x = y - S is then digit q), and >= S + nb (or
  // wraps) otherwise. S = (tc - bc) << w, nb = 2^w.
  const int wq_ = c.dh.width;
  const W kx_B = (DF == 1) ? (W)(bc << wq_) : (W)0;
  const W kx_S = (DF == 1) ? (W)((tc - bc) << wq_) : (W)0;
  const W kx_nb = (W)1 << wq_;
  const W kx_flag = kx_S + ((emit_all || store) ? kx_nb : (W)0);  // fast-path flag threshold on y
  // shared-window address of this lane's histogram copy (c.hist is the dynamic smem base)
  const unsigned hbase =
      (unsigned)__cvta_generic_to_shared(c.hist) + ((HC > 1 && DF != 3) ? (unsigned)(lane % HC) * 4u : 0u);
  const int shh2 = c.dh2.shift;
  const unsigned hmask2 = (1u << c.dh2.width) - 1u;
  const U xmask = sel_min ? (U)0 : (U)~(U)0;
  W wlo_seen = ~(W)0, whi_seen = 0;  // DF == 3: extremes of this thread's window members

  // Window [lo, hi] (DF == 3). code <= hi is tested on the RAW key bits b as (b ^ wx) <= hi: for
  // IEEE keys with sign bit S, code(b) <= hi <=> b ^ S <= hi when hi >= S (select-min; the
  // threshold key is non-negative, every negative key qualifies), <=> ~b <= hi when hi < S; the
  // select-max and unsigned cases are the complements.
  const W wlo = (W)c.lo, wspan = (W)c.span1;
  const W whi = (W)(wlo + wspan - 1);
  W wx = 0;
  if constexpr (DF == 3) {
    constexpr W S = (W)((W)1 << (KT<KIND>::R - 1));
    constexpr W ones = (W)(U)~(U)0;  // (U) again: ~ promotes 16-bit keys to int
    if constexpr (KT<KIND>::IEEE) {
      if (sel_min) wx = (whi >= S) ? S : ones;
      else wx = (whi < S) ? (W)(ones ^ S) : (W)0;
    } else {
      wx = sel_min ? (W)0 : ones;
    }
  }

  // Filter classification of digit q-1 (Alg1 L15-22): win = result, cand = candidate for pass q.
  auto classify = [&](U code, IdxT idx, bool valid, bool& win, bool& cand) {
    bool lt, eq;
    if constexpr (DF == 3) {  // sample-guided window
      win = valid && ((W)code < wlo);
      cand = valid && ((W)((W)code - wlo) < wspan);
      return;
    } else if constexpr (DF == 1) {
      const W h = (W)code >> sf;
      lt = (W)(h - bc) < (W)(tc - bc);
      eq = (h == tc);
    } else {
      const bool ce = (code == fc);
      const IdxT h = (IdxT)(idx >> sf);
      lt = ce && ((IdxT)(h - bi) < (IdxT)(ti - bi));
      eq = ce && (h == ti);
    }
    win = valid && (lt || (emit_all && eq));
    cand = valid && !emit_all && eq;
  };
  // Alg1 L19-20. Non-candidates count into a dummy bin instead of branching: a warp-uniform address
  // is aggregated by the shared atomic unit, so the common "no candidate" case is one cheap atomic
  // and no divergence.
  auto hist_cand = [&](U code, IdxT idx, bool cand) {
    unsigned d;
    if constexpr (DH == 2) d = (unsigned)(idx >> shh) & hmask;
    else d = (unsigned)((W)code >> shh) & hmask;
    d = (cand && do_hist) ? d : (unsigned)kDummyBin;
    shared_inc(hbase + d * (HC * 4));
  };

  // ---- the warp's tagged queue ----
  Q* const wq = c.wq;
  int qcnt = 0;
  auto flush_full = [&]() {
    __syncwarp();
    wq_flush<KIND, IdxT>(wq, qcnt, c.outc, c.bufc, c.ov, c.oi, c.kk, c.bco, c.bio, c.capa, sel_min, c.err, c.ioff);
    qcnt = 0;
    __syncwarp();
  };
  // one element per lane (all lanes call): tag 0 result, 1 candidate
  auto push1 = [&](bool pred, int tag, U code, IdxT idx) {
    const unsigned m = __ballot_sync(kFull, pred);
    if (!m) return;
    const int n = __popc(m);
    if (qcnt + n > Q::kCap) flush_full();
    if (pred) {
      const int pos = qcnt + __popc(m & lanemask_lt());
      wq->code[pos] = code;
      wq->idx[pos] = idx;
      wq->tag[pos] = (unsigned char)tag;
    }
    qcnt += n;
  };
  auto tag_of = [&](U code, IdxT idx) -> int {
    bool w, cd;
    classify(code, idx, true, w, cd);
    if constexpr (DF == 3) {
      if (cd) {  // window member: extremes + the pass-1 digit histogram of the window buffer
        wlo_seen = ((W)code < wlo_seen) ? (W)code : wlo_seen;
        whi_seen = ((W)code > whi_seen) ? (W)code : whi_seen;
        shared_inc(hbase + 4u * (unsigned)(((W)code >> shh) & hmask));
        shared_inc(hbase + 4u * (unsigned)(kHistSlots + (((W)code >> shh2) & hmask2)));
      }
    }
    return w ? 0 : ((cd && store) ? 1 : 2);
  };

  unsigned long long nread;
  if (c.srcL) {
    // ---- source = the input row L (contiguous slice per CTA, 16-byte vectors) ----
    const U* rowp = c.rowp;
    const uintptr_t mis = (uintptr_t)rowp & 15u;
    const int64_t head = mis ? std::min<int64_t>(c.len, (int64_t)((16u - mis) / sizeof(U))) : 0;
    const int64_t nvec = (c.len - head) / VEC;
    const int64_t tail0 = head + nvec * VEC;
    const uint4* vp = (const uint4*)(rowp + head);
    nread = c.len;

    auto index_of = [&](int64_t pos) -> IdxT {  // lazily: only results/candidates/index digits need it
      if constexpr (HASIDX) return (IdxT)c.rowi[pos];
      else return (IdxT)pos;
    };

    // Flagged elements of a tile -> the warp queue. Lane-local flags fl (bit b = element b of the
    // lane's tile); a warp scan of the flag counts gives every lane its queue slots, so the usual
    // case (a handful of flagged elements per warp tile) is one scan and one short loop per lane.
    // get(b, pos) returns the raw key of element b (shared-memory stage, registers or L2).
    auto drain = [&](auto fl, int64_t vb, int64_t vs, auto get) {
      using FlagT = decltype(fl);
      // usual case, at most one flagged element per lane: slots from one ballot (no scan chain)
      if (!__any_sync(kFull, (fl & (fl - 1)) != 0)) {
        const unsigned m = __ballot_sync(kFull, fl != 0);
        const int total = __popc(m);
        if (qcnt + total > Q::kCap) flush_full();
        if (fl) {
          const int qp = qcnt + __popc(m & lanemask_lt());
          const int b = ((sizeof(FlagT) == 8) ? __ffsll((long long)fl) : __ffs((int)fl)) - 1;
          const int64_t pos = head + (vb + (int64_t)(b / VEC) * vs) * VEC + (b % VEC);
          const U code = to_code_x<KIND>(get(b, pos), xmask);
          const IdxT idx = index_of(pos);
          wq->code[qp] = code;
          wq->idx[qp] = idx;
          wq->tag[qp] = (unsigned char)tag_of(code, idx);
        }
        qcnt += total;
        return;
      }
      while (true) {
        const int n = (sizeof(FlagT) == 8) ? __popcll((unsigned long long)fl) : __popc((unsigned)fl);
        int incl = n;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int y = __shfl_up_sync(kFull, incl, o);
          if (lane >= o) incl += y;
        }
        const int total = __shfl_sync(kFull, incl, 31);
        int qp = qcnt + incl - n;
        while (fl && qp < Q::kCap) {
          const int b = ((sizeof(FlagT) == 8) ? __ffsll((long long)fl) : __ffs((int)fl)) - 1;
          fl &= fl - 1;
          const int64_t pos = head + (vb + (int64_t)(b / VEC) * vs) * VEC + (b % VEC);
          const U code = to_code_x<KIND>(get(b, pos), xmask);
          const IdxT idx = index_of(pos);
          wq->code[qp] = code;
          wq->idx[qp] = idx;
          wq->tag[qp] = (unsigned char)tag_of(code, idx);
          ++qp;
        }
        const bool fits = qcnt + total <= Q::kCap;
        qcnt = fits ? qcnt + total : Q::kCap;
        if (qcnt == Q::kCap) flush_full();
        if (fits || !__any_sync(kFull, fl != 0)) break;
      }
    };

    // One thread's tile: NV 16-byte vectors at vector indices vb + u*vs. FULL: all valid.
    // sstage: shared-window address of the warp's staged tile (TMA path) or 0 (register path).
    auto process_tile = [&](const auto& r, int64_t vb, int64_t vlim, auto full_tag, int64_t vs, unsigned sstage) {
      constexpr bool FULL = decltype(full_tag)::value;
      constexpr int NV = (int)(sizeof(r) / sizeof(uint4));
      if constexpr (DF == 0) {
        // pass 1: the top digit needs no mask (code >> shh < 2^11)
#pragma unroll
        for (int u = 0; u < NV; ++u) {
          const bool valid = FULL || (vb + (int64_t)u * vs < vlim);
#pragma unroll
          for (int e = 0; e < VEC; ++e) {
            const U code = to_code_x<KIND>(vec_elem<U>(r[u], e), xmask);
            const unsigned d = (unsigned)((W)code >> shh);
            shared_inc(hbase + 4u * (valid ? d : (unsigned)kDummyBin));
          }
        }
        return;
      } else {
        using FlagT = std::conditional_t<(NV * VEC > 32), unsigned long long, unsigned>;
        FlagT fl = 0;  // elements that must leave through the queue (results / stored candidates)
        if constexpr (DF == 3) {
          // window pass: result (code < lo) or window member (lo <= code <= hi), together code <= hi,
          // tested on the raw bits: the lane's minimum of b ^ wx (one xor + one min per element), the
          // per-element flags only when the minimum hits (a few lanes per warp tile)
          W m = ~(W)0;
#pragma unroll
          for (int u = 0; u < NV; ++u) {
            const bool valid = FULL || (vb + (int64_t)u * vs < vlim);
#pragma unroll
            for (int e = 0; e < VEC; ++e) {
              const W t = (W)((W)vec_elem<U>(r[u], e) ^ wx);
              m = (valid && t < m) ? t : m;
            }
          }
          if (m <= whi) {
#pragma unroll
            for (int u = 0; u < NV; ++u) {
              const bool valid = FULL || (vb + (int64_t)u * vs < vlim);
#pragma unroll
              for (int e = 0; e < VEC; ++e)
                if (valid && (W)((W)vec_elem<U>(r[u], e) ^ wx) <= whi) fl |= (FlagT)1 << (u * VEC + e);
            }
          }
        } else if constexpr (DF == 1 && DH == 1) {
          // adjacent key digits: y = (code >> shh) - B places the elements whose higher digits match
          // the prefix at [S, S + nb) and the results below S (see the derivation at kx_* above)
#pragma unroll
          for (int u = 0; u < NV; ++u) {
            const bool valid = FULL || (vb + (int64_t)u * vs < vlim);
#pragma unroll
            for (int e = 0; e < VEC; ++e) {
              const U code = to_code_x<KIND>(vec_elem<U>(r[u], e), xmask);
              const W y = ((W)code >> shh) - kx_B;
              const unsigned d = (unsigned)min((W)(y - kx_S), (W)kDummyBin);
              shared_inc(hbase + (valid ? d : (unsigned)kDummyBin) * (HC * 4u));
              // result (y < S) or stored candidate / emit-all member (S <= y < S + nb): one compare
              if (valid && y < kx_flag) fl |= (FlagT)1 << (u * VEC + e);
            }
          }
        } else {
#pragma unroll
          for (int u = 0; u < NV; ++u) {
            const int64_t v = vb + (int64_t)u * vs;
            const bool valid = FULL || (v < vlim);
#pragma unroll
            for (int e = 0; e < VEC; ++e) {
              const U code = to_code_x<KIND>(vec_elem<U>(r[u], e), xmask);
              IdxT idx = 0;
              if constexpr (DF == 2 || DH == 2) {
                // the index is needed to classify (DF == 2) or to histogram a candidate (DH == 2)
                bool need = true;
                if constexpr (HASIDX) need = (DF == 2) ? (code == fc) : (((W)code >> sf) == tc);
                if (need && valid) idx = index_of(head + v * VEC + e);
              }
              bool win, cand;
              classify(code, idx, valid, win, cand);
              hist_cand(code, idx, cand);
              if (win || (cand && store)) fl |= (FlagT)1 << (u * VEC + e);
            }
          }
        }
        if (__any_sync(kFull, fl != 0)) {
          if (TMA && sstage) {
            drain(fl, vb, vs, [&](int b, int64_t) -> U {
              const unsigned a = sstage + (unsigned)((((b / VEC) * 32 + lane) * 16) + (b % VEC) * (int)sizeof(U));
              if constexpr (sizeof(U) == 2) { unsigned short t; asm volatile("ld.shared.u16 %0, [%1];" : "=h"(t) : "r"(a)); return (U)t; }
              else if constexpr (sizeof(U) == 4) { unsigned t; asm volatile("ld.shared.u32 %0, [%1];" : "=r"(t) : "r"(a)); return (U)t; }
              else { unsigned long long t; asm volatile("ld.shared.u64 %0, [%1];" : "=l"(t) : "r"(a)); return (U)t; }
            });
          } else {
#if AIRTOPK_SLOW_REG
            drain(fl, vb, vs, [&](int b, int64_t) -> U {
              const int u = b / VEC, e = b % VEC;
              uint4 v = r[0];
#pragma unroll
              for (int i = 1; i < NV; ++i) v = (u == i) ? r[i] : v;
              U out = vec_elem<U>(v, 0);
#pragma unroll
              for (int i = 1; i < VEC; ++i) out = (e == i) ? vec_elem<U>(v, i) : out;
              return out;
            });
#else
            drain(fl, vb, vs, [&](int, int64_t pos) -> U { return __ldcg(rowp + pos); });
#endif
          }
        }
      }
    };

    if constexpr (TMA) {
      // Per-CTA ring of NST stages of kTmaChunk bytes in grid-stride chunk order (chunk t -> CTA
      // t mod nslices of the row): thread 0 issues the bulk copies (completion counted on the
      // stage's full barrier), every warp consumes its NVT vectors per lane of a stage and arrives
      // on the stage's empty barrier; thread 0 refills a stage once all warps released it (lagged
      // by one iteration so it seldom waits).
      constexpr int NST = tma_stages<HC>();
      constexpr int NVT = (int)(kTmaChunk / 16 / BLOCK);
      static_assert(NVT >= 1 && kTmaChunk % (16 * BLOCK) == 0, "chunk = BLOCK x NVT 16-byte vectors");
      constexpr int64_t CV = (int64_t)BLOCK * NVT;  // vectors per chunk
      const unsigned ring = c.ring;
      const unsigned fullb = ring + NST * kTmaChunk, emptyb = fullb + 8u * NST;
      const int64_t nch = nvec / CV;
      const int64_t mine = (nch > c.slice) ? (nch - 1 - c.slice) / c.nslices + 1 : 0;
      // chunk of iteration i: c0 + i * cstep (all index arithmetic incremental: no 64-bit divisions
      // in the loop)
      const int64_t c0 = c.reverse ? (int64_t)c.slice + (mine - 1) * c.nslices : (int64_t)c.slice;
      const int64_t cstep = c.reverse ? -(int64_t)c.nslices : (int64_t)c.nslices;
      const uint4* const src0 = vp + c0 * CV;
      const int64_t sstep = cstep * CV;  // in 16-byte vectors
      if (!c.pre) tma_prologue<U, HC, BLOCK>(c.rowp, c.len, c.slice, c.nslices, c.reverse, ring);
      __syncthreads();
      int st = 0, pst = NST - 1;    // stage of this / the previous iteration
      unsigned ph = 0, pph = 1;     // their phase parities
      int64_t vb = c0 * CV + (int64_t)warp * NVT * 32 + lane;
      const uint4* refill = src0 + (int64_t)(NST - 1) * sstep;  // chunk of iteration i - 1 + NST
      for (int64_t i = 0; i < mine; ++i) {
        mbar_wait(fullb + 8u * st, ph);
        const unsigned sw = ring + st * kTmaChunk + (unsigned)(warp * NVT * 32 * 16);  // this warp's part
        uint4 r[NVT];
#pragma unroll
        for (int u = 0; u < NVT; ++u) r[u] = lds128(sw + (unsigned)((u * 32 + lane) * 16));
        process_tile(r, vb, nvec, std::true_type{}, (int64_t)32, sw);
        __syncwarp();
        if (lane == 0) mbar_arrive(emptyb + 8u * st);
        if (tid == 0 && i >= 1 && i - 1 + NST < mine) {  // refill the stage released one iteration ago
          mbar_wait(emptyb + 8u * pst, pph);
          fence_proxy_async_smem();
          mbar_arrive_expect_tx(fullb + 8u * pst, kTmaChunk);
          bulk_g2s(ring + pst * kTmaChunk, refill, kTmaChunk, fullb + 8u * pst);
        }
        refill += sstep;
        pst = st;
        pph = ph;
        if (++st == NST) {
          st = 0;
          ph ^= 1u;
        }
        vb += sstep;
      }
      if (nch * CV < nvec && c.slice == (int)(nch % c.nslices)) {  // the partial last chunk
        const int64_t vb = nch * CV + (int64_t)warp * NVT * 32 + lane;
        uint4 r[NVT];
#pragma unroll
        for (int u = 0; u < NVT; ++u) {
          const int64_t v = vb + (int64_t)u * 32;
          r[u] = (v < nvec) ? ldg_stream(vp + v) : make_uint4(0, 0, 0, 0);
        }
        process_tile(r, vb, nvec, std::false_type{}, (int64_t)32, 0u);
      }
    } else {
      // Grid-stride tile order: tile t (BLOCK*kUnroll 16-byte vectors, 32 KiB for 512 threads) goes
      // to slice t mod nslices, so at any moment the CTAs of a row read one compact, advancing region
      // of HBM. Measured on B200: zero DRAM over-fetch and 7.2-7.4 TB/s, vs 9% over-fetch and 6.3
      // TB/s when every CTA streams its own contiguous chunk (tools/microbench_hist.cu, profiles/).
      // `reverse` walks the tiles backwards (odd passes consume the tail the previous pass left in L2).
      const int64_t tile = (int64_t)BLOCK * kUnroll;
      const int64_t ntiles = nvec / tile;
      const int64_t mine = (ntiles > c.slice) ? (ntiles - 1 - c.slice) / c.nslices + 1 : 0;
      const int64_t t0 = c.reverse ? (int64_t)c.slice + (mine - 1) * c.nslices : (int64_t)c.slice;
      const int64_t vstep = (c.reverse ? -(int64_t)c.nslices : (int64_t)c.nslices) * tile;
      int64_t vb = t0 * tile + tid;
#if AIRTOPK_PREFETCH
      // software pipeline: the next tile's loads are in flight while this tile is classified
      if (mine > 0) {
        uint4 r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) r[u] = ldg_stream(vp + vb + (int64_t)u * BLOCK);
        for (int64_t i = 0; i < mine; ++i) {
          uint4 nx[kUnroll];
          const int64_t vn = (i + 1 < mine) ? vb + vstep : vb;
#pragma unroll
          for (int u = 0; u < kUnroll; ++u) nx[u] = ldg_stream(vp + vn + (int64_t)u * BLOCK);
          process_tile(r, vb, nvec, std::true_type{}, (int64_t)BLOCK, 0u);
#pragma unroll
          for (int u = 0; u < kUnroll; ++u) r[u] = nx[u];
          vb = vn;
        }
      }
#else
      for (int64_t i = 0; i < mine; ++i, vb += vstep) {
        uint4 r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) r[u] = ldg_stream(vp + vb + (int64_t)u * BLOCK);
        process_tile(r, vb, nvec, std::true_type{}, (int64_t)BLOCK, 0u);
      }
#endif
      if (ntiles * tile < nvec && c.slice == (int)(ntiles % c.nslices)) {  // the partial last tile
        const int64_t vb = ntiles * tile + tid;
        uint4 r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          const int64_t v = vb + (int64_t)u * BLOCK;
          r[u] = (v < nvec) ? ldg_stream(vp + v) : make_uint4(0, 0, 0, 0);
        }
        process_tile(r, vb, nvec, std::false_type{}, (int64_t)BLOCK, 0u);
      }
    }
    // scalar head (slice 0) and tail (last slice) of a misaligned / ragged row
    auto process_scalar = [&](int64_t i, bool valid) {
      const U code = to_code<KIND>(valid ? rowp[i] : (U)0, sel_min);
      if constexpr (DF == 0) {
        shared_inc(hbase + 4u * (valid ? (unsigned)(((W)code >> shh) & hmask) : (unsigned)kDummyBin));
      } else {
        const IdxT idx = valid ? index_of(i) : (IdxT)0;
        bool win, cand;
        classify(code, idx, valid, win, cand);
        if constexpr (DF != 3) hist_cand(code, idx, cand);
        const int tg = (win || cand) ? tag_of(code, idx) : 2;
        push1(tg != 2, tg, code, idx);
      }
    };
    for (int64_t hb = 0; hb < head; hb += BLOCK)
      if (c.slice == 0) process_scalar(hb + tid, hb + tid < head);
    for (int64_t tb = tail0; tb < c.len; tb += BLOCK)
      if (c.slice == c.nslices - 1) process_scalar(tb + tid, tb + tid < c.len);
  } else {
    // ---- source = candidate buffer written by the previous pass (codes + indices) ----
    const unsigned long long n = c.nbuf;
    const unsigned long long per = (n + c.nslices - 1) / c.nslices;
    const unsigned long long e0 = std::min<unsigned long long>(n, (unsigned long long)c.slice * per);
    const unsigned long long e1 = std::min<unsigned long long>(n, e0 + per);
    nread = n;
    if constexpr (DF == 0) {
      for (unsigned long long base = e0; base < e1; base += BLOCK) {
        const unsigned long long i = base + tid;
        const bool valid = i < e1;
        const U code = valid ? c.bcin[i] : (U)0;
        shared_inc(hbase + 4u * (valid ? (unsigned)(((W)code >> shh) & hmask) : (unsigned)kDummyBin));
      }
    } else if constexpr (DF != 3) {
      // BU coalesced entries per thread per iteration, all loads issued up front
      for (unsigned long long base = e0; base < e1; base += (unsigned long long)BLOCK * BU) {
        U code[BU];
        IdxT idx[BU];
#pragma unroll
        for (int j = 0; j < BU; ++j) {
          const unsigned long long i = base + (unsigned long long)j * BLOCK + tid;
          code[j] = (i < e1) ? c.bcin[i] : (U)0;
          idx[j] = (i < e1) ? c.biin[i] : (IdxT)0;
        }
#pragma unroll
        for (int j = 0; j < BU; ++j) {
          const bool valid = base + (unsigned long long)j * BLOCK + tid < e1;
          bool win, cand;
          classify(code[j], idx[j], valid, win, cand);
          hist_cand(code[j], idx[j], cand);
          push1(win || (cand && store), win ? 0 : 1, code[j], idx[j]);
        }
        pass_dbg(c.dbg, 0);
      }
    }
  }
  pass_dbg(c.dbg, 1);
  if constexpr (DF != 0) {
    // final flush of the partial queues, aggregated over the CTA: one global atomic per CTA and
    // destination instead of one per warp (same-address atomics serialise in L2: ~1 per ns)
    static_assert(NW <= 32, "one warp scans the per-warp counts");
    __shared__ unsigned long long s_base[2][NW];
    __shared__ unsigned s_n[NW];
    __syncwarp();
    const unsigned cnt = wq_counts(wq, qcnt);
    if (lane == 0) s_n[warp] = cnt;
    __syncthreads();
    if (warp == 0) {
      const unsigned x = (lane < NW) ? s_n[lane] : 0u;  // (results | candidates << 16) per warp
      unsigned incl = x;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned y = __shfl_up_sync(kFull, incl, o);
        if (lane >= o) incl += y;
      }
      const unsigned total = __shfl_sync(kFull, incl, 31);  // per-field sums < 2^16 (NW x kCap)
      unsigned long long b = 0;
      if (lane == 0 && (total & 0xffffu)) b = atomicAdd(c.outc, (unsigned long long)(total & 0xffffu));
      if (lane == 1 && (total >> 16)) b = atomicAdd(c.bufc, (unsigned long long)(total >> 16));
      const unsigned long long br = __shfl_sync(kFull, b, 0), bcb = __shfl_sync(kFull, b, 1);
      const unsigned ex = incl - x;
      if (lane < NW) {
        s_base[0][lane] = br + (ex & 0xffffu);
        s_base[1][lane] = bcb + (ex >> 16);
      }
    }
    __syncthreads();
    pass_dbg(c.dbg, 2);
    if (qcnt)
      wq_write<KIND, IdxT>(wq, qcnt, s_base[0][warp], s_base[1][warp], c.ov, c.oi, c.kk, c.bco, c.bio, c.capa,
                           sel_min, c.err, c.ioff);
    pass_dbg(c.dbg, 3);
  }
  if constexpr (DF == 3) {  // one atomic per warp: window-member extremes (the tail skips digits
                            // on which all members agree)
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const W a = shfl(wlo_seen, (lane + o) & 31), b = shfl(whi_seen, (lane + o) & 31);
      wlo_seen = a < wlo_seen ? a : wlo_seen;
      whi_seen = b > whi_seen ? b : whi_seen;
    }
    if (lane == 0 && whi_seen >= wlo_seen) {
      atomicMax(c.wnmin, ~(unsigned long long)wlo_seen);
      atomicMax(c.wmax, (unsigned long long)whi_seen);
    }
  }
  return nread;
}

// Single-CTA finish of a row: pass q reads a buffer of n <= kSmallFinish
// entries, all sharing the prefix of digits < q-1. Its filter of digit q-1 (Alg1 L15-22) emits the
// entries below the target digit j; among the C entries with digit q-1 == j the K smallest composite
// keys (code, index) — the lowest-index rule of reading 1 — are the rest of the result. With C small
// these are found by rank counting in shared memory instead of the remaining radix passes
// (rank(e) = #{e' : (code', idx') < (code, idx)}; keys are unique, so exactly K ranks are < K).
// The caller ends the row (grid engine: stop1 = q, so every later launch returns at once).
// sc, si: shared arrays of at least c.nbuf codes / indices.
template <int KIND, typename IdxT, int BLOCK>
__device__ void small_finish(const PassCtx<typename KT<KIND>::U, IdxT>& c, unsigned long long Kr,
                             typename KT<KIND>::U* sc, IdxT* si) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  __shared__ unsigned s_m;
  const int tid = threadIdx.x, lane = tid & 31;
  const int n = (int)c.nbuf;
  const Digit df = c.df;
  const unsigned long long jprev = (df.is_idx ? c.tidx : c.tcode) >> df.shift & ((1ull << df.width) - 1ull);
  if (tid == 0) s_m = 0;
  __syncthreads();
  auto emit = [&](bool pred, U code, IdxT idx) {  // warp-aggregated result append
    const unsigned m = __ballot_sync(kFull, pred);
    if (!m) return;
    unsigned long long b = 0;
    if (lane == 0) b = atomicAdd(c.outc, (unsigned long long)__popc(m));
    b = __shfl_sync(kFull, b, 0);
    if (pred) {
      const unsigned long long pos = b + __popc(m & lanemask_lt());
      if (pos < c.kk) {
        c.ov[pos] = from_code<KIND>(code, c.sel_min);
        c.oi[pos] = (int64_t)idx + c.ioff;
      } else {
        atomicOr(c.err, 1u);
      }
    }
  };
  for (int b0 = 0; b0 < n; b0 += BLOCK) {
    const int i = b0 + tid;
    const bool valid = i < n;
    const U code = valid ? c.bcin[i] : (U)0;
    const IdxT idx = valid ? c.biin[i] : (IdxT)0;
    const unsigned long long d = (df.is_idx ? (unsigned long long)idx : (unsigned long long)(W)code) >> df.shift &
                                 ((1ull << df.width) - 1ull);
    emit(valid && d < jprev, code, idx);
    const bool eq = valid && d == jprev;
    const unsigned m = __ballot_sync(kFull, eq);
    unsigned b = 0;
    if (lane == 0 && m) b = atomicAdd(&s_m, (unsigned)__popc(m));
    b = __shfl_sync(kFull, b, 0);
    if (eq) {
      const unsigned pos = b + __popc(m & lanemask_lt());
      sc[pos] = code;
      si[pos] = idx;
    }
  }
  __syncthreads();
  const int m = (int)s_m;
  for (int b0 = 0; b0 < m; b0 += BLOCK) {
    const int i = b0 + tid;
    bool sel = false;
    U code = 0;
    IdxT idx = 0;
    if (i < m) {
      code = sc[i];
      idx = si[i];
      unsigned long long rank = 0;
      if ((unsigned long long)m > Kr)
        for (int t = 0; t < m; ++t) rank += (sc[t] < code) || (sc[t] == code && si[t] < idx);
      sel = rank < Kr;
    }
    emit(sel, code, idx);
  }
  if (tid == 0 && (unsigned long long)m < Kr) atomicOr(c.err, 4u);
  __syncthreads();
}

}  // namespace airtopk
