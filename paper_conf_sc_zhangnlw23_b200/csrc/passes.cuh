// passes.cuh — the streaming body of one AIR Top-K pass, shared by both engines.
//
// One call processes this CTA's slice of the pass source (Alg1 L7-8: the input row L or the
// candidate buffer of the previous pass) and performs, per element,
//   DF (digit filtered, Alg1 L15-22): results (digit < target) -> output V/I; candidates
//       (digit == target) -> candidate buffer if C < N/alpha (L17-18);
//   DH (digit histogrammed, L12-13 / L19-20): candidates counted in the shared histogram.
// DF/DH: 0 none, 1 key digit, 2 index digit (the lowest-index tie-break digits).
//
// B200 choices (measured): 4 x 128-bit ld.global.nc.L1::no_allocate per
// thread in flight; per-element work is 3-4 integer ops and a predicated shared atomic
// (ATOMS.POPC.INC aggregates equal addresses within a warp); results/candidates, rare in most
// passes, leave through per-warp shared queues flushed with one global atomic per 64 entries and
// coalesced stores; the flagged element is re-read from L2 in the slow path so the tile registers
// die early (40 registers -> 3 CTAs x 512 threads per SM, no spills).
#pragma once

#include <algorithm>
#include <type_traits>

#include "device.cuh"
#include "tma.cuh"
#include <cuda_bf16.h>
#include <cuda_fp16.h>

namespace airtopk {

#ifndef AIRTOPK_SLOW_REG
#define AIRTOPK_SLOW_REG 0
#endif
#ifndef AIRTOPK_PREFETCH
#define AIRTOPK_PREFETCH 0
#endif
#ifndef AIRTOPK_UNROLL
#define AIRTOPK_UNROLL 4
#endif
constexpr int kUnroll = AIRTOPK_UNROLL;
constexpr int kQCap = 64;
constexpr int kTmaStages = 4;  // per-warp ring depth of the bulk-copy streaming loop
// Copies of the shared histogram in the filter passes: lane l counts into copy l % kHistCopies
// (interleaved bin-major so copies of one bin sit in different banks); cuts the same-address
// serialisation of shared atomics when many lanes hit a few bins (radix-adversarial passes).
constexpr int kHistCopies = 4;
// Extra histogram slot that absorbs the atomics of non-candidates / invalid lanes (never scanned).
constexpr int kDummyBin = kMaxBins;
constexpr int kHistSlots = kMaxBins + 32;  // per copy; the dummy bin + padding

// Conservative window prefilter for IEEE keys: true when some element of the tile may have
// code <= whi, by a floating-point compare against hv = the key whose code is whi (select-min;
// select-max mirrors it). x <=_total hv implies !(x >_fp hv): the IEEE total order refines the fp
// order (-0 < +0 only in the former) and every compare with a NaN is false, so no result or window
// member is missed; a false positive only sends the tile through the exact classification.
template <int KIND, bool SELMIN, int N>
__device__ __forceinline__ bool tile_maybe_le(const uint4 (&r)[N], uint32_t hv2) {
  if constexpr (KIND == K_F32) {
    const float h = __uint_as_float(hv2);
    bool any = false;
#pragma unroll
    for (int u = 0; u < N; ++u) {
      const uint32_t w[4] = {r[u].x, r[u].y, r[u].z, r[u].w};
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float x = __uint_as_float(w[e]);
        any |= SELMIN ? !(x > h) : !(x < h);
      }
    }
    return any;
  } else {
    unsigned acc = 0;
#pragma unroll
    for (int u = 0; u < N; ++u) {
      const uint32_t w[4] = {r[u].x, r[u].y, r[u].z, r[u].w};
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        if constexpr (KIND == K_F16) {
          const __half2 x = __halves2half2(__ushort_as_half((unsigned short)(w[e] & 0xffffu)),
                                           __ushort_as_half((unsigned short)(w[e] >> 16)));
          const __half2 h = __halves2half2(__ushort_as_half((unsigned short)(hv2 & 0xffffu)),
                                           __ushort_as_half((unsigned short)(hv2 >> 16)));
          acc |= SELMIN ? __hleu2_mask(x, h) : __hgeu2_mask(x, h);
        } else {
          const __nv_bfloat162 x = __halves2bfloat162(__ushort_as_bfloat16((unsigned short)(w[e] & 0xffffu)),
                                                      __ushort_as_bfloat16((unsigned short)(w[e] >> 16)));
          const __nv_bfloat162 h = __halves2bfloat162(__ushort_as_bfloat16((unsigned short)(hv2 & 0xffffu)),
                                                      __ushort_as_bfloat16((unsigned short)(hv2 >> 16)));
          acc |= SELMIN ? __hleu2_mask(x, h) : __hgeu2_mask(x, h);
        }
      }
    }
    return acc != 0;
  }
}

// +1 on a shared-window address (no return value): red.shared.add, which the hardware aggregates
// over lanes hitting the same address.
__device__ __forceinline__ void shared_inc(unsigned addr) {
  asm volatile("red.shared.add.u32 [%0], 1;" ::"r"(addr) : "memory");
}

template <typename U, typename IdxT>
struct WarpQ {
  static constexpr int kCap = (sizeof(U) + sizeof(IdxT) <= 8) ? kQCap : kQCap / 2;
  U code[kCap];
  IdxT idx[kCap];
};

template <int KIND, typename IdxT, int DF>
__host__ __device__ constexpr int hist_copies() {
  using U = typename KT<KIND>::U;
  return (DF == 0 || DF == 3) ? 1 : (sizeof(U) + sizeof(IdxT) <= 8 ? kHistCopies : 2);
}

// Store a warp queue's n entries at [base, base + n) of the destination (coalesced); entries at or
// beyond `limit` set the overflow flag instead. Out of line so the streaming loop stays small
// (I-cache). mode 0: results (value bits + int64 index), 1: candidates (code + index).
template <int KIND, typename IdxT>
__device__ __noinline__ void wq_write(const WarpQ<typename KT<KIND>::U, IdxT>* wq, int n, unsigned long long base,
                                      unsigned long long limit, typename KT<KIND>::U* dst_code, void* dst_idx,
                                      int mode, bool sel_min, unsigned* err) {
  const int lane = threadIdx.x & 31;
  for (int j = lane; j < n; j += 32) {
    const unsigned long long pos = base + j;
    if (pos < limit) {
      if (mode == 0) {
        dst_code[pos] = from_code<KIND>(wq->code[j], sel_min);
        ((int64_t*)dst_idx)[pos] = (int64_t)wq->idx[j];
      } else {
        dst_code[pos] = wq->code[j];
        ((IdxT*)dst_idx)[pos] = wq->idx[j];
      }
    } else {
      *err = mode == 0 ? 1u : 2u;
    }
  }
}

// Flush a full warp queue: ONE global atomic reserves n slots, then coalesced stores.
template <int KIND, typename IdxT>
__device__ __noinline__ void wq_flush(const WarpQ<typename KT<KIND>::U, IdxT>* wq, int n, unsigned long long* counter,
                                      unsigned long long limit, typename KT<KIND>::U* dst_code, void* dst_idx,
                                      int mode, bool sel_min, unsigned* err) {
  const int lane = threadIdx.x & 31;
  unsigned long long base = 0;
  if (lane == 0) base = atomicAdd(counter, (unsigned long long)n);
  base = __shfl_sync(kFull, base, 0);
  wq_write<KIND, IdxT>(wq, n, base, limit, dst_code, dst_idx, mode, sel_min, err);
}

// Warp-collective append of the lanes with `pred` to a shared-memory queue (flushes when full).
template <int KIND, typename IdxT>
__device__ __forceinline__ void wq_push(WarpQ<typename KT<KIND>::U, IdxT>* wq, int& cnt, bool pred,
                                        typename KT<KIND>::U code, IdxT idx, unsigned long long* counter,
                                        unsigned long long limit, typename KT<KIND>::U* dst_code, void* dst_idx,
                                        int mode, bool sel_min, unsigned* err) {
  const unsigned m = __ballot_sync(kFull, pred);
  if (!m) return;
  const int n = __popc(m);
  if (cnt + n > WarpQ<typename KT<KIND>::U, IdxT>::kCap) {
    __syncwarp();
    wq_flush<KIND, IdxT>(wq, cnt, counter, limit, dst_code, dst_idx, mode, sel_min, err);
    cnt = 0;
    __syncwarp();
  }
  if (pred) {
    const int pos = cnt + __popc(m & lanemask_lt());
    wq->code[pos] = code;
    wq->idx[pos] = idx;
  }
  cnt += n;
}

// Element b (0 .. kUnroll*VEC-1) of a thread's tile registers, selected without local memory.
template <typename U>
__device__ __forceinline__ U tile_elem(const uint4 (&r)[kUnroll], int b) {
  constexpr int VEC = 16 / sizeof(U);
  const int u = b / VEC, e = b % VEC;
  uint4 v = r[0];
#pragma unroll
  for (int i = 1; i < kUnroll; ++i) v = (u == i) ? r[i] : v;
  U out = vec_elem<U>(v, 0);
#pragma unroll
  for (int i = 1; i < VEC; ++i) out = (e == i) ? vec_elem<U>(v, i) : out;
  return out;
}

// Everything one pass of one row needs (built by the engine from its copy of the row state).
template <typename U, typename IdxT>
struct PassCtx {
  int q;
  bool emit_all, do_hist, srcL, store, sel_min, reverse;
  Digit dh, df;
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
  unsigned ring, bars;  // TMA streaming: shared-window addresses of the warp rings and their mbarriers
  WarpQ<U, IdxT>* oq;
  WarpQ<U, IdxT>* bq;
};

// Runs the pass over this CTA's slice; all queues are flushed on return. Returns the number of
// elements of the whole source (for the trace).
template <int KIND, typename IdxT, int DF, int DH, bool HASIDX, int BLOCK, int HCOPIES = 0, bool TMA = false,
          int BU = 4>
__device__ __forceinline__ unsigned long long run_pass(const PassCtx<typename KT<KIND>::U, IdxT>& c) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;  // shifted-key width
  constexpr int VEC = 16 / sizeof(U);
  constexpr int HC = HCOPIES > 0 ? HCOPIES : hist_copies<KIND, IdxT, DF>();  // histogram copies
  const int tid = threadIdx.x, lane = tid & 31;

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
  const unsigned hbase = (unsigned)__cvta_generic_to_shared(c.hist) + ((HC > 1) ? (unsigned)(lane % HC) * 4u : 0u);
  const U xmask = sel_min ? (U)0 : (U)~(U)0;
  int ocnt = 0, bcnt = 0;
  W wlo_seen = ~(W)0, whi_seen = 0;  // DF == 3: extremes of this thread's window members

  auto push_out = [&](bool pred, U code, IdxT idx) {
    wq_push<KIND, IdxT>(c.oq, ocnt, pred, code, idx, c.outc, c.kk, c.ov, c.oi, 0, sel_min, c.err);
  };
  auto push_buf = [&](bool pred, U code, IdxT idx) {
    wq_push<KIND, IdxT>(c.bq, bcnt, pred, code, idx, c.bufc, c.capa, c.bco, c.bio, 1, sel_min, c.err);
  };
  // Filter classification of digit q-1 (Alg1 L15-22): win = result, cand = candidate for pass q.
  const W wlo = (W)c.lo, wspan = (W)c.span1;
  const W whi = (W)(wlo + wspan - 1);  // DF == 3: window [lo, hi]
  // DF == 3 prefilter: the key whose code is whi (16-bit keys: in both halves)
  const uint32_t hv2 = (sizeof(U) == 2) ? ((uint32_t)from_code<KIND>((U)whi, sel_min) * 0x10001u)
                                        : (uint32_t)from_code<KIND>((U)whi, sel_min);
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
  // is aggregated by the shared atomic unit (ATOMS.POPC.INC), so the common "no candidate" case is
  // one cheap atomic and no divergence.
  auto hist_cand = [&](U code, IdxT idx, bool cand) {
    unsigned d;
    if constexpr (DH == 2) d = (unsigned)(idx >> shh) & hmask;
    else d = (unsigned)((W)code >> shh) & hmask;
    d = (cand && do_hist) ? d : (unsigned)kDummyBin;
    shared_inc(hbase + d * (HC * 4));
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

    // One thread's tile: kUnroll 16-byte vectors at vector indices vb + u*BLOCK. FULL: all valid.
    // vs = distance (in 16-byte vectors) between a thread's kUnroll vectors: BLOCK for CTA tiles read
    // with registers, 32 for warp tiles staged through shared memory by the bulk-copy engine
    // sstage: shared-window address of the warp's staged tile (TMA path) or 0 (register path): the
    // slow path then re-reads a flagged element from shared memory instead of L2
    auto process_tile = [&](const uint4 (&r)[kUnroll], int64_t vb, int64_t vlim, auto full_tag, int64_t vs,
                            unsigned sstage) {
      constexpr bool FULL = decltype(full_tag)::value;
      if constexpr (DF == 0) {
        // pass 1: the top digit needs no mask (code >> shh < 2^11)
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          const bool valid = FULL || (vb + (int64_t)u * vs < vlim);
#pragma unroll
          for (int e = 0; e < VEC; ++e) {
            const U code = to_code_x<KIND>(vec_elem<U>(r[u], e), xmask);
            const unsigned d = (unsigned)((W)code >> shh);
            shared_inc(hbase + 4u * (valid ? d : (unsigned)kDummyBin));
          }
        }
        return;
      }
      using FlagT = std::conditional_t<(kUnroll * VEC > 32), unsigned long long, unsigned>;
      FlagT fl = 0;  // elements that must leave through the queues (results / stored candidates)
      if constexpr (DF == 3) {
        // window pass: results below the window -> output, window members -> candidate buffer and
        // (slow path) the pass-1 histogram of the window members; a miss re-runs the paper's pass 1.
        // Floating-point keys first take one conservative fp compare per element (two per HSETP2 for
        // 16-bit keys): almost every tile holds neither result nor window member.
        bool maybe = true;  // (no early return: the whole warp must reach the slow-path votes)
        if constexpr (FULL && (KIND == K_F32 || KIND == K_F16 || KIND == K_BF16))
          maybe = sel_min ? tile_maybe_le<KIND, true>(r, hv2) : tile_maybe_le<KIND, false>(r, hv2);
        if (maybe) {
#pragma unroll
          for (int u = 0; u < kUnroll; ++u) {
            const bool valid = FULL || (vb + (int64_t)u * vs < vlim);
#pragma unroll
            for (int e = 0; e < VEC; ++e) {
              const U code = to_code_x<KIND>(vec_elem<U>(r[u], e), xmask);
              // result (code < lo) or window member (lo <= code <= hi): together simply code <= hi
              if (valid && (W)code <= whi) fl |= (FlagT)1 << (u * VEC + e);
            }
          }
        }
      } else if constexpr (DF == 1 && DH == 1) {
        // adjacent key digits: y = (code >> shh) - B places the elements whose higher digits match
        // the prefix at [S, S + nb) and the results below S (see the derivation at kx_* below)
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
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
        for (int u = 0; u < kUnroll; ++u) {
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
      // slow path (rare in most passes): results / candidates through the warp queues. The flagged
      // element is re-read (an L2 hit: this warp just streamed it) and re-classified, so the tile
      // registers die early.
      while (__any_sync(kFull, fl != 0)) {
        const bool has = fl != 0;
        const int b = has ? ((sizeof(FlagT) == 8) ? __ffsll((long long)fl) : __ffs((int)fl)) - 1 : 0;
        fl &= fl - 1;
        const int64_t pos = head + (vb + (int64_t)(b / VEC) * vs) * VEC + (b % VEC);
        U raw = 0;
        if (has) {
          if (TMA && sstage) {
            const unsigned a = sstage + (unsigned)((((b / VEC) * 32 + lane) * 16) + (b % VEC) * (int)sizeof(U));
            if constexpr (sizeof(U) == 2) { unsigned short t; asm volatile("ld.shared.u16 %0, [%1];" : "=h"(t) : "r"(a)); raw = (U)t; }
            else if constexpr (sizeof(U) == 4) { unsigned t; asm volatile("ld.shared.u32 %0, [%1];" : "=r"(t) : "r"(a)); raw = (U)t; }
            else { unsigned long long t; asm volatile("ld.shared.u64 %0, [%1];" : "=l"(t) : "r"(a)); raw = (U)t; }
          } else {
#if AIRTOPK_SLOW_REG
            raw = tile_elem<U>(r, b);
#else
            raw = __ldcg(rowp + pos);
#endif
          }
        }
        const U code = to_code_x<KIND>(raw, xmask);
        const IdxT idx = has ? index_of(pos) : (IdxT)0;
        bool w, cd;
        classify(code, idx, has, w, cd);
        if constexpr (DF == 3) {
          if (cd) {  // window member: extremes + the pass-1 digit histogram of the window buffer
            wlo_seen = ((W)code < wlo_seen) ? (W)code : wlo_seen;
            whi_seen = ((W)code > whi_seen) ? (W)code : whi_seen;
            shared_inc(hbase + 4u * (unsigned)((W)code >> shh));
          }
        }
        push_out(w, code, idx);
        if (store) push_buf(cd, code, idx);
      }
    };

    // Grid-stride tile order: tile t (BLOCK*kUnroll 16-byte vectors, 32 KiB for 512 threads) goes to
    // slice t mod nslices, so at any moment the CTAs of a row read one compact, advancing region of
    // HBM. Measured on B200: zero DRAM over-fetch and 7.2-7.4 TB/s, vs 9% over-fetch and 6.3 TB/s
    // when every CTA streams its own contiguous chunk (tools/microbench_hist.cu, profiles/).
    // `reverse` walks the tiles backwards (odd passes consume the tail the previous pass left in L2).
    if constexpr (TMA) {
      // Warp tiles of 32 x kUnroll 16-byte vectors (2 KiB for f32) in grid-stride order over all
      // warps of the row's CTAs; each warp streams its tiles through its own NST-stage shared ring
      // filled by the bulk-copy engine (lane 0 issues, the stage's mbarrier counts the bytes).
      constexpr int NW = BLOCK / 32;
      constexpr int64_t WT = 32 * kUnroll;
      constexpr unsigned WT_BYTES = (unsigned)(WT * 16);
      const int warp = tid >> 5;
      const int64_t G = (int64_t)c.nslices * NW, g = (int64_t)c.slice * NW + warp;
      const int64_t nwt = nvec / WT;
      const int64_t mine = (nwt > g) ? (nwt - 1 - g) / G + 1 : 0;
      auto wtile = [&](int64_t i) { return g + (c.reverse ? (mine - 1 - i) : i) * G; };
      const unsigned ring = c.ring + (unsigned)warp * (unsigned)(kTmaStages * WT_BYTES);
      const unsigned bars = c.bars + (unsigned)warp * (unsigned)(kTmaStages * 8);
      if (lane == 0) {
        for (int st = 0; st < kTmaStages; ++st) mbar_init(bars + 8u * st, 1);
        fence_mbar_init();
        for (int st = 0; st < kTmaStages && st < mine; ++st) {
          mbar_arrive_expect_tx(bars + 8u * st, WT_BYTES);
          bulk_g2s(ring + st * WT_BYTES, vp + wtile(st) * WT, WT_BYTES, bars + 8u * st);
        }
      }
      __syncwarp();
      for (int64_t i = 0; i < mine; ++i) {
        const int st = (int)(i % kTmaStages);
        mbar_wait(bars + 8u * st, (unsigned)((i / kTmaStages) & 1));
        uint4 r[kUnroll];
        const unsigned sbase = ring + st * WT_BYTES;
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) r[u] = lds128(sbase + (unsigned)((u * 32 + lane) * 16));
        process_tile(r, wtile(i) * WT + lane, nvec, std::true_type{}, (int64_t)32, sbase);
        __syncwarp();
        if (lane == 0 && i + kTmaStages < mine) {  // refill the consumed stage (kTmaStages-1 in flight)
          fence_proxy_async_smem();
          mbar_arrive_expect_tx(bars + 8u * st, WT_BYTES);
          bulk_g2s(sbase, vp + wtile(i + kTmaStages) * WT, WT_BYTES, bars + 8u * st);
        }
      }
      if (nwt * WT < nvec && g == (nwt % G)) {  // the partial last warp tile
        const int64_t vb = nwt * WT + lane;
        uint4 r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          const int64_t v = vb + (int64_t)u * 32;
          r[u] = (v < nvec) ? ldg_stream(vp + v) : make_uint4(0, 0, 0, 0);
        }
        process_tile(r, vb, nvec, std::false_type{}, (int64_t)32, 0u);
      }
    } else {
      const int64_t tile = (int64_t)BLOCK * kUnroll;
      const int64_t ntiles = nvec / tile;
      const int64_t mine = (ntiles > c.slice) ? (ntiles - 1 - c.slice) / c.nslices + 1 : 0;
  #if AIRTOPK_PREFETCH
      // software pipeline: the next tile's loads are in flight while this tile is classified
      if (mine > 0) {
        auto tile_of = [&](int64_t i) { return (int64_t)c.slice + (c.reverse ? (mine - 1 - i) : i) * c.nslices; };
        uint4 r[kUnroll];
        int64_t vb = tile_of(0) * tile + tid;
  #pragma unroll
        for (int u = 0; u < kUnroll; ++u) r[u] = ldg_stream(vp + vb + (int64_t)u * BLOCK);
        for (int64_t i = 0; i < mine; ++i) {
          uint4 nx[kUnroll];
          const int64_t vbn = (i + 1 < mine) ? tile_of(i + 1) * tile + tid : vb;
  #pragma unroll
          for (int u = 0; u < kUnroll; ++u) nx[u] = ldg_stream(vp + vbn + (int64_t)u * BLOCK);
          process_tile(r, vb, nvec, std::true_type{}, (int64_t)BLOCK, 0u);
  #pragma unroll
          for (int u = 0; u < kUnroll; ++u) r[u] = nx[u];
          vb = vbn;
        }
      }
  #else
      for (int64_t i = 0; i < mine; ++i) {
        const int64_t t = (int64_t)c.slice + (c.reverse ? (mine - 1 - i) : i) * c.nslices;
        const int64_t vb = t * tile + tid;
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
        if constexpr (DF == 3) {
          if (cand) {
            wlo_seen = ((W)code < wlo_seen) ? (W)code : wlo_seen;
            whi_seen = ((W)code > whi_seen) ? (W)code : whi_seen;
            shared_inc(hbase + 4u * (unsigned)((W)code >> shh));
          }
        }
        push_out(win, code, idx);
        if (store) push_buf(cand, code, idx);
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
          push_out(win, code[j], idx[j]);
          if (store) push_buf(cand, code[j], idx[j]);
        }
      }
    }
  }
  if constexpr (DF != 0) {
    // final flush of the partial queues, aggregated over the CTA: one global atomic per CTA and
    // destination instead of one per warp (same-address atomics serialise in L2: ~1 per ns)
    constexpr int NW = BLOCK / 32;
    static_assert(NW <= 32, "one warp scans the per-warp counts");
    __shared__ unsigned long long s_base[2][NW];
    __shared__ int s_n[2][NW];
    __syncwarp();
    if (lane == 0) {
      s_n[0][tid >> 5] = ocnt;
      s_n[1][tid >> 5] = bcnt;
    }
    __syncthreads();
    if ((tid >> 5) == 0) {
#pragma unroll
      for (int mode = 0; mode < 2; ++mode) {
        const unsigned x = (lane < NW) ? (unsigned)s_n[mode][lane] : 0u;
        unsigned incl = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const unsigned y = __shfl_up_sync(kFull, incl, o);
          if (lane >= o) incl += y;
        }
        const unsigned total = __shfl_sync(kFull, incl, 31);
        unsigned long long b = 0;
        if (lane == 0 && total) b = atomicAdd(mode ? c.bufc : c.outc, (unsigned long long)total);
        b = __shfl_sync(kFull, b, 0);
        if (lane < NW) s_base[mode][lane] = b + (incl - x);
      }
    }
    __syncthreads();
    if (ocnt) wq_write<KIND, IdxT>(c.oq, ocnt, s_base[0][tid >> 5], c.kk, c.ov, c.oi, 0, sel_min, c.err);
    if (bcnt) wq_write<KIND, IdxT>(c.bq, bcnt, s_base[1][tid >> 5], c.capa, c.bco, c.bio, 1, sel_min, c.err);
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

}  // namespace airtopk
