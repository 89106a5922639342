// device.cuh — device building blocks of the B200 AIR Top-K path (sm_100a).
//
// Paper: Zhang et al., "Parallel Top-K Algorithms on GPU", SC'23 — /root/reference/PAPER.md ("P:n").
// This header holds the per-element arithmetic every kernel shares:
//   * the order-preserving key transform ("binary representation"; reading 3/4 in DESIGN.md),
//   * the digit schedule: r key bits MSB-first in b = 11-bit digits, followed by the
//     row-index bits (the lowest-index tie-break realised as extra radix digits, reading 1),
//   * the filter classification of Algorithm 1 lines 15-22,
//   * warp-aggregated output/candidate appends and shared-memory histogram updates,
//   * the inclusive prefix sum + target-digit search of Algorithm 1 lines 24-28.
// Nothing here is shared with oracle/ (which has its own, independent implementation).
#pragma once

#include <cstdint>
#include <type_traits>
#include <cuda_runtime.h>

namespace airtopk {

constexpr int kDigitBits = 11;                  // b = 11
constexpr int kMaxBins = 1 << kDigitBits;       // 2048 histogram counters
constexpr unsigned kFull = 0xffffffffu;
constexpr int kTraceFields = 10;
constexpr int kTraceMaxPasses = 16;

enum Kind : int { K_F32 = 0, K_F16 = 1, K_BF16 = 2, K_F64 = 3, K_U32 = 4 };

template <int KIND> struct KT;
template <> struct KT<K_F32> { using U = uint32_t; static constexpr int R = 32; static constexpr bool IEEE = true; };
template <> struct KT<K_F16> { using U = uint16_t; static constexpr int R = 16; static constexpr bool IEEE = true; };
template <> struct KT<K_BF16> { using U = uint16_t; static constexpr int R = 16; static constexpr bool IEEE = true; };
template <> struct KT<K_F64> { using U = uint64_t; static constexpr int R = 64; static constexpr bool IEEE = true; };
template <> struct KT<K_U32> { using U = uint32_t; static constexpr int R = 32; static constexpr bool IEEE = false; };

// Order-preserving code: negative IEEE values have all bits flipped, non-negative ones get the
// sign bit set; the unsigned order of codes is then the IEEE total order. Select-max complements
// the code (the paper's "smallest without loss of generality").
template <int KIND>
__device__ __forceinline__ typename KT<KIND>::U to_code(typename KT<KIND>::U b, bool sel_min) {
  using U = typename KT<KIND>::U;
  U c;
  if constexpr (KT<KIND>::IEEE) {
    constexpr U sign = U(U(1) << (KT<KIND>::R - 1));
    c = (b & sign) ? U(~b) : U(b | sign);
  } else {
    c = b;
  }
  return sel_min ? c : U(~c);
}

// Branch-free form of to_code for the streaming loops: xmask = 0 (select-min) or all ones
// (select-max). b ^ (sign-extended sign | sign bit): flips every bit of negatives, sets the sign bit of
// non-negatives.
template <int KIND>
__device__ __forceinline__ typename KT<KIND>::U to_code_x(typename KT<KIND>::U b, typename KT<KIND>::U xmask) {
  using U = typename KT<KIND>::U;
  if constexpr (KT<KIND>::IEEE) {
    using S = std::make_signed_t<U>;
    constexpr U sign = U(U(1) << (KT<KIND>::R - 1));
    const U m = (U)((S)b >> (KT<KIND>::R - 1));
    return U(b ^ (m | sign) ^ xmask);
  } else {
    return U(b ^ xmask);
  }
}

template <int KIND>
__device__ __forceinline__ typename KT<KIND>::U from_code(typename KT<KIND>::U c, bool sel_min) {
  using U = typename KT<KIND>::U;
  if (!sel_min) c = U(~c);
  if constexpr (KT<KIND>::IEEE) {
    constexpr U sign = U(U(1) << (KT<KIND>::R - 1));
    return (c & sign) ? U(c & U(~sign)) : U(~c);
  } else {
    return c;
  }
}

// Digit q of the composite key (code : R bits || index : IB bits), most significant first.
struct Digit {
  int is_idx;
  int shift;
  int width;
};

__host__ __device__ __forceinline__ int code_passes(int R) { return (R + kDigitBits - 1) / kDigitBits; }
__host__ __device__ __forceinline__ int idx_passes(int IB) { return (IB + kDigitBits - 1) / kDigitBits; }

__host__ __device__ __forceinline__ Digit digit_of(int q, int R, int IB) {
  const int pc = code_passes(R);
  if (q < pc) {
    const int hi = R - kDigitBits * q;
    const int w = hi < kDigitBits ? hi : kDigitBits;
    return Digit{0, hi - w, w};
  }
  const int hi = IB - kDigitBits * (q - pc);
  const int w = hi < kDigitBits ? hi : kDigitBits;
  return Digit{1, hi - w, w};
}

// Per-row state shared by the CTAs of one row (the paper's K, C, C', target digit, Alg1 L1/L23-28).
// Zeroed by the launcher before the first kernel; "npass" = number of scans done so far.
struct alignas(128) RowState {
  unsigned long long K;          // remaining K after the last scan
  unsigned long long C;          // candidates of the next pass = hist[j] of the last scan
  unsigned long long Cp;         // C' = candidates counted by the last scan (C before it)
  unsigned long long tcode;      // fixed code bits (digits 0..npass-1 at their positions)
  unsigned long long tidx;       // fixed index bits
  unsigned long long out_count;  // results emitted so far
  unsigned long long buf_count[2];
  unsigned int ticket;           // "last thread block" detector
  int npass;
  int stop1;                     // 1 + pass after whose scan K == C (early stop); 0 = none
  unsigned int j;
  unsigned int error;            // 1 = output overflow (duplicate in_idx), 2 = buffer overflow
  int src1;                      // source of the next pass: 0 = input row L, s + 1 = buffer slot s
  int win_state;                 // sample-guided window: 0 off, 1 window holds the K-th key, 2 failed
  unsigned long long win_lo, win_hi;  // window [lo, hi] of codes chosen from the sample
  unsigned long long win_nmin, win_max;  // ~min and max code of the window members (atomicMax)
};

// no-op debug-stamp callback (kernels take a Stamp functor for optional %globaltimer stamps)
struct NoStamp {
  __device__ void operator()(int) const {}
};

template <typename T>
__device__ __forceinline__ T shfl(T v, int src) {
  if constexpr (sizeof(T) == 8) {
    unsigned long long x = (unsigned long long)v;
    return (T)__shfl_sync(kFull, x, src);
  } else {
    return (T)__shfl_sync(kFull, (unsigned)v, src);
  }
}

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

// Warp-aggregated slot allocation: one atomic per warp and predicate instead of one per element.
// Must be called by all 32 lanes. Returns the slot of this lane (valid only where pred).
__device__ __forceinline__ unsigned long long warp_alloc(bool pred, unsigned long long* counter, unsigned& mask) {
  mask = __ballot_sync(kFull, pred);
  unsigned long long base = 0;
  if (mask) {
    const int leader = __ffs(mask) - 1;
    if (lane_id() == leader) base = atomicAdd(counter, (unsigned long long)__popc(mask));
    base = __shfl_sync(kFull, base, leader);
  }
  return base + __popc(mask & lanemask_lt());
}

// "Last thread block" ticket: a device-scope acq_rel fetch-add. The release publishes the
// calling CTA's prior global writes (ordered before it by the __syncthreads that precedes the call);
// the acquire lets the last arriving CTA read everyone's. Cheaper than __threadfence (fence.sc.gpu).
__device__ __forceinline__ unsigned ticket_arrive(unsigned* t) {
  unsigned old;
  asm volatile("atom.add.acq_rel.gpu.u32 %0, [%1], 1;" : "=r"(old) : "l"(t) : "memory");
  return old;
}

// Programmatic dependent launch (PDL): wait for the previous kernel in the stream (its writes are
// then visible), and let the next kernel's CTAs be scheduled as ours retire. No-ops without PDL.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// 128-bit streaming load of read-only input (no L1 allocation).
__device__ __forceinline__ uint4 ldg_stream(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

template <typename U>
__device__ __forceinline__ U vec_elem(const uint4& v, int e) {
  if constexpr (sizeof(U) == 4) {
    return (U)((e == 0) ? v.x : (e == 1) ? v.y : (e == 2) ? v.z : v.w);
  } else if constexpr (sizeof(U) == 2) {
    const unsigned w = (e < 2) ? v.x : (e < 4) ? v.y : (e < 6) ? v.z : v.w;
    return (U)((e & 1) ? (w >> 16) : (w & 0xffffu));
  } else {
    return (e == 0) ? ((U)v.y << 32 | v.x) : ((U)v.w << 32 | v.z);
  }
}

// Shared-memory histogram update for one element slot per lane (all lanes call).
//   HMODE 0: plain shared atomics.
//   HMODE 1: warp-uniform fast path (all valid lanes share one digit -> one add), else plain.
//   HMODE 2: __match_any_sync aggregation (one add per distinct digit in the warp).
template <int HMODE>
__device__ __forceinline__ void hist_add(unsigned* sh, unsigned d, bool valid) {
  if constexpr (HMODE == 0) {
    if (valid) atomicAdd(&sh[d], 1u);
  } else if constexpr (HMODE == 1) {
    const unsigned vm = __ballot_sync(kFull, valid);
    if (!vm) return;
    const int leader = __ffs(vm) - 1;
    const unsigned d0 = __shfl_sync(kFull, d, leader);
    if (__all_sync(kFull, !valid || d == d0)) {
      if (lane_id() == leader) atomicAdd(&sh[d0], (unsigned)__popc(vm));
    } else if (valid) {
      atomicAdd(&sh[d], 1u);
    }
  } else {
    const unsigned key = valid ? d : 0xffffffffu;
    const unsigned grp = __match_any_sync(kFull, key);
    if (valid && (lane_id() == __ffs(grp) - 1)) atomicAdd(&sh[d], (unsigned)__popc(grp));
  }
}

// Block-wide exclusive scan of one 64-bit value per thread. `tmp` holds >= BLOCK/32 entries.
template <int BLOCK>
__device__ __forceinline__ unsigned long long block_exclusive_scan(unsigned long long v, unsigned long long* tmp,
                                                                   unsigned long long& total) {
  const int lane = lane_id(), warp = threadIdx.x >> 5;
  unsigned long long x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    unsigned long long y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) tmp[warp] = x;
  __syncthreads();
  if (warp == 0) {
    constexpr int NW = BLOCK / 32;
    unsigned long long w = (lane < NW) ? tmp[lane] : 0ull;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      unsigned long long y = __shfl_up_sync(kFull, w, o);
      if (lane >= o) w += y;
    }
    if (lane < NW) tmp[lane] = w;  // inclusive warp prefix
  }
  __syncthreads();
  const unsigned long long warp_excl = (warp == 0) ? 0ull : tmp[warp - 1];
  total = tmp[BLOCK / 32 - 1];
  __syncthreads();
  return warp_excl + x - v;
}

// Algorithm 1 L24-25: inclusive prefix sum of hist[0..nbins) and the target digit j with
// psum[j-1] < K <= psum[j]. `load(i)` returns the count of bin i. Exactly one thread
// finds j; results are published through shared memory to all threads.
struct ScanResult {
  unsigned j;
  unsigned long long before;  // psum[j-1]
  unsigned long long cnt;     // hist[j]
  unsigned long long total;   // psum[nbins-1]
};

template <int BLOCK, typename Load>
__device__ __forceinline__ ScanResult scan_choose(Load load, int nbins, unsigned long long K,
                                                  unsigned long long* tmp, ScanResult* res) {
  constexpr int BPT = (kMaxBins + BLOCK - 1) / BLOCK;
  unsigned long long c[BPT];
  unsigned long long s = 0;
#pragma unroll
  for (int i = 0; i < BPT; ++i) {
    const int b = threadIdx.x * BPT + i;
    c[i] = (b < nbins) ? load(b) : 0ull;
    s += c[i];
  }
  unsigned long long total;
  unsigned long long run = block_exclusive_scan<BLOCK>(s, tmp, total);
#pragma unroll
  for (int i = 0; i < BPT; ++i) {
    const unsigned long long before = run;
    run += c[i];
    if (before < K && run >= K) {
      res->j = threadIdx.x * BPT + i;
      res->before = before;
      res->cnt = c[i];
    }
  }
  if (threadIdx.x == 0) res->total = total;
  __syncthreads();
  ScanResult r = *res;
  __syncthreads();
  return r;
}

}  // namespace airtopk
