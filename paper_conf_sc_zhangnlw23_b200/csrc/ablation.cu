// ablation.cu — the paper's kernel-organisation ablations (§3.1).
//
// A deliberately plain multi-pass radix select with a RUNTIME digit width b and three kernel
// organisations, so the design choices the paper argues for can be measured on B200:
//   design 0, "naive" (Fig. 2): every iteration is FOUR kernels — histogram of digit d
//      over the candidates, inclusive prefix sum (one block), target-digit search (one block),
//      filter (results out, candidates to the buffer); the candidates are loaded twice per iteration;
//   design 1, "iteration-fused" (Fig. 3): kernel q filters digit q-1 AND histograms digit
//      q from one load (Alg1 L15-22), its last block computes the prefix sum and the target digit
//      (P:154), then ONE last-filter kernel — ceil(r/b) + 1 kernels;
//   design 2, "fused last filter" ("it is possible to fuse the last filtering kernel too"): as
//      design 1, but the last block of the last iteration also runs the final filter itself.
// b = 8 gives 4 iterations for 32-bit keys, b = 11 gives 3. Candidates are buffered only
// while C < N/alpha, early stop when K == C, lowest-index ties by continuing over the
// index digits (reading 1) — so every design returns exactly the same set as the engines.
// Keys of <= 32 bits, one row per blockIdx.y. This is an ablation harness, not a tuned engine
// (scalar loads, one histogram copy).
#include <algorithm>
#include <cstdint>

#include "../../include/airtopk.h"
#include "device.cuh"
#include "engine.h"

namespace airtopk {

constexpr int kAbBlock = 256;
constexpr int kAbMaxB = 11;

struct AbState {  // per row
  unsigned long long K, C, pcode, pidx, out, nbuf[2];
  int src;    // 0 = L, s + 1 = buffer slot s
  int stop;   // 1 + digit after whose scan K == C
  int done;
};

struct AbParams {
  const void* keys;
  int64_t batch, len, k;
  int sel_min, R, IB, b, P;  // P = digits of the composite key (code : R || index : IB)
  int64_t cap;               // buffer iff C <= cap (C * alpha < N)
  void* out_vals;
  int64_t* out_idx;
  AbState* st;
  unsigned* hist;            // [batch][2^b]
  unsigned long long* psum;  // [batch][2^b] (naive design)
  unsigned* ticket;          // [batch]
  unsigned* bcode;           // [2][batch][cap + 1]
  unsigned* bidx;
};

struct AbDigit {
  int is_idx, shift, width;
};

__device__ __forceinline__ AbDigit ab_digit(int q, int R, int IB, int b) {
  const int pc = (R + b - 1) / b;
  if (q < pc) {
    const int hi = R - b * q, w = hi < b ? hi : b;
    return AbDigit{0, hi - w, w};
  }
  const int hi = IB - b * (q - pc), w = hi < b ? hi : b;
  return AbDigit{1, hi - w, w};
}

// code / index value of digit d, and whether every digit above d matches the chosen prefix
__device__ __forceinline__ unsigned ab_val(const AbDigit& d, unsigned code, unsigned idx) {
  return ((d.is_idx ? idx : code) >> d.shift) & ((1u << d.width) - 1u);
}
__device__ __forceinline__ bool ab_prefix(const AbDigit& d, unsigned code, unsigned idx, const AbState& s, int R) {
  if (!d.is_idx) {
    const int top = d.shift + d.width;
    return top >= R ? true : ((code >> top) == (unsigned)(s.pcode >> top));
  }
  const int top = d.shift + d.width;
  return code == (unsigned)s.pcode && (top >= 32 ? true : ((idx >> top) == (unsigned)(s.pidx >> top)));
}

template <int KIND>
__device__ __forceinline__ unsigned ab_code(const AbParams& p, int64_t row, int64_t i) {
  using U = typename KT<KIND>::U;
  return (unsigned)to_code<KIND>(((const U*)p.keys)[row * p.len + i], p.sel_min != 0);
}

template <int KIND>
__device__ __forceinline__ void ab_emit(const AbParams& p, int64_t row, bool pred, unsigned code, unsigned idx) {
  using U = typename KT<KIND>::U;
  const unsigned m = __ballot_sync(kFull, pred);
  if (!m) return;
  const int lane = threadIdx.x & 31;
  unsigned long long b = 0;
  if (lane == 0) b = atomicAdd(&p.st[row].out, (unsigned long long)__popc(m));
  b = __shfl_sync(kFull, b, 0);
  if (pred) {
    const unsigned long long pos = b + __popc(m & lanemask_lt());
    if (pos < (unsigned long long)p.k) {
      ((U*)p.out_vals)[row * p.k + pos] = from_code<KIND>((U)code, p.sel_min != 0);
      p.out_idx[row * p.k + pos] = idx;
    }
  }
}

// Scan + target digit of digit q over hist (one block): Alg1 L24-28 / P:100-108.
__device__ void ab_scan_choose(const AbParams& p, int64_t row, int q, const unsigned* h, int nb, bool store_next,
                               int store_slot) {
  __shared__ unsigned long long tmp[kAbBlock / 32];
  __shared__ ScanResult res;
  AbState& s = p.st[row];
  const ScanResult r = scan_choose<kAbBlock>([&](int b) { return (unsigned long long)h[b]; }, nb, s.K, tmp, &res);
  if (threadIdx.x == 0) {
    const AbDigit d = ab_digit(q, p.R, p.IB, p.b);
    s.K -= r.before;
    s.C = r.cnt;
    if (!d.is_idx) s.pcode |= (unsigned long long)r.j << d.shift;
    else s.pidx |= (unsigned long long)r.j << d.shift;
    if (s.K == s.C) s.stop = q + 1;
    (void)store_next;
    (void)store_slot;
  }
  __syncthreads();
}

// Filter of digit f (results < j out, == j candidates to buffer `dst` when storing) and/or histogram
// of digit h over the candidates of the source. mode bit 1: filter, 2: histogram, 4: last block scans
// (fused design), 8: the last block also runs the final filter (design 2).
template <int KIND>
__global__ void __launch_bounds__(kAbBlock) ab_pass(const AbParams p, int q, int mode) {
  __shared__ unsigned sh[1 << kAbMaxB];
  __shared__ int last;
  const int64_t row = blockIdx.y;
  AbState& s = p.st[row];
  if (s.done) return;
  const bool FILT = mode & 1, HIST = mode & 2;
  const int f = q - 1;  // digit filtered (fused: q - 1; naive filter kernels pass q + 1)
  if (FILT && s.stop != 0 && s.stop - 1 < f) return;
  const bool emit_all = FILT && s.stop != 0 && s.stop - 1 == f;
  const bool hist_on = HIST && !emit_all;
  const AbDigit df = ab_digit(f >= 0 ? f : 0, p.R, p.IB, p.b);
  const AbDigit dh = ab_digit(q, p.R, p.IB, p.b);
  const int nb = 1 << dh.width;
  for (int i = threadIdx.x; i < nb; i += kAbBlock) sh[i] = 0;
  __syncthreads();
  const bool fromL = s.src == 0;
  const int islot = fromL ? 0 : s.src - 1, oslot = fromL ? 0 : 1 - islot;
  const unsigned long long n = fromL ? (unsigned long long)p.len : s.nbuf[islot];
  const bool store = FILT && !emit_all && s.C <= (unsigned long long)p.cap;
  const unsigned* ic = p.bcode + ((size_t)islot * p.batch + row) * (p.cap + 1);
  const unsigned* ii = p.bidx + ((size_t)islot * p.batch + row) * (p.cap + 1);
  unsigned* oc = p.bcode + ((size_t)oslot * p.batch + row) * (p.cap + 1);
  unsigned* oi = p.bidx + ((size_t)oslot * p.batch + row) * (p.cap + 1);
  const unsigned long long stride = (unsigned long long)gridDim.x * kAbBlock;
  for (unsigned long long b0 = (unsigned long long)blockIdx.x * kAbBlock; b0 < n; b0 += stride) {
    const unsigned long long i = b0 + threadIdx.x;
    const bool in = i < n;
    const unsigned code = in ? (fromL ? ab_code<KIND>(p, row, (int64_t)i) : ic[i]) : 0u;
    const unsigned idx = in ? (fromL ? (unsigned)i : ii[i]) : 0u;
    bool cand = in, win = false;
    if (FILT && in) {
      const bool pm = ab_prefix(df, code, idx, s, p.R);
      const unsigned v = ab_val(df, code, idx), j = (unsigned)(((df.is_idx ? s.pidx : s.pcode) >> df.shift) &
                                                               ((1u << df.width) - 1u));
      win = pm && (v < j || (emit_all && v == j));
      cand = pm && v == j && !emit_all;
    } else if (!FILT && in && q > 0) {
      // naive histogram kernel over L (no buffer): candidates are the elements matching the prefix
      cand = fromL ? ab_prefix(dh, code, idx, s, p.R) : true;
    }
    if (FILT) ab_emit<KIND>(p, row, win, code, idx);  // (every lane: warp-collective)
    if (store) {
      const unsigned m = __ballot_sync(kFull, cand);
      if (m) {
        unsigned long long base = 0;
        if ((threadIdx.x & 31) == 0) base = atomicAdd(&s.nbuf[oslot], (unsigned long long)__popc(m));
        base = __shfl_sync(kFull, base, 0);
        if (cand) {
          const unsigned long long pos = base + __popc(m & lanemask_lt());
          if (pos <= (unsigned long long)p.cap) {
            oc[pos] = code;
            oi[pos] = idx;
          }
        }
      }
    }
    if (hist_on && cand) atomicAdd(&sh[ab_val(dh, code, idx)], 1u);
  }
  if (!hist_on) {
    if (!(mode & 4)) return;
  }
  __syncthreads();
  unsigned* gh = p.hist + (size_t)row * (1 << kAbMaxB);
  if (hist_on)
    for (int i = threadIdx.x; i < nb; i += kAbBlock)
      if (sh[i]) atomicAdd(&gh[i], sh[i]);
  if (!(mode & 4)) return;
  // fused design: the last block of the row scans
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) last = ticket_arrive(&p.ticket[row]) == gridDim.x - 1;
  __syncthreads();
  if (!last) return;
  if (hist_on) {
    ab_scan_choose(p, row, q, gh, nb, false, 0);
    for (int i = threadIdx.x; i < (1 << kAbMaxB); i += kAbBlock) gh[i] = 0;
  }
  if (threadIdx.x == 0) {
    p.ticket[row] = 0;
    if (store) s.src = oslot + 1;
    s.nbuf[store ? 1 - oslot : oslot] = 0;
    if (FILT && !hist_on) s.done = 1;
  }
  __syncthreads();
  if ((mode & 8) && !s.done) {
    // design 2: this block alone runs the final filter of digit q over the candidates just stored
    // (or over L when the candidates were not stored)
    const AbDigit d = ab_digit(q, p.R, p.IB, p.b);
    const bool fl = s.src == 0;
    const int sl = fl ? 0 : s.src - 1;
    const unsigned long long m = fl ? (unsigned long long)p.len : s.nbuf[sl];
    const unsigned* c2 = p.bcode + ((size_t)sl * p.batch + row) * (p.cap + 1);
    const unsigned* i2 = p.bidx + ((size_t)sl * p.batch + row) * (p.cap + 1);
    const unsigned j = (unsigned)(((d.is_idx ? s.pidx : s.pcode) >> d.shift) & ((1u << d.width) - 1u));
    for (unsigned long long b0 = 0; b0 < m; b0 += kAbBlock) {
      const unsigned long long i = b0 + threadIdx.x;
      const bool in = i < m;
      const unsigned code = in ? (fl ? ab_code<KIND>(p, row, (int64_t)i) : c2[i]) : 0u;
      const unsigned idx = in ? (fl ? (unsigned)i : i2[i]) : 0u;
      const bool win = in && ab_prefix(d, code, idx, s, p.R) && ab_val(d, code, idx) <= j;
      ab_emit<KIND>(p, row, win, code, idx);
    }
    __syncthreads();
    if (threadIdx.x == 0) s.done = 1;
  }
}

// naive design: prefix sum (one block) and target-digit search (one block) as separate kernels
__global__ void __launch_bounds__(kAbBlock) ab_scan_kernel(const AbParams p, int q) {
  const int64_t row = blockIdx.x;
  if (p.st[row].done || (p.st[row].stop != 0 && p.st[row].stop - 1 < q)) return;
  const AbDigit d = ab_digit(q, p.R, p.IB, p.b);
  __shared__ unsigned long long tmp[kAbBlock / 32];
  const int nb = 1 << d.width;
  const unsigned* gh = p.hist + (size_t)row * (1 << kAbMaxB);
  unsigned long long* ps = p.psum + (size_t)row * (1 << kAbMaxB);
  constexpr int BPT = (1 << kAbMaxB) / kAbBlock;
  unsigned long long c[BPT], tot = 0;
  for (int i = 0; i < BPT; ++i) {
    const int b = threadIdx.x * BPT + i;
    c[i] = b < nb ? gh[b] : 0ull;
    tot += c[i];
  }
  unsigned long long total;
  unsigned long long run = block_exclusive_scan<kAbBlock>(tot, tmp, total);
  for (int i = 0; i < BPT; ++i) {
    run += c[i];
    const int b = threadIdx.x * BPT + i;
    if (b < nb) ps[b] = run;  // inclusive prefix sum
  }
}

__global__ void __launch_bounds__(kAbBlock) ab_choose_kernel(const AbParams p, int q) {
  const int64_t row = blockIdx.x;
  AbState& s = p.st[row];
  if (s.done || (s.stop != 0 && s.stop - 1 < q)) return;
  const AbDigit d = ab_digit(q, p.R, p.IB, p.b);
  const int nb = 1 << d.width;
  const unsigned long long* ps = p.psum + (size_t)row * (1 << kAbMaxB);
  unsigned* gh = p.hist + (size_t)row * (1 << kAbMaxB);
  for (int b = threadIdx.x; b < nb; b += kAbBlock) {
    const unsigned long long before = b ? ps[b - 1] : 0ull;
    if (before < s.K && s.K <= ps[b]) {  // psum[j-1] < K <= psum[j]
      s.K -= before;
      s.C = ps[b] - before;
      if (!d.is_idx) s.pcode |= (unsigned long long)b << d.shift;
      else s.pidx |= (unsigned long long)b << d.shift;
      if (s.K == s.C) s.stop = q + 1;
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < (1 << kAbMaxB); i += kAbBlock) gh[i] = 0;
}

// naive design: the filter kernel of digit q (after its scan / choose)
template <int KIND>
__global__ void __launch_bounds__(kAbBlock) ab_filter_kernel(const AbParams p, int q) {
  const int64_t row = blockIdx.y;
  AbState& s = p.st[row];
  if (s.done || (s.stop != 0 && s.stop - 1 < q)) return;
  const bool emit_all = (s.stop != 0 && s.stop - 1 == q) || q == p.P - 1;
  const AbDigit d = ab_digit(q, p.R, p.IB, p.b);
  const bool fromL = s.src == 0;
  const int islot = fromL ? 0 : s.src - 1, oslot = fromL ? 0 : 1 - islot;
  const unsigned long long n = fromL ? (unsigned long long)p.len : s.nbuf[islot];
  const bool store = !emit_all && s.C <= (unsigned long long)p.cap;
  const unsigned* ic = p.bcode + ((size_t)islot * p.batch + row) * (p.cap + 1);
  const unsigned* ii = p.bidx + ((size_t)islot * p.batch + row) * (p.cap + 1);
  unsigned* oc = p.bcode + ((size_t)oslot * p.batch + row) * (p.cap + 1);
  unsigned* oi = p.bidx + ((size_t)oslot * p.batch + row) * (p.cap + 1);
  const unsigned j = (unsigned)(((d.is_idx ? s.pidx : s.pcode) >> d.shift) & ((1u << d.width) - 1u));
  const unsigned long long stride = (unsigned long long)gridDim.x * kAbBlock;
  for (unsigned long long b0 = (unsigned long long)blockIdx.x * kAbBlock; b0 < n; b0 += stride) {
    const unsigned long long i = b0 + threadIdx.x;
    const bool in = i < n;
    const unsigned code = in ? (fromL ? ab_code<KIND>(p, row, (int64_t)i) : ic[i]) : 0u;
    const unsigned idx = in ? (fromL ? (unsigned)i : ii[i]) : 0u;
    const bool pm = in && ab_prefix(d, code, idx, s, p.R);
    const unsigned v = ab_val(d, code, idx);
    ab_emit<KIND>(p, row, pm && (v < j || (emit_all && v == j)), code, idx);
    const bool cand = pm && v == j && store;
    const unsigned m = __ballot_sync(kFull, cand);
    if (m) {
      unsigned long long base = 0;
      if ((threadIdx.x & 31) == 0) base = atomicAdd(&s.nbuf[oslot], (unsigned long long)__popc(m));
      base = __shfl_sync(kFull, base, 0);
      if (cand) {
        const unsigned long long pos = base + __popc(m & lanemask_lt());
        if (pos <= (unsigned long long)p.cap) {
          oc[pos] = code;
          oi[pos] = idx;
        }
      }
    }
  }
  // the last block switches the source for the next iteration (or ends the row)
  __shared__ int last;
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) last = ticket_arrive(&p.ticket[row]) == gridDim.x - 1;
  __syncthreads();
  if (!last || threadIdx.x != 0) return;
  p.ticket[row] = 0;
  if (emit_all) {
    s.done = 1;
  } else if (store) {
    s.src = oslot + 1;
    s.nbuf[1 - oslot] = 0;
  } else {
    s.nbuf[oslot] = 0;
  }
}

__global__ void ab_init(const AbParams p) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < p.batch; r += (int64_t)gridDim.x * blockDim.x) {
    AbState& s = p.st[r];
    s.K = (unsigned long long)p.k;
    s.C = (unsigned long long)p.len;
    s.pcode = s.pidx = s.out = 0;
    s.nbuf[0] = s.nbuf[1] = 0;
    s.src = s.stop = s.done = 0;
  }
}

}  // namespace airtopk

using namespace airtopk;

static int bits_of(uint64_t v) {
  int b = 0;
  while (v) {
    ++b;
    v >>= 1;
  }
  return b;
}

extern "C" {

size_t airtopk_ablation_workspace(airtopk_dtype dtype, int64_t batch, int64_t len, int64_t alpha) {
  if (batch < 1 || len < 1 || (int)dtype == AIRTOPK_F64 || alpha < 0) return 0;
  const int64_t cap = (len - 1) / (alpha > 0 ? alpha : 128);
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  return al(sizeof(AbState) * batch) + al((size_t)batch * (1 << kAbMaxB) * 4) + al((size_t)batch * (1 << kAbMaxB) * 8) +
         al((size_t)batch * 4) + 2 * al((size_t)2 * batch * (cap + 1) * 4);
}

airtopk_status airtopk_select_ablation(const void* keys, airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k,
                                       int select_min, void* out_vals, int64_t* out_idx, int design, int digit_bits,
                                       int64_t alpha, void* workspace, size_t workspace_bytes, airtopk_stream_t stream,
                                       int* kernels_out) {
  if (!keys || !out_vals || !out_idx || !workspace) return AIRTOPK_EINVAL;
  if ((int)dtype < AIRTOPK_F32 || (int)dtype > AIRTOPK_U32 || (int)dtype == AIRTOPK_F64) return AIRTOPK_EDTYPE;
  if (batch < 1 || batch > 65535 || len < 1 || len >= (int64_t(1) << 32) || k < 1 || k >= len) return AIRTOPK_EINVAL;
  if (design < 0 || design > 2 || (digit_bits != 8 && digit_bits != 11) || alpha < 0) return AIRTOPK_EINVAL;
  if (workspace_bytes < airtopk_ablation_workspace(dtype, batch, len, alpha)) return AIRTOPK_ENOSPACE;
  cudaStream_t s = (cudaStream_t)stream;
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  char* w = (char*)workspace;
  AbParams p;
  p.keys = keys;
  p.batch = batch;
  p.len = len;
  p.k = k;
  p.sel_min = select_min ? 1 : 0;
  p.R = key_bits((int)dtype);
  p.IB = std::max(1, bits_of((uint64_t)(len - 1)));
  p.b = digit_bits;
  p.P = (p.R + p.b - 1) / p.b + (p.IB + p.b - 1) / p.b;
  p.cap = (len - 1) / (alpha > 0 ? alpha : 128);
  p.out_vals = out_vals;
  p.out_idx = out_idx;
  p.st = (AbState*)w;
  w += al(sizeof(AbState) * batch);
  p.hist = (unsigned*)w;
  w += al((size_t)batch * (1 << kAbMaxB) * 4);
  p.psum = (unsigned long long*)w;
  w += al((size_t)batch * (1 << kAbMaxB) * 8);
  p.ticket = (unsigned*)w;
  w += al((size_t)batch * 4);
  p.bcode = (unsigned*)w;
  w += al((size_t)2 * batch * (p.cap + 1) * 4);
  p.bidx = (unsigned*)w;
  cudaError_t e = cudaMemsetAsync(workspace, 0, (size_t)(w - (char*)workspace), s);
  if (e != cudaSuccess) return AIRTOPK_ECUDA;
  ab_init<<<(unsigned)std::min<int64_t>((batch + 255) / 256, 64), 256, 0, s>>>(p);
  const int64_t per = std::max<int64_t>(1, std::min<int64_t>((len + kAbBlock * 8 - 1) / (kAbBlock * 8),
                                                             std::max<int64_t>(1, 148 * 8 / batch)));
  const dim3 grid((unsigned)per, (unsigned)batch);
  int nk = 0;
  auto pass = [&](int q, int mode) {
    switch ((int)dtype) {
      case AIRTOPK_F32: ab_pass<K_F32><<<grid, kAbBlock, 0, s>>>(p, q, mode); break;
      case AIRTOPK_F16: ab_pass<K_F16><<<grid, kAbBlock, 0, s>>>(p, q, mode); break;
      case AIRTOPK_BF16: ab_pass<K_BF16><<<grid, kAbBlock, 0, s>>>(p, q, mode); break;
      default: ab_pass<K_U32><<<grid, kAbBlock, 0, s>>>(p, q, mode); break;
    }
    ++nk;
  };
  auto filt = [&](int q) {
    switch ((int)dtype) {
      case AIRTOPK_F32: ab_filter_kernel<K_F32><<<grid, kAbBlock, 0, s>>>(p, q); break;
      case AIRTOPK_F16: ab_filter_kernel<K_F16><<<grid, kAbBlock, 0, s>>>(p, q); break;
      case AIRTOPK_BF16: ab_filter_kernel<K_BF16><<<grid, kAbBlock, 0, s>>>(p, q); break;
      default: ab_filter_kernel<K_U32><<<grid, kAbBlock, 0, s>>>(p, q); break;
    }
    ++nk;
  };
  if (design == 0) {
    // naive: per digit q: histogram (mode 2 over the candidates), scan, choose, filter
    for (int q = 0; q < p.P; ++q) {
      pass(q, 2);
      ab_scan_kernel<<<(unsigned)batch, kAbBlock, 0, s>>>(p, q);
      ab_choose_kernel<<<(unsigned)batch, kAbBlock, 0, s>>>(p, q);
      nk += 2;
      filt(q);
    }
  } else {
    // fused: kernel q = filter(q-1) + hist(q) + last-block scan; then the last filter kernel (design
    // 1) or none (design 2: the last block of the last iteration filters)
    for (int q = 0; q < p.P; ++q) pass(q, (q > 0 ? 1 : 0) | 2 | 4 | (design == 2 && q == p.P - 1 ? 8 : 0));
    if (design == 1) pass(p.P, 1 | 4);
  }
  if (kernels_out) *kernels_out = nk;
  return cudaGetLastError() == cudaSuccess ? AIRTOPK_OK : AIRTOPK_ECUDA;
}

}  // extern "C"
