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
//   * grid = batch x cpr CTAs of 512 threads, 3 CTAs/SM (444 CTAs fill the 148 SMs; measured
//     faster than 4/SM), each CTA a contiguous slice of its row;
//   * 4 x 128-bit ld.global.nc.L1::no_allocate loads in flight per thread (32 KiB per CTA tile);
//   * odd passes walk their slice backwards so the tail the previous pass left in the 126 MB L2 is
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
#include <type_traits>

#include "device.cuh"
#include "engine.h"
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
  int64_t* trace;
};

constexpr int kBlock = 512;
constexpr int kWarps = kBlock / 32;
constexpr int kMinBlocks = 3;

template <int KIND, typename IdxT, int DF, int DH, bool HASIDX>
__global__ void __launch_bounds__(kBlock, kMinBlocks) pass_kernel(const GridParams p, const int q) {
  using U = typename KT<KIND>::U;
  using CountT = std::conditional_t<sizeof(IdxT) == 8, unsigned long long, unsigned>;
  constexpr bool HAS_Q = DF != 0;
  constexpr int HC = hist_copies<KIND, IdxT, DF>();

  extern __shared__ unsigned sh_hist[];  // kMaxBins * HC counters (dynamic: may exceed 48 KB)
  __shared__ WarpQ<U, IdxT> sh_oq[HAS_Q ? kWarps : 1];
  __shared__ WarpQ<U, IdxT> sh_bq[(HAS_Q && DH != 0) ? kWarps : 1];
  __shared__ unsigned long long sh_tmp[kWarps];
  __shared__ ScanResult sh_res;
  __shared__ int sh_last;

  const int64_t row = blockIdx.x / p.cpr;
  const int cta = blockIdx.x % p.cpr;
  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  RowState* st = p.st + row;

  // ---- row state after scan q-1 ----
  const int stop1 = (DF != 0) ? st->stop1 : 0;
  if (DF != 0 && stop1 != 0 && stop1 - 1 < q - 1) return;  // finished by an earlier early stop
  PassCtx<U, IdxT> c;
  c.q = q;
  c.emit_all = (DF != 0) && ((stop1 != 0 && stop1 - 1 == q - 1) || DH == 0);
  c.do_hist = (DH != 0) && !c.emit_all;
  const unsigned long long Cprev = (DF != 0) ? st->C : (unsigned long long)p.len;  // C_{q-1}
  const unsigned long long Cpp = (DF != 0) ? st->Cp : (unsigned long long)p.len;   // C' = C_{q-2}
  c.srcL = (DF == 0) || (Cpp > (unsigned long long)p.cap_rule);                   // Alg1 L7
  c.store = c.do_hist && (DF != 0) && (Cprev <= (unsigned long long)p.cap_rule);  // Alg1 L17
  c.sel_min = p.sel_min != 0;
  c.reverse = (q & 1) != 0;  // walk back over what the previous pass left in L2
  c.dh = digit_of(q, KT<KIND>::R, p.IB);
  c.df = digit_of(DF != 0 ? q - 1 : 0, KT<KIND>::R, p.IB);
  c.tcode = (DF != 0) ? st->tcode : 0ull;
  c.tidx = (DF != 0) ? st->tidx : 0ull;
  c.rowp = (const U*)p.keys + row * p.len;
  c.rowi = HASIDX ? p.in_idx + row * p.len : nullptr;
  c.len = p.len;
  c.slice = cta;
  c.nslices = p.cpr;
  const int islot = (q - 1) & 1;
  c.bcin = (const U*)p.bcode + ((size_t)islot * p.batch + row) * p.cap_alloc;
  c.biin = (const IdxT*)p.bidx + ((size_t)islot * p.batch + row) * p.cap_alloc;
  c.nbuf = (DF != 0 && !c.srcL) ? st->buf_count[islot] : 0ull;
  c.ov = (U*)p.out_vals + row * p.k;
  c.oi = p.out_idx + row * p.k;
  c.outc = &st->out_count;
  c.kk = (unsigned long long)p.k;
  c.bco = (U*)p.bcode + ((size_t)(q & 1) * p.batch + row) * p.cap_alloc;
  c.bio = (IdxT*)p.bidx + ((size_t)(q & 1) * p.batch + row) * p.cap_alloc;
  c.bufc = &st->buf_count[q & 1];
  c.capa = (unsigned long long)p.cap_alloc;
  c.err = &st->error;
  c.hist = sh_hist;
  c.oq = &sh_oq[HAS_Q ? warp : 0];
  c.bq = &sh_bq[(HAS_Q && DH != 0) ? warp : 0];

  const bool hist_on = c.do_hist || DF == 0;
  if (hist_on) {
    for (int i = tid; i < kHistSlots * HC; i += kBlock) sh_hist[i] = 0;
    __syncthreads();
  }

  const unsigned long long nread = run_pass<KIND, IdxT, DF, DH, HASIDX, kBlock>(c);

  if (!hist_on) return;

  // ---- merge into the row histogram; the last CTA scans ----
  __syncthreads();
  const Digit dh = c.dh;
  CountT* gh = (CountT*)p.ghist + ((size_t)row * 2 + (q & 1)) * kMaxBins;
  const int nb = 1 << dh.width;
  for (int i = tid; i < nb; i += kBlock) {
    unsigned v = 0;
#pragma unroll
    for (int h = 0; h < HC; ++h) v += sh_hist[i * HC + h];
    if (v) atomicAdd(&gh[i], (CountT)v);
  }
  __threadfence();
  __syncthreads();
  if (tid == 0) sh_last = (atomicAdd(&st->ticket, 1u) == (unsigned)(p.cpr - 1));
  __syncthreads();
  if (!sh_last) return;
  __threadfence();

  const unsigned long long kk = (unsigned long long)p.k;
  const unsigned long long Kin = (DF == 0) ? kk : st->K;
  const unsigned long long Cin = Cprev;  // elements counted by this histogram
  const ScanResult r = scan_choose<kBlock>(
      [&](int b) { return (unsigned long long)__ldcg(&gh[b]); }, nb, Kin, sh_tmp, &sh_res);
  CountT* gh2 = (CountT*)p.ghist + ((size_t)row * 2 + ((q + 1) & 1)) * kMaxBins;
  for (int i = tid; i < kMaxBins; i += kBlock) gh2[i] = 0;
  if (tid == 0) {
    const unsigned long long newK = Kin - r.before, newC = r.cnt;   // Alg1 L26-28
    st->Cp = Cin;
    st->C = newC;
    st->K = newK;
    if (!dh.is_idx) st->tcode |= (unsigned long long)r.j << dh.shift;
    else st->tidx |= (unsigned long long)r.j << dh.shift;
    st->j = r.j;
    st->npass = q + 1;
    if (newK == newC) st->stop1 = q + 1;                             // early stop
    st->buf_count[(q + 1) & 1] = 0;
    st->ticket = 0;
    if (r.total != Cin) st->error |= 4u;
    if (p.trace && q < kTraceMaxPasses) {
      int64_t* t = p.trace + ((size_t)row * kTraceMaxPasses + q) * kTraceFields;
      t[0] = dh.width; t[1] = c.srcL; t[2] = c.store; t[3] = r.j; t[4] = (int64_t)newK; t[5] = (int64_t)newC;
      t[6] = (int64_t)Cin; t[7] = (int64_t)__ldcg(c.outc); t[8] = (newK == newC); t[9] = (int64_t)nread;
    }
  }
}

struct Events {
  void* const* ev;
  int n;
  void record(int i, cudaStream_t s) const {
    if (ev && i < n) cudaEventRecord((cudaEvent_t)ev[i], s);
  }
};

template <int KIND, typename IdxT, int DF, int DH>
constexpr size_t hist_smem_bytes() {
  return (size_t)kHistSlots * 4 * hist_copies<KIND, IdxT, DF>();
}

template <int KIND, typename IdxT, int DF, int DH, bool HASIDX>
cudaError_t launch_one(const GridParams& gp, unsigned grid, int q, cudaStream_t s) {
  constexpr size_t smem = hist_smem_bytes<KIND, IdxT, DF, DH>();
  static const cudaError_t attr = cudaFuncSetAttribute(pass_kernel<KIND, IdxT, DF, DH, HASIDX>,
                                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (attr != cudaSuccess) return attr;
  pass_kernel<KIND, IdxT, DF, DH, HASIDX><<<grid, kBlock, smem, s>>>(gp, q);
  return cudaSuccess;
}

template <int KIND, typename IdxT, bool HASIDX>
cudaError_t launch_grid_passes(const GridParams& gp, int64_t batch, const Events& ev, cudaStream_t s) {
  const unsigned grid = (unsigned)((long long)batch * gp.cpr);
  ev.record(0, s);
  for (int q = 0; q <= gp.P; ++q) {
    const int DF = q == 0 ? 0 : (digit_of(q - 1, KT<KIND>::R, gp.IB).is_idx ? 2 : 1);
    const int DH = q == gp.P ? 0 : (digit_of(q, KT<KIND>::R, gp.IB).is_idx ? 2 : 1);
    const int v = DF * 3 + DH;
    cudaError_t e;
    switch (v) {
      case 0 * 3 + 1: e = launch_one<KIND, IdxT, 0, 1, HASIDX>(gp, grid, q, s); break;
      case 1 * 3 + 1: e = launch_one<KIND, IdxT, 1, 1, HASIDX>(gp, grid, q, s); break;
      case 1 * 3 + 2: e = launch_one<KIND, IdxT, 1, 2, HASIDX>(gp, grid, q, s); break;
      case 2 * 3 + 2: e = launch_one<KIND, IdxT, 2, 2, HASIDX>(gp, grid, q, s); break;
      case 2 * 3 + 0: e = launch_one<KIND, IdxT, 2, 0, HASIDX>(gp, grid, q, s); break;
      default: return cudaErrorInvalidValue;
    }
    if (e != cudaSuccess) return e;
    ev.record(q + 1, s);
  }
  return cudaGetLastError();
}

template <int KIND>
cudaError_t launch_grid_kind(const SelectArgs& a, const Plan& pl, const GridParams& gp, cudaStream_t s) {
  const Events ev{a.events, a.n_events};
  if (a.in_idx) return launch_grid_passes<KIND, uint64_t, true>(gp, a.batch, ev, s);
  if (pl.idx64) return launch_grid_passes<KIND, uint64_t, false>(gp, a.batch, ev, s);
  return launch_grid_passes<KIND, uint32_t, false>(gp, a.batch, ev, s);
}

#define AIRTOPK_INSTANTIATE_GRID(KIND) \
  template cudaError_t launch_grid_kind<KIND>(const SelectArgs&, const Plan&, const GridParams&, cudaStream_t);

}  // namespace airtopk
