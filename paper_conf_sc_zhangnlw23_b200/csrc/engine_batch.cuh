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
//      [lo, hi] (the same estimator and 4-sigma+8 margin as sample_kernel); CTAs first issue L2 bulk
//      prefetches of the chunks they stream first, so HBM works during the sampling latency.
//   B  stream: the batch is cut into 64 KiB chunks, chunk c -> CTA c mod G (grid-stride over the
//      flattened batch: no wave quantisation, every SM streams ~equal bytes; the CTAs stream one
//      compact advancing region of HBM). Per element ONE compare of the raw key bits against the
//      transformed threshold hi (exact); the rare flagged keys (code <= hi) are written by their
//      warp to a FIXED slot of its (chunk, warp) — no atomics, no queues, no block barriers in the
//      streaming loop — and the warp stores the slot's count.
//   C  finish: CTA r gathers its row's slots (prefix sum over the slot counts) into shared memory
//      and registers, checks that the window holds the K-th key (R < K <= R + W, R = #codes < lo,
//      W = #members), emits the R results, then selects the K - R smallest members by radix passes
//      over the composite key (code || row index: lowest-index ties, reading 1) on the
//      register-resident entries: per pass a 2048-bin shared histogram, the inclusive scan and the
//      target digit j with psum[j-1] < K <= psum[j] (Alg1 L24-28), filter (digit < j ->
//      result, == j -> candidate), early stop when K == C.
//
// Exactness never depends on the sample: a row whose window misses (or overflows a slot or the
// finish capacity, or had no usable window) is marked win_state = 3 and the next, already enqueued,
// launch (the cluster engine in fallback mode, PDL) selects it from L with the paper's passes.
#pragma once

#include <cooperative_groups.h>

#include "device.cuh"
#include "engine.h"
#include "engine_grid.cuh"
#include "tma.cuh"

namespace airtopk {

constexpr int kBBlock = kBatchBlock;          // threads per CTA (1 CTA per SM)
constexpr int kBWarps = kBBlock / 32;
constexpr int kBUnroll = kBatchUnroll;        // 16-byte vectors per thread per chunk (64 KiB chunks)
static_assert(kBWarps == kBatchWarps, "host/device slot geometry");
constexpr int kBChunkVec = kBBlock * kBUnroll;  // 16-byte vectors per chunk
constexpr int kBWarpElems32 = 32 * kBUnroll * 4;  // f32 elements per (chunk, warp) slot: 512

// entries (results + window members) one row may stage in the finish: PER per thread in registers
template <int KIND>
__host__ __device__ constexpr int batch_per_thread() { return sizeof(typename KT<KIND>::U) == 8 ? 8 : 16; }
template <int KIND>
__host__ __device__ constexpr int batch_fcap() { return kBBlock * batch_per_thread<KIND>(); }
static_assert(batch_fcap<K_F64>() == kBatchBlock * 8 && batch_fcap<K_F32>() == kBatchBlock * 16, "batch_fcap_host");

struct BatchParams {
  const void* keys;
  int64_t batch, len, k;
  int sel_min;
  int IB;                 // index bits (lowest-index tie digits)
  void* out_vals;
  int64_t* out_idx;
  int64_t idx_off;
  RowState* st;
  unsigned short* cnt;    // [batch][nwc] entries written per (chunk, warp) slot (cap + 1 = overflow)
  void* scode;            // [batch][nwc][scap] codes
  unsigned* sidx;         // [batch][nwc][scap] row indices
  int nwc;                // slots per row = chunks per row * kBWarps
  int scap;               // entries per slot
  int cpc;                // chunks per row
  int nsamp;              // samples per row
  int early_stop;         // 0 on, -1 off
  int64_t* timing;        // optional (trace buffer): per CTA globaltimer stamps of the phases
  int64_t timing_n;       // int64 entries of `timing`
};

__device__ __forceinline__ void prefetch_l2(const void* p, unsigned bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}

// Phase A for one row (all threads of the CTA): window [lo, hi] from the sample order statistics.
template <int KIND>
__device__ void batch_sample_row(const BatchParams& p, int64_t row, void* scratch_v) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  constexpr int PER = kMaxSamples / kBBlock;
  __shared__ unsigned hist[2048 * kSampleHistCopies];
  __shared__ unsigned wsum[32];
  __shared__ W shw[8];
  __shared__ int sh_cnt[4];
  __shared__ W sh_red[64];
  W* scratch = (W*)scratch_v;
  RowState* st = p.st + row;
  const int nsamp = p.nsamp;
  const U* rowp = (const U*)p.keys + row * p.len;
  const U xmask = p.sel_min ? (U)0 : (U)~(U)0;
  constexpr int kRun = 32;
  const int nruns = nsamp / kRun;
  const int64_t stride = p.len / nruns;
  W v[PER];
  {
    U x[PER];
#pragma unroll
    for (int t = 0; t < PER; ++t) {
      const int slot = t * kBBlock + threadIdx.x;
      const int run = slot / kRun, e = slot % kRun;
      const int64_t pos = (int64_t)run * stride + (stride - kRun) / 2 + e;
      if (run < nruns) x[t] = __ldg(rowp + pos);
    }
#pragma unroll
    for (int t = 0; t < PER; ++t) {
      const int slot = t * kBBlock + threadIdx.x;
      v[t] = (slot < nsamp) ? (W)to_code_x<KIND>(x[t], xmask) : (W)0;
    }
  }
  const int tv = (nsamp - (int)threadIdx.x + kBBlock - 1) / kBBlock;  // valid v[t]: t < tv
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
    const W a = shfl(lmin, (threadIdx.x + o) & 31), b = shfl(lmax, (threadIdx.x + o) & 31);
    lmin = a < lmin ? a : lmin;
    lmax = b > lmax ? b : lmax;
  }
  if ((threadIdx.x & 31) == 0) {
    sh_red[threadIdx.x >> 5] = lmin;
    sh_red[32 + (threadIdx.x >> 5)] = lmax;
  }
  if (threadIdx.x == 0) sh_cnt[2] = 0;
  __syncthreads();
  W smin = sh_red[0], smax = sh_red[32];
#pragma unroll 8
  for (int i = 1; i < kBWarps; ++i) {
    smin = sh_red[i] < smin ? sh_red[i] : smin;
    smax = sh_red[32 + i] > smax ? sh_red[32 + i] : smax;
  }
  // expected sample rank of the K-th key, 4-sigma (+8) binomial margin (as sample_kernel)
  const double f = (double)p.k / (double)p.len;
  const double r = f * nsamp;
  const double m = 4.0 * sqrt(r * (1.0 - f)) + 8.0;
  const int rlo = (int)floor(r - m), rhi = (int)ceil(r + m);
  int state = 1;
  W lo = 0, hi = 0;
  if (rhi >= nsamp - 1) {
    state = 3;
  } else {
    const W diff = smin ^ smax;
    const int hb = diff ? (8 * (int)sizeof(W) - (sizeof(W) == 8 ? __clzll((long long)diff) : __clz((int)diff))) : 0;
    block_select_two<W, PER>(v, tv, scratch, rlo <= 0 ? -1 : rlo, rhi, smin, hb, hist, wsum, shw, sh_cnt, lo, hi);
    if (rlo <= 0) lo = 0;
    // estimated entries (results + members: every code <= hi) vs the finish capacity
    unsigned le = 0;
#pragma unroll
    for (int t = 0; t < PER; ++t) le += (t < tv) && v[t] <= hi;
    le = __reduce_add_sync(kFull, le);
    if ((threadIdx.x & 31) == 0 && le) atomicAdd(&sh_cnt[2], (int)le);
    __syncthreads();
    const double est = (double)sh_cnt[2] / nsamp * (double)p.len;
    if (est > 0.6 * (double)batch_fcap<KIND>()) state = 3;
  }
  if (threadIdx.x == 0) {
    st->win_lo = lo;
    st->win_hi = hi;
    st->win_state = state;
    st->out_count = 0;
    st->buf_count[0] = 0;
    st->buf_count[1] = 0;
    st->error = 0;
  }
  __syncthreads();
}

// Threshold of the raw-bit test: code(b) <= hi  <=>  (b ^ wx) <= hi (see run_pass, DF == 3).
template <int KIND>
__device__ __forceinline__ typename std::conditional_t<sizeof(typename KT<KIND>::U) == 8, unsigned long long, unsigned>
raw_xor_for(unsigned long long hi, bool sel_min) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  constexpr W S = (W)((W)1 << (KT<KIND>::R - 1));
  constexpr W ones = (W)(U)~(U)0;
  const W whi = (W)hi;
  if constexpr (KT<KIND>::IEEE) {
    if (sel_min) return (whi >= S) ? S : ones;
    return (whi < S) ? (W)(ones ^ S) : (W)0;
  } else {
    return sel_min ? (W)0 : ones;
  }
}

// Phase B for one chunk (all threads): flag code <= hi, write the warp's flagged keys to its slot.
template <int KIND>
__device__ __forceinline__ void batch_stream_chunk(const BatchParams& p, int64_t row, int ci, unsigned long long hi) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  constexpr int VEC = 16 / sizeof(U);
  constexpr int NE = kBUnroll * VEC;  // elements per thread per chunk
  using FlagT = std::conditional_t<(NE > 32), unsigned long long, unsigned>;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const bool sel_min = p.sel_min != 0;
  const W whi = (W)hi;
  const W wx = raw_xor_for<KIND>(hi, sel_min);
  const U xmask = sel_min ? (U)0 : (U)~(U)0;
  const int64_t nvec = p.len / VEC;  // rows are whole 16-byte vectors (checked on the host)
  const uint4* vp = (const uint4*)((const U*)p.keys + row * p.len);
  const int64_t vb = (int64_t)ci * kBChunkVec + tid;
  uint4 r[kBUnroll];
#pragma unroll
  for (int u = 0; u < kBUnroll; ++u) {
    const int64_t v = vb + (int64_t)u * kBBlock;
    r[u] = (v < nvec) ? ldg_stream(vp + v) : make_uint4(0xffffffffu, 0xffffffffu, 0xffffffffu, 0xffffffffu);
  }
  FlagT fl = 0;
  W m = ~(W)0;
#pragma unroll
  for (int u = 0; u < kBUnroll; ++u) {
    const bool valid = vb + (int64_t)u * kBBlock < nvec;
#pragma unroll
    for (int e = 0; e < VEC; ++e) {
      const W t = (W)((W)vec_elem<U>(r[u], e) ^ wx);
      m = (valid && t < m) ? t : m;
    }
  }
  if (m <= whi) {
#pragma unroll
    for (int u = 0; u < kBUnroll; ++u) {
      const bool valid = vb + (int64_t)u * kBBlock < nvec;
#pragma unroll
      for (int e = 0; e < VEC; ++e)
        if (valid && (W)((W)vec_elem<U>(r[u], e) ^ wx) <= whi) fl |= (FlagT)1 << (u * VEC + e);
    }
  }
  const size_t slot = (size_t)row * p.nwc + (size_t)ci * kBWarps + warp;
  int total = 0;
  if (__any_sync(kFull, fl != 0)) {
    const int n = (sizeof(FlagT) == 8) ? __popcll((unsigned long long)fl) : __popc((unsigned)fl);
    int incl = n;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(kFull, incl, o);
      if (lane >= o) incl += y;
    }
    total = __shfl_sync(kFull, incl, 31);
    int pos = incl - n;
    U* sc = (U*)p.scode + slot * p.scap;
    unsigned* si = p.sidx + slot * p.scap;
    while (fl) {
      const int b = ((sizeof(FlagT) == 8) ? __ffsll((long long)fl) : __ffs((int)fl)) - 1;
      fl &= fl - 1;
      if (pos < p.scap) {
        const int u = b / VEC, e = b % VEC;
        uint4 vv = r[0];
#pragma unroll
        for (int i = 1; i < kBUnroll; ++i) vv = (u == i) ? r[i] : vv;
        U raw = vec_elem<U>(vv, 0);
#pragma unroll
        for (int i = 1; i < VEC; ++i) raw = (e == i) ? vec_elem<U>(vv, i) : raw;
        sc[pos] = to_code_x<KIND>(raw, xmask);
        si[pos] = (unsigned)((vb + (int64_t)u * kBBlock) * VEC + e);
      }
      ++pos;
    }
  }
  if (lane == 0) p.cnt[slot] = (unsigned short)(total > p.scap ? p.scap + 1 : total);
}

// Phase C for one row (all threads): gather, check the window, emit results, select the members.
template <int KIND>
__device__ void batch_finish_row(const BatchParams& p, int64_t row, void* stage) {
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  constexpr int PER = batch_per_thread<KIND>();
  constexpr int FCAP = batch_fcap<KIND>();
  __shared__ unsigned long long s_tmp[kBWarps];
  __shared__ ScanResult s_res;
  __shared__ unsigned s_hist[kMaxBins];
  __shared__ unsigned long long s_tot[2];
  __shared__ unsigned s_out;
  __shared__ int s_bad;
  const int tid = threadIdx.x, lane = tid & 31;
  RowState* st = p.st + row;
  if (st->win_state != 1) return;  // (uniform) no window: the fallback launch selects the row
  const unsigned long long lo = st->win_lo, hi = st->win_hi;
  U* stc = (U*)stage;
  unsigned* sti = (unsigned*)((char*)stage + (size_t)FCAP * sizeof(U));
  // --- slot counts -> offsets (thread t owns slots [t*per, (t+1)*per)) ---
  const int nwc = p.nwc;
  const int per = (nwc + kBBlock - 1) / kBBlock;
  const unsigned short* cnt = p.cnt + (size_t)row * nwc;
  const int s0 = min(nwc, tid * per), s1 = min(nwc, s0 + per);
  unsigned long long mine = 0;
  int bad = 0;
  for (int s = s0; s < s1; ++s) {
    const int c = cnt[s];
    bad |= c > p.scap;
    mine += (unsigned)c;
  }
  if (tid == 0) s_bad = 0;
  __syncthreads();
  if (__any_sync(kFull, bad) && lane == 0) s_bad = 1;
  unsigned long long total;
  unsigned long long off = block_exclusive_scan<kBBlock>(mine, s_tmp, total);
  if (s_bad || total > (unsigned long long)FCAP || total < (unsigned long long)p.k) {
    if (tid == 0) st->win_state = 3;  // slot overflow / too many entries / window below the K-th key
    __syncthreads();
    return;
  }
  // --- gather the entries into shared memory (L2 reads), then into registers ---
  for (int s = s0; s < s1; ++s) {
    const int c = cnt[s];
    const U* sc = (const U*)p.scode + ((size_t)row * nwc + s) * p.scap;
    const unsigned* si = p.sidx + ((size_t)row * nwc + s) * p.scap;
    for (int j = 0; j < c; ++j) {
      stc[off + j] = __ldcg(sc + j);
      sti[off + j] = __ldcg(si + j);
    }
    off += c;
  }
  __syncthreads();
  const int n = (int)total;
  U vc[PER];
  unsigned vi[PER];
  unsigned valid = 0;  // bit t: register slot t holds an entry
  unsigned nres = 0;   // results (code < lo) held by this thread
#pragma unroll
  for (int t = 0; t < PER; ++t) {
    const int e = t * kBBlock + tid;
    vc[t] = (e < n) ? stc[e] : (U)0;
    vi[t] = (e < n) ? sti[e] : 0u;
    if (e < n) {
      valid |= 1u << t;
      nres += ((W)vc[t] < (W)lo);
    }
  }
  // --- window check: R < K <= R + W (W + R = n) ---
  nres = __reduce_add_sync(kFull, nres);
  if (tid == 0) { s_tot[0] = 0; s_out = 0; }
  __syncthreads();
  if (lane == 0 && nres) atomicAdd(&s_tot[0], (unsigned long long)nres);
  __syncthreads();
  const unsigned long long R = s_tot[0];
  const unsigned long long kk = (unsigned long long)p.k;
  if (!(R < kk && kk <= (unsigned long long)n)) {
    if (tid == 0) st->win_state = 3;
    __syncthreads();
    return;
  }
  U* ov = (U*)p.out_vals + row * p.k;
  int64_t* oi = p.out_idx + row * p.k;
  const bool sel_min = p.sel_min != 0;
  auto emit = [&](bool pred, U code, unsigned idx) {  // warp-aggregated output slots
    const unsigned m = __ballot_sync(kFull, pred);
    if (!m) return;
    unsigned b = 0;
    if (lane == 0) b = atomicAdd(&s_out, (unsigned)__popc(m));
    b = __shfl_sync(kFull, b, 0);
    if (pred) {
      const unsigned pos = b + __popc(m & lanemask_lt());
      ov[pos] = from_code<KIND>(code, sel_min);
      oi[pos] = (int64_t)idx + p.idx_off;
    }
  };
  // results: every code below the window
#pragma unroll
  for (int t = 0; t < PER; ++t) {
    const bool isr = ((valid >> t) & 1u) && (W)vc[t] < (W)lo;
    emit(isr, vc[t], vi[t]);
    if (isr) valid &= ~(1u << t);
  }
  // --- members: the K - R smallest composite keys (code || index), radix passes on registers ---
  unsigned long long Kr = kk - R, C = (unsigned long long)n - R;
  int q = 0;
  const int pc = code_passes(KT<KIND>::R), P = pc + idx_passes(p.IB);
  while (q < pc - 1) {  // digits on which lo and hi agree are common to every member
    const Digit d = digit_of(q, KT<KIND>::R, p.IB);
    if ((lo >> d.shift) != (hi >> d.shift)) break;
    ++q;
  }
  for (; q < P && !(Kr == C && p.early_stop == 0); ++q) {
    const Digit d = digit_of(q, KT<KIND>::R, p.IB);
    const unsigned dm = (1u << d.width) - 1u;
    const int nb = 1 << d.width;
    for (int i = tid; i < nb; i += kBBlock) s_hist[i] = 0;
    __syncthreads();
#pragma unroll
    for (int t = 0; t < PER; ++t) {
      if ((valid >> t) & 1u) {
        const unsigned dg = d.is_idx ? (vi[t] >> d.shift) & dm : (unsigned)((W)vc[t] >> d.shift) & dm;
        atomicAdd(&s_hist[dg], 1u);
      }
    }
    __syncthreads();
    const ScanResult r = scan_choose<kBBlock>([&](int b) { return (unsigned long long)s_hist[b]; }, nb, Kr, s_tmp,
                                             &s_res);
#pragma unroll
    for (int t = 0; t < PER; ++t) {
      const bool v = (valid >> t) & 1u;
      const unsigned dg = d.is_idx ? (vi[t] >> d.shift) & dm : (unsigned)((W)vc[t] >> d.shift) & dm;
      emit(v && dg < r.j, vc[t], vi[t]);
      if (!(v && dg == r.j)) valid &= ~(1u << t);
    }
    Kr -= r.before;
    C = r.cnt;
  }
  // early stop (K == C) or the last digit: every remaining candidate is a result
#pragma unroll
  for (int t = 0; t < PER; ++t) emit((valid >> t) & 1u, vc[t], vi[t]);
  __syncthreads();
  if (tid == 0) {
    st->out_count = s_out;
    st->win_state = 4;  // done
    if (s_out != (unsigned)kk) st->error |= 4u;
  }
}

template <int KIND>
__global__ void __launch_bounds__(kBBlock, 1) batch_kernel(const BatchParams p) {
  namespace cg = cooperative_groups;
  extern __shared__ __align__(16) unsigned char batch_smem[];
  cg::grid_group grid = cg::this_grid();
  const int G = (int)gridDim.x, cta = (int)blockIdx.x;
  auto stamp = [&](int f) {
    if (p.timing && threadIdx.x == 0 && (int64_t)cta * 8 + f < p.timing_n) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      p.timing[(int64_t)cta * 8 + f] = (int64_t)t;
    }
  };
  stamp(0);
  const int64_t nch = p.batch * (int64_t)p.cpc;
  // L2 prefetch of the first chunks this CTA streams in phase B (overlaps the sampling latency)
  if (threadIdx.x < 2) {
    const int64_t ch = cta + (int64_t)threadIdx.x * G;
    if (ch < nch) {
      using U = typename KT<KIND>::U;
      const int64_t row = ch / p.cpc, ci = ch % p.cpc;
      const int64_t e0 = ci * (int64_t)kBChunkVec * (16 / sizeof(U));
      const int64_t e1 = min(p.len, e0 + (int64_t)kBChunkVec * (16 / (int64_t)sizeof(U)));
      prefetch_l2((const U*)p.keys + row * p.len + e0, (unsigned)((e1 - e0) * sizeof(U)));
    }
  }
  for (int64_t row = cta; row < p.batch; row += G) batch_sample_row<KIND>(p, row, batch_smem);
  stamp(1);
  grid.sync();
  stamp(2);
  for (int64_t ch = cta; ch < nch; ch += G) {
    const int64_t row = ch / p.cpc;
    const int ci = (int)(ch - row * p.cpc);
    const RowState* st = p.st + row;
    if (st->win_state != 1) continue;
    batch_stream_chunk<KIND>(p, row, ci, st->win_hi);
  }
  stamp(3);
  grid.sync();
  stamp(4);
  for (int64_t row = cta; row < p.batch; row += G) batch_finish_row<KIND>(p, row, batch_smem);
  stamp(5);
}

template <int KIND>
constexpr size_t batch_smem_bytes() {
  using U = typename KT<KIND>::U;
  const size_t fin = (size_t)batch_fcap<KIND>() * (sizeof(U) + 4);
  const size_t samp = (size_t)kMaxSamples * (sizeof(U) == 8 ? 8 : 4);
  return fin > samp ? fin : samp;
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
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBBlock, smem);
  if (e != cudaSuccess) return e;
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
  p.nwc = pl.nwc;
  p.scap = pl.scap;
  p.cpc = pl.cpc;
  p.nsamp = pl.nsamp;
  p.early_stop = a.early_stop;
  p.timing = a.trace;
  p.timing_n = a.batch * kTraceMaxPasses * kTraceFields;
  const int G = num_sms() * std::min(occ, 1);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)G);
  cfg.blockDim = dim3(kBBlock);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
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
