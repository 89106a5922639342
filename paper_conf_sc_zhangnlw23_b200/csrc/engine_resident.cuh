// engine_resident.cuh — small rows held in shared memory: one thread-block cluster per row, the
// row read from HBM once, every radix pass on chip.
//
// "Small rows: one CTA or one cluster per row runs a2–a7 in one launch with
// block/cluster barriers and the row held on chip when it fits" (c1: one 256 KiB row). The
// cluster engine (engine_cluster.cuh) re-reads its row from L2 in every pass and merges the
// histograms with two cluster barriers; measured on c1 (profiles/r02_*): ~6 us per pass. Here:
//
//   load   CTA r of the cluster converts its slice of the row (at most kResCap keys) to codes in
//          shared memory (128-bit loads, one pass over HBM);
//   pass q the iteration-fused pass of the paper (Alg1 L11-22) over the shared slice:
//          filter digit q-1 (digit < j -> result, == j -> candidate) and histogram digit q of the
//          candidates; ONE cluster barrier; every CTA sums the CS histograms bin-wise through
//          distributed shared memory and scans them itself (Alg1 L24-28, psum[j-1] < K <= psum[j],
//          P:100-104) — identical results everywhere, no second barrier, no broadcast;
//          histograms are double-buffered so pass q+1 never overwrites what a slower CTA reads;
//   finish once C <= kResFin candidates remain (or K == C: early stop): one filter pass
//          emits the results and appends the candidates to CTA 0's shared buffer (DSMEM), one
//          barrier, and CTA 0 selects the K remaining with block_select_smem (finish.cuh).
//
// Keys are compared as composites (code : R bits || row index : IB bits): ties at the K-th key go to
// the lowest index (reading 1). Digits follow the paper's b = 11 split (digit_of).
#pragma once

#include <cooperative_groups.h>
#include <cstdlib>

#include "device.cuh"
#include "engine.h"
#include "finish.cuh"
#include "passes.cuh"
#include "tma.cuh"

namespace airtopk {

constexpr int kRBlock = 1024;
constexpr int kMaxResCluster = 16;
constexpr int kRWarps = kRBlock / 32;
constexpr int kResFin = kResidentFin;  // candidates CTA 0 finishes

template <int KIND>
__host__ __device__ constexpr int resident_cap() {
  return sizeof(typename KT<KIND>::U) == 8 ? kResidentCap / 2 : kResidentCap;
}

struct ResidentParams {
  const void* keys;
  int64_t batch, len, k;
  int sel_min;
  int IB;
  int P;            // code + index digits
  void* out_vals;
  int64_t* out_idx;
  int64_t idx_off;
  RowState* st;     // per row: out_count (output slots), error
  int nclusters;
  int slice;        // keys per CTA (a multiple of 8)
  int early_stop;   // 0 on, -1 off
  int vec_ok;       // rows are 16-byte aligned whole vectors
  int64_t* timing;  // optional debug stamps (trace buffer): per CTA 16 %globaltimer values
  int64_t timing_n;
};

__device__ __forceinline__ void rstamp(const ResidentParams& p, int f) {
  if (p.timing && threadIdx.x == 0 && (int64_t)blockIdx.x * 16 + f < p.timing_n) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    p.timing[(int64_t)blockIdx.x * 16 + f] = (int64_t)t;
  }
}

template <typename W>
struct ResShared {
  alignas(16) unsigned hist[2][kMaxBins + 32];  // this CTA's histogram of the current pass (read remotely) + dummy bin
  SelScratch<W, kRWarps> sel;
  unsigned long long tmp[kRWarps];
  ScanResult res;
  unsigned fin_cnt;            // CTA 0: candidates appended for the finish
  unsigned out_cnt;            // CTA 0: output slots handed out (distributed shared memory atomics:
                               // a cluster round trip instead of an L2 one per emitting warp)
};

template <int KIND>
__global__ void __launch_bounds__(kRBlock, 1) resident_kernel(const ResidentParams p) {
  namespace cg = cooperative_groups;
  using U = typename KT<KIND>::U;
  using W = std::conditional_t<sizeof(U) == 8, unsigned long long, unsigned>;
  constexpr int VEC = 16 / sizeof(U);
  extern __shared__ __align__(16) unsigned char res_smem[];
  __shared__ ResShared<W> sh;
  cg::cluster_group cl = cg::this_cluster();
  // PDL: launched while the previous kernel of the stream runs; nothing global is touched before
  // its writes are visible. The next launch may then be scheduled (its launch latency overlaps us).
  pdl_wait();
  pdl_trigger();
  const int CS = (int)cl.num_blocks(), crank = (int)cl.block_rank();
  const int cid = blockIdx.x / CS;
  const int tid = threadIdx.x, lane = tid & 31;
  const bool sel_min = p.sel_min != 0;
  const U xmask = sel_min ? (U)0 : (U)~(U)0;
  U* codes = (U*)res_smem;
  U* fcode = (U*)(res_smem + (size_t)p.slice * sizeof(U));              // CTA 0: finish candidates
  unsigned* fidx = (unsigned*)(res_smem + (size_t)p.slice * sizeof(U) + (size_t)kResFin * sizeof(U));
  U* fcode0 = cl.map_shared_rank(fcode, 0);
  unsigned* fidx0 = cl.map_shared_rank(fidx, 0);
  unsigned* fcnt0 = cl.map_shared_rank(&sh.fin_cnt, 0);
  unsigned* out0 = cl.map_shared_rank(&sh.out_cnt, 0);
  const unsigned long long kk = (unsigned long long)p.k;
  rstamp(p, 0);

#pragma unroll 1
  for (int64_t row = cid; row < p.batch; row += p.nclusters) {
    RowState* st = p.st + row;
    const U* rowp = (const U*)p.keys + row * p.len;
    U* ov = (U*)p.out_vals + row * p.k;
    int64_t* oi = p.out_idx + row * p.k;
    const int64_t s0 = (int64_t)crank * p.slice;
    const int nl = (int)max((int64_t)0, min((int64_t)p.slice, p.len - s0));  // keys of this CTA
    if (crank == 0 && tid == 0) {
      st->error = 0;
      sh.fin_cnt = 0;
      sh.out_cnt = 0;
    }
    // ---- load: the slice as codes (one read of the row) ----
    if (p.vec_ok) {
      const uint4* vp = (const uint4*)(rowp + s0);
      const int nv = nl / VEC;
#pragma unroll 4
      for (int v = tid; v < nv; v += kRBlock) {
        const uint4 x = ldg_stream(vp + v);
        U c[VEC];
#pragma unroll
        for (int e = 0; e < VEC; ++e) c[e] = to_code_x<KIND>(vec_elem<U>(x, e), xmask);
        uint4 y;
        if constexpr (sizeof(U) == 4) y = make_uint4(c[0], c[1], c[2], c[3]);
        else if constexpr (sizeof(U) == 2)
          y = make_uint4(c[0] | (unsigned)c[1] << 16, c[2] | (unsigned)c[3] << 16, c[4] | (unsigned)c[5] << 16,
                         c[6] | (unsigned)c[7] << 16);
        else y = make_uint4((unsigned)c[0], (unsigned)(c[0] >> 32), (unsigned)c[1], (unsigned)(c[1] >> 32));
        ((uint4*)codes)[v] = y;
      }
    } else {
#pragma unroll 4
      for (int e = tid; e < nl; e += kRBlock) codes[e] = to_code_x<KIND>(__ldg(rowp + s0 + e), xmask);
    }
    __syncthreads();
    rstamp(p, 1);
    auto emit = [&](bool pred, U code, unsigned idx) {  // warp-aggregated output slots
      const unsigned m = __ballot_sync(kFull, pred);
      if (!m) return;
      unsigned b = 0;
      if (lane == 0) b = atomicAdd(out0, (unsigned)__popc(m));
      b = __shfl_sync(kFull, b, 0);
      if (pred) {
        const unsigned long long pos = (unsigned long long)b + __popc(m & lanemask_lt());
        if (pos < kk) {
          ov[pos] = from_code<KIND>(code, sel_min);
          oi[pos] = (int64_t)idx + p.idx_off;
        } else {
          atomicOr(&st->error, 1u);
        }
      }
    };
    // ---- radix passes over the shared slice ----
    unsigned long long K = kk, C = (unsigned long long)p.len, tcode = 0, tidx = 0;
    int q = 0;
#pragma unroll 1
    for (;; ++q) {
      const Digit dh = digit_of(q, KT<KIND>::R, p.IB);
      const Digit df = digit_of(q > 0 ? q - 1 : 0, KT<KIND>::R, p.IB);
      const unsigned hm = (1u << dh.width) - 1u, fm = (1u << df.width) - 1u;
      unsigned* hist = sh.hist[q & 1];
      for (int i = tid; i < (1 << dh.width); i += kRBlock) hist[i] = 0;
      if (tid == 0) hist[kMaxBins] = 0;
      __syncthreads();
      const W tc = (W)(tcode >> df.shift), bc = tc & ~(W)fm;
      const unsigned ti = (unsigned)(tidx >> df.shift), bi = ti & ~fm;
#pragma unroll 2
      for (int e0 = 0; e0 < nl; e0 += kRBlock) {
        const int e = e0 + tid;
        const bool in = e < nl;
        const U code = in ? codes[e] : (U)0;
        const unsigned idx = (unsigned)(s0 + e);
        bool cand = in, win = false;
        if (q > 0 && in) {
          if (!df.is_idx) {
            const W h = (W)code >> df.shift;
            win = (W)(h - bc) < (W)(tc - bc);
            cand = h == tc;
          } else {
            const bool ce = (W)code == (W)tcode;
            const unsigned h = idx >> df.shift;
            win = ce && (unsigned)(h - bi) < (unsigned)(ti - bi);
            cand = ce && h == ti;
          }
        }
        if (__any_sync(kFull, win)) emit(win, code, idx);
        // red.shared.add (equal addresses in a warp are aggregated by the hardware); non-candidates
        // hit the dummy bin instead of branching (passes.cuh)
        const unsigned d = cand ? (dh.is_idx ? (idx >> dh.shift) & hm : (unsigned)((W)code >> dh.shift) & hm)
                                : (unsigned)kMaxBins;
        shared_inc(smem_addr(hist) + 4u * d);
      }
      rstamp(p, 2 + 3 * min(q, 2));
      cl.sync();  // every CTA's histogram of digit q is complete
      rstamp(p, 3 + 3 * min(q, 2));
      // sum the CS histograms bin-wise (DSMEM) and scan: the same j, K, C in every CTA. Thread t
      // owns bins 2t, 2t+1 (scan_choose's split): ONE 8-byte remote load per cluster rank, all CS
      // loads in flight together (a rolled loop of 4-byte loads serialised ~16 DSMEM round trips)
      static_assert((kMaxBins + kRBlock - 1) / kRBlock == 2, "two bins per thread");
      unsigned s0 = 0, s1 = 0;
      {
        uint2 x[kMaxResCluster];
#pragma unroll
        for (int rr = 0; rr < kMaxResCluster; ++rr)
          if (rr < CS) x[rr] = *(const uint2*)(cl.map_shared_rank(hist, rr) + 2 * tid);
#pragma unroll
        for (int rr = 0; rr < kMaxResCluster; ++rr)
          if (rr < CS) {
            s0 += x[rr].x;
            s1 += x[rr].y;
          }
      }
      const ScanResult r = scan_choose<kRBlock>([&](int b) { return (unsigned long long)((b & 1) ? s1 : s0); },
                                                1 << dh.width, K, sh.tmp, &sh.res);
      rstamp(p, 4 + 3 * min(q, 2));
      K -= r.before;
      C = r.cnt;
      if (!dh.is_idx) tcode |= (unsigned long long)r.j << dh.shift;
      else tidx |= (unsigned long long)r.j << dh.shift;
      if ((K == C && p.early_stop == 0) || C <= (unsigned long long)kResFin || q == p.P - 1) break;
    }
    // ---- finish: results of digit q leave; candidates go to CTA 0 unless they are all results ----
    const bool all = (K == C);
    {
      const Digit df = digit_of(q, KT<KIND>::R, p.IB);
      const unsigned fm = (1u << df.width) - 1u;
      const W tc = (W)(tcode >> df.shift), bc = tc & ~(W)fm;
      const unsigned ti = (unsigned)(tidx >> df.shift), bi = ti & ~fm;
#pragma unroll 2
      for (int e0 = 0; e0 < nl; e0 += kRBlock) {
        const int e = e0 + tid;
        const bool in = e < nl;
        const U code = in ? codes[e] : (U)0;
        const unsigned idx = (unsigned)(s0 + e);
        bool win = false, cand = false;
        if (in) {
          if (!df.is_idx) {
            const W h = (W)code >> df.shift;
            win = (W)(h - bc) < (W)(tc - bc);
            cand = h == tc;
          } else {
            const bool ce = (W)code == (W)tcode;
            const unsigned h = idx >> df.shift;
            win = ce && (unsigned)(h - bi) < (unsigned)(ti - bi);
            cand = ce && h == ti;
          }
        }
        emit(win || (cand && all), code, idx);
        const bool app = cand && !all;
        const unsigned m = __ballot_sync(kFull, app);
        if (m) {
          unsigned b = 0;
          if (lane == 0) b = atomicAdd(fcnt0, (unsigned)__popc(m));
          b = __shfl_sync(kFull, b, 0);
          if (app) {
            const unsigned pos = b + __popc(m & lanemask_lt());
            if (pos < (unsigned)kResFin) {
              fcode0[pos] = code;
              fidx0[pos] = idx;
            }
          }
        }
      }
    }
    rstamp(p, 11);
    cl.sync();  // CTA 0's candidate buffer is complete
    rstamp(p, 12);
    if (crank == 0 && !all) {
      const int n = (int)min(sh.fin_cnt, (unsigned)kResFin);
      const int tcnt = (n + kRBlock - 1) / kRBlock;
      unsigned valid = 0;
      for (int t = 0; t < tcnt; ++t)
        if (tid + t * kRBlock < n) valid |= 1u << t;
      block_select_smem<KIND, kRBlock>(fcode, fidx, tcnt, valid, K, (unsigned long long)n, p.IB, p.early_stop == 0,
                                       sh.sel, emit);
      if (tid == 0 && sh.fin_cnt != C) atomicOr(&st->error, 4u);
    }
    __syncthreads();
    if (crank == 0 && tid == 0) {
      st->out_count = sh.out_cnt;
      if (sh.out_cnt != (unsigned)kk) atomicOr(&st->error, 4u);
    }
    rstamp(p, 13);
    cl.sync();  // the row is complete before its buffers are reused
  }
  rstamp(p, 14);
}

template <int KIND>
cudaError_t launch_resident_kind(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s) {
  using U = typename KT<KIND>::U;
  auto kern = resident_kernel<KIND>;
  const size_t smem = (size_t)pl.rslice * sizeof(U) + (size_t)kResFin * (sizeof(U) + 4);
  // the attribute is an upper bound: set once to the largest slice any call may use
  constexpr size_t smem_max = (size_t)resident_cap<KIND>() * sizeof(U) + (size_t)kResFin * (sizeof(U) + 4);
  cudaError_t e = func_attr(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_max);
  if (e != cudaSuccess) return e;
  e = func_attr(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  if (e != cudaSuccess) return e;
  ResidentParams p;
  p.keys = a.keys;
  p.batch = a.batch;
  p.len = a.len;
  p.k = a.k;
  p.sel_min = a.sel_min;
  p.IB = pl.IB;
  p.P = pl.P;
  p.out_vals = a.out_vals;
  p.out_idx = a.out_idx;
  p.idx_off = a.idx_off;
  p.st = (RowState*)((char*)ws + pl.off_state);
  p.slice = pl.rslice;
  p.early_stop = a.early_stop;
  p.timing = a.trace;
  p.timing_n = a.trace ? (a.trace_len > 0 ? a.trace_len : a.batch * kTraceMaxPasses * kTraceFields) : 0;
  p.vec_ok = ((uintptr_t)a.keys % 16 == 0) && ((size_t)a.len * sizeof(U)) % 16 == 0 ? 1 : 0;
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = pl.csize;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.blockDim = dim3(kRBlock);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cfg.gridDim = dim3((unsigned)pl.csize);
  int maxc = 0;
  const int key = pl.csize * 1024 + (int)(smem >> 10);
  if (!occ_cache_get((const void*)kern, key, &maxc)) {
    e = cudaOccupancyMaxActiveClusters(&maxc, kern, &cfg);
    if (e != cudaSuccess) return e;
    occ_cache_put((const void*)kern, key, maxc);
  }
  if (maxc < 1) return cudaErrorInvalidConfiguration;
  p.nclusters = (int)std::min<int64_t>(a.batch, (int64_t)maxc);
  if (getenv("AIRTOPK_RES_ONECLUSTER")) p.nclusters = 1;  // debug: rows one after another (warm caches)
  cfg.gridDim = dim3((unsigned)(p.nclusters * pl.csize));
  cfg.numAttrs = 2;  // + PDL (the occupancy query above ran on the cluster shape alone)
  if (a.events && a.n_events > 0) cudaEventRecord((cudaEvent_t)a.events[0], s);
  e = cudaLaunchKernelEx(&cfg, kern, p);
  if (a.events && a.n_events > 1) cudaEventRecord((cudaEvent_t)a.events[1], s);
  return e;
}

#define AIRTOPK_INSTANTIATE_RESIDENT(KIND) \
  template cudaError_t launch_resident_kind<KIND>(const SelectArgs&, const Plan&, void*, cudaStream_t);

}  // namespace airtopk
