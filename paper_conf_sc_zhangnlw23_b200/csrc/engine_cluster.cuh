// engine_cluster.cuh — one thread-block cluster per row, every pass in ONE launch.
//
// Same per-pass arithmetic as the grid engine (run_pass in passes.cuh: Algorithm 1 L7-22 of
// P:130), but the per-pass synchronisation of the paper's multi-kernel design (kernel boundaries +
// "last thread block" scan) is replaced by Blackwell thread-block-cluster hardware:
//   * a cluster of CS CTAs (CS <= 16) owns a row; clusters loop persistently over rows;
//   * after a pass, the CS shared-memory histograms are merged through distributed shared memory
//     (DSMEM): CTA r sums bin segment r across the cluster, publishes its segment total to every
//     CTA, and the CTA whose segment holds the K-th element finds j (psum[j-1] < K <= psum[j],
//     P:100-104) and broadcasts it — three cluster barriers, no global atomics, no extra launch;
//   * every CTA keeps an identical copy of the row state (K, C, C', prefix), so the next pass starts
//     right after the barrier; the row is re-read from L2 (a cluster's rows in flight fit the 126 MB
//     L2), candidates go to a per-cluster buffer (C < N/alpha rule), results to the output
//     through the same warp queues as the grid engine.
// Used for batched rows and small rows (c1, c2), where the grid engine's per-pass launches and
// last-block scans dominate.
#pragma once

#include <algorithm>
#include <cooperative_groups.h>
#include <cstdlib>

#include "device.cuh"
#include "engine.h"
#include "passes.cuh"

namespace airtopk {

namespace cg = cooperative_groups;

constexpr int kCBlock = 512;
constexpr int kCWarps = kCBlock / 32;
constexpr int kMaxCluster = 16;
struct ClusterParams {
  const void* keys;
  const int64_t* in_idx;
  int64_t batch, len, k;
  int sel_min;
  int P, IB;
  void* out_vals;
  int64_t* out_idx;
  RowState* st;  // per row (same workspace layout as the grid engine; counters, window outcome)
  void* bcode;   // per row: 2 x cap_alloc codes   (slot-major: [slot][row][cap])
  void* bidx;    // per row: 2 x cap_alloc indices
  int64_t cap_rule, cap_alloc;
  int nclusters;
  int early_stop;  // 0 on, -1 off (ablation)
  int64_t idx_off; // added to every output index (airtopk_select_shard)
  int tail;      // 1: continue rows after the grid engine's window pass;
                 // 2: fallback after the batched engine: only rows with win_state == 3, from L
  int tail_q;    // tail mode: the grid engine ran passes q < tail_q after the window pass
  int timing_stride;  // int64 slots per CTA in `timing` (8; 24 with the merge-phase stamps, debug)
  int64_t* timing;  // optional: per CTA [globaltimer at start, at end, rows done, passes run, end of passes 1-4]
  const unsigned* fail;  // tail == 2: [0] = number of rows to redo, [1 + i] = the rows
};

struct ClusterShared {
  unsigned long long res_before, res_cnt;  // target digit result, written remotely by the owner
  unsigned res_j;
  unsigned long long tmp[kCWarps];
  ScanResult scan;
};

// The cluster engine keeps ONE histogram copy: its passes are short, so zeroing/merging copies
// costs more than the same-bin serialisation they avoid.
template <int KIND, typename IdxT, int DF, int DH, bool HASIDX>
__device__ __forceinline__ unsigned long long cluster_pass(PassCtx<typename KT<KIND>::U, IdxT>& c) {
  // 8 buffer entries per thread per iteration: the few CTAs of a cluster need deep memory-level
  // parallelism to stream a candidate buffer from L2
  return run_pass<KIND, IdxT, DF, DH, HASIDX, kCBlock, 1, false, 8>(c);
}

template <int KIND, typename IdxT, bool HASIDX>
__global__ void __launch_bounds__(kCBlock, 1) cluster_kernel(const ClusterParams p) {
  using U = typename KT<KIND>::U;
  constexpr int HC = 1;
  extern __shared__ unsigned sh_hist[];  // kHistSlots counters
  __shared__ WarpQ<U, IdxT> sh_wq[kCWarps];
  __shared__ ClusterShared cs;
  __shared__ __align__(16) unsigned sh_seg[kMaxBins];  // the cluster's merged histogram (each CTA's copy)

  cg::cluster_group cl = cg::this_cluster();
  const int CS = (int)cl.num_blocks();
  const int crank = (int)cl.block_rank();
  const int cid = blockIdx.x / CS;
  const int tid = threadIdx.x, warp = tid >> 5;
  const bool sel_min = p.sel_min != 0;
  const unsigned long long N = (unsigned long long)p.len;
  const unsigned long long kk = (unsigned long long)p.k;
  const unsigned long long cap = (unsigned long long)p.cap_rule;

  // PDL (every mode): the previous launch — the window pass or the batch kernel in tail / fallback
  // mode, any kernel standalone — has finished and its writes are visible; the next launch may be
  // scheduled while we run
  pdl_wait();
  pdl_trigger();
  unsigned long long t_start = 0;
  int n_rows = 0, n_passes = 0;
  if (p.timing && tid == 0) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_start));
  // debug timing of the merge / scan phases of the first two passes (slots 8 + 5 * pass + phase)
  auto stamp = [&](int phase) {
    if (p.timing && p.timing_stride >= 24 && tid == 0 && n_passes >= 1 && n_passes <= 2) {
      unsigned long long tp;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tp));
      p.timing[(int64_t)blockIdx.x * p.timing_stride + 8 + 5 * (n_passes - 1) + phase] = (int64_t)tp;
    }
  };

  const int64_t nrows = (p.tail == 2) ? (int64_t)p.fail[0] : p.batch;  // fallback: only the failed rows
  for (int64_t it = cid; it < nrows; it += p.nclusters) {
    const int64_t row = (p.tail == 2) ? (int64_t)p.fail[1 + it] : it;
    RowState* st = p.st + row;
    unsigned long long K = kk, C = N, Cp = N, tcode = 0, tidx = 0;
    int stop1 = 0, src1 = 0;  // src1: 0 = the input row L, s + 1 = candidate buffer slot s
    int q0 = 0;
    const int ws = p.tail == 1 ? st->win_state : 0;
    if (p.tail != 1) {  // standalone: the row's counters start at zero (no memset launch before the kernel)
      if (crank == 0 && tid == 0) {
        st->out_count = 0;
        st->buf_count[0] = 0;
        st->buf_count[1] = 0;
        st->error = 0;
      }
      cl.sync();
    }
    if (p.tail == 1 && (ws == 1 || p.tail_q > 0)) {
      // continue the row from its state: after the window pass (which scanned pass 1 over the window
      // buffer) or after the grid passes q < tail_q
      K = st->K;
      C = st->C;
      Cp = st->Cp;
      src1 = st->src1;
      tcode = st->tcode;
      tidx = st->tidx;
      stop1 = st->stop1;
      q0 = st->npass;
    }
    if (ws == 1) {
      // Every window member lies in [wmin, wmax]: while all key bits above digit q agree between the
      // two (so no result of an earlier digit is pending), pass q's histogram is a single bin (j = that
      // digit, K and C unchanged) and the pass is skipped — the paper's adaptivity applied to the
      // digits.
      const unsigned long long wmin = ~st->win_nmin, wmax = st->win_max;
      const int pc = code_passes(KT<KIND>::R);
      while (stop1 == 0 && q0 < pc) {
        const Digit d = digit_of(q0, KT<KIND>::R, p.IB);
        if ((wmin >> d.shift) != (wmax >> d.shift)) break;
        tcode |= ((wmin >> d.shift) & ((1ull << d.width) - 1ull)) << d.shift;
        ++q0;
      }
    }
    for (int q = q0; q <= p.P; ++q) {
      if (stop1 != 0 && stop1 - 1 < q - 1) break;
      const int DF = q == 0 ? 0 : (digit_of(q - 1, KT<KIND>::R, p.IB).is_idx ? 2 : 1);
      const int DH = q == p.P ? 0 : (digit_of(q, KT<KIND>::R, p.IB).is_idx ? 2 : 1);
      const int sslot = (src1 == 1) ? 1 : 0;
      PassCtx<U, IdxT> c;
      c.q = q;
      c.emit_all = (DF != 0) && ((stop1 != 0 && stop1 - 1 == q - 1) || DH == 0);
      c.do_hist = (DH != 0) && !c.emit_all;
      c.srcL = (src1 == 0);                                      // Alg1 L7-8
      c.store = c.do_hist && (DF != 0) && (C <= cap);           // Alg1 L17
      c.sel_min = sel_min;
      c.reverse = (q & 1) != 0;
      c.dh = digit_of(q, KT<KIND>::R, p.IB);
      c.df = digit_of(DF != 0 ? q - 1 : 0, KT<KIND>::R, p.IB);
      c.tcode = tcode;
      c.tidx = tidx;
      c.lo = 0;
      c.wnmin = nullptr;
      c.wmax = nullptr;
      c.span1 = 0;
      c.rowp = (const U*)p.keys + row * p.len;
      c.rowi = HASIDX ? p.in_idx + row * p.len : nullptr;
      c.len = p.len;
      c.slice = crank;
      c.nslices = CS;
      const int islot = src1 > 0 ? src1 - 1 : 0;
      c.bcin = (const U*)p.bcode + ((size_t)islot * p.batch + row) * p.cap_alloc;
      c.biin = (const IdxT*)p.bidx + ((size_t)islot * p.batch + row) * p.cap_alloc;
      c.nbuf = (src1 > 0) ? __ldcg(&st->buf_count[islot]) : 0ull;
      c.ov = (U*)p.out_vals + row * p.k;
      c.oi = p.out_idx + row * p.k;
      c.ioff = p.idx_off;
      c.outc = &st->out_count;
      c.kk = kk;
      c.bco = (U*)p.bcode + ((size_t)sslot * p.batch + row) * p.cap_alloc;
      c.bio = (IdxT*)p.bidx + ((size_t)sslot * p.batch + row) * p.cap_alloc;
      c.bufc = &st->buf_count[sslot];
      c.capa = (unsigned long long)p.cap_alloc;
      c.err = &st->error;
      c.hist = sh_hist;
      c.ring = 0;
      c.wq = &sh_wq[warp];
      const bool hist_on = c.do_hist || DF == 0;
      if (hist_on) {
        for (int i = tid; i < kHistSlots * HC; i += kCBlock) sh_hist[i] = 0;
      }
      __syncthreads();
      switch (DF * 3 + DH) {
        case 0 * 3 + 1: cluster_pass<KIND, IdxT, 0, 1, HASIDX>(c); break;
        case 1 * 3 + 1: cluster_pass<KIND, IdxT, 1, 1, HASIDX>(c); break;
        case 1 * 3 + 2: cluster_pass<KIND, IdxT, 1, 2, HASIDX>(c); break;
        case 2 * 3 + 2: cluster_pass<KIND, IdxT, 2, 2, HASIDX>(c); break;
        default: cluster_pass<KIND, IdxT, 2, 0, HASIDX>(c); break;
      }
      ++n_passes;
      if (p.timing && tid == 0 && n_passes <= 4) {
        unsigned long long tp;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tp));
        p.timing[(int64_t)blockIdx.x * p.timing_stride + 3 + n_passes] = (int64_t)tp;
      }
      if (!hist_on) break;  // emit-all pass: the row is complete

      // ---- histogram merge + scan (replaces the last-block scan) ----
      const int nb = 1 << c.dh.width;
      if (CS == 1) {
        // one CTA per row: its histogram is the row's; scan it in place
        __syncthreads();
        const ScanResult r = scan_choose<kCBlock>(
            [&](int b) { return (unsigned long long)sh_hist[b]; }, nb, K, cs.tmp, &cs.scan);
        if (tid == 0) {
          cs.res_j = r.j;
          cs.res_before = r.before;
          cs.res_cnt = r.cnt;
        }
        if (c.store) src1 = sslot + 1;  // the buffer this pass wrote feeds the next one
        if (tid == 0) st->buf_count[src1 == 1 ? 1 : 0] = 0;  // next pass's output buffer
        __syncthreads();
      } else {
        cl.sync();  // (B) every CTA's histogram and appends are complete
        stamp(0);
        // CTA r owns bins [r*seg, (r+1)*seg): sums them over the cluster (all CS DSMEM loads of a bin
        // in flight at once) and stores the sums into EVERY CTA's full merged histogram (sh_seg), so
        // that after the next barrier each CTA scans all bins locally (no remote loads on the scan)
        const int seg = (nb + CS - 1) / CS;
        const int b0 = crank * seg;
        for (int b = tid; b < seg; b += kCBlock) {
          if (b0 + b < nb) {
            unsigned v = 0;
            for (int r0 = 0; r0 < CS; r0 += 4) {  // 4 DSMEM loads in flight (few registers)
              unsigned x[4];
#pragma unroll
              for (int i = 0; i < 4; ++i) x[i] = (r0 + i < CS) ? cl.map_shared_rank(sh_hist, r0 + i)[b0 + b] : 0u;
              v += x[0] + x[1] + x[2] + x[3];
            }
            for (int rr = 0; rr < CS; ++rr) cl.map_shared_rank(sh_seg, rr)[b0 + b] = v;
          }
        }
        stamp(1);
        if (c.store) src1 = sslot + 1;
        if (crank == 0 && tid == 0) st->buf_count[src1 == 1 ? 1 : 0] = 0;  // next pass's output buffer
        cl.sync();  // (C) merged histogram complete everywhere; remote reads of sh_hist done
        stamp(2);
        const ScanResult r = scan_choose<kCBlock>(
            [&](int b) { return (unsigned long long)sh_seg[b]; }, nb, K, cs.tmp, &cs.scan);
        if (tid == 0) {
          cs.res_j = r.j;
          cs.res_before = r.before;
          cs.res_cnt = r.cnt;
        }
        __syncthreads();
        stamp(3);
      }
      const unsigned j = cs.res_j;
      const unsigned long long newK = K - cs.res_before, newC = cs.res_cnt;   // Alg1 L26-28
      Cp = C;
      C = newC;
      K = newK;
      if (!c.dh.is_idx) tcode |= (unsigned long long)j << c.dh.shift;
      else tidx |= (unsigned long long)j << c.dh.shift;
      if (newK == newC && p.early_stop == 0) stop1 = q + 1;                                       // early stop
    }
    cl.sync();  // the cluster finishes the row before its buffers are reused
    ++n_rows;
  }
  if (p.timing && tid == 0) {
    unsigned long long t_end;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_end));
    int64_t* t = p.timing + (int64_t)blockIdx.x * p.timing_stride;
    t[0] = (int64_t)t_start; t[1] = (int64_t)t_end; t[2] = n_rows; t[3] = n_passes;
  }
}

}  // namespace airtopk

namespace airtopk {

template <int KIND, typename IdxT, bool HASIDX>
cudaError_t launch_cluster_t(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s, int tail) {
  auto kern = cluster_kernel<KIND, IdxT, HASIDX>;
  constexpr size_t smem = (size_t)kHistSlots * 4;
  const cudaError_t attr1 = func_attr(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  const cudaError_t attr2 = func_attr(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  if (attr1 != cudaSuccess) return attr1;
  if (attr2 != cudaSuccess) return attr2;
  char* base = (char*)ws;
  cudaError_t e = cudaSuccess;
  ClusterParams p;
  p.keys = a.keys;
  p.in_idx = a.in_idx;
  p.batch = a.batch;
  p.len = a.len;
  p.k = a.k;
  p.sel_min = a.sel_min;
  p.P = pl.P;
  p.IB = pl.IB;
  p.out_vals = a.out_vals;
  p.out_idx = a.out_idx;
  p.st = (RowState*)(base + pl.off_state);
  p.bcode = base + pl.off_bcode;
  p.bidx = base + pl.off_bidx;
  p.cap_rule = pl.cap_rule;
  p.cap_alloc = pl.cap_alloc;
  p.tail = tail;
  p.early_stop = a.early_stop;
  p.idx_off = a.idx_off;
  p.tail_q = pl.tail_q;
  // standalone cluster engine: the trace buffer receives per-CTA timing instead (not in tail /
  // fallback mode: the trace then belongs to the engine that ran before)
  p.timing = tail ? nullptr : a.trace;
  p.fail = (const unsigned*)(base + pl.off_bfail);
  p.timing_stride = getenv("AIRTOPK_CLUSTER_TIMING") ? 24 : 8;

  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = pl.csize;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.blockDim = dim3(kCBlock, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cfg.attrs = at;
  cfg.numAttrs = 1;  // (the occupancy query below runs on the cluster shape alone; PDL added for the launch)
  cfg.gridDim = dim3((unsigned)pl.csize, 1, 1);
  int maxc = 0;
  if (!occ_cache_get((const void*)kern, pl.csize * 4 + (tail ? 1 : 0), &maxc)) {
    e = cudaOccupancyMaxActiveClusters(&maxc, kern, &cfg);
    if (e != cudaSuccess) return e;
    occ_cache_put((const void*)kern, pl.csize * 4 + (tail ? 1 : 0), maxc);
  }
  if (maxc < 1) return cudaErrorInvalidConfiguration;
  const int64_t ncl = std::min<int64_t>(a.batch, (int64_t)maxc);
  // the per-CTA timing must fit the caller's trace buffer (batch x kTraceMaxPasses x kTraceFields
  // int64 or trace_len, airtopk.h): otherwise no timing (debug only) — never an out-of-bounds write
  //
  if (p.timing && ncl * pl.csize * (int64_t)p.timing_stride >
                      (a.trace_len > 0 ? a.trace_len : a.batch * kTraceMaxPasses * kTraceFields))
    p.timing = nullptr;
  p.nclusters = (int)ncl;
  cfg.gridDim = dim3((unsigned)(ncl * pl.csize), 1, 1);
  cfg.numAttrs = 2;
  if (!tail && a.events && a.n_events > 0) cudaEventRecord((cudaEvent_t)a.events[0], s);
  e = cudaLaunchKernelEx(&cfg, kern, p);
  if (!tail && a.events && a.n_events > 1) cudaEventRecord((cudaEvent_t)a.events[1], s);
  return e;
}

template <int KIND>
cudaError_t launch_cluster_kind(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s, int tail) {
  if (a.in_idx) return launch_cluster_t<KIND, uint64_t, true>(a, pl, ws, s, tail);
  if (pl.idx64) return launch_cluster_t<KIND, uint64_t, false>(a, pl, ws, s, tail);
  return launch_cluster_t<KIND, uint32_t, false>(a, pl, ws, s, tail);
}

#define AIRTOPK_INSTANTIATE_CLUSTER(KIND) \
  template cudaError_t launch_cluster_kind<KIND>(const SelectArgs&, const Plan&, void*, cudaStream_t, int);

}  // namespace airtopk
