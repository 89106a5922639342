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

#include <cooperative_groups.h>

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
  unsigned long long* counters;  // per row: out_count, buf_count[2], error (zeroed by the launcher)
  void* bcode;                   // per cluster: 2 x cap_alloc codes
  void* bidx;                    // per cluster: 2 x cap_alloc indices
  int64_t cap_rule, cap_alloc;
  int nclusters;
};

struct ClusterShared {
  unsigned long long segtot[kMaxCluster];  // segment totals, written remotely by each CTA
  unsigned long long res_before, res_cnt;  // target digit result, written remotely by the owner
  unsigned res_j;
  unsigned long long tmp[kCWarps];
  ScanResult scan;
};

template <int KIND, typename IdxT, int DF, int DH, bool HASIDX>
__device__ __forceinline__ unsigned long long cluster_pass(PassCtx<typename KT<KIND>::U, IdxT>& c) {
  return run_pass<KIND, IdxT, DF, DH, HASIDX, kCBlock>(c);
}

template <int KIND, typename IdxT, bool HASIDX>
__global__ void __launch_bounds__(kCBlock, 1) cluster_kernel(const ClusterParams p) {
  using U = typename KT<KIND>::U;
  constexpr int HC = hist_copies<KIND, IdxT, 1>();
  extern __shared__ unsigned sh_hist[];  // kMaxBins * HC
  __shared__ WarpQ<U, IdxT> sh_oq[kCWarps];
  __shared__ WarpQ<U, IdxT> sh_bq[kCWarps];
  __shared__ ClusterShared cs;
  __shared__ unsigned sh_seg[kMaxBins];  // this CTA's merged bin segment

  cg::cluster_group cl = cg::this_cluster();
  const int CS = (int)cl.num_blocks();
  const int crank = (int)cl.block_rank();
  const int cid = blockIdx.x / CS;
  const int tid = threadIdx.x, warp = tid >> 5;
  const bool sel_min = p.sel_min != 0;
  const unsigned long long N = (unsigned long long)p.len;
  const unsigned long long kk = (unsigned long long)p.k;
  const unsigned long long cap = (unsigned long long)p.cap_rule;

  U* const bcode0 = (U*)p.bcode + (size_t)cid * 2 * p.cap_alloc;
  IdxT* const bidx0 = (IdxT*)p.bidx + (size_t)cid * 2 * p.cap_alloc;

  for (int64_t row = cid; row < p.batch; row += p.nclusters) {
    unsigned long long* ctr = p.counters + row * 4;
    unsigned long long K = kk, C = N, Cp = N, tcode = 0, tidx = 0;
    int stop1 = 0;
    for (int q = 0; q <= p.P; ++q) {
      if (stop1 != 0 && stop1 - 1 < q - 1) break;
      const int DF = q == 0 ? 0 : (digit_of(q - 1, KT<KIND>::R, p.IB).is_idx ? 2 : 1);
      const int DH = q == p.P ? 0 : (digit_of(q, KT<KIND>::R, p.IB).is_idx ? 2 : 1);
      PassCtx<U, IdxT> c;
      c.q = q;
      c.emit_all = (DF != 0) && ((stop1 != 0 && stop1 - 1 == q - 1) || DH == 0);
      c.do_hist = (DH != 0) && !c.emit_all;
      c.srcL = (DF == 0) || (Cp > cap);
      c.store = c.do_hist && (DF != 0) && (C <= cap);
      c.sel_min = sel_min;
      c.reverse = (q & 1) != 0;
      c.dh = digit_of(q, KT<KIND>::R, p.IB);
      c.df = digit_of(DF != 0 ? q - 1 : 0, KT<KIND>::R, p.IB);
      c.tcode = tcode;
      c.tidx = tidx;
      c.rowp = (const U*)p.keys + row * p.len;
      c.rowi = HASIDX ? p.in_idx + row * p.len : nullptr;
      c.len = p.len;
      c.slice = crank;
      c.nslices = CS;
      const int islot = (q - 1) & 1;
      c.bcin = bcode0 + (size_t)islot * p.cap_alloc;
      c.biin = bidx0 + (size_t)islot * p.cap_alloc;
      c.nbuf = (DF != 0 && !c.srcL) ? __ldcg(&ctr[1 + islot]) : 0ull;
      c.ov = (U*)p.out_vals + row * p.k;
      c.oi = p.out_idx + row * p.k;
      c.outc = &ctr[0];
      c.kk = kk;
      c.bco = bcode0 + (size_t)(q & 1) * p.cap_alloc;
      c.bio = bidx0 + (size_t)(q & 1) * p.cap_alloc;
      c.bufc = &ctr[1 + (q & 1)];
      c.capa = (unsigned long long)p.cap_alloc;
      c.err = (unsigned*)&ctr[3];
      c.hist = sh_hist;
      c.oq = &sh_oq[warp];
      c.bq = &sh_bq[warp];
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
      if (!hist_on) break;  // emit-all pass: the row is complete

      // ---- cluster-wide histogram merge + scan (replaces the last-block scan) ----
      cl.sync();  // (B) every CTA's histogram and appends are complete
      const int hc = (DF == 0) ? 1 : HC;   // copies used by this pass
      const int nb = 1 << c.dh.width;
      const int seg = (nb + CS - 1) / CS;
      const int b0 = crank * seg;
      unsigned long long mytot = 0;
      for (int i = tid; i < seg; i += kCBlock) {
        const int b = b0 + i;
        unsigned v = 0;
        if (b < nb) {
          for (int r = 0; r < CS; ++r) {
            const unsigned* rh = cl.map_shared_rank(sh_hist, r);
            for (int h = 0; h < hc; ++h) v += rh[b * hc + h];
          }
        }
        sh_seg[i] = v;
        mytot += v;
      }
      // block reduction of mytot
      {
        unsigned long long tot;
        (void)block_exclusive_scan<kCBlock>(mytot, cs.tmp, tot);
        if (tid == 0) {
          for (int r = 0; r < CS; ++r) cl.map_shared_rank(&cs, r)->segtot[crank] = tot;
        }
      }
      cl.sync();  // (C) all segment totals published; all remote reads of sh_hist done
      unsigned long long before_seg = 0;
      int owner = -1;
      {
        unsigned long long run = 0;
        for (int r = 0; r < CS; ++r) {
          const unsigned long long t = cs.segtot[r];
          if (owner < 0 && run < K && run + t >= K) { owner = r; before_seg = run; }
          run += t;
        }
      }
      if (crank == owner) {
        const unsigned long long Kseg = K - before_seg;
        const ScanResult r = scan_choose<kCBlock>(
            [&](int b) { return (unsigned long long)sh_seg[b]; }, seg, Kseg, cs.tmp, &cs.scan);
        if (tid == 0) {
          for (int rr = 0; rr < CS; ++rr) {
            ClusterShared* o = cl.map_shared_rank(&cs, rr);
            o->res_j = (unsigned)(b0 + r.j);
            o->res_before = before_seg + r.before;
            o->res_cnt = r.cnt;
          }
        }
      }
      if (crank == 0 && tid == 0) ctr[1 + ((q + 1) & 1)] = 0;  // buffer slot of pass q+1
      cl.sync();  // (D) result visible everywhere
      const unsigned j = cs.res_j;
      const unsigned long long newK = K - cs.res_before, newC = cs.res_cnt;   // Alg1 L26-28
      Cp = C;
      C = newC;
      K = newK;
      if (!c.dh.is_idx) tcode |= (unsigned long long)j << c.dh.shift;
      else tidx |= (unsigned long long)j << c.dh.shift;
      if (newK == newC) stop1 = q + 1;                                       // early stop
    }
    cl.sync();  // the cluster finishes the row before its buffers are reused
  }
}

}  // namespace airtopk

namespace airtopk {

template <int KIND, typename IdxT, bool HASIDX>
cudaError_t launch_cluster_t(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s) {
  auto kern = cluster_kernel<KIND, IdxT, HASIDX>;
  constexpr size_t smem = (size_t)kHistSlots * 4 * hist_copies<KIND, IdxT, 1>();
  static const cudaError_t attr1 = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  static const cudaError_t attr2 = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  if (attr1 != cudaSuccess) return attr1;
  if (attr2 != cudaSuccess) return attr2;
  char* base = (char*)ws;
  cudaError_t e = cudaMemsetAsync(base + pl.off_state, 0, (size_t)a.batch * 32, s);
  if (e != cudaSuccess) return e;
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
  p.counters = (unsigned long long*)(base + pl.off_state);
  p.bcode = base + pl.off_bcode;
  p.bidx = base + pl.off_bidx;
  p.cap_rule = pl.cap_rule;
  p.cap_alloc = pl.cap_alloc;

  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = pl.csize;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.blockDim = dim3(kCBlock, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cfg.gridDim = dim3((unsigned)pl.csize, 1, 1);
  int maxc = 0;
  e = cudaOccupancyMaxActiveClusters(&maxc, kern, &cfg);
  if (e != cudaSuccess) return e;
  if (maxc < 1) return cudaErrorInvalidConfiguration;
  const int64_t ncl = std::min<int64_t>({a.batch, (int64_t)maxc, (int64_t)pl.max_clusters});
  p.nclusters = (int)ncl;
  cfg.gridDim = dim3((unsigned)(ncl * pl.csize), 1, 1);
  if (a.events && a.n_events > 0) cudaEventRecord((cudaEvent_t)a.events[0], s);
  e = cudaLaunchKernelEx(&cfg, kern, p);
  if (a.events && a.n_events > 1) cudaEventRecord((cudaEvent_t)a.events[1], s);
  return e;
}

template <int KIND>
cudaError_t launch_cluster_kind(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s) {
  if (a.in_idx) return launch_cluster_t<KIND, uint64_t, true>(a, pl, ws, s);
  if (pl.idx64) return launch_cluster_t<KIND, uint64_t, false>(a, pl, ws, s);
  return launch_cluster_t<KIND, uint32_t, false>(a, pl, ws, s);
}

#define AIRTOPK_INSTANTIATE_CLUSTER(KIND) \
  template cudaError_t launch_cluster_kind<KIND>(const SelectArgs&, const Plan&, void*, cudaStream_t);

}  // namespace airtopk
