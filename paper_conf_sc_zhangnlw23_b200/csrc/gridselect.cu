// gridselect.cu — GridSelect, the paper's second top-K algorithm (§4).
//
// WarpSelect with ONE shared queue per warp and multiple thread blocks:
//   * every warp keeps its K best elements so far as a sorted list in shared memory and a 32-entry
//     queue in shared memory ("the size of the shared queue is set to 32");
//   * parallel two-step insertion (Fig. 5): each lane compares its element with the K-th
//     best known so far; a warp ballot gives every qualified lane a unique queue position; lanes
//     whose position is < 32 insert at once; if the queue is then full, it is sorted (bitonic, across
//     the 32 lanes) and merged into the list, the threshold is updated, and the lanes whose position
//     was >= 32 insert at position - 32 (after re-checking against the new threshold);
//   * multiple thread blocks: a row is split over G CTAs x W warps; each warp writes its list
//     to the workspace, and the last CTA of the row (atomic ticket) runs the same warp
//     procedure over the G*W*K candidates and writes the row's K results.
// Elements are compared as composite keys (order-preserving code : 32 bits || row index : 32 bits),
// so ties at the K-th value go to the lowest indices (reading 1) and all keys are distinct.
// Scope: keys of <= 32 bits, len < 2^32, K <= kGsMaxK. Output rows come out sorted (ascending in
// the selection order).
#include <algorithm>

#include "device.cuh"
#include "engine.h"

namespace airtopk {

constexpr int kGsWarps = 8;
constexpr int kGsBlock = kGsWarps * 32;
constexpr int kGsMaxK = 256;
constexpr unsigned long long kGsInf = ~0ull;  // sorts after every real composite key

struct GsParams {
  const void* keys;
  int64_t batch, len, k;
  int sel_min;
  void* out_vals;
  int64_t* out_idx;
  unsigned long long* cand;  // [batch][G * kGsWarps][k] per-warp sorted lists
  unsigned* ticket;          // [batch]
  int G;                     // CTAs per row
  int64_t per_warp;          // elements per warp slice
};

struct GsWarp {
  unsigned long long list[2][kGsMaxK];  // sorted K best (double buffer for the merge)
  unsigned long long q[32];             // the shared queue
};

// Bitonic sort of one value per lane, ascending by lane (15 compare-exchange steps over shuffles).
__device__ __forceinline__ unsigned long long warp_sort32(unsigned long long v) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int size = 2; size <= 32; size <<= 1) {
#pragma unroll
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      const unsigned long long o = __shfl_xor_sync(kFull, v, stride);
      const bool up = ((lane & size) == 0);
      const bool lower = ((lane & stride) == 0);
      const unsigned long long mn = v < o ? v : o, mx = v < o ? o : v;
      v = (lower == up) ? mn : mx;
    }
  }
  return v;
}

// Queue full (or final flush): sort the queue, merge it into the sorted list keeping the K smallest
// (stable merge by ranks: list entry i goes to i + #{queue < it}, queue entry j to
// j + #{list <= it}), return the new K-th best (the insertion threshold).
__device__ __forceinline__ unsigned long long gs_flush(GsWarp& w, int& cur, int K, int qn) {
  const int lane = threadIdx.x & 31;
  const unsigned long long qv = warp_sort32(lane < qn ? w.q[lane] : kGsInf);
  w.q[lane] = qv;
  __syncwarp();
  const unsigned long long* L = w.list[cur];
  unsigned long long* Nn = w.list[cur ^ 1];
  for (int i = lane; i < K; i += 32) {
    const unsigned long long x = L[i];
    int lo = 0, hi = 32;  // #{queue < x}
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (w.q[mid] < x) lo = mid + 1; else hi = mid;
    }
    if (i + lo < K) Nn[i + lo] = x;
  }
  {
    int lo = 0, hi = K;  // #{list <= qv}
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (L[mid] <= qv) lo = mid + 1; else hi = mid;
    }
    if (lane + lo < K) Nn[lane + lo] = qv;
  }
  __syncwarp();
  cur ^= 1;
  return w.list[cur][K - 1];
}

// Two-step insertion of one element per lane: returns the updated queue fill.
__device__ __forceinline__ int gs_insert(GsWarp& w, int& cur, int K, unsigned long long x, unsigned long long& thr,
                                         int qn) {
  bool ok = x < thr;
  const unsigned m = __ballot_sync(kFull, ok);
  if (!m) return qn;
  const int pos = qn + __popc(m & lanemask_lt());
  if (ok && pos < 32) w.q[pos] = x;  // step 1
  qn += __popc(m);
  if (qn >= 32) {
    __syncwarp();
    thr = gs_flush(w, cur, K, 32);
    ok = ok && pos >= 32 && x < thr;  // step 2: the overflow, shifted down by 32
    const unsigned m2 = __ballot_sync(kFull, ok);
    if (ok) w.q[__popc(m2 & lanemask_lt())] = x;
    qn = __popc(m2);
  }
  __syncwarp();
  return qn;
}

// One warp's GridSelect over n composite keys produced by get(i) (i < n), kGsUnroll elements per
// lane loaded up front (memory-level parallelism), element (t, lane) of a round = base + 32 t + lane.
// Returns with the warp's list (w.list[cur]) holding its K best.
constexpr int kGsUnroll = 16;
template <typename Get>
__device__ __forceinline__ void gs_warp_run(GsWarp& w, int& cur, int K, int64_t n, Get get) {
  const int lane = threadIdx.x & 31;
  for (int i = lane; i < kGsMaxK; i += 32) w.list[cur][i] = kGsInf;
  __syncwarp();
  unsigned long long thr = kGsInf;
  int qn = 0;
  for (int64_t b = 0; b < n; b += 32 * kGsUnroll) {
    unsigned long long x[kGsUnroll];
#pragma unroll
    for (int t = 0; t < kGsUnroll; ++t) {
      const int64_t i = b + 32 * t + lane;
      x[t] = (i < n) ? get(i) : kGsInf;
    }
#pragma unroll
    for (int t = 0; t < kGsUnroll; ++t) qn = gs_insert(w, cur, K, x[t], thr, qn);
  }
  if (qn > 0) gs_flush(w, cur, K, qn);
}

template <int KIND>
__global__ void __launch_bounds__(kGsBlock) gridselect_kernel(const GsParams p) {
  using U = typename KT<KIND>::U;
  __shared__ GsWarp sw[kGsWarps];
  __shared__ int sh_last;
  const int64_t row = blockIdx.x / p.G;
  const int cta = blockIdx.x % p.G;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int K = (int)p.k;
  const bool sel_min = p.sel_min != 0;
  const U* rowp = (const U*)p.keys + row * p.len;
  GsWarp& w = sw[warp];
  int cur = 0;
  // this warp's slice of the row
  const int64_t gw = (int64_t)cta * kGsWarps + warp;
  const int64_t e0 = std::min<int64_t>(p.len, gw * p.per_warp), e1 = std::min<int64_t>(p.len, e0 + p.per_warp);
  gs_warp_run(w, cur, K, e1 - e0, [&](int64_t i) -> unsigned long long {
    const int64_t pos = e0 + i;
    return ((unsigned long long)to_code<KIND>(__ldg(rowp + pos), sel_min) << 32) | (unsigned long long)pos;
  });
  unsigned long long* cand = p.cand + (size_t)row * p.G * kGsWarps * K;
  for (int i = lane; i < K; i += 32) cand[gw * K + i] = w.list[cur][i];
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) sh_last = (ticket_arrive(&p.ticket[row]) == (unsigned)(p.G - 1));
  __syncthreads();
  if (!sh_last) return;
  // last CTA of the row: the same procedure over the G * W candidate lists (split over its warps),
  // then warp 0 over the W lists of its warps
  const int64_t nc = (int64_t)p.G * kGsWarps * K;
  const int64_t per = (nc + kGsWarps - 1) / kGsWarps;
  const int64_t c0 = std::min<int64_t>(nc, warp * per), c1 = std::min<int64_t>(nc, c0 + per);
  cur = 0;
  gs_warp_run(w, cur, K, c1 - c0, [&](int64_t i) { return __ldcg(cand + c0 + i); });
  __syncthreads();
  if (warp != 0) {
    // publish this warp's list in its queue-independent buffer for warp 0
    if (cur != 1) {
      for (int i = lane; i < K; i += 32) w.list[1][i] = w.list[0][i];
    }
  }
  __syncthreads();
  if (warp == 0) {
    // warp 0: keep its own list, then insert every other warp's list through the queue
    unsigned long long thr = w.list[cur][K - 1];
    int qn = 0;
    for (int ow = 1; ow < kGsWarps; ++ow) {
      const unsigned long long* src = sw[ow].list[1];
      for (int b = 0; b < K; b += 32) {
        const int i = b + lane;
        qn = gs_insert(w, cur, K, (i < K) ? src[i] : kGsInf, thr, qn);
      }
    }
    if (qn > 0) gs_flush(w, cur, K, qn);
    U* ov = (U*)p.out_vals + row * p.k;
    int64_t* oi = p.out_idx + row * p.k;
    for (int i = lane; i < K; i += 32) {
      const unsigned long long x = w.list[cur][i];
      ov[i] = from_code<KIND>((U)(x >> 32), sel_min);
      oi[i] = (int64_t)(x & 0xffffffffull);
    }
  }
  if (threadIdx.x == 0) p.ticket[row] = 0;
}

bool gridselect_supported(const SelectArgs& a) {
  return a.in_idx == nullptr && key_bits(a.kind) <= 32 && a.len < (int64_t(1) << 32) && a.k <= kGsMaxK;
}

// CTAs per row: >= 1K elements per warp, at most enough CTAs to fill the SMs a few times over
int gridselect_ctas(const SelectArgs& a) {
  const int64_t per_cta = (int64_t)kGsWarps * 1024;
  int64_t g = (a.len + per_cta - 1) / per_cta;
  g = std::min<int64_t>(g, std::max<int64_t>(1, (int64_t)num_sms() * 8 / a.batch));
  return (int)std::max<int64_t>(1, g);
}

size_t gridselect_workspace(const SelectArgs& a, int G) {
  const size_t cand = (size_t)a.batch * G * kGsWarps * a.k * 8;
  return ((cand + 255) / 256) * 256 + ((size_t)a.batch * 4 + 255) / 256 * 256;
}

template <int KIND>
static cudaError_t launch_gs(const GsParams& p, cudaStream_t s) {
  gridselect_kernel<KIND><<<(unsigned)(p.batch * p.G), kGsBlock, 0, s>>>(p);
  return cudaGetLastError();
}

cudaError_t run_gridselect(const SelectArgs& a, void* ws, size_t ws_bytes, cudaStream_t s) {
  GsParams p;
  p.G = gridselect_ctas(a);
  if (ws_bytes < gridselect_workspace(a, p.G)) return cudaErrorInvalidValue;
  p.keys = a.keys;
  p.batch = a.batch;
  p.len = a.len;
  p.k = a.k;
  p.sel_min = a.sel_min;
  p.out_vals = a.out_vals;
  p.out_idx = a.out_idx;
  p.cand = (unsigned long long*)ws;
  const size_t cand = (size_t)a.batch * p.G * kGsWarps * a.k * 8;
  p.ticket = (unsigned*)((char*)ws + ((cand + 255) / 256) * 256);
  p.per_warp = (a.len + (int64_t)p.G * kGsWarps - 1) / ((int64_t)p.G * kGsWarps);
  cudaError_t e = cudaMemsetAsync(p.ticket, 0, (size_t)a.batch * 4, s);
  if (e != cudaSuccess) return e;
  if (a.events && a.n_events > 0) cudaEventRecord((cudaEvent_t)a.events[0], s);
  switch (a.kind) {
    case K_F32: e = launch_gs<K_F32>(p, s); break;
    case K_F16: e = launch_gs<K_F16>(p, s); break;
    case K_BF16: e = launch_gs<K_BF16>(p, s); break;
    case K_U32: e = launch_gs<K_U32>(p, s); break;
    default: return cudaErrorInvalidValue;
  }
  if (a.events && a.n_events > 1) cudaEventRecord((cudaEvent_t)a.events[1], s);
  return e;
}

}  // namespace airtopk
