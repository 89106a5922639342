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
//   * multiple thread blocks: a row is split over G CTAs x W warps.
// B200 additions:
//   * K up to 2048 ("the largest K that WarpSelect, BlockSelect, and GridSelect support is
//     2048"): the lists live in dynamic shared memory, W = 8 warps per CTA for K <= 1024, fewer above;
//   * 128-bit loads of the row (4 f32 / 8 f16 keys per lane per load);
//   * a threshold shared by every warp of the row: after each merge a warp publishes its K-th best
//     with a 64-bit atomicMin to a per-row word and adopts the row minimum — any warp's K-th best
//     bounds the row's K-th best, so elements at or above it can never be results and skip the queue;
//   * the W lists of a CTA are merged in the CTA before anything is written (G lists of K reach the
//     final merge, not G*W), and the last CTA (ticket, as P:154) splits the G lists over its W warps
//     and merges their W results.
// Per-thread queues (Fig. 11 ablation; engine AIRTOPK_ENGINE_GRIDSELECT_PTQ): each lane
// keeps a 2-entry queue in registers like BlockSelect; when any lane's queue is full, all lanes' queues
// are flushed through the same sort + merge.
// Elements are compared as composite keys (order-preserving code : 32 bits || row index : 32 bits),
// so ties at the K-th value go to the lowest indices (reading 1) and all keys are distinct.
// Scope: keys of <= 32 bits, len < 2^32, K <= kGsMaxK. Output rows come out sorted (ascending in
// the selection order).
#include <algorithm>

#include "device.cuh"
#include "engine.h"

namespace airtopk {

constexpr int kGsMaxWarps = 8;
constexpr int kGsMaxK = 2048;
constexpr int kGsPtq = 2;                     // per-thread queue length (ablation variant)
constexpr size_t kGsSmemCap = 200 * 1024;     // dynamic shared memory for the warp lists
constexpr unsigned long long kGsInf = ~0ull;  // sorts after every real composite key

struct GsParams {
  const void* keys;
  int64_t batch, len, k;
  int kcap;                  // K rounded up to 32 (list stride)
  int sel_min;
  void* out_vals;
  int64_t* out_idx;
  unsigned long long* cand;  // [batch][G][k] per-CTA sorted lists
  unsigned long long* rthr;  // [batch] shared row threshold (atomicMin)
  unsigned* ticket;          // [batch]
  int G;                     // CTAs per row
  int64_t per_warp;          // elements per warp slice (a multiple of the vector width)
  int vec_ok;                // rows are 16-byte aligned whole vectors
};

// Per-warp shared state: two sorted lists (double buffer for the merge) and the queue.
struct GsWarpView {
  unsigned long long* list[2];
  unsigned long long* q;
};

__device__ __forceinline__ GsWarpView gs_view(unsigned char* smem, int warp, int kcap) {
  unsigned long long* base = (unsigned long long*)smem + (size_t)warp * (2 * kcap + 32);
  return GsWarpView{{base, base + kcap}, base + 2 * kcap};
}

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
__device__ __noinline__ unsigned long long gs_flush(GsWarpView& w, int& cur, int K, int qn) {
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

// Merge two sorted lists A, B of K unique keys into out (the K smallest of the union), one warp:
// A[i] lands at i + #{B < A[i]}, B[j] at j + #{A < B[j]} (binary searches; positions >= K dropped).
__device__ __noinline__ void gs_merge2(const unsigned long long* A, const unsigned long long* B, unsigned long long* out,
                                      int K) {
  const int lane = threadIdx.x & 31;
  for (int i = lane; i < K; i += 32) {
    const unsigned long long a = A[i], b = B[i];
    int lo = 0, hi = K;  // #{B < a}
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (B[mid] < a) lo = mid + 1; else hi = mid;
    }
    if (i + lo < K) out[i + lo] = a;
    lo = 0;
    hi = K;  // #{A < b}
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (A[mid] < b) lo = mid + 1; else hi = mid;
    }
    if (i + lo < K) out[i + lo] = b;
  }
  __syncwarp();
}

// The CTA's W sorted lists (buffer 0 of every warp) -> one, by a tree of pairwise merges (log2 W
// levels, the merges of a level in parallel); returns with the result in warp 0's buffer 0.
__device__ __forceinline__ void gs_cta_merge(unsigned char* smem, int W, int kcap, int K) {
  const int warp = threadIdx.x >> 5;
  for (int st = 1; st < W; st <<= 1) {
    __syncthreads();
    if ((warp % (2 * st)) == 0 && warp + st < W) {
      GsWarpView a = gs_view(smem, warp, kcap), b = gs_view(smem, warp + st, kcap);
      gs_merge2(a.list[0], b.list[0], a.list[1], K);
      const int lane = threadIdx.x & 31;
      for (int i = lane; i < K; i += 32) a.list[0][i] = a.list[1][i];
      __syncwarp();
    }
  }
  __syncthreads();
}

// The warp's insertion state: threshold (own K-th best, lowered by the row threshold), queue fill,
// per-thread queue (ablation variant).
struct GsIns {
  unsigned long long thr;
  int qn;
  unsigned long long tq[kGsPtq];
  int tn;
};

// Publish / adopt the shared row threshold after a merge.
__device__ __forceinline__ void gs_share(GsIns& s, unsigned long long* rthr) {
  const int lane = threadIdx.x & 31;
  unsigned long long r = 0;
  if (lane == 0) r = atomicMin(rthr, s.thr);  // returns the previous row minimum
  r = __shfl_sync(kFull, r, 0);
  s.thr = r < s.thr ? r : s.thr;
}

// Two-step insertion of one element per lane.
template <int QMODE>
__device__ __forceinline__ void gs_insert(GsWarpView& w, int& cur, int K, unsigned long long x, GsIns& s,
                                          unsigned long long* rthr) {
  if constexpr (QMODE == 0) {
    bool ok = x < s.thr;
    const unsigned m = __ballot_sync(kFull, ok);
    if (!m) return;
    const int pos = s.qn + __popc(m & lanemask_lt());
    if (ok && pos < 32) w.q[pos] = x;  // step 1
    s.qn += __popc(m);
    if (s.qn >= 32) {
      __syncwarp();
      s.thr = gs_flush(w, cur, K, 32);
      if (rthr) gs_share(s, rthr);
      ok = ok && pos >= 32 && x < s.thr;  // step 2: the overflow, shifted down by 32
      const unsigned m2 = __ballot_sync(kFull, ok);
      if (ok) w.q[__popc(m2 & lanemask_lt())] = x;
      s.qn = __popc(m2);
    }
    __syncwarp();
  } else {
    // per-thread queues (BlockSelect style): each lane appends to its own register queue
    const bool ok = x < s.thr;
    if (ok) {
#pragma unroll
      for (int t = 0; t < kGsPtq; ++t)
        if (t == s.tn) s.tq[t] = x;
      ++s.tn;
    }
    if (__any_sync(kFull, s.tn == kGsPtq)) {
      // one lane's queue is full: every lane's queue goes through the sort + merge (kGsPtq rounds)
      const int lane = threadIdx.x & 31;
#pragma unroll
      for (int t = 0; t < kGsPtq; ++t) {
        w.q[lane] = (t < s.tn) ? s.tq[t] : kGsInf;
        __syncwarp();
        s.thr = gs_flush(w, cur, K, 32);
      }
      if (rthr) gs_share(s, rthr);
      s.tn = 0;
    }
  }
}

template <int QMODE>
__device__ __forceinline__ void gs_drain(GsWarpView& w, int& cur, int K, GsIns& s) {
  const int lane = threadIdx.x & 31;
  if constexpr (QMODE == 0) {
    if (s.qn > 0) s.thr = gs_flush(w, cur, K, s.qn);
    s.qn = 0;
  } else {
#pragma unroll
    for (int t = 0; t < kGsPtq; ++t) {
      if (__any_sync(kFull, t < s.tn)) {
        w.q[lane] = (t < s.tn) ? s.tq[t] : kGsInf;
        __syncwarp();
        s.thr = gs_flush(w, cur, K, 32);
      }
    }
    s.tn = 0;
  }
}

__device__ __forceinline__ void gs_reset(GsWarpView& w, int cur, int kcap, GsIns& s) {
  const int lane = threadIdx.x & 31;
  for (int i = lane; i < kcap; i += 32) w.list[cur][i] = kGsInf;
  __syncwarp();
  s.thr = kGsInf;
  s.qn = 0;
  s.tn = 0;
}

// One warp over n composite keys get(i) (i < n), kGsUnroll keys per lane loaded up front.
constexpr int kGsUnroll = 16;
template <int QMODE, typename Get>
__device__ __forceinline__ void gs_warp_run(GsWarpView& w, int& cur, int K, int64_t n, GsIns& s,
                                            unsigned long long* rthr, Get get) {
  const int lane = threadIdx.x & 31;
  for (int64_t b = 0; b < n; b += 32 * kGsUnroll) {
    if (rthr) {  // adopt the row threshold once per round
      const unsigned long long r = __ldcg(rthr);
      s.thr = r < s.thr ? r : s.thr;
    }
    unsigned long long x[kGsUnroll];
#pragma unroll
    for (int t = 0; t < kGsUnroll; ++t) {
      const int64_t i = b + 32 * t + lane;
      x[t] = (i < n) ? get(i) : kGsInf;
    }
#pragma unroll
    for (int t = 0; t < kGsUnroll; ++t) gs_insert<QMODE>(w, cur, K, x[t], s, rthr);
  }
}

template <int KIND, int QMODE>
__global__ void __launch_bounds__(kGsMaxWarps * 32) gridselect_kernel(const GsParams p) {
  using U = typename KT<KIND>::U;
  constexpr int VEC = 16 / sizeof(U);
  extern __shared__ __align__(16) unsigned char gs_smem[];
  __shared__ int sh_last;
  const int W = (int)(blockDim.x >> 5);
  const int64_t row = blockIdx.x / p.G;
  const int cta = blockIdx.x % p.G;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int K = (int)p.k;
  const bool sel_min = p.sel_min != 0;
  const U xmask = sel_min ? (U)0 : (U)~(U)0;
  const U* rowp = (const U*)p.keys + row * p.len;
  unsigned long long* rthr = p.rthr + row;
  GsWarpView w = gs_view(gs_smem, warp, p.kcap);
  int cur = 0;
  GsIns s;
  gs_reset(w, cur, p.kcap, s);
  // ---- this warp's slice of the row ----
  const int64_t gw = (int64_t)cta * W + warp;
  const int64_t e0 = std::min<int64_t>(p.len, gw * p.per_warp), e1 = std::min<int64_t>(p.len, e0 + p.per_warp);
  if (p.vec_ok) {
    // 128-bit loads: lane handles vectors lane, lane + 32, ...; the VEC keys of a vector are
    // inserted one after another (every lane inserts its e-th key in the same step)
    const uint4* vp = (const uint4*)(rowp + e0);
    const int64_t nv = (e1 - e0) / VEC;
    constexpr int VU = kGsUnroll / VEC > 0 ? kGsUnroll / VEC : 1;
    for (int64_t b = 0; b < nv; b += 32 * VU) {
      const unsigned long long r = __ldcg(rthr);
      s.thr = r < s.thr ? r : s.thr;
      uint4 v[VU];
#pragma unroll
      for (int t = 0; t < VU; ++t) {
        const int64_t i = b + 32 * t + lane;
        v[t] = (i < nv) ? ldg_stream(vp + i) : make_uint4(0, 0, 0, 0);
      }
#pragma unroll
      for (int t = 0; t < VU; ++t) {
        const int64_t i = b + 32 * t + lane;
#pragma unroll
        for (int e = 0; e < VEC; ++e) {
          const unsigned long long pos = (unsigned long long)(e0 + i * VEC + e);
          const unsigned long long x =
              (i < nv) ? ((unsigned long long)to_code_x<KIND>(vec_elem<U>(v[t], e), xmask) << 32) | pos : kGsInf;
          gs_insert<QMODE>(w, cur, K, x, s, rthr);
        }
      }
    }
  } else {
    gs_warp_run<QMODE>(w, cur, K, e1 - e0, s, rthr, [&](int64_t i) -> unsigned long long {
      const int64_t pos = e0 + i;
      return ((unsigned long long)to_code_x<KIND>(__ldg(rowp + pos), xmask) << 32) | (unsigned long long)pos;
    });
  }
  gs_drain<QMODE>(w, cur, K, s);
  // ---- the CTA's W lists -> one (warp 0 inserts the others' lists through its queue) ----
  if (cur != 0) {  // every warp's final list in buffer 0
    for (int i = lane; i < K; i += 32) w.list[0][i] = w.list[1][i];
    __syncwarp();
    cur = 0;
  }
  gs_cta_merge(gs_smem, W, p.kcap, K);
  if (warp == 0) {
    unsigned long long* cand = p.cand + ((size_t)row * p.G + cta) * K;
    for (int i = lane; i < K; i += 32) cand[i] = w.list[cur][i];
  }
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) sh_last = (ticket_arrive(&p.ticket[row]) == (unsigned)(p.G - 1));
  __syncthreads();
  if (!sh_last) return;
  // ---- last CTA of the row: the G lists split over its W warps, then warp 0 merges the W results ----
  const unsigned long long* cand = p.cand + (size_t)row * p.G * K;
  const int64_t nc = (int64_t)p.G * K;
  const int64_t per = (nc + W - 1) / W;
  const int64_t c0 = std::min<int64_t>(nc, warp * per), c1 = std::min<int64_t>(nc, c0 + per);
  cur = 0;
  gs_reset(w, cur, p.kcap, s);
  {  // keys <= the row threshold may be results (it is itself some list's K-th best): insert x <= it
    const unsigned long long r = __ldcg(rthr);
    s.thr = (r == kGsInf) ? r : r + 1;
  }
  gs_warp_run<0>(w, cur, K, c1 - c0, s, nullptr, [&](int64_t i) { return __ldcg(cand + c0 + i); });
  gs_drain<0>(w, cur, K, s);
  if (cur != 0) {
    for (int i = lane; i < K; i += 32) w.list[0][i] = w.list[1][i];
    __syncwarp();
    cur = 0;
  }
  gs_cta_merge(gs_smem, W, p.kcap, K);
  if (warp == 0) {
    U* ov = (U*)p.out_vals + row * p.k;
    int64_t* oi = p.out_idx + row * p.k;
    for (int i = lane; i < K; i += 32) {
      const unsigned long long x = w.list[cur][i];
      ov[i] = from_code<KIND>((U)(x >> 32), sel_min);
      oi[i] = (int64_t)(x & 0xffffffffull);
    }
  }
  if (threadIdx.x == 0) {
    p.ticket[row] = 0;
    *rthr = kGsInf;  // ready for the next call on this workspace
  }
}

bool gridselect_supported(const SelectArgs& a) {
  return a.in_idx == nullptr && key_bits(a.kind) <= 32 && a.len < (int64_t(1) << 32) && a.k <= kGsMaxK;
}

static int gs_kcap(const SelectArgs& a) { return (int)((a.k + 31) / 32 * 32); }

// warps per CTA: 8, fewer when the K-entry lists would exceed the shared-memory budget
static int gs_warps(const SelectArgs& a) {
  const size_t per = (size_t)(2 * gs_kcap(a) + 32) * 8;
  return (int)std::max<size_t>(1, std::min<size_t>(kGsMaxWarps, kGsSmemCap / per));
}

// CTAs per row: >= 1K elements per warp, at most enough CTAs to fill the SMs a few times over
int gridselect_ctas(const SelectArgs& a) {
  const int64_t per_cta = (int64_t)gs_warps(a) * 1024;
  int64_t g = (a.len + per_cta - 1) / per_cta;
  g = std::min<int64_t>(g, std::max<int64_t>(1, (int64_t)num_sms() * 4 / a.batch));
  return (int)std::max<int64_t>(1, g);
}

size_t gridselect_workspace(const SelectArgs& a, int G) {
  const size_t cand = (size_t)a.batch * G * a.k * 8;
  return ((cand + 255) / 256) * 256 + ((size_t)a.batch * 8 + 255) / 256 * 256 +
         ((size_t)a.batch * 4 + 255) / 256 * 256;
}

template <int KIND, int QMODE>
static cudaError_t launch_gs(const GsParams& p, int W, cudaStream_t s) {
  const size_t smem = (size_t)W * (2 * p.kcap + 32) * 8;
  cudaError_t e = func_attr(gridselect_kernel<KIND, QMODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kGsSmemCap);
  if (e != cudaSuccess) return e;
  gridselect_kernel<KIND, QMODE><<<(unsigned)(p.batch * p.G), (unsigned)(W * 32), smem, s>>>(p);
  return cudaGetLastError();
}

cudaError_t run_gridselect(const SelectArgs& a, void* ws, size_t ws_bytes, cudaStream_t s) {
  GsParams p;
  p.G = gridselect_ctas(a);
  if (ws_bytes < gridselect_workspace(a, p.G)) return cudaErrorInvalidValue;
  const int W = gs_warps(a);
  p.keys = a.keys;
  p.batch = a.batch;
  p.len = a.len;
  p.k = a.k;
  p.kcap = gs_kcap(a);
  p.sel_min = a.sel_min;
  p.out_vals = a.out_vals;
  p.out_idx = a.out_idx;
  p.cand = (unsigned long long*)ws;
  const size_t cand = ((size_t)a.batch * p.G * a.k * 8 + 255) / 256 * 256;
  p.rthr = (unsigned long long*)((char*)ws + cand);
  p.ticket = (unsigned*)((char*)ws + cand + ((size_t)a.batch * 8 + 255) / 256 * 256);
  const int vec = 16 / key_bytes(a.kind);
  p.vec_ok = ((uintptr_t)a.keys % 16 == 0) && (a.len % vec == 0) ? 1 : 0;
  const int64_t slices = (int64_t)p.G * W;
  p.per_warp = ((a.len + slices - 1) / slices + vec - 1) / vec * vec;
  // row thresholds = +inf (all ones), tickets = 0
  cudaError_t e = cudaMemsetAsync(p.rthr, 0xff, (size_t)a.batch * 8, s);
  if (e != cudaSuccess) return e;
  e = cudaMemsetAsync(p.ticket, 0, (size_t)a.batch * 4, s);
  if (e != cudaSuccess) return e;
  if (a.events && a.n_events > 0) cudaEventRecord((cudaEvent_t)a.events[0], s);
  const bool ptq = a.engine == 7;
  switch (a.kind) {
    case K_F32: e = ptq ? launch_gs<K_F32, 1>(p, W, s) : launch_gs<K_F32, 0>(p, W, s); break;
    case K_F16: e = ptq ? launch_gs<K_F16, 1>(p, W, s) : launch_gs<K_F16, 0>(p, W, s); break;
    case K_BF16: e = ptq ? launch_gs<K_BF16, 1>(p, W, s) : launch_gs<K_BF16, 0>(p, W, s); break;
    case K_U32: e = ptq ? launch_gs<K_U32, 1>(p, W, s) : launch_gs<K_U32, 0>(p, W, s); break;
    default: return cudaErrorInvalidValue;
  }
  if (a.events && a.n_events > 1) cudaEventRecord((cudaEvent_t)a.events[1], s);
  return e;
}

}  // namespace airtopk
