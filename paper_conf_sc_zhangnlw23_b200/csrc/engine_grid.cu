// engine_grid.cu — host side of the grid engine: parameter set-up, per-kind dispatch, and the
// K == N trivial path. The kernels live in engine_grid.cuh and are instantiated per key type in
// engine_grid_<kind>.cu (parallel compilation).
#include "engine_batch.cuh"
#include "engine_resident.cuh"
#include "engine_cluster.cuh"
#include "engine_grid.cuh"

#include <cstdlib>

namespace airtopk {

extern template cudaError_t launch_grid_kind<K_F32>(const SelectArgs&, const Plan&, const GridParams&, void*, cudaStream_t);
extern template cudaError_t launch_grid_kind<K_F16>(const SelectArgs&, const Plan&, const GridParams&, void*, cudaStream_t);
extern template cudaError_t launch_grid_kind<K_BF16>(const SelectArgs&, const Plan&, const GridParams&, void*, cudaStream_t);
extern template cudaError_t launch_grid_kind<K_F64>(const SelectArgs&, const Plan&, const GridParams&, void*, cudaStream_t);
extern template cudaError_t launch_grid_kind<K_U32>(const SelectArgs&, const Plan&, const GridParams&, void*, cudaStream_t);
int grid_occupancy_f32(int idx64);
extern template cudaError_t launch_batch_kind<K_F32>(const SelectArgs&, const Plan&, void*, cudaStream_t);
extern template cudaError_t launch_resident_kind<K_F32>(const SelectArgs&, const Plan&, void*, cudaStream_t);
extern template cudaError_t launch_batch_kind<K_F16>(const SelectArgs&, const Plan&, void*, cudaStream_t);
extern template cudaError_t launch_resident_kind<K_F16>(const SelectArgs&, const Plan&, void*, cudaStream_t);
extern template cudaError_t launch_batch_kind<K_BF16>(const SelectArgs&, const Plan&, void*, cudaStream_t);
extern template cudaError_t launch_resident_kind<K_BF16>(const SelectArgs&, const Plan&, void*, cudaStream_t);
extern template cudaError_t launch_batch_kind<K_F64>(const SelectArgs&, const Plan&, void*, cudaStream_t);
extern template cudaError_t launch_resident_kind<K_F64>(const SelectArgs&, const Plan&, void*, cudaStream_t);
extern template cudaError_t launch_batch_kind<K_U32>(const SelectArgs&, const Plan&, void*, cudaStream_t);
extern template cudaError_t launch_resident_kind<K_U32>(const SelectArgs&, const Plan&, void*, cudaStream_t);
extern template cudaError_t launch_cluster_kind<K_F32>(const SelectArgs&, const Plan&, void*, cudaStream_t, int);
extern template cudaError_t launch_cluster_kind<K_F16>(const SelectArgs&, const Plan&, void*, cudaStream_t, int);
extern template cudaError_t launch_cluster_kind<K_BF16>(const SelectArgs&, const Plan&, void*, cudaStream_t, int);
extern template cudaError_t launch_cluster_kind<K_F64>(const SelectArgs&, const Plan&, void*, cudaStream_t, int);
extern template cudaError_t launch_cluster_kind<K_U32>(const SelectArgs&, const Plan&, void*, cudaStream_t, int);

// K == N ("a trivial case"): every element is a result, in index order.
template <typename U>
__global__ void trivial_kernel(const U* keys, int64_t total, U* ov, int64_t* oi, int64_t len, int64_t ioff) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    ov[i] = keys[i];
    oi[i] = i % len + ioff;
  }
}

int grid_blocks_per_sm(const SelectArgs& a, int idx64) {
  (void)a;
  int n = grid_occupancy_f32(idx64);
  return n < 1 ? kMinBlocks : std::min(n, kMinBlocks);
}

int grid_vec_chunk(int kind) { return kBlock * kUnroll * (16 / key_bytes(kind)); }

cudaError_t run_grid(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s) {
  char* base = (char*)ws;
  cudaError_t e = cudaMemsetAsync(base + pl.off_state, 0, pl.off_bcode - pl.off_state, s);
  if (e != cudaSuccess) return e;
  GridParams gp;
  gp.keys = a.keys;
  gp.in_idx = a.in_idx;
  gp.batch = a.batch;
  gp.len = a.len;
  gp.k = a.k;
  gp.sel_min = a.sel_min;
  gp.P = pl.P;
  gp.IB = pl.IB;
  gp.out_vals = a.out_vals;
  gp.out_idx = a.out_idx;
  gp.st = (RowState*)(base + pl.off_state);
  gp.ghist = base + pl.off_hist;
  gp.bcode = base + pl.off_bcode;
  gp.bidx = base + pl.off_bidx;
  gp.cap_rule = pl.cap_rule;
  gp.cap_alloc = pl.cap_alloc;
  gp.cpr = pl.cpr;
  gp.cpr_buf = pl.cpr_buf;
  gp.trace = a.trace;
  gp.samp = base + pl.off_samp;
  gp.nsms = num_sms();
  gp.early_stop = a.early_stop;
  gp.idx_off = a.idx_off;
  gp.thist = base + pl.off_thist;
  gp.tstamp = nullptr;
  if (a.trace && getenv("AIRTOPK_TAIL_STAMPS")) gp.tstamp = a.trace;  // debug (tools/tail_stamps.py)
  gp.tcnt = (unsigned long long*)(base + pl.off_tcnt);
  {
    static const char* env2 = getenv("AIRTOPK_SMALL_FINISH");  // A/B knob (0 = off)
    gp.small_finish = env2 ? std::min(atoi(env2), kSmallFinish) : kSmallFinish;
  }
  switch (a.kind) {
    case K_F32: return launch_grid_kind<K_F32>(a, pl, gp, ws, s);
    case K_F16: return launch_grid_kind<K_F16>(a, pl, gp, ws, s);
    case K_BF16: return launch_grid_kind<K_BF16>(a, pl, gp, ws, s);
    case K_F64: return launch_grid_kind<K_F64>(a, pl, gp, ws, s);
    case K_U32: return launch_grid_kind<K_U32>(a, pl, gp, ws, s);
  }
  return cudaErrorInvalidValue;
}

cudaError_t run_batch(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s) {
  switch (a.kind) {
    case K_F32: return launch_batch_kind<K_F32>(a, pl, ws, s);
    case K_F16: return launch_batch_kind<K_F16>(a, pl, ws, s);
    case K_BF16: return launch_batch_kind<K_BF16>(a, pl, ws, s);
    case K_F64: return launch_batch_kind<K_F64>(a, pl, ws, s);
    case K_U32: return launch_batch_kind<K_U32>(a, pl, ws, s);
  }
  return cudaErrorInvalidValue;
}

cudaError_t run_resident(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s) {
  // (no memset: the kernel resets each row's counters itself)
  switch (a.kind) {
    case K_F32: return launch_resident_kind<K_F32>(a, pl, ws, s);
    case K_F16: return launch_resident_kind<K_F16>(a, pl, ws, s);
    case K_BF16: return launch_resident_kind<K_BF16>(a, pl, ws, s);
    case K_F64: return launch_resident_kind<K_F64>(a, pl, ws, s);
    case K_U32: return launch_resident_kind<K_U32>(a, pl, ws, s);
  }
  return cudaErrorInvalidValue;
}

cudaError_t run_cluster(const SelectArgs& a, const Plan& pl, void* ws, cudaStream_t s) {
  switch (a.kind) {
    case K_F32: return launch_cluster_kind<K_F32>(a, pl, ws, s, 0);
    case K_F16: return launch_cluster_kind<K_F16>(a, pl, ws, s, 0);
    case K_BF16: return launch_cluster_kind<K_BF16>(a, pl, ws, s, 0);
    case K_F64: return launch_cluster_kind<K_F64>(a, pl, ws, s, 0);
    case K_U32: return launch_cluster_kind<K_U32>(a, pl, ws, s, 0);
  }
  return cudaErrorInvalidValue;
}

template <int KIND>
__global__ void pad_kernel(typename KT<KIND>::U* ov, int64_t* oi, int64_t n, int64_t pad_base, int sel_min) {
  using U = typename KT<KIND>::U;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    ov[i] = from_code<KIND>((U)~(U)0, sel_min != 0);  // the largest code: sorts after every key
    oi[i] = pad_base + i;
  }
}

cudaError_t run_pad(int kind, int sel_min, void* vals, int64_t* idx, int64_t n, int64_t pad_base, cudaStream_t s) {
  const unsigned blocks = (unsigned)std::min<int64_t>((n + 255) / 256, 1024);
  switch (kind) {
    case K_F32: pad_kernel<K_F32><<<blocks, 256, 0, s>>>((uint32_t*)vals, idx, n, pad_base, sel_min); break;
    case K_F16: pad_kernel<K_F16><<<blocks, 256, 0, s>>>((uint16_t*)vals, idx, n, pad_base, sel_min); break;
    case K_BF16: pad_kernel<K_BF16><<<blocks, 256, 0, s>>>((uint16_t*)vals, idx, n, pad_base, sel_min); break;
    case K_F64: pad_kernel<K_F64><<<blocks, 256, 0, s>>>((uint64_t*)vals, idx, n, pad_base, sel_min); break;
    case K_U32: pad_kernel<K_U32><<<blocks, 256, 0, s>>>((uint32_t*)vals, idx, n, pad_base, sel_min); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

// Sorted output option: one CTA per row sorts its K (code, index) pairs ascending — bitonic network
// over the next power of two in shared memory (padding sorts last), values re-derived from the codes.
template <int KIND>
__global__ void __launch_bounds__(1024) sort_rows_kernel(typename KT<KIND>::U* ov, int64_t* oi, int64_t k,
                                                         int sel_min) {
  using U = typename KT<KIND>::U;
  extern __shared__ __align__(16) unsigned long long srt[];
  unsigned long long* sc = srt;               // codes (as 64-bit)
  unsigned long long* si = srt + kSortMaxK;   // indices
  const int64_t row = blockIdx.x;
  int n = 1;
  while (n < k) n <<= 1;
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    const bool in = i < k;
    sc[i] = in ? (unsigned long long)to_code<KIND>(ov[row * k + i], sel_min != 0) : ~0ull;
    si[i] = in ? (unsigned long long)oi[row * k + i] : ~0ull;
  }
  __syncthreads();
  for (int size = 2; size <= n; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      for (int i = threadIdx.x; i < n / 2; i += blockDim.x) {
        const int a = 2 * i - (i & (stride - 1)), b = a + stride;  // pair (a, b), a's bit `stride` clear
        const bool up = (a & size) == 0;
        const unsigned long long ca = sc[a], cb = sc[b], ia = si[a], ib = si[b];
        const bool gt = ca > cb || (ca == cb && ia > ib);
        if (gt == up) {
          sc[a] = cb; sc[b] = ca;
          si[a] = ib; si[b] = ia;
        }
      }
      __syncthreads();
    }
  }
  for (int i = threadIdx.x; i < k; i += blockDim.x) {
    ov[row * k + i] = from_code<KIND>((U)sc[i], sel_min != 0);
    oi[row * k + i] = (int64_t)si[i];
  }
}

cudaError_t run_sort_rows(const SelectArgs& a, cudaStream_t s) {
  const size_t smem = (size_t)2 * kSortMaxK * 8;
  const unsigned g = (unsigned)a.batch;
  cudaError_t e = cudaSuccess;
  switch (a.kind) {
    case K_F32:
      if ((e = func_attr(sort_rows_kernel<K_F32>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) == cudaSuccess)
        sort_rows_kernel<K_F32><<<g, 1024, smem, s>>>((uint32_t*)a.out_vals, a.out_idx, a.k, a.sel_min);
      break;
    case K_F16:
      if ((e = func_attr(sort_rows_kernel<K_F16>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) == cudaSuccess)
        sort_rows_kernel<K_F16><<<g, 1024, smem, s>>>((uint16_t*)a.out_vals, a.out_idx, a.k, a.sel_min);
      break;
    case K_BF16:
      if ((e = func_attr(sort_rows_kernel<K_BF16>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) == cudaSuccess)
        sort_rows_kernel<K_BF16><<<g, 1024, smem, s>>>((uint16_t*)a.out_vals, a.out_idx, a.k, a.sel_min);
      break;
    case K_F64:
      if ((e = func_attr(sort_rows_kernel<K_F64>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) == cudaSuccess)
        sort_rows_kernel<K_F64><<<g, 1024, smem, s>>>((uint64_t*)a.out_vals, a.out_idx, a.k, a.sel_min);
      break;
    case K_U32:
      if ((e = func_attr(sort_rows_kernel<K_U32>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) == cudaSuccess)
        sort_rows_kernel<K_U32><<<g, 1024, smem, s>>>((uint32_t*)a.out_vals, a.out_idx, a.k, a.sel_min);
      break;
  }
  if (e != cudaSuccess) return e;
  return cudaGetLastError();
}

__global__ void status_kernel(const RowState* st, int64_t batch, unsigned* status) {
  unsigned e = 0;
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < batch; r += (int64_t)gridDim.x * blockDim.x)
    e |= st[r].error;
  e = __reduce_or_sync(kFull, e);
  if ((threadIdx.x & 31) == 0 && e) atomicOr(status, e);
}

cudaError_t collect_status(const SelectArgs& a, const Plan& p, void* ws, cudaStream_t s) {
  const unsigned blocks = (unsigned)std::min<int64_t>((a.batch + 255) / 256, 148);
  status_kernel<<<blocks, 256, 0, s>>>((const RowState*)((char*)ws + p.off_state), a.batch, a.status);
  return cudaGetLastError();
}

cudaError_t run_trivial(const SelectArgs& a, cudaStream_t s) {
  const int64_t total = a.batch * a.len;
  const int threads = 256;
  const long long blocks = std::min<long long>((total + threads - 1) / threads, 148LL * 16);
  switch (key_bytes(a.kind)) {
    case 2: trivial_kernel<uint16_t><<<(unsigned)blocks, threads, 0, s>>>((const uint16_t*)a.keys, total, (uint16_t*)a.out_vals, a.out_idx, a.len, a.idx_off); break;
    case 4: trivial_kernel<uint32_t><<<(unsigned)blocks, threads, 0, s>>>((const uint32_t*)a.keys, total, (uint32_t*)a.out_vals, a.out_idx, a.len, a.idx_off); break;
    default: trivial_kernel<uint64_t><<<(unsigned)blocks, threads, 0, s>>>((const uint64_t*)a.keys, total, (uint64_t*)a.out_vals, a.out_idx, a.len, a.idx_off); break;
  }
  return cudaGetLastError();
}

}  // namespace airtopk
