// p2p.cu — the split-row exchange over peer memory ("top 0.1 % of the
// gradients ... across workers").
//
// The NCCL all-gather of the split-row path is replaced by ONE push kernel per rank: every rank stores
// its k (value, global index) entries straight into slot `rank` of EVERY rank's gather buffers
// (peer pointers opened with CUDA IPC; over NVLink 5 / NVSwitch the stores are P2P writes), then —
// after a system-scope fence and a last-CTA ticket, so every store of the launch is visible first —
// sets its flag word in every peer's flag array to the call's epoch. A one-CTA wait kernel on each
// rank spins (acquire loads) until all world flags carry the epoch; the merge select
// (airtopk_select_with_idx) is stream-ordered after it. Host-side the library only enqueues.
#include <algorithm>
#include <cstdint>
#include <cstring>

#include <cuda.h>

#include "../../include/airtopk.h"
#include "device.cuh"
#include "engine.h"

namespace airtopk {

constexpr int kP2PMaxWorld = 64;

// cuMemGetAddressRange through the runtime's driver entry point (no link-time libcuda dependency:
// the library must load on machines without a driver, e.g. for the C-ABI tests)
static CUresult addr_range(CUdeviceptr* base, size_t* size, CUdeviceptr p) {
  using Fn = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
  static Fn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !f)
      return CUDA_ERROR_NOT_FOUND;
    fn = (Fn)f;
  }
  return fn(base, size, p);
}

struct PushParams {
  const unsigned char* vals;  // this rank's k values (esz bytes each)
  const int64_t* idx;         // this rank's k global indices
  int64_t k;
  int esz;
  int world, rank;
  unsigned epoch;
  unsigned* ticket;                        // local: CTAs done (reset by the last one)
  unsigned char* peer_vals[kP2PMaxWorld];  // [world * k] gather buffers of every rank (IPC-mapped)
  int64_t* peer_idx[kP2PMaxWorld];
  unsigned* peer_flags[kP2PMaxWorld];      // [world] flag words of every rank
};

__global__ void push_kernel(const PushParams p) {
  // copy: 16-byte chunks of the value and index slots, every peer
  const int64_t vbytes = p.k * p.esz, ibytes = p.k * 8;
  const int64_t v16 = vbytes / 16, i16 = ibytes / 16;
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, nth = (int64_t)gridDim.x * blockDim.x;
  for (int r = 0; r < p.world; ++r) {
    unsigned char* dv = p.peer_vals[r] + (size_t)p.rank * vbytes;
    unsigned char* di = (unsigned char*)(p.peer_idx[r] + (size_t)p.rank * p.k);
    const bool va = (((uintptr_t)dv | (uintptr_t)p.vals) & 15u) == 0;
    if (va) {
      for (int64_t i = tid; i < v16; i += nth) ((uint4*)dv)[i] = ((const uint4*)p.vals)[i];
      for (int64_t i = v16 * 16 + tid; i < vbytes; i += nth) dv[i] = p.vals[i];
    } else {
      for (int64_t i = tid; i < vbytes; i += nth) dv[i] = p.vals[i];
    }
    const bool ia = (((uintptr_t)di | (uintptr_t)p.idx) & 15u) == 0;
    if (ia) {
      for (int64_t i = tid; i < i16; i += nth) ((uint4*)di)[i] = ((const uint4*)p.idx)[i];
      for (int64_t i = i16 * 16 + tid; i < ibytes; i += nth) di[i] = ((const unsigned char*)p.idx)[i];
    } else {
      for (int64_t i = tid; i < ibytes; i += nth) di[i] = ((const unsigned char*)p.idx)[i];
    }
  }
  // publish: every store of this CTA is visible system-wide before the ticket; the last CTA then
  // raises this rank's flag in every peer (release)
  __threadfence_system();
  __syncthreads();
  __shared__ bool last;
  if (threadIdx.x == 0) last = atomicAdd(p.ticket, 1u) == gridDim.x - 1;
  __syncthreads();
  if (!last) return;
  __threadfence_system();
  if (threadIdx.x < (unsigned)p.world) {
    unsigned* f = p.peer_flags[threadIdx.x] + p.rank;
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(f), "r"(p.epoch) : "memory");
  }
  if (threadIdx.x == 0) *p.ticket = 0;
}

__global__ void wait_kernel(const unsigned* flags, int world, unsigned epoch) {
  if (threadIdx.x < (unsigned)world) {
    unsigned v;
    do {
      asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(flags + threadIdx.x) : "memory");
      if (v != epoch) __nanosleep(256);
    } while (v != epoch);
  }
  __syncthreads();
}

}  // namespace airtopk

using namespace airtopk;

extern "C" {

airtopk_status airtopk_ipc_handle(const void* dev_ptr, void* handle_out, uint64_t* offset_out) {
  if (!dev_ptr || !handle_out || !offset_out) return AIRTOPK_EINVAL;
  // the handle names the whole allocation: report where dev_ptr lies inside it (caching allocators
  // hand out pieces of larger cudaMalloc blocks)
  CUdeviceptr base = 0;
  size_t size = 0;
  if (addr_range(&base, &size, (CUdeviceptr)dev_ptr) != CUDA_SUCCESS) return AIRTOPK_ECUDA;
  cudaIpcMemHandle_t h;
  const cudaError_t e = cudaIpcGetMemHandle(&h, (void*)base);
  if (e != cudaSuccess) return AIRTOPK_ECUDA;
  std::memcpy(handle_out, &h, sizeof(h));
  *offset_out = (uint64_t)((CUdeviceptr)dev_ptr - base);
  return AIRTOPK_OK;
}

airtopk_status airtopk_ipc_open(const void* handle, uint64_t offset, void** dev_ptr_out) {
  if (!handle || !dev_ptr_out) return AIRTOPK_EINVAL;
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle, sizeof(h));
  void* base = nullptr;
  const cudaError_t e = cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) return AIRTOPK_ECUDA;
  *dev_ptr_out = (char*)base + offset;
  return AIRTOPK_OK;
}

airtopk_status airtopk_ipc_close(void* dev_ptr) {
  if (!dev_ptr) return AIRTOPK_EINVAL;
  CUdeviceptr base = 0;
  size_t size = 0;
  if (addr_range(&base, &size, (CUdeviceptr)dev_ptr) != CUDA_SUCCESS) return AIRTOPK_ECUDA;
  return cudaIpcCloseMemHandle((void*)base) == cudaSuccess ? AIRTOPK_OK : AIRTOPK_ECUDA;
}

airtopk_status airtopk_shard_push(const void* vals, const int64_t* idx, int64_t k, airtopk_dtype dtype, int world,
                                  int rank, void* const* peer_vals, int64_t* const* peer_idx,
                                  uint32_t* const* peer_flags, uint32_t epoch, uint32_t* ticket,
                                  airtopk_stream_t stream) {
  if (!vals || !idx || !peer_vals || !peer_idx || !peer_flags || !ticket) return AIRTOPK_EINVAL;
  if (k < 1 || world < 1 || world > kP2PMaxWorld || rank < 0 || rank >= world || epoch == 0) return AIRTOPK_EINVAL;
  if ((int)dtype < AIRTOPK_F32 || (int)dtype > AIRTOPK_U32) return AIRTOPK_EDTYPE;
  PushParams p;
  p.vals = (const unsigned char*)vals;
  p.idx = idx;
  p.k = k;
  p.esz = key_bytes((int)dtype);
  p.world = world;
  p.rank = rank;
  p.epoch = epoch;
  p.ticket = ticket;
  for (int r = 0; r < world; ++r) {
    if (!peer_vals[r] || !peer_idx[r] || !peer_flags[r]) return AIRTOPK_EINVAL;
    p.peer_vals[r] = (unsigned char*)peer_vals[r];
    p.peer_idx[r] = peer_idx[r];
    p.peer_flags[r] = peer_flags[r];
  }
  const int64_t work = (k * 8 + 15) / 16;
  const unsigned blocks = (unsigned)std::max<int64_t>(1, std::min<int64_t>((work + 255) / 256, 148));
  push_kernel<<<blocks, 256, 0, (cudaStream_t)stream>>>(p);
  return cudaGetLastError() == cudaSuccess ? AIRTOPK_OK : AIRTOPK_ECUDA;
}

airtopk_status airtopk_wait_flags(const uint32_t* flags, int world, uint32_t epoch, airtopk_stream_t stream) {
  if (!flags || world < 1 || world > kP2PMaxWorld || epoch == 0) return AIRTOPK_EINVAL;
  wait_kernel<<<1, 64, 0, (cudaStream_t)stream>>>(flags, world, epoch);
  return cudaGetLastError() == cudaSuccess ? AIRTOPK_OK : AIRTOPK_ECUDA;
}

}  // extern "C"
