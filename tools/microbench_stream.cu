// microbench_stream.cu — how to stream 4 GiB of f32 keys through the SMs at the HBM limit on B200,
// with the window pass's per-element work (one conservative fp compare per element, a rare slow path).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/mbs tools/microbench_stream.cu
// Variants: register loads (16 B or 32 B per load, L2 prefetch hints, CTAs/SM, unroll), per-warp
// bulk-copy rings (stages x tile size), per-CTA bulk-copy ring (one producer, all warps consume).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

__global__ void fill(float* x, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint32_t u = (uint32_t)(mix64(12345 + (i + 1) * 0x9E3779B97F4A7C15ULL) >> 32);
    x[i] = (float)u * 2.3283064365386963e-10f + 1.1641532182693481e-10f;
  }
}

template <int HINT>
__device__ __forceinline__ uint4 ld16(const uint4* p) {
  uint4 r;
  if (HINT == 0)
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  else if (HINT == 1)
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  else
    asm volatile("ld.global.nc.L1::no_allocate.L2::128B.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

struct u8x { uint32_t v[8]; };
__device__ __forceinline__ u8x ld32(const void* p) {
  u8x r;
  asm volatile("ld.global.nc.L1::no_allocate.v8.u32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]), "=r"(r.v[6]), "=r"(r.v[7])
               : "l"(p));
  return r;
}

__device__ __forceinline__ bool any_le(const uint32_t* w, int n, float h) {
  bool a = false;
#pragma unroll
  for (int i = 0; i < 16; ++i)
    if (i < n) a |= !(__uint_as_float(w[i]) > h);
  return a;
}

// register loads, grid-stride tiles of BS*U vectors
template <int BS, int U, int HINT>
__global__ void __launch_bounds__(BS) reg16(const float* x, int64_t n, float h, unsigned* hits) {
  const uint4* vp = (const uint4*)x;
  const int64_t nvec = n / 4, tile = (int64_t)U * BS;
  unsigned cnt = 0;
  for (int64_t base = (int64_t)blockIdx.x * tile; base + tile <= nvec; base += (int64_t)gridDim.x * tile) {
    uint4 r[U];
#pragma unroll
    for (int u = 0; u < U; ++u) r[u] = ld16<HINT>(vp + base + u * BS + threadIdx.x);
    bool a = false;
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint32_t w[4] = {r[u].x, r[u].y, r[u].z, r[u].w};
      a |= any_le(w, 4, h);
    }
    if (__any_sync(~0u, a)) cnt += __popc(__ballot_sync(~0u, a));
  }
  if (cnt && threadIdx.x % 32 == 0) atomicAdd(hits, cnt);
}

template <int BS, int U>
__global__ void __launch_bounds__(BS) reg32(const float* x, int64_t n, float h, unsigned* hits) {
  const int64_t nv = n / 8, tile = (int64_t)U * BS;
  unsigned cnt = 0;
  for (int64_t base = (int64_t)blockIdx.x * tile; base + tile <= nv; base += (int64_t)gridDim.x * tile) {
    u8x r[U];
#pragma unroll
    for (int u = 0; u < U; ++u) r[u] = ld32(x + (base + u * BS + threadIdx.x) * 8);
    bool a = false;
#pragma unroll
    for (int u = 0; u < U; ++u) a |= any_le(r[u].v, 8, h);
    if (__any_sync(~0u, a)) cnt += __popc(__ballot_sync(~0u, a));
  }
  if (cnt && threadIdx.x % 32 == 0) atomicAdd(hits, cnt);
}

// ---- bulk copy primitives
__device__ __forceinline__ unsigned saddr(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned bar, unsigned c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(c) : "memory"); }
__device__ __forceinline__ void expect_tx(unsigned bar, unsigned b) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(b) : "memory"); }
__device__ __forceinline__ void arrive(unsigned bar) { asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory"); }
__device__ __forceinline__ void bulk(unsigned dst, const void* src, unsigned bytes, unsigned bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
__device__ __forceinline__ void bulk_hint(unsigned dst, const void* src, unsigned bytes, unsigned bar, uint64_t pol) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(dst), "l"(src), "r"(bytes), "r"(bar), "l"(pol) : "memory");
}
__device__ __forceinline__ void wait(unsigned bar, unsigned par) {
  unsigned ok = 0;
  while (!ok)
    asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}" : "=r"(ok) : "r"(bar), "r"(par) : "memory");
}
__device__ __forceinline__ uint4 lds128(unsigned a) {
  uint4 r;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "r"(a));
  return r;
}

// per-warp ring: ST stages of TB bytes (TB = 32 lanes x V vectors x 16 B)
template <int BS, int ST, int V>
__global__ void __launch_bounds__(BS, 1) tma_warp(const float* x, int64_t n, float h, unsigned* hits) {
  extern __shared__ __align__(128) unsigned char sm[];
  constexpr unsigned TB = 32 * V * 16;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const unsigned ring = saddr(sm) + warp * ST * TB;
  __shared__ __align__(8) uint64_t bars_[BS / 32][ST];
  const unsigned bars = saddr(&bars_[warp][0]);
  const int64_t G = (int64_t)gridDim.x * (BS / 32), g = (int64_t)blockIdx.x * (BS / 32) + warp;
  const int64_t ntile = (int64_t)n * 4 / TB;
  const int64_t mine = ntile > g ? (ntile - 1 - g) / G + 1 : 0;
  const char* src = (const char*)x;
  if (lane == 0) {
    for (int s = 0; s < ST; ++s) mbar_init(bars + 8 * s, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    for (int s = 0; s < ST && s < mine; ++s) {
      expect_tx(bars + 8 * s, TB);
      bulk(ring + s * TB, src + (g + s * G) * TB, TB, bars + 8 * s);
    }
  }
  __syncwarp();
  unsigned cnt = 0;
  for (int64_t i = 0; i < mine; ++i) {
    const int s = (int)(i % ST);
    wait(bars + 8 * s, (unsigned)((i / ST) & 1));
    bool a = false;
#pragma unroll
    for (int u = 0; u < V; ++u) {
      const uint4 r = lds128(ring + s * TB + (u * 32 + lane) * 16);
      const uint32_t w[4] = {r.x, r.y, r.z, r.w};
      a |= any_le(w, 4, h);
    }
    if (__any_sync(~0u, a)) cnt += __popc(__ballot_sync(~0u, a));
    __syncwarp();
    if (lane == 0 && i + ST < mine) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      expect_tx(bars + 8 * s, TB);
      bulk(ring + s * TB, src + (g + (i + ST) * G) * TB, TB, bars + 8 * s);
    }
  }
  if (cnt && lane == 0) atomicAdd(hits, cnt);
}

// per-CTA ring: ST stages of CB bytes; thread 0 produces, every warp consumes its 1/NW of a stage,
// then arrives on the stage's "empty" barrier (count NW)
template <int BS, int ST, int CB>
__global__ void __launch_bounds__(BS, 1) tma_cta(const float* x, int64_t n, float h, unsigned* hits) {
  extern __shared__ __align__(128) unsigned char sm[];
  constexpr int NW = BS / 32;
  constexpr int VPT = CB / 16 / BS;  // vectors per thread per stage
  __shared__ __align__(8) uint64_t full_[ST], empty_[ST];
  const unsigned ring = saddr(sm), fb = saddr(full_), eb = saddr(empty_);
  const int64_t nchunk = (int64_t)n * 4 / CB;
  const int64_t mine = nchunk > blockIdx.x ? (nchunk - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  const char* src = (const char*)x;
  if (threadIdx.x == 0) {
    for (int s = 0; s < ST; ++s) { mbar_init(fb + 8 * s, 1); mbar_init(eb + 8 * s, NW); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0)
    for (int s = 0; s < ST && s < mine; ++s) {
      expect_tx(fb + 8 * s, CB);
      bulk(ring + s * CB, src + (blockIdx.x + (int64_t)s * gridDim.x) * CB, CB, fb + 8 * s);
    }
  unsigned cnt = 0;
  for (int64_t i = 0; i < mine; ++i) {
    const int s = (int)(i % ST);
    const unsigned par = (unsigned)((i / ST) & 1);
    wait(fb + 8 * s, par);
    bool a = false;
#pragma unroll
    for (int u = 0; u < VPT; ++u) {
      const uint4 r = lds128(ring + s * CB + (u * BS + threadIdx.x) * 16);
      const uint32_t w[4] = {r.x, r.y, r.z, r.w};
      a |= any_le(w, 4, h);
    }
    if (__any_sync(~0u, a)) cnt += __popc(__ballot_sync(~0u, a));
    __syncwarp();
    if (threadIdx.x % 32 == 0) arrive(eb + 8 * s);
    if (threadIdx.x == 0 && i + ST < mine) {
      wait(eb + 8 * s, par);  // every warp has consumed stage s
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      expect_tx(fb + 8 * s, CB);
      bulk(ring + s * CB, src + (blockIdx.x + (i + ST) * (int64_t)gridDim.x) * CB, CB, fb + 8 * s);
    }
  }
  if (cnt && threadIdx.x % 32 == 0) atomicAdd(hits, cnt);
}

// tma_cta variants: LAG refills the stage released one iteration earlier (as libairtopk does);
// OFF places the ring OFF bytes into dynamic shared memory (after a histogram, as libairtopk does)
template <int BS, int ST, int CB, int LAG, int OFF>
__global__ void __launch_bounds__(BS, 1) tma_cta2(const float* x, int64_t n, float h, unsigned* hits) {
  extern __shared__ __align__(128) unsigned char sm[];
  constexpr int NW = BS / 32;
  constexpr int VPT = CB / 16 / BS;
  const unsigned ring = saddr(sm) + OFF, fb = ring + ST * CB, eb = fb + 8 * ST;
  const int64_t nchunk = (int64_t)n * 4 / CB;
  const int64_t mine = nchunk > blockIdx.x ? (nchunk - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  const char* src = (const char*)x;
  if (threadIdx.x == 0) {
    for (int s = 0; s < ST; ++s) { mbar_init(fb + 8 * s, 1); mbar_init(eb + 8 * s, NW); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    for (int s = 0; s < ST && s < mine; ++s) {
      expect_tx(fb + 8 * s, CB);
      bulk(ring + s * CB, src + (blockIdx.x + (int64_t)s * gridDim.x) * CB, CB, fb + 8 * s);
    }
  }
  __syncthreads();
  unsigned cnt = 0;
  for (int64_t i = 0; i < mine; ++i) {
    const int s = (int)(i % ST);
    wait(fb + 8 * s, (unsigned)((i / ST) & 1));
    bool a = false;
#pragma unroll
    for (int u = 0; u < VPT; ++u) {
      const uint4 r = lds128(ring + s * CB + ((threadIdx.x / 32) * VPT * 32 + u * 32 + threadIdx.x % 32) * 16);
      const uint32_t w[4] = {r.x, r.y, r.z, r.w};
      a |= any_le(w, 4, h);
    }
    if (__any_sync(~0u, a)) cnt += __popc(__ballot_sync(~0u, a));
    __syncwarp();
    if (threadIdx.x % 32 == 0) arrive(eb + 8 * s);
    const int64_t j = i - LAG;
    if (threadIdx.x == 0 && j >= 0 && j + ST < mine) {
      const int sp = (int)(j % ST);
      wait(eb + 8 * sp, (unsigned)((j / ST) & 1));
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      expect_tx(fb + 8 * sp, CB);
      bulk(ring + sp * CB, src + (blockIdx.x + (j + ST) * (int64_t)gridDim.x) * CB, CB, fb + 8 * sp);
    }
  }
  if (cnt && threadIdx.x % 32 == 0) atomicAdd(hits, cnt);
}

template <typename F>
void timeit(const char* name, int grid, F launch, int64_t n) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int w = 0; w < 3; ++w) launch();
  cudaEventRecord(a);
  const int it = 10;
  for (int w = 0; w < it; ++w) launch();
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  ms /= it;
  cudaError_t e = cudaGetLastError();
  printf("%-34s grid=%4d  %.3f ms  %6.0f GB/s %s\n", name, grid, ms, n * 4.0 / (ms * 1e-3) / 1e9,
         e == cudaSuccess ? "" : cudaGetErrorString(e));
}

int main(int argc, char** argv) {
  const int64_t n = 1LL << 30;
  float* x;
  unsigned* hits;
  cudaMalloc(&x, n * 4);
  cudaMalloc(&hits, 4);
  fill<<<148 * 8, 512>>>(x, n);
  cudaDeviceSynchronize();
  const float h = 0.0024f;
  char nm[64];
  // memcpy reference (read + write bytes / 2 = read rate equivalent)
  {
    float* y;
    cudaMalloc(&y, (n / 2) * 4);
    timeit("cudaMemcpy D2D 2GiB (rd+wr)", 0, [&] { cudaMemcpyAsync(y, x, (n / 2) * 4, cudaMemcpyDeviceToDevice); }, n);
    cudaFree(y);
  }
#define REG16(BS, U, HINT, BPS)                                                                  \
  snprintf(nm, sizeof nm, "reg16 bs%d u%d hint%d bps%d", BS, U, HINT, BPS);                      \
  timeit(nm, 148 * BPS, [&] { reg16<BS, U, HINT><<<148 * BPS, BS>>>(x, n, h, hits); }, n);
  REG16(512, 4, 0, 2) REG16(512, 4, 0, 3) REG16(512, 4, 1, 2) REG16(512, 4, 1, 3) REG16(512, 4, 2, 2)
  REG16(256, 4, 0, 4) REG16(256, 4, 0, 6) REG16(256, 8, 0, 4) REG16(1024, 4, 0, 1) REG16(1024, 2, 0, 2)
  REG16(512, 2, 0, 4) REG16(512, 8, 0, 2) REG16(256, 4, 1, 6)
#define REG32(BS, U, BPS)                                                                        \
  snprintf(nm, sizeof nm, "reg32 bs%d u%d bps%d", BS, U, BPS);                                   \
  timeit(nm, 148 * BPS, [&] { reg32<BS, U><<<148 * BPS, BS>>>(x, n, h, hits); }, n);
  REG32(512, 2, 2) REG32(512, 2, 3) REG32(512, 4, 2) REG32(256, 2, 4) REG32(512, 1, 4)
#define TW(BS, ST, V, BPS)                                                                                      \
  {                                                                                                             \
    const int smem = (BS / 32) * ST * 32 * V * 16;                                                              \
    cudaFuncSetAttribute(tma_warp<BS, ST, V>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);               \
    snprintf(nm, sizeof nm, "tma_warp bs%d st%d tile%dB bps%d", BS, ST, 32 * V * 16, BPS);                      \
    timeit(nm, 148 * BPS, [&] { tma_warp<BS, ST, V><<<148 * BPS, BS, smem>>>(x, n, h, hits); }, n);            \
  }
  TW(512, 4, 4, 1) TW(512, 2, 4, 1) TW(512, 3, 4, 1) TW(512, 6, 4, 1) TW(512, 2, 8, 1) TW(512, 3, 8, 1)
  TW(256, 4, 4, 2) TW(256, 3, 8, 2) TW(512, 2, 4, 2) TW(256, 4, 8, 1) TW(512, 2, 2, 1) TW(512, 4, 2, 1)
#define TC(BS, ST, CB, BPS)                                                                                     \
  {                                                                                                             \
    const int smem = ST * CB;                                                                                   \
    cudaFuncSetAttribute(tma_cta<BS, ST, CB>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);               \
    snprintf(nm, sizeof nm, "tma_cta bs%d st%d chunk%dK bps%d", BS, ST, CB / 1024, BPS);                        \
    timeit(nm, 148 * BPS, [&] { tma_cta<BS, ST, CB><<<148 * BPS, BS, smem>>>(x, n, h, hits); }, n);            \
  }
  TC(512, 4, 16384, 1) TC(512, 8, 16384, 1) TC(512, 4, 32768, 1) TC(512, 6, 32768, 1) TC(512, 3, 65536, 1)
  TC(256, 4, 16384, 2) TC(256, 6, 16384, 2) TC(256, 3, 32768, 2) TC(512, 12, 16384, 1) TC(256, 8, 8192, 2)
#define TC2(BS, ST, CB, LAG, OFF)                                                                               \
  {                                                                                                             \
    const int smem = OFF + ST * (CB + 16);                                                                      \
    cudaFuncSetAttribute(tma_cta2<BS, ST, CB, LAG, OFF>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);    \
    snprintf(nm, sizeof nm, "tma_cta2 st%d %dK lag%d off%d", ST, CB / 1024, LAG, OFF);                          \
    timeit(nm, 148, [&] { tma_cta2<BS, ST, CB, LAG, OFF><<<148, BS, smem>>>(x, n, h, hits); }, n);             \
  }
  TC2(512, 12, 16384, 0, 0) TC2(512, 12, 16384, 1, 0) TC2(512, 12, 16384, 0, 8320) TC2(512, 12, 16384, 1, 8320)
  TC2(512, 8, 16384, 1, 8320) TC2(512, 6, 32768, 1, 8320) TC2(512, 6, 32768, 0, 0) TC2(512, 4, 32768, 0, 0)
  TC2(512, 12, 16384, 0, 1024) TC2(512, 12, 16384, 0, 4096)
  cudaError_t e = cudaGetLastError();
  printf("err=%s\n", cudaGetErrorString(e));
  return 0;
}
