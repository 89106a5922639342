// engine_grid.cu — the iteration-fused multi-CTA engine (one launch per radix pass).
//
// Algorithm 1 of the paper, as reconstructed in SURVEY.md §8(c)-0, mapped to B200:
//   host (Alg1 L1-5): memset the per-row state, then enqueue P+1 launches of grid_pass_kernel
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
// B200 mapping: grid = batch x cpr CTAs of 512 threads (cpr sized to fill 148 SMs), each CTA a
// contiguous slice of its row, 128-bit ld.global.nc.L1::no_allocate loads x4 unrolled, 2048-bin
// shared histogram merged with global red.add of the nonzero bins only, warp-aggregated appends
// (one atomic per warp and predicate) for results and candidates.
#include <algorithm>
#include <type_traits>

#include "device.cuh"
#include "engine.h"

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
constexpr int kUnroll = 4;
constexpr int kMinBlocks = 2;

template <int KIND, typename IdxT, bool HASIDX, int HMODE>
__global__ void __launch_bounds__(kBlock, kMinBlocks) grid_pass_kernel(const GridParams p, const int q) {
  using U = typename KT<KIND>::U;
  using CountT = std::conditional_t<sizeof(IdxT) == 8, unsigned long long, unsigned>;
  constexpr int R = KT<KIND>::R;
  constexpr int VEC = 16 / sizeof(U);

  __shared__ unsigned sh_hist[kMaxBins];
  __shared__ unsigned long long sh_tmp[kBlock / 32];
  __shared__ ScanResult sh_res;
  __shared__ int sh_last;

  const int64_t row = blockIdx.x / p.cpr;
  const int cta = blockIdx.x % p.cpr;
  const int tid = threadIdx.x;
  RowState* st = p.st + row;

  // ---- row state after scan q-1 ----
  const int stop1 = (q > 0) ? st->stop1 : 0;
  if (q > 0 && stop1 != 0 && stop1 - 1 < q - 1) return;  // finished by an earlier early stop
  const bool emit_all = (q > 0) && ((stop1 != 0 && stop1 - 1 == q - 1) || q == p.P);
  const bool do_hist = !emit_all;
  const unsigned long long Cprev = (q > 0) ? st->C : (unsigned long long)p.len;   // C_{q-1}
  const unsigned long long Cpp = (q > 0) ? st->Cp : (unsigned long long)p.len;    // C' = C_{q-2}
  const bool srcL = (q == 0) || (Cpp > (unsigned long long)p.cap_rule);            // Alg1 L7
  const bool store = do_hist && q > 0 && (Cprev <= (unsigned long long)p.cap_rule);  // Alg1 L17
  const bool sel_min = p.sel_min != 0;

  const Digit dh = digit_of(q, R, p.IB);
  const Digit df = digit_of(q > 0 ? q - 1 : 0, R, p.IB);

  U tgt_c = 0, base_c = 0, full_code = 0;
  IdxT tgt_i = 0, base_i = 0;
  if (q > 0) {
    const unsigned long long tc = st->tcode, ti = st->tidx;
    if (!df.is_idx) {
      tgt_c = (U)(tc >> df.shift);
      base_c = (U)(tgt_c & (U)~(U)((1u << df.width) - 1u));
    } else {
      full_code = (U)tc;
      tgt_i = (IdxT)(ti >> df.shift);
      base_i = (IdxT)(tgt_i & ~(IdxT)((1u << df.width) - 1u));
    }
  }

  if (do_hist) {
    for (int i = tid; i < kMaxBins; i += kBlock) sh_hist[i] = 0;
    __syncthreads();
  }

  unsigned long long* outc = &st->out_count;
  unsigned long long* bufc = &st->buf_count[q & 1];
  U* const bc_out = (U*)p.bcode + ((size_t)(q & 1) * p.batch + row) * p.cap_alloc;
  IdxT* const bi_out = (IdxT*)p.bidx + ((size_t)(q & 1) * p.batch + row) * p.cap_alloc;
  U* const ov = (U*)p.out_vals + row * p.k;
  int64_t* const oi = p.out_idx + row * p.k;
  const unsigned hmask = (1u << dh.width) - 1u;
  const unsigned long long kk = (unsigned long long)p.k;
  const unsigned long long capa = (unsigned long long)p.cap_alloc;

  auto process = [&](U code, IdxT idx, bool valid) {
    bool cand;
    if (q == 0) {
      cand = valid;
    } else {
      bool lt, eq;
      if (!df.is_idx) {
        const U h = (U)(code >> df.shift);
        lt = (h >= base_c) & (h < tgt_c);
        eq = (h == tgt_c);
      } else {
        const bool ce = (code == full_code);
        const IdxT h = (IdxT)(idx >> df.shift);
        lt = ce & (h >= base_i) & (h < tgt_i);
        eq = ce & (h == tgt_i);
      }
      const bool win = valid & (lt | (emit_all & eq));
      cand = valid & !emit_all & eq;
      unsigned m;
      const unsigned long long pos = warp_alloc(win, outc, m);  // Alg1 L22: add e to V
      if (win) {
        if (pos < kk) {
          ov[pos] = from_code<KIND>(code, sel_min);
          oi[pos] = (int64_t)idx;
        } else {
          st->error = 1u;
        }
      }
      if (store) {                                              // Alg1 L17-18
        const unsigned long long bpos = warp_alloc(cand, bufc, m);
        if (cand) {
          if (bpos < capa) {
            bc_out[bpos] = code;
            bi_out[bpos] = idx;
          } else {
            st->error = 2u;
          }
        }
      }
    }
    if (do_hist) {                                              // Alg1 L12-13 / L19-20
      const unsigned d = dh.is_idx ? ((unsigned)(idx >> dh.shift) & hmask) : ((unsigned)(code >> dh.shift) & hmask);
      hist_add<HMODE>(sh_hist, d, cand);
    }
  };

  unsigned long long nread;
  if (srcL) {
    // ---- source = the input row L (contiguous slice per CTA, 16-byte vectors) ----
    const U* rowp = (const U*)p.keys + row * p.len;
    const int64_t* rowi = HASIDX ? p.in_idx + row * p.len : nullptr;
    const uintptr_t mis = (uintptr_t)rowp & 15u;
    const int64_t head = mis ? std::min<int64_t>(p.len, (int64_t)((16u - mis) / sizeof(U))) : 0;
    const int64_t nvec = (p.len - head) / VEC;
    const int64_t tail0 = head + nvec * VEC;
    const int64_t per = (nvec + p.cpr - 1) / p.cpr;
    const int64_t v0 = std::min<int64_t>(nvec, (int64_t)cta * per);
    const int64_t v1 = std::min<int64_t>(nvec, v0 + per);
    const uint4* vp = (const uint4*)(rowp + head);
    nread = p.len;
    for (int64_t base = v0; base < v1; base += (int64_t)kBlock * kUnroll) {
      uint4 r[kUnroll];
#pragma unroll
      for (int u = 0; u < kUnroll; ++u) {
        const int64_t v = base + (int64_t)u * kBlock + tid;
        r[u] = (v < v1) ? ldg_stream(vp + v) : make_uint4(0, 0, 0, 0);
      }
#pragma unroll
      for (int u = 0; u < kUnroll; ++u) {
        const int64_t v = base + (int64_t)u * kBlock + tid;
        const bool valid = v < v1;
#pragma unroll
        for (int e = 0; e < VEC; ++e) {
          const int64_t i = head + v * VEC + e;
          const IdxT idx = HASIDX ? (valid ? (IdxT)rowi[i] : (IdxT)0) : (IdxT)i;
          process(to_code<KIND>(vec_elem<U>(r[u], e), sel_min), idx, valid);
        }
      }
    }
    if (cta == 0 && head > 0) {
      const int64_t i = tid;
      const bool valid = i < head;
      const U bits = valid ? rowp[i] : (U)0;
      const IdxT idx = HASIDX ? (valid ? (IdxT)rowi[i] : (IdxT)0) : (IdxT)i;
      process(to_code<KIND>(bits, sel_min), idx, valid);
    }
    if (cta == p.cpr - 1 && tail0 < p.len) {
      const int64_t i = tail0 + tid;
      const bool valid = i < p.len;
      const U bits = valid ? rowp[i] : (U)0;
      const IdxT idx = HASIDX ? (valid ? (IdxT)rowi[i] : (IdxT)0) : (IdxT)i;
      process(to_code<KIND>(bits, sel_min), idx, valid);
    }
  } else {
    // ---- source = candidate buffer written by kernel q-1 (codes + indices) ----
    const int slot = (q - 1) & 1;
    const unsigned long long n = st->buf_count[slot];
    const U* bc = (const U*)p.bcode + ((size_t)slot * p.batch + row) * p.cap_alloc;
    const IdxT* bi = (const IdxT*)p.bidx + ((size_t)slot * p.batch + row) * p.cap_alloc;
    const unsigned long long per = (n + p.cpr - 1) / p.cpr;
    const unsigned long long e0 = std::min<unsigned long long>(n, (unsigned long long)cta * per);
    const unsigned long long e1 = std::min<unsigned long long>(n, e0 + per);
    nread = n;
    for (unsigned long long base = e0; base < e1; base += kBlock) {
      const unsigned long long i = base + tid;
      const bool valid = i < e1;
      const U code = valid ? bc[i] : (U)0;
      const IdxT idx = valid ? bi[i] : (IdxT)0;
      process(code, idx, valid);
    }
  }

  if (!do_hist) return;

  // ---- merge into the row histogram; the last CTA scans ----
  __syncthreads();
  CountT* gh = (CountT*)p.ghist + ((size_t)row * 2 + (q & 1)) * kMaxBins;
  const int nb = 1 << dh.width;
  for (int i = tid; i < nb; i += kBlock) {
    const unsigned v = sh_hist[i];
    if (v) atomicAdd(&gh[i], (CountT)v);
  }
  __threadfence();
  __syncthreads();
  if (tid == 0) sh_last = (atomicAdd(&st->ticket, 1u) == (unsigned)(p.cpr - 1));
  __syncthreads();
  if (!sh_last) return;
  __threadfence();

  const unsigned long long Kin = (q == 0) ? kk : st->K;
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
      t[0] = dh.width; t[1] = srcL; t[2] = store; t[3] = r.j; t[4] = (int64_t)newK; t[5] = (int64_t)newC;
      t[6] = (int64_t)Cin; t[7] = (int64_t)__ldcg(outc); t[8] = (newK == newC); t[9] = (int64_t)nread;
    }
  }
}

// K == N ("a trivial case"): every element is a result, in index order.
template <typename U>
__global__ void trivial_kernel(const U* keys, int64_t total, U* ov, int64_t* oi, int64_t len) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    ov[i] = keys[i];
    oi[i] = i % len;
  }
}

namespace {

int hmode_from_env() {
  static int m = [] {
    const char* e = getenv("AIRTOPK_HMODE");
    return e ? atoi(e) : 1;
  }();
  return m;
}

struct Events {
  void* const* ev;
  int n;
  void record(int i, cudaStream_t s) const {
    if (ev && i < n) cudaEventRecord((cudaEvent_t)ev[i], s);
  }
};

template <int KIND, typename IdxT, bool HASIDX, int HMODE>
cudaError_t launch_passes(const GridParams& gp, int64_t batch, const Events& ev, cudaStream_t s) {
  const long long grid = (long long)batch * gp.cpr;
  ev.record(0, s);
  for (int q = 0; q <= gp.P; ++q) {
    grid_pass_kernel<KIND, IdxT, HASIDX, HMODE><<<(unsigned)grid, kBlock, 0, s>>>(gp, q);
    ev.record(q + 1, s);
  }
  return cudaGetLastError();
}

template <int KIND, typename IdxT, bool HASIDX>
cudaError_t launch_h(const GridParams& gp, int64_t batch, const Events& ev, cudaStream_t s) {
  if constexpr (KIND == K_F32 && !HASIDX && sizeof(IdxT) == 4) {
    switch (hmode_from_env()) {
      case 0: return launch_passes<KIND, IdxT, HASIDX, 0>(gp, batch, ev, s);
      case 2: return launch_passes<KIND, IdxT, HASIDX, 2>(gp, batch, ev, s);
      default: break;
    }
  }
  return launch_passes<KIND, IdxT, HASIDX, 1>(gp, batch, ev, s);
}

template <int KIND>
cudaError_t launch_kind(const SelectArgs& a, const Plan& pl, const GridParams& gp, cudaStream_t s) {
  const Events ev{a.events, a.n_events};
  if (a.in_idx) return launch_h<KIND, uint64_t, true>(gp, a.batch, ev, s);
  if (pl.idx64) return launch_h<KIND, uint64_t, false>(gp, a.batch, ev, s);
  return launch_h<KIND, uint32_t, false>(gp, a.batch, ev, s);
}

}  // namespace

int grid_blocks_per_sm(const SelectArgs& a, int idx64) {
  int n = 0;
  cudaError_t e;
  if (idx64) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, grid_pass_kernel<K_F32, uint64_t, false, 1>, kBlock, 0);
  else e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, grid_pass_kernel<K_F32, uint32_t, false, 1>, kBlock, 0);
  (void)a;
  if (e != cudaSuccess || n < 1) n = kMinBlocks;
  return n;
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
  gp.trace = a.trace;
  switch (a.kind) {
    case K_F32: return launch_kind<K_F32>(a, pl, gp, s);
    case K_F16: return launch_kind<K_F16>(a, pl, gp, s);
    case K_BF16: return launch_kind<K_BF16>(a, pl, gp, s);
    case K_F64: return launch_kind<K_F64>(a, pl, gp, s);
    case K_U32: return launch_kind<K_U32>(a, pl, gp, s);
  }
  return cudaErrorInvalidValue;
}

cudaError_t run_trivial(const SelectArgs& a, cudaStream_t s) {
  const int64_t total = a.batch * a.len;
  const int threads = 256;
  const long long blocks = std::min<long long>((total + threads - 1) / threads, 148LL * 16);
  switch (key_bytes(a.kind)) {
    case 2: trivial_kernel<uint16_t><<<(unsigned)blocks, threads, 0, s>>>((const uint16_t*)a.keys, total, (uint16_t*)a.out_vals, a.out_idx, a.len); break;
    case 4: trivial_kernel<uint32_t><<<(unsigned)blocks, threads, 0, s>>>((const uint32_t*)a.keys, total, (uint32_t*)a.out_vals, a.out_idx, a.len); break;
    default: trivial_kernel<uint64_t><<<(unsigned)blocks, threads, 0, s>>>((const uint64_t*)a.keys, total, (uint64_t*)a.out_vals, a.out_idx, a.len); break;
  }
  return cudaGetLastError();
}

}  // namespace airtopk
