// engine.h — internal (non-ABI) interface between the C-ABI layer (api.cu) and the engines.
#pragma once

#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>

namespace airtopk {

struct SelectArgs {
  const void* keys = nullptr;
  const int64_t* in_idx = nullptr;  // with_idx variant: caller-given index values (else positions)
  int idx_bits = 0;                 // with_idx variant: index value width
  int kind = 0;                     // Kind
  int64_t batch = 0, len = 0, k = 0;
  int sel_min = 1;
  void* out_vals = nullptr;
  int64_t* out_idx = nullptr;
  int64_t alpha = 128;
  int engine = 0;
  int ctas_per_row = 0;
  int cluster_size = 0;
  int window = 0;                   // sample-guided window: 0 auto, 1 on, -1 off
  int tma = 0;                      // bulk-copy streaming: 0 auto, 1 on, -1 off
  int early_stop = 0;               // 0 on, -1 off (ablation)
  int64_t idx_off = 0;              // added to every output index (airtopk_select_shard)
  unsigned* status = nullptr;       // optional device word: row error flags OR-ed in after the select
  int sorted = 0;                   // 1: rows sorted in selection order after the select (K <= 4096)
  int64_t* trace = nullptr;
  int64_t trace_len = 0;  // int64 entries of trace (0: batch * kTraceMaxPasses * kTraceFields)
  void* const* events = nullptr;    // optional cudaEvent_t[n_events] recorded around launches
  int n_events = 0;
};

// Resolved launch plan (host side).
struct Plan {
  int engine;        // 1 grid, 2 cluster, 3 trivial copy (K == N), 4 GridSelect, 5 batched, 6 resident cluster
  int idx64;         // 64-bit internal indices
  int R;             // key bits
  int IB;            // index bits appended to the key for the lowest-index tie-break
  int P;             // radix passes (code + index digits)
  int64_t cap_rule;  // buffer iff C <= cap_rule  (== C * alpha < N)
  int64_t cap_alloc; // entries allocated per candidate buffer
  int cpr;           // CTAs per row (grid engine)
  int cpr_buf;       // CTAs per row of the register-load passes after a bulk-copy window pass
  int csize;         // CTAs per cluster (cluster engine)
  int max_clusters;  // cluster engine: clusters the workspace has candidate buffers for
  int nsamp;         // grid engine: samples per row for the sample-guided window (0 = off)
  int tail;          // grid engine: finish after the window pass with one cluster-engine launch
  int tail_q;        // ... after the grid passes q < tail_q (0: right after the window pass)
  int tma;           // grid engine: stream rows through bulk-copy (TMA) shared rings, 1 CTA/SM
  int fused;         // grid engine, batch 1: every pass after the window pass in one cooperative launch
  // batched engine (engine 5, engine_batch.cuh): eligible by shape; slot geometry
  int batch_ok;      // the shape qualifies (alignment is checked at run time)
  int bnsamp;        // samples per row
  int cpc;           // 32 KiB chunks per row
  int nwc;           // slots per row (one per chunk)
  int scap;          // entries per slot
  int rslice;        // resident-cluster engine: keys per CTA
  size_t off_state, off_hist, off_thist, off_tcnt, off_bcode, off_bidx, off_samp, off_bcnt, off_bslot, off_bsidx,
      off_bfail, bytes;
};

// cudaFuncSetAttribute once per (kernel, current device, attribute, value): the runtime applies
// function attributes per device, so a process selecting on several GPUs sets them on each.
cudaError_t func_attr(const void* func, cudaFuncAttribute attr, int value);
template <typename F>
cudaError_t func_attr(F* func, cudaFuncAttribute attr, int value) {
  return func_attr(reinterpret_cast<const void*>(func), attr, value);
}

// Memoised occupancy queries (per kernel, current device and parameter): the runtime queries cost
// microseconds of host time, which the small configs (c1, c2 shards) cannot afford per call.
bool occ_cache_get(const void* f, int param, int* out);
void occ_cache_put(const void* f, int param, int value);

int key_bits(int kind);
int num_sms();  // SMs of the current device (cached per thread)
int key_bytes(int kind);
Plan make_plan(const SelectArgs& a);
cudaError_t run_grid(const SelectArgs& a, const Plan& p, void* ws, cudaStream_t s);
cudaError_t run_cluster(const SelectArgs& a, const Plan& p, void* ws, cudaStream_t s);
cudaError_t run_batch(const SelectArgs& a, const Plan& p, void* ws, cudaStream_t s);
cudaError_t run_resident(const SelectArgs& a, const Plan& p, void* ws, cudaStream_t s);
// batched engine constants shared with the host plan (engine_batch.cuh)
constexpr int kBatchBlock = 1024, kBatchWarps = 32;
#ifndef AIRTOPK_BATCH_GROUPS
#define AIRTOPK_BATCH_GROUPS 4        // phase-B consumer warp groups (take ring stages in turn)
#endif
#ifndef AIRTOPK_BATCH_STAGE_BYTES
#define AIRTOPK_BATCH_STAGE_BYTES 24576
#endif
constexpr int kBatchStage = AIRTOPK_BATCH_STAGE_BYTES;      // bytes per chunk (one bulk-copy ring stage)
constexpr int kBatchFcap = 16384;    // entries (results + window members) one row may stage in the finish
// resident-cluster engine (engine_resident.cuh)
constexpr int kResidentCap = 32768;  // keys per CTA held in shared memory (<= 4-byte keys; half for 8-byte)
constexpr int kResidentFin = 2048;   // candidates CTA 0 finishes
cudaError_t run_trivial(const SelectArgs& a, cudaStream_t s);
// K entries that sort last in the selection order (multi-GPU shard shorter than K): value bits of the
// maximum code, indices pad_base + j
cudaError_t run_pad(int kind, int sel_min, void* vals, int64_t* idx, int64_t n, int64_t pad_base, cudaStream_t s);
// sort every row's K results in selection order (one CTA per row, bitonic in shared memory, K <= 4096)
cudaError_t run_sort_rows(const SelectArgs& a, cudaStream_t s);
constexpr int64_t kSortMaxK = 4096;
// OR the error flags of every row state of a grid / cluster engine workspace into *a.status
cudaError_t collect_status(const SelectArgs& a, const Plan& p, void* ws, cudaStream_t s);
int grid_blocks_per_sm(const SelectArgs& a, int idx64);
// GridSelect: keys of <= 32 bits, len < 2^32, K <= 256
bool gridselect_supported(const SelectArgs& a);
int gridselect_ctas(const SelectArgs& a);
size_t gridselect_workspace(const SelectArgs& a, int G);
cudaError_t run_gridselect(const SelectArgs& a, void* ws, size_t ws_bytes, cudaStream_t s);

}  // namespace airtopk
