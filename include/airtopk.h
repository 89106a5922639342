/*
 * airtopk.h — C ABI of the B200-native AIR Top-K library (libairtopk.so).
 *
 * AIR Top-K = Adaptive and Iteration-fused Radix Top-K, Zhang, Li, Naruse, Wang, SC'23
 * (/root/reference/PAPER.md; "P:n" below = line n of that file).
 *
 * Operation (§2.1 "Problem Statement"): for each row L of `len` elements and
 * K = k in [1, len], produce a value list V and an index list I of length K with
 * L[I[i]] = V[i] and V[i] <= L[j] for every j not in I — the K smallest elements
 * ("without loss of generality") or, with select_min = 0, the K largest.
 * Batches of rows with the same len and K are solved together (§5.1).
 *
 * Method (all on the GPU, the host only enqueues kernels — P:50):
 *   multi-pass MSD radix select over order-preserving key bits with b = 11-bit digits
 *   (§2.3): per pass a histogram, an inclusive prefix sum, the target digit j
 *   with psum[j-1] < K <= psum[j], and a filter that emits definite winners and keeps the
 *   candidates; filter(i-1) and histogram(i) fused in one kernel (§3.1); the scan run by
 *   the last CTA to finish; candidates buffered only while C < N/alpha, else the next pass
 *   re-reads the input (§3.2, alpha = 128 as in P:210); early stop when K == C (§3.3).
 *
 * Semantics fixed by this library where the paper is silent:
 *   - Order: IEEE-754 total order of the key bits (-NaN < -inf < ... < -0 < +0 < ... < +inf < +NaN);
 *     u32 keys use their natural order. No floating-point arithmetic is performed on keys.
 *   - Ties at the K-th key are broken by LOWEST index (row-local index; for
 *     airtopk_select_with_idx, by the smallest in_idx VALUE).
 *   - out_vals are raw bit copies of the selected input elements (NaN payloads, -0.0 preserved).
 *   - The order of the K results within a row is UNSPECIFIED.
 *
 * Layout: keys are row-major [batch][len], contiguous, in DEVICE memory (any alignment of the
 * element type). out_vals is [batch][k] of the key type, out_idx is [batch][k] int64, both device
 * memory, row-local indices in [0, len). Outputs must not alias keys or the workspace.
 *
 * Ownership: the caller owns every buffer. The library never frees, retains or writes through
 * caller pointers other than out_vals / out_idx / workspace, and never modifies keys.
 * Calls are stateless and re-entrant: concurrent calls on different streams must use distinct
 * workspaces (the convenience entry points allocate their own with cudaMallocAsync).
 *
 * Asynchrony / errors: every entry point except airtopk_select_host only ENQUEUES work on
 * `stream` (no host synchronisation, no device->host copy) and returns:
 *   AIRTOPK_OK         work enqueued;
 *   AIRTOPK_EINVAL     null pointer, batch < 1, len < 1, k < 1 or k > len (K in [1, N]);
 *   AIRTOPK_EDTYPE     unknown dtype;
 *   AIRTOPK_ENOSPACE   workspace smaller than airtopk_workspace_bytes(...);
 *   AIRTOPK_ECUDA      a CUDA launch/allocation failed (airtopk_last_cuda_error() has the code);
 *   AIRTOPK_EDEVICE    (synchronous calls only: airtopk_select_host) the kernels flagged an
 *                      inconsistency, e.g. duplicate in_idx values (see airtopk_options.status).
 * Faults inside kernels surface at the caller's next synchronisation, as with any CUDA library.
 * Inconsistencies the kernels detect (more than K results or fewer, which only duplicate in_idx
 * values can cause) are reported through the optional device word airtopk_options.status.
 * Nothing is written to the outputs when a status other than AIRTOPK_OK is returned.
 */
#ifndef AIRTOPK_H_
#define AIRTOPK_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* cudaStream_t without requiring cuda_runtime.h; 0 = the legacy default stream. */
typedef struct CUstream_st* airtopk_stream_t;

typedef enum {
  AIRTOPK_OK = 0,
  AIRTOPK_EINVAL = 1,
  AIRTOPK_EDTYPE = 2,
  AIRTOPK_ENOSPACE = 3,
  AIRTOPK_ECUDA = 4,
  AIRTOPK_EDEVICE = 5
} airtopk_status;

/* Bits OR-ed into *airtopk_options.status (device-detected inconsistencies; 0 = none). */
#define AIRTOPK_ERR_OUTPUT_OVERFLOW 1u  /* more than K results in a row (duplicate in_idx values) */
#define AIRTOPK_ERR_BUFFER_OVERFLOW 2u  /* a candidate buffer overflowed outside the window pass */
#define AIRTOPK_ERR_COUNT 4u            /* histogram total != candidates, or fewer than K results */

typedef enum {
  AIRTOPK_F32 = 0,  /* IEEE binary32, r = 32 bits: 3 radix passes of 11/11/10 bits */
  AIRTOPK_F16 = 1,  /* IEEE binary16, r = 16: 2 passes (11/5) */
  AIRTOPK_BF16 = 2, /* bfloat16, r = 16: 2 passes */
  AIRTOPK_F64 = 3,  /* IEEE binary64, r = 64: 6 passes (5 x 11 + 9) */
  AIRTOPK_U32 = 4   /* unsigned 32-bit integers, natural order */
} airtopk_dtype;

/* Engine selection (airtopk_options.engine). */
typedef enum {
  AIRTOPK_ENGINE_AUTO = 0,
  AIRTOPK_ENGINE_GRID = 1,    /* multi-CTA per row, one launch per pass, last-CTA scan */
  AIRTOPK_ENGINE_CLUSTER = 2, /* one thread-block cluster per row, all passes in one launch */
  AIRTOPK_ENGINE_GRIDSELECT = 4, /* the paper's second algorithm (§4): per-warp shared
                                   32-entry queue with two-step ballot insertion, sorted per-warp
                                   top-K lists, a row-wide shared threshold, CTA lists merged by the
                                   last CTA of the row. Same results (lowest-index ties). Only for
                                   keys of <= 32 bits, len < 2^32 and K <= 2048, else
                                   AIRTOPK_EINVAL. Rows come out sorted. Never chosen by AUTO. */
  AIRTOPK_ENGINE_BATCH = 5,     /* batched rows in ONE cooperative launch: per-row sample window,
                                   single read of every row into fixed per-chunk slots,
                                   per-row shared-memory finish; rows whose window fails are redone
                                   by a cluster-engine launch. Needs 16-byte aligned rows and a
                                   window that fits 16K entries per row, else AIRTOPK_EINVAL. */
  AIRTOPK_ENGINE_RESIDENT = 6,  /* rows of <= 512K keys (256K for f64) held in the shared memory of
                                   a thread-block cluster: one HBM read, every pass on chip. */
  AIRTOPK_ENGINE_GRIDSELECT_PTQ = 7 /* GridSelect with per-thread register queues instead of the
                                   shared queue: the Fig. 11 ablation. Same scope. */
} airtopk_engine;

/* Tuning / ablation knobs. Pass NULL for the defaults. */
typedef struct {
  int64_t alpha;        /* adaptive-buffer parameter: buffer candidates iff C * alpha < len.
                           0 = default 128; alpha >= len = never buffer; 1 = buffer
                           whenever at least one element was eliminated. Must be >= 0. */
  int32_t engine;       /* airtopk_engine; 0 = auto */
  int32_t ctas_per_row; /* grid engine: CTAs per row; 0 = auto (fills the 148 SMs) */
  int32_t cluster_size; /* cluster / resident engine: CTAs per cluster (1,2,4,8,16); 0 = auto */
  int32_t n_events;     /* number of entries in `events` */
  int64_t* trace;       /* optional DEVICE buffer of batch * AIRTOPK_TRACE_MAX_PASSES * 10 int64:
                           per-row state after each scan (width, src_is_input, stored, j, K, C, C',
                           emitted_so_far, early_stop, elements_read); unused slots untouched.
                           Grid engine only. NULL = no trace. */
  void* const* events;  /* optional array of n_events cudaEvent_t (created by the caller) recorded on
                           `stream` around the launches: events[0] before the first kernel,
                           events[i+1] after launch i — lets a caller time each kernel with CUDA
                           events on the launching stream. NULL = none. */
  int32_t window;       /* sample-guided window pass: 0 = auto (grid engine,
                           len >= 2^18), 1 = on, -1 = off (the paper's passes only). Exact either way. */
  int32_t tma;          /* grid engine streaming: 0 = auto (bulk-copy rings for a few long rows), 1 = bulk
                           copies (cp.async.bulk into a per-CTA ring of 32 KiB stages, mbarrier handshake),
                           -1 = register loads. */
  int32_t early_stop;   /* early stopping: 0 = on (default), -1 = off (the Fig. 10 ablation:
                           the passes continue after K == C; results identical). */
  uint32_t* status;     /* optional DEVICE word: after the select the library ORs every row's
                           AIRTOPK_ERR_* flags into it (one extra tiny launch; the caller zeroes it and
                           reads it after synchronising). NULL = not collected. Radix engines only. */
  int32_t sorted;       /* 1: every row's K results come out sorted in the selection order (ascending
                           keys for select-min, descending for select-max; equal keys by ascending
                           index) — one extra launch, K <= 4096 (else AIRTOPK_EINVAL). 0 = unordered
                           (GridSelect rows are always sorted). */
  int64_t trace_len;    /* int64 entries of `trace` (0 = the size stated there). The cluster, batched and
                           resident engines write per-CTA debug timing stamps into `trace` instead of
                           the per-row records; they never write past trace_len entries. */
} airtopk_options;

#define AIRTOPK_TRACE_MAX_PASSES 16

/* Bytes of device workspace a call with these arguments needs (grows with batch * len / alpha:
 * two candidate buffers of floor((len-1)/alpha) entries per row). 0 on invalid arguments. */
size_t airtopk_workspace_bytes(airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k);
size_t airtopk_workspace_bytes_ex(airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k,
                                  const airtopk_options* opt);

/* Generic entry point. workspace: device memory of at least airtopk_workspace_bytes_ex(...) bytes,
 * 256-byte aligned, owned by the caller, not used concurrently by another call. */
airtopk_status airtopk_select(const void* keys, airtopk_dtype dtype, int64_t batch, int64_t len,
                              int64_t k, int select_min, void* out_vals, int64_t* out_idx,
                              void* workspace, size_t workspace_bytes, airtopk_stream_t stream);
airtopk_status airtopk_select_ex(const void* keys, airtopk_dtype dtype, int64_t batch, int64_t len,
                                 int64_t k, int select_min, void* out_vals, int64_t* out_idx,
                                 void* workspace, size_t workspace_bytes, airtopk_stream_t stream,
                                 const airtopk_options* opt);

/* north_star signature, one per dtype: the workspace is taken from the stream-ordered pool
 * (cudaMallocAsync / cudaFreeAsync on `stream`), so these are also fully asynchronous.
 * 16-bit keys are passed as their raw uint16_t bit patterns. */
airtopk_status airtopk_select_f32(const float* keys, int64_t batch, int64_t len, int64_t k, int select_min,
                                  float* out_vals, int64_t* out_idx, airtopk_stream_t stream);
airtopk_status airtopk_select_f16(const uint16_t* keys, int64_t batch, int64_t len, int64_t k, int select_min,
                                  uint16_t* out_vals, int64_t* out_idx, airtopk_stream_t stream);
airtopk_status airtopk_select_bf16(const uint16_t* keys, int64_t batch, int64_t len, int64_t k, int select_min,
                                   uint16_t* out_vals, int64_t* out_idx, airtopk_stream_t stream);
airtopk_status airtopk_select_f64(const double* keys, int64_t batch, int64_t len, int64_t k, int select_min,
                                  double* out_vals, int64_t* out_idx, airtopk_stream_t stream);
airtopk_status airtopk_select_u32(const uint32_t* keys, int64_t batch, int64_t len, int64_t k, int select_min,
                                  uint32_t* out_vals, int64_t* out_idx, airtopk_stream_t stream);

/* Merge select for candidates gathered from several GPUs: a single row of
 * `len` keys whose elements carry caller-given index VALUES in_idx[len] (device, int64, distinct,
 * each in [0, 2^idx_bits)). Selects the K smallest (largest) keys, ties by smallest in_idx value;
 * out_idx receives in_idx values. idx_bits in [1, 63]. */
size_t airtopk_workspace_bytes_with_idx(airtopk_dtype dtype, int64_t len, int64_t k, int idx_bits);
airtopk_status airtopk_select_with_idx(const void* keys, const int64_t* in_idx, int idx_bits,
                                       airtopk_dtype dtype, int64_t len, int64_t k, int select_min,
                                       void* out_vals, int64_t* out_idx, void* workspace,
                                       size_t workspace_bytes, airtopk_stream_t stream);

/* Same with options (alpha, engine 1/2, status word, events, ...). */
airtopk_status airtopk_select_with_idx_ex(const void* keys, const int64_t* in_idx, int idx_bits,
                                          airtopk_dtype dtype, int64_t len, int64_t k, int select_min,
                                          void* out_vals, int64_t* out_idx, void* workspace,
                                          size_t workspace_bytes, airtopk_stream_t stream,
                                          const airtopk_options* opt);

/* Multi-GPU split row ("top 0.1% ... across workers").
 * One row of total_len keys is split into contiguous shards, one per rank. Each rank calls
 * airtopk_select_shard on its shard (len keys starting at global index shard_offset): it writes
 * exactly k entries — the min(k, len) smallest (largest) keys of the shard with GLOBAL indices
 * (local index + shard_offset; ties by lowest index, P:78 reading), and, when len < k, k - len pad
 * entries whose key sorts after every key (the maximum code) with indices pad_base + j, j < k - len.
 * The caller picks pad_base = total_len + rank * k so pad indices never collide. out_vals [k] of
 * the key type, out_idx [k] int64, device memory; the k entries of every rank are gathered
 * (one NCCL all-gather, or peer stores) into [world * k] arrays, and airtopk_select_with_idx with
 * idx_bits = airtopk_merge_idx_bits(total_len, world, k) gives the global top-k on every rank
 * (exact: a global top-k element has < k predecessors in (code, index) order, hence < k in its own
 * shard). Workspace: airtopk_workspace_bytes_shard(dtype, len, k) bytes, 256-aligned, device. */
size_t airtopk_workspace_bytes_shard(airtopk_dtype dtype, int64_t len, int64_t k);
airtopk_status airtopk_select_shard(const void* keys, airtopk_dtype dtype, int64_t len, int64_t k,
                                    int select_min, int64_t shard_offset, int64_t pad_base,
                                    void* out_vals, int64_t* out_idx, void* workspace,
                                    size_t workspace_bytes, airtopk_stream_t stream);
/* Index width of the merge select: bits of total_len + world * k - 1 (0 on invalid arguments). */
int airtopk_merge_idx_bits(int64_t total_len, int world, int64_t k);

/* Collective-fused split-row exchange over peer memory:
 * the NCCL all-gather replaced by direct stores into every rank's gather buffers (CUDA IPC; P2P over
 * NVLink / NVSwitch). Set-up (once per buffer set): each rank exports its gather buffers and flag
 * array with airtopk_ipc_handle (a 64-byte handle + the offset of the pointer inside its allocation),
 * the handles are exchanged out of band (e.g. torch.distributed all_gather_object), and every rank
 * opens its peers' with airtopk_ipc_open (and later airtopk_ipc_close). Per call, with a fresh
 * nonzero epoch (the same on every rank, e.g. a call counter):
 *   airtopk_shard_push   one launch: this rank's k values + global indices (from
 *                        airtopk_select_shard) are stored into slot `rank` of EVERY rank's gather
 *                        buffers (peer_vals[r] / peer_idx[r], r < world, this rank's own included),
 *                        then this rank's flag (peer_flags[r][rank]) is set to epoch in every rank
 *                        after all its stores are visible (system-scope fence + release store);
 *                        `ticket` is one zeroed device word owned by this rank (reset by the kernel);
 *   airtopk_wait_flags   one-CTA launch that returns once flags[0..world) all equal epoch (acquire);
 *                        the merge select enqueued after it sees every rank's entries.
 * Values are raw key bits of `dtype`, indices int64, buffers [world * k] on each rank's device. */
airtopk_status airtopk_ipc_handle(const void* dev_ptr, void* handle_out, uint64_t* offset_out);
airtopk_status airtopk_ipc_open(const void* handle, uint64_t offset, void** dev_ptr_out);
airtopk_status airtopk_ipc_close(void* dev_ptr);
airtopk_status airtopk_shard_push(const void* vals, const int64_t* idx, int64_t k, airtopk_dtype dtype, int world,
                                  int rank, void* const* peer_vals, int64_t* const* peer_idx,
                                  uint32_t* const* peer_flags, uint32_t epoch, uint32_t* ticket,
                                  airtopk_stream_t stream);
airtopk_status airtopk_wait_flags(const uint32_t* flags, int world, uint32_t epoch, airtopk_stream_t stream);

/* The paper's kernel-organisation ablations (§3.1), a plain radix
 * select with a runtime digit width: design 0 = naive (Fig. 2: histogram, prefix sum, target digit,
 * filter as four kernels per iteration), 1 = iteration-fused (Fig. 3: filter + histogram in one
 * kernel, scan in its last block, then a last-filter kernel), 2 = 1 with the last filter fused into the
 * last iteration. digit_bits 8 or 11. Same results as airtopk_select (lowest-index
 * ties). Keys of <= 32 bits, len < 2^32, 1 <= k < len, batch <= 65535; workspace from
 * airtopk_ablation_workspace. *kernels_out (optional) receives the launches enqueued. */
size_t airtopk_ablation_workspace(airtopk_dtype dtype, int64_t batch, int64_t len, int64_t alpha);
airtopk_status airtopk_select_ablation(const void* keys, airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k,
                                       int select_min, void* out_vals, int64_t* out_idx, int design, int digit_bits,
                                       int64_t alpha, void* workspace, size_t workspace_bytes,
                                       airtopk_stream_t stream, int* kernels_out);

/* End-to-end convenience with HOST buffers: copies keys host->device, selects, copies the results
 * device->host and SYNCHRONISES `stream` before returning. Pinned (page-locked) host memory gives
 * asynchronous DMA; pageable memory works but is staged by the driver. Device staging (keys,
 * outputs, workspace) is a per-thread, per-device cudaMalloc cache that grows on demand and is
 * released when the calling thread exits. */
airtopk_status airtopk_select_host(const void* h_keys, airtopk_dtype dtype, int64_t batch, int64_t len,
                                   int64_t k, int select_min, void* h_out_vals, int64_t* h_out_idx,
                                   airtopk_stream_t stream);

/* How a call with these arguments would run (no device work; may query the current device's SM
 * count). Lets callers count launches and label measurements. */
typedef struct {
  int32_t engine;        /* airtopk_engine actually used (3 = K == len trivial copy) */
  int32_t passes;        /* radix passes P (key digits + index digits) */
  int32_t launches;      /* kernel launches per call, excluding the workspace memset */
  int32_t ctas_per_row;  /* grid engine */
  int32_t cluster_size;  /* cluster engine */
  int32_t index_bits;    /* bits of the row index appended for the lowest-index tie-break */
  int64_t buffer_cap;    /* candidate-buffer capacity per row (floor((len-1)/alpha)) */
  size_t workspace_bytes;
} airtopk_plan;

airtopk_status airtopk_describe(airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k,
                                const airtopk_options* opt, airtopk_plan* out);

/* Human-readable status; never NULL. */
const char* airtopk_status_str(airtopk_status s);
/* cudaError_t (as int) of the most recent AIRTOPK_ECUDA on this thread; 0 if none. */
int airtopk_last_cuda_error(void);
/* Library version, e.g. "0.1.0". */
const char* airtopk_version(void);

#ifdef __cplusplus
}
#endif

#endif /* AIRTOPK_H_ */
