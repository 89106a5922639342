// api.cu — the C ABI of libairtopk.so (declared and documented in include/airtopk.h).
//
// Argument validation (K in [1, N]), dtype dispatch, workspace carve-up and launch
// sequencing. Every entry point except airtopk_select_host only enqueues work on the caller's
// stream (the iteration-fused property: the CPU only launches kernels, P:50/P:142/P:158).
#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>
#include <set>
#include <tuple>
#include <cmath>
#include <cstring>

#include <nvtx3/nvToolsExt.h>

#include "../../include/airtopk.h"
#include "device.cuh"
#include "engine.h"

namespace airtopk {

namespace {
thread_local int g_last_cuda_error = 0;

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

int bits_needed(uint64_t v) {  // number of bits to represent v (0 for v == 0)
  int b = 0;
  while (v) { ++b; v >>= 1; }
  return b;
}

}  // namespace

cudaError_t func_attr(const void* f, cudaFuncAttribute attr, int value) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  // the attribute holds ONE value per (kernel, device): remember the value last set, re-set on change
  using Key = std::tuple<const void*, int, int>;
  static std::mutex mu;
  static std::map<Key, int> cur;
  const Key key{f, dev, (int)attr};
  {
    std::lock_guard<std::mutex> g(mu);
    auto it = cur.find(key);
    if (it != cur.end() && it->second == value) return cudaSuccess;
  }
  e = cudaFuncSetAttribute(f, attr, value);
  if (e == cudaSuccess) {
    std::lock_guard<std::mutex> g(mu);
    cur[key] = value;
  }
  return e;
}

namespace {
std::mutex g_occ_mu;
std::map<std::tuple<const void*, int, int>, int> g_occ;
}  // namespace

bool occ_cache_get(const void* f, int param, int* out) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return false;
  std::lock_guard<std::mutex> g(g_occ_mu);
  auto it = g_occ.find(std::make_tuple(f, dev, param));
  if (it == g_occ.end()) return false;
  *out = it->second;
  return true;
}

void occ_cache_put(const void* f, int param, int value) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return;
  std::lock_guard<std::mutex> g(g_occ_mu);
  g_occ[std::make_tuple(f, dev, param)] = value;
}

int num_sms() {
  static thread_local int dev_cached = -1, sms_cached = 148;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 148;
  if (dev != dev_cached) {
    int n = 0;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && n > 0) sms_cached = n;
    dev_cached = dev;
  }
  return sms_cached;
}

int key_bits(int kind) {
  switch (kind) {
    case K_F32: return 32;
    case K_F16: return 16;
    case K_BF16: return 16;
    case K_F64: return 64;
    case K_U32: return 32;
  }
  return -1;
}

int key_bytes(int kind) { return key_bits(kind) / 8; }

int grid_vec_chunk(int kind);

// Workspace layout (all offsets 256-aligned):
//   [RowState x batch][2 histograms x 2048 counters x batch][code buffers 2 x batch x cap][index buffers]
// batched engine: samples per row = len / div (clamped to 4K..16K); env AIRTOPK_BATCH_SAMP_DIV: A/B knob
static int64_t batch_samp_div() {
  static const int64_t d = [] {
    const char* e = getenv("AIRTOPK_BATCH_SAMP_DIV");
    return (e && atoll(e) > 0) ? (int64_t)atoll(e) : (int64_t)128;
  }();
  return d;
}

Plan make_plan(const SelectArgs& a) {
  Plan p{};
  p.R = key_bits(a.kind);
  if (!a.in_idx && a.k == a.len) {
    p.engine = 3;
    return p;
  }
  if (a.engine == 4 || a.engine == 7) {  // GridSelect (the paper's second algorithm; 7: per-thread queues)
    p.engine = 4;
    p.cpr = gridselect_ctas(a);
    p.bytes = gridselect_workspace(a, p.cpr);
    return p;
  }
  p.idx64 = (a.in_idx != nullptr) || (a.len > (int64_t(1) << 32));
  p.IB = a.in_idx ? a.idx_bits : bits_needed((uint64_t)(a.len - 1));
  p.P = code_passes(p.R) + idx_passes(p.IB);
  const int64_t alpha = a.alpha > 0 ? a.alpha : 128;
  p.cap_rule = (a.len - 1) / alpha;                   // C * alpha < N  <=>  C <= (N-1)/alpha
  p.cap_alloc = (int64_t)align_up((size_t)p.cap_rule, 8);
  p.engine = 1;
  p.max_clusters = (int)std::min<int64_t>(a.batch, 2 * 148);
  const size_t isz = p.idx64 ? 8 : 4;
  const size_t csz = isz;  // histogram counter width
  p.off_state = 0;
  p.off_hist = align_up(sizeof(RowState) * (size_t)a.batch, 256);
  // fused tail (batch 1): 3 rotating histograms + per-pass buffer counts, zeroed with the state
  p.off_thist = p.off_hist + align_up((size_t)a.batch * 2 * kMaxBins * csz, 256);
  p.off_tcnt = p.off_thist + (a.batch == 1 ? align_up((size_t)3 * kMaxBins * csz, 256) : 0);
  p.off_bcode = p.off_tcnt + (a.batch == 1 ? 256 : 0);
  p.off_bidx = p.off_bcode + align_up((size_t)2 * a.batch * p.cap_alloc * key_bytes(a.kind), 256);
  // sample-guided window (grid engine, position indices): stratified samples, 4K..16K
  p.nsamp = 0;
  if (!a.in_idx && (a.window > 0 || (a.window == 0 && a.len >= (int64_t(1) << 18)))) {
    // samples are read in whole 128-byte lines (32 consecutive elements): len/64 capped at 16K
    // costs <= 1/64 of the row's bytes; at least 4K samples keep the window small vs N/alpha
    int64_t ns = std::min<int64_t>(std::max<int64_t>(a.len / 128, 4096), 16384);
    ns = std::min<int64_t>(ns, a.len / 2) / 32 * 32;
    if (key_bytes(a.kind) == 8) ns = std::min<int64_t>(ns, 8192);  // sample_kernel shared memory
    p.nsamp = ns >= 1024 ? (int)ns : 0;
  }
  p.off_samp = p.off_bidx + align_up((size_t)2 * a.batch * p.cap_alloc * isz, 256);
  p.bytes = p.off_samp + align_up((size_t)a.batch * p.nsamp * (key_bytes(a.kind) == 8 ? 8 : 4), 256);
  // batched engine (engine_batch.cuh): qualifies by shape when the window of every row is expected
  // to fit the per-row finish capacity; the fallback for missed rows uses the regions above
  p.batch_ok = 0;
  p.off_bcnt = p.off_bslot = p.off_bsidx = p.off_bfail = p.bytes;
  if (!a.in_idx && a.window >= 0 && (a.engine == 0 || a.engine == 5) && a.len >= (int64_t(1) << 14) &&
      a.len < (int64_t(1) << 31)) {
    const int es = key_bytes(a.kind), vec = 16 / es;
    int64_t ns = std::min<int64_t>(std::max<int64_t>(a.len / batch_samp_div(), 4096), 16384);
    ns = std::min<int64_t>(ns, a.len / 2) / 32 * 32;
    if (es == 8) ns = std::min<int64_t>(ns, 8192);
    const double f = (double)a.k / (double)a.len, r = f * (double)ns;
    const double rhi = std::ceil(r + 4.0 * std::sqrt(r * (1.0 - f)) + 8.0);
    const double per_row = rhi / (double)ns * (double)a.len;  // expected entries <= hi
    if (ns >= 1024 && rhi < (double)(ns - 1) && per_row <= 0.5 * kBatchFcap) {
      const int64_t chunk = kBatchStage / es;
      const double e_slot = (double)(kBatchStage / 16) * vec * rhi / (double)ns;  // expected entries per chunk
      p.batch_ok = 1;
      p.bnsamp = (int)ns;
      p.cpc = (int)((a.len + chunk - 1) / chunk);
      p.nwc = p.cpc;  // one slot per chunk (shared by the consumer group's warps)
      // the true count below hi can be ~2x the estimate (hi is a sample order statistic of rank
      // ~rhi: relative spread ~1/sqrt(rhi)), plus a 6-sigma Poisson margin per chunk; a multiple of
      // 16 entries: slots start on 32-byte sectors (the group leader pads to whole sectors)
      const double e2 = 2.0 * e_slot;
      p.scap = (int)align_up((size_t)std::ceil(e2 + 6.0 * std::sqrt(e2) + 8.0), 16);
      const size_t nslot = (size_t)a.batch * p.nwc;
      p.off_bcnt = p.bytes;
      p.off_bslot = p.off_bcnt + align_up(nslot * 2, 256);
      p.off_bsidx = p.off_bslot + align_up(nslot * p.scap * es, 256);
      p.off_bfail = p.off_bsidx + align_up(nslot * p.scap * 4, 256);
      p.bytes = p.off_bfail + align_up((size_t)(a.batch + 1) * 4, 256);
    }
  }
  return p;
}

// Engine choice: the cluster engine (one launch, DSMEM scans) for batched
// and small rows, the grid engine (one launch per pass, whole GPU per row) for long rows.
static int auto_engine(const SelectArgs& a) {
  if (a.window > 0 && !a.in_idx) return 1;  // window requested: grid window pass (+ cluster tail)
  // split-row merges of >= 2^18 gathered candidates: the grid passes (tools/merge_ab.py: 8 x 2^16
  // candidates 46 us vs 61 us in one cluster)
  if (a.in_idx && a.len >= (int64_t(1) << 18)) return 1;
  if (a.len <= (int64_t(1) << 19)) return 2;  // one launch: measured fastest from 2^17 to 2^19 keys per row
  return 1;
}

static int auto_cluster_size(const SelectArgs& a) {
  if (a.cluster_size > 0) return a.cluster_size;
  int64_t c = (a.len + 4095) / 4096;  // >= 4096 elements per CTA
  // batches: no more CTAs per row than keep every row of a wave resident (rows run concurrently)
  if (a.batch > 1) c = std::min<int64_t>(c, std::max<int64_t>(1, (int64_t)num_sms() / a.batch));
  int cs = 1;
  while (cs < 16 && cs < c) cs <<= 1;
  return cs;
}

constexpr double kTailPerCTA = 4096.0;  // expected window entries per cluster-tail CTA

static bool batch_aligned(const SelectArgs& a) {
  return ((uintptr_t)a.keys % 16) == 0 && ((size_t)a.len * key_bytes(a.kind)) % 16 == 0;
}

// Resident-cluster engine: rows held in shared memory (a cluster of CS CTAs, <= kResidentCap keys
// each). CS: enough CTAs to hold the row; for latency ~8K keys per CTA while the batch leaves SMs free.
static bool resident_fits(const SelectArgs& a) {
  const int64_t cap = key_bytes(a.kind) == 8 ? kResidentCap / 2 : kResidentCap;
  return !a.in_idx && a.len <= 16 * cap && a.len < (int64_t(1) << 31);
}

static void resident_geometry(const SelectArgs& a, Plan& p) {
  const int64_t cap = key_bytes(a.kind) == 8 ? kResidentCap / 2 : kResidentCap;
  auto pow2ceil = [](int64_t v) { int64_t c = 1; while (c < v) c <<= 1; return c; };
  const int64_t cmin = pow2ceil((a.len + cap - 1) / cap);
  int64_t clat = pow2ceil((a.len + 8191) / 8192);
  clat = std::min<int64_t>(clat, std::max<int64_t>(1, (int64_t)num_sms() / a.batch));
  int64_t cs = std::min<int64_t>(16, std::max(cmin, clat));
  if (a.cluster_size > 0) cs = std::max<int64_t>(cmin, a.cluster_size);
  p.csize = (int)cs;
  p.rslice = (int)(((a.len + cs - 1) / cs + 7) / 8 * 8);
}

static void choose_launch(const SelectArgs& a, Plan& p) {
  if (p.engine == 3 || p.engine == 4) return;  // (4: GridSelect, either queue variant)
  // AUTO (tools/engine_ab.py, profiles/r02_engine_ab.txt, L2 flushed between selects): the
  // resident cluster wins for rows of <= 2^14 keys at any batch and for a single row of <= 2^16
  if (a.engine == 6 || (a.engine == 0 && a.window == 0 && resident_fits(a) && a.trace == nullptr &&
                        (a.len <= (int64_t(1) << 14) || (a.batch == 1 && a.len <= (int64_t(1) << 16))))) {
    if (resident_fits(a)) {
      p.engine = 6;
      resident_geometry(a, p);
      return;
    }
  }
  // batched engine: explicit, or AUTO for batches with enough 64 KiB chunks to cover the SMs
  if (p.batch_ok && batch_aligned(a) && (a.trace == nullptr || a.engine == 5) &&
      (a.engine == 5 || (a.engine == 0 && a.window == 0 && a.batch >= 2 && (int64_t)a.batch * p.cpc >= num_sms()))) {
    p.engine = 5;
    p.csize = auto_cluster_size(a);  // fallback launch (cluster engine)
    p.nsamp = p.bnsamp;
    return;
  }
  p.engine = a.engine > 0 && a.engine != 5 && a.engine != 6 ? a.engine : auto_engine(a);
  if (p.engine == 2) {
    p.csize = auto_cluster_size(a);
    return;
  }
  // rows of fewer than 2^26 keys: the sample + window (+ tail) launches cost more than the second
  // read of L they save (tools/engine_ab.py: 1 x 2^22 keys 36 us without vs 51 us with the window,
  // 1 x 2^24 63 vs 73 us, 100 x 2^20 with K = 32768 334 vs 723 us); the paper's passes run instead
  if (a.window == 0 && a.engine == 0 && a.len < (int64_t(1) << 26) && !a.in_idx) p.nsamp = 0;
  // Cluster tail (one cluster-engine launch runs every pass after the window pass) for small windows:
  // opt-in only (AIRTOPK_CLUSTER_TAIL=1, A/B). Measured (tools/probe_tail.py, profiles/r02_probe_tail.txt):
  // on well-behaved rows it equals the fused cooperative tail (batch 1) or the grid passes
  // (batches), but a window that misses or is rejected restarts the row inside one cluster — a
  // constant 2^26-key row with K = 10 took 2.68 ms there vs 0.36 ms on the grid.
  p.tail = 0;
  if (p.nsamp > 0 && a.window >= 0 && getenv("AIRTOPK_CLUSTER_TAIL") != nullptr) {
    const double f = (double)a.k / (double)a.len, r = f * p.nsamp;
    const double rhi = r + 4.0 * std::sqrt(r * (1.0 - f)) + 9.0;  // sample_kernel's margin
    const double expect = rhi / p.nsamp * (double)a.len;
    if (a.engine == 0 && expect <= 16.0 * kTailPerCTA) {
      p.tail = 1;
      p.tail_q = 0;
      int cs = 1;
      while (cs < 16 && cs * kTailPerCTA < expect) cs <<= 1;
      p.csize = a.cluster_size > 0 ? a.cluster_size : cs;
    }
  }
  // batch 1 (no trace, no tail): every pass after the window pass in one cooperative launch
  // (window = -1 keeps the paper's one-kernel-per-pass structure: the P:146-156 ablations)
  p.fused = (p.engine == 1 && a.batch == 1 && !a.in_idx && (a.trace == nullptr || getenv("AIRTOPK_TAIL_STAMPS")) &&
             !p.tail && a.window >= 0 &&
             getenv("AIRTOPK_NO_FUSED") == nullptr) ? 1 : 0;
  // bulk-copy streaming for a few long rows (every SM busy with 1 CTA); register loads otherwise
  p.tma = 0;
  if (!a.in_idx && !p.idx64 && a.tma >= 0 &&
      (a.tma > 0 || (a.batch * 2 <= num_sms() && a.len >= (int64_t(1) << 22))))
    p.tma = 1;
  if (a.ctas_per_row > 0) {
    p.cpr = p.cpr_buf = a.ctas_per_row;
    return;
  }
  const int64_t target = (int64_t)num_sms() * (p.tma ? 1 : grid_blocks_per_sm(a, p.idx64));
  const int64_t chunk = grid_vec_chunk(a.kind);
  const int64_t maxc = std::max<int64_t>(1, (a.len + chunk - 1) / chunk);
  // whole waves: batch x cpr <= target CTAs (a partial second wave costs more than idle slots)
  int64_t c = std::max<int64_t>(1, target / a.batch);
  p.cpr = (int)std::max<int64_t>(1, std::min<int64_t>(c, maxc));
  // Batches whose rows do not fill the slots evenly (c2: 100 rows x 2 CTAs on 296 slots leaves some
  // SMs with half the work of others): several waves of shorter CTAs (>= 16 tiles each) balance the
  // SMs (measured on c2: 8 CTAs per row 128 us vs 2 per row 141 us).
  if (a.batch > 1 && 10 * a.batch * p.cpr < 9 * target)
    p.cpr = (int)std::max<int64_t>(p.cpr, std::min<int64_t>(maxc / 16, 4 * c));
  // After a bulk-copy window pass the next passes read the (small) window buffer: they run the
  // register-load kernel, whose 3 CTAs/SM hide the queue and load latencies (measured 2-3x faster).
  const int64_t cb = std::max<int64_t>(1, (int64_t)num_sms() * grid_blocks_per_sm(a, p.idx64) / a.batch);
  p.cpr_buf = p.tma ? (int)std::max<int64_t>(1, std::min<int64_t>(cb, maxc)) : p.cpr;
}

static bool valid_kind(int dt) { return dt >= AIRTOPK_F32 && dt <= AIRTOPK_U32; }

static airtopk_status validate(const SelectArgs& a) {
  if (!valid_kind(a.kind)) return AIRTOPK_EDTYPE;
  if (!a.keys || !a.out_vals || !a.out_idx) return AIRTOPK_EINVAL;
  if (a.batch < 1 || a.len < 1 || a.k < 1 || a.k > a.len) return AIRTOPK_EINVAL;
  if (a.alpha < 0) return AIRTOPK_EINVAL;
  if (a.engine < 0 || a.engine > 7 || a.engine == 3) return AIRTOPK_EINVAL;
  if ((a.engine == 4 || a.engine == 7) && !gridselect_supported(a)) return AIRTOPK_EINVAL;
  if (a.window < -1 || a.window > 1) return AIRTOPK_EINVAL;
  if (a.early_stop < -1 || a.early_stop > 0) return AIRTOPK_EINVAL;
  if (a.in_idx && (a.batch != 1 || a.idx_bits < 1 || a.idx_bits > 63)) return AIRTOPK_EINVAL;
  if (a.sorted < 0 || a.sorted > 1 || (a.sorted && a.k > kSortMaxK)) return AIRTOPK_EINVAL;
  return AIRTOPK_OK;
}

static airtopk_status fail_cuda(cudaError_t e) {
  g_last_cuda_error = (int)e;
  return AIRTOPK_ECUDA;
}

// NVTX range around everything one select enqueues (the paper's per-call measurement unit, P:210;
// lets nsys / ncu --nvtx delimit a select). No cost without an attached tool.
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

static airtopk_status run(const SelectArgs& a, void* ws, size_t ws_bytes, cudaStream_t s) {
  airtopk_status st = validate(a);
  if (st != AIRTOPK_OK) return st;
  NvtxRange nvtx(a.in_idx ? "airtopk_select_with_idx" : "airtopk_select");
  Plan p = make_plan(a);
  if (p.engine == 3) {
    cudaError_t e = run_trivial(a, s);
    if (e == cudaSuccess && a.sorted) e = run_sort_rows(a, s);
    return e == cudaSuccess ? AIRTOPK_OK : fail_cuda(e);
  }
  if (!ws || ws_bytes < p.bytes) return AIRTOPK_ENOSPACE;
  if (((uintptr_t)ws & 255u) != 0) return AIRTOPK_EINVAL;
  if (p.engine == 4) {
    cudaError_t e = run_gridselect(a, ws, ws_bytes, s);
    return e == cudaSuccess ? AIRTOPK_OK : fail_cuda(e);
  }
  choose_launch(a, p);
  if ((a.engine == 5 || a.engine == 6) && p.engine != a.engine) return AIRTOPK_EINVAL;  // shape not eligible
  if (p.engine == 2 && (p.csize < 1 || p.csize > 16 || (p.csize & (p.csize - 1)))) return AIRTOPK_EINVAL;
  cudaError_t e = (p.engine == 2)   ? run_cluster(a, p, ws, s)
                  : (p.engine == 5) ? run_batch(a, p, ws, s)
                  : (p.engine == 6) ? run_resident(a, p, ws, s)
                                    : run_grid(a, p, ws, s);
  if (e == cudaSuccess && a.sorted) e = run_sort_rows(a, s);
  if (e == cudaSuccess && a.status) e = collect_status(a, p, ws, s);
  return e == cudaSuccess ? AIRTOPK_OK : fail_cuda(e);
}

static SelectArgs make_args(const void* keys, int dt, int64_t batch, int64_t len, int64_t k, int select_min,
                            void* out_vals, int64_t* out_idx, const airtopk_options* opt) {
  SelectArgs a;
  a.keys = keys;
  a.kind = dt;
  a.batch = batch;
  a.len = len;
  a.k = k;
  a.sel_min = select_min ? 1 : 0;
  a.out_vals = out_vals;
  a.out_idx = out_idx;
  if (opt) {
    a.alpha = opt->alpha;
    a.engine = opt->engine;
    a.ctas_per_row = opt->ctas_per_row;
    a.cluster_size = opt->cluster_size;
    a.trace = opt->trace;
    a.trace_len = opt->trace_len;
    a.events = opt->events;
    a.n_events = opt->events ? opt->n_events : 0;
    a.window = opt->window;
    a.tma = opt->tma;
    a.early_stop = opt->early_stop;
    a.status = opt->status;
    a.sorted = opt->sorted;
  }
  if (a.alpha == 0) a.alpha = 128;
  return a;
}

static airtopk_status run_pooled(const SelectArgs& a, cudaStream_t s) {
  airtopk_status st = validate(a);
  if (st != AIRTOPK_OK) return st;
  Plan p = make_plan(a);
  void* ws = nullptr;
  if (p.engine != 3 && p.bytes) {
    cudaError_t e = cudaMallocAsync(&ws, p.bytes, s);
    if (e != cudaSuccess) return fail_cuda(e);
  }
  st = run(a, ws, p.bytes, s);
  if (ws) {
    cudaError_t e = cudaFreeAsync(ws, s);
    if (e != cudaSuccess && st == AIRTOPK_OK) st = fail_cuda(e);
  }
  return st;
}

}  // namespace airtopk

using namespace airtopk;

extern "C" {

size_t airtopk_workspace_bytes_ex(airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k,
                                  const airtopk_options* opt) {
  int64_t dummy_out = 0;
  SelectArgs a = make_args((const void*)1, (int)dtype, batch, len, k, 1, (void*)1, &dummy_out, opt);
  if (validate(a) != AIRTOPK_OK) return 0;
  Plan p = make_plan(a);
  return p.engine == 3 ? 0 : p.bytes;
}

size_t airtopk_workspace_bytes(airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k) {
  return airtopk_workspace_bytes_ex(dtype, batch, len, k, nullptr);
}

airtopk_status airtopk_select_ex(const void* keys, airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k,
                                 int select_min, void* out_vals, int64_t* out_idx, void* workspace,
                                 size_t workspace_bytes, airtopk_stream_t stream, const airtopk_options* opt) {
  SelectArgs a = make_args(keys, (int)dtype, batch, len, k, select_min, out_vals, out_idx, opt);
  return run(a, workspace, workspace_bytes, (cudaStream_t)stream);
}

airtopk_status airtopk_select(const void* keys, airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k,
                              int select_min, void* out_vals, int64_t* out_idx, void* workspace,
                              size_t workspace_bytes, airtopk_stream_t stream) {
  return airtopk_select_ex(keys, dtype, batch, len, k, select_min, out_vals, out_idx, workspace, workspace_bytes,
                           stream, nullptr);
}

#define AIRTOPK_TYPED(NAME, T, DT)                                                                        \
  airtopk_status NAME(const T* keys, int64_t batch, int64_t len, int64_t k, int select_min, T* out_vals,  \
                      int64_t* out_idx, airtopk_stream_t stream) {                                        \
    SelectArgs a = make_args(keys, DT, batch, len, k, select_min, out_vals, out_idx, nullptr);            \
    return run_pooled(a, (cudaStream_t)stream);                                                           \
  }

AIRTOPK_TYPED(airtopk_select_f32, float, AIRTOPK_F32)
AIRTOPK_TYPED(airtopk_select_f16, uint16_t, AIRTOPK_F16)
AIRTOPK_TYPED(airtopk_select_bf16, uint16_t, AIRTOPK_BF16)
AIRTOPK_TYPED(airtopk_select_f64, double, AIRTOPK_F64)
AIRTOPK_TYPED(airtopk_select_u32, uint32_t, AIRTOPK_U32)
#undef AIRTOPK_TYPED

size_t airtopk_workspace_bytes_with_idx(airtopk_dtype dtype, int64_t len, int64_t k, int idx_bits) {
  int64_t dummy = 0;
  SelectArgs a = make_args((const void*)1, (int)dtype, 1, len, k, 1, (void*)1, &dummy, nullptr);
  a.in_idx = &dummy;
  a.idx_bits = idx_bits;
  if (validate(a) != AIRTOPK_OK) return 0;
  return make_plan(a).bytes;
}

airtopk_status airtopk_select_with_idx(const void* keys, const int64_t* in_idx, int idx_bits, airtopk_dtype dtype,
                                       int64_t len, int64_t k, int select_min, void* out_vals, int64_t* out_idx,
                                       void* workspace, size_t workspace_bytes, airtopk_stream_t stream) {
  if (!in_idx) return AIRTOPK_EINVAL;
  SelectArgs a = make_args(keys, (int)dtype, 1, len, k, select_min, out_vals, out_idx, nullptr);
  a.in_idx = in_idx;
  a.idx_bits = idx_bits;
  return run(a, workspace, workspace_bytes, (cudaStream_t)stream);
}

airtopk_status airtopk_select_host(const void* h_keys, airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k,
                                   int select_min, void* h_out_vals, int64_t* h_out_idx, airtopk_stream_t stream) {
  if (!h_keys || !h_out_vals || !h_out_idx) return AIRTOPK_EINVAL;
  if (!valid_kind((int)dtype)) return AIRTOPK_EDTYPE;
  if (batch < 1 || len < 1 || k < 1 || k > len) return AIRTOPK_EINVAL;
  cudaStream_t s = (cudaStream_t)stream;
  const size_t es = key_bytes((int)dtype);
  const size_t in_b = (size_t)batch * len * es, ov_b = (size_t)batch * k * es, oi_b = (size_t)batch * k * 8;
  SelectArgs a = make_args(nullptr, (int)dtype, batch, len, k, select_min, nullptr, nullptr, nullptr);
  Plan p = make_plan(a);
  const size_t ws_b = p.engine == 3 ? 0 : p.bytes;
  const size_t o1 = align_up(in_b, 256), o2 = o1 + align_up(ov_b, 256), o3 = o2 + align_up(oi_b, 256);
  const size_t o4 = o3 + align_up(ws_b, 256);  // the device status word
  // device staging cached per thread and device (this call synchronises before returning, so the
  // next call on this thread may reuse it); grows on demand, released at thread exit
  struct Staging {
    char* ptr = nullptr;
    size_t bytes = 0;
    int dev = -1;
    ~Staging() { if (ptr) cudaFree(ptr); }
  };
  static thread_local Staging stg;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return fail_cuda(e);
  if (stg.dev != dev || stg.bytes < o4 + 256) {
    if (stg.ptr) {
      cudaStreamSynchronize(s);
      cudaFree(stg.ptr);
      stg.ptr = nullptr;
    }
    if ((e = cudaMalloc((void**)&stg.ptr, o4 + 256)) != cudaSuccess) {
      stg.bytes = 0;
      return fail_cuda(e);
    }
    stg.bytes = o4 + 256;
    stg.dev = dev;
  }
  char* d = stg.ptr;
  unsigned* dstatus = (unsigned*)(d + o4);
  airtopk_status st = AIRTOPK_OK;
  if ((e = cudaMemcpyAsync(d, h_keys, in_b, cudaMemcpyHostToDevice, s)) != cudaSuccess) st = fail_cuda(e);
  if (st == AIRTOPK_OK && (e = cudaMemsetAsync(dstatus, 0, sizeof(unsigned), s)) != cudaSuccess) st = fail_cuda(e);
  if (st == AIRTOPK_OK) {
    a.keys = d;
    a.out_vals = d + o1;
    a.out_idx = (int64_t*)(d + o2);
    a.status = dstatus;
    st = run(a, ws_b ? d + o3 : nullptr, ws_b, s);
  }
  if (st == AIRTOPK_OK && (e = cudaMemcpyAsync(h_out_vals, d + o1, ov_b, cudaMemcpyDeviceToHost, s)) != cudaSuccess)
    st = fail_cuda(e);
  if (st == AIRTOPK_OK && (e = cudaMemcpyAsync(h_out_idx, d + o2, oi_b, cudaMemcpyDeviceToHost, s)) != cudaSuccess)
    st = fail_cuda(e);
  unsigned hstatus = 0;
  if (st == AIRTOPK_OK && (e = cudaMemcpyAsync(&hstatus, dstatus, sizeof(unsigned), cudaMemcpyDeviceToHost, s)) !=
                              cudaSuccess)
    st = fail_cuda(e);
  if ((e = cudaStreamSynchronize(s)) != cudaSuccess && st == AIRTOPK_OK) st = fail_cuda(e);
  if (st == AIRTOPK_OK && hstatus != 0) st = AIRTOPK_EDEVICE;
  return st;
}

airtopk_status airtopk_select_with_idx_ex(const void* keys, const int64_t* in_idx, int idx_bits, airtopk_dtype dtype,
                                          int64_t len, int64_t k, int select_min, void* out_vals, int64_t* out_idx,
                                          void* workspace, size_t workspace_bytes, airtopk_stream_t stream,
                                          const airtopk_options* opt) {
  if (!in_idx) return AIRTOPK_EINVAL;
  SelectArgs a = make_args(keys, (int)dtype, 1, len, k, select_min, out_vals, out_idx, opt);
  if (a.engine == 4) return AIRTOPK_EINVAL;
  a.in_idx = in_idx;
  a.idx_bits = idx_bits;
  a.window = 0;
  return run(a, workspace, workspace_bytes, (cudaStream_t)stream);
}

int airtopk_merge_idx_bits(int64_t total_len, int world, int64_t k) {
  if (total_len < 1 || world < 1 || k < 1) return 0;
  // real global indices < total_len; pad indices total_len + r*k + j < total_len + world*k
  const int b = bits_needed((uint64_t)(total_len + (int64_t)world * k - 1));
  return b < 1 ? 1 : b;
}

size_t airtopk_workspace_bytes_shard(airtopk_dtype dtype, int64_t len, int64_t k) {
  if (len < 1 || k < 1) return 0;
  return airtopk_workspace_bytes(dtype, 1, len, std::min(k, len));
}

airtopk_status airtopk_select_shard(const void* keys, airtopk_dtype dtype, int64_t len, int64_t k, int select_min,
                                    int64_t shard_offset, int64_t pad_base, void* out_vals, int64_t* out_idx,
                                    void* workspace, size_t workspace_bytes, airtopk_stream_t stream) {
  if (!keys || !out_vals || !out_idx) return AIRTOPK_EINVAL;
  if (!valid_kind((int)dtype)) return AIRTOPK_EDTYPE;
  if (len < 1 || k < 1 || shard_offset < 0 || pad_base < 0) return AIRTOPK_EINVAL;
  NvtxRange nvtx("airtopk_select_shard");
  const int64_t kk = std::min(k, len);
  SelectArgs a = make_args(keys, (int)dtype, 1, len, kk, select_min, out_vals, out_idx, nullptr);
  a.idx_off = shard_offset;
  airtopk_status st = run(a, workspace, workspace_bytes, (cudaStream_t)stream);
  if (st != AIRTOPK_OK || kk == k) return st;
  cudaError_t e = run_pad(a.kind, a.sel_min, (char*)out_vals + (size_t)kk * key_bytes(a.kind), out_idx + kk, k - kk,
                          pad_base, (cudaStream_t)stream);
  return e == cudaSuccess ? AIRTOPK_OK : fail_cuda(e);
}

airtopk_status airtopk_describe(airtopk_dtype dtype, int64_t batch, int64_t len, int64_t k,
                                const airtopk_options* opt, airtopk_plan* out) {
  if (!out) return AIRTOPK_EINVAL;
  int64_t dummy = 0;
  SelectArgs a = make_args((const void*)256, (int)dtype, batch, len, k, 1, (void*)1, &dummy, opt);
  airtopk_status st = validate(a);
  if (st != AIRTOPK_OK) return st;
  Plan p = make_plan(a);
  const size_t bytes = p.engine == 3 ? 0 : p.bytes;
  choose_launch(a, p);
  std::memset(out, 0, sizeof(*out));
  out->engine = p.engine;
  out->passes = p.P;
  out->launches = (p.engine == 3 || p.engine == 4 || p.engine == 6) ? 1 : (p.engine == 2 ? 1 : p.engine == 5 ? 2
                  : p.fused ? 1 + (p.nsamp > 0 ? 2 : 0)
                  : (p.tail ? 3 + p.tail_q : p.P + 1 + (p.nsamp > 0 ? 2 : 0)));
  out->ctas_per_row = (p.engine == 1 || p.engine == 4) ? p.cpr : 0;
  out->cluster_size = (p.engine == 2 || p.engine == 5 || p.engine == 6 || p.tail) ? p.csize : 0;
  out->index_bits = p.IB;
  out->buffer_cap = p.cap_rule;
  out->workspace_bytes = bytes;
  return AIRTOPK_OK;
}

const char* airtopk_status_str(airtopk_status s) {
  switch (s) {
    case AIRTOPK_OK: return "AIRTOPK_OK: success";
    case AIRTOPK_EINVAL: return "AIRTOPK_EINVAL: invalid argument (null pointer, batch/len/k out of range, k > len)";
    case AIRTOPK_EDTYPE: return "AIRTOPK_EDTYPE: unknown dtype";
    case AIRTOPK_ENOSPACE: return "AIRTOPK_ENOSPACE: workspace too small";
    case AIRTOPK_ECUDA: return "AIRTOPK_ECUDA: CUDA error (see airtopk_last_cuda_error)";
    case AIRTOPK_EDEVICE: return "AIRTOPK_EDEVICE: the kernels detected inconsistent input (e.g. duplicate in_idx values)";
  }
  return "AIRTOPK: unknown status";
}

int airtopk_last_cuda_error(void) { return g_last_cuda_error; }

const char* airtopk_version(void) { return "0.1.0"; }

}  // extern "C"
