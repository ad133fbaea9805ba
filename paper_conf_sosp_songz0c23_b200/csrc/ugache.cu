// ugache.cu -- C ABI of libugache: context, host-table mapping, peers, fill, extract.
//
// See include/ugache.h for the contract of every entry point.  The per-batch path is
// ugache_extract -> K1 locate_bucket_kernel -> K2 factored_gather_kernel (kernels.cuh),
// two launches on the caller's stream with no host synchronisation and no collective.
#include <cuda_runtime.h>
#include <sys/mman.h>

#include <algorithm>
#include <cstddef>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "kernels.cuh"
#include "ugache_internal.h"

struct ugache_ctx {
  ugache_config cfg{};
  ugache_plan plan{};
  int device = 0;
  int sm_count = 0;
  // host table (source G)
  const uint8_t *host_table = nullptr;
  const uint8_t *host_table_dev = nullptr;
  std::vector<const void *> pinned;  // host ranges this ctx registered (refcounted globally)
  // host tier (UGACHE_FLAG_HOST_TIER): rank-ordered copy of every row, host-resident ranks
  // first (slot of rank r = (r - band_end) mod N)
  uint8_t *tier_owned = nullptr;
  size_t tier_owned_bytes = 0;
  const uint8_t *tier_dev = nullptr;
  std::vector<uint32_t> h_tier_slot;  // tier slot of every key (host-side, for refresh)
  uint32_t *d_tier_slot = nullptr;    // device copy, uploaded by the first refresh
  // this GPU's cache slab and location table
  uint8_t *slab = nullptr;
  uint64_t slab_bytes = 0;
  uint64_t n_slots = 0;
  uint64_t *d_slot_keys = nullptr;
  uint64_t slot_keys_cap = 0;
  std::vector<uint64_t> h_slot_keys;  // host copy of the slot list (refresh diffs)
  uint64_t *d_loc = nullptr;
  // cache refresh: 0 idle, 1 evicted (LT transitional), 2 content written,
  // 3 staged for the chunked protocol (ugache_refresh_chunk)
  int refresh_state = 0;
  uint64_t *d_loc_new = nullptr;
  std::vector<uint64_t> new_slot_keys;
  std::vector<uint64_t> refresh_slots;  // changed slots of this GPU, ascending
  uint64_t refresh_changed = 0, refresh_pos = 0;
  uint64_t *d_refresh = nullptr;  // changed (slot, key) lists staged for the content step
  // sources
  const uint8_t *src_base[ug::kMaxSrc] = {};
  void *ipc_mapped[UGACHE_MAX_GPUS] = {};
  bool peers_ready = false;
  bool filled = false;
  // scratch
  ugk::Ctrl *d_ctrl = nullptr;
  unsigned long long *d_timeline = nullptr;  // per-CTA role timeline (kMaxSmId x kTimelineWords)
  uint64_t *d_buckets = nullptr;
  uint64_t bucket_cap = 0;
  void *d_keys_stage = nullptr;
  size_t keys_stage_bytes = 0;
  void *d_out_stage = nullptr;
  size_t out_stage_bytes = 0;
  uint64_t *d_host_sorted = nullptr;
  uint64_t *d_queues = nullptr;  // single-pass queues, num_src x queue_cap, ~0 between launches
  uint64_t queue_cap = 0;
  uint32_t *d_qctr = nullptr;    // single-pass sub-queue counts / heads, zero between launches
  uint32_t *d_ranges = nullptr;  // 2 * kMaxRanges counters
  uint32_t range_shift = 0, n_ranges = 1;
  int host_sort = 1;
  uint32_t host_sort_min = ugk::kHostSortMin;  // max(kHostSortMin, host 2 MB pages)
  int host_dynamic = 1;  // size the host role from the host bucket when it is sparse
  int warp_dedication = 0;            // UGACHE_OPT_DEDICATION
  int wd_host_warps = 1, wd_peer_warps = 1;  // warp-granular dedication: warps per SM
  int host_rows = ugk::kRowsInFlight;        // env UGACHE_HOST_ROWS (1, 2, 4, 8)
  int host_walk = 1;                         // UGACHE_OPT_HOST_WALK
  int preorder = 1;                          // UGACHE_OPT_PREORDER (env UGACHE_PREORDER)
  int hist_smem = 1;                         // env UGACHE_HIST_SMEM (fused: per-CTA histogram)
  int host_segments = 2;                     // env UGACHE_HOST_SEGMENTS (ordered host copy)
  int locate_spread = 1;                     // env UGACHE_LOCATE_SPREAD (fused: tile size from n)
  int local_pace = 0;                        // env UGACHE_LOCAL_PACE (ns, experiment)
  int reg_kernel_ck = 8;                     // env UGACHE_REG_KERNEL_CK: keys per chunk of K3r (sparse
                                             // host, every source inline); 0 = K3's register path
  uint64_t small_batch_keys = 32768;         // env UGACHE_SMALL_BATCH: auto path reads peers inline
                                             // in the single pass up to this many keys
  uint64_t walk_keys_per_sm = 1024;          // env UGACHE_WALK_KEYS_PER_SM: a sparse host bucket is
                                             // walked only if keys <= walkers x this (else ordered)
  int local_warps = 0;                       // env UGACHE_LOCAL_WARPS (dense host: warps per SM on local rows)
  int stream_ck = 0;                         // env UGACHE_STREAM_CK (single pass: max keys per chunk)
  int sparse_host_regpath = 1;               // env UGACHE_SPARSE_HOST_REGPATH
  int fused = 2;                             // UGACHE_OPT_FUSED: 0 off, 1 on, 2 auto
  int early_walk = 0;                        // UGACHE_OPT_EARLY_WALK (env UGACHE_EARLY_WALK)
  int local_bulk = 2;                        // UGACHE_OPT_LOCAL_BULK (0 off, 1 on, 2 auto, 3)
  int stream = 2;                            // UGACHE_OPT_STREAM (0 off, 1 on, 2 auto)
  int inline_mask = UGACHE_INLINE_HOST;      // UGACHE_OPT_INLINE
  int stream_k = 1, stream_host_last = 0, stream_host_cap = 0, stream_static = 1, stream_nap = 100,
      stream_prefetch = 0, stream_coop = 0, stream_regstore = 0,
      stream_peer_warps = ugk::kGatherWarps, local_sms = 0, stream_group = 0;  // single-pass env knobs
  int host_warps = ugk::kHostWarps;  // env UGACHE_HOST_WARPS (A0 calibration knob)
  int stage_host_io = 0;             // env UGACHE_STAGE_HOST_IO=1: stage pinned host I/O too
  std::vector<int> smids;  // sorted %smid values of the device (one per SM)
  // dedication / mode
  int host_sms = 0, peer_sms = 0;
  int mode = UGACHE_MODE_FACTORED;
  // timing
  bool timing = false;
  bool timing_valid = false;
  bool last_fused = false;  // last timed extract ran K1+K2 as one launch
  bool last_single_pass = false;  // last timed extract ran the single pass (K3)
  uint32_t *h_mirror = nullptr;  // pinned {n, host count, launches} of the last launch (Ctrl)
  cudaEvent_t ev[3] = {};
  int last_launches = 0;
  // message-based baseline: 0 idle, 1 local part done (buckets valid), 2 requests packed
  int msg_state = 0;
  uint64_t msg_counts[ug::kMaxSrc] = {};
  void *msg_out = nullptr;
  uint64_t last_n = 0;
  cudaStream_t last_stream = nullptr;
  std::string err;
};

namespace {

// Dynamic shared memory requested only to guarantee one gather CTA per SM, so that the
// CTA index -> role mapping is also an SM -> role mapping (P:1620-1627 used MPS for this).
constexpr size_t kOneCtaPerSmSmem = ugk::kGatherSmem;
// UGACHE_OPT_FUSED = auto: batches up to this many keys run K1 + K2 in one launch.
constexpr uint64_t kFusedAutoMaxKeys = 1u << 20;
// UGACHE_OPT_STREAM = auto: the single pass only for rows up to this size.
constexpr uint32_t kStreamAutoMaxRow = 1024;

std::mutex g_reg_mu;
std::map<const void *, int> g_reg_count;  // host-table registrations owned by this library

ugache_status cuda_fail(ugache_ctx *ctx, cudaError_t e, const char *what) {
  if (ctx) {
    char buf[512];
    snprintf(buf, sizeof(buf), "%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
    ctx->err = buf;
  }
  (void)cudaGetLastError();
  return e == cudaErrorMemoryAllocation ? UGACHE_ENOMEM : UGACHE_ECUDA;
}

#define UG_CUDA(ctx, call)                                  \
  do {                                                      \
    cudaError_t _e = (call);                                \
    if (_e != cudaSuccess) return cuda_fail(ctx, _e, #call); \
  } while (0)

ugache_status fail(ugache_ctx *ctx, ugache_status st, const char *msg) {
  if (ctx) ctx->err = msg;
  return st;
}

bool is_device_pointer(const void *p, int *device) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    (void)cudaGetLastError();
    return false;
  }
  if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) {
    if (device) *device = a.device;
    return true;
  }
  return false;
}

enum class MemKind { kDevice, kPinned, kPageable };

// Where a caller buffer lives; for pinned host memory also its device-mapped address.
MemKind mem_kind(const void *p, void **mapped) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    (void)cudaGetLastError();
    return MemKind::kPageable;
  }
  if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) return MemKind::kDevice;
  if (a.type == cudaMemoryTypeHost && a.devicePointer) {
    *mapped = a.devicePointer;
    return MemKind::kPinned;
  }
  return MemKind::kPageable;
}

bool is_pinned_host(const void *p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    (void)cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeHost;
}

// Page-lock and map a host range (refcounted per address across contexts of the process)
// and return its device address.  Already-pinned memory is used as is.
ugache_status pin_host(ugache_ctx *ctx, const void *p, size_t bytes, const uint8_t **dev) {
  {
    std::lock_guard<std::mutex> lk(g_reg_mu);
    auto it = g_reg_count.find(p);
    if (it != g_reg_count.end()) {
      it->second++;
      ctx->pinned.push_back(p);
    } else if (!is_pinned_host(p)) {
      cudaError_t e = cudaHostRegister(const_cast<void *>(p), bytes,
                                       cudaHostRegisterMapped | cudaHostRegisterPortable |
                                           cudaHostRegisterReadOnly);
      if (e != cudaSuccess) {
        (void)cudaGetLastError();
        e = cudaHostRegister(const_cast<void *>(p), bytes,
                             cudaHostRegisterMapped | cudaHostRegisterPortable);
      }
      if (e != cudaSuccess) return cuda_fail(ctx, e, "cudaHostRegister");
      g_reg_count[p] = 1;
      ctx->pinned.push_back(p);
    }
  }
  void *dptr = nullptr;
  UG_CUDA(ctx, cudaHostGetDevicePointer(&dptr, const_cast<void *>(p), 0));
  *dev = static_cast<const uint8_t *>(dptr);
  return UGACHE_OK;
}

void unpin_all(ugache_ctx *ctx) {
  std::lock_guard<std::mutex> lk(g_reg_mu);
  for (const void *p : ctx->pinned) {
    auto it = g_reg_count.find(p);
    if (it != g_reg_count.end() && --it->second == 0) {
      cudaHostUnregister(const_cast<void *>(p));
      (void)cudaGetLastError();
      g_reg_count.erase(it);
    }
  }
  ctx->pinned.clear();
}

// Scratch of the extract kernels.  The queue sentinels (~0) and sub-queue counters (0) are
// initialised on the extract stream itself: a caller's non-blocking stream is not ordered
// after the legacy default stream, so a plain cudaMemset could land after the first launch.
ugache_status ensure_scratch(ugache_ctx *ctx, uint64_t n, cudaStream_t s) {
  if (n <= ctx->bucket_cap) return UGACHE_OK;
  uint64_t cap = std::max<uint64_t>(n, 1024);
  if (ctx->d_buckets) {
    UG_CUDA(ctx, cudaDeviceSynchronize());
    cudaFree(ctx->d_buckets);
    ctx->d_buckets = nullptr;
    ctx->bucket_cap = 0;
  }
  if (ctx->d_host_sorted) {
    cudaFree(ctx->d_host_sorted);
    ctx->d_host_sorted = nullptr;
  }
  if (ctx->d_queues) {
    cudaFree(ctx->d_queues);
    ctx->d_queues = nullptr;
  }
  const size_t bytes = (size_t)(ctx->cfg.num_gpus + 1) * cap * sizeof(uint64_t);
  UG_CUDA(ctx, cudaMalloc(&ctx->d_buckets, bytes));
  // sub-queues round each one up to whole chunks: room for one extra chunk per sub-queue
  ctx->queue_cap = cap + (uint64_t)(ctx->sm_count + 1) * ugk::kStreamChunk;
  const size_t qbytes = (size_t)(ctx->cfg.num_gpus + 1) * ctx->queue_cap * sizeof(uint64_t);
  UG_CUDA(ctx, cudaMalloc(&ctx->d_queues, qbytes));
  UG_CUDA(ctx, cudaMemsetAsync(ctx->d_queues, 0xFF, qbytes, s));
  if (!ctx->d_qctr) {
    const size_t cb = 2 * (size_t)ugk::kMaxSrc * ugk::kMaxSmId * sizeof(uint32_t);
    UG_CUDA(ctx, cudaMalloc(&ctx->d_qctr, cb));
    UG_CUDA(ctx, cudaMemsetAsync(ctx->d_qctr, 0, cb, s));
  }
  UG_CUDA(ctx, cudaMalloc(&ctx->d_host_sorted, cap * sizeof(uint64_t)));
  ctx->bucket_cap = cap;
  return UGACHE_OK;
}

ugache_status ensure_stage(ugache_ctx *ctx, void **buf, size_t *have, size_t need) {
  if (need <= *have) return UGACHE_OK;
  if (*buf) {
    UG_CUDA(ctx, cudaDeviceSynchronize());
    cudaFree(*buf);
    *buf = nullptr;
    *have = 0;
  }
  UG_CUDA(ctx, cudaMalloc(buf, need));
  *have = need;
  return UGACHE_OK;
}

// Core-dedication inputs of the gather kernel.  The roles themselves are
// resolved on the device from the per-source counts: positions [0, H) of the SM order are
// host SMs, then peer_sms positions per peer, then local.  The SM order is a stride
// permutation of the sorted SM ids, so every role is spread over the whole chip (all GPCs,
// both dies) -- on the B200 box the host source's zero-copy throughput scales with the
// number of GPCs issuing requests.
void build_roles(const ugache_ctx *ctx, ugk::GatherParams *gp, int *grid) {
  const int G = ctx->cfg.num_gpus, me = ctx->cfg.rank;
  const int S = (int)ctx->smids.size();
  gp->num_sms = S;
  gp->host_sms = ctx->host_sms;
  gp->peer_sms = G > 1 ? ctx->peer_sms : 0;
  gp->n_peers = 0;
  for (int j = 0; j < G; ++j)
    if (j != me) gp->peer_src[gp->n_peers++] = j;
  gp->host_sms_max = ctx->host_dynamic ? std::max(ctx->host_sms, S - gp->n_peers * gp->peer_sms)
                                       : ctx->host_sms;
  gp->host_sort_min = ctx->host_sort_min;
  gp->host_dense_min = ctx->host_sort_min;
  gp->warp_dedication = ctx->warp_dedication;
  gp->host_rows = ctx->host_rows;
  gp->peer_warps = ctx->wd_peer_warps;
  gp->host_warps = ctx->warp_dedication ? ctx->wd_host_warps : ctx->host_warps;
  memset(gp->sm_pos, S - 1, sizeof(gp->sm_pos));
  int stride = (int)(S * 0.6180339887) | 1;
  while (std::__gcd(stride, S) != 1) stride += 2;
  for (int pos = 0; pos < S; ++pos)
    gp->sm_pos[ctx->smids[(size_t)((int64_t)pos * stride % S)]] = (uint8_t)pos;
  *grid = S;
}

// Caller-provided placement (ugache_init_with_placement): checks that this GPU's table
// resolves every key to a valid source / row and that its own slots hold the keys that map
// to them (peer slots are the peers' business; the placement checker covers them).
ugache_status check_given_placement(ugache_ctx *ctx, const ugache_config *cfg, const uint64_t *loc,
                                    const uint64_t *slots, uint64_t n_slots) {
  const uint64_t N = cfg->num_rows, C = cfg->capacity_rows;
  const int G = cfg->num_gpus, me = cfg->rank;
  if (n_slots > C || (n_slots && !slots)) return fail(ctx, UGACHE_EINVAL, "slot list exceeds capacity");
  for (uint64_t s = 0; s < n_slots; ++s)
    if (slots[s] >= N) return fail(ctx, UGACHE_EINVAL, "slot key out of range");
  bool ok = true;
#pragma omp parallel for reduction(&& : ok)
  for (int64_t k = 0; k < (int64_t)N; ++k) {
    const uint64_t src = loc[k] >> UGACHE_LOC_SRC_SHIFT, row = loc[k] & UGACHE_LOC_ROW_MASK;
    bool good = src <= (uint64_t)G;
    if (good && src == (uint64_t)G) good = row == (uint64_t)k;
    if (good && src == (uint64_t)me) good = row < n_slots && slots[row] == (uint64_t)k;
    if (good && src < (uint64_t)G) good = row < C;
    ok = ok && good;
  }
  return ok ? UGACHE_OK : fail(ctx, UGACHE_EINVAL, "location table does not resolve every key");
}

// MemAvailable of /proc/meminfo in bytes (0 if unknown).
uint64_t host_mem_available() {
  FILE *f = fopen("/proc/meminfo", "r");
  if (!f) return 0;
  char line[256];
  uint64_t kb = 0;
  while (fgets(line, sizeof(line), f))
    if (sscanf(line, "MemAvailable: %lu kB", &kb) == 1) break;
  fclose(f);
  return kb * 1024;
}

ugache_status init_common(ugache_ctx *ctx, const ugache_config *cfg, const void *host_table,
                          const std::vector<uint32_t> &order, const void *host_tier,
                          const uint64_t *given_loc = nullptr, const uint64_t *given_slots = nullptr,
                          uint64_t given_n = 0) {
  const uint64_t N = cfg->num_rows, R = cfg->row_bytes;
  const int G = cfg->num_gpus;
  ugache_status st = pin_host(ctx, host_table, (size_t)(N * R), &ctx->host_table_dev);
  if (st != UGACHE_OK) return st;
  ctx->host_table = static_cast<const uint8_t *>(host_table);
  const uint64_t tier_rows = N;  // every row (a refresh may send any key to the host)
  if (cfg->flags & UGACHE_FLAG_HOST_TIER) {
    const void *tier = host_tier;
    if (!tier) {  // build this ctx's own rank-ordered host tier
      const uint64_t avail = host_mem_available();
      if (avail && tier_rows * R > avail / 10 * 9)
        return fail(ctx, UGACHE_ENOMEM, "the host tier (another copy of every row) does not fit host RAM");
      ctx->tier_owned_bytes = (size_t)(tier_rows * R);
      void *m = mmap(nullptr, ctx->tier_owned_bytes, PROT_READ | PROT_WRITE,
                     MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
      if (m == MAP_FAILED) {
        ctx->tier_owned_bytes = 0;
        return fail(ctx, UGACHE_ENOMEM, "mmap of the host tier failed");
      }
      madvise(m, ctx->tier_owned_bytes, MADV_HUGEPAGE);
      ctx->tier_owned = static_cast<uint8_t *>(m);
      ug::fill_host_tier(static_cast<const uint8_t *>(host_table), (uint32_t)R, order.data(),
                         ctx->plan.band_end, N, ctx->tier_owned);
      tier = ctx->tier_owned;
    }
    st = pin_host(ctx, tier, (size_t)(tier_rows * R), &ctx->tier_dev);
    if (st != UGACHE_OK) return st;
    try {
      ctx->h_tier_slot.resize(N);
    } catch (const std::bad_alloc &) {
      return fail(ctx, UGACHE_ENOMEM, "host allocation of the tier slot map failed");
    }
    const uint64_t be = ctx->plan.band_end;
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < (int64_t)N; ++r)
      ctx->h_tier_slot[order[r]] = (uint32_t)(((uint64_t)r + N - be) % N);
  }

  // location table and slot list of this rank
  std::vector<uint64_t> loc;
  std::vector<uint64_t> slots;
  try {
    loc.resize(N);
    slots.resize(std::max<uint64_t>(ctx->plan.capacity_rows, 1));
  } catch (const std::bad_alloc &) {
    return fail(ctx, UGACHE_ENOMEM, "host allocation of the location table failed");
  }
  if (given_loc) {
    st = check_given_placement(ctx, cfg, given_loc, given_slots, given_n);
    if (st != UGACHE_OK) return st;
    std::memcpy(loc.data(), given_loc, N * sizeof(uint64_t));
    if (given_n) std::memcpy(slots.data(), given_slots, given_n * sizeof(uint64_t));
    ctx->n_slots = given_n;
  } else {
    st = ug::build_placement(cfg, order.data(), &ctx->plan, cfg->rank, loc.data(), slots.data(),
                             &ctx->n_slots);
    if (st != UGACHE_OK) return fail(ctx, st, "build_placement failed");
  }

  ctx->slab_bytes = std::max<uint64_t>(ctx->plan.capacity_rows, 1) * R;
  UG_CUDA(ctx, cudaMalloc(&ctx->slab, ctx->slab_bytes));
  UG_CUDA(ctx, cudaMalloc(&ctx->d_loc, N * sizeof(uint64_t)));
  UG_CUDA(ctx, cudaMemcpy(ctx->d_loc, loc.data(), N * sizeof(uint64_t), cudaMemcpyHostToDevice));
  if (ctx->n_slots) {
    UG_CUDA(ctx, cudaMalloc(&ctx->d_slot_keys, ctx->n_slots * sizeof(uint64_t)));
    UG_CUDA(ctx, cudaMemcpy(ctx->d_slot_keys, slots.data(), ctx->n_slots * sizeof(uint64_t),
                            cudaMemcpyHostToDevice));
    ctx->slot_keys_cap = ctx->n_slots;
  }
  ctx->h_slot_keys.assign(slots.begin(), slots.begin() + (ptrdiff_t)ctx->n_slots);
  UG_CUDA(ctx, cudaMalloc(&ctx->d_ctrl, sizeof(ugk::Ctrl)));
  UG_CUDA(ctx, cudaMemset(ctx->d_ctrl, 0, sizeof(ugk::Ctrl)));
  UG_CUDA(ctx, cudaMalloc(&ctx->d_timeline, ugk::kMaxSmId * ugk::kTimelineWords * sizeof(unsigned long long)));
  {  // pinned mirror of the last launch's {n, host count, launches} (path choice, K3)
    UG_CUDA(ctx, cudaHostAlloc(reinterpret_cast<void **>(&ctx->h_mirror), 4 * sizeof(uint32_t),
                               cudaHostAllocMapped));
    std::memset(ctx->h_mirror, 0, 4 * sizeof(uint32_t));
    void *dm = nullptr;
    UG_CUDA(ctx, cudaHostGetDevicePointer(&dm, ctx->h_mirror, 0));
    UG_CUDA(ctx, cudaMemcpy(reinterpret_cast<uint8_t *>(ctx->d_ctrl) + offsetof(ugk::Ctrl, host_mirror), &dm,
                            sizeof(dm), cudaMemcpyHostToDevice));
  }
  UG_CUDA(ctx, cudaMalloc(&ctx->d_ranges, 2 * ugk::kMaxRanges * sizeof(uint32_t)));
  UG_CUDA(ctx, cudaMemset(ctx->d_ranges, 0, 2 * ugk::kMaxRanges * sizeof(uint32_t)));
  // host key ranges: the smallest power-of-two rows per range giving <= kMaxRanges ranges
  // over the host source's rows (the tier's slots when it is on, else the table's keys)
  {
    const uint64_t hr = std::max<uint64_t>(N, 1);
    ctx->range_shift = 0;
    while (((hr - 1) >> ctx->range_shift) + 1 > (uint64_t)ugk::kMaxRanges) ++ctx->range_shift;
    ctx->n_ranges = (uint32_t)(((hr - 1) >> ctx->range_shift) + 1);
  }
  {  // ordering pays once host rows share translation pages: >= 1 key per 2 MB of host source
    const uint64_t host_rows = ctx->tier_dev ? N - ctx->plan.band_end : N;
    const uint64_t pages = (host_rows * R) >> 21;
    ctx->host_sort_min = (uint32_t)std::min<uint64_t>(std::max<uint64_t>(ugk::kHostSortMin, pages),
                                                      0xFFFFFFFFull);
  }
  if (const char *e = getenv("UGACHE_HOST_SORT_MIN")) ctx->host_sort_min = (uint32_t)atoll(e);
  if (const char *e = getenv("UGACHE_HOST_DYNAMIC")) ctx->host_dynamic = atoi(e) != 0;
  if (const char *e = getenv("UGACHE_HOST_ROWS")) ctx->host_rows = atoi(e);
  if (const char *e = getenv("UGACHE_EARLY_WALK")) ctx->early_walk = atoi(e) != 0;
  if (const char *e = getenv("UGACHE_PREORDER")) ctx->preorder = atoi(e) != 0;

  if (const char *e = getenv("UGACHE_HIST_SMEM")) ctx->hist_smem = atoi(e) != 0;
  if (const char *e = getenv("UGACHE_LOCATE_SPREAD")) ctx->locate_spread = atoi(e) != 0;
  if (const char *e = getenv("UGACHE_LOCAL_PACE")) ctx->local_pace = std::max(0, std::min(1000000, atoi(e)));
  if (const char *e = getenv("UGACHE_LOCAL_WARPS")) ctx->local_warps = std::max(0, std::min(ugk::kGatherWarps, atoi(e)));
  if (const char *e = getenv("UGACHE_SPARSE_HOST_REGPATH")) ctx->sparse_host_regpath = atoi(e) != 0;
  if (const char *e = getenv("UGACHE_STREAM_CK")) {
    int v = atoi(e), ck = 4;
    while (ck < v && ck < 32) ck <<= 1;
    ctx->stream_ck = v > 0 ? ck : 0;
  }
  if (const char *e = getenv("UGACHE_HOST_SEGMENTS")) ctx->host_segments = std::max(1, std::min(8, atoi(e)));
  if (const char *e = getenv("UGACHE_LOCAL_BULK")) ctx->local_bulk = std::max(0, std::min(3, atoi(e)));
  if (const char *e = getenv("UGACHE_STAGE_HOST_IO")) ctx->stage_host_io = atoi(e) != 0;
  if (const char *e = getenv("UGACHE_STREAM_K")) ctx->stream_k = std::max(1, std::min(ugk::kStreamK, atoi(e)));
  if (const char *e = getenv("UGACHE_STREAM_HOST_LAST")) ctx->stream_host_last = atoi(e) != 0;
  {  // row payload L2 policy (kernels.cuh c_row_evict_first), per device
    int ef = 0;
    if (const char *e = getenv("UGACHE_ROW_EVICT_FIRST")) ef = atoi(e) != 0;
    UG_CUDA(ctx, cudaMemcpyToSymbol(ugk::c_row_evict_first, &ef, sizeof(ef)));
    int lf = 1;
    if (const char *e = getenv("UGACHE_LT_EVICT_FIRST")) lf = atoi(e) != 0;
    UG_CUDA(ctx, cudaMemcpyToSymbol(ugk::c_lt_evict_first, &lf, sizeof(lf)));
  }
  if (const char *e = getenv("UGACHE_INLINE")) ctx->inline_mask = atoi(e) & (UGACHE_INLINE_HOST | UGACHE_INLINE_PEERS);
  if (const char *e = getenv("UGACHE_REG_KERNEL_CK")) {
    const int v = atoi(e);
    ctx->reg_kernel_ck = v <= 0 ? 0 : v <= 4 ? 4 : v <= 8 ? 8 : v <= 16 ? 16 : 32;
  }
  if (const char *e = getenv("UGACHE_SMALL_BATCH")) ctx->small_batch_keys = strtoull(e, nullptr, 10);
  if (const char *e = getenv("UGACHE_WALK_KEYS_PER_SM")) ctx->walk_keys_per_sm = strtoull(e, nullptr, 10);
  if (const char *e = getenv("UGACHE_STREAM_GROUP"))
    ctx->stream_group = std::max(0, std::min(ugk::kStreamGroupMax, atoi(e)));
  if (const char *e = getenv("UGACHE_LOCAL_SMS")) ctx->local_sms = std::max(0, atoi(e));
  if (const char *e = getenv("UGACHE_STREAM_PEER_WARPS"))
    ctx->stream_peer_warps = std::max(1, std::min(ugk::kGatherWarps, atoi(e)));
  if (const char *e = getenv("UGACHE_STREAM_REGSTORE")) ctx->stream_regstore = atoi(e) != 0;
  if (const char *e = getenv("UGACHE_STREAM_COOP")) ctx->stream_coop = atoi(e) != 0;
  if (const char *e = getenv("UGACHE_STREAM_PREFETCH")) ctx->stream_prefetch = atoi(e);
  if (const char *e = getenv("UGACHE_STREAM_NAP")) ctx->stream_nap = std::max(0, atoi(e));
  if (const char *e = getenv("UGACHE_STREAM_STATIC")) ctx->stream_static = std::max(0, atoi(e));
  if (const char *e = getenv("UGACHE_STREAM_HOST_CAP")) ctx->stream_host_cap = std::max(0, atoi(e));
  if (const char *e = getenv("UGACHE_STREAM")) ctx->stream = std::max(0, std::min(2, atoi(e)));
  if (const char *e = getenv("UGACHE_HOST_WARPS")) ctx->host_warps = std::max(1, std::min(ugk::kGatherWarps, atoi(e)));
  for (int i = 0; i < 3; ++i) UG_CUDA(ctx, cudaEventCreate(&ctx->ev[i]));
  ctx->src_base[cfg->rank] = ctx->slab;
  ctx->src_base[G] = ctx->tier_dev ? ctx->tier_dev : ctx->host_table_dev;
  ctx->peers_ready = (G == 1);
  ctx->host_sms = ctx->plan.host_sms;
  ctx->peer_sms = ctx->plan.peer_sms;
  {  // SM ids of this device (role table index)
    uint32_t *d_ids = nullptr;
    UG_CUDA(ctx, cudaMalloc(&d_ids, ctx->sm_count * sizeof(uint32_t)));
    UG_CUDA(ctx, cudaFuncSetAttribute(ugk::smid_probe_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)kOneCtaPerSmSmem));
    void *args[] = {&d_ids};
    cudaError_t e = cudaLaunchCooperativeKernel((const void *)ugk::smid_probe_kernel, dim3(ctx->sm_count),
                                                dim3(32), args, kOneCtaPerSmSmem, nullptr);
    std::vector<uint32_t> ids(ctx->sm_count);
    if (e == cudaSuccess) e = cudaMemcpy(ids.data(), d_ids, ids.size() * 4, cudaMemcpyDeviceToHost);
    cudaFree(d_ids);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "smid probe");
    std::sort(ids.begin(), ids.end());
    for (size_t i = 0; i < ids.size(); ++i) {
      if (ids[i] >= (uint32_t)ugk::kMaxSmId || (i && ids[i] == ids[i - 1]))
        return fail(ctx, UGACHE_ECUDA, "unexpected %smid layout");
      ctx->smids.push_back((int)ids[i]);
    }
  }
  UG_CUDA(ctx, cudaFuncSetAttribute(ugk::factored_gather_kernel,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kOneCtaPerSmSmem));
  UG_CUDA(ctx, cudaFuncSetAttribute(ugk::fused_extract_kernel<int64_t>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kOneCtaPerSmSmem));
  UG_CUDA(ctx, cudaFuncSetAttribute(ugk::fused_extract_kernel<uint32_t>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kOneCtaPerSmSmem));
  UG_CUDA(ctx, cudaFuncSetAttribute(ugk::stream_extract_kernel<int64_t>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kOneCtaPerSmSmem));
  UG_CUDA(ctx, cudaFuncSetAttribute(ugk::stream_extract_kernel<uint32_t>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kOneCtaPerSmSmem));
  UG_CUDA(ctx, cudaFuncSetAttribute(ugk::random_dispatch_kernel<int64_t>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kOneCtaPerSmSmem));
  UG_CUDA(ctx, cudaFuncSetAttribute(ugk::random_dispatch_kernel<uint32_t>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kOneCtaPerSmSmem));
  return UGACHE_OK;
}

ugache_status begin(ugache_ctx *ctx) {
  UG_CUDA(ctx, cudaSetDevice(ctx->device));
  return UGACHE_OK;
}

}  // namespace

extern "C" {

int32_t ugache_version(void) { return UGACHE_VERSION; }

const char *ugache_error_string(ugache_status st) {
  switch (st) {
    case UGACHE_OK: return "ok";
    case UGACHE_EINVAL: return "invalid argument";
    case UGACHE_ECUDA: return "CUDA error";
    case UGACHE_ENOMEM: return "out of memory";
    case UGACHE_ESTATE: return "invalid call order";
    case UGACHE_EPEER: return "peer mapping failed";
    case UGACHE_EKEY: return "key out of range";
  }
  return "unknown status";
}

namespace {
thread_local std::string g_init_err;  // detail of this thread's last failed init
}

const char *ugache_last_error_message(const ugache_ctx *ctx) {
  return ctx ? ctx->err.c_str() : g_init_err.c_str();
}

static ugache_status init_impl(ugache_ctx **out, const ugache_config *cfg, const void *host_table,
                               const float *hotness, const uint64_t *order_in,
                               const ugache_plan *plan_in, const void *host_tier,
                               const uint64_t *given_loc = nullptr,
                               const uint64_t *given_slots = nullptr, uint64_t given_n = 0) {
  if (!out || !cfg || !host_table) return UGACHE_EINVAL;
  *out = nullptr;
  // rows are read with 16-byte vector loads and cp.async.bulk: 16-byte aligned sources only
  if (reinterpret_cast<uintptr_t>(host_table) % 16 || reinterpret_cast<uintptr_t>(host_tier) % 16)
    return UGACHE_EINVAL;
  if (cfg->rank < 0 || cfg->rank >= cfg->num_gpus) return UGACHE_EINVAL;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev <= 0) {
    (void)cudaGetLastError();
    return UGACHE_ECUDA;
  }
  if (cfg->device < 0 || cfg->device >= ndev) return UGACHE_EINVAL;
  ugache_ctx *ctx = new (std::nothrow) ugache_ctx();
  if (!ctx) return UGACHE_ENOMEM;
  ctx->cfg = *cfg;
  ctx->device = cfg->device;
  ugache_status st = begin(ctx);
  if (st == UGACHE_OK) {
    cudaError_t e = cudaDeviceGetAttribute(&ctx->sm_count, cudaDevAttrMultiProcessorCount, ctx->device);
    if (e != cudaSuccess) st = cuda_fail(ctx, e, "cudaDeviceGetAttribute");
  }
  std::vector<uint32_t> order;
  if (st == UGACHE_OK && given_loc) {  // caller-provided placement: no solve
    ug::Params p;
    st = ug::resolve_params(cfg, ctx->sm_count, &p);
    if (st == UGACHE_OK && (cfg->flags & UGACHE_FLAG_HOST_TIER)) st = UGACHE_EINVAL;
    if (st == UGACHE_OK) {
      ugache_plan &pl = ctx->plan;
      std::memset(&pl, 0, sizeof(pl));
      pl.policy = -1;
      pl.num_gpus = cfg->num_gpus;
      pl.capacity_rows = std::min<uint64_t>(cfg->capacity_rows, cfg->num_rows);
      pl.band_end = cfg->num_rows;  // no host tier
      pl.T_local = p.T_L, pl.T_peer = p.T_P, pl.T_host = p.T_H;
      pl.R_local = p.R_L, pl.R_peer = p.R_P, pl.R_host = p.R_H;
      pl.host_sms = p.host_sms, pl.peer_sms = p.peer_sms, pl.num_sms = p.S;
    }
  } else if (st == UGACHE_OK) {
    if (order_in && plan_in) {
      ug::Params p;
      st = ug::resolve_params(cfg, ctx->sm_count, &p);
      if (st == UGACHE_OK) {
        // order must be a permutation of [0, N): a key missing from it would keep a host
        // location whose tier slot lies outside the tier
        order.resize(cfg->num_rows);
        std::vector<uint8_t> seen(cfg->num_rows, 0);
        for (uint64_t i = 0; i < cfg->num_rows; ++i) {
          if (order_in[i] >= cfg->num_rows || seen[order_in[i]]) { st = UGACHE_EINVAL; break; }
          seen[order_in[i]] = 1;
          order[i] = (uint32_t)order_in[i];
        }
        ctx->plan = *plan_in;
        if (plan_in->num_gpus != cfg->num_gpus || plan_in->host_sms != p.host_sms ||
            plan_in->peer_sms != p.peer_sms)
          st = UGACHE_EINVAL;
        const uint64_t cap = std::min<uint64_t>(cfg->capacity_rows, cfg->num_rows);
        if (plan_in->capacity_rows > cap || plan_in->k > plan_in->capacity_rows ||
            plan_in->band_end < plan_in->k || plan_in->band_end > cfg->num_rows)
          st = UGACHE_EINVAL;
        if (plan_in->num_sms > ctx->sm_count) st = UGACHE_EINVAL;
      }
    } else {
      st = ug::solve(cfg, ctx->sm_count, hotness, order, &ctx->plan);
    }
    if (st == UGACHE_OK && ctx->plan.num_sms > ctx->sm_count) st = UGACHE_EINVAL;
  }
  if (st == UGACHE_OK)
    st = init_common(ctx, cfg, host_table, order, host_tier, given_loc, given_slots, given_n);
  if (st != UGACHE_OK) {
    g_init_err = ctx->err;
    ugache_destroy(ctx);
    return st;
  }
  *out = ctx;
  return UGACHE_OK;
}

ugache_status ugache_init(ugache_ctx **ctx, const ugache_config *cfg, const void *host_table,
                          const float *hotness) {
  return init_impl(ctx, cfg, host_table, hotness, nullptr, nullptr, nullptr);
}

ugache_status ugache_init_with_plan(ugache_ctx **ctx, const ugache_config *cfg,
                                    const void *host_table, const uint64_t *order,
                                    const ugache_plan *plan, const void *host_tier) {
  if (!order || !plan) return UGACHE_EINVAL;
  return init_impl(ctx, cfg, host_table, nullptr, order, plan, host_tier);
}

ugache_status ugache_init_with_placement(ugache_ctx **ctx, const ugache_config *cfg,
                                         const void *host_table, const uint64_t *loc,
                                         const uint64_t *slot_keys, uint64_t n_slots) {
  if (!loc) return UGACHE_EINVAL;
  return init_impl(ctx, cfg, host_table, nullptr, nullptr, nullptr, nullptr, loc, slot_keys, n_slots);
}

ugache_status ugache_get_plan(const ugache_ctx *ctx, ugache_plan *plan) {
  if (!ctx || !plan) return UGACHE_EINVAL;
  *plan = ctx->plan;
  return UGACHE_OK;
}

ugache_status ugache_slab(const ugache_ctx *ctx, void **dev_ptr, uint64_t *bytes, uint64_t *n_slots) {
  if (!ctx) return UGACHE_EINVAL;
  if (dev_ptr) *dev_ptr = ctx->slab;
  if (bytes) *bytes = ctx->slab_bytes;
  if (n_slots) *n_slots = ctx->n_slots;
  return UGACHE_OK;
}

ugache_status ugache_ipc_handle(ugache_ctx *ctx, void *buf, size_t *len) {
  if (!ctx || !buf || !len) return UGACHE_EINVAL;
  if (*len < sizeof(cudaIpcMemHandle_t)) return UGACHE_EINVAL;
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  cudaIpcMemHandle_t h;
  UG_CUDA(ctx, cudaIpcGetMemHandle(&h, ctx->slab));
  memcpy(buf, &h, sizeof(h));
  *len = sizeof(h);
  return UGACHE_OK;
}

ugache_status ugache_open_peers(ugache_ctx *ctx, const void *all_handles, size_t len_each) {
  if (!ctx || !all_handles || len_each < sizeof(cudaIpcMemHandle_t)) return UGACHE_EINVAL;
  if (ctx->peers_ready && ctx->cfg.num_gpus > 1) return fail(ctx, UGACHE_ESTATE, "peers already set");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  const uint8_t *hb = static_cast<const uint8_t *>(all_handles);
  for (int j = 0; j < ctx->cfg.num_gpus; ++j) {
    if (j == ctx->cfg.rank) continue;
    cudaIpcMemHandle_t h;
    memcpy(&h, hb + (size_t)j * len_each, sizeof(h));
    void *p = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
      cuda_fail(ctx, e, "cudaIpcOpenMemHandle");
      return UGACHE_EPEER;
    }
    ctx->ipc_mapped[j] = p;
    ctx->src_base[j] = static_cast<const uint8_t *>(p);
  }
  ctx->peers_ready = true;
  return UGACHE_OK;
}

ugache_status ugache_set_peer_slabs(ugache_ctx *ctx, const void *const *slabs) {
  if (!ctx || !slabs) return UGACHE_EINVAL;
  for (int j = 0; j < ctx->cfg.num_gpus; ++j) {
    if (j == ctx->cfg.rank) continue;
    if (!slabs[j] || reinterpret_cast<uintptr_t>(slabs[j]) % 16) return UGACHE_EINVAL;
    int dev = -1;
    if (!is_device_pointer(slabs[j], &dev)) return fail(ctx, UGACHE_EPEER, "peer slab is not device memory");
    if (dev != ctx->device) {
      int can = 0;
      cudaDeviceCanAccessPeer(&can, ctx->device, dev);
      if (!can) return fail(ctx, UGACHE_EPEER, "no peer access to the slab's device");
      ugache_status st = begin(ctx);
      if (st != UGACHE_OK) return st;
      cudaError_t e = cudaDeviceEnablePeerAccess(dev, 0);
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) {
        cuda_fail(ctx, e, "cudaDeviceEnablePeerAccess");
        return UGACHE_EPEER;
      }
      (void)cudaGetLastError();
    }
    ctx->src_base[j] = static_cast<const uint8_t *>(slabs[j]);
  }
  ctx->peers_ready = true;
  return UGACHE_OK;
}

ugache_status ugache_fill(ugache_ctx *ctx, void *stream) {
  if (!ctx) return UGACHE_EINVAL;
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (ctx->n_slots) {
    ugk::FillParams fp;
    fp.slot_idx = nullptr;
    fp.slot_keys = ctx->d_slot_keys;
    fp.table = ctx->host_table_dev;
    fp.slab = ctx->slab;
    fp.n_slots = ctx->n_slots;
    fp.row_bytes = ctx->cfg.row_bytes;
    const int grid = ctx->sm_count * 8;
    ugk::fill_kernel<<<grid, 256, 0, s>>>(fp);
    UG_CUDA(ctx, cudaGetLastError());
  }
  ctx->filled = true;
  return UGACHE_OK;
}

// ---- cache refresh (section 7.2) -------------------------------------------
namespace {
// Host location of key k while a refresh redirects it: the tier slot, or the key itself.
uint64_t host_entry(const ugache_ctx *ctx, uint64_t k) {
  const uint64_t tag = (uint64_t)ctx->cfg.num_gpus << UGACHE_LOC_SRC_SHIFT;
  return tag | (ctx->tier_dev ? (uint64_t)ctx->h_tier_slot[k] : k);
}

// Stage a new placement: checked like ugache_init_with_placement (host rows = keys), its
// host rows translated to tier slots when the ctx has a tier, uploaded next to the current
// table; the changed slots of this GPU (slot, new key) uploaded for the content steps.
ugache_status refresh_stage(ugache_ctx *ctx, const uint64_t *new_loc, const uint64_t *new_slot_keys,
                            uint64_t n_new_slots, cudaStream_t s) {
  if (ctx->refresh_state != 0) return fail(ctx, UGACHE_ESTATE, "refresh already in progress");
  if (!ctx->filled) return fail(ctx, UGACHE_ESTATE, "refresh before fill");
  ugache_status st = check_given_placement(ctx, &ctx->cfg, new_loc, new_slot_keys, n_new_slots);
  if (st != UGACHE_OK) return st;
  st = begin(ctx);
  if (st != UGACHE_OK) return st;
  const uint64_t N = ctx->cfg.num_rows;
  const int G = ctx->cfg.num_gpus;
  UG_CUDA(ctx, cudaStreamSynchronize(s));
  if (!ctx->d_loc_new) UG_CUDA(ctx, cudaMalloc(&ctx->d_loc_new, N * sizeof(uint64_t)));
  if (ctx->tier_dev) {
    std::vector<uint64_t> tr(N);
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < (int64_t)N; ++k)
      tr[k] = (new_loc[k] >> UGACHE_LOC_SRC_SHIFT) == (uint64_t)G ? host_entry(ctx, (uint64_t)k) : new_loc[k];
    UG_CUDA(ctx, cudaMemcpy(ctx->d_loc_new, tr.data(), N * sizeof(uint64_t), cudaMemcpyHostToDevice));
    if (!ctx->d_tier_slot) {
      UG_CUDA(ctx, cudaMalloc(&ctx->d_tier_slot, N * sizeof(uint32_t)));
      UG_CUDA(ctx, cudaMemcpy(ctx->d_tier_slot, ctx->h_tier_slot.data(), N * sizeof(uint32_t),
                              cudaMemcpyHostToDevice));
    }
  } else {
    UG_CUDA(ctx, cudaMemcpy(ctx->d_loc_new, new_loc, N * sizeof(uint64_t), cudaMemcpyHostToDevice));
  }
  ctx->new_slot_keys.assign(new_slot_keys, new_slot_keys + n_new_slots);
  std::vector<uint64_t> keys;
  ctx->refresh_slots.clear();
  for (uint64_t i = 0; i < ctx->new_slot_keys.size(); ++i)
    if (i >= ctx->h_slot_keys.size() || ctx->h_slot_keys[i] != ctx->new_slot_keys[i]) {
      ctx->refresh_slots.push_back(i);
      keys.push_back(ctx->new_slot_keys[i]);
    }
  ctx->refresh_changed = ctx->refresh_slots.size();
  ctx->refresh_pos = 0;
  cudaFree(ctx->d_refresh);
  ctx->d_refresh = nullptr;
  UG_CUDA(ctx, cudaMalloc(&ctx->d_refresh, 2 * std::max<size_t>(keys.size(), 1) * sizeof(uint64_t)));
  if (!keys.empty()) {
    UG_CUDA(ctx, cudaMemcpy(ctx->d_refresh, ctx->refresh_slots.data(), keys.size() * 8, cudaMemcpyHostToDevice));
    UG_CUDA(ctx, cudaMemcpy(ctx->d_refresh + keys.size(), keys.data(), keys.size() * 8, cudaMemcpyHostToDevice));
  }
  return UGACHE_OK;
}

// Keys whose current location is a GPU slot in [lo, hi) and changes -> host (the host holds
// every entry), so nobody reaches those slots while their content is rewritten.
ugache_status refresh_evict(ugache_ctx *ctx, uint64_t lo, uint64_t hi, cudaStream_t s) {
  ugk::refresh_evict_kernel<<<ctx->sm_count * 8, 256, 0, s>>>(
      ctx->d_loc, ctx->d_loc_new, ctx->cfg.num_rows, (uint64_t)ctx->cfg.num_gpus << UGACHE_LOC_SRC_SHIFT,
      ctx->tier_dev ? ctx->d_tier_slot : nullptr, (uint64_t)ctx->cfg.num_gpus, lo, hi);
  UG_CUDA(ctx, cudaGetLastError());
  return UGACHE_OK;
}

// Rewrite the changed slots of this GPU with index in [a, b) of the changed list.
ugache_status refresh_fill(ugache_ctx *ctx, uint64_t a, uint64_t b, int32_t max_sms, cudaStream_t s) {
  if (b <= a) return UGACHE_OK;
  ugk::FillParams fp;
  fp.slot_idx = ctx->d_refresh + a;
  fp.slot_keys = ctx->d_refresh + ctx->refresh_changed + a;
  fp.table = ctx->host_table_dev;
  fp.slab = ctx->slab;
  fp.n_slots = b - a;
  fp.row_bytes = ctx->cfg.row_bytes;
  // throttle: at most max_sms SMs' worth of CTAs
  const int sms = max_sms ? std::min<int>(max_sms, ctx->sm_count) : ctx->sm_count;
  ugk::fill_kernel<<<sms * 8, 256, 0, s>>>(fp);
  UG_CUDA(ctx, cudaGetLastError());
  return UGACHE_OK;
}
}  // namespace

ugache_status ugache_refresh_begin(ugache_ctx *ctx, const uint64_t *new_loc,
                                   const uint64_t *new_slot_keys, uint64_t n_new_slots,
                                   void *stream) {
  if (!ctx || !new_loc) return UGACHE_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  ugache_status st = refresh_stage(ctx, new_loc, new_slot_keys, n_new_slots, s);
  if (st != UGACHE_OK) return st;
  st = refresh_evict(ctx, 0, ~0ull, s);
  if (st != UGACHE_OK) return st;
  ctx->refresh_state = 1;
  return UGACHE_OK;
}

ugache_status ugache_refresh_content(ugache_ctx *ctx, int32_t max_sms, uint64_t max_rows,
                                     uint64_t *remaining, void *stream) {
  if (!ctx || max_sms < 0) return UGACHE_EINVAL;
  if (ctx->refresh_state != 1) return fail(ctx, UGACHE_ESTATE, "refresh_content before refresh_begin");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  const uint64_t total = ctx->refresh_changed, lo = ctx->refresh_pos;
  const uint64_t hi = max_rows ? std::min(total, lo + max_rows) : total;
  st = refresh_fill(ctx, lo, hi, max_sms, static_cast<cudaStream_t>(stream));  // asynchronous
  if (st != UGACHE_OK) return st;
  ctx->refresh_pos = hi;
  if (remaining) *remaining = total - hi;
  if (hi == total) ctx->refresh_state = 2;
  return UGACHE_OK;
}

ugache_status ugache_refresh_stage(ugache_ctx *ctx, const uint64_t *new_loc,
                                   const uint64_t *new_slot_keys, uint64_t n_new_slots,
                                   void *stream) {
  if (!ctx || !new_loc) return UGACHE_EINVAL;
  ugache_status st = refresh_stage(ctx, new_loc, new_slot_keys, n_new_slots, static_cast<cudaStream_t>(stream));
  if (st != UGACHE_OK) return st;
  ctx->refresh_state = 3;
  return UGACHE_OK;
}

ugache_status ugache_refresh_chunk(ugache_ctx *ctx, int32_t step, uint64_t slot_lo, uint64_t slot_hi,
                                   int32_t max_sms, void *stream) {
  if (!ctx || max_sms < 0 || slot_hi < slot_lo) return UGACHE_EINVAL;
  if (ctx->refresh_state != 3) return fail(ctx, UGACHE_ESTATE, "refresh_chunk before refresh_stage");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  switch (step) {
    case UGACHE_REFRESH_EVICT: return refresh_evict(ctx, slot_lo, slot_hi, s);
    case UGACHE_REFRESH_FILL: {
      const auto &v = ctx->refresh_slots;
      const uint64_t a = (uint64_t)(std::lower_bound(v.begin(), v.end(), slot_lo) - v.begin());
      const uint64_t b = (uint64_t)(std::lower_bound(v.begin(), v.end(), slot_hi) - v.begin());
      return refresh_fill(ctx, a, b, max_sms, s);
    }
    case UGACHE_REFRESH_INSTALL:
      ugk::refresh_install_kernel<<<ctx->sm_count * 8, 256, 0, s>>>(
          ctx->d_loc, ctx->d_loc_new, ctx->cfg.num_rows, (uint64_t)ctx->cfg.num_gpus, slot_lo, slot_hi);
      UG_CUDA(ctx, cudaGetLastError());
      return UGACHE_OK;
  }
  return UGACHE_EINVAL;
}

ugache_status ugache_refresh_commit(ugache_ctx *ctx, void *stream) {
  if (!ctx) return UGACHE_EINVAL;
  if (ctx->refresh_state != 2 && ctx->refresh_state != 3)
    return fail(ctx, UGACHE_ESTATE, "refresh_commit before refresh_content / refresh_stage");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const uint64_t N = ctx->cfg.num_rows;
  UG_CUDA(ctx, cudaMemcpyAsync(ctx->d_loc, ctx->d_loc_new, N * sizeof(uint64_t), cudaMemcpyDeviceToDevice, s));
  const uint64_t ns = ctx->new_slot_keys.size();
  if (ns > ctx->slot_keys_cap) {
    UG_CUDA(ctx, cudaStreamSynchronize(s));
    cudaFree(ctx->d_slot_keys);
    ctx->d_slot_keys = nullptr;
    UG_CUDA(ctx, cudaMalloc(&ctx->d_slot_keys, ns * sizeof(uint64_t)));
    ctx->slot_keys_cap = ns;
  }
  if (ns)
    UG_CUDA(ctx, cudaMemcpyAsync(ctx->d_slot_keys, ctx->new_slot_keys.data(), ns * sizeof(uint64_t),
                                 cudaMemcpyHostToDevice, s));
  UG_CUDA(ctx, cudaStreamSynchronize(s));
  ctx->h_slot_keys.swap(ctx->new_slot_keys);
  ctx->new_slot_keys.clear();
  ctx->refresh_slots.clear();
  ctx->n_slots = ns;
  cudaFree(ctx->d_loc_new);
  ctx->d_loc_new = nullptr;
  cudaFree(ctx->d_refresh);
  ctx->d_refresh = nullptr;
  ctx->plan.policy = -1;  // the placement no longer comes from this ctx's solve
  ctx->refresh_state = 0;
  return UGACHE_OK;
}

// ---- A0 calibration (Fig. 6) ------------------------------------------------
namespace {
uint64_t calib_mix(uint64_t &x) {  // splitmix64 step (sample rows only)
  uint64_t z = (x += 0x9E3779B97F4A7C15ull);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// n sorted uniform random rows of [0, span) as sample entries (row << 32 | i)
void calib_sample(std::vector<uint64_t> &ents, uint64_t span, uint32_t n, uint64_t seed) {
  std::vector<uint64_t> rows(n);
  for (uint32_t i = 0; i < n; ++i) rows[i] = span ? calib_mix(seed) % span : 0;
  std::sort(rows.begin(), rows.end());
  const size_t off = ents.size();
  ents.resize(off + n);
  for (uint32_t i = 0; i < n; ++i) ents[off + i] = (rows[i] << 32) | i;
}

// The swept point whose bandwidth first reaches 90 % of the best one (reading R13).
int calib_pick(const int32_t *ks, const double *bw, int n) {
  double best = 0;
  for (int i = 0; i < n; ++i) best = std::max(best, bw[i]);
  for (int i = 0; i < n; ++i)
    if (bw[i] >= 0.9 * best) return i;
  return n - 1;
}
}  // namespace

ugache_status ugache_calibrate(ugache_ctx *ctx, uint32_t sample_rows, ugache_calibration *out) {
  if (!ctx || !out) return UGACHE_EINVAL;
  if (!ctx->filled || !ctx->peers_ready) return fail(ctx, UGACHE_ESTATE, "calibrate before fill/peers");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  std::memset(out, 0, sizeof(*out));
  const uint32_t n = sample_rows ? std::min<uint32_t>(sample_rows, 1u << 22) : 65536u;
  const int G = ctx->cfg.num_gpus, me = ctx->cfg.rank;
  const uint32_t R = ctx->cfg.row_bytes;
  const uint64_t N = ctx->cfg.num_rows;
  const int roles_max = std::max(1, G - 1);
  ugk::CalibParams cp{};
  int S = 0;
  {
    ugk::GatherParams gp{};
    build_roles(ctx, &gp, &S);
    std::memcpy(cp.sm_pos, gp.sm_pos, sizeof(cp.sm_pos));
  }
  for (int j = 0; j < ugk::kMaxSrc; ++j) cp.base[j] = ctx->src_base[j];
  cp.n_ents = n;
  cp.row_bytes = R;
  uint64_t *d_ents = nullptr;
  uint8_t *d_out = nullptr, *d_flush = nullptr;
  uint32_t *d_cursor = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  const size_t flush_bytes = 256u << 20;
  auto cleanup = [&]() {
    cudaFree(d_ents);
    cudaFree(d_out);
    cudaFree(d_flush);
    cudaFree(d_cursor);
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
  };
  cudaError_t ce = cudaMalloc(&d_ents, (size_t)std::max(roles_max, 8) * n * sizeof(uint64_t));
  const uint32_t n_local = n * 8;  // the local gather needs a larger sample to outlast the launch
  if (ce == cudaSuccess) ce = cudaMalloc(&d_out, (size_t)std::max<uint64_t>((uint64_t)roles_max * n, n_local) * R);
  if (ce == cudaSuccess) ce = cudaMalloc(&d_flush, flush_bytes);
  if (ce == cudaSuccess) ce = cudaMalloc(&d_cursor, ugk::kMaxSrc * sizeof(uint32_t));
  if (ce == cudaSuccess) ce = cudaEventCreate(&e0);
  if (ce == cudaSuccess) ce = cudaEventCreate(&e1);
  if (ce == cudaSuccess)
    ce = cudaFuncSetAttribute(ugk::calib_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kOneCtaPerSmSmem);
  if (ce != cudaSuccess) {
    cleanup();
    return cuda_fail(ctx, ce, "calibration buffers");
  }
  cp.ents = d_ents;
  cp.out = d_out;
  cp.cursor = d_cursor;
  // time one configuration: median of 3 cold launches (L2 flushed before each), bytes/s
  auto run = [&](int k, int n_roles, double *bw) -> cudaError_t {
    cp.k = k;
    cp.n_roles = n_roles;
    float ms[3];
    for (int rep = 0; rep < 3; ++rep) {
      cudaError_t e = cudaMemsetAsync(d_flush, rep + 1, flush_bytes, nullptr);
      if (e == cudaSuccess) e = cudaMemsetAsync(d_cursor, 0, ugk::kMaxSrc * sizeof(uint32_t), nullptr);
      if (e == cudaSuccess) e = cudaEventRecord(e0, nullptr);
      void *args[] = {&cp};
      if (e == cudaSuccess)
        e = cudaLaunchCooperativeKernel((const void *)ugk::calib_kernel, dim3(S), dim3(ugk::kGatherThreads), args,
                                        kOneCtaPerSmSmem, nullptr);
      if (e == cudaSuccess) e = cudaEventRecord(e1, nullptr);
      if (e == cudaSuccess) e = cudaEventSynchronize(e1);
      if (e == cudaSuccess) e = cudaEventElapsedTime(&ms[rep], e0, e1);
      if (e != cudaSuccess) return e;
    }
    std::sort(ms, ms + 3);
    *bw = (double)n_roles * cp.n_ents * R / (ms[1] * 1e-3);
    return cudaSuccess;
  };
  std::vector<uint64_t> ents;
  uint64_t seed = 0x55474143ull ^ ((uint64_t)me << 32);
  // host source: uniform rows of the whole host source, sorted (range-ordered reads)
  calib_sample(ents, N, n, seed++);
  ce = cudaMemcpy(d_ents, ents.data(), ents.size() * 8, cudaMemcpyHostToDevice);
  cp.src_id[0] = G;
  const int host_ks[] = {1, 2, 3, 4, 6, 8, 10, 12, 14, 16, 20, 24, 32, 48, 64, 96, 128, 148};
  for (int k : host_ks) {
    if (ce != cudaSuccess || k > S || out->n_host_points >= UGACHE_CALIB_MAX_POINTS) break;
    double bw = 0;
    ce = run(k, 1, &bw);
    out->host_points_sms[out->n_host_points] = k;
    out->host_points_bw[out->n_host_points++] = bw;
  }
  if (ce == cudaSuccess && out->n_host_points) {
    const int i = calib_pick(out->host_points_sms, out->host_points_bw, out->n_host_points);
    out->host_sms = out->host_points_sms[i];
    out->bw_host = out->host_points_bw[i];
  }
  // local slab: every SM
  if (ce == cudaSuccess) {
    ents.clear();
    calib_sample(ents, std::max<uint64_t>(ctx->n_slots, 1), n_local, seed++);
    ce = cudaMemcpy(d_ents, ents.data(), ents.size() * 8, cudaMemcpyHostToDevice);
    cp.src_id[0] = me;
    cp.n_ents = n_local;
    if (ce == cudaSuccess) ce = run(S, 1, &out->bw_local);
    cp.n_ents = n;
  }
  // peers: all at once, k SMs per peer (all-to-all ingress)
  if (ce == cudaSuccess && G > 1) {
    ents.clear();
    int r = 0;
    for (int j = 0; j < G; ++j) {
      if (j == me) continue;
      calib_sample(ents, std::max<uint64_t>(ctx->plan.capacity_rows, 1), n, seed++);
      cp.src_id[r++] = j;
    }
    ce = cudaMemcpy(d_ents, ents.data(), ents.size() * 8, cudaMemcpyHostToDevice);
    const int kmax = std::max(1, (S - std::max(out->host_sms, 1)) / (G - 1));
    const int peer_ks[] = {1, 2, 3, 4, 6, 8, 10, 12, 16, 20, 24, 32, 40, 48, 64, 96, 128, 148};
    for (int k : peer_ks) {
      if (ce != cudaSuccess || k > kmax || out->n_peer_points >= UGACHE_CALIB_MAX_POINTS) break;
      double bw = 0;
      ce = run(k, G - 1, &bw);
      out->peer_points_sms[out->n_peer_points] = k;
      out->peer_points_bw[out->n_peer_points++] = bw;
    }
    if (ce == cudaSuccess && out->n_peer_points) {
      const int i = calib_pick(out->peer_points_sms, out->peer_points_bw, out->n_peer_points);
      out->peer_sms = out->peer_points_sms[i];
      out->bw_peer = out->peer_points_bw[i];
    }
  }
  out->sample_rows = n;
  cleanup();
  if (ce != cudaSuccess) return cuda_fail(ctx, ce, "calibration");
  return UGACHE_OK;
}

ugache_status ugache_set_dedication(ugache_ctx *ctx, int32_t host_sms, int32_t peer_sms) {
  if (!ctx || host_sms < 0 || peer_sms < 0) return UGACHE_EINVAL;
  const int hs = host_sms ? host_sms : ctx->host_sms;
  const int ps = peer_sms ? peer_sms : ctx->peer_sms;
  const int G = ctx->cfg.num_gpus;
  if (hs < 1 || hs > ctx->sm_count) return UGACHE_EINVAL;
  if (G > 1 && (ps < 1 || (int64_t)hs + (int64_t)(G - 1) * ps > ctx->sm_count)) return UGACHE_EINVAL;
  ctx->host_sms = hs;
  ctx->peer_sms = ps;
  return UGACHE_OK;
}

ugache_status ugache_set_mode(ugache_ctx *ctx, int32_t mode) {
  if (!ctx || (mode != UGACHE_MODE_FACTORED && mode != UGACHE_MODE_RANDOM_DISPATCH))
    return UGACHE_EINVAL;
  ctx->mode = mode;
  return UGACHE_OK;
}

ugache_status ugache_set_option(ugache_ctx *ctx, int32_t option, int64_t value) {
  if (!ctx) return UGACHE_EINVAL;
  switch (option) {
    case UGACHE_OPT_HOST_ORDERING: ctx->host_sort = value != 0; return UGACHE_OK;
    case UGACHE_OPT_STAGE_HOST_IO: ctx->stage_host_io = value != 0; return UGACHE_OK;
    case UGACHE_OPT_HOST_WARPS:
      if (value < 1 || value > ugk::kGatherWarps) return UGACHE_EINVAL;
      ctx->host_warps = (int)value;
      return UGACHE_OK;
    case UGACHE_OPT_HOST_WALK: ctx->host_walk = value != 0; return UGACHE_OK;
    case UGACHE_OPT_PREORDER: ctx->preorder = value != 0; return UGACHE_OK;
    case UGACHE_OPT_FUSED:
      if (value < 0 || value > 2) return UGACHE_EINVAL;
      ctx->fused = (int)value;
      return UGACHE_OK;
    case UGACHE_OPT_EARLY_WALK:
      if (value < 0 || value > 1) return UGACHE_EINVAL;
      ctx->early_walk = (int)value;
      return UGACHE_OK;
    case UGACHE_OPT_LOCAL_BULK:
      if (value < 0 || value > 3) return UGACHE_EINVAL;
      ctx->local_bulk = (int)value;
      return UGACHE_OK;
    case UGACHE_OPT_STREAM:
      if (value < 0 || value > 2) return UGACHE_EINVAL;
      ctx->stream = (int)value;
      return UGACHE_OK;
    case UGACHE_OPT_INLINE:
      if (value < 0 || value > (UGACHE_INLINE_HOST | UGACHE_INLINE_PEERS)) return UGACHE_EINVAL;
      ctx->inline_mask = (int)value;
      return UGACHE_OK;
    case UGACHE_OPT_DEDICATION:
      if (value != UGACHE_DEDICATE_SMS && value != UGACHE_DEDICATE_WARPS) return UGACHE_EINVAL;
      ctx->warp_dedication = value == UGACHE_DEDICATE_WARPS;
      return UGACHE_OK;
    case UGACHE_OPT_WARP_HOST:
    case UGACHE_OPT_WARP_PEER: {
      const int hw = option == UGACHE_OPT_WARP_HOST ? (int)value : ctx->wd_host_warps;
      const int pw = option == UGACHE_OPT_WARP_PEER ? (int)value : ctx->wd_peer_warps;
      if (value < 1 || hw + (ctx->cfg.num_gpus - 1) * pw > ugk::kGatherWarps) return UGACHE_EINVAL;
      ctx->wd_host_warps = hw;
      ctx->wd_peer_warps = pw;
      return UGACHE_OK;
    }
  }
  return UGACHE_EINVAL;
}

namespace {
ugache_status extract_impl(ugache_ctx *ctx, const void *keys, int32_t key_type, uint64_t n,
                           void *out, void *stream, bool msg_local) {
  if (!ctx) return UGACHE_EINVAL;
  ctx->msg_state = 0;
  if (key_type != UGACHE_KEY_I64 && key_type != UGACHE_KEY_U32) return UGACHE_EINVAL;
  if (n >= (1ull << 32)) return UGACHE_EINVAL;
  if (!ctx->filled || !ctx->peers_ready) return fail(ctx, UGACHE_ESTATE, "extract before fill/peers");
  ctx->last_n = n;
  ctx->last_launches = 0;
  ctx->timing_valid = false;
  if (n == 0) return UGACHE_OK;
  if (!keys || !out) return UGACHE_EINVAL;
  if (reinterpret_cast<uintptr_t>(keys) % (key_type == UGACHE_KEY_I64 ? 8 : 4))
    return fail(ctx, UGACHE_EINVAL, "keys must be aligned to the key size");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const uint32_t R = ctx->cfg.row_bytes;
  const size_t key_bytes = key_type == UGACHE_KEY_I64 ? 8 : 4;

  // Host buffers: pinned (page-locked, mapped) ones are read / written in place by the
  // kernels over PCIe -- the H2D of the keys and the D2H of the rows are fused into the
  // locate and gather kernels; pageable ones are staged through ctx-owned device buffers.
  const void *dkeys = keys;
  void *mapped = nullptr;
  const MemKind kkind = mem_kind(keys, &mapped);
  if (kkind == MemKind::kPinned && !ctx->stage_host_io) {
    dkeys = mapped;
  } else if (kkind != MemKind::kDevice) {
    st = ensure_stage(ctx, &ctx->d_keys_stage, &ctx->keys_stage_bytes, n * key_bytes);
    if (st != UGACHE_OK) return st;
    UG_CUDA(ctx, cudaMemcpyAsync(ctx->d_keys_stage, keys, n * key_bytes, cudaMemcpyHostToDevice, s));
    dkeys = ctx->d_keys_stage;
  }
  uint8_t *dout = static_cast<uint8_t *>(out);
  const MemKind okind = mem_kind(out, &mapped);
  const bool staged_out = okind == MemKind::kPageable || (okind == MemKind::kPinned && ctx->stage_host_io);
  if (staged_out) {
    st = ensure_stage(ctx, &ctx->d_out_stage, &ctx->out_stage_bytes, n * (size_t)R);
    if (st != UGACHE_OK) return st;
    dout = static_cast<uint8_t *>(ctx->d_out_stage);
  } else {
    if (okind == MemKind::kPinned) dout = static_cast<uint8_t *>(mapped);
    if (reinterpret_cast<uintptr_t>(dout) % 16 != 0)
      return fail(ctx, UGACHE_EINVAL, "out must be 16-byte aligned");
  }
  const bool host_out = staged_out;

  if (ctx->mode == UGACHE_MODE_RANDOM_DISPATCH) {
    ugk::RandomParams rp;
    rp.keys = dkeys;
    rp.loc = ctx->d_loc;
    rp.ctrl = ctx->d_ctrl;
    for (int j = 0; j < ugk::kMaxSrc; ++j) rp.base[j] = ctx->src_base[j];
    rp.out = dout;
    rp.num_rows = ctx->cfg.num_rows;
    rp.n = (uint32_t)n;
    rp.row_bytes = R;
    rp.num_src = ctx->cfg.num_gpus + 1;
    if (ctx->timing) UG_CUDA(ctx, cudaEventRecord(ctx->ev[0], s));
    if (ctx->timing) UG_CUDA(ctx, cudaEventRecord(ctx->ev[1], s));
    if (key_type == UGACHE_KEY_I64)
      ugk::random_dispatch_kernel<int64_t><<<ctx->sm_count, ugk::kGatherThreads, kOneCtaPerSmSmem, s>>>(rp);
    else
      ugk::random_dispatch_kernel<uint32_t><<<ctx->sm_count, ugk::kGatherThreads, kOneCtaPerSmSmem, s>>>(rp);
    UG_CUDA(ctx, cudaGetLastError());
    ctx->last_launches = 1;
  } else {
    st = ensure_scratch(ctx, n, s);
    if (st != UGACHE_OK) return st;
    ugk::LocateParams lp;
    lp.keys = dkeys;
    lp.loc = ctx->d_loc;
    lp.buckets = ctx->d_buckets;
    lp.ctrl = ctx->d_ctrl;
    lp.out = dout;
    lp.num_rows = ctx->cfg.num_rows;
    lp.bucket_cap = ctx->bucket_cap;
    lp.n = (uint32_t)n;
    lp.row_bytes = R;
    lp.num_src = ctx->cfg.num_gpus + 1;
    lp.hist = 0;
    lp.items = ugk::kLocateItems;
    lp.range_shift = ctx->range_shift;
    lp.range_count = ctx->d_ranges;
    ugk::GatherParams gp{};
    gp.buckets = ctx->d_buckets;
    gp.ctrl = ctx->d_ctrl;
    for (int j = 0; j < ugk::kMaxSrc; ++j) gp.base[j] = ctx->src_base[j];
    gp.out = dout;
    gp.bucket_cap = ctx->bucket_cap;
    gp.row_bytes = R;
    gp.num_src = ctx->cfg.num_gpus + 1;
    gp.local_src = ctx->cfg.rank;
    gp.host_sorted = ctx->d_host_sorted;
    gp.range_count = ctx->d_ranges;
    gp.range_cursor = ctx->d_ranges + ugk::kMaxRanges;
    gp.range_shift = ctx->range_shift;
    gp.n_ranges = ctx->n_ranges;
    gp.host_sort = ctx->host_sort;
    gp.keys = dkeys;
    gp.loc = ctx->d_loc;
    gp.num_rows = ctx->cfg.num_rows;
    gp.n_keys = (uint32_t)n;
    gp.keys_u32 = key_type == UGACHE_KEY_U32;
    gp.host_walk = ctx->host_walk;
    gp.host_warps = ctx->host_warps;
    gp.local_bulk = R <= ugk::kBulkWarpBytes / 2 ? ctx->local_bulk : 0;
    gp.early_walk = ctx->early_walk && ctx->host_walk && ctx->host_sort && !ctx->warp_dedication && !msg_local;
    gp.inline_host = (ctx->inline_mask & UGACHE_INLINE_HOST) != 0;
    gp.inline_peer = (ctx->inline_mask & UGACHE_INLINE_PEERS) != 0;
    gp.queues = ctx->d_queues;
    gp.queue_cap = ctx->queue_cap;
    gp.stream_regstore = ctx->stream_regstore;
    gp.stream_peer_warps = ctx->stream_peer_warps;
    gp.local_sms = ctx->local_sms;
    gp.stream_group = ctx->stream_group;
    gp.qctr = ctx->d_qctr;
    gp.stream_bulk = R <= ugk::kBulkWarpBytes / 2 && ctx->local_bulk != 0;
    gp.stream_k = ctx->stream_k;
    gp.stream_ck = 32;
    {  // small batches: fewer keys per chunk, so that every warp of the grid gets one
      const uint64_t warps = (uint64_t)ctx->sm_count * ugk::kGatherWarps;
      const uint64_t per = (n + warps - 1) / warps;
      if (per < 32) {
        uint32_t ck = 4;
        while (ck < per) ck <<= 1;
        gp.stream_ck = (int32_t)ck;
        gp.stream_k = 1;
      }
      if (ctx->stream_ck > 0) {  // env UGACHE_STREAM_CK: keys per chunk (4..32, power of 2)
        gp.stream_ck = std::min<int32_t>(gp.stream_ck, ctx->stream_ck);
        gp.stream_k = 1;
      }
    }
    gp.stream_host_last = ctx->stream_host_last;
    gp.stream_host_cap = ctx->stream_host_cap;
    gp.stream_static = ctx->stream_static;
    gp.stream_nap = ctx->stream_nap;
    gp.stream_prefetch = ctx->stream_prefetch;
    gp.stream_queues = (!gp.inline_host && ctx->host_sms > 0) || (!gp.inline_peer && ctx->cfg.num_gpus > 1);
    gp.preorder = 0;
    gp.hist_smem = ctx->hist_smem;
    gp.host_segments = ctx->host_segments;
    gp.local_pace = ctx->local_pace;
    gp.local_warps = ctx->local_warps;
    gp.timeline = ctx->timing ? ctx->d_timeline : nullptr;
    if (gp.timeline)
      UG_CUDA(ctx, cudaMemsetAsync(gp.timeline, 0, ugk::kMaxSmId * ugk::kTimelineWords * sizeof(unsigned long long), s));
    int grid = 0;
    build_roles(ctx, &gp, &grid);
    if (msg_local) {  // message baseline: no SM reads a peer; the peer buckets stay for msg_*
      gp.n_peers = 0;
      gp.peer_sms = 0;
      gp.host_sms_max = ctx->host_dynamic ? std::max(ctx->host_sms, gp.num_sms) : ctx->host_sms;
    }
    // A sparse host bucket is walked in input order by the host-role SMs (host_walk), which
    // re-reads every key's location entry: that pays only when most SMs walk (G = 1).  With
    // peer roles holding most SMs the walkers are few (12-15 at G = 2..8) and the walk took
    // 0.40-0.50 ms for 3-4K host rows of a 500K-key batch, against 0.16 ms ordered
    // (placement grid), so there every non-empty host bucket is ordered.
    if (ctx->host_walk && 2 * gp.host_sms_max < gp.num_sms &&
        n > (uint64_t)gp.host_sms_max * ctx->walk_keys_per_sm)
      gp.host_sort_min = 1;
    // single pass unless the last launch on this ctx (its counts mirrored to pinned host
    // memory by the kernel) had a host bucket dense enough for range-ordered reads; rows
    // above 1 KB stay on the two-phase path (measured faster there)
    bool stream = !msg_local && !ctx->warp_dedication && ctx->stream != 0;
    // Expected host keys of this batch: scaled from the previous launch on this ctx (its
    // counts mirrored to pinned host memory by the kernel, no synchronisation), or, before
    // the first launch, from the plan's host hotness mass (keys x host_mass_frac).
    const volatile uint32_t *m = ctx->h_mirror;
    const uint64_t pn = m[0], ph = m[1];
    const double exp_host = (m[2] && pn) ? (double)ph * (double)n / (double)pn
                                         : (double)n * ctx->plan.host_mass_frac;
    if (stream && ctx->stream == 2) {
      // with peer rows queued to dedicated SMs the two-phase kernel measured faster (fake
      // peers), so auto takes the single pass only without peer queues
      const bool peer_queues = ctx->cfg.num_gpus > 1 && !(ctx->inline_mask & UGACHE_INLINE_PEERS);
      // A small batch is latency-bound: its rows fit in flight at once and no link saturates,
      // so dedication buys nothing while the two-phase kernel's grid barrier puts every
      // row's latency behind the whole locate pass; it takes the single pass with its peer
      // rows read inline (fake peers, 2K-20K keys: 25-37 us -> 12-22 us)
      const bool small = n <= ctx->small_batch_keys;
      stream = R <= kStreamAutoMaxRow && (!peer_queues || small) &&
               !(ctx->host_sort && exp_host >= (double)ctx->host_sort_min);
      if (stream && peer_queues) {
        gp.inline_peer = 1;
        gp.stream_queues = !gp.inline_host && ctx->host_sms > 0;
      }
    }
    const bool fused = ctx->fused == 1 || (ctx->fused == 2 && n <= kFusedAutoMaxKeys);
    bool reg_kernel = false;
    if (stream && ctx->sparse_host_regpath && exp_host >= 0.005 * (double)n && ctx->stream_ck == 0) {
      // a sparse but present host bucket (cold host rows, latency-bound): the register path
      // with 16-key chunks keeps fewer host requests in flight per warp and measured faster
      // than the TMA slots on distinct DLR-shaped batches
      gp.stream_bulk = 0;
      gp.stream_ck = std::min<int32_t>(gp.stream_ck, 16);
      gp.stream_k = 1;
      if (!gp.stream_queues && ctx->reg_kernel_ck > 0) {  // every source inline: the lean K3r
        reg_kernel = true;
        gp.stream_ck = ctx->reg_kernel_ck;
      }
    }
    if (!stream && ctx->preorder && ctx->host_sort && !gp.early_walk) {
      // two-phase paths: the locate pass builds the host range histogram, and every CTA of the
      // gather scatters a slice of the host bucket into range order (kernels.cuh preorder_host)
      lp.hist = 1;
      gp.preorder = 1;
    }
    if (stream) {  // K3: one cooperative launch, no grid barrier
      if (ctx->timing) {
        UG_CUDA(ctx, cudaEventRecord(ctx->ev[0], s));
        UG_CUDA(ctx, cudaEventRecord(ctx->ev[1], s));
      }
      void *kargs[] = {&lp, &gp};
      const void *fn = key_type == UGACHE_KEY_I64 ? (const void *)ugk::stream_extract_kernel<int64_t>
                                                  : (const void *)ugk::stream_extract_kernel<uint32_t>;
      if (reg_kernel) {
        const void *rf = key_type == UGACHE_KEY_I64 ? (const void *)ugk::stream_extract_reg_kernel<int64_t>
                                                    : (const void *)ugk::stream_extract_reg_kernel<uint32_t>;
        UG_CUDA(ctx, cudaLaunchKernel(rf, dim3(2 * ctx->sm_count), dim3(ugk::kGatherThreads), kargs, 0, s));
      } else if (gp.stream_queues || ctx->stream_coop) {
        UG_CUDA(ctx, cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(ugk::kGatherThreads), kargs,
                                                 kOneCtaPerSmSmem, s));
      } else {  // no queues: no CTA waits on another, a plain launch is enough
        UG_CUDA(ctx, cudaLaunchKernel(fn, dim3(grid), dim3(ugk::kGatherThreads), kargs, kOneCtaPerSmSmem, s));
      }
      ctx->last_launches = 1;
      ctx->last_fused = false;
      ctx->last_single_pass = true;
    } else if (fused) {  // K1 + K2 in one cooperative launch
      // tiles of 512 x items keys, items the smallest count that covers the batch with one
      // tile per CTA (up to kLocateItems): the locate work spreads over every SM
      const uint64_t per = (n + (uint64_t)grid * ugk::kGatherThreads - 1) / ((uint64_t)grid * ugk::kGatherThreads);
      if (ctx->locate_spread) lp.items = (int32_t)std::max<uint64_t>(1, std::min<uint64_t>(ugk::kLocateItems, per));
      if (ctx->timing) {
        UG_CUDA(ctx, cudaEventRecord(ctx->ev[0], s));
        UG_CUDA(ctx, cudaEventRecord(ctx->ev[1], s));
      }
      void *kargs[] = {&lp, &gp};
      const void *fn = key_type == UGACHE_KEY_I64 ? (const void *)ugk::fused_extract_kernel<int64_t>
                                                  : (const void *)ugk::fused_extract_kernel<uint32_t>;
      UG_CUDA(ctx, cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(ugk::kGatherThreads), kargs,
                                               kOneCtaPerSmSmem, s));
      ctx->last_launches = 1;
      ctx->last_fused = true;
      ctx->last_single_pass = false;
    } else {
      const unsigned lgrid = (unsigned)((n + ugk::kLocateTile - 1) / ugk::kLocateTile);
      if (ctx->timing) UG_CUDA(ctx, cudaEventRecord(ctx->ev[0], s));
      if (key_type == UGACHE_KEY_I64)
        ugk::locate_bucket_kernel<int64_t><<<lgrid, ugk::kLocateThreads, 0, s>>>(lp);
      else
        ugk::locate_bucket_kernel<uint32_t><<<lgrid, ugk::kLocateThreads, 0, s>>>(lp);
      UG_CUDA(ctx, cudaGetLastError());
      if (ctx->timing) UG_CUDA(ctx, cudaEventRecord(ctx->ev[1], s));
      void *kargs[] = {&gp};
      UG_CUDA(ctx, cudaLaunchCooperativeKernel((const void *)ugk::factored_gather_kernel, dim3(grid),
                                               dim3(ugk::kGatherThreads), kargs, kOneCtaPerSmSmem, s));
      ctx->last_launches = 2;
      ctx->last_fused = false;
      ctx->last_single_pass = false;
    }
  }
  if (ctx->timing) {
    UG_CUDA(ctx, cudaEventRecord(ctx->ev[2], s));
    ctx->timing_valid = true;
  }
  if (host_out) UG_CUDA(ctx, cudaMemcpyAsync(out, dout, n * (size_t)R, cudaMemcpyDeviceToHost, s));
  ctx->last_stream = s;
  return UGACHE_OK;
}
}  // namespace

ugache_status ugache_extract(ugache_ctx *ctx, const void *keys, int32_t key_type, uint64_t n,
                             void *out, void *stream) {
  return extract_impl(ctx, keys, key_type, n, out, stream, false);
}

// ---------------------------------------------------------------- message-based baseline
ugache_status ugache_msg_extract_local(ugache_ctx *ctx, const void *keys, int32_t key_type,
                                       uint64_t n, void *out, void *stream) {
  if (!ctx) return UGACHE_EINVAL;
  if (ctx->mode != UGACHE_MODE_FACTORED) return fail(ctx, UGACHE_ESTATE, "message path needs the factored mode");
  void *unused = nullptr;
  if (n && out && mem_kind(out, &unused) != MemKind::kDevice)
    return fail(ctx, UGACHE_EINVAL, "message path: out must be device memory");
  ugache_status st = extract_impl(ctx, keys, key_type, n, out, stream, true);
  if (st != UGACHE_OK) return st;
  ctx->msg_state = 1;
  ctx->msg_out = out;
  return UGACHE_OK;
}

namespace {
void msg_segments(const ugache_ctx *ctx, ugk::MsgParams *mp) {
  const int G = ctx->cfg.num_gpus, me = ctx->cfg.rank;
  mp->buckets = ctx->d_buckets;
  mp->bucket_cap = ctx->bucket_cap;
  mp->n_seg = 0;
  uint64_t off = 0;
  for (int j = 0; j < G; ++j) {
    if (j == me) continue;
    mp->seg[mp->n_seg].src = (uint32_t)j;
    mp->seg[mp->n_seg].count = (uint32_t)ctx->msg_counts[j];
    mp->seg[mp->n_seg].off = off;
    off += ctx->msg_counts[j];
    ++mp->n_seg;
  }
  mp->total = off;
  mp->row_bytes = ctx->cfg.row_bytes;
}
unsigned msg_grid(const ugache_ctx *ctx, uint64_t rows_or_items, unsigned per_block) {
  const uint64_t b = (rows_or_items + per_block - 1) / per_block;
  return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(b, (uint64_t)ctx->sm_count * 8));
}
}  // namespace

ugache_status ugache_msg_requests(ugache_ctx *ctx, uint64_t *counts, uint32_t *req, void *stream) {
  if (!ctx || !counts) return UGACHE_EINVAL;
  if (ctx->msg_state != 1) return fail(ctx, UGACHE_ESTATE, "msg_requests without msg_extract_local");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  const int S = ctx->cfg.num_gpus + 1;
  if (ctx->last_n == 0 || ctx->last_launches == 0) {
    for (int j = 0; j < S; ++j) ctx->msg_counts[j] = 0;
  } else {
    UG_CUDA(ctx, cudaStreamSynchronize(ctx->last_stream));
    ugk::Ctrl c;
    UG_CUDA(ctx, cudaMemcpy(&c, ctx->d_ctrl, sizeof(c), cudaMemcpyDeviceToHost));
    for (int j = 0; j < S; ++j) ctx->msg_counts[j] = c.stat_counts[j];
  }
  for (int j = 0; j < S; ++j) counts[j] = ctx->msg_counts[j];
  ugk::MsgParams mp{};
  msg_segments(ctx, &mp);
  mp.req = req;
  if (mp.total) {
    if (!req) return UGACHE_EINVAL;
    ugk::msg_pack_kernel<<<msg_grid(ctx, mp.total, 256), 256, 0, static_cast<cudaStream_t>(stream)>>>(mp);
    UG_CUDA(ctx, cudaGetLastError());
  }
  ctx->msg_state = 2;
  return UGACHE_OK;
}

ugache_status ugache_msg_serve(ugache_ctx *ctx, const uint32_t *req_in, uint64_t n_req, void *send,
                               void *stream) {
  if (!ctx) return UGACHE_EINVAL;
  if (!n_req) return UGACHE_OK;
  if (!req_in || !send) return UGACHE_EINVAL;
  if (!ctx->filled) return fail(ctx, UGACHE_ESTATE, "serve before fill");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  ugk::MsgParams mp{};
  mp.total = n_req;
  mp.req_in = req_in;
  mp.slab = ctx->slab;
  mp.slab_rows = ctx->plan.capacity_rows;
  mp.rows_out = static_cast<uint8_t *>(send);
  mp.row_bytes = ctx->cfg.row_bytes;
  ugk::msg_copy_kernel<false><<<msg_grid(ctx, n_req, 16 * ugk::kRowsInFlight), 512, 0,
                                static_cast<cudaStream_t>(stream)>>>(mp);
  UG_CUDA(ctx, cudaGetLastError());
  return UGACHE_OK;
}

ugache_status ugache_msg_scatter(ugache_ctx *ctx, const void *replies, void *out, void *stream) {
  if (!ctx) return UGACHE_EINVAL;
  if (ctx->msg_state != 2) return fail(ctx, UGACHE_ESTATE, "msg_scatter without msg_requests");
  if (out != ctx->msg_out) return fail(ctx, UGACHE_EINVAL, "msg_scatter: out differs from msg_extract_local's");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  ugk::MsgParams mp{};
  msg_segments(ctx, &mp);
  ctx->msg_state = 0;
  if (!mp.total) return UGACHE_OK;
  if (!replies || !out) return UGACHE_EINVAL;
  mp.rows_in = static_cast<const uint8_t *>(replies);
  mp.rows_out = static_cast<uint8_t *>(out);
  ugk::msg_copy_kernel<true><<<msg_grid(ctx, mp.total, 16 * ugk::kRowsInFlight), 512, 0,
                               static_cast<cudaStream_t>(stream)>>>(mp);
  UG_CUDA(ctx, cudaGetLastError());
  return UGACHE_OK;
}

ugache_status ugache_last_batch_stats(ugache_ctx *ctx, uint64_t *per_source, uint64_t *bad_keys) {
  if (!ctx) return UGACHE_EINVAL;
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  const int S = ctx->cfg.num_gpus + 1;
  if (ctx->last_n == 0 || ctx->last_launches == 0) {
    if (per_source) for (int j = 0; j < S; ++j) per_source[j] = 0;
    if (bad_keys) *bad_keys = 0;
    return UGACHE_OK;
  }
  UG_CUDA(ctx, cudaStreamSynchronize(ctx->last_stream));
  ugk::Ctrl c;
  UG_CUDA(ctx, cudaMemcpy(&c, ctx->d_ctrl, sizeof(c), cudaMemcpyDeviceToHost));
  if (per_source) for (int j = 0; j < S; ++j) per_source[j] = c.stat_counts[j];
  if (bad_keys) *bad_keys = c.stat_bad;
  return UGACHE_OK;
}

ugache_status ugache_enable_timing(ugache_ctx *ctx, int32_t on) {
  if (!ctx) return UGACHE_EINVAL;
  ctx->timing = on != 0;
  ctx->timing_valid = false;
  return UGACHE_OK;
}

ugache_status ugache_last_batch_timing(ugache_ctx *ctx, float *ms_locate, float *ms_gather) {
  if (!ctx) return UGACHE_EINVAL;
  if (!ctx->timing_valid) return fail(ctx, UGACHE_ESTATE, "no timed extract");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  UG_CUDA(ctx, cudaEventSynchronize(ctx->ev[2]));
  float a = 0, b = 0;
  UG_CUDA(ctx, cudaEventElapsedTime(&a, ctx->ev[0], ctx->ev[1]));
  UG_CUDA(ctx, cudaEventElapsedTime(&b, ctx->ev[1], ctx->ev[2]));
  if (ctx->last_single_pass && ctx->mode == UGACHE_MODE_FACTORED) {
    b += a;  // single pass: no separate locate phase
    a = 0.f;
  } else if (ctx->last_fused && ctx->mode == UGACHE_MODE_FACTORED) {
    // one launch: split it at the grid barrier with the kernel's own %globaltimer stamps
    ugk::Ctrl c;
    UG_CUDA(ctx, cudaMemcpy(&c, ctx->d_ctrl, sizeof(c), cudaMemcpyDeviceToHost));
    const float loc = c.t_located > c.t_start ? (float)((c.t_located - c.t_start) * 1e-6) : 0.f;
    a = std::min(loc, b);
    b -= a;
  }
  if (ms_locate) *ms_locate = a;
  if (ms_gather) *ms_gather = b;
  return UGACHE_OK;
}

ugache_status ugache_last_batch_phases(ugache_ctx *ctx, float *ms) {
  if (!ctx || !ms) return UGACHE_EINVAL;
  if (!ctx->last_fused || ctx->last_launches == 0 || ctx->mode != UGACHE_MODE_FACTORED)
    return fail(ctx, UGACHE_ESTATE, "last extract was not a fused launch");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  UG_CUDA(ctx, cudaStreamSynchronize(ctx->last_stream));
  ugk::Ctrl c;
  UG_CUDA(ctx, cudaMemcpy(&c, ctx->d_ctrl, sizeof(c), cudaMemcpyDeviceToHost));
  auto rel = [&](unsigned long long t) { return t > c.t_start ? (float)((t - c.t_start) * 1e-6) : 0.f; };
  ms[0] = rel(c.t_located);
  ms[1] = rel(c.t_ordered);
  ms[2] = rel(c.t_host_done);
  ms[3] = rel(c.t_loc_last);
  ms[4] = rel(c.t_end);
  return UGACHE_OK;
}

ugache_status ugache_last_batch_timeline(ugache_ctx *ctx, float *out, int32_t *num_ctas) {
  if (!ctx || !out || !num_ctas) return UGACHE_EINVAL;
  if (!ctx->last_fused || ctx->last_launches == 0 || ctx->mode != UGACHE_MODE_FACTORED || !ctx->timing)
    return fail(ctx, UGACHE_ESTATE, "last extract was not a fused launch with timing on");
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  UG_CUDA(ctx, cudaStreamSynchronize(ctx->last_stream));
  const int S = (int)ctx->smids.size();
  std::vector<unsigned long long> t((size_t)S * ugk::kTimelineWords);
  UG_CUDA(ctx, cudaMemcpy(t.data(), ctx->d_timeline, t.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost));
  ugk::Ctrl c;
  UG_CUDA(ctx, cudaMemcpy(&c, ctx->d_ctrl, sizeof(c), cudaMemcpyDeviceToHost));
  auto rel = [&](unsigned long long v) { return v > c.t_start ? (float)((v - c.t_start) * 1e-6) : 0.f; };
  for (int i = 0; i < S; ++i) {
    const unsigned long long *w = &t[(size_t)i * ugk::kTimelineWords];
    out[i * 5 + 0] = (float)w[0];
    for (int k = 1; k < 5; ++k) out[i * 5 + k] = rel(w[k]);
  }
  *num_ctas = S;
  return UGACHE_OK;
}

ugache_status ugache_last_launch_count(const ugache_ctx *ctx, int32_t *launches) {
  if (!ctx || !launches) return UGACHE_EINVAL;
  *launches = ctx->last_launches;
  return UGACHE_OK;
}

ugache_status ugache_last_extract_path(const ugache_ctx *ctx, int32_t *path) {
  if (!ctx || !path) return UGACHE_EINVAL;
  if (ctx->last_launches == 0) *path = UGACHE_PATH_NONE;
  else if (ctx->mode == UGACHE_MODE_RANDOM_DISPATCH) *path = UGACHE_PATH_RANDOM;
  else if (ctx->last_single_pass) *path = UGACHE_PATH_SINGLE_PASS;
  else if (ctx->last_fused) *path = UGACHE_PATH_FUSED;
  else *path = UGACHE_PATH_SPLIT;
  return UGACHE_OK;
}

ugache_status ugache_export_placement(ugache_ctx *ctx, uint64_t *loc, uint64_t *slot_keys,
                                      uint64_t *n_slots) {
  if (!ctx) return UGACHE_EINVAL;
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  if (loc)
    UG_CUDA(ctx, cudaMemcpy(loc, ctx->d_loc, ctx->cfg.num_rows * sizeof(uint64_t), cudaMemcpyDeviceToHost));
  if (slot_keys && ctx->n_slots)
    UG_CUDA(ctx, cudaMemcpy(slot_keys, ctx->d_slot_keys, ctx->n_slots * sizeof(uint64_t),
                            cudaMemcpyDeviceToHost));
  if (n_slots) *n_slots = ctx->n_slots;
  return UGACHE_OK;
}

ugache_status ugache_read_slab(ugache_ctx *ctx, uint64_t first, uint64_t count, void *dst) {
  if (!ctx || (!dst && count)) return UGACHE_EINVAL;
  if (first > ctx->plan.capacity_rows || count > ctx->plan.capacity_rows - first) return UGACHE_EINVAL;
  if (!count) return UGACHE_OK;
  ugache_status st = begin(ctx);
  if (st != UGACHE_OK) return st;
  const uint64_t R = ctx->cfg.row_bytes;
  UG_CUDA(ctx, cudaDeviceSynchronize());
  UG_CUDA(ctx, cudaMemcpy(dst, ctx->slab + first * R, count * R, cudaMemcpyDeviceToHost));
  return UGACHE_OK;
}

ugache_status ugache_destroy(ugache_ctx *ctx) {
  if (!ctx) return UGACHE_OK;
  if (cudaSetDevice(ctx->device) == cudaSuccess) {
    cudaDeviceSynchronize();
    for (int j = 0; j < UGACHE_MAX_GPUS; ++j)
      if (ctx->ipc_mapped[j]) cudaIpcCloseMemHandle(ctx->ipc_mapped[j]);
    cudaFree(ctx->slab);
    cudaFree(ctx->d_loc);
    cudaFree(ctx->d_slot_keys);
    cudaFree(ctx->d_ctrl);
    cudaFree(ctx->d_timeline);
    cudaFree(ctx->d_buckets);
    cudaFree(ctx->d_keys_stage);
    cudaFree(ctx->d_out_stage);
    cudaFree(ctx->d_host_sorted);
    cudaFree(ctx->d_queues);
    cudaFree(ctx->d_qctr);
    if (ctx->h_mirror) cudaFreeHost(ctx->h_mirror);
    cudaFree(ctx->d_ranges);
    cudaFree(ctx->d_loc_new);
    cudaFree(ctx->d_refresh);
    cudaFree(ctx->d_tier_slot);
    for (int i = 0; i < 3; ++i)
      if (ctx->ev[i]) cudaEventDestroy(ctx->ev[i]);
  }
  unpin_all(ctx);
  if (ctx->tier_owned) munmap(ctx->tier_owned, ctx->tier_owned_bytes);
  (void)cudaGetLastError();
  delete ctx;
  return UGACHE_OK;
}

}  // extern "C"
