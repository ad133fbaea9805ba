/*
 * ugache.h -- C ABI of the B200-native UGache factored-embedding-extraction library.
 *
 * Citations "P:n" are lines of the paper text (PAPER.md of dblp/paper_conf_sosp_songz0c23,
 * "UGache: A Unified GPU Cache for Embedding-based Deep Learning", SOSP'23).
 *
 * The hot path (ugache_extract) is the paper's extract() (section 3.2) executed
 * with the factored extraction mechanism (section 5.3): every key is located
 * through this GPU's location table (the per-GPU "hashtable" of <GPU_i, Offset>),
 * keys are grouped by source, SMs dedicated to each non-local source (host
 * DRAM over PCIe, each peer GPU over NVLink/NVSwitch) copy their group, and local HBM work
 * pads the ragged non-local time.  The placement is solved on the host
 * (section 6) and filled once (Filler).
 *
 * Conventions that hold for every function:
 *  - Errors: every function returns a ugache_status; nothing throws or aborts across the
 *    ABI.  UGACHE_EINVAL = bad argument / size / alignment; UGACHE_ESTATE = wrong call
 *    order; UGACHE_ECUDA = a CUDA runtime call failed (text in ugache_last_error_message);
 *    UGACHE_ENOMEM = device or host allocation failed; UGACHE_EPEER = peer mapping failed.
 *  - Pointers are plain host or device addresses.  Streams are cudaStream_t passed as
 *    void* (NULL = legacy default stream).
 *  - Keys are integer row ids in [0, num_rows).  An out-of-range key (including a negative
 *    int64) yields an all-zero output row and is counted in bad_keys (R2).
 *  - Sizes: num_rows < 2^32, batch n < 2^32, row_bytes a positive multiple of 16.
 *  - One ugache_ctx per (process, GPU rank).  A ctx is not re-entrant: calls on one ctx
 *    must not overlap; extracts on one ctx are ordered by the caller's streams.
 */
#ifndef UGACHE_H_
#define UGACHE_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define UGACHE_VERSION 1
#define UGACHE_MAX_GPUS 16
/* Location-table entry: (src << 56) | row.  src = j < G: GPU j's cache slab, row = slot;
 * src = G: host DRAM, row = key (the host holds every entry), or the host-tier
 * slot when UGACHE_FLAG_HOST_TIER is set. */
#define UGACHE_LOC_SRC_SHIFT 56
#define UGACHE_LOC_ROW_MASK ((((uint64_t)1) << 56) - 1)

typedef struct ugache_ctx ugache_ctx;

typedef enum {
  UGACHE_OK = 0,
  UGACHE_EINVAL = 1,
  UGACHE_ECUDA = 2,
  UGACHE_ENOMEM = 3,
  UGACHE_ESTATE = 4,
  UGACHE_EPEER = 5,
  UGACHE_EKEY = 6
} ugache_status;

/* Cache policies run through the same kernels (P:385-413 replication / partition;
 * UGACHE = hotness-driven hot-replicate / warm-partition chosen by the section 6.2 model). */
typedef enum {
  UGACHE_POLICY_UGACHE = 0,
  UGACHE_POLICY_REPLICATION = 1,
  UGACHE_POLICY_PARTITION = 2
} ugache_policy;

typedef enum { UGACHE_KEY_I64 = 0, UGACHE_KEY_U32 = 1 } ugache_key_type;

/* Extraction mechanism.  FACTORED = the paper's FEM (section 5.3).  RANDOM_DISPATCH = the
 * unfactored peer-based baseline (section 5.2): keys dispatched to warps in
 * input order, each warp locates on the fly and reads whichever source (ablation only). */
typedef enum { UGACHE_MODE_FACTORED = 0, UGACHE_MODE_RANDOM_DISPATCH = 1 } ugache_mode;

typedef struct {
  uint64_t num_rows;      /* N: entries of the (concatenated) embedding table            */
  uint32_t row_bytes;     /* R: bytes per entry (D * sizeof(dtype)), multiple of 16       */
  uint32_t reserved0;     /* must be 0                                                    */
  uint64_t capacity_rows; /* C: per-GPU cache capacity in entries (Cap_j) */
  int32_t num_gpus;       /* G in [1, UGACHE_MAX_GPUS]                                    */
  int32_t rank;           /* this GPU's index in [0, G)                                   */
  int32_t device;         /* CUDA device ordinal used by this ctx                         */
  int32_t policy;         /* ugache_policy                                                */
  double bw_local;        /* bytes/s of local HBM gathers for the model; 0 = default      */
  double bw_peer;         /* bytes/s of NVLink ingress per GPU; 0 = default               */
  double bw_host;         /* bytes/s of host->GPU zero-copy reads; 0 = default            */
  int32_t host_sms;       /* SMs dedicated to host extraction; 0 = default  */
  int32_t peer_sms;       /* SMs dedicated to each peer; 0 = floor((S-host)/(G-1));
                             a measured cap (ugache_calibrate) is applied with
                             ugache_set_dedication -- DESIGN.md R14                           */
  int32_t num_sms;        /* S; 0 = the device's SM count (148 on B200)                   */
  int32_t flags;          /* UGACHE_FLAG_* bits; other bits must be 0                     */
} ugache_config;

/* Host tier (reading R24): the entries that no GPU caches (hotness
 * ranks >= band_end) are read from a pinned host copy laid out in hotness-rank order
 * instead of the caller's key-ordered table, so host reads concentrate in a dense prefix
 * of host address space.  Location-table rows of the host source are then tier slots
 * (slot t holds the key of rank (band_end + t) mod N) instead of keys; the tier holds all N
 * rows so that a cache refresh can redirect any evicted key to it. */
#define UGACHE_FLAG_HOST_TIER 1

/* Solver output (section 6.2 model evaluated for the chosen placement). */
typedef struct {
  int32_t policy;          /* policy solved for                                         */
  int32_t num_gpus;        /* G                                                         */
  uint64_t capacity_rows;  /* effective C = min(C, N)                                   */
  uint64_t k;              /* hotness ranks [0,k) replicated on every GPU               */
  uint64_t band_end;       /* ranks [k,band_end) partitioned round-robin; rest on host  */
  double z;                /* modeled batch extraction time (s) of the chosen placement */
  double z_replication;    /* z at k = C                                                */
  double z_partition;      /* z at k = 0                                                */
  double T_local, T_peer, T_host;  /* T_{i<-j} per entry (s)               */
  double R_local, R_peer, R_host;  /* R_{i<-j} core ratios                   */
  int32_t host_sms, peer_sms, num_sms, reserved;
  double host_mass_frac;   /* hotness mass of the host-resident ranks (>= band_end) over the
                              total: the expected host share of a batch's keys (hotness =
                              expected accesses per batch, R6).  The extract path
                              choice uses it until this ctx has run a launch.  0 = unknown
                              (ugache_init_with_placement).                                */
} ugache_plan;

/* ---- host-only placement solver (no GPU needed) ------------------------------------ */

/* Solve the cache placement (section 6) for cfg (rank/device ignored).
 * hotness: N floats (access frequency; NULL = uniform; NaN/Inf -> EINVAL;
 * values <= 0 count as 0).  order: optional out, N entries, order[r] = key of hotness rank
 * r (ties by lower key).  plan: out.  Deterministic; O(N) memory + O(C*G) model sweep. */
ugache_status ugache_solve(const ugache_config *cfg, const float *hotness, uint64_t *order,
                           ugache_plan *plan);

/* Build GPU `gpu`'s location table and slot list for a solved plan.
 * order: N entries from ugache_solve.  loc: out, N entries (UGACHE_LOC_* encoding).
 * slot_keys: out, capacity_rows entries (key cached in each slot of GPU gpu's slab);
 * n_slots: out, number of filled slots (<= capacity). */
ugache_status ugache_build_placement(const ugache_config *cfg, const uint64_t *order,
                                     const ugache_plan *plan, int32_t gpu, uint64_t *loc,
                                     uint64_t *slot_keys, uint64_t *n_slots);

/* Host tier (UGACHE_FLAG_HOST_TIER): number of tier rows -- N: the tier holds every row in
 * hotness-rank order rotated so the host-resident ranks [band_end, N) come first (slot t =
 * rank (band_end + t) mod N); the cached ranks' slots serve keys a refresh evicts. */
uint64_t ugache_host_tier_rows(const ugache_plan *plan, uint64_t num_rows);

/* Fill a caller-provided host tier: tier[t*R ..) = table row order[(band_end + t) mod N]
 * for t < N (parallel host copy, no GPU).  tier: ugache_host_tier_rows * R bytes. */
ugache_status ugache_fill_host_tier(const ugache_config *cfg, const uint64_t *order,
                                    const ugache_plan *plan, const void *host_table,
                                    void *tier);

/* ---- context lifecycle -------------------------------------------------------------- */

/* Create the ctx of GPU cfg->rank on device cfg->device: solve the placement, build this
 * GPU's location table in HBM, allocate the cache slab (C x R bytes, its own cudaMalloc so
 * it can be IPC-exported) and the bucket scratch.  host_table: N*R bytes, 16-byte aligned
 * (else EINVAL), caller-owned, must outlive the ctx and stay unmodified (read-only access); it is page-locked and
 * mapped with cudaHostRegister unless already pinned.  hotness: as for ugache_solve,
 * copied.  The cache is NOT filled: call ugache_fill, connect peers, then barrier. */
ugache_status ugache_init(ugache_ctx **ctx, const ugache_config *cfg, const void *host_table,
                          const float *hotness);

/* Same as ugache_init but with a precomputed order/plan (every rank of a process group can
 * share one solve).  order: N entries, a permutation of [0, N) (else EINVAL); plan from
 * ugache_solve with the same cfg (its capacity_rows <= min(C, N), k <= capacity_rows <=
 * band_end <= N, and the same SM dedication, else EINVAL).
 * host_tier: with UGACHE_FLAG_HOST_TIER, an optional caller-owned tier already filled by
 * ugache_fill_host_tier (shared by the ranks of a node; pinned by the library unless
 * already pinned; must outlive the ctx); NULL = the ctx builds and owns its own tier.
 * ugache_init with the flag always builds its own. */
ugache_status ugache_init_with_plan(ugache_ctx **ctx, const ugache_config *cfg,
                                    const void *host_table, const uint64_t *order,
                                    const ugache_plan *plan, const void *host_tier);

/* Same, with a placement computed elsewhere (e.g. the block-level MILP of section 6.3,
 * P:1520-1566, which may replicate an entry on any subset of GPUs): loc = this GPU's
 * location table (N entries, UGACHE_LOC_* encoding, host rows = keys), slot_keys = the keys
 * of its slots 0..n_slots-1 (n_slots <= capacity_rows).  Checked: every key resolves to
 * GPU j < G with row < capacity, or to the host with row == key; every key mapped to this
 * GPU sits in the named slot.  UGACHE_FLAG_HOST_TIER is not supported here (EINVAL).  The
 * plan reports policy -1, k = 0, band_end = N, z = 0. */
ugache_status ugache_init_with_placement(ugache_ctx **ctx, const ugache_config *cfg,
                                         const void *host_table, const uint64_t *loc,
                                         const uint64_t *slot_keys, uint64_t n_slots);

ugache_status ugache_get_plan(const ugache_ctx *ctx, ugache_plan *plan);

/* Device address and size of this GPU's cache slab (for in-process peers / checks). */
ugache_status ugache_slab(const ugache_ctx *ctx, void **dev_ptr, uint64_t *bytes,
                          uint64_t *n_slots);

/* Export this GPU's slab as a cudaIpcMemHandle_t.  buf: out, *len in: capacity, out: bytes
 * written (64).  Peer-based access in a unified address space. */
ugache_status ugache_ipc_handle(ugache_ctx *ctx, void *buf, size_t *len);

/* Map every peer's slab.  all_handles: G handles of len_each bytes in rank order (this
 * rank's entry is ignored).  Opened with cudaIpcMemLazyEnablePeerAccess.  -> EPEER. */
ugache_status ugache_open_peers(ugache_ctx *ctx, const void *all_handles, size_t len_each);

/* In-process alternative to IPC: slabs[j] = device address of GPU j's slab, reachable from
 * this ctx's device (same device, or peer access enabled), 16-byte aligned.  slabs[rank] is
 * ignored. */
ugache_status ugache_set_peer_slabs(ugache_ctx *ctx, const void *const *slabs);

/* Filler: copy this GPU's cached rows from the host table into its slab
 * (zero-copy gather over PCIe), asynchronously on stream.  Peers must be filled (and a
 * barrier passed) before any GPU extracts from them. */
ugache_status ugache_fill(ugache_ctx *ctx, void *stream);

/* THE HOT PATH.  out[i*R .. (i+1)*R) = table row keys[i] for i < n (output in
 * key order P:626-627).  keys: n keys of key_type, device or host memory, aligned to the
 * key size (else EINVAL).  out: n*R bytes,
 * device or host memory, 16-byte aligned.  Device buffers: fully asynchronous on stream,
 * no host synchronisation, no collective; keys/out must stay valid until the stream
 * reaches the work.  Pinned (page-locked) host buffers: read / written in place by the
 * kernels over PCIe (zero-copy; UGACHE_OPT_STAGE_HOST_IO = 1 stages them instead).
 * Pageable host buffers: staged through ctx-owned device buffers with async copies on the
 * same stream.  With any host buffer the caller synchronises the stream before reading
 * out.  n == 0: no work.  Requires ugache_fill and, for G > 1, peers (else ESTATE). */
ugache_status ugache_extract(ugache_ctx *ctx, const void *keys, int32_t key_type, uint64_t n,
                             void *out, void *stream);

/* ---- message-based baseline -----------------------
 * The design UGache argues against: "a GPU sends keys to the GPU caching them, which then
 * looks up and sends back the values" and the requester must "reorder ... back to the
 * original key order".  Same placement, location table and kernels as the
 * factored path; the peer rows travel through two all-to-all exchanges done by the CALLER
 * (NCCL via torch.distributed), never through peer loads.  Per batch, on every GPU:
 *   1. ugache_msg_extract_local(keys, out): locate + bucket every key, copy the local and
 *      host rows into out (peer SMs = 0); the peer buckets stay in the ctx.
 *   2. ugache_msg_requests(counts, req): synchronises the stream, returns the per-source
 *      key counts (G+1 entries as ugache_last_batch_stats) and packs the slot ids wanted
 *      from each peer into req (device, >= sum of the peer counts u32 entries), peers in
 *      rank order.  The caller exchanges counts and req (all-to-all).
 *   3. ugache_msg_serve(req_in, n_req, send): on the owner, send[i] = slab row req_in[i]
 *      (device buffers; n_req*R bytes).  The caller all-to-alls send back.
 *   4. ugache_msg_scatter(replies, out): replies packed in the same peer order as req;
 *      out[out_idx] = reply row.  out must be the out of step 1.
 * Steps 2-4 must follow step 1 of the same batch on the same ctx with no extract in
 * between (ESTATE otherwise).  Device memory only for req/send/replies/out.  Not for the
 * hot path: it exists to measure the paper's message-based comparison (Fig. 4 / Fig. 13). */
ugache_status ugache_msg_extract_local(ugache_ctx *ctx, const void *keys, int32_t key_type,
                                       uint64_t n, void *out, void *stream);
ugache_status ugache_msg_requests(ugache_ctx *ctx, uint64_t *counts, uint32_t *req, void *stream);
ugache_status ugache_msg_serve(ugache_ctx *ctx, const uint32_t *req_in, uint64_t n_req, void *send,
                               void *stream);
ugache_status ugache_msg_scatter(ugache_ctx *ctx, const void *replies, void *out, void *stream);

/* ---- cache refresh (section 7.2) ----------------------------------------
 * "Refresher evicts old entries and inserts new entries into UGache's hashtable and cache
 * content ... Refresher waits for a foreground batch between the update of hashtable and
 * cache content".  new_loc / new_slot_keys: as for ugache_init_with_placement
 * (checked the same way; host rows = keys -- with UGACHE_FLAG_HOST_TIER the library maps
 * them to tier slots, the tier holding every row).  Every call below is asynchronous on
 * stream except where noted; between steps the CALLER makes every GPU of the group reach
 * the same step (barrier) and, where stated, lets one foreground batch finish.  Wrong
 * order -> ESTATE.
 *
 * Whole-table protocol (three calls per GPU):
 *   1. ugache_refresh_begin(new placement): stage it (synchronises stream; uploads the new
 *      table), then every key whose location changes is pointed at the host (which holds
 *      every entry); extracts stay correct and read those keys from host DRAM.
 *      -> all GPUs, then >= 1 foreground batch + barrier
 *   2. ugache_refresh_content(max_sms, max_rows, &remaining): rewrite the next max_rows
 *      (0 = all) slots whose key changes from the host table with at most max_sms SMs'
 *      worth of CTAs (0 = all) -- the refresh granularity / resource throttle of
 *      P:1611-1616; call again while remaining > 0.  -> all GPUs: synchronise the stream,
 *      then barrier
 *   3. ugache_refresh_commit: install the new location table and slot list (synchronises).
 *
 * Chunked protocol (the incremental refill of SURVEY.md 8(f) row 3): only one slot range is
 * in transition at a time, so at most that chunk's keys are redirected to the host.
 *   ugache_refresh_stage(new placement)                 (synchronous; no table change)
 *   for each slot range [lo, hi) covering [0, capacity_rows), on every GPU:
 *     ugache_refresh_chunk(EVICT, lo, hi): keys whose current location is a GPU slot in
 *        [lo, hi) and changes -> host.   -> all GPUs, >= 1 foreground batch + barrier
 *     ugache_refresh_chunk(FILL, lo, hi, max_sms): rewrite this GPU's changed slots in
 *        [lo, hi).   -> all GPUs: synchronise the stream, then barrier
 *     ugache_refresh_chunk(INSTALL, lo, hi): keys whose new location is a GPU slot in
 *        [lo, hi) take it.
 *   ugache_refresh_commit                                (synchronous) */
enum { UGACHE_REFRESH_EVICT = 0, UGACHE_REFRESH_FILL = 1, UGACHE_REFRESH_INSTALL = 2 };
ugache_status ugache_refresh_begin(ugache_ctx *ctx, const uint64_t *new_loc,
                                   const uint64_t *new_slot_keys, uint64_t n_new_slots,
                                   void *stream);
ugache_status ugache_refresh_content(ugache_ctx *ctx, int32_t max_sms, uint64_t max_rows,
                                     uint64_t *remaining, void *stream);
ugache_status ugache_refresh_stage(ugache_ctx *ctx, const uint64_t *new_loc,
                                   const uint64_t *new_slot_keys, uint64_t n_new_slots,
                                   void *stream);
ugache_status ugache_refresh_chunk(ugache_ctx *ctx, int32_t step, uint64_t slot_lo,
                                   uint64_t slot_hi, int32_t max_sms, void *stream);
ugache_status ugache_refresh_commit(ugache_ctx *ctx, void *stream);

/* Section 6.2 model value z (seconds) of a given placement under hotness (P:1359-1385,
 * P:1497-1498): locs[i] = GPU i's location table (N entries, UGACHE_LOC_* encoding; only
 * the source field is used), hotness = N floats (NULL = uniform; <= 0 counts as 0; NaN/Inf
 * -> EINVAL), T_{i<-j} / R_{i<-j} from plan.  The Refresher's trigger compares the current
 * placement's z under fresh hotness with a new solve's z.  Host-only. */
ugache_status ugache_model_time(const ugache_plan *plan, int32_t num_gpus, uint64_t num_rows,
                                const uint64_t *const *locs, const float *hotness, double *z);

/* ---- A0 calibration (Fig. 6; section 5.3) -------------------
 * Bandwidth vs the number of SMs dedicated to a source, measured through this ctx's own
 * sources with the extract kernels' SM placement (roles spread over the chip): the host
 * source (tier or table: sorted uniform random rows, the range-ordered host reads), every
 * peer at once (k SMs per peer, all-to-all ingress), and the local slab (all SMs).  L2 is
 * flushed before every timed launch.  "Realistic contention": call it on every
 * rank of the group at the same time (caller barrier before), so the host link and each
 * GPU's NVLink egress carry the load of all G readers.  Synchronous (uses the legacy
 * stream and a temporary 256 MiB device buffer).  Results (reading R13 of DESIGN.md):
 *   host_sms = the smallest swept SM count reaching >= 90 % of the best host bandwidth;
 *   bw_host  = the bandwidth at host_sms (bytes/s of row payload);
 *   peer_sms = the same rule on the aggregate peer ingress with k SMs per peer, capped at
 *              floor((S - host_sms) / (G - 1)) (0 when G == 1 or peers are not connected);
 *   bw_peer  = aggregate ingress at peer_sms (the ugache_config bw_peer unit);
 *   bw_local = local random-row gather with every SM (bytes/s of rows read).
 * The curves are returned point by point.  Requires ugache_fill (and peers when G > 1). */
#define UGACHE_CALIB_MAX_POINTS 24
typedef struct {
  int32_t host_sms, peer_sms;
  double bw_local, bw_peer, bw_host;
  int32_t n_host_points, n_peer_points;
  int32_t host_points_sms[UGACHE_CALIB_MAX_POINTS];
  double host_points_bw[UGACHE_CALIB_MAX_POINTS];
  int32_t peer_points_sms[UGACHE_CALIB_MAX_POINTS];
  double peer_points_bw[UGACHE_CALIB_MAX_POINTS];
  uint32_t sample_rows;      /* rows per source per timed launch */
  int32_t reserved;
} ugache_calibration;
ugache_status ugache_calibrate(ugache_ctx *ctx, uint32_t sample_rows, ugache_calibration *out);

/* Core dedication override: SMs for host and for each peer; local gets the
 * rest plus padding.  0 keeps the current value.  Only affects later extracts. */
ugache_status ugache_set_dedication(ugache_ctx *ctx, int32_t host_sms, int32_t peer_sms);

/* ugache_mode; FACTORED by default. */
ugache_status ugache_set_mode(ugache_ctx *ctx, int32_t mode);

/* Tuning options (ugache_set_option); none changes the output bytes.
 *  UGACHE_OPT_HOST_ORDERING (default 1): a dense host bucket is ordered by key range before
 *    it is copied (by every CTA right after the locate pass with UGACHE_OPT_PREORDER, else by
 *    the host CTAs), so the rows in flight cover a small window of host address space
 *    (translation reach of the host aperture); the host SMs then copy
 *    it as two concurrent segments (env UGACHE_HOST_SEGMENTS); 0 = copy in bucket order.
 *  UGACHE_OPT_STAGE_HOST_IO (default 0): 1 = stage pinned host keys/out through device
 *    buffers + cudaMemcpyAsync instead of zero-copy access from the kernels.
 *  UGACHE_OPT_HOST_WARPS (default 12, 1..16): warps per host CTA that read host rows; the
 *    others pad local work (A0 calibration knob).
 *  UGACHE_OPT_DEDICATION: UGACHE_DEDICATE_SMS = the paper's core dedication, whole SMs per
 *    source; UGACHE_DEDICATE_WARPS = the same dedication at warp granularity:
 *    on every SM, UGACHE_OPT_WARP_HOST warps serve the host and UGACHE_OPT_WARP_PEER warps
 *    serve each peer, the others start on local rows.
 *  UGACHE_OPT_WARP_HOST / UGACHE_OPT_WARP_PEER (default 1 / 1): warps per SM in
 *    UGACHE_DEDICATE_WARPS mode; host + (G-1) * peer <= 16.
 *  UGACHE_OPT_HOST_WALK (default 1): when the host bucket is sparse (fewer keys than 2 MB
 *    pages of host source), every SM not dedicated to a peer first walks the batch's keys in
 *    input order and copies the host rows it meets (paced, input-ordered host requests),
 *    then pads local work; 0 = copy the sparse host bucket with dedicated SMs. */
typedef enum {
  UGACHE_OPT_HOST_ORDERING = 0,
  UGACHE_OPT_STAGE_HOST_IO = 1,
  UGACHE_OPT_HOST_WARPS = 2,
  UGACHE_OPT_DEDICATION = 3,
  UGACHE_OPT_WARP_HOST = 4,
  UGACHE_OPT_WARP_PEER = 5,
  UGACHE_OPT_HOST_WALK = 6,
  UGACHE_OPT_FUSED = 7,
  UGACHE_OPT_LOCAL_BULK = 8,
  UGACHE_OPT_EARLY_WALK = 9,
  UGACHE_OPT_STREAM = 10,
  UGACHE_OPT_INLINE = 11,
  UGACHE_OPT_PREORDER = 12
} ugache_option;
/* UGACHE_OPT_PREORDER (default 1): on the two-phase paths (fused / split) with host
 *   ordering on, the locate pass counts each host entry into its key-range histogram, and
 *   right after the locate | gather boundary every CTA of the launch scans the histogram
 *   and scatters its slice of the host bucket into range order; the host-copy warps start
 *   as soon as all CTAs are done.  0 = the host CTAs alone order the bucket after the
 *   boundary (histogram | barrier | scan | scatter | barrier).  Same output bytes. */
/* UGACHE_OPT_STREAM: single-pass extraction (K3, its own cooperative kernel).  Warps take
 *   64-key chunks (a static schedule: warp w takes chunks w, w + W, ...), locate them (A1)
 *   and copy local rows at once (A4: local extraction tolerates every core);
 *   rows of a queued source go to that source's queue, drained only by the SMs dedicated to
 *   it (A2/A3), which locate chunks themselves while their queue is empty.
 *   Rows move through per-lane TMA shared-memory slots (cp.async.bulk in and out, up to
 *   12 KB in flight per warp).  No grid barrier and no bucket round trip for local rows.
 *   0 = off (locate | grid barrier | factored gather); 1 = always; 2 (default) = for rows of
 *   at most 1 KB and no queued peer source (G = 1, or UGACHE_INLINE_PEERS, or a small batch
 *   of at most 32768 keys -- env UGACHE_SMALL_BATCH -- whose peer rows are then read inline:
 *   a latency-bound batch saturates no link, so dedication buys nothing), unless this
 *   batch is expected to have a host bucket dense enough for range-ordered reads: expected
 *   host keys = the last launch's host count scaled to this batch's size (the kernel mirrors
 *   its counts to pinned host memory, so the choice needs no synchronisation), or, before
 *   the first launch of the ctx, n x plan.host_mass_frac.  Ignored with
 *   UGACHE_DEDICATE_WARPS and on the message path.  Timing reports the whole launch as
 *   the gather phase (locate = 0).
 * UGACHE_OPT_INLINE: bit mask of the sources whose rows the locating warp copies itself in
 *   single-pass mode instead of queueing them for dedicated SMs: UGACHE_INLINE_HOST (default)
 *   -- on the B200 box sparse host rows are latency/translation-bound,
 *   so spreading them over every warp beats a bounded set of dedicated warps -- and
 *   UGACHE_INLINE_PEERS (ablation: no peer dedication). */
enum { UGACHE_INLINE_HOST = 1, UGACHE_INLINE_PEERS = 2 };
/* UGACHE_OPT_EARLY_WALK (default 0): 1 = in the fused launch, CTAs left without a locate
 *   tile start the input-order host walk at once, so host rows overlap the locate phase;
 *   the ordered host path then skips the walked keys.  Needs HOST_WALK and HOST_ORDERING on
 *   and SM-granular dedication.  Off by default: measured on B200, concurrent host reads
 *   stretch the locate phase 2-10x.
 * UGACHE_OPT_LOCAL_BULK: local rows (A4) move HBM -> shared -> HBM as TMA cp.async.bulk
 *   copies (no registers per row, ~196 KB in flight per SM) instead of LDG.128 / STG.128
 *   through registers.  0 = never, 1 = always, 2 (default) = unless the host bucket is
 *   dense enough for range-ordered reads (a PCIe-bound batch, where the register path's
 *   local burst interferes less with the host reads), 3 = on CTAs without a host role.
 *   Rows larger than 6 KB always use the register path.
 * UGACHE_OPT_FUSED: 0 = locate+bucket and gather as two launches; 1 = one cooperative
 * launch (grid barrier between the phases); 2 (default) = fused for batches of up to 2^20
 * keys.  Timing (ugache_last_batch_timing) splits the fused launch at its grid barrier
 * (device %globaltimer stamps): locate = start .. barrier, gather = the rest. */
typedef enum { UGACHE_DEDICATE_SMS = 0, UGACHE_DEDICATE_WARPS = 1 } ugache_dedication;
ugache_status ugache_set_option(ugache_ctx *ctx, int32_t option, int64_t value);

/* Per-source key counts of the last extract: per_source[j] for GPU j (j == rank: local),
 * per_source[G] for host (G+1 entries); bad_keys: out-of-range keys.  Synchronises with
 * the last extract.  Per-source hit rates as in Fig. 14. */
ugache_status ugache_last_batch_stats(ugache_ctx *ctx, uint64_t *per_source,
                                      uint64_t *bad_keys);

/* When enabled, extract records CUDA events around its locate+bucket and gather kernels on
 * the extract stream; ugache_last_batch_timing synchronises and returns their durations. */
ugache_status ugache_enable_timing(ugache_ctx *ctx, int32_t on);
ugache_status ugache_last_batch_timing(ugache_ctx *ctx, float *ms_locate, float *ms_gather);

/* Diagnostic phase split of the last fused (K1+K2) launch from the kernel's %globaltimer
 * stamps, in ms from the kernel's start (CTA 0's first instruction): ms[0] = grid barrier
 * released (locate done), ms[1] = host bucket range-ordered (0 if the ordered host path
 * did not run), ms[2] = last host-copy warp done (0 likewise), ms[3] = the last CTA
 * finished its locate tiles, ms[4] = the last CTA of the launch finished.  ms: 5 floats.
 * Synchronises with the last extract.  ESTATE when the last extract was not a fused
 * launch. */
ugache_status ugache_last_batch_phases(ugache_ctx *ctx, float *ms);

/* Per-CTA role timeline of the last fused (K1+K2) launch, for the paper's per-source time
 * split (Fig. 8's picture; §5.3): one CTA per SM, listed in the chip-spreading
 * order the roles are assigned in.  out[5*i .. 5*i+4] for position i = {role source id (GPU
 * j = peer j or this rank = local, num_gpus = host, num_gpus + 1 = warp-granular dedication:
 * every SM mixes roles; the role-done stamp is then 0), CTA start, gather start (grid barrier
 * and host pre-ordering done), own role done (local padding follows), CTA done}, times in
 * ms from the kernel's start.  out: caller-owned, 5 * (SM count) floats (<= 5 * 256);
 * *num_ctas = SM count.  Needs ugache_enable_timing(ctx, 1) before the extract (the stamps
 * cost four %globaltimer reads per CTA).  Synchronises with the last extract.  ESTATE when
 * the last extract was not a fused launch with timing on. */
ugache_status ugache_last_batch_timeline(ugache_ctx *ctx, float *out, int32_t *num_ctas);

/* Number of kernel launches the last extract issued (for launch accounting). */
ugache_status ugache_last_launch_count(const ugache_ctx *ctx, int32_t *launches);

/* Which path the last extract took (roofline accounting): UGACHE_PATH_NONE (n = 0),
 * UGACHE_PATH_SPLIT (K1 + K2, two launches), UGACHE_PATH_FUSED (K1 + grid barrier + K2, one
 * cooperative launch), UGACHE_PATH_SINGLE_PASS (K3), UGACHE_PATH_RANDOM (unfactored K2'). */
enum { UGACHE_PATH_NONE = 0, UGACHE_PATH_SPLIT = 1, UGACHE_PATH_FUSED = 2, UGACHE_PATH_SINGLE_PASS = 3,
       UGACHE_PATH_RANDOM = 4 };
ugache_status ugache_last_extract_path(const ugache_ctx *ctx, int32_t *path);

/* Copy out this GPU's location table (N entries) and slot list (capacity entries) for the
 * placement checker.  Synchronous. */
ugache_status ugache_export_placement(ugache_ctx *ctx, uint64_t *loc, uint64_t *slot_keys,
                                      uint64_t *n_slots);

/* Copy slots [first, first+count) of this GPU's slab to host memory dst (count*R bytes). */
ugache_status ugache_read_slab(ugache_ctx *ctx, uint64_t first, uint64_t count, void *dst);

/* Release device memory, peer mappings and the host-table registration. NULL is a no-op. */
ugache_status ugache_destroy(ugache_ctx *ctx);

const char *ugache_error_string(ugache_status st);
/* Detail text of the ctx's last error (CUDA error name and call, ...); with ctx == NULL,
 * the detail of the calling thread's last failed ugache_init* (the ctx is gone). */
const char *ugache_last_error_message(const ugache_ctx *ctx);
int32_t ugache_version(void);

#ifdef __cplusplus
}
#endif
#endif /* UGACHE_H_ */
