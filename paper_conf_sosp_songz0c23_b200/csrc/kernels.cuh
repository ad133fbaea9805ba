// kernels.cuh -- sm_100a kernels of the factored extraction path.
//
//  K1 locate_bucket_kernel : key -> location-table entry -> per-source bucket
//                            (locate; grouping)
//  K2 factored_gather_kernel : one CTA per SM, CTA role = source; non-local roles copy
//                            their bucket first, then every CTA pads the local bucket
//                            through an atomic cursor (FEM)
//  K3 stream_extract_kernel : single pass -- chunks located and copied at once through
//                            per-lane TMA slots; queued sources drained by their dedicated
//                            SMs from per-CTA sub-queues (no grid barrier, no local bucket)
//  K3r stream_extract_reg_kernel : single pass, register variant for a sparse host bucket
//                            with every source inline (8-key chunks, 8 rows per warp step)
//  K2' random_dispatch_kernel : unfactored peer-based baseline, ablation only
//  K5 fill_kernel          : Filler, host rows -> this GPU's cache slab
//
// Nothing here is a contraction: every step is integer address arithmetic plus 16-byte
// vector copies, so the kernels are written for HBM / NVLink / PCIe bandwidth (coalesced
// 16-B lanes, many independent rows in flight per warp, streaming store hints).
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

#include "ugache.h"

namespace ugk {

constexpr int kMaxSrc = UGACHE_MAX_GPUS + 1;
constexpr int kLocateThreads = 256;
constexpr int kLocateItems = 8;  // keys per thread -> 2048-key tile per CTA
constexpr int kLocateTile = kLocateThreads * kLocateItems;
constexpr int kGatherThreads = 512;  // 16 warps; one CTA per SM (forced via smem)
constexpr int kGatherWarps = kGatherThreads / 32;
constexpr int kRowsInFlight = 8;     // rows per warp per step (U)
constexpr int kLocalChunk = 64;      // rows per local-cursor claim
constexpr int kHostWarps = 12;       // warps per host CTA reading host rows (A0 calibration, round 2)
constexpr uint32_t kFullMask = 0xFFFFFFFFu;
constexpr int kMaxSmId = 256;        // role table size, indexed by %smid

// Device control block (one per ctx).  counts/local_cursor/done/bad are consumed and reset
// by the last CTA of every gather launch, so consecutive extracts need no memset.
struct Ctrl {
  uint32_t counts[kMaxSrc];
  uint32_t local_cursor;
  uint32_t done;
  uint32_t bad;
  uint32_t stat_counts[kMaxSrc];
  uint32_t stat_bad;
  uint32_t host_arrive[2];  // intra-role barriers of the host CTAs
  uint32_t host_cursor;     // dynamic cursor over the range-ordered host bucket
  uint32_t host_seg_cursor[8];  // per-segment cursors (host_segments > 1)
  uint32_t grid_arrive;     // grid barrier of the fused locate+gather kernel
  uint32_t walk_cursor;     // input-order host walk: next key index to claim
  unsigned long long t_start;    // fused kernel: %globaltimer at CTA 0's start (ns)
  unsigned long long t_located;  // fused kernel: %globaltimer when CTA 0 leaves the grid barrier
  unsigned long long t_ordered;  // ordered host path: host CTA 0 done ordering the host bucket
  unsigned long long t_host_done;  // ordered host path: last host-copy warp done (atomicMax)
  // single-pass (streaming) extraction
  uint32_t qhead[kMaxSrc];  // consumer cursor of each source's queue
  uint32_t chunk_cursor;    // next key chunk to locate
  uint32_t keys_done;       // keys whose chunk is fully located (queued or copied)
  uint32_t stat_n;          // keys of the last launch (auto mode: previous batch's host density)
  uint32_t last_stream;     // 1 = the last launch ran the single-pass path
  // host pre-ordering (range histogram built during locate): CTAs done scattering their
  // slice of the host bucket into range order
  uint32_t pre_arrive;
  unsigned long long t_loc_max;   // latest %globaltimer at which a CTA finished its locate tiles
  unsigned long long t_loc_last;  // t_loc_max of the last launch (published by finish_launch)
  unsigned long long t_end;       // %globaltimer when the last CTA of the last launch finished
  // pinned, device-mapped host words {n, host count, launches} written by the last CTA of
  // every launch: the host picks the next batch's path from them without synchronising.
  // The launch count is kept here (mirror_seq) so the kernel only WRITES host memory: a
  // read of the mirror would put a PCIe round trip (and a cold translation) on every
  // launch's tail.
  uint32_t mirror_seq;
  volatile uint32_t *host_mirror;
};

__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Host-bucket range ordering: host rows are read in ascending
// key-range order so that the rows in flight span a small window of host address space
// (IOMMU/ATS translation reach), instead of the whole table.
constexpr int kMaxRanges = 4096;
constexpr uint32_t kHostSortMin = 4096;  // never order fewer host keys than this
constexpr int kRowsPerSmRound = kGatherWarps * kRowsInFlight;  // rows one SM keeps in flight

// Dynamic shared memory of the gather kernels: [host range table | per-warp bulk slots].
// Its size (> half of the SM's 228 KB) also guarantees one gather CTA per SM.
constexpr uint32_t kRangeTabBytes = kMaxRanges * 4;
constexpr uint32_t kBulkWarpBytes = 12 * 1024;          // TMA staging per warp (24 rows of 512 B)
constexpr int kBulkMaxSlots = 32;                       // slots (rows) per warp
constexpr uint32_t kGatherSmem = kRangeTabBytes + kGatherWarps * kBulkWarpBytes;  // 208 KB

struct LocateParams {
  const void *keys;
  const uint64_t *loc;       // N entries, (src << 56) | row
  uint64_t *buckets;         // num_src x bucket_cap entries, (row << 32) | out_idx
  Ctrl *ctrl;
  uint8_t *out;              // for zero rows of out-of-range keys
  uint64_t num_rows;
  uint64_t bucket_cap;
  uint32_t n;
  uint32_t row_bytes;
  int32_t num_src;
  // host pre-ordering: histogram of the host rows' key ranges, built while locating
  int32_t items;             // keys per thread per tile (1..kLocateItems): the fused kernel
                             // sizes tiles so the batch spreads over every CTA
  int32_t hist;              // 1 = count every host entry into range_count
  uint32_t range_shift;      // range = row >> range_shift
  uint32_t *range_count;     // kMaxRanges counters, zero between launches
};

struct GatherParams {
  const uint64_t *buckets;
  Ctrl *ctrl;
  const uint8_t *base[kMaxSrc];  // row base address of each source
  uint8_t *out;
  uint64_t bucket_cap;
  uint32_t row_bytes;
  int32_t num_src;
  int32_t local_src;
  // core dedication, resolved per launch on the device from the counts
  int32_t num_sms;
  int32_t host_sms;                // calibrated host SMs (dense host bucket)
  int32_t host_sms_max;            // cap for a sparse host bucket (S - peers' SMs)
  int32_t peer_sms;                // SMs per peer
  int32_t n_peers;                 // G - 1
  int32_t peer_src[kMaxSrc];       // the peer GPU ids, in role order
  uint32_t host_sort_min;          // host keys needed for range-ordered reads
  uint32_t host_dense_min;         // host keys that make the batch PCIe-bound (the ctx's
                                   // ordering threshold; host_sort_min may be lowered below it)
  uint8_t sm_pos[kMaxSmId];        // position of SM %smid in the chip-spreading order
  // host range ordering
  uint64_t *host_sorted;           // bucket_cap entries of scratch
  uint32_t *range_count;           // kMaxRanges, zero between launches
  uint32_t *range_cursor;          // kMaxRanges, zero between launches
  uint32_t range_shift;            // range = row >> range_shift
  uint32_t n_ranges;               // <= kMaxRanges
  int32_t host_sort;               // 0 = read the host bucket in bucket order
  int32_t host_warps;              // SM mode: warps per host CTA copying host rows;
                                   // warp mode: host warps on every SM
  int32_t peer_warps;              // warp mode: warps per peer on every SM
  int32_t warp_dedication;         // 0 = SM-granular roles (paper), 1 = warp-granular roles
  int32_t host_rows;               // rows per warp step on the unordered host path (1,2,4,8)
  // sparse host bucket: input-order walk over the batch (host_walk)
  const void *keys;                // the batch's keys (device)
  const uint64_t *loc;             // this GPU's location table
  uint64_t num_rows;
  uint32_t n_keys;
  int32_t keys_u32;                // key type: 0 = int64, 1 = uint32
  int32_t host_walk;               // 1 = sparse host buckets use the input-order walk
  int32_t early_walk;              // fused kernel: CTAs without a locate tile walk for host rows
  int32_t local_bulk;              // local rows by TMA bulk copies: 0 never, 1 always, 2 unless
                                   // the host bucket is dense, 3 on CTAs without a host role
  // single-pass extraction (fused kernel only; stream_body)
  int32_t inline_host;             // single pass: host rows copied by the locating warp
  int32_t inline_peer;             // single pass: peer rows copied by the locating warp (ablation)
  uint64_t *queues;                // num_src x bucket_cap entries, ~0 between launches
  int32_t stream_bulk;             // single pass: inline rows through TMA slots (StreamSlots)
  int32_t stream_k;                // single pass: keys per lane per chunk (1 or 2)
  int32_t stream_ck;               // single pass: lanes holding a key per step (32; 4..16 for
                                   // small batches, so every warp gets a chunk)
  int32_t stream_host_last;        // single pass: non-local inline rows after the local ones
  int32_t stream_host_cap;         // single pass: non-local rows in flight per warp (0 = slots)
  int32_t stream_static;           // single pass: static chunk schedule instead of the cursor
  int32_t stream_nap;              // single pass: ns a warp sleeps when all its slots are in flight
  int32_t stream_prefetch;         // single pass: locating warps prefetch the next chunks' keys/entries
  int32_t stream_queues;           // single pass: some source is queued (consumers exist)
  uint64_t queue_cap;              // single pass: entries per source in `queues`
  int32_t stream_regstore;         // single pass: slots leave by warp-wide stores, not bulk copies
  int32_t stream_peer_warps;       // single pass: consumer warps per peer-dedicated CTA
  int32_t local_sms;               // two-phase, dense host: SMs copying local rows (0 = all)
  int32_t stream_group;            // single pass: chunks per group with non-local rows first (<= 1 off)
  uint32_t *qctr;                  // single pass: [2][kMaxSrc][kMaxSmId] sub-queue counts / heads
  int32_t preorder;                // the locate pass built the host range histogram: every CTA
                                   // scatters a slice of the host bucket (preorder_host)
  int32_t hist_smem;               // fused kernel: the histogram is aggregated per CTA in shared
                                   // memory before the global atomics
  int32_t host_segments;           // ordered host copy: the ordered bucket is split into this many
                                   // segments read concurrently (1 = one cursor, in order)
  int32_t local_pace;              // dense host bucket: ns a local-copy warp sleeps after each
                                   // chunk (spreads the local burst over the host-bound step)
  int32_t local_warps;             // dense host bucket: warps per non-host SM copying local rows
                                   // (0 = all 16)
  unsigned long long *timeline;    // per-CTA role timeline (timing on): kTimelineWords per
                                   // chip position, see gather_body; nullptr = off
};
// Per-CTA role timeline (fused kernel, diagnostics): [role source, CTA start, gather start
// (after the grid barrier and pre-ordering), own role done (last warp), CTA done (last
// warp)], %globaltimer ns; zeroed by the host before each timed launch.
constexpr int kTimelineWords = 5;

struct RandomParams {
  const void *keys;
  const uint64_t *loc;
  Ctrl *ctrl;
  const uint8_t *base[kMaxSrc];
  uint8_t *out;
  uint64_t num_rows;
  uint32_t n;
  uint32_t row_bytes;
  int32_t num_src;
};

struct FillParams {
  const uint64_t *slot_idx;   // destination slot of entry i (nullptr: slot i)
  const uint64_t *slot_keys;
  const uint8_t *table;  // device-mapped host table
  uint8_t *slab;
  uint64_t n_slots;
  uint32_t row_bytes;
};

// ---------------------------------------------------------------------------- helpers
// 1 = row payload reads (LDG.128 and TMA bulk) carry an L2 evict_first policy, so the
// streamed rows do not push longer-lived lines (location-table sectors, the GMMU's cached
// translations of the host aperture) out of L2 between batches.  Set at ctx init.
__device__ __constant__ int c_row_evict_first;
// 1 (default) = location-table lookups carry the L2 evict_first policy: the random 8-B
// lookups (one >= 64-B line each) then stop displacing longer-lived L2 lines between batches
// -- on the B200 box that keeps the host aperture's translation state warm from one batch
// to the next (steady state)
__device__ __constant__ int c_lt_evict_first;

__device__ __forceinline__ uint64_t l2_policy_evict_first() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ uint4 ld_nc_v4(const void *p) {
  uint4 r;
  if (c_row_evict_first) {
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p), "l"(l2_policy_evict_first()));
  } else {
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                 : "l"(p));
  }
  return r;
}
__device__ __forceinline__ void st_cs_v4(void *p, const uint4 &v) {
  asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y),
               "r"(v.z), "r"(v.w)
               : "memory");
}
__device__ __forceinline__ uint64_t ld_lt_u64(const uint64_t *p) {  // location-table lookup
  uint64_t r;
  if (c_lt_evict_first) {
    asm volatile("ld.global.nc.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(r) : "l"(p), "l"(l2_policy_evict_first()));
  } else {
    asm volatile("ld.global.nc.u64 %0, [%1];" : "=l"(r) : "l"(p));
  }
  return r;
}
__device__ __forceinline__ uint64_t ld_nc_u64(const uint64_t *p) {
  uint64_t r;
  asm volatile("ld.global.nc.u64 %0, [%1];" : "=l"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// Warp copies up to U rows.  ent: bucket entries (row << 32 | out_idx), read by lanes < U.
// All U loads of a lane are issued before its stores (U * 16 B in flight per lane per
// vector step).  Rows of R bytes = V 16-byte vectors; lanes stride over V.
template <int U>
__device__ __forceinline__ void copy_rows(const uint8_t *__restrict__ base,
                                          uint8_t *__restrict__ out, uint32_t R,
                                          const uint64_t *__restrict__ ent, int nvalid,
                                          int lane) {
  const uint64_t e = (lane < nvalid) ? ent[lane] : 0ull;
  uint64_t eu[U];
#pragma unroll
  for (int u = 0; u < U; ++u) eu[u] = __shfl_sync(kFullMask, e, u);
  const uint32_t V = R >> 4;
  for (uint32_t j = lane; j < V; j += 32) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (u < nvalid) v[u] = ld_nc_v4(base + (eu[u] >> 32) * (uint64_t)R + (uint64_t)j * 16u);
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (u < nvalid)
        st_cs_v4(out + (eu[u] & 0xFFFFFFFFull) * (uint64_t)R + (uint64_t)j * 16u, v[u]);
  }
}

__device__ __forceinline__ void zero_row(uint8_t *dst, uint32_t R) {
  const uint4 z = make_uint4(0, 0, 0, 0);
  for (uint32_t j = 0; j < (R >> 4); ++j) *reinterpret_cast<uint4 *>(dst + (uint64_t)j * 16) = z;
}

template <typename KeyT>
__device__ __forceinline__ bool key_in_range(KeyT k, uint64_t N) {
  if constexpr (sizeof(KeyT) == 8) return k >= 0 && (uint64_t)k < N;
  else return (uint64_t)k < N;
}

// Last CTA of a gather launch publishes stats and re-arms the control block.
// The last CTA of a launch publishes the batch's statistics and re-arms the control block
// for the next launch.  Its threads split the work (one source per thread, the scalar resets
// on another warp): a single thread doing it all chained ~20 dependent L2 round trips (and,
// before mirror_seq, a PCIe read) onto every launch's tail -- 5-7 us at G = 8.
__device__ __forceinline__ void finish_launch(Ctrl *ctrl, int num_src, uint32_t n, uint32_t streamed) {
  __shared__ uint32_t s_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    s_last = atomicAdd(&ctrl->done, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  volatile Ctrl *c = ctrl;
  const int t = threadIdx.x;
  if (t < num_src) {
    const uint32_t v = c->counts[t];
    c->stat_counts[t] = v;
    c->counts[t] = 0;
    c->qhead[t] = 0;
    if (t == num_src - 1 && c->host_mirror) c->host_mirror[1] = v;
  } else if (t >= 32 && t < 40) {
    c->host_seg_cursor[t - 32] = 0;
  } else if (t == 64) {
    c->stat_bad = c->bad;
    c->bad = 0;
    c->t_loc_last = c->t_loc_max;
    c->t_loc_max = 0;
  } else if (t == 96) {
    c->chunk_cursor = 0;
    c->keys_done = 0;
    c->stat_n = n;
    c->last_stream = streamed;
    c->local_cursor = 0;
    c->host_arrive[0] = 0;
    c->host_arrive[1] = 0;
    c->host_cursor = 0;
    c->grid_arrive = 0;
    c->walk_cursor = 0;
    c->pre_arrive = 0;
  }
  __syncthreads();
  if (t == 0) {
    if (c->host_mirror) {
      const uint32_t seq = c->mirror_seq + 1;
      c->mirror_seq = seq;
      c->host_mirror[0] = n;
      c->host_mirror[2] = seq;
    }
    c->t_end = globaltimer_ns();
    __threadfence();
    c->done = 0;
  }
}

// ---------------------------------------------------------------------------- K1
// One tile of K1 (THREADS x kLocateItems keys) processed by one CTA.  s_cnt / s_base are
// shared arrays of kMaxSrc entries; the function starts and ends with a CTA barrier.
template <typename KeyT, int THREADS>
__device__ __forceinline__ void locate_tile(const LocateParams &p, uint64_t tile,
                                            uint32_t *s_cnt, uint32_t *s_base,
                                            uint32_t *s_hist = nullptr) {
  const int tid = threadIdx.x, lane = tid & 31;
  __syncthreads();
  if (tid < kMaxSrc) s_cnt[tid] = 0;
  __syncthreads();
  const KeyT *keys = static_cast<const KeyT *>(p.keys);
  const int items = p.items;
  const uint64_t tile0 = tile * (uint64_t)(THREADS * items);

  KeyT k[kLocateItems];
  uint64_t e[kLocateItems];
#pragma unroll
  for (int it = 0; it < kLocateItems; ++it) {  // coalesced key loads
    const uint64_t i = tile0 + (uint64_t)it * THREADS + tid;
    k[it] = (it < items && i < p.n) ? keys[i] : (KeyT)0;
  }
#pragma unroll
  for (int it = 0; it < kLocateItems; ++it) {  // random location-table reads, all in flight
    const uint64_t i = tile0 + (uint64_t)it * THREADS + tid;
    e[it] = (it < items && i < p.n && key_in_range<KeyT>(k[it], p.num_rows)) ? ld_lt_u64(p.loc + (uint64_t)k[it])
                                                                             : ~0ull;
  }
  int src[kLocateItems];
  uint32_t pos[kLocateItems];
  uint32_t nbad = 0;
#pragma unroll
  for (int it = 0; it < kLocateItems; ++it) {
    const uint64_t i = tile0 + (uint64_t)it * THREADS + tid;
    int s = -1;
    if (it < items && i < p.n) {
      if (e[it] != ~0ull) {
        s = (int)(e[it] >> UGACHE_LOC_SRC_SHIFT);
      } else {
        zero_row(p.out + i * (uint64_t)p.row_bytes, p.row_bytes);  // out-of-range key
        ++nbad;
      }
    }
    // warp-aggregated per-source slot reservation in shared memory
    const uint32_t peers = __match_any_sync(kFullMask, s);
    const int leader = __ffs(peers) - 1;
    uint32_t b = 0;
    if (s >= 0 && lane == leader) b = atomicAdd(&s_cnt[s], (uint32_t)__popc(peers));
    b = __shfl_sync(kFullMask, b, leader);
    src[it] = s;
    pos[it] = b + __popc(peers & lanemask_lt());
  }
  if (nbad) atomicAdd(&p.ctrl->bad, nbad);
  __syncthreads();
  if (tid < p.num_src && s_cnt[tid]) s_base[tid] = atomicAdd(&p.ctrl->counts[tid], s_cnt[tid]);
  __syncthreads();
#pragma unroll
  for (int it = 0; it < kLocateItems; ++it) {
    if (src[it] >= 0) {
      const uint64_t i = tile0 + (uint64_t)it * THREADS + tid;
      const uint32_t row = (uint32_t)(e[it] & UGACHE_LOC_ROW_MASK);
      p.buckets[(uint64_t)src[it] * p.bucket_cap + s_base[src[it]] + pos[it]] =
          ((uint64_t)row << 32) | (uint64_t)i;
      if (p.hist && src[it] == p.num_src - 1)
        atomicAdd(s_hist ? &s_hist[row >> p.range_shift] : &p.range_count[row >> p.range_shift], 1u);
    }
  }
}

template <typename KeyT>
__global__ void __launch_bounds__(kLocateThreads)
    locate_bucket_kernel(const LocateParams p) {
  __shared__ uint32_t s_cnt[kMaxSrc];
  __shared__ uint32_t s_base[kMaxSrc];
  locate_tile<KeyT, kLocateThreads>(p, blockIdx.x, s_cnt, s_base);
}

// Barrier among the `n` CTAs of one role.  The gather kernel is launched cooperatively
// (one CTA per SM), so every CTA of a role is co-resident.
__device__ __forceinline__ void role_barrier(uint32_t *ctr, uint32_t n) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(ctr, 1u);
    uint32_t v;
    do {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
      if (v < n) __nanosleep(64);
    } while (v < n);
  }
  __syncthreads();
}

// Wait (without arriving) until n CTAs have arrived at a role_barrier counter.
__device__ __forceinline__ void role_wait(const uint32_t *ctr, uint32_t n) {
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t v;
    do {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
      if (v < n) __nanosleep(64);
    } while (v < n);
  }
  __syncthreads();
}

// Exclusive scan of src[0..n) (global) into dst[0..n) (shared); n <= kMaxRanges.
__device__ __forceinline__ void block_exclusive_scan(const uint32_t *src, uint32_t *dst, uint32_t n) {
  __shared__ uint32_t s_warp[32];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nt = blockDim.x;
  const uint32_t per = (n + nt - 1) / nt;
  const uint32_t lo = min(n, tid * per), hi = min(n, lo + per);
  uint32_t sum = 0;
  for (uint32_t i = lo; i < hi; ++i) sum += src[i];
  uint32_t incl = sum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(kFullMask, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) s_warp[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    const int nw = nt >> 5;
    uint32_t w = lane < nw ? s_warp[lane] : 0, wi = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(kFullMask, wi, o);
      if (lane >= o) wi += y;
    }
    if (lane < nw) s_warp[lane] = wi - w;
  }
  __syncthreads();
  uint32_t run = s_warp[warp] + incl - sum;
  for (uint32_t i = lo; i < hi; ++i) {
    const uint32_t v = src[i];
    dst[i] = run;
    run += v;
  }
  __syncthreads();
}

// In-order copy of the range-ordered host bucket: warps claim U consecutive entries from a
// shared cursor (next claim prefetched), so the rows in flight are the most recent claims.
template <int U>
__device__ __forceinline__ void host_copy_ordered(const GatherParams &p, uint32_t cnt, int lane,
                                                  uint32_t gwarp) {
  const uint8_t *base = p.base[p.num_src - 1];
  const int K = min(max(p.host_segments, 1), 8);
  if (K > 1) {
    // K contiguous segments of the ordered bucket read at once (warp w starts on segment
    // w mod K, then helps the others): the rows in flight mix dense and sparse key ranges
    for (int t = 0; t < K; ++t) {
      const uint32_t sg = (gwarp + (uint32_t)t) % (uint32_t)K;
      const uint32_t lo = (uint32_t)((uint64_t)cnt * sg / K), hi = (uint32_t)((uint64_t)cnt * (sg + 1) / K);
      while (true) {
        uint32_t e0 = 0;
        if (lane == 0) e0 = lo + atomicAdd(&p.ctrl->host_seg_cursor[sg], (uint32_t)U);
        e0 = __shfl_sync(kFullMask, e0, 0);
        if (e0 >= hi) break;
        copy_rows<U>(base, p.out, p.row_bytes, p.host_sorted + e0, (int)min((uint32_t)U, hi - e0), lane);
      }
    }
    return;
  }
  uint32_t next = 0;
  if (lane == 0) next = atomicAdd(&p.ctrl->host_cursor, (uint32_t)U);
  next = __shfl_sync(kFullMask, next, 0);
  while (next < cnt) {
    const uint32_t e0 = next;
    if (lane == 0) next = atomicAdd(&p.ctrl->host_cursor, (uint32_t)U);
    next = __shfl_sync(kFullMask, next, 0);
    copy_rows<U>(base, p.out, p.row_bytes, p.host_sorted + e0, (int)min((uint32_t)U, cnt - e0), lane);
  }
}

// Range ordering of the host bucket into p.host_sorted: histogram -> barrier -> scan ->
// scatter -> barrier.  CTAs h = 0..H-1 cooperate with all their threads.  Entries whose key
// index is below `walked` were already copied by the input-order walk (fused kernel, before
// its grid barrier) and are dropped.  Returns the number of ordered entries.
__device__ __forceinline__ uint32_t host_order(const GatherParams &p, const uint64_t *b,
                                               uint32_t cnt, int h, int H, uint32_t *s_tab,
                                               uint32_t walked) {
  const int tid = threadIdx.x;
  const uint32_t lo = (uint32_t)((uint64_t)cnt * h / H), hi = (uint32_t)((uint64_t)cnt * (h + 1) / H);
  for (uint32_t i = tid; i < p.n_ranges; i += blockDim.x) s_tab[i] = 0;
  __syncthreads();
  for (uint32_t e = lo + tid; e < hi; e += blockDim.x) {
    const uint64_t ent = b[e];
    if ((uint32_t)ent >= walked) atomicAdd(&s_tab[(uint32_t)(ent >> 32) >> p.range_shift], 1u);
  }
  __syncthreads();
  for (uint32_t i = tid; i < p.n_ranges; i += blockDim.x)
    if (s_tab[i]) atomicAdd(&p.range_count[i], s_tab[i]);
  role_barrier(&p.ctrl->host_arrive[0], (uint32_t)H);
  block_exclusive_scan(p.range_count, s_tab, p.n_ranges);
  const uint32_t total = s_tab[p.n_ranges - 1] + p.range_count[p.n_ranges - 1];
  for (uint32_t e = lo + tid; e < hi; e += blockDim.x) {
    const uint64_t ent = b[e];
    if ((uint32_t)ent < walked) continue;
    const uint32_t r = (uint32_t)(ent >> 32) >> p.range_shift;
    p.host_sorted[s_tab[r] + atomicAdd(&p.range_cursor[r], 1u)] = ent;
  }
  role_barrier(&p.ctrl->host_arrive[1], (uint32_t)H);
  {  // every host CTA is past its scatter: re-arm my slice of the range counters
    const uint32_t zlo = p.n_ranges * h / H, zhi = p.n_ranges * (h + 1) / H;
    for (uint32_t i = zlo + tid; i < zhi; i += blockDim.x) {
      p.range_count[i] = 0;
      p.range_cursor[i] = 0;
    }
  }
  return total;
}

// Range ordering without the host CTAs' serial prefix (gp.preorder): the locate pass already
// counted every host entry into range_count, so right after the locate | gather boundary
// EVERY CTA of the launch scans the counts (4096 entries, on-chip) and scatters its
// 1/gridDim slice of the host bucket into range order, then arrives on pre_arrive.  The
// host-copy warps start once all CTAs arrived (host_role_preordered) -- a few microseconds
// instead of the host CTAs' histogram | barrier | scan | scatter | barrier sequence.  With a
// sparse host bucket the histogram is unused and each CTA re-arms its slice of it.
__device__ __forceinline__ void preorder_host(const GatherParams &p, uint32_t *s_tab, uint32_t pos,
                                              uint32_t S) {
  const int tid = threadIdx.x;
  const int host_src = p.num_src - 1;
  const uint32_t cnt = *(volatile const uint32_t *)&p.ctrl->counts[host_src];
  if (cnt < p.host_sort_min) {
    const uint32_t zlo = p.n_ranges * pos / S, zhi = p.n_ranges * (pos + 1) / S;
    for (uint32_t i = zlo + tid; i < zhi; i += blockDim.x) p.range_count[i] = 0;
    return;
  }
  block_exclusive_scan(p.range_count, s_tab, p.n_ranges);
  const uint64_t *b = p.buckets + (uint64_t)host_src * p.bucket_cap;
  const uint32_t lo = (uint32_t)((uint64_t)cnt * pos / S), hi = (uint32_t)((uint64_t)cnt * (pos + 1) / S);
  // The CTA reserves one block per non-empty range (one global atomic per (CTA, range)
  // instead of one per entry: the hot head of the tier puts thousands of a batch's host
  // keys in its first ranges, and per-entry atomics on their cursors serialised), then
  // places its entries with shared-memory cursors.  s_loc lives in the first TMA staging
  // buffers, idle until the gather starts (after this function's last barrier).
  uint32_t *s_loc = s_tab + kMaxRanges;
  for (uint32_t i = tid; i < p.n_ranges; i += blockDim.x) s_loc[i] = 0;
  __syncthreads();
  for (uint32_t e = lo + tid; e < hi; e += blockDim.x)
    atomicAdd(&s_loc[(uint32_t)(b[e] >> 32) >> p.range_shift], 1u);
  __syncthreads();
  for (uint32_t i = tid; i < p.n_ranges; i += blockDim.x) {
    const uint32_t c = s_loc[i];
    if (c) s_loc[i] = s_tab[i] + atomicAdd(&p.range_cursor[i], c);
  }
  __syncthreads();
  for (uint32_t e = lo + tid; e < hi; e += blockDim.x) {
    const uint64_t ent = b[e];
    p.host_sorted[atomicAdd(&s_loc[(uint32_t)(ent >> 32) >> p.range_shift], 1u)] = ent;
  }
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    atomicAdd(&p.ctrl->pre_arrive, 1u);
  }
}

// After preorder_host: wait until every CTA scattered its slice, then re-arm slice h of H of
// the range counters (every CTA has read range_count and bumped range_cursor by now).
__device__ __forceinline__ void preorder_wait(const GatherParams &p, uint32_t h, uint32_t H) {
  role_wait(&p.ctrl->pre_arrive, gridDim.x);
  const uint32_t zlo = p.n_ranges * h / H, zhi = p.n_ranges * (h + 1) / H;
  for (uint32_t i = zlo + threadIdx.x; i < zhi; i += blockDim.x) {
    p.range_count[i] = 0;
    p.range_cursor[i] = 0;
  }
}

// Input-order host walk (sparse host buckets, and the fused kernel's early walk): warps
// claim kWalkChunk consecutive keys from a shared cursor, re-read their location entries and
// copy the host rows among them.  Stops when the keys run out or, with stop != nullptr, once
// *stop reaches stop_at (checked between claims, so every claimed chunk completes).
constexpr uint32_t kWalkChunk = 64;
__device__ __forceinline__ void host_walk_copy(const GatherParams &p, int warp, int lane,
                                          const uint32_t *stop, uint32_t stop_at) {
  __shared__ uint64_t s_ent[kGatherWarps][kRowsInFlight];
  const int host_src = p.num_src - 1;
  while (true) {
    uint32_t c0 = 0;
    if (lane == 0) {
      bool go = true;
      if (stop) {
        uint32_t v;
        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(stop) : "memory");
        go = v < stop_at;
      }
      c0 = go ? atomicAdd(&p.ctrl->walk_cursor, kWalkChunk) : 0xFFFFFFFFu;
    }
    c0 = __shfl_sync(kFullMask, c0, 0);
    if (c0 >= p.n_keys) return;
    const uint32_t c1 = min(p.n_keys, c0 + kWalkChunk);
    for (uint32_t e0 = c0; e0 < c1; e0 += kRowsInFlight) {
      const int nv = (int)min((uint32_t)kRowsInFlight, c1 - e0);
      uint64_t ent = ~0ull;
      if (lane < nv) {
        const uint64_t i = e0 + lane;
        const int64_t k = p.keys_u32 ? (int64_t)static_cast<const uint32_t *>(p.keys)[i]
                                     : static_cast<const int64_t *>(p.keys)[i];
        if (k >= 0 && (uint64_t)k < p.num_rows) {
          const uint64_t l = ld_lt_u64(p.loc + k);
          if ((int)(l >> UGACHE_LOC_SRC_SHIFT) == host_src) ent = ((l & UGACHE_LOC_ROW_MASK) << 32) | i;
        }
      }
      const uint32_t m = __ballot_sync(kFullMask, ent != ~0ull);
      if (ent != ~0ull) s_ent[warp][__popc(m & lanemask_lt())] = ent;  // compact to lanes 0..
      __syncwarp();
      if (m) copy_rows<kRowsInFlight>(p.base[host_src], p.out, p.row_bytes, s_ent[warp], __popc(m), lane);
      __syncwarp();
    }
  }
}

// Host role (SM-granular dedication) with range ordering: the host CTAs order the bucket,
// then `host_warps` warps of each copy rows in order; the other warps pad local work.
__device__ __forceinline__ void host_role_sorted(const GatherParams &p, const uint64_t *b,
                                                 uint32_t cnt, int h, int H, uint32_t *s_tab,
                                                 uint32_t walked) {
  if (p.preorder) preorder_wait(p, (uint32_t)h, (uint32_t)H);  // ordered by every CTA already
  else cnt = host_order(p, b, cnt, h, H, s_tab, walked);
  if (h == 0 && threadIdx.x == 0) p.ctrl->t_ordered = globaltimer_ns();  // phase stamp
  if ((int)(threadIdx.x >> 5) >= p.host_warps) return;  // window control
  host_copy_ordered<kRowsInFlight>(p, cnt, threadIdx.x & 31, (uint32_t)(h * p.host_warps) + (threadIdx.x >> 5));
  if ((threadIdx.x & 31) == 0) atomicMax(&p.ctrl->t_host_done, globaltimer_ns());
}

// Static warp striding of W warps (this one = gw) over a bucket of cnt rows of one source,
// U rows per warp step.
template <int U>
__device__ __forceinline__ void stride_copy_u(const GatherParams &p, const uint64_t *b, uint32_t cnt,
                                              const uint8_t *base, uint32_t gw, uint32_t W, int lane) {
  for (uint32_t e0 = gw * U; e0 < cnt; e0 += W * U)
    copy_rows<U>(base, p.out, p.row_bytes, b + e0, (int)min((uint32_t)U, cnt - e0), lane);
}

__device__ __forceinline__ void stride_copy(const GatherParams &p, const uint64_t *b, uint32_t cnt,
                                            const uint8_t *base, uint32_t gw, uint32_t W, int lane,
                                            int rows = kRowsInFlight) {
  switch (rows) {
    case 1: stride_copy_u<1>(p, b, cnt, base, gw, W, lane); break;
    case 2: stride_copy_u<2>(p, b, cnt, base, gw, W, lane); break;
    case 4: stride_copy_u<4>(p, b, cnt, base, gw, W, lane); break;
    default: stride_copy_u<kRowsInFlight>(p, b, cnt, base, gw, W, lane); break;
  }
}

// ---------------------------------------------------------------------------- TMA bulk
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  }
}
// global -> shared, completion counted on bar (bytes multiple of 16, 16-B aligned)
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
  if (c_row_evict_first) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], "
        "%4;" ::"r"(smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(l2_policy_evict_first())
        : "memory");
  } else {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
  }
}
// shared -> global, tracked by this thread's bulk groups; policy: an L2 cache policy
// (evict_first for the output stream, like st.global.cs on the register path)
__device__ __forceinline__ void bulk_s2g(void *dst, const void *src, uint32_t bytes, uint64_t policy) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(dst),
               "r"(smem_u32(src)), "r"(bytes), "l"(policy)
               : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ uint64_t l2_evict_first_policy() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ void bulk_wait_read_all() {
  asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
// cp.async (LDGSTS) of one 4/8-byte word into shared memory: a load with no register held
// while it is in flight (single-pass locate pipeline, stream_prefetch = 2)
__device__ __forceinline__ void cp_async_word(void *smem, const void *g, int bytes, bool evict_first) {
  if (bytes == 8 && evict_first)
    asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 8, %2;" ::"r"(smem_u32(smem)), "l"(g),
                 "l"(l2_policy_evict_first())
                 : "memory");
  else if (bytes == 8)
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(smem)), "l"(g) : "memory");
  else
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(smem)), "l"(g) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// Rows per local-cursor claim: kLocalChunk for big buckets; smaller (a multiple of 8, at
// least 8) when the bucket would leave warps of the grid without a claim, so a medium batch
// spreads its local rows over every warp instead of chaining 8 dependent steps on a few.
__device__ __forceinline__ uint32_t local_chunk_rows(uint32_t cnt, int num_sms) {
  const uint32_t warps = (uint32_t)num_sms * kGatherWarps;
  const uint32_t per = (cnt + warps - 1) / warps;
  return min((uint32_t)kLocalChunk, max(8u, (per + 7u) & ~7u));
}

// Local bucket drained by TMA bulk copies (A4 on B200): each row goes HBM -> shared memory
// -> HBM as two cp.async.bulk operations, no registers hold row data, so one SM keeps
// 16 warps x 24 rows = 196 KB in flight (LDG.128 at 128 registers/thread: 64 KB).  Lane u
// of a warp owns slots {d*U + u}: step g loads group g (U consecutive bucket entries of the
// warp's current chunk) into buffer g % depth and stores group g - (depth - 1) from its
// buffer, so depth - 1 groups of loads overlap every store.  Chunks come from the same
// atomic cursor as the LDG path (padding by every SM whose own group drained).
__device__ __forceinline__ void local_bulk_copy(const GatherParams &p, uint8_t *wsmem, uint64_t *bars,
                                                uint32_t *oidx, int lane) {
  const uint32_t R = p.row_bytes;
  const int slots = min(kBulkMaxSlots, (int)(kBulkWarpBytes / R));
  const int U = min(kRowsInFlight, slots / 2);
  const int depth = slots / U;
  const uint32_t cnt = p.ctrl->counts[p.local_src];
  const uint64_t *b = p.buckets + (uint64_t)p.local_src * p.bucket_cap;
  const uint8_t *base = p.base[p.local_src];
  if (lane < U)
    for (int d = 0; d < depth; ++d) mbar_init(&bars[d * U + lane], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const uint64_t out_policy = l2_evict_first_policy();
  uint32_t phase = 0;     // bit d: parity of buffer d's barrier for this lane
  uint32_t g = 0;         // groups issued by this warp
  uint32_t valid = 0;     // bit d: this lane loaded a row into buffer d, store pending
  auto store_group = [&](uint32_t h) {  // wait for group h's row and send it to out
    const int d = (int)(h % (uint32_t)depth);
    if (lane < U && (valid >> d & 1u)) {
      const int slot = d * U + lane;
      mbar_wait(&bars[slot], (phase >> d) & 1u);
      phase ^= 1u << d;
      bulk_s2g(p.out + (uint64_t)oidx[slot] * R, wsmem + (uint32_t)slot * R, R, out_policy);
      valid &= ~(1u << d);
    }
  };
  uint32_t next = 0;
  const uint32_t lc = local_chunk_rows(cnt, p.num_sms);
  if (lane == 0) next = atomicAdd(&p.ctrl->local_cursor, lc);
  next = __shfl_sync(kFullMask, next, 0);
  while (next < cnt) {
    const uint32_t c0 = next, c1 = min(cnt, c0 + lc);
    if (lane == 0) next = atomicAdd(&p.ctrl->local_cursor, lc);  // prefetch claim
    next = __shfl_sync(kFullMask, next, 0);
    for (uint32_t e0 = c0; e0 < c1; e0 += (uint32_t)U, ++g) {
      const int d = (int)(g % (uint32_t)depth);
      if (lane < U && e0 + lane < c1) {
        const uint64_t ent = b[e0 + lane];
        const int slot = d * U + lane;
        bulk_wait_read_all();  // this slot's previous store has left shared memory
        oidx[slot] = (uint32_t)(ent & 0xFFFFFFFFull);
        mbar_expect_tx(&bars[slot], R);
        bulk_g2s(wsmem + (uint32_t)slot * R, base + (ent >> 32) * (uint64_t)R, R, &bars[slot]);
        valid |= 1u << d;
      }
      if (g + 1 >= (uint32_t)depth) store_group(g + 1 - depth);
    }
  }
  for (uint32_t h = g + 1 > (uint32_t)depth ? g + 1 - depth : 0; h < g; ++h) store_group(h);
  bulk_wait_all();
}

// ---------------------------------------------------------------------------- K2
__device__ __forceinline__ void gather_body(const GatherParams &p, uint32_t *s_dyn) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // Role of this CTA = role of the SM it runs on (one CTA per SM, cooperative launch):
  // the B200 replacement of the paper's MPS core limits.  SMs are taken in
  // the order of a chip-spreading permutation (sm_pos): [host | peer_0 | ... | local].
  uint32_t smid;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  const int pos = smid < (uint32_t)kMaxSmId ? p.sm_pos[smid] : p.num_sms - 1;
  const int host_src = p.num_src - 1;
  if (p.preorder) preorder_host(p, s_dyn, blockIdx.x, gridDim.x);
  unsigned long long *tl = p.timeline ? p.timeline + pos * kTimelineWords : nullptr;
  if (tl && threadIdx.x == 0) tl[2] = globaltimer_ns();
  const uint32_t n_host = p.ctrl->counts[host_src];
  const bool host_dense = p.host_sort && n_host >= p.host_sort_min;
  const uint32_t R = p.row_bytes;
  // keys [0, walked) were walked for host rows before the fused kernel's grid barrier
  const uint32_t walked = min(*(volatile const uint32_t *)&p.ctrl->walk_cursor, p.n_keys);
  bool host_cta = false;  // SM-granular mode: this CTA holds a host role

  if (p.warp_dedication) {
    if (tl && threadIdx.x == 0) tl[0] = (unsigned long long)p.num_src;  // mixed roles (timeline)
    // Warp-granular dedication: on EVERY SM, warps [0, hw) serve the
    // host and the next pw warps each peer; the rest start on local work.  Concurrency per
    // slow source stays bounded (S*hw or S*pw warps) while the requests come from all GPCs
    // and no SM idles behind a slow link.
    const int S = p.num_sms, hw = p.host_warps, pw = p.peer_warps;
    const uint64_t *bh = p.buckets + (uint64_t)host_src * p.bucket_cap;
    uint32_t n_ord = 0;
    if (host_dense && p.preorder) {
      preorder_wait(p, blockIdx.x, gridDim.x);
      n_ord = n_host;
    } else if (host_dense) {
      n_ord = host_order(p, bh, n_host, pos, S, s_dyn, 0);
    }
    if (warp < hw) {
      if (host_dense) host_copy_ordered<kRowsInFlight>(p, n_ord, lane, (uint32_t)(pos * hw + warp));
      else stride_copy(p, bh, n_host, p.base[host_src], (uint32_t)(pos * hw + warp), (uint32_t)(S * hw), lane,
                       p.host_rows);
    } else if (warp < hw + p.n_peers * pw) {
      const int j = p.peer_src[(warp - hw) / pw];
      stride_copy(p, p.buckets + (uint64_t)j * p.bucket_cap, p.ctrl->counts[j], p.base[j],
                  (uint32_t)(pos * pw + (warp - hw) % pw), (uint32_t)(S * pw), lane);
    }
  } else {
  // Host SMs: the calibrated count when the host bucket is dense enough for ordered reads
  // (throughput-bound); otherwise enough SMs to put the whole bucket in flight in about one
  // round (latency-bound), capped so every peer keeps its dedicated SMs.  Every CTA derives
  // the same split from the same counts.
  const bool host_walk = p.host_walk && !host_dense && n_host > 0;
  int H = p.host_sms;
  if (host_walk)
    H = p.host_sms_max;  // every SM not dedicated to a peer walks the batch for host rows
  else if (!host_dense)
    H = max(H, min(p.host_sms_max, (int)((n_host + kRowsPerSmRound - 1) / kRowsPerSmRound)));
  int my_src, my_idx, role_ctas;
  if (pos < H) {
    my_src = host_src, my_idx = pos, role_ctas = H;
    host_cta = true;
  } else if (pos - H < p.n_peers * p.peer_sms) {
    my_src = p.peer_src[(pos - H) / p.peer_sms];
    my_idx = (pos - H) % p.peer_sms, role_ctas = p.peer_sms;
  } else {
    my_src = p.local_src, my_idx = 0, role_ctas = 0;
  }

  if (my_src == host_src && host_walk) {
    // Sparse host bucket: the host SMs walk the batch's keys in input order (re-reading
    // their location entries) and copy the host rows they meet, continuing where the fused
    // kernel's early walk stopped.  Measured on the B200 box, sparse cold host rows are read
    // ~1.6x faster in this paced input order than from the dense host bucket, whose rows
    // would all be requested at once.
    host_walk_copy(p, warp, lane, nullptr, 0);
  } else if (my_src == host_src && host_dense) {
    host_role_sorted(p, p.buckets + (uint64_t)host_src * p.bucket_cap, n_host, my_idx, role_ctas,
                     s_dyn, walked);
  } else if (my_src != p.local_src) {
    // dedicated non-local extraction: static warp striding over this source's bucket
    const uint32_t cnt = p.ctrl->counts[my_src];
    const uint64_t *b = p.buckets + (uint64_t)my_src * p.bucket_cap;
    const uint8_t *base = p.base[my_src];
    stride_copy(p, b, cnt, base, (uint32_t)my_idx * kGatherWarps + warp,
                (uint32_t)role_ctas * kGatherWarps, lane, my_src == host_src ? p.host_rows : kRowsInFlight);

  }
  if (tl) {  // own role done: the CTA's last warp to leave its role (local padding follows)
    if (threadIdx.x == 0) tl[0] = (unsigned long long)my_src;
    if (lane == 0) atomicMax(&tl[3], globaltimer_ns());
  }
  }
  // Dense host bucket: optionally only `local_sms` SMs (in chip-spreading order, after the
  // host / peer roles) copy local rows, spreading the local burst over the host-bound step
  // (experiment: does a gentler local stream interfere less with host translation?)
  if (host_dense && p.local_sms > 0 && !host_cta && pos >= p.num_sms - p.local_sms) {
    // this SM is not one of the local_sms -- fall through only if it is a dedicated SM
  } else if (host_dense && p.local_sms > 0 && !host_cta) {
    finish_launch(p.ctrl, p.num_src, p.n_keys, 0);
    return;
  }
  // local group: dedicated local CTAs start here; others pad once their group drains
  // TMA bulk local copies (1 always; 2 = unless the host bucket is dense -- with a
  // PCIe-bound batch the register path's gentler local burst keeps the host reads faster,
  // DESIGN.md section 6; 3 = on every CTA without a host role)
  // "dense" for the local path means PCIe-bound by the ctx's own threshold: a host bucket
  // ordered only because few SMs would walk it (G > 1) is no reason to slow the local burst
  const bool pcie_bound = host_dense && n_host >= p.host_dense_min;
  const bool use_bulk = p.local_bulk == 1 || (p.local_bulk == 2 && !pcie_bound) ||
                        (p.local_bulk == 3 && !host_cta);
  // dense host bucket: optionally only `local_warps` warps of each non-host SM copy local
  // rows (a lower local request rate spread over the host-bound step)
  const bool local_warp = !(host_dense && p.local_warps > 0 && !host_cta && warp >= p.local_warps);
  if (!local_warp) {
    // nothing: this warp leaves the local rows to the SM's first local_warps warps
  } else if (use_bulk) {
    __shared__ __align__(8) uint64_t s_bars[kGatherWarps][kBulkMaxSlots];
    __shared__ uint32_t s_oidx[kGatherWarps][kBulkMaxSlots];
    local_bulk_copy(p, reinterpret_cast<uint8_t *>(s_dyn) + kRangeTabBytes + warp * kBulkWarpBytes,
                    s_bars[warp], s_oidx[warp], lane);
  } else {
    const uint32_t cnt = p.ctrl->counts[p.local_src];
    const uint64_t *b = p.buckets + (uint64_t)p.local_src * p.bucket_cap;
    const uint8_t *base = p.base[p.local_src];
    uint32_t next = 0;
    const uint32_t lc = local_chunk_rows(cnt, p.num_sms);
    if (lane == 0) next = atomicAdd(&p.ctrl->local_cursor, lc);
    next = __shfl_sync(kFullMask, next, 0);
    while (next < cnt) {
      const uint32_t c0 = next, c1 = min(cnt, c0 + lc);
      if (lane == 0) next = atomicAdd(&p.ctrl->local_cursor, lc);  // prefetch claim
      next = __shfl_sync(kFullMask, next, 0);
      for (uint32_t e0 = c0; e0 < c1; e0 += kRowsInFlight)
        copy_rows<kRowsInFlight>(base, p.out, R, b + e0, (int)min((uint32_t)kRowsInFlight, c1 - e0),
                                 lane);
      if (host_dense && p.local_pace > 0) __nanosleep((unsigned)p.local_pace);
    }
  }
  if (tl && lane == 0) atomicMax(&tl[4], globaltimer_ns());
  finish_launch(p.ctrl, p.num_src, p.n_keys, 0);
}

__global__ void __launch_bounds__(kGatherThreads, 1)
    factored_gather_kernel(const GatherParams p) {
  extern __shared__ __align__(16) uint32_t s_dyn[];
  gather_body(p, s_dyn);
}

// ---------------------------------------------------------------------------- single pass
// Single-pass extraction (K3, the fused kernel's `stream` path).  The locate of A1 and the
// copies of A3/A4 overlap instead of meeting at a grid barrier: warps claim 64-key chunks in
// input order, look their keys up, copy the rows they may copy themselves at once (local
// rows -- local extraction "can tolerate all GPU cores", P:1096-1103 -- plus inline host /
// peer rows) and append every other row to its source's queue, which only that source's
// dedicated SMs drain (A2/A3 core dedication).  Local rows never touch a
// bucket, so the 16 B/key bucket round trip and the locate->gather barrier disappear.
// Queues hold (row << 32 | out_idx) entries and are ~0 between launches: a consumer claims
// an index from the queue's head cursor and waits for the entry to be written; it writes ~0
// back after reading it.  A source's queue is final once every chunk is located
// (keys_done == n; reservations precede the increment).
constexpr int kStreamK = 2;                          // keys per lane per chunk
constexpr uint32_t kStreamChunk = 32u * kStreamK;    // keys per chunk (one warp)
constexpr uint32_t kNoClaim = 0xFFFFFFFFu;
constexpr int kStreamRegRows = 4;                    // rows per step of the register path (R > 6 KB)
constexpr int kStreamGroupMax = 8;                   // chunks per group, non-local rows first

__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_u64(uint64_t *p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Warp copies up to U rows; lane u < nvalid holds row u's source address and output index.
template <int U>
__device__ __forceinline__ void copy_addr_rows(uint8_t *__restrict__ out, uint32_t R, uint64_t src,
                                               uint32_t oidx, int nvalid, int lane) {
  uint64_t su[U];
  uint32_t du[U];
#pragma unroll
  for (int u = 0; u < U; ++u) {
    su[u] = __shfl_sync(kFullMask, src, u);
    du[u] = __shfl_sync(kFullMask, oidx, u);
  }
  const uint32_t V = R >> 4;
  for (uint32_t j = lane; j < V; j += 32) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (u < nvalid) v[u] = ld_nc_v4(reinterpret_cast<const uint8_t *>(su[u]) + (uint64_t)j * 16u);
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (u < nvalid) st_cs_v4(out + (uint64_t)du[u] * R + (uint64_t)j * 16u, v[u]);
  }
}

// One chunk: locate its keys, queue the rows of queued sources, copy the rest (non-local
// inline rows first, so their longer latencies start first).  s_addr / s_idx: this warp's
// kStreamChunk-entry copy list; s_inl: per-CTA counts of inline rows per source.
// Asynchronous row slots of one warp (single pass, rows <= 6 KB): lane u < nslots owns one
// R-byte shared-memory slot and its mbarrier.  A row moves source -> slot by one
// cp.async.bulk (TMA) and slot -> out by another, both issued by its lane; a lane takes a
// new row as soon as its slot's row has landed, so a slow row (a cold host read) holds one
// lane's slot while the other lanes keep streaming local rows: up to nslots rows in flight
// per warp (12 KB), no registers held per row, and a row's latency is off the warp's
// critical path.  A slot whose store was issued in this round is reused one round later
// (its store has usually left shared memory by then, so the reuse wait is short).
struct StreamSlots {
  uint8_t *buf;       // this lane's slot
  uint64_t *bar;      // this lane's mbarrier
  uint64_t policy;    // L2 policy of the output stores (evict_first)
  uint32_t oidx;      // output row of the slot's pending row
  uint32_t phase;     // mbarrier parity
  uint32_t busy;      // a row is on its way into the slot
  uint32_t slow;      // ... and it comes from a non-local source
  int nslots;         // 0: register path (copy_addr_rows)
  int slow_cap;       // max non-local rows in flight per warp
  uint32_t nap;       // ns to sleep when every slot is in flight
  int regstore;       // landed rows leave by warp-wide 16-B stores instead of a bulk copy
  uint8_t *wbase;     // slot 0 of this warp

  __device__ __forceinline__ void init(uint8_t *wbuf, uint64_t *wbars, uint32_t R, int lane, bool on, int cap,
                                       uint32_t nap_ns, int reg_store) {
    nap = nap_ns;
    regstore = reg_store;
    wbase = wbuf;
    nslots = on ? min(32, (int)(kBulkWarpBytes / R)) : 0;
    slow_cap = cap > 0 ? cap : 32;
    buf = wbuf + (uint32_t)lane * R;
    bar = wbars + lane;
    phase = 0, busy = 0, slow = 0, oidx = 0;
    policy = l2_evict_first_policy();
    if (lane < nslots) mbar_init(bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncwarp();
  }
  __device__ __forceinline__ bool landed() const {
    uint32_t done;
    asm volatile(
        "{ .reg .pred p; mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(phase)
        : "memory");
    return done != 0;
  }
  __device__ __forceinline__ void retire(uint8_t *out, uint32_t R) {  // slot -> out
    phase ^= 1u;
    busy = 0;
    slow = 0;
    bulk_s2g(out + (uint64_t)oidx * R, buf, R, policy);
  }
  // regstore: the whole warp copies every landed slot to out (16 B per lane per step) and
  // the slots are free at once (no bulk store to wait for).
  __device__ __forceinline__ void retire_warp(bool ready, uint8_t *out, uint32_t R, int lane) {
    uint32_t m = __ballot_sync(kFullMask, ready);
    if (!m) return;
    const uint32_t V = R >> 4;
    while (m) {
      const int u = __ffs(m) - 1;
      m &= m - 1;
      const uint32_t o = __shfl_sync(kFullMask, oidx, u);
      const uint8_t *src = wbase + (uint32_t)u * R;
      for (uint32_t j = lane; j < V; j += 32)
        st_cs_v4(out + (uint64_t)o * R + (uint64_t)j * 16u, *reinterpret_cast<const uint4 *>(src + j * 16u));
    }
    if (ready) {
      phase ^= 1u;
      busy = 0;
      slow = 0;
    }
    __syncwarp();
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // reads before the next TMA writes
  }
  // Copy list entries [0, nl): free lanes take the next entries in list order; entries
  // [sb, se) are non-local rows, at most slow_cap of them in flight per warp.
  __device__ __forceinline__ void feed(const uint64_t *s_addr, const uint32_t *s_idx, uint32_t nl,
                                       uint32_t sb, uint32_t se, uint8_t *out, uint32_t R, int lane) {
    uint32_t next = 0;
    while (next < nl) {
      if (regstore) retire_warp(lane < nslots && busy && landed(), out, R, lane);
      const bool free_lane = lane < nslots && !busy;  // free before this round's bulk retirements
      if (!regstore && lane < nslots && busy && landed()) retire(out, R);
      const uint32_t fm = __ballot_sync(kFullMask, free_lane);
      const uint32_t in_slow = (uint32_t)__popc(__ballot_sync(kFullMask, busy && slow));
      uint32_t t = min((uint32_t)__popc(fm), nl - next);
      const uint32_t s0 = max(next, sb), s1 = min(next + t, se);
      const uint32_t allowed = (uint32_t)slow_cap > in_slow ? (uint32_t)slow_cap - in_slow : 0u;
      if (s1 > s0 && s1 - s0 > allowed) t = s0 + allowed - next;
      if (!t) {  // every slot in flight: yield the issue slots to the SM's other warps
        if (nap) __nanosleep(nap);
        continue;
      }
      const uint32_t e = next + __popc(fm & lanemask_lt());
      if (free_lane && e < next + t) {
        if (!regstore) bulk_wait_read_all();  // this lane's previous store has left the slot
        oidx = s_idx[e];
        slow = e >= sb && e < se;
        mbar_expect_tx(bar, R);
        bulk_g2s(buf, reinterpret_cast<const void *>(s_addr[e]), R, bar);
        busy = 1;
      }
      next += t;
    }
  }
  __device__ __forceinline__ void drain(uint8_t *out, uint32_t R, int lane) {
    if (regstore) {
      if (lane < nslots && busy) mbar_wait(bar, phase);
      retire_warp(lane < nslots && busy, out, R, lane);
    } else if (lane < nslots && busy) {
      mbar_wait(bar, phase);
      retire(out, R);
    }
    bulk_wait_all();
    __syncwarp();
  }
};

// Sub-queues (single pass): the queue of source s is split into one sub-queue per CTA
// dedicated to s, so each is drained by one CTA's warps (no grid-wide claim contention):
// chunk c's rows of s go to sub-queue c mod P_s, of capacity ceil(nchunks / P_s) * chunk.
__device__ __forceinline__ int stream_role_ctas(const GatherParams &gp, int s) {
  if (s == gp.num_src - 1) return gp.inline_host ? 0 : gp.host_sms;
  return gp.inline_peer ? 0 : gp.peer_sms;
}
__device__ __forceinline__ uint32_t *sub_count(const GatherParams &gp, int s, int j) {
  return gp.qctr + (uint32_t)s * kMaxSmId + (uint32_t)j;
}
__device__ __forceinline__ uint32_t *sub_head(const GatherParams &gp, int s, int j) {
  return gp.qctr + (uint32_t)(kMaxSrc + s) * kMaxSmId + (uint32_t)j;
}
__device__ __forceinline__ uint64_t *sub_queue(const GatherParams &gp, int s, int j, uint32_t nchunks,
                                               uint32_t chunk) {
  const uint32_t P = (uint32_t)stream_role_ctas(gp, s);
  const uint64_t cap = (uint64_t)((nchunks + P - 1) / P) * chunk;
  return gp.queues + (uint64_t)s * gp.queue_cap + (uint64_t)j * cap;
}

template <typename KeyT>
__device__ __forceinline__ void stream_keys(const LocateParams &lp, const GatherParams &gp, uint32_t c, int lane,
                                            KeyT (&k)[kStreamK]) {
  const KeyT *keys = static_cast<const KeyT *>(lp.keys);
  const uint32_t K = (uint32_t)gp.stream_k, ck = (uint32_t)gp.stream_ck, i0 = c * ck * K;
#pragma unroll
  for (int it = 0; it < kStreamK; ++it) {
    const uint32_t i = i0 + it * ck + lane;
    k[it] = (it < (int)K && (uint32_t)lane < ck && i < lp.n) ? keys[i] : (KeyT)0;
  }
}
template <typename KeyT>
__device__ __forceinline__ void stream_locs(const LocateParams &lp, const GatherParams &gp, uint32_t c, int lane,
                                            const KeyT (&k)[kStreamK], uint64_t (&e)[kStreamK]) {
  const uint32_t K = (uint32_t)gp.stream_k, ck = (uint32_t)gp.stream_ck, i0 = c * ck * K;
#pragma unroll
  for (int it = 0; it < kStreamK; ++it) {
    const uint32_t i = i0 + it * ck + lane;
    e[it] = (it < (int)K && (uint32_t)lane < ck && i < lp.n && key_in_range<KeyT>(k[it], lp.num_rows))
                ? ld_lt_u64(lp.loc + (uint64_t)k[it])
                : ~0ull;
  }
}

// Chunk c whose location entries e[] are loaded (stream_keys + stream_locs).
// PART 0: the whole chunk; 1: everything but its local rows (locate bookkeeping, queued
// entries, inline non-local rows, keys_done); 2: only its local rows (after PART 1).
template <typename KeyT, int PART = 0>
__device__ __forceinline__ void stream_chunk_located(const LocateParams &lp, const GatherParams &gp, uint32_t c,
                                                     const uint64_t (&e)[kStreamK], int lane, uint64_t *s_addr,
                                                     uint32_t *s_idx, uint32_t *s_inl, StreamSlots &sl) {
  const uint32_t K = (uint32_t)gp.stream_k, ck = (uint32_t)gp.stream_ck, chunk = ck * K;
  const uint32_t R = gp.row_bytes, n = lp.n, i0 = c * chunk;
  const int host_src = gp.num_src - 1;
  int s[kStreamK];
  uint32_t nbad = 0;
  bool any_queued = false;
#pragma unroll
  for (int it = 0; it < kStreamK; ++it) {
    const uint32_t i = i0 + it * ck + lane;
    s[it] = -1;
    if (it < (int)K && (uint32_t)lane < ck && i < n) {
      if (e[it] != ~0ull) {
        s[it] = (int)(e[it] >> UGACHE_LOC_SRC_SHIFT);
      } else if (PART != 2) {
        zero_row(gp.out + (uint64_t)i * R, R);  // out-of-range key
        ++nbad;
      }
    }
    if (PART == 2) continue;
    const int si = s[it];
    const bool inl = si >= 0 && (si == gp.local_src || (si == host_src ? gp.inline_host : gp.inline_peer));
    const int qs = (si >= 0 && !inl) ? si : -1;
    any_queued |= __any_sync(kFullMask, qs >= 0);
    // queued rows: warp-aggregated reservation on the source's queue, then the entry
    const uint32_t qpeers = __match_any_sync(kFullMask, qs);
    const int qleader = __ffs(qpeers) - 1;
    uint32_t b = 0;
    const int qj = qs >= 0 ? (int)(c % (uint32_t)stream_role_ctas(gp, qs)) : 0;
    if (qs >= 0 && lane == qleader) b = atomicAdd(sub_count(gp, qs, qj), (uint32_t)__popc(qpeers));
    b = __shfl_sync(kFullMask, b, qleader);
    if (qs >= 0)
      st_relaxed_u64(sub_queue(gp, qs, qj, (n + chunk - 1) / chunk, chunk) + b + __popc(qpeers & lanemask_lt()),
                     ((e[it] & UGACHE_LOC_ROW_MASK) << 32) | (uint64_t)i);
    // inline rows: per-CTA statistics
    const int is = inl ? si : -1;
    const uint32_t ipeers = __match_any_sync(kFullMask, is);
    if (is >= 0 && lane == __ffs(ipeers) - 1) atomicAdd(&s_inl[is], (uint32_t)__popc(ipeers));
  }
  if (nbad) atomicAdd(&gp.ctrl->bad, nbad);
  // copy list: [inline non-local rows | local rows] (or local first with stream_host_last)
  uint32_t nl = 0, slow_b = 0, slow_e = 0;
#pragma unroll
  for (int pass = 0; pass < 2; ++pass) {
    const bool slow_pass = (pass == 0) != (gp.stream_host_last != 0);
    if ((PART == 1 && !slow_pass) || (PART == 2 && slow_pass)) continue;
    if (slow_pass) slow_b = nl;
#pragma unroll
    for (int it = 0; it < kStreamK; ++it) {
      const int si = s[it];
      const bool take = si >= 0 && (!slow_pass ? si == gp.local_src
                                               : si != gp.local_src &&
                                                     (si == host_src ? gp.inline_host : gp.inline_peer));
      const uint32_t m = __ballot_sync(kFullMask, take);
      if (take) {
        const uint32_t at = nl + __popc(m & lanemask_lt());
        s_addr[at] = reinterpret_cast<uint64_t>(gp.base[si]) + (e[it] & UGACHE_LOC_ROW_MASK) * (uint64_t)R;
        s_idx[at] = i0 + it * ck + lane;
      }
      nl += __popc(m);
    }
    if (slow_pass) slow_e = nl;
  }
  __syncwarp();
  if (sl.nslots) {
    sl.feed(s_addr, s_idx, nl, slow_b, slow_e, gp.out, R, lane);
  } else {
    for (uint32_t g0 = 0; g0 < nl; g0 += kStreamRegRows) {
      const int nv = (int)min((uint32_t)kStreamRegRows, nl - g0);
      const uint64_t a = lane < nv ? s_addr[g0 + lane] : 0ull;
      const uint32_t o = lane < nv ? s_idx[g0 + lane] : 0u;
      copy_addr_rows<kStreamRegRows>(gp.out, R, a, o, nv, lane);
    }
  }
  __syncwarp();
  // keys_done only serves consumers (a queue is final once every key is located); with no
  // queued source in this launch nobody reads it.  A chunk that reserved queue entries
  // orders the reservations before its increment; one that reserved none needs no fence.
  if (PART != 2 && gp.stream_queues) {
    if (any_queued) {
      __threadfence();
      __syncwarp();
    }
    if (lane == 0) atomicAdd(&gp.ctrl->keys_done, min(chunk, n - i0));
  }
}

template <typename KeyT>
__device__ __forceinline__ void stream_chunk(const LocateParams &lp, const GatherParams &gp, uint32_t c, int lane,
                                             uint64_t *s_addr, uint32_t *s_idx, uint32_t *s_inl, StreamSlots &sl) {
  KeyT k[kStreamK];
  uint64_t e[kStreamK];
  stream_keys<KeyT>(lp, gp, c, lane, k);
  stream_locs<KeyT>(lp, gp, c, lane, k, e);
  stream_chunk_located<KeyT>(lp, gp, c, e, lane, s_addr, s_idx, s_inl, sl);
}

// Dedicated warp: claim up to one entry per TMA slot (register path: kStreamRegRows) of
// source s's sub-queue j and copy them.
// Returns false when nothing was reserved beyond the queue head.
__device__ __forceinline__ bool stream_consume(const GatherParams &gp, int s, int j, uint32_t nchunks,
                                               uint32_t chunk, int lane, uint64_t *s_addr, uint32_t *s_idx,
                                               StreamSlots &sl) {
  // Claims never pass the reservation counter (CAS), so every claimed entry is being
  // written by a producer that does not block: waiting for it cannot deadlock even when
  // every warp of the grid is a consumer.
  uint32_t claim = kNoClaim, take = 0;
  if (lane == 0) {
    uint32_t *head = sub_head(gp, s, j);
    const uint32_t *count = sub_count(gp, s, j);
    uint32_t h = ld_relaxed_u32(head);
    while (true) {
      const uint32_t c = ld_relaxed_u32(count);
      if (h >= c) break;
      const uint32_t t = min(sl.nslots ? (uint32_t)sl.nslots : (uint32_t)kStreamRegRows, c - h);
      const uint32_t old = atomicCAS(head, h, h + t);
      if (old == h) {
        claim = h, take = t;
        break;
      }
      h = old;
    }
  }
  claim = __shfl_sync(kFullMask, claim, 0);
  if (claim == kNoClaim) return false;
  take = __shfl_sync(kFullMask, take, 0);
  uint64_t *q = sub_queue(gp, s, j, nchunks, chunk);
  const uint32_t idx = claim + lane;
  uint64_t ent = ~0ull;
  if ((uint32_t)lane < take) {
    while ((ent = ld_relaxed_u64(q + idx)) == ~0ull) __nanosleep(20);  // producer mid-write
    q[idx] = ~0ull;  // re-arm for the next launch
  }
  const int nv = (int)take;
  const uint64_t a = ent != ~0ull ? reinterpret_cast<uint64_t>(gp.base[s]) + (ent >> 32) * (uint64_t)gp.row_bytes : 0ull;
  if (sl.nslots) {  // through this warp's TMA slots, like the inline rows
    __syncwarp();
    if (lane < nv) {
      s_addr[lane] = a;
      s_idx[lane] = (uint32_t)ent;
    }
    __syncwarp();
    sl.feed(s_addr, s_idx, (uint32_t)nv, 0, (uint32_t)nv, gp.out, gp.row_bytes, lane);
    __syncwarp();
  } else if (nv) {
    copy_addr_rows<kStreamRegRows>(gp.out, gp.row_bytes, a, (uint32_t)ent, nv, lane);
  }
  return true;
}

template <typename KeyT>
__device__ __forceinline__ void stream_body(const LocateParams &lp, const GatherParams &gp, uint32_t *s_dyn,
                                            uint32_t pos) {
  __shared__ uint32_t s_inl[kMaxSrc];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t n = lp.n, chunk = (uint32_t)gp.stream_ck * (uint32_t)gp.stream_k,
                 nchunks = (n + chunk - 1) / chunk;
  uint64_t *s_addr = reinterpret_cast<uint64_t *>(s_dyn) + warp * kStreamChunk;
  uint32_t *s_idx = reinterpret_cast<uint32_t *>(s_dyn + 2 * kGatherWarps * kStreamChunk) + warp * kStreamChunk;
  __shared__ __align__(8) uint64_t s_slot_bars[kGatherWarps][32];
  if (threadIdx.x < kMaxSrc) s_inl[threadIdx.x] = 0;
  StreamSlots sl;
  sl.init(reinterpret_cast<uint8_t *>(s_dyn) + kRangeTabBytes + warp * kBulkWarpBytes, s_slot_bars[warp],
          gp.row_bytes, lane, gp.stream_bulk != 0, gp.stream_host_cap, (uint32_t)gp.stream_nap,
          gp.stream_regstore);
  __syncthreads();
  // roles of the queued sources, as in gather_body: [host | peer_0 | ... | local]
  const int host_src = gp.num_src - 1;
  const int H = gp.inline_host ? 0 : gp.host_sms;
  const int P = gp.inline_peer ? 0 : gp.peer_sms;
  int role_src = -1, role_j = 0;  // this CTA's queued source and its sub-queue
  if ((int)pos < H) {
    role_src = host_src, role_j = (int)pos;
  } else if ((int)pos - H < gp.n_peers * P) {
    role_src = gp.peer_src[((int)pos - H) / P], role_j = ((int)pos - H) % P;
  }
  // consumer warps of a dedicated CTA: host_warps (host) / stream_peer_warps (peers); the
  // CTA's other warps locate chunks like everyone else
  const int consumers = role_src == host_src ? gp.host_warps : gp.stream_peer_warps;
  const int my_src = warp < consumers ? role_src : -1;
  Ctrl *ctrl = gp.ctrl;
  // chunk claims: dynamic (atomic cursor, input order over time) or static (warp gw takes
  // chunks gw, gw + W, ...: every warp works on the same window of keys at a time)
  // stream_static >= 2: static for the full rounds of W chunks but the last (stream_static
  // - 2), then the dynamic cursor for the remaining chunks (balances the tail)
  uint32_t static_next = pos * kGatherWarps + warp;
  const uint32_t static_stride = gridDim.x * kGatherWarps;
  uint32_t static_end = 0;
  if (gp.stream_static == 1) {
    static_end = nchunks;
  } else if (gp.stream_static >= 2) {
    const uint32_t rounds = nchunks / static_stride, keep = (uint32_t)(gp.stream_static - 2);
    static_end = (rounds > keep ? rounds - keep : 0) * static_stride;
  }
  auto claim_chunk = [&]() -> uint32_t {
    uint32_t c = kNoClaim;
    if (static_next < static_end) {
      c = static_next;
      static_next += static_stride;
    } else if (gp.stream_static == 1) {
      c = kNoClaim;
    } else if (lane == 0 && static_end + ld_relaxed_u32(&ctrl->chunk_cursor) < nchunks) {
      c = static_end + atomicAdd(&ctrl->chunk_cursor, 1u);
    }
    return __shfl_sync(kFullMask, c, 0);
  };
  if (my_src < 0 && gp.stream_prefetch == 2 && gp.stream_k == 1 && gp.stream_ck == 32) {
    // locating warp, pipelined through shared memory with cp.async (no register holds a
    // load in flight): the keys of chunk i+2 and the location entries of chunk i+1 land
    // while chunk i's rows are fed to the slots, so the key -> entry dependent loads leave
    // the warp's critical path.  Each lane stages only its own key / entry (lane-private
    // words: cp.async.wait_group alone orders them).  Entries alternate between two
    // buffers so a new entry never lands on one that is still being read.
    __shared__ __align__(8) uint64_t s_pf[kGatherWarps][3][32];
    KeyT *pk = reinterpret_cast<KeyT *>(s_pf[warp][0]);
    const KeyT *keys = static_cast<const KeyT *>(lp.keys);
    const bool ef = c_lt_evict_first != 0;
    auto lane_key = [&](uint32_t c) { return c < nchunks && c * 32u + (uint32_t)lane < n; };
    uint32_t c0 = claim_chunk(), c1 = kNoClaim, buf = 0;
    bool v0 = false;  // this lane's key of chunk c0 is in range (its entry is staged)
    if (c0 < nchunks) {
      if (lane_key(c0)) {
        const KeyT k = keys[c0 * 32u + lane];
        v0 = key_in_range<KeyT>(k, lp.num_rows);
        if (v0) cp_async_word(&s_pf[warp][1][lane], lp.loc + (uint64_t)k, 8, ef);
      }
      c1 = claim_chunk();
      if (lane_key(c1)) cp_async_word(&pk[lane], keys + c1 * 32u + lane, (int)sizeof(KeyT), false);
    }
    cp_async_commit();
    while (c0 < nchunks) {
      cp_async_wait_all();
      uint64_t e[kStreamK];
#pragma unroll
      for (int it = 0; it < kStreamK; ++it) e[it] = ~0ull;
      e[0] = v0 ? s_pf[warp][1 + buf][lane] : ~0ull;
      const uint32_t c2 = c1 < nchunks ? claim_chunk() : kNoClaim;
      bool v1 = false;
      if (lane_key(c1)) {
        const KeyT k = pk[lane];
        v1 = key_in_range<KeyT>(k, lp.num_rows);
        if (v1) cp_async_word(&s_pf[warp][2 - buf][lane], lp.loc + (uint64_t)k, 8, ef);
      }
      if (lane_key(c2)) cp_async_word(&pk[lane], keys + c2 * 32u + lane, (int)sizeof(KeyT), false);
      cp_async_commit();
      stream_chunk_located<KeyT>(lp, gp, c0, e, lane, s_addr, s_idx, s_inl, sl);
      c0 = c1, c1 = c2, v0 = v1, buf ^= 1u;
    }
    cp_async_wait_all();
  } else if (my_src < 0 && gp.stream_prefetch) {
    // locating warp, software-pipelined two deep: the keys of chunk i+2 and the location
    // entries of chunk i+1 are in flight while chunk i's rows are fed to the slots
    KeyT k1[kStreamK];
    uint64_t e0[kStreamK], e1[kStreamK];
    uint32_t c0 = claim_chunk(), c1 = kNoClaim;
    if (c0 < nchunks) {
      stream_keys<KeyT>(lp, gp, c0, lane, k1);
      stream_locs<KeyT>(lp, gp, c0, lane, k1, e0);
      c1 = claim_chunk();
      if (c1 < nchunks) stream_keys<KeyT>(lp, gp, c1, lane, k1);
    }
    while (c0 < nchunks) {
      if (c1 < nchunks) stream_locs<KeyT>(lp, gp, c1, lane, k1, e1);
      const uint32_t c2 = c1 < nchunks ? claim_chunk() : kNoClaim;
      if (c2 < nchunks) stream_keys<KeyT>(lp, gp, c2, lane, k1);
      stream_chunk_located<KeyT>(lp, gp, c0, e0, lane, s_addr, s_idx, s_inl, sl);
      c0 = c1;
      c1 = c2;
#pragma unroll
      for (int it = 0; it < kStreamK; ++it) e0[it] = e1[it];
    }
  } else if (my_src < 0 && gp.stream_group > 1 && gp.stream_k == 1) {
    // locating warp, non-local rows first: locate a group of up to kStreamGroupMax chunks,
    // put every non-local (host) row of the group in flight, then feed the local rows --
    // a cold host row's latency then overlaps all of the group's local work
    bool more = true;
    while (more) {
      uint32_t cs[kStreamGroupMax];
      uint64_t es[kStreamGroupMax];
      KeyT ks[kStreamGroupMax];
#pragma unroll
      for (int g = 0; g < kStreamGroupMax; ++g) {
        const bool want = more && g < gp.stream_group;
        cs[g] = want ? claim_chunk() : kNoClaim;
        if (want && cs[g] >= nchunks) more = false;
        const uint32_t i = cs[g] * (uint32_t)gp.stream_ck + lane;
        ks[g] = (cs[g] < nchunks && (uint32_t)lane < (uint32_t)gp.stream_ck && i < n)
                    ? static_cast<const KeyT *>(lp.keys)[i] : (KeyT)0;
      }
#pragma unroll
      for (int g = 0; g < kStreamGroupMax; ++g) {
        const uint32_t i = cs[g] * (uint32_t)gp.stream_ck + lane;
        es[g] = (cs[g] < nchunks && (uint32_t)lane < (uint32_t)gp.stream_ck && i < n &&
                 key_in_range<KeyT>(ks[g], lp.num_rows))
                    ? ld_lt_u64(lp.loc + (uint64_t)ks[g])
                    : ~0ull;
      }
#pragma unroll
      for (int g = 0; g < kStreamGroupMax; ++g)
        if (cs[g] < nchunks) {
          const uint64_t e1[kStreamK] = {es[g]};
          stream_chunk_located<KeyT, 1>(lp, gp, cs[g], e1, lane, s_addr, s_idx, s_inl, sl);
        }
#pragma unroll
      for (int g = 0; g < kStreamGroupMax; ++g)
        if (cs[g] < nchunks) {
          const uint64_t e1[kStreamK] = {es[g]};
          stream_chunk_located<KeyT, 2>(lp, gp, cs[g], e1, lane, s_addr, s_idx, s_inl, sl);
        }
    }
  } else if (my_src < 0) {  // locating warp: chunks until none are left
    while (true) {
      const uint32_t c = claim_chunk();
      if (c >= nchunks) break;
      stream_chunk<KeyT>(lp, gp, c, lane, s_addr, s_idx, s_inl, sl);
    }
  } else {  // dedicated warp: drain my source's queue; locate chunks while it is empty
    bool chunks_left = true;
    while (true) {
      if (stream_consume(gp, my_src, role_j, nchunks, chunk, lane, s_addr, s_idx, sl)) continue;
      uint32_t c = chunks_left ? claim_chunk() : kNoClaim;
      if (c >= nchunks) chunks_left = false;
      if (c < nchunks) {
        stream_chunk<KeyT>(lp, gp, c, lane, s_addr, s_idx, s_inl, sl);
        continue;
      }
      int fin = 0;
      if (lane == 0)
        fin = ld_acquire_u32(&ctrl->keys_done) >= n &&
              ld_relaxed_u32(sub_head(gp, my_src, role_j)) >= ld_relaxed_u32(sub_count(gp, my_src, role_j));
      if (__shfl_sync(kFullMask, fin, 0)) break;
      __nanosleep(64);
    }
  }
  sl.drain(gp.out, gp.row_bytes, lane);
  __syncthreads();
  if (threadIdx.x < gp.num_src && s_inl[threadIdx.x]) atomicAdd(&ctrl->counts[threadIdx.x], s_inl[threadIdx.x]);
  if (role_src >= 0 && threadIdx.x == 0) {  // my sub-queue is drained: publish its count, re-arm it
    uint32_t *cnt = sub_count(gp, role_src, role_j);
    atomicAdd(&ctrl->counts[role_src], *cnt);
    *cnt = 0;
    *sub_head(gp, role_src, role_j) = 0;
  }
  finish_launch(ctrl, gp.num_src, n, 1);
}

// ---------------------------------------------------------------------------- K1+K2 fused
// One cooperative launch per batch: every CTA locates + buckets tiles of 512 x 8 keys, a
// grid-wide barrier publishes the buckets and counts, then the same CTAs run the factored
// gather.  Saves a launch and the inter-kernel gap for small batches (DLR-shaped).
template <typename KeyT>
__global__ void __launch_bounds__(kGatherThreads, 1)
    fused_extract_kernel(const LocateParams lp, const GatherParams gp) {
  extern __shared__ __align__(16) uint32_t s_dyn[];
  __shared__ uint32_t s_cnt[kMaxSrc];
  __shared__ uint32_t s_base[kMaxSrc];
  const uint32_t kTile = kGatherThreads * (uint32_t)lp.items;
  const uint32_t ntiles = (lp.n + kTile - 1) / kTile;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    gp.ctrl->t_start = globaltimer_ns();
    gp.ctrl->t_ordered = 0;
    gp.ctrl->t_host_done = 0;  // diagnostic stamps; host copies finish >> 1 us later
  }
  // Tiles go to CTAs in chip-spreading order; CTAs left without a tile start the input-order
  // host walk at once (the host rows of a sparse batch then overlap the locate phase, as in
  // the unfactored kernel) until every tile is located.  Keys walked here are skipped by the
  // ordered host path after the barrier (host_order's `walked`).
  // Walkers never arrive at the barrier (it counts the locating CTAs only), so a walker
  // finishing its last chunk delays nobody; claimed chunks are always completed by their
  // claimer, so skipping [0, walked) in the ordered path stays exact.
  uint32_t smid;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  const uint32_t pos = smid < (uint32_t)kMaxSmId ? gp.sm_pos[smid] : blockIdx.x;
  if (gp.timeline && threadIdx.x == 0) gp.timeline[pos * kTimelineWords + 1] = globaltimer_ns();
  const bool walker = gp.early_walk && pos >= ntiles;
  const uint32_t arrivals = gp.early_walk ? min(gridDim.x, ntiles) : gridDim.x;
  uint32_t *s_hist = (lp.hist && gp.hist_smem) ? s_dyn : nullptr;  // the range-table area
  if (s_hist) {
    for (uint32_t i = threadIdx.x; i < gp.n_ranges; i += blockDim.x) s_hist[i] = 0;
    __syncthreads();
  }
  for (uint32_t t = pos; t < ntiles; t += gridDim.x)
    locate_tile<KeyT, kGatherThreads>(lp, t, s_cnt, s_base, s_hist);
  __syncthreads();
  if (s_hist && pos < ntiles)
    for (uint32_t i = threadIdx.x; i < gp.n_ranges; i += blockDim.x)
      if (s_hist[i]) atomicAdd(&lp.range_count[i], s_hist[i]);
  if (threadIdx.x == 0) atomicMax(&gp.ctrl->t_loc_max, globaltimer_ns());  // diagnostic stamp
  if (walker) {
    host_walk_copy(gp, threadIdx.x >> 5, threadIdx.x & 31, &gp.ctrl->grid_arrive, arrivals);
    role_wait(&gp.ctrl->grid_arrive, arrivals);
  } else {
    role_barrier(&gp.ctrl->grid_arrive, arrivals);
  }
  if (pos == 0 && threadIdx.x == 0) gp.ctrl->t_located = globaltimer_ns();
  gather_body(gp, s_dyn);
}

// ---------------------------------------------------------------------------- K3
// Single-pass extraction (stream_body): its own kernel, so its register allocation does
// not constrain the locate | barrier | gather kernel's.  Cooperative launch, one CTA per SM.
template <typename KeyT>
__global__ void __launch_bounds__(kGatherThreads, 1)
    stream_extract_kernel(const LocateParams lp, const GatherParams gp) {
  extern __shared__ __align__(16) uint32_t s_dyn[];
  // With queued sources the CTA's role is its SM's (cooperative launch, one CTA per SM);
  // without, no warp ever waits on another, the launch is a plain one and CTA b takes
  // position b of the static chunk schedule.
  uint32_t pos = blockIdx.x;
  if (gp.stream_queues) {
    uint32_t smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    pos = smid < (uint32_t)kMaxSmId ? gp.sm_pos[smid] : blockIdx.x;
  }
  stream_body<KeyT>(lp, gp, s_dyn, pos);
}

// ---------------------------------------------------------------------------- K3r
// Single pass, register variant, for batches whose every source is read inline (no queued
// source: G = 1 or peers inline) and whose host bucket is sparse (cold host rows, latency-
// bound).  Each warp takes chunks of stream_ck (<= 32) keys on the
// static schedule, locates them, and copies its rows RegRows at a time straight from the
// lanes that located them (no copy list in shared memory, no TMA slots, no queue
// bookkeeping): a lean kernel whose registers leave room for 8 rows in flight per warp
// step and two CTAs per SM.  Same output, same per-source counts as K3.
constexpr int kRegRows = 8;
template <typename KeyT>
__global__ void __launch_bounds__(kGatherThreads, 2)
    stream_extract_reg_kernel(const LocateParams lp, const GatherParams gp) {
  __shared__ uint32_t s_inl[kMaxSrc];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x < kMaxSrc) s_inl[threadIdx.x] = 0;
  __syncthreads();
  const uint32_t n = lp.n, ck = (uint32_t)gp.stream_ck, R = gp.row_bytes;
  const uint32_t nchunks = (n + ck - 1) / ck;
  const uint32_t W = gridDim.x * (blockDim.x >> 5);
  const KeyT *keys = static_cast<const KeyT *>(lp.keys);
  uint32_t nbad = 0;
  for (uint32_t c = blockIdx.x * (blockDim.x >> 5) + warp; c < nchunks; c += W) {
    const uint32_t i = c * ck + (uint32_t)lane;
    int s = -1;
    uint64_t a = 0;
    if ((uint32_t)lane < ck && i < n) {
      const KeyT k = keys[i];
      if (key_in_range<KeyT>(k, lp.num_rows)) {
        const uint64_t e = ld_lt_u64(lp.loc + (uint64_t)k);
        s = (int)(e >> UGACHE_LOC_SRC_SHIFT);
        a = reinterpret_cast<uint64_t>(gp.base[s]) + (e & UGACHE_LOC_ROW_MASK) * (uint64_t)R;
      } else {
        zero_row(gp.out + (uint64_t)i * R, R);  // out-of-range key
        ++nbad;
      }
    }
    const uint32_t peers = __match_any_sync(kFullMask, s);
    if (s >= 0 && lane == __ffs(peers) - 1) atomicAdd(&s_inl[s], (uint32_t)__popc(peers));
    // rows of this chunk, kRegRows per step, taken from the lanes that located them
    const uint32_t m = __ballot_sync(kFullMask, s >= 0);
    const int nrows = __popc(m);
    for (int g0 = 0; g0 < nrows; g0 += kRegRows) {
      const int nv = min(kRegRows, nrows - g0);
      // lane u < nv takes the (g0 + u)-th located lane's row
      const int srcl = lane < nv ? (int)__fns(m, 0, g0 + lane + 1) : 0;
      const uint64_t au = __shfl_sync(kFullMask, a, srcl);
      const uint32_t ou = c * ck + (uint32_t)srcl;
      copy_addr_rows<kRegRows>(gp.out, R, au, ou, nv, lane);
    }
  }
  if (nbad) atomicAdd(&gp.ctrl->bad, nbad);
  __syncthreads();
  if (threadIdx.x < gp.num_src && s_inl[threadIdx.x]) atomicAdd(&gp.ctrl->counts[threadIdx.x], s_inl[threadIdx.x]);
  finish_launch(gp.ctrl, gp.num_src, n, 1);
}

// ---------------------------------------------------------------------------- K2'
template <typename KeyT>
__global__ void __launch_bounds__(kGatherThreads, 1)
    random_dispatch_kernel(const RandomParams p) {
  __shared__ uint32_t s_cnt[kMaxSrc];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x < kMaxSrc) s_cnt[threadIdx.x] = 0;
  __syncthreads();
  const KeyT *keys = static_cast<const KeyT *>(p.keys);
  const uint32_t R = p.row_bytes, V = R >> 4;
  const uint32_t W = gridDim.x * kGatherWarps;
  uint32_t nbad = 0;
  for (uint32_t e0 = (blockIdx.x * kGatherWarps + warp) * kRowsInFlight; e0 < p.n;
       e0 += W * kRowsInFlight) {
    const int nvalid = (int)min((uint32_t)kRowsInFlight, p.n - e0);
    int s = -2;
    uint64_t rr = 0;
    if (lane < nvalid) {
      const KeyT k = keys[e0 + lane];
      if (key_in_range<KeyT>(k, p.num_rows)) {
        const uint64_t e = ld_lt_u64(p.loc + (uint64_t)k);
        s = (int)(e >> UGACHE_LOC_SRC_SHIFT);
        rr = e & UGACHE_LOC_ROW_MASK;
      } else {
        s = -1;
        ++nbad;
      }
    }
    const uint32_t peers = __match_any_sync(kFullMask, s);
    if (s >= 0 && lane == __ffs(peers) - 1) atomicAdd(&s_cnt[s], (uint32_t)__popc(peers));
    int su[kRowsInFlight];
    uint64_t ru[kRowsInFlight];
#pragma unroll
    for (int u = 0; u < kRowsInFlight; ++u) {
      su[u] = __shfl_sync(kFullMask, s, u);
      ru[u] = __shfl_sync(kFullMask, rr, u);
    }
    for (uint32_t j = lane; j < V; j += 32) {
      uint4 v[kRowsInFlight];
#pragma unroll
      for (int u = 0; u < kRowsInFlight; ++u)
        if (su[u] >= 0) v[u] = ld_nc_v4(p.base[su[u]] + ru[u] * R + (uint64_t)j * 16u);
        else v[u] = make_uint4(0, 0, 0, 0);
#pragma unroll
      for (int u = 0; u < kRowsInFlight; ++u)
        if (su[u] >= -1) st_cs_v4(p.out + (uint64_t)(e0 + u) * R + (uint64_t)j * 16u, v[u]);
    }
  }
  if (nbad) atomicAdd(&p.ctrl->bad, nbad);
  __syncthreads();
  if (threadIdx.x < p.num_src && s_cnt[threadIdx.x])
    atomicAdd(&p.ctrl->counts[threadIdx.x], s_cnt[threadIdx.x]);
  finish_launch(p.ctrl, p.num_src, p.n, 0);
}

// ---------------------------------------------------------------------------- probe
// One CTA per SM (cooperative launch): record the %smid values of this device.
__global__ void __launch_bounds__(32, 1) smid_probe_kernel(uint32_t *smids) {
  if (threadIdx.x == 0) {
    uint32_t smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    smids[blockIdx.x] = smid;
  }
}

// ---------------------------------------------------------------------------- A0 calibrate
// Bandwidth vs the number of SMs dedicated to a source (A0, Fig. 6): one CTA per
// SM (cooperative launch, the gather kernels' shared-memory footprint); the CTA at position
// pos of the chip-spreading SM order reads for role pos / k (role r < n_roles: source
// src_id[r]), so each source gets k SMs spread over the chip exactly as the extract
// kernels place their roles.  A role's warps claim kRowsInFlight entries at a time from its
// sample list (row << 32 | out row, ascending rows) and copy them with copy_rows.
struct CalibParams {
  const uint8_t *base[kMaxSrc];
  const uint64_t *ents;      // n_roles x n_ents sample entries
  uint8_t *out;              // n_roles x n_ents rows
  uint32_t *cursor;          // n_roles claim cursors, zero before the launch
  uint32_t n_ents;
  uint32_t row_bytes;
  int32_t n_roles;
  int32_t k;                 // SMs per role
  int32_t src_id[kMaxSrc];
  uint8_t sm_pos[kMaxSmId];
};

__global__ void __launch_bounds__(kGatherThreads, 1) calib_kernel(const CalibParams p) {
  uint32_t smid;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  const int pos = smid < (uint32_t)kMaxSmId ? p.sm_pos[smid] : (int)blockIdx.x;
  const int role = pos / p.k;
  if (role >= p.n_roles) return;
  const int lane = threadIdx.x & 31;
  const uint64_t *e = p.ents + (uint64_t)role * p.n_ents;
  uint8_t *out = p.out + (uint64_t)role * p.n_ents * p.row_bytes;
  const uint8_t *base = p.base[p.src_id[role]];
  while (true) {
    uint32_t e0 = 0;
    if (lane == 0) e0 = atomicAdd(&p.cursor[role], (uint32_t)kRowsInFlight);
    e0 = __shfl_sync(kFullMask, e0, 0);
    if (e0 >= p.n_ents) break;
    copy_rows<kRowsInFlight>(base, out, p.row_bytes, e + e0, (int)min((uint32_t)kRowsInFlight, p.n_ents - e0),
                             lane);
  }
}

// ---------------------------------------------------------------------------- K5
__global__ void __launch_bounds__(256) fill_kernel(const FillParams p) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t W = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  const uint32_t V = p.row_bytes >> 4;
  for (uint64_t s0 = warp * kRowsInFlight; s0 < p.n_slots; s0 += W * kRowsInFlight) {
    const int nvalid = (int)min((uint64_t)kRowsInFlight, p.n_slots - s0);
    const uint64_t key = lane < nvalid ? p.slot_keys[s0 + lane] : 0ull;
    const uint64_t dst = lane < nvalid ? (p.slot_idx ? p.slot_idx[s0 + lane] : s0 + lane) : 0ull;
    uint64_t ku[kRowsInFlight], du[kRowsInFlight];
#pragma unroll
    for (int u = 0; u < kRowsInFlight; ++u) {
      ku[u] = __shfl_sync(kFullMask, key, u);
      du[u] = __shfl_sync(kFullMask, dst, u);
    }
    for (uint32_t j = lane; j < V; j += 32) {
      uint4 v[kRowsInFlight];
#pragma unroll
      for (int u = 0; u < kRowsInFlight; ++u)
        if (u < nvalid) v[u] = ld_nc_v4(p.table + ku[u] * p.row_bytes + (uint64_t)j * 16u);
#pragma unroll
      for (int u = 0; u < kRowsInFlight; ++u)
        if (u < nvalid)
          *reinterpret_cast<uint4 *>(p.slab + du[u] * p.row_bytes + (uint64_t)j * 16u) = v[u];
    }
  }
}

// ---------------------------------------------------------------------------- message path
// The message-based baseline ("peer-based" vs "message-based" extraction): the
// requester sends the slot ids it needs to each owner, the owner gathers them into a
// contiguous send buffer, the rows travel back in a collective, and the requester
// scatters them into key order.  Only the three device steps are here; the two
// all-to-all exchanges are the caller's (NCCL through torch.distributed).
struct MsgSeg {
  uint32_t src;    // peer GPU id (bucket index)
  uint32_t count;  // entries of that bucket
  uint64_t off;    // first entry of this peer's segment in the packed request / reply
};

struct MsgParams {
  const uint64_t *buckets;
  uint64_t bucket_cap;
  MsgSeg seg[kMaxSrc];
  int32_t n_seg;
  uint64_t total;
  uint32_t *req;             // pack: out, one slot id per entry
  const uint32_t *req_in;    // serve: in
  const uint8_t *slab;       // serve: this GPU's cache slab
  uint64_t slab_rows;        // serve: rows >= slab_rows zero-fill (never produced by a valid LT)
  const uint8_t *rows_in;    // scatter: replies, packed in segment order
  uint8_t *rows_out;         // serve: send buffer / scatter: out
  uint32_t row_bytes;
};

__device__ __forceinline__ int msg_segment(const MsgParams &p, uint64_t i) {
  int s = 0;
  while (s + 1 < p.n_seg && i >= p.seg[s + 1].off) ++s;
  return s;
}

__global__ void __launch_bounds__(256) msg_pack_kernel(const MsgParams p) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < p.total;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const MsgSeg g = p.seg[msg_segment(p, i)];
    p.req[i] = (uint32_t)(p.buckets[(uint64_t)g.src * p.bucket_cap + (i - g.off)] >> 32);
  }
}

// Warp per U rows: serve (slab[req[i]] -> send[i]) or scatter (reply[i] -> out[out_idx]).
template <bool SCATTER>
__global__ void __launch_bounds__(512) msg_copy_kernel(const MsgParams p) {
  const int lane = threadIdx.x & 31;
  const uint64_t W = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  const uint32_t R = p.row_bytes, V = R >> 4;
  for (uint64_t e0 = (((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * kRowsInFlight; e0 < p.total;
       e0 += W * kRowsInFlight) {
    const int nv = (int)min((uint64_t)kRowsInFlight, p.total - e0);
    uint64_t s_row = 0, d_row = 0;
    bool zero = false;
    if (lane < nv) {
      const uint64_t i = e0 + lane;
      if (SCATTER) {
        const MsgSeg g = p.seg[msg_segment(p, i)];
        s_row = i;
        d_row = p.buckets[(uint64_t)g.src * p.bucket_cap + (i - g.off)] & 0xFFFFFFFFull;
      } else {
        s_row = p.req_in[i];
        d_row = i;
        zero = s_row >= p.slab_rows;
      }
    }
    const uint8_t *src = SCATTER ? p.rows_in : p.slab;
    uint64_t su[kRowsInFlight], du[kRowsInFlight];
    bool zu[kRowsInFlight];
#pragma unroll
    for (int u = 0; u < kRowsInFlight; ++u) {
      su[u] = __shfl_sync(kFullMask, s_row, u);
      du[u] = __shfl_sync(kFullMask, d_row, u);
      zu[u] = __shfl_sync(kFullMask, zero, u);
    }
    for (uint32_t j = lane; j < V; j += 32) {
      uint4 v[kRowsInFlight];
#pragma unroll
      for (int u = 0; u < kRowsInFlight; ++u)
        if (u < nv) v[u] = zu[u] ? make_uint4(0, 0, 0, 0) : ld_nc_v4(src + su[u] * R + (uint64_t)j * 16u);
#pragma unroll
      for (int u = 0; u < kRowsInFlight; ++u)
        if (u < nv) st_cs_v4(p.rows_out + du[u] * R + (uint64_t)j * 16u, v[u]);
    }
  }
}

// ---------------------------------------------------------------------------- refresh
// Cache refresh, hashtable step: every key whose CURRENT location is a GPU slot
// in [lo, hi) and whose location changes is pointed at the host first (which holds every
// entry; tier slot tier_slot[k] when the host tier is on, else row = key), so no reader can
// reach a slot whose content is about to be rewritten.  Unchanged and host keys stay.
__global__ void __launch_bounds__(256) refresh_evict_kernel(uint64_t *loc, const uint64_t *loc_new,
                                                            uint64_t N, uint64_t host_tag,
                                                            const uint32_t *tier_slot, uint64_t G,
                                                            uint64_t lo, uint64_t hi) {
  for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < N;
       k += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t a = loc[k];
    const uint64_t row = a & UGACHE_LOC_ROW_MASK;
    if ((a >> UGACHE_LOC_SRC_SHIFT) < G && row >= lo && row < hi && a != loc_new[k])
      loc[k] = host_tag | (tier_slot ? (uint64_t)tier_slot[k] : k);
  }
}

// Cache refresh, install step of a chunk: keys whose NEW location is a GPU slot in [lo, hi)
// take it (the slot's content was rewritten by its owner before this runs).
__global__ void __launch_bounds__(256) refresh_install_kernel(uint64_t *loc, const uint64_t *loc_new,
                                                              uint64_t N, uint64_t G, uint64_t lo,
                                                              uint64_t hi) {
  for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < N;
       k += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t b = loc_new[k];
    const uint64_t row = b & UGACHE_LOC_ROW_MASK;
    if ((b >> UGACHE_LOC_SRC_SHIFT) < G && row >= lo && row < hi) loc[k] = b;
  }
}

}  // namespace ugk
