// ugache_internal.h -- shared declarations of the libugache implementation (not ABI).
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "ugache.h"

namespace ug {

constexpr int kMaxSrc = UGACHE_MAX_GPUS + 1;
constexpr int kDefaultNumSms = 148;
// Default core dedication for host extraction: "a small number of cores for host"
// (P:1211-1213).  Set from the A0 calibration on B200 (DESIGN.md section "calibration").
constexpr int kDefaultHostSms = 12;
// Default model bandwidths (bytes/s) when the caller passes 0 (R11):
//  local = MEASURED_PEAKS.json hbm_gbs (STREAM-style copy on this pool's B200s),
//  peer  = measured B200 peer copy per direction (B200_PROFILING.md: 770 GB/s),
//  host  = calibrated zero-copy throughput of random 512-B host rows with range-ordered
//          reads on the B200 box (tools/calibrate.py, gnn_pa: 34.4 GB/s; the sequential
//          pinned-H2D DMA peak is 55.6 GB/s).
constexpr double kDefaultBwLocal = 6457.7e9;
constexpr double kDefaultBwPeer = 770e9;
constexpr double kDefaultBwHost = 34.4e9;

struct Params {
  int S, host_sms, peer_sms;
  double T_L, T_P, T_H, R_L, R_P, R_H;
};

ugache_status resolve_params(const ugache_config *cfg, int device_sms, Params *p);
ugache_status solve(const ugache_config *cfg, int device_sms, const float *hotness,
                    std::vector<uint32_t> &order, ugache_plan *plan);
ugache_status build_placement(const ugache_config *cfg, const uint32_t *order,
                              const ugache_plan *plan, int gpu, uint64_t *loc,
                              uint64_t *slot_keys, uint64_t *n_slots);
void fill_host_tier(const uint8_t *table, uint32_t R, const uint64_t *order, uint64_t be,
                    uint64_t N, uint8_t *tier);
void fill_host_tier(const uint8_t *table, uint32_t R, const uint32_t *order, uint64_t be,
                    uint64_t N, uint8_t *tier);

}  // namespace ug
