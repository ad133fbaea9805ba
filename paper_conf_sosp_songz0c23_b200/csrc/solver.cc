// solver.cc -- host-side cache-placement solver of UGache (section 6).
//
// The placement family is hot-replicate / warm-partition (ref [39]), which the
// paper rejects as a *general* solver only because it assumes a uniform fully-connected
// platform; a B200 NVSwitch node is exactly that (R11, R22).  The member of the
// family is chosen by minimising the paper's extraction-time model (section 6.2,
// P:1304-1501) exactly over the replicated-prefix length k in [0, C]:
//
//   ranks [0,k)           replicated on every GPU           (replication)
//   ranks [k, band_end)   round-robin over GPUs by rank     (partition,   P:395-398)
//   ranks >= band_end     host DRAM                         (fallback,    P:1369-1370)
//
//   t^j_i = T_{i<-j} * sum_e h_e a^e_{i<-j}
//   t_i   = max( max_j t^j_i , sum_j R_{i<-j} t^j_i )
//   z     = max_i t_i
//
// Every k is evaluated in O(G) from prefix sums of the sorted hotness (per-GPU band masses
// come from residue-class prefix sums), so the search is exact, O(N log) sort + O(C*G).
#include <algorithm>
#include <cmath>
#include <cstring>
#include <vector>

#include <omp.h>

#include "ugache_internal.h"

namespace ug {

ugache_status resolve_params(const ugache_config *cfg, int device_sms, Params *p) {
  if (!cfg || !p) return UGACHE_EINVAL;
  const int G = cfg->num_gpus;
  if (G < 1 || G > UGACHE_MAX_GPUS) return UGACHE_EINVAL;
  if (cfg->num_rows == 0 || cfg->num_rows >= (1ull << 32)) return UGACHE_EINVAL;
  if (cfg->row_bytes == 0 || (cfg->row_bytes % 16) != 0) return UGACHE_EINVAL;
  if (cfg->reserved0 != 0 || (cfg->flags & ~UGACHE_FLAG_HOST_TIER) != 0) return UGACHE_EINVAL;
  if (cfg->policy < UGACHE_POLICY_UGACHE || cfg->policy > UGACHE_POLICY_PARTITION)
    return UGACHE_EINVAL;
  if (cfg->bw_local < 0 || cfg->bw_peer < 0 || cfg->bw_host < 0) return UGACHE_EINVAL;
  if (cfg->host_sms < 0 || cfg->peer_sms < 0 || cfg->num_sms < 0) return UGACHE_EINVAL;
  const int S = cfg->num_sms ? cfg->num_sms : (device_sms > 0 ? device_sms : kDefaultNumSms);
  const int host_sms = cfg->host_sms ? cfg->host_sms : std::min(kDefaultHostSms, S - 1);
  const double R = (double)cfg->row_bytes;
  const double bl = cfg->bw_local > 0 ? cfg->bw_local : kDefaultBwLocal;
  const double bp = cfg->bw_peer > 0 ? cfg->bw_peer : kDefaultBwPeer;
  const double bh = cfg->bw_host > 0 ? cfg->bw_host : kDefaultBwHost;
  // SMs per peer: the paper's even split of the SMs left after the host.  The
  // B200 refinement -- cap it at the NVLink tolerance -- is a
  // measurement: ugache_calibrate under all-to-all load, applied by the caller
  // (ugache_set_dedication; bench.py does at N > 1).  DESIGN.md R14.
  int peer_sms = 0;
  if (G > 1) peer_sms = cfg->peer_sms ? cfg->peer_sms : (S - host_sms) / (G - 1);
  if (host_sms < 1 || host_sms >= S) return UGACHE_EINVAL;
  if (G > 1 && (peer_sms < 1 || (int64_t)host_sms + (int64_t)(G - 1) * peer_sms > S))
    return UGACHE_EINVAL;
  p->S = S;
  p->host_sms = host_sms;
  p->peer_sms = peer_sms;
  p->T_L = R / bl;
  p->T_P = R / (bp / (double)std::max(G - 1, 1));  // 1/(G-1) of the link per peer
  p->T_H = R / bh;
  p->R_L = 1.0;                                      // local padding may use every core
  p->R_P = (double)peer_sms / (double)S;
  p->R_H = (double)host_sms / (double)S;
  return UGACHE_OK;
}

// Stable LSD radix sort of (descending hotness, ascending key): the input is in key order,
// so a stable sort on the 32-bit transformed hotness alone breaks ties by key.
static void sort_by_hotness(const float *h, uint64_t N, std::vector<uint32_t> &order) {
  order.resize(N);
  std::vector<uint32_t> kin(N), kout(N), vout(N);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < (int64_t)N; ++i) {
    float x = h[i];
    uint32_t b;
    if (!(x > 0.0f)) x = 0.0f;  // <= 0 and -0.0 -> +0.0 (NaN rejected earlier)
    std::memcpy(&b, &x, 4);
    kin[i] = ~b;                // ascending ~bits == descending value for x >= 0
    order[i] = (uint32_t)i;
  }
  const int T = std::max(1, std::min(omp_get_max_threads(), 64));
  std::vector<uint64_t> hist((size_t)T * 65536);
  uint32_t *ksrc = kin.data(), *kdst = kout.data();
  uint32_t *vsrc = order.data(), *vdst = vout.data();
  for (int pass = 0; pass < 2; ++pass) {
    const int shift = pass * 16;
    std::fill(hist.begin(), hist.end(), 0);
#pragma omp parallel num_threads(T)
    {
      const int t = omp_get_thread_num();
      const uint64_t lo = N * (uint64_t)t / T, hi = N * (uint64_t)(t + 1) / T;
      uint64_t *ht = hist.data() + (size_t)t * 65536;
      for (uint64_t i = lo; i < hi; ++i) ht[(ksrc[i] >> shift) & 0xFFFF]++;
#pragma omp barrier
#pragma omp single
      {
        uint64_t run = 0;
        for (int d = 0; d < 65536; ++d)
          for (int tt = 0; tt < T; ++tt) {
            uint64_t c = hist[(size_t)tt * 65536 + d];
            hist[(size_t)tt * 65536 + d] = run;
            run += c;
          }
      }
      for (uint64_t i = lo; i < hi; ++i) {
        const uint64_t pos = ht[(ksrc[i] >> shift) & 0xFFFF]++;
        kdst[pos] = ksrc[i];
        vdst[pos] = vsrc[i];
      }
    }
    std::swap(ksrc, kdst);
    std::swap(vsrc, vdst);
  }
  if (vsrc != order.data()) std::memcpy(order.data(), vsrc, N * sizeof(uint32_t));
}

namespace {
struct Sweep {
  uint64_t N, C;
  int G;
  Params p;
  std::vector<double> P;  // P[r] = sum of sorted hotness over ranks < r, r <= limit
  std::vector<double> Q;  // Q[r] = hs[r] + Q[r-G]  (residue-class prefix), r < limit
  double total = 0;
  uint64_t limit = 0;

  double class_sum(uint64_t c, uint64_t a, uint64_t b) const {  // ranks r = c mod G in [a,b)
    if (a >= b) return 0.0;
    const uint64_t Gu = (uint64_t)G;
    const uint64_t first = a + ((c + Gu - (a % Gu)) % Gu);
    if (first >= b) return 0.0;
    const uint64_t last = first + ((b - 1 - first) / Gu) * Gu;
    return Q[last] - (first >= Gu ? Q[first - Gu] : 0.0);
  }

  uint64_t band_end(uint64_t k) const { return std::min<uint64_t>(N, k + (uint64_t)G * (C - k)); }

  // z(k) and, optionally, the per-source modeled times of GPU `gpu`.
  double z(uint64_t k) const {
    const uint64_t be = band_end(k);
    const double rep = P[k];
    const double host = total - P[be];
    double m[UGACHE_MAX_GPUS];
    double msum = 0;
    for (int g = 0; g < G; ++g) {
      m[g] = class_sum((k + (uint64_t)g) % (uint64_t)G, k, be);
      msum += m[g];
    }
    // top-2 band masses for max over peers j != i
    int a1 = 0;
    for (int g = 1; g < G; ++g) if (m[g] > m[a1]) a1 = g;
    double second = 0;
    for (int g = 0; g < G; ++g) if (g != a1) second = std::max(second, m[g]);
    double zmax = 0;
    for (int i = 0; i < G; ++i) {
      const double tl = p.T_L * (rep + m[i]);
      const double pmax = (G > 1) ? (i == a1 ? second : m[a1]) : 0.0;
      const double tp_sum = p.T_P * (msum - m[i]);
      const double th = p.T_H * host;
      double ti = std::max(std::max(tl, p.T_P * pmax), th);
      ti = std::max(ti, p.R_L * tl + p.R_P * tp_sum + p.R_H * th);
      zmax = std::max(zmax, ti);
    }
    return zmax;
  }
};
}  // namespace

ugache_status solve(const ugache_config *cfg, int device_sms, const float *hotness,
                    std::vector<uint32_t> &order, ugache_plan *plan) {
  Params p;
  ugache_status st = resolve_params(cfg, device_sms, &p);
  if (st != UGACHE_OK) return st;
  const uint64_t N = cfg->num_rows;
  const int G = cfg->num_gpus;
  if (hotness) {
    bool ok = true;
#pragma omp parallel for reduction(&& : ok)
    for (int64_t i = 0; i < (int64_t)N; ++i) ok = ok && std::isfinite(hotness[i]);
    if (!ok) return UGACHE_EINVAL;
    sort_by_hotness(hotness, N, order);
  } else {
    order.resize(N);
#pragma omp parallel for
    for (int64_t i = 0; i < (int64_t)N; ++i) order[i] = (uint32_t)i;
  }
  Sweep sw;
  sw.N = N;
  sw.C = std::min<uint64_t>(cfg->capacity_rows, N);
  sw.G = G;
  sw.p = p;
  const uint64_t C = sw.C;
  sw.limit = std::min<uint64_t>(N, (uint64_t)G * C);
  sw.P.assign(sw.limit + 1, 0.0);
  sw.Q.assign(sw.limit, 0.0);
  {
    long double run = 0.0L;
    for (uint64_t r = 0; r < sw.limit; ++r) {
      const float x = hotness ? hotness[order[r]] : 1.0f;
      const double hx = x > 0.0f ? (double)x : 0.0;
      run += (long double)hx;
      sw.P[r + 1] = (double)run;
    }
    // residue-class prefix sums in long double per class
    std::vector<long double> acc((size_t)G, 0.0L);
    for (uint64_t r = 0; r < sw.limit; ++r) {
      const float x = hotness ? hotness[order[r]] : 1.0f;
      const double hx = x > 0.0f ? (double)x : 0.0;
      long double &a = acc[r % (uint64_t)G];
      a += (long double)hx;
      sw.Q[r] = (double)a;
    }
    long double tot = run;
    if (hotness) {
      long double tail = 0.0L;
#pragma omp parallel for reduction(+ : tail)
      for (int64_t r = (int64_t)sw.limit; r < (int64_t)N; ++r) {
        const float x = hotness[order[r]];
        tail += (long double)(x > 0.0f ? (double)x : 0.0);
      }
      tot += tail;
    } else {
      tot += (long double)(N - sw.limit);
    }
    sw.total = (double)tot;
  }

  uint64_t best_k = C;
  double best_z = sw.z(C);
  const double z_rep = best_z;
  const double z_part = sw.z(0);
  if (cfg->policy == UGACHE_POLICY_PARTITION && G > 1) {  // G = 1: every policy is k = C
    best_k = 0;
    best_z = z_part;
  } else if (cfg->policy == UGACHE_POLICY_UGACHE && G > 1) {
    // k from C down to 0; strict improvement required, so ties keep the larger k.
    for (uint64_t kk = C; kk-- > 0;) {
      const double zk = sw.z(kk);
      if (zk < best_z * (1.0 - 1e-12)) {
        best_z = zk;
        best_k = kk;
      }
    }
  }
  std::memset(plan, 0, sizeof(*plan));
  plan->policy = cfg->policy;
  plan->num_gpus = G;
  plan->capacity_rows = C;
  plan->k = best_k;
  plan->band_end = sw.band_end(best_k);
  plan->z = best_z;
  plan->z_replication = z_rep;
  plan->z_partition = z_part;
  plan->T_local = p.T_L;
  plan->T_peer = p.T_P;
  plan->T_host = p.T_H;
  plan->R_local = p.R_L;
  plan->R_peer = p.R_P;
  plan->R_host = p.R_H;
  plan->host_sms = p.host_sms;
  plan->peer_sms = p.peer_sms;
  plan->num_sms = p.S;
  {
    const uint64_t be = plan->band_end;
    plan->host_mass_frac = sw.total > 0 ? std::max(0.0, sw.total - sw.P[be]) / sw.total : 0.0;
  }
  return UGACHE_OK;
}

ugache_status build_placement(const ugache_config *cfg, const uint32_t *order,
                              const ugache_plan *plan, int gpu, uint64_t *loc,
                              uint64_t *slot_keys, uint64_t *n_slots) {
  const uint64_t N = cfg->num_rows;
  const int G = cfg->num_gpus;
  if (gpu < 0 || gpu >= G || !plan || plan->num_gpus != G) return UGACHE_EINVAL;
  const uint64_t C = plan->capacity_rows, k = plan->k, be = plan->band_end;
  if (k > C || be > N || be < k || C > N) return UGACHE_EINVAL;
  const uint64_t host_tag = (uint64_t)G << UGACHE_LOC_SRC_SHIFT;
  if (loc) {
#pragma omp parallel for schedule(static)
    for (int64_t key = 0; key < (int64_t)N; ++key) loc[key] = host_tag | (uint64_t)key;
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < (int64_t)k; ++r)
      loc[order[r]] = ((uint64_t)gpu << UGACHE_LOC_SRC_SHIFT) | (uint64_t)r;
#pragma omp parallel for schedule(static)
    for (int64_t r = (int64_t)k; r < (int64_t)be; ++r) {
      const uint64_t d = (uint64_t)r - k;
      const uint64_t owner = d % (uint64_t)G, slot = k + d / (uint64_t)G;
      loc[order[r]] = (owner << UGACHE_LOC_SRC_SHIFT) | slot;
    }
    if (cfg->flags & UGACHE_FLAG_HOST_TIER) {  // host rows are tier slots: rank - band_end
#pragma omp parallel for schedule(static)
      for (int64_t r = (int64_t)be; r < (int64_t)N; ++r)
        loc[order[r]] = host_tag | ((uint64_t)r - be);
    }
  }
  uint64_t ns = k;
  if (be - k > (uint64_t)gpu) ns += (be - k - (uint64_t)gpu + (uint64_t)G - 1) / (uint64_t)G;
  if (ns > C) return UGACHE_EINVAL;
  if (slot_keys) {
    for (uint64_t r = 0; r < k; ++r) slot_keys[r] = order[r];
    for (uint64_t s = k; s < ns; ++s) slot_keys[s] = order[k + (s - k) * (uint64_t)G + (uint64_t)gpu];
  }
  if (n_slots) *n_slots = ns;
  return UGACHE_OK;
}

// tier[t] = table[order[(be + t) mod N]] for t < N (parallel, first touch by the copying
// thread): the host-resident ranks [be, N) first, in rank order, then the cached ranks
// [0, be) -- the slots a cache refresh may redirect evicted keys to.
template <typename OrderT>
void fill_host_tier_impl(const uint8_t *table, uint32_t R, const OrderT *order, uint64_t be,
                         uint64_t N, uint8_t *tier) {
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < (int64_t)N; ++t) {
    const uint64_t r = ((uint64_t)t + be) % N;
    std::memcpy(tier + (uint64_t)t * R, table + (uint64_t)order[r] * R, R);
  }
}

void fill_host_tier(const uint8_t *table, uint32_t R, const uint64_t *order, uint64_t be,
                    uint64_t N, uint8_t *tier) {
  fill_host_tier_impl(table, R, order, be, N, tier);
}

void fill_host_tier(const uint8_t *table, uint32_t R, const uint32_t *order, uint64_t be,
                    uint64_t N, uint8_t *tier) {
  fill_host_tier_impl(table, R, order, be, N, tier);
}

}  // namespace ug

extern "C" {

ugache_status ugache_solve(const ugache_config *cfg, const float *hotness, uint64_t *order,
                           ugache_plan *plan) {
  if (!cfg || !plan) return UGACHE_EINVAL;
  std::vector<uint32_t> ord;
  ugache_status st = ug::solve(cfg, 0, hotness, ord, plan);
  if (st != UGACHE_OK) return st;
  if (order) {
#pragma omp parallel for
    for (int64_t i = 0; i < (int64_t)cfg->num_rows; ++i) order[i] = ord[i];
  }
  return UGACHE_OK;
}

ugache_status ugache_build_placement(const ugache_config *cfg, const uint64_t *order,
                                     const ugache_plan *plan, int32_t gpu, uint64_t *loc,
                                     uint64_t *slot_keys, uint64_t *n_slots) {
  if (!cfg || !order || !plan) return UGACHE_EINVAL;
  ug::Params p;
  ugache_status st = ug::resolve_params(cfg, 0, &p);
  if (st != UGACHE_OK) return st;
  std::vector<uint32_t> ord(cfg->num_rows);
  for (uint64_t i = 0; i < cfg->num_rows; ++i) {
    if (order[i] >= cfg->num_rows) return UGACHE_EINVAL;
    ord[i] = (uint32_t)order[i];
  }
  return ug::build_placement(cfg, ord.data(), plan, gpu, loc, slot_keys, n_slots);
}

ugache_status ugache_model_time(const ugache_plan *plan, int32_t num_gpus, uint64_t num_rows,
                                const uint64_t *const *locs, const float *hotness, double *z) {
  if (!plan || !locs || !z || num_gpus < 1 || num_gpus > UGACHE_MAX_GPUS || num_rows == 0)
    return UGACHE_EINVAL;
  const int G = num_gpus, M = G + 1;
  for (int i = 0; i < G; ++i)
    if (!locs[i]) return UGACHE_EINVAL;
  // mass[i][j] = sum of hotness over the keys GPU i reads from source j
  std::vector<double> mass((size_t)G * M, 0.0);
  bool ok = true;
  for (int i = 0; i < G; ++i) {
    std::vector<double> m(M, 0.0);
#pragma omp parallel
    {
      std::vector<double> part(M, 0.0);
      bool good = true;
#pragma omp for schedule(static)
      for (int64_t k = 0; k < (int64_t)num_rows; ++k) {
        const uint64_t src = locs[i][k] >> UGACHE_LOC_SRC_SHIFT;
        const float h = hotness ? hotness[k] : 1.0f;
        if (src > (uint64_t)G || !std::isfinite(h)) good = false;
        else part[src] += h > 0.0f ? (double)h : 0.0;
      }
#pragma omp critical
      {
        for (int j = 0; j < M; ++j) m[j] += part[j];
        ok = ok && good;
      }
    }
    for (int j = 0; j < M; ++j) mass[(size_t)i * M + j] = m[j];
  }
  if (!ok) return UGACHE_EINVAL;
  // t^j_i = T_{i<-j} * mass, t_i = max(max_j t^j_i, sum_j R_{i<-j} t^j_i), z = max_i t_i
  double zmax = 0.0;
  for (int i = 0; i < G; ++i) {
    double tmax = 0.0, area = 0.0;
    for (int j = 0; j < M; ++j) {
      const bool host = j == G, local = j == i;
      const double T = host ? plan->T_host : (local ? plan->T_local : plan->T_peer);
      const double Rr = host ? plan->R_host : (local ? plan->R_local : plan->R_peer);
      const double t = T * mass[(size_t)i * M + j];
      tmax = std::max(tmax, t);
      area += Rr * t;
    }
    zmax = std::max(zmax, std::max(tmax, area));
  }
  *z = zmax;
  return UGACHE_OK;
}

uint64_t ugache_host_tier_rows(const ugache_plan *plan, uint64_t num_rows) {
  if (!plan || plan->band_end > num_rows) return 0;
  return num_rows;
}

ugache_status ugache_fill_host_tier(const ugache_config *cfg, const uint64_t *order,
                                    const ugache_plan *plan, const void *host_table,
                                    void *tier) {
  if (!cfg || !order || !plan || !host_table) return UGACHE_EINVAL;
  ug::Params p;
  ugache_status st = ug::resolve_params(cfg, 0, &p);
  if (st != UGACHE_OK) return st;
  const uint64_t N = cfg->num_rows, be = plan->band_end;
  if (be > N) return UGACHE_EINVAL;
  if (!tier) return UGACHE_EINVAL;
  ug::fill_host_tier(static_cast<const uint8_t *>(host_table), cfg->row_bytes, order, be, N,
                     static_cast<uint8_t *>(tier));
  return UGACHE_OK;
}

}  // extern "C"
