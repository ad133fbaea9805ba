// tools/host_split_probe.cu -- round-2 verdict item 3, second lever: does copy-engine DMA
// of a CPU-gathered slice of the host bucket add bandwidth alongside the zero-copy reads?
// Standalone (not part of libugache); prints CSV.
//
//   host_split_probe <tier_rows> <draws> <nbatches> [threads_list] [fractions]
//
// The host source is an anonymous THP buffer of tier_rows x 512 B, cudaHostRegister'ed (the
// library's host tier).  Each batch's host bucket is `draws` draws of a continuous Zipf(1.2)
// over tier ranks [r0, r0 + tier_rows) (r0 = tier_rows / 9, gnn_pa's band end at c = 10 %),
// deduplicated and sorted (the library's range ordering).  Every batch is distinct and the
// L2 is flushed (1 GiB write) before every leg, so no leg sees another's translations warm.
//
// Legs (ms per batch, median over batches):
//   zc      the ordered zero-copy copy: 12 SMs spread over the chip, 12 warps, 8 rows/warp
//   cpu     T host threads gather the bucket into a pinned staging buffer (memcpy per row)
//   dma     one cudaMemcpyAsync of the staged bucket to HBM
//   pipe    cpu + dma pipelined in 4096-row chunks (threads gather chunk i+1 while i moves)
//   split f the sparse cold end (last f of the sorted bucket) through pipe, the rest through
//           zc, concurrently; wall time from launch until both are done
#include <cuda_runtime.h>
#include <sys/mman.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <string>
#include <thread>
#include <vector>

#define CK(x)                                                                              \
  do {                                                                                     \
    cudaError_t e = (x);                                                                   \
    if (e != cudaSuccess) {                                                                \
      fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e));    \
      exit(1);                                                                             \
    }                                                                                      \
  } while (0)

constexpr int R = 512;
constexpr uint32_t kChunk = 4096;

__device__ __forceinline__ uint4 ldnc(const void *p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

__global__ void smid_kernel(uint32_t *ids) {
  uint32_t s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  if (threadIdx.x == 0) ids[blockIdx.x] = s;
}

// the library's host_copy_ordered loop: warps claim 8 consecutive entries from a cursor
__global__ void __launch_bounds__(512, 1)
    zc_copy(const uint8_t *tab, const uint32_t *rows, uint32_t n, uint8_t *out, const uint8_t *active,
            int warps, uint32_t *cursor) {
  constexpr int U = 8;
  uint32_t s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (!active[s] || warp >= warps) return;
  uint32_t next = 0;
  if (lane == 0) next = atomicAdd(cursor, (uint32_t)U);
  next = __shfl_sync(~0u, next, 0);
  while (next < n) {
    const uint32_t e0 = next;
    if (lane == 0) next = atomicAdd(cursor, (uint32_t)U);
    next = __shfl_sync(~0u, next, 0);
    const int nv = (int)min((uint32_t)U, n - e0);
    const uint32_t r = lane < nv ? rows[e0 + lane] : 0u;
    uint32_t ru[U];
#pragma unroll
    for (int u = 0; u < U; ++u) ru[u] = __shfl_sync(~0u, r, u);
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (u < nv) v[u] = ldnc(tab + (uint64_t)ru[u] * R + lane * 16);
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (u < nv) *(uint4 *)(out + (uint64_t)(e0 + u) * R + lane * 16) = v[u];
  }
}

static double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

// T threads gather rows[0..n) of tab into stage; chunk c is ready when left[c] reaches 0
struct Gather {
  const uint8_t *tab;
  const uint32_t *rows;
  uint32_t n;
  uint8_t *stage;
  std::vector<std::atomic<int>> *left;  // threads still working on chunk c
};

static void gather_worker(Gather *g, int T, int t) {
  const uint32_t nch = (g->n + kChunk - 1) / kChunk;
  for (uint32_t c = 0; c < nch; ++c) {
    const uint32_t b = c * kChunk, e = std::min(g->n, b + kChunk);
    const uint32_t lo = b + (e - b) * t / T, hi = b + (e - b) * (t + 1) / T;
    for (uint32_t i = lo; i < hi; ++i) memcpy(g->stage + (uint64_t)i * R, g->tab + (uint64_t)g->rows[i] * R, R);
    (*g->left)[c].fetch_sub(1, std::memory_order_release);
  }
}

// CPU gather + chunked DMA to dst; returns when every copy is enqueued (caller syncs stream)
static void pipe_run(const uint8_t *tab, const uint32_t *rows, uint32_t n, uint8_t *stage, uint8_t *dst,
                     int T, cudaStream_t st, bool dma) {
  if (n == 0) return;
  const uint32_t nch = (n + kChunk - 1) / kChunk;
  std::vector<std::atomic<int>> left(nch);
  for (auto &l : left) l.store(T);
  Gather g{tab, rows, n, stage, &left};
  std::vector<std::thread> th;
  for (int t = 0; t < T; ++t) th.emplace_back(gather_worker, &g, T, t);
  for (uint32_t c = 0; c < nch; ++c) {
    while (left[c].load(std::memory_order_acquire) != 0) {
    }
    const uint64_t b = (uint64_t)c * kChunk, en = std::min<uint64_t>(n, b + kChunk);
    if (dma) CK(cudaMemcpyAsync(dst + b * R, stage + b * R, (en - b) * R, cudaMemcpyHostToDevice, st));
  }
  for (auto &t : th) t.join();
}

int main(int argc, char **argv) {
  if (argc < 4) {
    fprintf(stderr, "usage: %s tier_rows draws nbatches [threads,..] [f,..]\n", argv[0]);
    return 2;
  }
  const uint64_t N = strtoull(argv[1], nullptr, 10);
  const uint64_t draws = strtoull(argv[2], nullptr, 10);
  const int nb = atoi(argv[3]);
  std::vector<int> tlist = {4, 8, 16};
  std::vector<double> flist = {0.1, 0.2, 0.3, 0.4, 0.5};
  auto parse = [](const char *s, auto &v) {
    v.clear();
    std::string x = s;
    size_t p = 0;
    while (p < x.size()) {
      size_t q = x.find(',', p);
      if (q == std::string::npos) q = x.size();
      v.push_back(atof(x.substr(p, q - p).c_str()));
      p = q + 1;
    }
  };
  if (argc > 4) parse(argv[4], tlist);
  if (argc > 5) parse(argv[5], flist);

  // batches: continuous Zipf(1.2) over ranks [r0, r0 + N), dedup, sort
  const double a = 1.2, r0 = (double)(N / 9), r1 = r0 + (double)N;
  const double A = std::pow(r0, 1 - a), B = std::pow(r1, 1 - a);
  std::vector<std::vector<uint32_t>> batches(nb);
  for (int i = 0; i < nb; ++i) {
    std::mt19937_64 rng(0x5eed + i);
    std::uniform_real_distribution<double> U01(0, 1);
    auto &v = batches[i];
    v.reserve(draws);
    for (uint64_t d = 0; d < draws; ++d) {
      const double r = std::pow(A + U01(rng) * (B - A), 1 / (1 - a));
      v.push_back((uint32_t)std::min<double>(N - 1, std::floor(r - r0)));
    }
    std::sort(v.begin(), v.end());
    v.erase(std::unique(v.begin(), v.end()), v.end());
  }
  size_t maxn = 0;
  for (auto &v : batches) maxn = std::max(maxn, v.size());
  fprintf(stderr, "tier %llu rows (%.1f GB), %d batches of ~%zu unique host rows\n", (unsigned long long)N,
          N * 512.0 / 1e9, nb, maxn);

  const size_t bytes = N * (size_t)R;
  uint8_t *h = (uint8_t *)mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  if (h == MAP_FAILED) { perror("mmap"); return 1; }
  madvise(h, bytes, MADV_HUGEPAGE);
  {
    std::vector<std::thread> th;
    for (int t = 0; t < 16; ++t)
      th.emplace_back([=] {
        const uint64_t lo = N * t / 16, hi = N * (t + 1) / 16;
        memset(h + lo * R, 1 + t, (hi - lo) * R);
        for (uint64_t r = lo; r < hi; ++r) memcpy(h + r * R, &r, 8);  // rows tell themselves apart
      });
    for (auto &t : th) t.join();
  }
  const double tpin = now_ms();
  CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
  fprintf(stderr, "pinned in %.1f s\n", (now_ms() - tpin) / 1e3);
  uint8_t *dtab;
  CK(cudaHostGetDevicePointer((void **)&dtab, h, 0));

  int S;
  CK(cudaDeviceGetAttribute(&S, cudaDevAttrMultiProcessorCount, 0));
  uint32_t *dids;
  CK(cudaMalloc(&dids, S * 4));
  CK(cudaFuncSetAttribute(zc_copy, cudaFuncAttributeMaxDynamicSharedMemorySize, 120 << 10));
  CK(cudaFuncSetAttribute(smid_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 120 << 10));
  smid_kernel<<<S, 32, 120 << 10>>>(dids);
  std::vector<uint32_t> ids(S);
  CK(cudaMemcpy(ids.data(), dids, S * 4, cudaMemcpyDeviceToHost));
  std::sort(ids.begin(), ids.end());
  uint8_t *dact;
  CK(cudaMalloc(&dact, 256));
  {
    std::vector<uint8_t> act(256, 0);
    for (int i = 0; i < 12; ++i) act[ids[(size_t)i * S / 12]] = 1;
    CK(cudaMemcpy(dact, act.data(), 256, cudaMemcpyHostToDevice));
  }
  std::vector<uint32_t *> dr(nb);
  for (int i = 0; i < nb; ++i) {
    CK(cudaMalloc(&dr[i], batches[i].size() * 4));
    CK(cudaMemcpy(dr[i], batches[i].data(), batches[i].size() * 4, cudaMemcpyHostToDevice));
  }
  uint8_t *out, *stage, *flush;
  uint32_t *dcur;
  CK(cudaMalloc(&out, maxn * R));
  CK(cudaMalloc(&flush, 1 << 30));
  CK(cudaMalloc(&dcur, 4));
  CK(cudaHostAlloc((void **)&stage, maxn * R, cudaHostAllocPortable));
  memset(stage, 0, maxn * R);
  cudaStream_t s1, s2;
  CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));

  // host DMA peak: 1 GiB pinned -> device, best of 5
  double dma_peak = 0;
  {
    uint8_t *hb, *db;
    CK(cudaHostAlloc((void **)&hb, 1 << 30, cudaHostAllocPortable));
    memset(hb, 3, 1 << 30);
    CK(cudaMalloc(&db, 1 << 30));
    for (int i = 0; i < 5; ++i) {
      const double t0 = now_ms();
      CK(cudaMemcpyAsync(db, hb, 1 << 30, cudaMemcpyHostToDevice, s1));
      CK(cudaStreamSynchronize(s1));
      dma_peak = std::max(dma_peak, (1 << 30) / ((now_ms() - t0) * 1e-3) / 1e9);
    }
    CK(cudaFree(db));
    CK(cudaFreeHost(hb));
  }
  fprintf(stderr, "pinned H2D DMA peak %.1f GB/s, %d host threads available\n", dma_peak,
          (int)std::thread::hardware_concurrency());

  auto flush_l2 = [&](int i) {
    CK(cudaMemsetAsync(flush, i & 0xff, 1 << 30, s1));
    CK(cudaStreamSynchronize(s1));
  };
  auto zc_launch = [&](int i, uint32_t off, uint32_t cnt) {
    CK(cudaMemsetAsync(dcur, 0, 4, s1));
    if (cnt) zc_copy<<<S, 512, 120 << 10, s1>>>(dtab, dr[i] + off, cnt, out + (uint64_t)off * R, dact, 12, dcur);
  };
  auto median = [](std::vector<double> v) {
    std::sort(v.begin(), v.end());
    return v[v.size() / 2];
  };
  printf("leg,threads,f,ms,host_rows,GBps\n");
  auto report = [&](const char *leg, int T, double f, std::vector<double> &ms) {
    double rows = 0;
    for (auto &b : batches) rows += b.size();
    rows /= nb;
    const double m = median(ms);
    printf("%s,%d,%.2f,%.4f,%.0f,%.2f\n", leg, T, f, m, rows, rows * R / (m * 1e-3) / 1e9);
    fflush(stdout);
  };
  // each leg walks the batches in a different rotation, so no batch is re-read soon after
  int rot = 0;
  auto order = [&](int j) { return (j + rot) % nb; };
  {  // zc
    std::vector<double> ms;
    for (int j = 0; j < nb; ++j) {
      const int i = order(j);
      flush_l2(j);
      const double t0 = now_ms();
      zc_launch(i, 0, (uint32_t)batches[i].size());
      CK(cudaStreamSynchronize(s1));
      ms.push_back(now_ms() - t0);
    }
    report("zc", 0, 0, ms);
    rot += 3;
  }
  for (int T : tlist) {  // cpu alone, then pipe
    std::vector<double> mc, md, mp;
    for (int j = 0; j < nb; ++j) {
      const int i = order(j);
      const uint32_t n = (uint32_t)batches[i].size();
      flush_l2(j);
      double t0 = now_ms();
      pipe_run(h, batches[i].data(), n, stage, nullptr, T, s2, false);
      mc.push_back(now_ms() - t0);
      t0 = now_ms();
      CK(cudaMemcpyAsync(out, stage, (size_t)n * R, cudaMemcpyHostToDevice, s2));
      CK(cudaStreamSynchronize(s2));
      md.push_back(now_ms() - t0);
    }
    rot += 3;
    for (int j = 0; j < nb; ++j) {
      const int i = order(j);
      flush_l2(j);
      const double t0 = now_ms();
      pipe_run(h, batches[i].data(), (uint32_t)batches[i].size(), stage, out, T, s2, true);
      CK(cudaStreamSynchronize(s2));
      mp.push_back(now_ms() - t0);
    }
    rot += 3;
    report("cpu", T, 1, mc);
    report("dma", T, 1, md);
    report("pipe", T, 1, mp);
  }
  int last = 0;
  for (int T : tlist) {
    for (double f : flist) {
      std::vector<double> ms;
      for (int j = 0; j < nb; ++j) {
        const int i = order(j);
        last = i;
        const uint32_t n = (uint32_t)batches[i].size();
        const uint32_t nz = (uint32_t)std::lround(n * (1 - f));
        flush_l2(j);
        const double t0 = now_ms();
        zc_launch(i, 0, nz);
        pipe_run(h, batches[i].data() + nz, n - nz, stage, out + (uint64_t)nz * R, T, s2, true);
        CK(cudaStreamSynchronize(s2));
        CK(cudaStreamSynchronize(s1));
        ms.push_back(now_ms() - t0);
      }
      rot += 3;
      report("split", T, f, ms);
    }
  }
  // parity of the last split against the table (spot check, the probe's own sanity)
  {
    const int i = last;
    std::vector<uint8_t> o((size_t)batches[i].size() * R);
    CK(cudaMemcpy(o.data(), out, o.size(), cudaMemcpyDeviceToHost));
    size_t bad = 0;
    for (size_t k = 0; k < batches[i].size(); ++k)
      bad += memcmp(o.data() + k * R, h + (uint64_t)batches[i][k] * R, R) != 0;
    fprintf(stderr, "last split batch: %zu / %zu rows differ\n", bad, batches[i].size());
  }
  return 0;
}
