// tools/host_order_probe.cu -- A0 follow-up ("the host source"):
// how fast can the host rows of ONE real batch be read from pinned host memory, and in
// which order / with how many SMs, warps and rows in flight?  Standalone (not part of
// libugache); prints CSV.
//
//   host_order_probe <rows.bin> <table_rows>
//
// rows.bin: uint32 host-row ids of one batch in batch order (tools/host_order_probe.py
// writes the gnn_pa host bucket in host-tier layout).  The table is anonymous THP memory,
// cudaHostRegister'ed, of table_rows x 512 B.
//
// Orders: 0 = batch order, 1 = 4096 ranges (the library's ordering), 2 = 32768 ranges,
// 3 = full sort.  Copy: warps of the active CTAs claim U consecutive entries from a global
// cursor (the library's host_copy_ordered).  Active CTAs are chosen by %smid, spread over
// the chip (every (S/H)-th SM id in ascending order).  (An earlier copy-engine leg with one
// 512-B copy per row was removed: that batched-copy call is closed on this GPU pool.)
#include <cuda.h>
#include <cuda_runtime.h>
#include <sys/mman.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <string>
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

template <int U>
__global__ void __launch_bounds__(512, 1)
    ordered_copy(const uint8_t *tab, const uint32_t *rows, uint32_t n, uint8_t *out,
                 const uint8_t *active, int warps, uint32_t *cursor) {
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

int main(int argc, char **argv) {
  if (argc < 3) {
    fprintf(stderr, "usage: %s rows.bin table_rows\n", argv[0]);
    return 2;
  }
  // argv[1]: one or more comma-separated row files (distinct batches, cycled per rep)
  std::vector<std::vector<uint32_t>> batches;
  {
    std::string list = argv[1];
    size_t p0 = 0;
    while (p0 <= list.size()) {
      size_t p1 = list.find(',', p0);
      if (p1 == std::string::npos) p1 = list.size();
      FILE *f = fopen(list.substr(p0, p1 - p0).c_str(), "rb");
      if (!f) { perror("rows"); return 1; }
      std::vector<uint32_t> v;
      uint32_t x;
      while (fread(&x, 4, 1, f) == 1) v.push_back(x);
      fclose(f);
      batches.push_back(v);
      p0 = p1 + 1;
    }
  }
  const std::vector<uint32_t> &batch = batches[0];
  const uint64_t N = strtoull(argv[2], nullptr, 10);
  const uint32_t n = (uint32_t)batch.size();
  const size_t bytes = N * R;
  fprintf(stderr, "%u rows over %.1f GB\n", n, bytes / 1e9);
  // argv[3]: 1 = also cudaHostRegisterReadOnly (what libugache asks for first)
  const int ro = argc > 3 ? atoi(argv[3]) : 0;
  // argv[4]: 1 = quick (orders 0/1, a few shapes)
  const int quick = argc > 4 ? atoi(argv[4]) : 0;
  // argv[5]: host allocation: 0 mmap + MADV_HUGEPAGE, 1 mmap + MADV_NOHUGEPAGE,
  // 2 cudaHostAlloc, 3 VMM host (cuMemCreate HOST_NUMA), 4 mmap MAP_HUGETLB (2 MB hugetlbfs)
  const int amode = argc > 5 ? atoi(argv[5]) : 0;
  uint8_t *h = nullptr, *dtab = nullptr;
  auto par_memset = [&](uint8_t *p) {
    std::vector<std::thread> th;
    const int T = 16;
    for (int t = 0; t < T; ++t)
      th.emplace_back([=] { memset(p + bytes * t / T, 1, bytes * (t + 1) / T - bytes * t / T); });
    for (auto &t : th) t.join();
  };
  if (amode == 2) {
    CK(cudaHostAlloc((void **)&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
    par_memset(h);
    CK(cudaHostGetDevicePointer((void **)&dtab, h, 0));
  } else if (amode == 3) {
    CK(cudaFree(0));
    CUmemAllocationProp prop = {};
    prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    prop.location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA;
    prop.location.id = 0;
    size_t g = 0;
    cuMemGetAllocationGranularity(&g, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED);
    const size_t sz = (bytes + g - 1) / g * g;
    CUmemGenericAllocationHandle hd;
    if (cuMemCreate(&hd, sz, &prop, 0) != CUDA_SUCCESS) { fprintf(stderr, "cuMemCreate failed\n"); return 1; }
    CUdeviceptr va;
    if (cuMemAddressReserve(&va, sz, g, 0, 0) != CUDA_SUCCESS || cuMemMap(va, sz, 0, hd, 0) != CUDA_SUCCESS) {
      fprintf(stderr, "reserve/map failed\n");
      return 1;
    }
    CUmemAccessDesc ad[2] = {};
    ad[0].location.type = CU_MEM_LOCATION_TYPE_DEVICE; ad[0].location.id = 0;
    ad[0].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    ad[1].location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA; ad[1].location.id = 0;
    ad[1].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    if (cuMemSetAccess(va, sz, ad, 2) != CUDA_SUCCESS) {
      if (cuMemSetAccess(va, sz, ad, 1) != CUDA_SUCCESS) { fprintf(stderr, "setaccess failed\n"); return 1; }
      CK(cudaMemset((void *)va, 1, bytes));
      CK(cudaDeviceSynchronize());
    } else {
      par_memset((uint8_t *)va);
    }
    fprintf(stderr, "vmm host granularity %zu\n", g);
    h = dtab = (uint8_t *)va;
  } else {
    int fl = MAP_PRIVATE | MAP_ANONYMOUS | (amode == 4 ? MAP_HUGETLB : 0);
    h = (uint8_t *)mmap(nullptr, bytes, PROT_READ | PROT_WRITE, fl, -1, 0);
    if (h == MAP_FAILED) { perror("mmap"); return 1; }
    if (amode != 4) madvise(h, bytes, amode == 1 ? MADV_NOHUGEPAGE : MADV_HUGEPAGE);
    par_memset(h);
    CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable |
                                      (ro ? cudaHostRegisterReadOnly : 0)));
    CK(cudaHostGetDevicePointer((void **)&dtab, h, 0));
  }
  {
    FILE *m = fopen("/proc/meminfo", "r");
    char line[256];
    while (m && fgets(line, sizeof line, m))
      if (strstr(line, "AnonHugePages") || strstr(line, "HugePages_")) fprintf(stderr, "%s", line);
    if (m) fclose(m);
  }
  int S;
  CK(cudaDeviceGetAttribute(&S, cudaDevAttrMultiProcessorCount, 0));
  uint32_t *dids;
  CK(cudaMalloc(&dids, S * 4));
  CK(cudaFuncSetAttribute(ordered_copy<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 120 << 10));
  CK(cudaFuncSetAttribute(ordered_copy<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 120 << 10));
  CK(cudaFuncSetAttribute(ordered_copy<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 120 << 10));
  CK(cudaFuncSetAttribute(smid_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 120 << 10));
  smid_kernel<<<S, 32, 120 << 10>>>(dids);
  std::vector<uint32_t> ids(S);
  CK(cudaMemcpy(ids.data(), dids, S * 4, cudaMemcpyDeviceToHost));
  std::sort(ids.begin(), ids.end());
  uint32_t *drows, *dcur;
  uint8_t *out, *dact;
  CK(cudaMalloc(&drows, (size_t)n * 4));
  CK(cudaMalloc(&dcur, 4));
  CK(cudaMalloc(&dact, 256));
  CK(cudaMalloc(&out, (size_t)n * R));
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const uint32_t maxrow = *std::max_element(batch.begin(), batch.end());
  printf("order,sms,warps,U,ms,GBps,first_pass_ms\n");
  size_t maxn = 0;
  for (auto &v : batches) maxn = std::max(maxn, v.size());
  const int nb = (int)batches.size();
  std::vector<uint32_t *> dr(nb);
  for (int i = 0; i < nb; ++i) CK(cudaMalloc(&dr[i], batches[i].size() * 4));
  uint8_t *out2;
  CK(cudaMalloc(&out2, maxn * R));
  // cold: 1 GiB device buffer written between launches (flushes L2, not the host TLBs)
  uint8_t *flush;
  CK(cudaMalloc(&flush, 1 << 30));
  for (int order : {0, 1, 2, 3}) {
    if (quick && order > 1) continue;
    std::vector<uint32_t> rows = batch;
    for (int i = 0; i < nb; ++i) {
      std::vector<uint32_t> r = batches[i];
      const uint32_t mx = *std::max_element(r.begin(), r.end());
      if (order == 3) {
        std::sort(r.begin(), r.end());
      } else if (order > 0) {
        const int nr = order == 1 ? 4096 : 32768;
        int shift = 0;
        while (((uint64_t)mx >> shift) >= (uint64_t)nr) ++shift;
        std::stable_sort(r.begin(), r.end(), [=](uint32_t p, uint32_t q) { return (p >> shift) < (q >> shift); });
      }
      CK(cudaMemcpy(dr[i], r.data(), r.size() * 4, cudaMemcpyHostToDevice));
      if (i == 0) rows = r;
    }
    for (int H : {8, 12, 16, 24, 32, 48, 148}) {
      std::vector<uint8_t> act(256, 0);
      for (int i = 0; i < H; ++i) act[ids[(size_t)i * S / H]] = 1;
      CK(cudaMemcpy(dact, act.data(), 256, cudaMemcpyHostToDevice));
      for (int warps : {4, 8, 16}) {
        for (int U : {4, 8, 16}) {
          if (order == 0 && U != 8) continue;
          if (quick && (U != 8 || (warps != 8 && warps != 16) || (H != 12 && H != 48))) continue;
          double tot = 0, tot_first = 0;
          uint64_t rows_tot = 0;
          for (int rep = 0; rep < 2; ++rep) {
            for (int i = 0; i < nb; ++i) {
              const uint32_t ni = (uint32_t)batches[i].size();
              CK(cudaMemset(flush, rep + i, 1 << 30));
              CK(cudaMemset(dcur, 0, 4));
              cudaEventRecord(a);
              if (U == 4) ordered_copy<4><<<S, 512, 120 << 10>>>(dtab, dr[i], ni, out2, dact, warps, dcur);
              if (U == 8) ordered_copy<8><<<S, 512, 120 << 10>>>(dtab, dr[i], ni, out2, dact, warps, dcur);
              if (U == 16) ordered_copy<16><<<S, 512, 120 << 10>>>(dtab, dr[i], ni, out2, dact, warps, dcur);
              cudaEventRecord(b);
              CK(cudaEventSynchronize(b));
              float ms;
              cudaEventElapsedTime(&ms, a, b);
              if (rep == 0) tot_first += ms;
              else { tot += ms; rows_tot += ni; }
            }
          }
          // ms = mean per batch over the 2nd pass; first = mean over the 1st pass
          printf("%d,%d,%d,%d,%.4f,%.2f,%.4f\n", order, H, warps, U, tot / nb,
                 (double)rows_tot * R / (tot * 1e-3) / 1e9, tot_first / nb);
          fflush(stdout);
        }
      }
    }
  }
  // sequential reference: rows 0..n-1
  {
    std::vector<uint32_t> rows(n);
    for (uint32_t i = 0; i < n; ++i) rows[i] = i;
    CK(cudaMemcpy(drows, rows.data(), (size_t)n * 4, cudaMemcpyHostToDevice));
    for (int H : {12, 32, 148}) {
      std::vector<uint8_t> act(256, 0);
      for (int i = 0; i < H; ++i) act[ids[(size_t)i * S / H]] = 1;
      CK(cudaMemcpy(dact, act.data(), 256, cudaMemcpyHostToDevice));
      float best = 1e9;
      for (int rep = 0; rep < 3; ++rep) {
        CK(cudaMemset(dcur, 0, 4));
        cudaEventRecord(a);
        ordered_copy<8><<<S, 512, 120 << 10>>>(dtab, drows, n, out, dact, 16, dcur);
        cudaEventRecord(b);
        CK(cudaEventSynchronize(b));
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        best = std::min(best, ms);
      }
      printf("seq,%d,16,8,%.4f,%.2f\n", H, best, (double)n * R / (best * 1e-3) / 1e9);
    }
  }
  return 0;
}
