// tools/pcie_probe.cu -- A0 calibration microbenchmark (Fig. 6 analog) for the
// host source on a B200 box: bandwidth of random 512-B row reads from pinned, mapped host
// memory vs (a) number of SMs, (b) access instruction (LDG.128 per lane vs one
// cp.async.bulk per row into shared memory), (c) rows in flight, (d) table size.
// Standalone (not part of libugache); prints CSV.
#include <cuda.h>
#include <cuda_runtime.h>
#include <sys/mman.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <algorithm>

#define CK(x)                                                                       \
  do {                                                                              \
    cudaError_t e = (x);                                                            \
    if (e != cudaSuccess) {                                                         \
      fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e)); \
      exit(1);                                                                      \
    }                                                                               \
  } while (0)

__device__ __forceinline__ uint4 ldnc(const void *p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

// LDG: warp per row, U rows in flight; rows[i] random row ids; writes to out (device).
template <int U>
__global__ void __launch_bounds__(512, 1) ldg_kernel(const uint8_t *tab, const uint32_t *rows, uint32_t n,
                                                  uint8_t *out, int R) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t W = gridDim.x * (blockDim.x >> 5);
  const int V = R >> 4;
  for (uint32_t e0 = (blockIdx.x * (blockDim.x >> 5) + warp) * U; e0 < n; e0 += W * U) {
    uint32_t r = lane < U && e0 + lane < n ? rows[e0 + lane] : 0;
    uint32_t ru[U];
#pragma unroll
    for (int u = 0; u < U; ++u) ru[u] = __shfl_sync(0xffffffff, r, u);
    for (int j = lane; j < V; j += 32) {
      uint4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = ldnc(tab + (uint64_t)ru[u] * R + j * 16);
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (e0 + u < n) *(uint4 *)(out + (uint64_t)(e0 + u) * R + j * 16) = v[u];
    }
  }
}

// Bulk: each warp owns S stages of one row each in smem; lane 0 issues cp.async.bulk
// global->shared (R bytes), mbarrier completion; then the warp stores the row to out.
template <int S>
__global__ void __launch_bounds__(512, 1) bulk_kernel(const uint8_t *tab, const uint32_t *rows, uint32_t n,
                                                   uint8_t *out, int R) {
  extern __shared__ __align__(128) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  uint8_t *buf = smem + (size_t)warp * S * R;
  __shared__ __align__(8) uint64_t bars[16 * S];
  uint64_t *bar = bars + warp * S;
  if (lane < S) {
    uint32_t a = (uint32_t)__cvta_generic_to_shared(&bar[lane]);
    asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(a));
  }
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const uint32_t W = gridDim.x * nw;
  uint32_t phase[S];
#pragma unroll
  for (int s = 0; s < S; ++s) phase[s] = 0;
  // iterate over groups of S rows per warp
  for (uint32_t e0 = (blockIdx.x * nw + warp) * S; e0 < n; e0 += W * S) {
    if (lane == 0) {
#pragma unroll
      for (int s = 0; s < S; ++s) {
        if (e0 + s < n) {
          const uint32_t r = rows[e0 + s];
          uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar[s]);
          uint32_t d = (uint32_t)__cvta_generic_to_shared(buf + s * R);
          asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(b), "r"(R) : "memory");
          asm volatile(
              "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d),
              "l"(tab + (uint64_t)r * R), "r"(R), "r"(b)
              : "memory");
        }
      }
    }
    __syncwarp();
#pragma unroll
    for (int s = 0; s < S; ++s) {
      if (e0 + s < n) {
        uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar[s]);
        uint32_t done = 0;
        while (!done) {
          asm volatile(
              "{ .reg .pred p; mbarrier.try_wait.parity.shared.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
              : "=r"(done) : "r"(b), "r"(phase[s]) : "memory");
        }
        phase[s] ^= 1;
        for (int j = lane; j < (R >> 4); j += 32)
          *(uint4 *)(out + (uint64_t)(e0 + s) * R + j * 16) = *(const uint4 *)(buf + s * R + j * 16);
      }
    }
    __syncwarp();
  }
}

int main(int argc, char **argv) {
  const size_t table_gb = argc > 1 ? atoll(argv[1]) : 8;
  const int alloc_mode = argc > 2 ? atoi(argv[2]) : 0;  // 0 mmap+THP+register, 1 cudaHostAlloc, 2 mmap no THP
  const int quick = argc > 3 ? atoi(argv[3]) : 0;
  const int order_mode = argc > 4 ? atoi(argv[4]) : 0;  // 0 random, 1 sorted, k>1: grouped into k ranges
  const int R = 512;
  const size_t bytes = table_gb << 30;
  const uint64_t N = bytes / R;
  const uint32_t n = 200000;
  void *h = nullptr;
  if (alloc_mode == 3) {
    cudaFree(0);
    CUmemAllocationProp prop = {};
    prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    prop.location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA;
    prop.location.id = 0;
    size_t gmin = 0, grec = 0;
    cuMemGetAllocationGranularity(&gmin, &prop, CU_MEM_ALLOC_GRANULARITY_MINIMUM);
    cuMemGetAllocationGranularity(&grec, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED);
    fprintf(stderr, "vmm host granularity min %zu rec %zu\n", gmin, grec);
    CUmemGenericAllocationHandle hd;
    CUresult r = cuMemCreate(&hd, bytes, &prop, 0);
    if (r != CUDA_SUCCESS) { fprintf(stderr, "cuMemCreate failed %d\n", (int)r); exit(1); }
    CUdeviceptr va;
    r = cuMemAddressReserve(&va, bytes, grec > gmin ? grec : gmin, 0, 0);
    if (r != CUDA_SUCCESS) { fprintf(stderr, "reserve failed %d\n", (int)r); exit(1); }
    r = cuMemMap(va, bytes, 0, hd, 0);
    if (r != CUDA_SUCCESS) { fprintf(stderr, "map failed %d\n", (int)r); exit(1); }
    CUmemAccessDesc ad[2] = {};
    ad[0].location.type = CU_MEM_LOCATION_TYPE_DEVICE; ad[0].location.id = 0;
    ad[0].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    ad[1].location.type = CU_MEM_LOCATION_TYPE_HOST_NUMA; ad[1].location.id = 0;
    ad[1].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    r = cuMemSetAccess(va, bytes, ad, 2);
    if (r != CUDA_SUCCESS) { fprintf(stderr, "setaccess(2) failed %d, device only\n", (int)r);
      r = cuMemSetAccess(va, bytes, ad, 1); if (r != CUDA_SUCCESS) { fprintf(stderr, "setaccess failed %d\n", (int)r); exit(1);} 
      CK(cudaMemset((void*)va, 1, bytes)); CK(cudaDeviceSynchronize());
    } else {
      memset((void *)va, 1, bytes);
    }
    h = (void *)va;
  } else if (alloc_mode == 1) {
    CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
    memset(h, 1, bytes);
  } else {
    h = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
    madvise(h, bytes, alloc_mode == 2 ? MADV_NOHUGEPAGE : MADV_HUGEPAGE);
    memset(h, 1, bytes);
    CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
  }
  uint8_t *dtab;
  if (alloc_mode == 3) dtab = (uint8_t *)h; else CK(cudaHostGetDevicePointer((void **)&dtab, h, 0));
  std::vector<uint32_t> rows(n);
  uint64_t x = 88172645463325252ull;
  for (uint32_t i = 0; i < n; ++i) {
    x ^= x << 13; x ^= x >> 7; x ^= x << 17;
    rows[i] = (uint32_t)(x % N);
  }
  if (order_mode == 1) {
    std::sort(rows.begin(), rows.end());
  } else if (order_mode > 1) {
    const uint64_t span = (N + order_mode - 1) / order_mode;
    std::stable_sort(rows.begin(), rows.end(),
                     [&](uint32_t x1, uint32_t x2) { return x1 / span < x2 / span; });
  }
  uint32_t *drows;
  uint8_t *out;
  CK(cudaMalloc(&drows, n * 4));
  CK(cudaMalloc(&out, (size_t)n * R));
  CK(cudaMemcpy(drows, rows.data(), n * 4, cudaMemcpyHostToDevice));
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  CK(cudaFuncSetAttribute(bulk_kernel<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16 * 4 * R));
  CK(cudaFuncSetAttribute(bulk_kernel<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16 * 8 * R));
  CK(cudaFuncSetAttribute(bulk_kernel<16>, cudaFuncAttributeMaxDynamicSharedMemorySize, 16 * 16 * R));
  printf("table_gb,method,depth,sms,ms,GBps\n");
  const int sms_list[] = {1, 2, 4, 8, 16, 24, 32, 48, 64, 96, 148};
  for (int method = 0; method < 2; ++method) {
    if (quick && method == 1) continue;
    for (int depth : {4, 8, 16}) {
      if (quick && depth != 8) continue;
      for (int sms : sms_list) {
        if (quick && sms != 8 && sms != 32 && sms != 148) continue;
        float best = 1e9;
        for (int rep = 0; rep < 3; ++rep) {
          cudaEventRecord(a);
          if (method == 0) {
            if (depth == 4) ldg_kernel<4><<<sms, 512>>>(dtab, drows, n, out, R);
            if (depth == 8) ldg_kernel<8><<<sms, 512>>>(dtab, drows, n, out, R);
            if (depth == 16) ldg_kernel<16><<<sms, 512>>>(dtab, drows, n, out, R);
          } else {
            if (depth == 4) bulk_kernel<4><<<sms, 512, 16 * 4 * R>>>(dtab, drows, n, out, R);
            if (depth == 8) bulk_kernel<8><<<sms, 512, 16 * 8 * R>>>(dtab, drows, n, out, R);
            if (depth == 16) bulk_kernel<16><<<sms, 512, 16 * 16 * R>>>(dtab, drows, n, out, R);
          }
          cudaEventRecord(b);
          CK(cudaEventSynchronize(b));
          float ms;
          cudaEventElapsedTime(&ms, a, b);
          if (ms < best) best = ms;
        }
        CK(cudaGetLastError());
        printf("%zu/%d/o%d,%s,%d,%d,%.3f,%.2f\n", table_gb, alloc_mode, order_mode, method ? "bulk" : "ldg", depth, sms, best,
               (double)n * R / (best * 1e-3) / 1e9);
        fflush(stdout);
      }
    }
  }
  if (quick) return 0;
  // contiguous rows (sequential) reference with LDG, all SMs
  for (uint32_t i = 0; i < n; ++i) rows[i] = i;
  CK(cudaMemcpy(drows, rows.data(), n * 4, cudaMemcpyHostToDevice));
  for (int sms : {8, 32, 148}) {
    float best = 1e9;
    for (int rep = 0; rep < 3; ++rep) {
      cudaEventRecord(a);
      ldg_kernel<8><<<sms, 512>>>(dtab, drows, n, out, R);
      cudaEventRecord(b);
      CK(cudaEventSynchronize(b));
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (ms < best) best = ms;
    }
    printf("%zu/%d,ldg_seq,8,%d,%.3f,%.2f\n", table_gb, alloc_mode, sms, best, (double)n * R / (best * 1e-3) / 1e9);
  }
  return 0;
}
