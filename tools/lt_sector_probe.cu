// tools/lt_sector_probe.cu -- how many L2 sectors / DRAM bytes does one random 8-byte
// location-table lookup cost on B200?  500K random u64 loads from an 888 MB array (gnn_pa's
// location table), one per thread, summed into a sink; run under ncu for
// lts__t_sectors_srcunit_tex_op_read.sum and dram__bytes_read.sum.  Variants: 0 ld.global.nc,
// 1 ld.global.cg, 2 with cudaLimitMaxL2FetchGranularity = 32, 3 a 16-byte cp.async.bulk (TMA)
// of the aligned pair holding the entry.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <random>

__global__ void lookups(const uint64_t *__restrict__ t, const uint32_t *__restrict__ idx, uint32_t n,
                        unsigned long long *sink, int cg) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint64_t v;
  const uint64_t *p = t + idx[i];
  if (cg) asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p));
  else asm volatile("ld.global.nc.u64 %0, [%1];" : "=l"(v) : "l"(p));
  if (v == 0x12345) atomicAdd(sink, 1ull);
}

__global__ void lookups_tma(const uint64_t *__restrict__ t, const uint32_t *__restrict__ idx, uint32_t n,
                            unsigned long long *sink) {
  __shared__ __align__(16) uint64_t buf[256][2];
  __shared__ __align__(8) uint64_t bar[256];
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar[threadIdx.x]);
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(&buf[threadIdx.x][0]);
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  if (i >= n) return;
  const uint32_t k = idx[i];
  const uint64_t *p = t + (k & ~1u);
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], 16;" ::"r"(b) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 16, [%2];"
               ::"r"(d), "l"(p), "r"(b) : "memory");
  uint32_t done = 0;
  while (!done)
    asm volatile("{ .reg .pred q; mbarrier.try_wait.parity.shared::cta.b64 q, [%1], 0; selp.u32 %0, 1, 0, q; }"
                 : "=r"(done) : "r"(b) : "memory");
  const uint64_t v = buf[threadIdx.x][k & 1u];
  if (v == 0x12345) atomicAdd(sink, 1ull);
}

int main(int argc, char **argv) {
  const int variant = argc > 1 ? atoi(argv[1]) : 0;
  const uint64_t N = 111000000ull;
  const uint32_t n = 500000;
  uint64_t *t;
  uint32_t *idx;
  unsigned long long *sink;
  cudaMalloc(&t, N * 8);
  cudaMemset(t, 1, N * 8);
  cudaMalloc(&idx, n * 4);
  cudaMalloc(&sink, 8);
  std::vector<uint32_t> h(n);
  std::mt19937_64 rng(1);
  for (auto &x : h) x = (uint32_t)(rng() % N);
  cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice);
  if (variant == 2) cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, 32);
  uint8_t *flush;
  cudaMalloc(&flush, 256 << 20);
  for (int r = 0; r < 3; ++r) {
    cudaMemset(flush, r, 256 << 20);
    if (variant == 3) lookups_tma<<<(n + 255) / 256, 256>>>(t, idx, n, sink);
    else lookups<<<(n + 255) / 256, 256>>>(t, idx, n, sink, variant == 1);
  }
  cudaDeviceSynchronize();
  printf("variant %d: %s\n", variant, cudaGetErrorString(cudaGetLastError()));
  return 0;
}
