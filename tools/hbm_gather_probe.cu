// tools/hbm_gather_probe.cu -- ceiling of the local-HBM row gather (A4) on one B200.
// out[i] = slab[rows[i]] for n random rows of R bytes from a large device slab, with the
// L2 flushed between launches.  Variants: LDG.128 rows-in-flight U x warps per SM (the
// library's register path), TMA bulk global->shared->global (with / without evict-first
// L2 hints), and a STREAM-style cudaMemcpy D2D reference.  Standalone; prints CSV.
//   hbm_gather_probe [slab_gb=57] [n=500000] [R=512]
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <random>
#include <vector>

#define CK(x)                                                                           \
  do {                                                                                  \
    cudaError_t e = (x);                                                                \
    if (e != cudaSuccess) {                                                             \
      fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e)); \
      exit(1);                                                                          \
    }                                                                                   \
  } while (0)

__device__ __forceinline__ uint4 ldnc(const void *p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ void stcs(void *p, const uint4 &v) {
  asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}

// LDG path: warps claim U rows from a cursor (chunked like the library), U loads in flight
template <int U>
__global__ void __launch_bounds__(512) ldg_gather(const uint8_t *slab, const uint32_t *rows, uint32_t n,
                                                  uint8_t *out, uint32_t R, uint32_t *cursor, int seq_out) {
  const int lane = threadIdx.x & 31;
  const uint32_t V = R >> 4;
  uint32_t next = 0;
  if (lane == 0) next = atomicAdd(cursor, 64u);
  next = __shfl_sync(~0u, next, 0);
  while (next < n) {
    const uint32_t c0 = next, c1 = min(n, c0 + 64u);
    if (lane == 0) next = atomicAdd(cursor, 64u);
    next = __shfl_sync(~0u, next, 0);
    for (uint32_t e0 = c0; e0 < c1; e0 += U) {
      const int nv = (int)min((uint32_t)U, c1 - e0);
      const uint32_t r = lane < nv ? rows[e0 + lane] : 0;
      uint32_t ru[U];
#pragma unroll
      for (int u = 0; u < U; ++u) ru[u] = __shfl_sync(~0u, r, u);
      for (uint32_t j = lane; j < V; j += 32) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u)
          if (u < nv) v[u] = ldnc(slab + (uint64_t)ru[u] * R + j * 16);
#pragma unroll
        for (int u = 0; u < U; ++u)
          if (u < nv) {
            const uint64_t o = seq_out ? (e0 + u) : (uint64_t)((e0 + u) * 2654435761u % n);
            stcs(out + o * R + j * 16, v[u]);
          }
      }
    }
  }
}

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

// TMA bulk: each warp owns `slots` rows of smem; lane u issues loads for slot u (+U*d)
template <bool HINT>
__global__ void __launch_bounds__(512, 1) bulk_gather(const uint8_t *slab, const uint32_t *rows, uint32_t n,
                                                      uint8_t *out, uint32_t R, uint32_t *cursor, int seq_out,
                                                      int U, int depth) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) uint64_t bars[16][32];
  __shared__ uint32_t oidx[16][32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint8_t *ws = sm + (size_t)warp * U * depth * R;
  uint64_t pol = 0;
  if (HINT) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  if (lane < U)
    for (int d = 0; d < depth; ++d)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bars[warp][d * U + lane])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  uint32_t phase = 0, valid = 0, g = 0;
  auto store = [&](uint32_t h) {
    const int d = (int)(h % depth);
    if (lane < U && (valid >> d & 1u)) {
      const int s = d * U + lane;
      uint32_t done = 0;
      while (!done)
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                     : "=r"(done) : "r"(su32(&bars[warp][s])), "r"((phase >> d) & 1u) : "memory");
      phase ^= 1u << d;
      if (HINT)
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(
                         out + (uint64_t)oidx[warp][s] * R), "r"(su32(ws + s * R)), "r"(R), "l"(pol) : "memory");
      else
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(out + (uint64_t)oidx[warp][s] * R),
                     "r"(su32(ws + s * R)), "r"(R) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      valid &= ~(1u << d);
    }
  };
  uint32_t next = 0;
  if (lane == 0) next = atomicAdd(cursor, 64u);
  next = __shfl_sync(~0u, next, 0);
  while (next < n) {
    const uint32_t c0 = next, c1 = min(n, c0 + 64u);
    if (lane == 0) next = atomicAdd(cursor, 64u);
    next = __shfl_sync(~0u, next, 0);
    for (uint32_t e0 = c0; e0 < c1; e0 += U, ++g) {
      const int d = (int)(g % depth);
      if (lane < U && e0 + lane < c1) {
        const int s = d * U + lane;
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        const uint32_t i = e0 + lane;
        oidx[warp][s] = seq_out ? i : (uint32_t)(i * 2654435761u % n);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bars[warp][s])), "r"(R)
                     : "memory");
        const uint8_t *src = slab + (uint64_t)rows[i] * R;
        if (HINT)
          asm volatile(
              "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
                  su32(ws + s * R)), "l"(src), "r"(R), "r"(su32(&bars[warp][s])), "l"(pol) : "memory");
        else
          asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                           su32(ws + s * R)), "l"(src), "r"(R), "r"(su32(&bars[warp][s])) : "memory");
        valid |= 1u << d;
      }
      if (g + 1 >= (uint32_t)depth) store(g + 1 - depth);
    }
  }
  for (uint32_t h = g + 1 > (uint32_t)depth ? g + 1 - depth : 0; h < g; ++h) store(h);
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main(int argc, char **argv) {
  const size_t slab_gb = argc > 1 ? atoll(argv[1]) : 57;
  const uint32_t n = argc > 2 ? atoi(argv[2]) : 500000;
  const uint32_t R = argc > 3 ? atoi(argv[3]) : 512;
  const uint64_t N = (slab_gb << 30) / R;
  uint8_t *slab, *out, *flush;
  CK(cudaMalloc(&slab, N * R));
  CK(cudaMemset(slab, 3, N * R));
  CK(cudaMalloc(&out, (size_t)n * R));
  CK(cudaMalloc(&flush, 512u << 20));
  std::vector<uint32_t> rows(n);
  std::mt19937_64 rng(7);
  for (auto &r : rows) r = (uint32_t)(rng() % N);
  uint32_t *drows, *cur;
  CK(cudaMalloc(&drows, n * 4));
  CK(cudaMalloc(&cur, 4));
  CK(cudaMemcpy(drows, rows.data(), n * 4, cudaMemcpyHostToDevice));
  int S;
  CK(cudaDeviceGetAttribute(&S, cudaDevAttrMultiProcessorCount, 0));
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const double bytes = 2.0 * n * R;
  auto timeit = [&](auto launch) {
    float best = 1e9, tot = 0;
    for (int rep = 0; rep < 6; ++rep) {
      CK(cudaMemset(flush, rep, 512u << 20));
      CK(cudaMemset(cur, 0, 4));
      cudaEventRecord(a);
      launch();
      cudaEventRecord(b);
      CK(cudaEventSynchronize(b));
      CK(cudaGetLastError());
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (rep) tot += ms;
      best = std::min(best, ms);
    }
    return tot / 5;
  };
  printf("variant,seq_out,blocks_per_sm,threads,U,depth,ms,GBps_rw\n");
  {  // STREAM-style reference: D2D copy of n*R bytes
    float ms = timeit([&] { CK(cudaMemcpyAsync(out, slab, (size_t)n * R, cudaMemcpyDeviceToDevice)); });
    printf("memcpy_d2d,1,0,0,0,0,%.4f,%.1f\n", ms, bytes / (ms * 1e-3) / 1e9);
  }
  for (int seq = 0; seq < 2; ++seq) {
    for (int bps : {1, 2, 4}) {
      for (int thr : {256, 512}) {
        for (int U : {4, 8}) {
          if (bps * thr > 2048) continue;
          if (thr == 512 && bps > 1 && U == 8) continue;  // register file
          float ms = timeit([&] {
            if (U == 4) ldg_gather<4><<<S * bps, thr>>>(slab, drows, n, out, R, cur, seq);
            else ldg_gather<8><<<S * bps, thr>>>(slab, drows, n, out, R, cur, seq);
          });
          printf("ldg,%d,%d,%d,%d,0,%.4f,%.1f\n", seq, bps, thr, U, ms, bytes / (ms * 1e-3) / 1e9);
          fflush(stdout);
        }
      }
    }
    for (int hint = 0; hint < 2; ++hint) {
      for (int U : {4, 8}) {
        for (int depth : {2, 3, 4}) {
          const size_t smem = (size_t)16 * U * depth * R;
          if (smem > 200 * 1024 || U * depth > 32) continue;
          if (hint) CK(cudaFuncSetAttribute(bulk_gather<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
          else CK(cudaFuncSetAttribute(bulk_gather<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
          float ms = timeit([&] {
            if (hint) bulk_gather<true><<<S, 512, smem>>>(slab, drows, n, out, R, cur, seq, U, depth);
            else bulk_gather<false><<<S, 512, smem>>>(slab, drows, n, out, R, cur, seq, U, depth);
          });
          printf("bulk%s,%d,1,512,%d,%d,%.4f,%.1f\n", hint ? "_ef" : "", seq, U, depth, ms, bytes / (ms * 1e-3) / 1e9);
          fflush(stdout);
        }
      }
    }
  }
  return 0;
}
