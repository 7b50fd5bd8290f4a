// Streaming-read ceilings on B200 (builder tooling): max over a 16 GiB u64 array via
//  (1) vectorized LDG grid-stride, (2) per-warp 1-D TMA bulk ring (no processing),
//  (3) same ring + a trivial per-lane max over the staged keys.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include "../paper_conf_sc_mandulakgfhs24_b200/csrc/kernels.cuh"
using namespace lm;

__global__ void k_ldg(const ulonglong2* __restrict__ a, int64_t n2, unsigned long long* out) {
  uint64_t b = 0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + 3 * stride < n2; i += 4 * stride) {
    ulonglong2 x0 = __ldg(a + i), x1 = __ldg(a + i + stride), x2 = __ldg(a + i + 2 * stride), x3 = __ldg(a + i + 3 * stride);
    b = umax64(b, umax64(umax64(x0.x, x0.y), umax64(x1.x, x1.y)));
    b = umax64(b, umax64(umax64(x2.x, x2.y), umax64(x3.x, x3.y)));
  }
  for (; i < n2; i += stride) { ulonglong2 x = __ldg(a + i); b = umax64(b, umax64(x.x, x.y)); }
  if (b == 0x12345) atomicAdd(out, 1ull);
}

template <int TILE, int RING, int WARPS, bool WORK>
__global__ void __launch_bounds__(32 * WARPS) k_tma(const uint64_t* adj, int64_t ntiles, unsigned long long* out) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  unsigned char* my = smem + (size_t)warp * (RING * TILE * 8 + 64);
  uint64_t* bars = reinterpret_cast<uint64_t*>(my + RING * TILE * 8);
  const int64_t gw = (int64_t)blockIdx.x * WARPS + warp, nwt = (int64_t)gridDim.x * WARPS;
  if (lane == 0) { for (int s = 0; s < RING; ++s) mbar_init(&bars[s], 1); fence_mbar_init(); }
  __syncwarp();
  const uint64_t pol = policy_evict_first();
  auto issue = [&](int64_t t, int s) {
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(&bars[s], TILE * 8);
    tma_bulk_g2s(my + s * TILE * 8, adj + t * TILE, TILE * 8, &bars[s], pol);
  };
  if (lane == 0) for (int s = 0; s < RING; ++s) { int64_t t = gw + s * nwt; if (t < ntiles) issue(t, s); }
  uint64_t b = 0;
  for (int64_t k = 0;; ++k) {
    const int64_t t = gw + k * nwt;
    if (t >= ntiles) break;
    const int s = (int)(k % RING);
    while (!mbar_try_wait(&bars[s], (uint32_t)((k / RING) & 1))) {}
    if (WORK) {
      const uint64_t* K = reinterpret_cast<const uint64_t*>(my + s * TILE * 8);
      for (int j = lane; j < TILE; j += 32) b = umax64(b, K[j]);
    }
    __syncwarp();
    const int64_t tn = t + RING * nwt;
    if (lane == 0 && tn < ntiles) issue(tn, s);
  }
  if (b == 0x12345) atomicAdd(out, 1ull);
}

template <int TILE, int RING, int WARPS, bool WORK>
float run_tma(const uint64_t* d, int64_t n, unsigned long long* out) {
  const size_t sm = (size_t)WARPS * (RING * TILE * 8 + 64);
  cudaFuncSetAttribute(k_tma<TILE, RING, WARPS, WORK>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tma<TILE, RING, WARPS, WORK>, 32 * WARPS, sm);
  const int64_t ntiles = n / TILE;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float best = 1e9;
  for (int it = 0; it < 5; ++it) {
    cudaEventRecord(a);
    k_tma<TILE, RING, WARPS, WORK><<<occ * 148, 32 * WARPS, sm>>>(d, ntiles, out);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); best = std::min(best, ms);
  }
  printf("tma TILE=%d RING=%d WARPS=%d work=%d occ=%d: %.3f ms  %.0f GB/s\n", TILE, RING, WARPS, (int)WORK, occ, best, n * 8.0 / best / 1e6);
  return best;
}

int main() {
  const int64_t n = (16ll << 30) / 8;
  uint64_t* d; cudaMalloc(&d, n * 8); cudaMemset(d, 1, n * 8);
  unsigned long long* out; cudaMalloc(&out, 8);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int blocks : {148 * 4, 148 * 8, 148 * 16, 148 * 32}) {
    float best = 1e9;
    for (int it = 0; it < 5; ++it) {
      cudaEventRecord(a); k_ldg<<<blocks, 256>>>((const ulonglong2*)d, n / 2, out); cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b); best = std::min(best, ms);
    }
    printf("ldg blocks=%d: %.3f ms  %.0f GB/s\n", blocks, best, n * 8.0 / best / 1e6);
  }
  run_tma<512, 3, 4, false>(d, n, out);
  run_tma<512, 6, 4, false>(d, n, out);
  run_tma<1024, 4, 2, false>(d, n, out);
  run_tma<1024, 4, 4, false>(d, n, out);
  run_tma<2048, 4, 2, false>(d, n, out);
  run_tma<4096, 3, 1, false>(d, n, out);
  run_tma<512, 3, 4, true>(d, n, out);
  run_tma<1024, 4, 2, true>(d, n, out);
  run_tma<2048, 4, 2, true>(d, n, out);
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
