// graphgen_cuda.cu -- the same seeded generators as graphgen.cpp, on the GPU (bench/test input
// preparation only; holds none of the matching method's arithmetic).  Both sides include
// gg_common.h, so graphs are bit-identical by construction (tests/test_gpu_graphgen.py).
//
// ER / R-MAT CSR build, bucketed by source-vertex range so any scale fits in HBM:
//   1. gg_cuda_count : entries per bucket (both directions of every non-loop edge)
//   2. per bucket    : gg_cuda_emit (keys u<<32|v of entries whose u lies in the bucket)
//                      -> gg_cuda_sort_unique (CUB radix sort + unique: sorted, deduplicated rows)
//                      -> gg_cuda_scatter (col, w, first-entry index of each row)
//   3. (python)       offsets = suffix-min fill of the row starts
// Compiled with -fmad=false so the fp64 weight modes round exactly as on the host.
#include <cuda_runtime.h>

#include <cub/cub.cuh>
#include <cstdint>

#include "gg_common.h"

namespace {

struct GenSpec {
  int kind;  // 0 = ER, 1 = R-MAT
  GGEr er;
  GGRmat rm;
  __device__ __forceinline__ void edge(int64_t i, int64_t* u, int64_t* v) const {
    if (kind == 0) er.edge(i, u, v);
    else rm.edge(i, u, v);
  }
};

GenSpec make_spec(int kind, int64_t n, int scale, uint64_t seed, double a, double b, double c) {
  GenSpec s;
  s.kind = kind;
  s.er = gg_make_er(n, seed);
  s.rm = gg_make_rmat(scale > 0 ? scale : 1, seed, a, b, c);
  return s;
}

__global__ void k_count(GenSpec g, int64_t M, int shift, int nb, unsigned long long* counts) {
  extern __shared__ unsigned long long sh[];
  for (int i = threadIdx.x; i < nb; i += blockDim.x) sh[i] = 0;
  __syncthreads();
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M; i += stride) {
    int64_t u, v;
    g.edge(i, &u, &v);
    if (u == v) continue;
    atomicAdd(&sh[u >> shift], 1ull);
    atomicAdd(&sh[v >> shift], 1ull);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < nb; i += blockDim.x)
    if (sh[i]) atomicAdd(&counts[i], sh[i]);
}

__device__ __forceinline__ void append(bool p, uint64_t key, uint64_t* out,
                                       unsigned long long* cur) {
  const unsigned b = __ballot_sync(0xffffffffu, p);
  if (!b) return;
  const int lane = threadIdx.x & 31, leader = __ffs(b) - 1;
  unsigned long long base = 0;
  if (lane == leader) base = atomicAdd(cur, (unsigned long long)__popc(b));
  base = __shfl_sync(0xffffffffu, base, leader);
  unsigned lt;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
  if (p) out[base + __popc(b & lt)] = key;
}

__global__ void k_emit(GenSpec g, int64_t M, int64_t lo, int64_t hi, uint64_t* keys,
                       unsigned long long* cur) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t M32 = (M + 31) & ~31ll;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M32; i += stride) {
    int64_t u = 0, v = 0;
    if (i < M) g.edge(i, &u, &v);
    const bool ok = i < M && u != v;
    append(ok && u >= lo && u < hi, ((uint64_t)u << 32) | (uint64_t)v, keys, cur);
    append(ok && v >= lo && v < hi, ((uint64_t)v << 32) | (uint64_t)u, keys, cur);
  }
}

// col/w are written at out_base + j (out_base = base: whole-graph device arrays; 0: a per-bucket
// buffer that the caller copies out); first[] always gets the global entry index base + j
__global__ void k_scatter(const uint64_t* __restrict__ keys, int64_t cnt, int64_t base,
                          int64_t out_base, uint64_t ws, int mode, int32_t* col, float* w,
                          int64_t* first) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < cnt; j += stride) {
    const uint64_t k = keys[j];
    const int64_t u = (int64_t)(k >> 32), v = (int64_t)(uint32_t)k;
    col[out_base + j] = (int32_t)v;
    w[out_base + j] = gg_weight(ws, mode, u, v, 1);
    if (j == 0 || (keys[j - 1] >> 32) != (k >> 32)) first[u] = base + j;
  }
}

// mesh: degree, fill, and per-row weights
__device__ __forceinline__ bool mesh_keep(uint64_t s, int keep, int64_t a, int64_t b) {
  if (keep >= 1000) return true;
  const int64_t lo = a < b ? a : b, hi = a < b ? b : a;
  return (int)(gg_hash2(s, (uint64_t)lo, (uint64_t)hi) % 1000u) < keep;
}
__device__ __forceinline__ int mesh_nbrs(int64_t side, uint64_t s, int keep, int64_t id,
                                         int64_t out[4]) {
  const int64_t x = id % side, y = id / side;
  int k = 0;
  if (y > 0 && mesh_keep(s, keep, id, id - side)) out[k++] = id - side;
  if (x > 0 && mesh_keep(s, keep, id, id - 1)) out[k++] = id - 1;
  if (x + 1 < side && mesh_keep(s, keep, id, id + 1)) out[k++] = id + 1;
  if (y + 1 < side && mesh_keep(s, keep, id, id + side)) out[k++] = id + side;
  return k;
}
__global__ void k_mesh_deg(int64_t side, uint64_t s, int keep, int64_t* deg) {
  const int64_t n = side * side, stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    int64_t t[4];
    deg[i] = mesh_nbrs(side, s, keep, i, t);
  }
}
__global__ void k_mesh_fill(int64_t side, uint64_t s, int keep, const int64_t* offs, int32_t* col,
                            float* w, uint64_t ws, int mode) {
  const int64_t n = side * side, stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    int64_t t[4];
    const int k = mesh_nbrs(side, s, keep, i, t);
    for (int j = 0; j < k; ++j) {
      col[offs[i] + j] = (int32_t)t[j];
      w[offs[i] + j] = gg_weight(ws, mode, i, t[j], side);
    }
  }
}

int grid_of(int64_t work) {
  int64_t b = (work + 255) / 256;
  if (b > 148 * 64) b = 148 * 64;
  if (b < 1) b = 1;
  return (int)b;
}

}  // namespace

extern "C" {

int gg_cuda_count(int kind, int64_t n, int scale, uint64_t seed, double a, double b, double c,
                  int64_t M, int shift, int nb, unsigned long long* d_counts, void* stream) {
  GenSpec g = make_spec(kind, n, scale, seed, a, b, c);
  k_count<<<grid_of(M), 256, (size_t)nb * 8, (cudaStream_t)stream>>>(g, M, shift, nb, d_counts);
  return (int)cudaGetLastError();
}

int gg_cuda_emit(int kind, int64_t n, int scale, uint64_t seed, double a, double b, double c,
                 int64_t M, int64_t lo, int64_t hi, uint64_t* d_keys, unsigned long long* d_cur,
                 void* stream) {
  GenSpec g = make_spec(kind, n, scale, seed, a, b, c);
  k_emit<<<grid_of(M), 256, 0, (cudaStream_t)stream>>>(g, M, lo, hi, d_keys, d_cur);
  return (int)cudaGetLastError();
}

// temp bytes needed by gg_cuda_sort_unique for `cnt` keys
int64_t gg_cuda_temp_bytes(int64_t cnt) {
  size_t t1 = 0, t2 = 0;
  cub::DoubleBuffer<uint64_t> db(nullptr, nullptr);
  cub::DeviceRadixSort::SortKeys(nullptr, t1, db, cnt, 0, 64);
  cub::DeviceSelect::Unique(nullptr, t2, (uint64_t*)nullptr, (uint64_t*)nullptr,
                            (int64_t*)nullptr, cnt);
  return (int64_t)(t1 > t2 ? t1 : t2);
}

// sort keys[0:cnt) (alt = scratch of cnt keys) and deduplicate into whichever buffer does not hold
// the sorted keys; *which_out = 0 if the result is in d_keys, 1 if in d_alt; *d_nout = count.
int gg_cuda_sort_unique(uint64_t* d_keys, uint64_t* d_alt, int64_t cnt, int begin_bit, int end_bit,
                        void* d_temp, int64_t temp_bytes, int64_t* d_nout, int* which_out,
                        void* stream) {
  cudaStream_t st = (cudaStream_t)stream;
  size_t tb = (size_t)temp_bytes;
  cub::DoubleBuffer<uint64_t> db(d_keys, d_alt);
  cudaError_t e = cub::DeviceRadixSort::SortKeys(d_temp, tb, db, cnt, begin_bit, end_bit, st);
  if (e) return (int)e;
  uint64_t* out = (db.Current() == d_keys) ? d_alt : d_keys;
  *which_out = (out == d_keys) ? 0 : 1;
  tb = (size_t)temp_bytes;
  e = cub::DeviceSelect::Unique(d_temp, tb, db.Current(), out, d_nout, cnt, st);
  return (int)e;
}

int gg_cuda_scatter(const uint64_t* d_keys, int64_t cnt, int64_t base, uint64_t seed, int mode,
                    int32_t* d_col, float* d_w, int64_t* d_first, void* stream) {
  const uint64_t ws = gg_mix64(seed ^ 0x77u);
  k_scatter<<<grid_of(cnt), 256, 0, (cudaStream_t)stream>>>(d_keys, cnt, base, base, ws, mode,
                                                           d_col, d_w, d_first);
  return (int)cudaGetLastError();
}

// same, but col/w of this bucket land at d_col[0..cnt) (for host-side assembly of big graphs)
int gg_cuda_scatter_local(const uint64_t* d_keys, int64_t cnt, int64_t base, uint64_t seed, int mode,
                          int32_t* d_col, float* d_w, int64_t* d_first, void* stream) {
  const uint64_t ws = gg_mix64(seed ^ 0x77u);
  k_scatter<<<grid_of(cnt), 256, 0, (cudaStream_t)stream>>>(d_keys, cnt, base, 0, ws, mode, d_col,
                                                           d_w, d_first);
  return (int)cudaGetLastError();
}

int gg_cuda_mesh_deg(int64_t side, int keep_permille, uint64_t seed, int64_t* d_deg, void* stream) {
  const uint64_t s = gg_mix64(seed ^ 0x3E5u);
  k_mesh_deg<<<grid_of(side * side), 256, 0, (cudaStream_t)stream>>>(side, s, keep_permille, d_deg);
  return (int)cudaGetLastError();
}

int gg_cuda_mesh_fill(int64_t side, int keep_permille, uint64_t seed, const int64_t* d_offs,
                      int32_t* d_col, float* d_w, uint64_t wseed, int mode, void* stream) {
  const uint64_t s = gg_mix64(seed ^ 0x3E5u);
  const uint64_t ws = gg_mix64(wseed ^ 0x77u);
  k_mesh_fill<<<grid_of(side * side), 256, 0, (cudaStream_t)stream>>>(side, s, keep_permille,
                                                                     d_offs, d_col, d_w, ws, mode);
  return (int)cudaGetLastError();
}

}  // extern "C"
