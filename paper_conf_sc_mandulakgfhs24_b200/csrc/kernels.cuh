// kernels.cuh -- sm_100a kernels of the pointer-based locally dominant matching hot path.
//
// Paper: Mandulak et al., SC'24.  "P:N" = PAPER.md line N.  Design and rooflines: DESIGN.md.
//
// Data on the device (one graph, one GPU):
//   offs   int64[n+1]        CSR row pointers
//   adj    uint64[m (+pad)]  packed keys  key = (float_bits(w) << 32) | neighbour.  For w > 0
//                            finite, integer order of keys == the strict per-vertex order
//                            "heavier weight, then larger neighbour id" (R1), so the
//                            pointer argmax of Alg. 3 L5-8 is a plain u64 max.
//   noffs  int64[n_nz+1]     start of every NON-EMPTY row (+ m): the round-1 sweep's row index
//   nzr    int32[n_nz]       vertex id of every non-empty row
//   tile_nz int32[ntiles+1]  non-empty row containing the first entry of each sweep tile
//   best   uint64[n]         the pointer of each vertex as its full key (0 = no candidate);
//                            ptr[u] = (uint32)best[u]   (Alg. 3 "pointers")
//   bits   uint32[(n+31)/32] matched bitmap ("mate[u] != empty", Alg. 3 L5/L6 P:147-148)
//   L      int32[]           live list: unmatched vertices holding a valid pointer
//   F[b]   int32[]           frontier (vertices whose target was matched), binned by degree
#pragma once
#include <cstdint>
#include <cooperative_groups.h>
#include <cuda.h>
#include <cuda_runtime.h>

namespace lm {

namespace cg = cooperative_groups;

constexpr int kDegBins = 4;            // frontier degree bins (rows scanned by the pointer kernels)
constexpr int kDecided = 4;            // frontier list of rows whose pointer the key cache decided
constexpr int kBins = 5;               // frontier lists: the degree bins + the decided list
#ifndef LM_BIN0
#define LM_BIN0 8
#endif
#ifndef LM_BIN1
#define LM_BIN1 64
#endif
#ifndef LM_BIN2
#define LM_BIN2 2048
#endif
// frontier degree bins: <= kBinDeg0 one lane, <= kBinDeg1 a sub-warp group, <= kBinDeg2 a warp,
// else a CTA (group sizes: LM_B*_G in lmatch.cu)
constexpr int kBinDeg0 = LM_BIN0, kBinDeg1 = LM_BIN1, kBinDeg2 = LM_BIN2;

// Adjacency view: entries [0, R) in HBM, [R, m) in pinned host memory mapped into the device
// address space (out-of-core mode; R = m otherwise).  host_off is pre-offset by -R.
// Out-of-core with the host-row key cache (NEXT-1): indices >= M0 address the cache (HBM),
// cache_off pre-offset by -M0, so a frontier entry can be redirected to cached keys.
#ifndef LM_ADJ_NOALLOC
#define LM_ADJ_NOALLOC 0  // 1 = frontier row reads bypass L1 (keep L1 for the bitmap probes)
#endif
// L2 policy of the frontier rounds: the row keys a pointer kernel reads are
// used once per round, while the matched bitmap (n/8 bytes, 8 MB at 2^26) is probed for almost
// every key; LM_KEY_HINT = 1 loads the keys L1::no_allocate with an L2 evict_first policy and
// LM_BIT_HINT = 1 probes the bitmap with an L2 evict_last policy, so the key stream does not push
// the bitmap out of L2.
#ifndef LM_KEY_HINT
#define LM_KEY_HINT 0
#endif
#ifndef LM_BIT_HINT
#define LM_BIT_HINT 0
#endif
__device__ __forceinline__ uint64_t l2_policy_first() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t l2_policy_last() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t ld_stream_u64(const uint64_t* p) {
#if LM_KEY_HINT
  uint64_t v;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(l2_policy_first()));
  return v;
#elif LM_ADJ_NOALLOC
  uint64_t v;
  asm("ld.global.nc.L1::no_allocate.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
#else
  return __ldg(p);
#endif
}
// the bitmap word holding vertex v's matched bit, as probed by the pointer phase
__device__ __forceinline__ uint32_t probe_word(const uint32_t* __restrict__ bits, uint32_t v) {
#if LM_BIT_HINT
  uint32_t x;
  asm("ld.global.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(x) : "l"(bits + (v >> 5)), "l"(l2_policy_last()));
  return x;
#else
  return bits[v >> 5];
#endif
}
struct AdjView {
  const uint64_t* dev;
  const uint64_t* host_off;
  int64_t R;
  const uint64_t* cache_off = nullptr;
  int64_t M0 = INT64_MAX;
  // out of core, residual rows (NEXT-1): host rows copied into HBM when first rescanned, at
  // indices >= M2 (res_off pre-offset by -M2)
  const uint64_t* res_off = nullptr;
  int64_t M2 = INT64_MAX;
  __device__ __forceinline__ uint64_t at(int64_t j) const {
    return j < R ? ld_stream_u64(dev + j)
                 : (j < M0 ? host_off[j] : (j < M2 ? __ldg(cache_off + j) : __ldg(res_off + j)));
  }
  __device__ __forceinline__ uint64_t* ptr(int64_t j) const {
    return const_cast<uint64_t*>(j < R ? dev + j : host_off + j);
  }
};

// --------------------------------------------------------------------------- small helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ bool bit_test(const uint32_t* __restrict__ bits, uint32_t v) {
  return (bits[v >> 5] >> (v & 31)) & 1u;
}
// max over a group of lanes of a packed key: two 32-bit max reductions (weight bits, then the
// neighbour id among the lanes holding the winning weight bits) -- equal to the u64 max.
__device__ __forceinline__ uint64_t group_max_key(uint64_t key, unsigned mask) {
  const uint32_t hi = (uint32_t)(key >> 32);
  const uint32_t mhi = __reduce_max_sync(mask, hi);
  const uint32_t lo = (hi == mhi) ? (uint32_t)key : 0u;
  const uint32_t mlo = __reduce_max_sync(mask, lo);
  return ((uint64_t)mhi << 32) | mlo;
}
// insert x into a descending register list (keeps the K largest)
template <int K>
__device__ __forceinline__ void topk_insert(uint64_t (&t)[K], uint64_t x) {
#pragma unroll
  for (int i = 0; i < K; ++i) {
    const uint64_t a = t[i];
    const bool gt = x > a;
    t[i] = gt ? x : a;
    x = gt ? a : x;
  }
}

// K warp-wide pops of the per-lane descending lists: lane r < K receives the r-th largest key
// (u64 max; equal keys of a repeated edge are popped one at a time).
template <int K>
__device__ __forceinline__ uint64_t warp_topk_pop(uint64_t (&t)[K]) {
  const int lane = threadIdx.x & 31;
  uint64_t mine = 0ull;
#pragma unroll
  for (int r = 0; r < K; ++r) {
    const uint64_t mx = group_max_key(t[0], 0xffffffffu);
    if (lane == r) mine = mx;
    const unsigned own = __ballot_sync(0xffffffffu, mx != 0ull && t[0] == mx);
    if (own && lane == __ffs(own) - 1) {
#pragma unroll
      for (int i = 0; i < K - 1; ++i) t[i] = t[i + 1];
      t[K - 1] = 0ull;
    }
  }
  return mine;
}

__device__ __forceinline__ int bin_of(int64_t deg) {
  return deg <= kBinDeg0 ? 0 : deg <= kBinDeg1 ? 1 : deg <= kBinDeg2 ? 2 : 3;
}
__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned r;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
  return r;
}
// warp-aggregated append: every lane with `pred` gets a unique slot in list[]; one atomic/warp.
// Must be called by all 32 lanes.
__device__ __forceinline__ void warp_append(bool pred, int32_t val, int32_t* list,
                                            unsigned long long* counter) {
  const unsigned b = __ballot_sync(0xffffffffu, pred);
  if (!b) return;
  const int lane = threadIdx.x & 31;
  const int leader = __ffs(b) - 1;
  unsigned long long base = 0;
  if (lane == leader) base = atomicAdd(counter, (unsigned long long)__popc(b));
  base = __shfl_sync(0xffffffffu, base, leader);
  if (pred) list[base + __popc(b & lanemask_lt())] = val;
}

// ------------------------------------------------------------------ mbarrier + TMA bulk copy
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile(
      "{\n .reg .b64 st;\n mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n}\n" ::"r"(
          smem_u32(bar)),
      "r"(bytes)
      : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      " selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
// 1-D TMA bulk copy global -> shared (cp.async.bulk; SASS UBLKCP), completion on `bar`.
// dst/src 16-byte aligned, bytes a multiple of 16.  Adjacency is streamed once: evict-first.
__device__ __forceinline__ void tma_bulk_g2s(void* dst, const void* src, uint32_t bytes,
                                             uint64_t* bar, uint64_t policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1], %2, [%3], %4;" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}

// =============================================================================================
// =============================================================================================
// A1 ingest: pack + validate  (adj[j] = bits(w[j]) << 32 | col[j]; PAPER.md:96 CSR arrays)
// =============================================================================================
struct PackErr {
  unsigned long long first_bad;  // smallest bad entry index (ULLONG_MAX = none)
  unsigned long long bad_offsets;
};

__global__ void k_pack(const int32_t* __restrict__ col, const float* __restrict__ w, int64_t cnt,
                       int64_t n, uint64_t* __restrict__ adj, int64_t base, PackErr* err) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < cnt; j += stride) {
    const int32_t c = col[j];
    const uint32_t wb = __float_as_uint(w[j]);
    // finite, > 0, not -0.0: sign bit clear, exponent != 255, not +0
    const bool ok = c >= 0 && (int64_t)c < n && (wb >> 31) == 0 && ((wb >> 23) & 0xffu) != 0xffu &&
                    wb != 0u;
    if (!ok) atomicMin(&err->first_bad, (unsigned long long)(base + j));
    adj[j] = ((uint64_t)wb << 32) | (uint32_t)c;
  }
}

// Self-loops are ignored (simple graph): their keys become 0, which never wins a max, so
// no kernel on the hot path needs a per-entry self test.  8 lanes per row.
__global__ void k_zap_self_loops(const int64_t* __restrict__ offs, AdjView adj, int64_t n,
                                 int64_t vbase, unsigned long long* count) {
  const int lane8 = threadIdx.x & 7;
  const int64_t g0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 3;
  const int64_t gs = ((int64_t)gridDim.x * blockDim.x) >> 3;
  unsigned long long c = 0;
  for (int64_t u = g0; u < n; u += gs)
    for (int64_t j = offs[u] + lane8; j < offs[u + 1]; j += 8)
      if ((uint32_t)adj.at(j) == (uint32_t)(u + vbase) && adj.at(j) != 0ull) {
        *adj.ptr(j) = 0ull;
        ++c;
      }
  for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(count, c);
}

// number of vertices in each frontier degree bin (static capacity of the bin lists)
__global__ void k_bin_sizes(const int64_t* __restrict__ offs, int64_t n, unsigned long long* cnt) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  unsigned long long c[kDegBins] = {0, 0, 0, 0};
  for (int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; u < n; u += stride) {
    const int64_t d = offs[u + 1] - offs[u];
    if (d > 0) ++c[bin_of(d)];
  }
#pragma unroll
  for (int b = 0; b < kDegBins; ++b) {
    for (int o = 16; o; o >>= 1) c[b] += __shfl_xor_sync(0xffffffffu, c[b], o);
    if ((threadIdx.x & 31) == 0 && c[b]) atomicAdd(&cnt[b], c[b]);
  }
}

__global__ void k_check_offsets(const int64_t* __restrict__ offs, int64_t n, int64_t m,
                                PackErr* err) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    bool bad = offs[i + 1] < offs[i];
    if (i == 0 && offs[0] != 0) bad = true;
    if (i == n - 1 && offs[n] != m) bad = true;
    if (bad) atomicMin(&err->bad_offsets, (unsigned long long)i);
  }
}

// validate_level 2: sum over entries of H(u,v,w) - H(v,u,w) (mod 2^64) is 0 iff the multiset of
// (u,v,w) equals that of (v,u,w) (w.h.p. for a 64-bit mixing hash).  8 lanes per row.
__device__ __forceinline__ uint64_t mix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
__global__ void k_symhash(const int64_t* __restrict__ offs, AdjView adj, int64_t n,
                          unsigned long long* acc) {
  const int lane8 = threadIdx.x & 7;
  const int64_t g0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 3;
  const int64_t gs = ((int64_t)gridDim.x * blockDim.x) >> 3;
  uint64_t s = 0;
  for (int64_t u = g0; u < n; u += gs) {
    for (int64_t j = offs[u] + lane8; j < offs[u + 1]; j += 8) {
      const uint64_t k = adj.at(j);
      if (k == 0) continue;  // zeroed self-loop
      const uint64_t v = (uint32_t)k, wb = k >> 32;
      s += mix64(mix64((uint64_t)u * 0x100000001B3ull ^ v) ^ wb) -
           mix64(mix64(v * 0x100000001B3ull ^ (uint64_t)u) ^ wb);
    }
  }
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) atomicAdd(acc, (unsigned long long)s);
}

// validate_level 2, repeated edges: entries [base, base + cnt) as (neighbour << 32 | weight bits)
// keys, so a segmented ascending sort groups each row's copies of one neighbour together
__global__ void k_dup_keys(AdjView adj, int64_t base, int64_t cnt, uint64_t* __restrict__ out) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += stride) {
    const uint64_t k = adj.at(base + i);
    out[i] = (k << 32) | (k >> 32);
  }
}
// ... and neighbouring sorted keys of one row with the same neighbour must be equal; *bad = the
// smallest offending row (global id row0 + r).  8 lanes per row.
__global__ void k_dup_check(const uint64_t* __restrict__ keys, const int32_t* __restrict__ seg,
                            int64_t nrows, int64_t row0, unsigned long long* bad) {
  const int lane8 = threadIdx.x & 7;
  const int64_t g0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 3;
  const int64_t gs = ((int64_t)gridDim.x * blockDim.x) >> 3;
  for (int64_t r = g0; r < nrows; r += gs)
    for (int64_t j = (int64_t)seg[r] + 1 + lane8; j < (int64_t)seg[r + 1]; j += 8) {
      const uint64_t a = keys[j - 1], b = keys[j];
      if ((a >> 32) == (b >> 32) && a != b) atomicMin(bad, (unsigned long long)(row0 + r));
    }
}

// =============================================================================================
// A1 ingest: index of non-empty rows for the round-1 sweep (exclusive scan, 3 kernels)
// =============================================================================================
constexpr int kScanThreads = 1024;
constexpr int kScanItems = 4;
constexpr int kScanBlock = kScanThreads * kScanItems;

__device__ __forceinline__ int64_t block_excl_scan(int64_t x, int64_t* total) {
  __shared__ int64_t warp_sums[33];  // [0,32): exclusive warp prefixes, [32]: block total
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int64_t incl = x;
  for (int o = 1; o < 32; o <<= 1) {
    const int64_t y = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) warp_sums[wid] = incl;
  __syncthreads();
  if (wid == 0) {
    const int nw = blockDim.x >> 5;
    const int64_t v = lane < nw ? warp_sums[lane] : 0;
    int64_t vi = v;
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t y = __shfl_up_sync(0xffffffffu, vi, o);
      if (lane >= o) vi += y;
    }
    if (lane < nw) warp_sums[lane] = vi - v;
    if (lane == 31) warp_sums[32] = vi;
  }
  __syncthreads();
  const int64_t res = warp_sums[wid] + incl - x;
  if (total) *total = warp_sums[32];
  __syncthreads();
  return res;
}

__global__ void k_nz_count(const int64_t* __restrict__ offs, int64_t n, int64_t* blocksum) {
  const int64_t b0 = (int64_t)blockIdx.x * kScanBlock + threadIdx.x * kScanItems;
  int64_t c = 0;
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    const int64_t i = b0 + k;
    if (i < n) c += offs[i + 1] > offs[i];
  }
  int64_t tot;
  block_excl_scan(c, &tot);
  if (threadIdx.x == 0) blocksum[blockIdx.x] = tot;
}

// single-block exclusive scan of nb block sums (in place); writes grand total to *total.
__global__ void k_scan_blocksums(int64_t* bs, int64_t nb, int64_t* total) {
  __shared__ int64_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int64_t base = 0; base < nb; base += blockDim.x) {
    const int64_t i = base + threadIdx.x;
    const int64_t x = i < nb ? bs[i] : 0;
    int64_t tot;
    const int64_t ex = block_excl_scan(x, &tot);
    if (i < nb) bs[i] = carry + ex;
    __syncthreads();
    if (threadIdx.x == 0) carry += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0) *total = carry;
}

__global__ void k_nz_scatter(const int64_t* __restrict__ offs, int64_t n,
                             const int64_t* __restrict__ blockoff, int32_t* nzr, int64_t* noffs) {
  const int64_t b0 = (int64_t)blockIdx.x * kScanBlock + threadIdx.x * kScanItems;
  int64_t c = 0;
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    const int64_t i = b0 + k;
    if (i < n) c += offs[i + 1] > offs[i];
  }
  int64_t pos = blockoff[blockIdx.x] + block_excl_scan(c, nullptr);
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    const int64_t i = b0 + k;
    if (i < n && offs[i + 1] > offs[i]) {
      nzr[pos] = (int32_t)i;
      noffs[pos] = offs[i];
      ++pos;
    }
  }
}

// tile_nz[t] = last non-empty row r with noffs[r] <= t*tile (t < ntiles); tile_nz[ntiles]=n_nz-1
__global__ void k_tile_rows(const int64_t* __restrict__ noffs, int64_t n_nz, int64_t ntiles,
                            int64_t tile, int32_t* tile_nz) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t <= ntiles; t += stride) {
    if (t == ntiles) { tile_nz[t] = (int32_t)(n_nz - 1); continue; }
    const int64_t e = t * tile;
    int64_t lo = 0, hi = n_nz - 1;
    while (lo < hi) {
      const int64_t mid = (lo + hi + 1) >> 1;
      if (noffs[mid] <= e) lo = mid; else hi = mid - 1;
    }
    tile_nz[t] = (int32_t)lo;
  }
}

// =============================================================================================
// =============================================================================================
// per-run reset: matched bitmap, counters, and best[] of the rows the sweep merges with
// atomicMax (rows crossing a sweep-tile boundary; listed at create time).
// =============================================================================================
struct RoundState;
__device__ __forceinline__ uint32_t round_tag(const RoundState* st);
__global__ void k_reset(uint32_t* bits, int64_t nwords, uint64_t* best,
                        const int32_t* __restrict__ atomic_rows, int64_t n_atomic,
                        unsigned long long* counters, int ncounters, uint32_t* live,
                        int64_t n_live, const RoundState* st) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (int64_t i = tid; i < nwords; i += stride) bits[i] = 0u;
  // A7 pruning: live[u] = tag << 16 | live count is valid only under this run's tag; when the
  // 16-bit tag is about to wrap (or on the first run) old entries could alias, so clear them
  if (live) {
    const uint32_t t = round_tag(st);
    if (t == 0u || t == 0xffffu)
      for (int64_t i = tid; i < n_live; i += stride) live[i] = 0u;
  }
  for (int64_t i = tid; i < n_atomic; i += stride) best[atomic_rows[i]] = 0ull;
  if (tid < ncounters) counters[tid] = 0ull;
}

// =============================================================================================
// A2 round-1 pointer sweep (SETPOINTERS over all vertices, Alg. 3 L1-9 P:141-151).
//
// Edge-centric, warp-private tiles: the adjacency is cut into fixed tiles of TILE entries
// regardless of row boundaries, so every warp streams equal bytes (hub rows and degree-1 rows
// alike).  Each warp owns a ring of RING shared-memory stages; its lane 0 keeps RING-1 tiles in
// flight with 1-D TMA bulk copies (cp.async.bulk -> UBLKCP) completing on the stage's mbarrier:
// the tile's packed keys plus the window of its rows' start offsets (low 32 bits) and vertex ids.
// No CTA-wide barrier anywhere: warps never wait for each other.  Per tile, from shared memory:
//   * lane l takes row r0+l of the window; a row with fewer than 32 in-tile entries is scanned by
//     its lane alone; longer rows are then scanned by the whole warp, one after the other
//     (32 consecutive keys per step, conflict-free) and reduced across the warp;
//   * a row wholly inside the tile stores its max key (the pointer); a row crossing a tile
//     boundary merges its partial max with a global atomicMax on the u64 key (order independent
//     => identical to one sequential scan; such rows are zeroed by k_reset).
// Self-loop keys were zeroed at ingest (k_zap_self_loops).  No bitmap test in round 1.
// =============================================================================================
#ifndef LM_SWEEP_LONG
#define LM_SWEEP_LONG 32  // in-tile rows with at least this many entries are reduced by the warp
#endif
#ifndef LM_SWEEP_WCHAINS
#define LM_SWEEP_WCHAINS 4  // independent max chains per lane of a warp-reduced (long) row: 4 or 2
#endif
#ifndef LM_SWEEP_LCHAINS
#define LM_SWEEP_LCHAINS 2  // independent max chains of a lane-reduced (short) row: 2 (measured 2.98 vs 3.00 ms) or 4
#endif
#ifndef LM_SWEEP_MID
#define LM_SWEEP_MID 0  // 1 = rows of 8..31 in-tile entries by 8-lane groups (build knob)
#endif
__device__ __forceinline__ uint64_t umax64(uint64_t a, uint64_t b) { return a > b ? a : b; }
// The sweep's key max on the FP64 pipe (LM_SWEEP_DMAX): a packed key float_bits(w) << 32 | col
// with w > 0 finite (validated at ingest) or 0 is the bit pattern of a non-negative, finite,
// non-NaN double (exponent field <= 0x7F7), and for such doubles the IEEE order is the unsigned
// integer order of the bit patterns -- so DSETP + 2 FSEL computes exactly the u64 max, off the
// integer ALU pipe that bounds the sweep (2 ISETP + 2 SEL per key otherwise).
#ifndef LM_SWEEP_DMAX
#define LM_SWEEP_DMAX 1
#endif
__device__ __forceinline__ uint64_t kmax64(uint64_t a, uint64_t b) {
#if LM_SWEEP_DMAX
  const double x = __longlong_as_double((long long)a), y = __longlong_as_double((long long)b);
  return (uint64_t)__double_as_longlong(y > x ? y : x);
#else
  return a > b ? a : b;
#endif
}
// the same order for the frontier kernels' key compares and selects (LM_FRONT_DMAX): keys held as
// doubles compare with DSETP and select with FSEL, off the integer ALU pipe
#ifndef LM_FRONT_DMAX
#define LM_FRONT_DMAX 0  // measured neutral (the frontier kernels are latency-bound): 11.48 vs 11.48 ms
#endif
__device__ __forceinline__ double kd_of(uint64_t k) { return __longlong_as_double((long long)k); }
__device__ __forceinline__ uint64_t ku_of(double d) { return (uint64_t)__double_as_longlong(d); }
// max(b, key) unless key is the self-loop entry of vertex `self`
__device__ __forceinline__ uint64_t umax_skip(uint64_t b, uint64_t key, uint32_t self) {
  return ((uint32_t)key != self && key > b) ? key : b;
}

// Resident key cache ("key cache"): the round-1 sweep also keeps the kKC
// largest keys of every row, descending (0-padded), in kc[u][0..kKC).  From round 2 on, a vertex
// whose target was matched takes its new pointer from the cache when one of them is available:
// every key of the row above the first available cached key is cached and matched, and matched
// is permanent (R3), so that key is the row maximum over available neighbours -- exactly Alg. 1's
// pointer (L4).  Only rows whose cached keys are all matched (and that hold more than the
// cached keys) are scanned again.  A row crossing a sweep tile writes its per-tile top-kKC into
// xpart[tile][slot] (slot 0: the row began before the tile; 1: it continues after it), merged by
// k_kc_merge.
#ifndef LM_KC
#define LM_KC 4  // keys per row in the resident key cache (2 or 4; 2 = the row maximum and the next key)
#endif
constexpr int kKC = LM_KC;
static_assert(kKC == 2 || kKC == 4, "key cache width must be 2 or 4");
// top-2 update of a descending pair (t0 >= t1): branch-free, two u64 max and one u64 min
__device__ __forceinline__ void top2_insert(uint64_t& t0, uint64_t& t1, uint64_t k) {
#if LM_SWEEP_DMAX
  // the same key order on the FP64 pipe (see kmax64)
  const double d = kd_of(k), a0 = kd_of(t0), a1 = kd_of(t1);
  const double lo = d < a0 ? d : a0;
  t1 = ku_of(lo > a1 ? lo : a1);
  t0 = ku_of(d > a0 ? d : a0);
#else
  const uint64_t lo = k < t0 ? k : t0;
  t1 = lo > t1 ? lo : t1;
  t0 = k > t0 ? k : t0;
#endif
}
// merge two descending pairs into the descending top-2 of their union
__device__ __forceinline__ void top2_merge(uint64_t& t0, uint64_t& t1, uint64_t o0, uint64_t o1) {
#if LM_SWEEP_DMAX
  const double a0 = kd_of(t0), a1 = kd_of(t1), b0 = kd_of(o0), b1 = kd_of(o1);
  const double lo = b0 < a0 ? b0 : a0;
  const double hi1 = b1 > a1 ? b1 : a1;
  t1 = ku_of(lo > hi1 ? lo : hi1);
  t0 = ku_of(b0 > a0 ? b0 : a0);
#else
  const uint64_t lo = o0 < t0 ? o0 : t0;
  const uint64_t hi1 = o1 > t1 ? o1 : t1;
  t1 = lo > hi1 ? lo : hi1;
  t0 = o0 > t0 ? o0 : t0;
#endif
}
// insert key k into the descending list t0 >= t1 >= t2 >= t3 (keeps the kKC largest)
__device__ __forceinline__ void top4_insert(uint64_t& t0, uint64_t& t1, uint64_t& t2, uint64_t& t3,
                                            uint64_t k) {
  if (k > t3) {
    t3 = k;
    if (t3 > t2) { const uint64_t x = t2; t2 = t3; t3 = x; }
    if (t2 > t1) { const uint64_t x = t1; t1 = t2; t2 = x; }
    if (t1 > t0) { const uint64_t x = t0; t0 = t1; t1 = x; }
  }
}

struct SweepArgs {
  const uint64_t* adj;       // keys of entry tile_begin*TILE onward (HBM or a streamed chunk)
  uint64_t* zap;             // ZAP variant only: writable adjacency (self-loop keys -> 0)
  unsigned long long* zapped;
  uint32_t vbase;            // ZAP only: global id of local row 0 (partitioned handles)
  const uint32_t* noffs_lo;  // low 32 bits of each non-empty row's start (+ m)
  const int32_t* nzr;
  const int32_t* tile_nz;
  uint64_t* best;
  int64_t m;
  int64_t tile_begin;        // tiles [tile_begin, ntiles) of this launch
  int64_t ntiles;
  uint64_t* kc = nullptr;    // KC variant: key cache [n][kKC]
  uint64_t* xpart = nullptr; // KC variant: per-tile partial lists of crossing rows [ntiles][2][kKC]
};

template <int TILE, int RING, int WARPS, int WCAP>
struct SweepCfg {
  static constexpr int kTile = TILE;
  static constexpr int kRing = RING;
  static constexpr int kWarps = WARPS;
  static constexpr int kThreads = 32 * WARPS;
  static constexpr int kKeys = TILE + 2;   // u64 slots per stage
  static constexpr int kWin = WCAP;        // u32 row starts / ids staged per stage (rows beyond
                                           // the cap are read from global memory)
  static constexpr size_t kStageBytes = (size_t)kKeys * 8 + 2 * (size_t)kWin * 4;
  static constexpr size_t kWarpBytes = RING * kStageBytes + ((RING * 8 + 8 + 15) / 16) * 16;
  static constexpr size_t kSmem = WARPS * kWarpBytes;
  static_assert(WCAP % 4 == 0, "window cap must be a multiple of 4 entries");
  static_assert(kStageBytes % 16 == 0 && kWarpBytes % 16 == 0, "TMA needs 16-byte alignment");
};

template <int TILE, int RING, int WARPS, int WCAP, bool ZAP = false, bool KC = false>
__global__ void __launch_bounds__(32 * WARPS) k_sweep(SweepArgs A) {
  // ZAP: the one-time ingest pass -- same tiles and rows, but instead of the max it zeroes the
  // keys of self-loops (col == row; simple graph) in place.
  using C = SweepCfg<TILE, RING, WARPS, WCAP>;
  extern __shared__ __align__(128) unsigned char smem[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  unsigned char* my = smem + (size_t)warp * C::kWarpBytes;
  uint64_t* bars = reinterpret_cast<uint64_t*>(my + RING * C::kStageBytes);
  auto keys_of = [&](int s) { return reinterpret_cast<uint64_t*>(my + s * C::kStageBytes); };
  auto win_of = [&](int s) {
    return reinterpret_cast<uint32_t*>(my + s * C::kStageBytes + (size_t)C::kKeys * 8);
  };
  auto ids_of = [&](int s) {
    return reinterpret_cast<int32_t*>(my + s * C::kStageBytes + (size_t)C::kKeys * 8 +
                                      (size_t)C::kWin * 4);
  };
  (void)ids_of;

  const int64_t gw = A.tile_begin + (int64_t)blockIdx.x * WARPS + warp;
  const int64_t nwt = (int64_t)gridDim.x * WARPS;
  if (lane == 0) {
    for (int s = 0; s < RING; ++s) mbar_init(&bars[s], 1);
    fence_mbar_init();
  }
  __syncwarp();

  const uint64_t pol = policy_evict_first();
  // lane 0 only: TMA-load tile t (row window [a, bp]) into stage s
  auto issue = [&](int64_t t, int s, int32_t a, int32_t bp) {
    const int64_t e0 = t * TILE;
    const int64_t len = min((int64_t)TILE, A.m - e0);
    const uint32_t kbytes = (uint32_t)(((len + 1) & ~1ll) * 8);
    const int64_t a4 = a & ~3ll;
    const int64_t wcnt = min((int64_t)bp + 2 - a4, (int64_t)WCAP);
    const uint32_t wbytes = (uint32_t)(((wcnt + 3) & ~3ll) * 4);
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(&bars[s], kbytes + 2 * wbytes);
    tma_bulk_g2s(keys_of(s), A.adj + (t - A.tile_begin) * TILE, kbytes, &bars[s], pol);
    tma_bulk_g2s(win_of(s), A.noffs_lo + a4, wbytes, &bars[s], pol);
    tma_bulk_g2s(ids_of(s), A.nzr + a4, wbytes, &bars[s], pol);
  };
  // lane s holds the row window of the tile now in stage s; lane 0 prefetches the next one
  int32_t my_a = 0, my_bp = 0, nx_a = 0, nx_bp = 0;
  if (lane < RING) {
    const int64_t t = gw + (int64_t)lane * nwt;
    if (t < A.ntiles) { my_a = A.tile_nz[t]; my_bp = A.tile_nz[t + 1]; }
  }
  __syncwarp();
  for (int s = 0; s < RING; ++s) {
    const int64_t t = gw + (int64_t)s * nwt;
    const int32_t a = __shfl_sync(0xffffffffu, my_a, s), bp = __shfl_sync(0xffffffffu, my_bp, s);
    if (lane == 0 && t < A.ntiles) issue(t, s, a, bp);
  }
  if (lane == 0) {
    const int64_t t = gw + (int64_t)RING * nwt;
    if (t < A.ntiles) { nx_a = A.tile_nz[t]; nx_bp = A.tile_nz[t + 1]; }
  }

  for (int64_t k = 0;; ++k) {
    const int64_t t = gw + k * nwt;
    if (t >= A.ntiles) break;
    const int s = (int)(k % RING);
    const int32_t a = __shfl_sync(0xffffffffu, my_a, s), bp = __shfl_sync(0xffffffffu, my_bp, s);
    while (!mbar_try_wait(&bars[s], (uint32_t)((k / RING) & 1))) {
    }
    const uint64_t* K = keys_of(s);
    const uint32_t* Ws = win_of(s);
    const int32_t* Is = ids_of(s);
    const int lo = a & 3, hi = bp - (a & ~3);
    const int64_t a4 = a & ~3ll;
    const int64_t ts = t * TILE;
    const int len = (int)min((int64_t)TILE, A.m - ts);
    const uint32_t ts32 = (uint32_t)ts;
    // window accessors: staged entries from shared memory, the (rare) overflow from global
    auto Wr = [&](int r) -> uint32_t { return r < WCAP ? Ws[r] : __ldg(A.noffs_lo + a4 + r); };
    auto Ir = [&](int r) -> int32_t { return r < WCAP ? Is[r] : __ldg(A.nzr + a4 + r); };

    for (int r0 = lo; r0 <= hi; r0 += 32) {
      const int r = r0 + lane;
      int32_t rs = 0, re = 0;
      int L = 0;
      uint32_t vid = 0;
      if (r <= hi) {
        rs = (int32_t)(Wr(r) - ts32);
        re = (int32_t)(Wr(r + 1) - ts32);
        L = min(re, len) - max(rs, 0);
        vid = (uint32_t)Ir(r);
      }
      const bool inside = rs >= 0 && re <= len;
      // short rows: a lane each
      if (ZAP) {
        // every entry of the window's rows inside this tile, lane-per-row then warp-per-row
        if (L > 0 && L < 32) {
          for (int j = max(rs, 0), je = min(re, len); j < je; ++j)
            if ((uint32_t)K[j] == vid + A.vbase && K[j] != 0ull) {
              A.zap[ts + j] = 0ull;
              atomicAdd(A.zapped, 1ull);
            }
        }
        unsigned zm = __ballot_sync(0xffffffffu, L >= 32);
        while (zm) {
          const int l = __ffs(zm) - 1;
          zm &= zm - 1;
          const int32_t ja = __shfl_sync(0xffffffffu, max(rs, 0), l);
          const int32_t jb = __shfl_sync(0xffffffffu, min(re, len), l);
          const uint32_t v = __shfl_sync(0xffffffffu, vid, l);
          for (int j = ja + lane; j < jb; j += 32)
            if ((uint32_t)K[j] == v + A.vbase && K[j] != 0ull) {
              A.zap[ts + j] = 0ull;
              atomicAdd(A.zapped, 1ull);
            }
        }
        continue;
      }
#if LM_SWEEP_MID
      // medium rows (8 <= L < 32): 8-lane groups, four rows per step, so the lane-per-row loop
      // below only runs as long as the longest row under 8 entries (no long divergent tail)
      unsigned mm = __ballot_sync(0xffffffffu, L >= 8 && L < 32);
      while (mm) {
        const int q = lane >> 3, gl = lane & 7;
        unsigned m2 = mm;
        for (int i = 0; i < q && m2; ++i) m2 &= m2 - 1;
        const int l = m2 ? __ffs(m2) - 1 : 0;
        const bool has = m2 != 0u;
        for (int i = 0; i < 4 && mm; ++i) mm &= mm - 1;
        const int32_t ja = __shfl_sync(0xffffffffu, max(rs, 0), l);
        const int32_t jl = __shfl_sync(0xffffffffu, min(re, len), l);
        const int32_t jb = has ? jl : ja;
        const uint32_t v = __shfl_sync(0xffffffffu, vid, l);
        const bool ins = __shfl_sync(0xffffffffu, (int)inside, l) != 0;
        uint64_t b0 = 0, b1 = 0;
        int j = ja + gl;
        for (; j + 8 < jb; j += 16) {
          b0 = kmax64(b0, K[j]);
          b1 = kmax64(b1, K[j + 8]);
        }
        if (j < jb) b0 = kmax64(b0, K[j]);
        const unsigned gmask = 0xffu << (q * 8);
        const uint64_t b = group_max_key(kmax64(b0, b1), gmask);
        if (has && gl == 0) {
          if (ins) A.best[v] = b;
          else if (b) atomicMax(reinterpret_cast<unsigned long long*>(&A.best[v]), (unsigned long long)b);
        }
      }
      if (L > 0 && L < 8) {
#else
      if (KC && L > 0 && L < LM_SWEEP_LONG) {
        // the row's 4 largest keys (descending); rows wholly in the tile store them in the cache
        uint64_t t0 = 0, t1 = 0, t2 = 0, t3 = 0;
        if constexpr (kKC == 2) {
          // two independent top-2 chains, merged
          uint64_t u0 = 0, u1 = 0;
          int j = max(rs, 0);
          const int je = min(re, len);
          for (; j + 1 < je; j += 2) {
            top2_insert(t0, t1, K[j]);
            top2_insert(u0, u1, K[j + 1]);
          }
          if (j < je) top2_insert(t0, t1, K[j]);
          top2_merge(t0, t1, u0, u1);
        } else {
          for (int j = max(rs, 0), je = min(re, len); j < je; ++j) top4_insert(t0, t1, t2, t3, K[j]);
        }
        ulonglong2* c = inside ? reinterpret_cast<ulonglong2*>(A.kc + (size_t)vid * kKC)
                               : reinterpret_cast<ulonglong2*>(A.xpart + ((size_t)t * 2 + (rs < 0 ? 0 : 1)) * kKC);
        if (inside) A.best[vid] = t0;
        c[0] = make_ulonglong2(t0, t1);
        if constexpr (kKC == 4) c[1] = make_ulonglong2(t2, t3);
      }
      if (!KC && L > 0 && L < LM_SWEEP_LONG) {
#endif
#if LM_SWEEP_LCHAINS == 2
        uint64_t b0 = 0, b1 = 0;  // 2 independent max chains (short rows: less tail and combine)
        int j = max(rs, 0);
        const int je = min(re, len);
        for (; j + 1 < je; j += 2) {
          b0 = kmax64(b0, K[j]);
          b1 = kmax64(b1, K[j + 1]);
        }
        if (j < je) b0 = kmax64(b0, K[j]);
        const uint64_t b = kmax64(b0, b1);
#else
        uint64_t b0 = 0, b1 = 0, b2 = 0, b3 = 0;  // 4 independent max chains
        int j = max(rs, 0);
        const int je = min(re, len);
        for (; j + 3 < je; j += 4) {
          b0 = kmax64(b0, K[j]);
          b1 = kmax64(b1, K[j + 1]);
          b2 = kmax64(b2, K[j + 2]);
          b3 = kmax64(b3, K[j + 3]);
        }
        if (j < je) b0 = kmax64(b0, K[j]);  // <= 3 left: independent, predicated
        if (j + 1 < je) b1 = kmax64(b1, K[j + 1]);
        if (j + 2 < je) b2 = kmax64(b2, K[j + 2]);
        const uint64_t b = kmax64(kmax64(b0, b1), kmax64(b2, b3));
#endif
        if (inside) A.best[vid] = b;
        else if (b) atomicMax(reinterpret_cast<unsigned long long*>(&A.best[vid]), (unsigned long long)b);
      }
      // long rows: the whole warp, one row at a time
      unsigned lm = __ballot_sync(0xffffffffu, L >= LM_SWEEP_LONG);
      while (lm) {
        const int l = __ffs(lm) - 1;
        lm &= lm - 1;
        const int32_t ja = __shfl_sync(0xffffffffu, max(rs, 0), l);
        const int32_t jb = __shfl_sync(0xffffffffu, min(re, len), l);
        const uint32_t v = __shfl_sync(0xffffffffu, vid, l);
        const bool ins = __shfl_sync(0xffffffffu, (int)inside, l) != 0;
        if (KC) {
          // per-lane top 4 over the lane's keys, then 4 warp-wide pops: lane q < 4 holds the
          // row segment's q-th largest key
          uint64_t tt[kKC] = {};
          uint64_t mine;
          if constexpr (kKC == 2) {
            // per-lane top-2 over two chains, then a butterfly top-2 merge; lane q < 2 takes key q
            uint64_t u0 = 0, u1 = 0;
            int j = ja + lane;
            for (; j + 32 < jb; j += 64) {
              top2_insert(tt[0], tt[1], K[j]);
              top2_insert(u0, u1, K[j + 32]);
            }
            if (j < jb) top2_insert(tt[0], tt[1], K[j]);
            top2_merge(tt[0], tt[1], u0, u1);
#pragma unroll
            for (int o = 16; o; o >>= 1) {
              const uint64_t o0 = __shfl_xor_sync(0xffffffffu, tt[0], o);
              const uint64_t o1 = __shfl_xor_sync(0xffffffffu, tt[1], o);
              top2_merge(tt[0], tt[1], o0, o1);
            }
            mine = lane == 0 ? tt[0] : tt[1];
          } else {
            for (int j = ja + lane; j < jb; j += 32) top4_insert(tt[0], tt[1], tt[2], tt[3], K[j]);
            mine = warp_topk_pop<kKC>(tt);
          }
          const bool rs_neg = __shfl_sync(0xffffffffu, (int)(rs < 0), l) != 0;
          uint64_t* dst = ins ? A.kc + (size_t)v * kKC : A.xpart + ((size_t)t * 2 + (rs_neg ? 0 : 1)) * kKC;
          if (lane < kKC) dst[lane] = mine;
          if (ins && lane == 0) A.best[v] = mine;
          continue;
        }
#if LM_SWEEP_WCHAINS == 2
        uint64_t b0 = 0, b1 = 0;  // 2 independent max chains per lane
        int j = ja + lane;
        for (; j + 32 < jb; j += 64) {
          b0 = kmax64(b0, K[j]);
          b1 = kmax64(b1, K[j + 32]);
        }
        if (j < jb) b0 = kmax64(b0, K[j]);
        const uint64_t b = group_max_key(kmax64(b0, b1), 0xffffffffu);
#else
        uint64_t b0 = 0, b1 = 0, b2 = 0, b3 = 0;  // 4 independent max chains
        int j = ja + lane;
        for (; j + 96 < jb; j += 128) {
          b0 = kmax64(b0, K[j]);
          b1 = kmax64(b1, K[j + 32]);
          b2 = kmax64(b2, K[j + 64]);
          b3 = kmax64(b3, K[j + 96]);
        }
        if (j < jb) b0 = kmax64(b0, K[j]);  // <= 3 steps left: independent, predicated
        if (j + 32 < jb) b1 = kmax64(b1, K[j + 32]);
        if (j + 64 < jb) b2 = kmax64(b2, K[j + 64]);
        const uint64_t b = group_max_key(kmax64(kmax64(b0, b1), kmax64(b2, b3)), 0xffffffffu);
#endif
        if (lane == 0) {
          if (ins) A.best[v] = b;
          else if (b) atomicMax(reinterpret_cast<unsigned long long*>(&A.best[v]), (unsigned long long)b);
        }
      }
    }
    __syncwarp();
    // refill stage s with tile k + RING; prefetch the window of tile k + RING + 1
    const int64_t tn = t + (int64_t)RING * nwt;
    if (lane == 0 && tn < A.ntiles) issue(tn, s, nx_a, nx_bp);
    {
      const int32_t na = __shfl_sync(0xffffffffu, nx_a, 0), nbp = __shfl_sync(0xffffffffu, nx_bp, 0);
      if (lane == s) { my_a = na; my_bp = nbp; }
    }
    if (lane == 0) {
      const int64_t t2 = tn + nwt;
      if (t2 < A.ntiles) { nx_a = A.tile_nz[t2]; nx_bp = A.tile_nz[t2 + 1]; }
    }
  }
}

// =============================================================================================
// A2 round-1 pointer sweep, v2: swizzled 2-D TMA tiles + merge-path style segmented reduction.
//
// The adjacency is viewed as a 2-D tensor [ceil(m/16)][16] of u64 keys (128-byte rows) and each
// warp-private tile of TILE entries is fetched with ONE cp.async.bulk.tensor.2d (SASS UTMALDG)
// using the 128-byte swizzle, so lane l can read its 16 CONTIGUOUS keys (one 128-B row) with
// 8 conflict-free 16-byte shared loads (the swizzle spreads the lanes' chunks over all banks).
// The tile's row window (row starts, vertex ids) comes with two 1-D bulk copies.
// Each 512-entry pass: lane l walks entries [16l, 16l+16) of the pass in order, keeps the max key
// of the current row segment, and stores every row that begins and ends inside its 16 entries;
// rows spanning lanes are combined by ONE 5-step segmented max-scan over the lanes' open tail
// segments; a row still open at the end of a pass is carried to the next pass in registers; a
// row crossing the tile boundary is merged with a global atomicMax on its u64 key (zeroed by
// k_reset).  u64 max is order independent => identical to one sequential scan of each row.
// =============================================================================================
struct Sweep2DArgs {
  const uint32_t* noffs_lo;  // low 32 bits of each non-empty row's start (+ m)
  const int32_t* nzr;
  const int32_t* tile_nz;
  uint64_t* best;
  int64_t m;
  int64_t ntiles;
};

template <int TILE, int RING, int WARPS, int WCAP>
struct Sweep2DCfg {
  static constexpr int kTile = TILE;
  static constexpr int kThreads = 32 * WARPS;
  static constexpr int kPasses = TILE / 512;
  static constexpr size_t kKeyBytes = (size_t)TILE * 8;  // multiple of 1024 (swizzle atom)
  static constexpr size_t kWinBytes = 2 * (size_t)WCAP * 4;
  static constexpr size_t kWarpBytes =
      ((RING * kKeyBytes + RING * kWinBytes + RING * 8 + 8 + 1023) / 1024) * 1024;
  static constexpr size_t kSmem = WARPS * kWarpBytes + 1024;  // + runtime 1024-B alignment slack
  static_assert(TILE % 512 == 0 && TILE / 16 <= 256, "tile = k*512 entries, box <= 256 rows");
  static_assert(WCAP % 4 == 0, "window cap must be a multiple of 4 entries");
};

__device__ __forceinline__ void tma_tensor2d_g2s(void* dst, const void* tmap, int c0, int c1,
                                                 uint64_t* bar, uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%2, %3}], [%4], %5;" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(tmap)), "r"(c0), "r"(c1), "r"(smem_u32(bar)), "l"(policy)
      : "memory");
}

template <int TILE, int RING, int WARPS, int WCAP>
__global__ void __launch_bounds__(32 * WARPS)
    k_sweep2d(const __grid_constant__ CUtensorMap tmap, Sweep2DArgs A) {
  using C = Sweep2DCfg<TILE, RING, WARPS, WCAP>;
  extern __shared__ unsigned char smem_raw[];
  unsigned char* smem = reinterpret_cast<unsigned char*>(
      (reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  unsigned char* my = smem + (size_t)warp * C::kWarpBytes;
  unsigned char* keys0 = my;                                    // RING x kKeyBytes (1024-aligned)
  unsigned char* wins0 = my + RING * C::kKeyBytes;              // RING x (starts[WCAP], ids[WCAP])
  uint64_t* bars = reinterpret_cast<uint64_t*>(wins0 + RING * C::kWinBytes);

  const int64_t gw = (int64_t)blockIdx.x * WARPS + warp;
  const int64_t nwt = (int64_t)gridDim.x * WARPS;
  if (lane == 0) {
    for (int s = 0; s < RING; ++s) mbar_init(&bars[s], 1);
    fence_mbar_init();
  }
  __syncwarp();

  const uint64_t pol = policy_evict_first();
  auto issue = [&](int64_t t, int s, int32_t a, int32_t bp) {  // lane 0 only
    const int64_t a4 = a & ~3ll;
    const int64_t wcnt = min((int64_t)bp + 2 - a4, (int64_t)WCAP);
    const uint32_t wbytes = (uint32_t)(((wcnt + 3) & ~3ll) * 4);
    unsigned char* w = wins0 + s * C::kWinBytes;
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(&bars[s], (uint32_t)C::kKeyBytes + 2 * wbytes);
    tma_tensor2d_g2s(keys0 + s * C::kKeyBytes, &tmap, 0, (int)(t * (TILE / 16)), &bars[s], pol);
    tma_bulk_g2s(w, A.noffs_lo + a4, wbytes, &bars[s], pol);
    tma_bulk_g2s(w + WCAP * 4, A.nzr + a4, wbytes, &bars[s], pol);
  };
  int32_t my_a = 0, my_bp = 0, nx_a = 0, nx_bp = 0;
  if (lane < RING) {
    const int64_t t = gw + (int64_t)lane * nwt;
    if (t < A.ntiles) { my_a = A.tile_nz[t]; my_bp = A.tile_nz[t + 1]; }
  }
  __syncwarp();
  for (int s = 0; s < RING; ++s) {
    const int64_t t = gw + (int64_t)s * nwt;
    const int32_t a = __shfl_sync(0xffffffffu, my_a, s), bp = __shfl_sync(0xffffffffu, my_bp, s);
    if (lane == 0 && t < A.ntiles) issue(t, s, a, bp);
  }
  if (lane == 0) {
    const int64_t t = gw + (int64_t)RING * nwt;
    if (t < A.ntiles) { nx_a = A.tile_nz[t]; nx_bp = A.tile_nz[t + 1]; }
  }

  for (int64_t k = 0;; ++k) {
    const int64_t t = gw + k * nwt;
    if (t >= A.ntiles) break;
    const int s = (int)(k % RING);
    const int32_t a = __shfl_sync(0xffffffffu, my_a, s), bp = __shfl_sync(0xffffffffu, my_bp, s);
    while (!mbar_try_wait(&bars[s], (uint32_t)((k / RING) & 1))) {
    }
    const unsigned char* K = keys0 + s * C::kKeyBytes;
    const uint32_t* Ws = reinterpret_cast<const uint32_t*>(wins0 + s * C::kWinBytes);
    const int32_t* Is = reinterpret_cast<const int32_t*>(wins0 + s * C::kWinBytes + WCAP * 4);
    const int lo = a & 3, hi = bp - (a & ~3);
    const int64_t a4 = a & ~3ll;
    const int64_t ts = t * TILE;
    const int len = (int)min((int64_t)TILE, A.m - ts);
    const uint32_t ts32 = (uint32_t)ts;
    auto rel = [&](int r) -> int32_t {
      return (int32_t)((r < WCAP ? Ws[r] : __ldg(A.noffs_lo + a4 + r)) - ts32);
    };
    auto idr = [&](int r) -> uint32_t {
      return (uint32_t)(r < WCAP ? Is[r] : __ldg(A.nzr + a4 + r));
    };

    int carryR = -1;        // row left open by the previous pass (window index), or -1
    uint64_t carryV = 0;
    int rlo = lo;           // search lower bound (rows before it ended in earlier passes)
#pragma unroll 1
    for (int p = 0; p < C::kPasses; ++p) {
      const int pbase = p * 512;
      if (pbase >= len) break;
      const int e0 = pbase + lane * 16;
      const int e1 = min(e0 + 16, len);
      const bool has = e0 < len;
      // row containing e0: last r in [rlo, hi] with rel(r) <= e0
      int r = rlo;
      if (has) {
        int h = hi;
        while (r < h) {
          const int mid = (r + h + 1) >> 1;
          if (rel(mid) <= e0) r = mid; else h = mid - 1;
        }
      }
      int32_t rs = has ? rel(r) : 0, re = has ? rel(r + 1) : 0;
      uint32_t vid = has ? idr(r) : 0;
      // my 16 keys: one swizzled 128-byte row of the tile
      ulonglong2 kv[8];
      if (has) {
        const int R = e0 >> 4;
        const unsigned char* rowp = K + R * 128;
#pragma unroll
        for (int c = 0; c < 8; ++c)
          kv[c] = *reinterpret_cast<const ulonglong2*>(rowp + ((c ^ (R & 7)) << 4));
      }
      const bool firstOpen = has && rs < e0;
      const int firstR = r;
      const int32_t f_rs = rs, f_re = re;
      const uint32_t f_vid = vid;
      bool firstClosed = false;
      uint64_t firstVal = 0, b = 0;
#pragma unroll
      for (int q = 0; q < 16; ++q) {
        const int e = e0 + q;
        if (e < e1) {
          if (e >= re) {  // the current row segment ends before e
            if (r == firstR && firstOpen) { firstClosed = true; firstVal = b; }
            else A.best[vid] = b;  // began and ended inside my 16 entries
            ++r;
            rs = re;
            re = rel(r + 1);
            vid = idr(r);
            b = 0;
          }
          const uint64_t key = (q & 1) ? kv[q >> 1].y : kv[q >> 1].x;
          b = umax64(b, key);
        }
      }
      const bool lastOpen = has && re > e1;
      if (has && !lastOpen) {  // the last segment ends exactly at e1
        if (r == firstR && firstOpen) { firstClosed = true; firstVal = b; }
        else A.best[vid] = b;
      }
      // segmented max-scan over the lanes' open tail segments
      uint64_t T = lastOpen ? b : 0ull;
      bool H = !(lastOpen && r == firstR && firstOpen);
      if (lane == 0 && !H && carryR == r) T = umax64(T, carryV);
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint64_t tu = __shfl_up_sync(0xffffffffu, T, d);
        const bool hu = __shfl_up_sync(0xffffffffu, (int)H, d) != 0;
        if (lane >= d && !H) { T = umax64(T, tu); H = hu; }
      }
      const uint64_t Tprev = __shfl_up_sync(0xffffffffu, T, 1);
      if (firstClosed) {
        uint64_t tot = firstVal;
        if (lane > 0) tot = umax64(tot, Tprev);
        else if (carryR == firstR) tot = umax64(tot, carryV);
        if (f_rs >= 0 && f_re <= len) A.best[f_vid] = tot;
        else if (tot) atomicMax(reinterpret_cast<unsigned long long*>(&A.best[f_vid]),
                                (unsigned long long)tot);
      }
      if (lastOpen && e1 == len && T)  // crosses the tile end
        atomicMax(reinterpret_cast<unsigned long long*>(&A.best[vid]), (unsigned long long)T);
      // carry the row left open at the end of this pass
      const bool open31 = __shfl_sync(0xffffffffu, (int)(lastOpen && e1 < len), 31) != 0;
      carryR = open31 ? __shfl_sync(0xffffffffu, r, 31) : -1;
      carryV = __shfl_sync(0xffffffffu, T, 31);
      rlo = __shfl_sync(0xffffffffu, r, 31);
    }
    __syncwarp();
    const int64_t tn = t + (int64_t)RING * nwt;
    if (lane == 0 && tn < A.ntiles) issue(tn, s, nx_a, nx_bp);
    {
      const int32_t na = __shfl_sync(0xffffffffu, nx_a, 0), nbp = __shfl_sync(0xffffffffu, nx_bp, 0);
      if (lane == s) { my_a = na; my_bp = nbp; }
    }
    if (lane == 0) {
      const int64_t t2 = tn + nwt;
      if (t2 < A.ntiles) { nx_a = A.tile_nz[t2]; nx_bp = A.tile_nz[t2 + 1]; }
    }
  }
}

// rows the sweep merges with atomicMax: those crossing a tile boundary (one entry per boundary;
// a row crossing several boundaries appears several times, which is harmless for zeroing)
__global__ void k_atomic_rows(const int64_t* __restrict__ noffs, const int32_t* __restrict__ nzr,
                              const int32_t* __restrict__ tile_nz, int64_t ntiles, int64_t tile,
                              int32_t* out, unsigned long long* count) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t lim = (ntiles + 31) & ~31ll;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < lim; i += stride) {
    bool cross = false;
    int32_t v = 0;
    if (i >= 1 && i < ntiles) {
      const int32_t r = tile_nz[i];
      cross = noffs[r] < i * tile;
      v = nzr[r];
    }
    warp_append(cross, v, out, count);
  }
}

// key cache: the non-empty rows (nz index) that cross a sweep-tile boundary, each listed once
__global__ void k_kc_xrows(const int64_t* __restrict__ noffs, int64_t n_nz, int64_t tile,
                           int32_t* out, unsigned long long* count) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t lim = (n_nz + 31) & ~31ll;
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < lim; r += stride) {
    const bool cross = r < n_nz && noffs[r] / tile != (noffs[r + 1] - 1) / tile;
    warp_append(cross, (int32_t)r, out, count);
  }
}
// key cache: merge the per-tile partial top-kKC lists of every crossing row (tiles tf..tl; the
// row continues after tile tf -> slot 1 there, began before every later tile -> slot 0) into its
// cache line and its pointer best[u] (the row maximum).  One warp per row.
__global__ void k_kc_merge(const int32_t* __restrict__ xrows, const unsigned long long* __restrict__ nx,
                           const int64_t* __restrict__ noffs, const int32_t* __restrict__ nzr,
                           const uint64_t* __restrict__ xpart, int64_t tile, uint64_t* __restrict__ kc,
                           uint64_t* __restrict__ best) {
  const int lane = threadIdx.x & 31;
  const int64_t cnt = (int64_t)*nx;
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t ws = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = w0; i < cnt; i += ws) {
    const int64_t r = xrows[i];
    const int64_t tf = noffs[r] / tile, tl = (noffs[r + 1] - 1) / tile;
    uint64_t t[kKC] = {};
    for (int64_t tt = tf + lane; tt <= tl; tt += 32) {
      const ulonglong2* p = reinterpret_cast<const ulonglong2*>(xpart + ((size_t)tt * 2 + (tt == tf ? 1 : 0)) * kKC);
#pragma unroll
      for (int h = 0; h < kKC / 2; ++h) {
        const ulonglong2 a = p[h];
        topk_insert<kKC>(t, a.x);
        topk_insert<kKC>(t, a.y);
      }
    }
    const uint64_t mine = warp_topk_pop<kKC>(t);
    const uint32_t u = (uint32_t)nzr[r];
    if (lane < kKC) kc[(size_t)u * kKC + lane] = mine;
    if (lane == 0) best[u] = mine;
  }
}

__global__ void k_low32(const int64_t* __restrict__ noffs, int64_t cnt, uint32_t* lo) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += stride)
    lo[i] = (uint32_t)noffs[i];
}

// =============================================================================================
// Rounds >= 2.  Device counters (unsigned long long, kNumCounters):
//   [8 * set]               |S| of pair set `set` (stable live pairs)
//   [8 * set + 1 + b]       |F_b| of frontier set `set`, degree bin b
//   [16]                    adjacency entries of all frontiers produced so far (stats)
// Lists: S = uint64 pairs (u | ptr u << 32).  Frontier bins = 16-byte entries
//   .x = u | ptr << 32 (the pointer kernel overwrites ptr with the new pointer)
//   .y = row start | degree << 40 (degree >= 2^24 stored as kBigDeg: read offs instead)
// so the pointer kernel streams its row without a dependent offs[] lookup.
// =============================================================================================
constexpr int kNumCounters = 24;
constexpr int kCntSwept = 16;
constexpr int kCntCache = 17;  // [17] rows served by the out-of-core cache, [18] host entries read
constexpr int kCntN = 20;      // A6 push frontier: |N_r|, the vertices newly matched this round
constexpr int kCntPushRounds = 21;  // rounds whose next frontier the push step built
__host__ __device__ constexpr int cnt_S(int set) { return 8 * set; }
__host__ __device__ constexpr int cnt_F(int set, int b) { return 8 * set + 1 + b; }
constexpr uint32_t kNoPtr = 0xffffffffu;
constexpr uint64_t kBigDeg = (1ull << 24) - 1;

__device__ __forceinline__ uint64_t make_pair(uint32_t lo, uint32_t hi) {
  return (uint64_t)lo | ((uint64_t)hi << 32);
}
__device__ __forceinline__ void row_range(const ulonglong2& e, const int64_t* __restrict__ offs,
                                          int64_t vbase, int64_t* s, int64_t* en) {
  const uint64_t d = e.y >> 40;
  *s = (int64_t)(e.y & ((1ull << 40) - 1));
  *en = d == kBigDeg ? offs[(int64_t)(uint32_t)e.x - vbase + 1] : *s + (int64_t)d;
}

// One frontier list, structure of arrays (round 2): p[i] = u | ptr << 32 (the pair the match and
// the compaction read: 8 B per entry instead of 16), r[i] = row start | degree << 40 (read by the
// pointer kernels with it).  list[i] returns both as a ulonglong2 (.x = p, .y = r).
struct FL {
  uint64_t* p;
  uint64_t* r;
  __device__ __forceinline__ ulonglong2 operator[](int64_t i) const { return make_ulonglong2(p[i], r[i]); }
  __device__ __forceinline__ void put(int64_t i, const ulonglong2& e) const {
    p[i] = e.x;
    r[i] = e.y;
  }
};
struct Bins {
  FL list[kBins];
};

// Device-resident round bookkeeping, so the round loop needs no host decision: the same launch
// sequence runs host-driven or as a captured CUDA graph with a conditional WHILE node.
struct RoundState {
  int cur;               // index of the set holding the current live pairs S and frontier F
  int cont;              // 1 = another round follows (host-driven mode reads it)
  long long rounds;      // pointing phases executed (round 1 = the sweep)
  long long max_rounds;
  long long ftot;        // sum of frontier sizes over rounds >= 2
  long long log_len;     // rows written to the per-round log
  long long log_cap;
  unsigned long long swept_prev;
  uint32_t tag;          // per-run tag of the A7 live counts (1..65535, advanced by k_round_init)
  uint32_t push;         // A6 push frontier active (persistent kernel; set by end_round_body)
};
__device__ __forceinline__ uint32_t round_tag(const RoundState* st) {
  return *reinterpret_cast<const volatile uint32_t*>(&st->tag);
}
struct RoundArgs {
  uint64_t* S[2];
  Bins F[2];
  unsigned long long* cnt;  // kNumCounters; set s = cnt_S(s), cnt_F(s, b)
  RoundState* st;
  long long* log;           // [log_cap][3]: |F_r|, |S_r| + |F_r|, E(F_r)
  uint32_t* live;           // A7 pruning: per-vertex live counts (nullptr = pruning off)
  const uint64_t* kc;       // resident key cache [n][kKC] (nullptr = off)
  uint64_t* best;           // per-vertex pointers (the compaction writes the cache-decided ones)
  uint32_t* N;              // A6 push frontier: vertices newly matched this round (nullptr = off)
  unsigned long long push_min_live;  // ... used once the live list is at least this long
};

// A2 pointer phase on the frontier (rounds >= 2): G lanes per vertex (degree-binned).
//   best[u] = max{ adj[j] : j in row(u), !matched(col) }   (Alg. 3 L5-8)
// Keys are loaded U at a time per lane and the bitmap words of the candidates (keys above the
// running max at batch start) are fetched together, so no L2 round trip sits on the loop-carried
// max.  Zeroed self-loop keys never qualify.  The new pointer goes to best[u] and into the slot.
#ifndef LM_PROBE3_MIN_G
#define LM_PROBE3_MIN_G 32  // two-phase probing only for warp and CTA rows (measured: it slows
                            // the 1- and 8-lane bins, speeds up the 32-lane and CTA bins ~10%)
#endif
#ifndef LM_PROBE
#define LM_PROBE 3  // bitmap probes per batch: 0 = all candidates in parallel, 1 = descending, 2 = top first,
                    // 3 = two-phase (lane tops, then only keys above the group's best)
#endif
#ifndef LM_R1_NOFFS
#define LM_R1_NOFFS 1  // round-1 compaction reads frontier rows' ranges from noffs (item order)
#endif
#ifndef LM_MATCH_V
#define LM_MATCH_V 4  // frontier entries per thread step in the match, loads batched (1 -> 4: -0.4%)
#endif
#ifndef LM_MAX1
#define LM_MAX1 1  // two-phase probe: lane max first, then one compare with the running best (0 = per-key test)
#endif
#ifndef LM_IDX32
#define LM_IDX32 0  // 1 = resident rows indexed with 32-bit offsets from the row start
#endif
#ifndef LM_RES_FAST
#define LM_RES_FAST 1  // rows wholly in the HBM-resident prefix load keys straight from adj.dev
#endif
#ifndef LM_UB_FILTER
#define LM_UB_FILTER 0  // 1 = keys at or above the vertex's previous pointer are skipped (R3)
#endif
#ifndef LM_LIST_PF
#define LM_LIST_PF 0  // 1 = binned pointer kernels prefetch the group's next frontier entry
#endif
#ifndef LM_QEXIT
#define LM_QEXIT 0  // 1 = sub-warp groups skip the key columns past the row end (group-uniform)
#endif
// RES: the row lies in the HBM-resident prefix (e <= R), so keys are plain loads from adj.dev
// instead of AdjView's per-key region test (decided once per row; group-uniform)
template <int G, int U, bool RES>
__device__ __forceinline__ uint64_t scan_row_available_t(const AdjView adj,
                                                         const uint32_t* __restrict__ bits,
                                                         int64_t s, int64_t e, int gl,
                                                         unsigned rmask, uint64_t ub = ~0ull) {
  (void)ub;
  uint64_t b = 0;
  (void)rmask;
#if LM_IDX32
  // resident rows: 32-bit offsets from the row start (a row has < 2^31 entries)
  const uint64_t* rp = adj.dev + s;
  const int32_t len32 = RES ? (int32_t)(e - s) : 0;
#endif
#if LM_QEXIT
  // sub-warp groups (G = 2..16): a batch touches only the ceil(rest / G) key columns the row
  // still has, so a 12-entry row in a 16 x 4 group costs one column of loads and probes, not 4
  if (G > 1 && G < LM_PROBE3_MIN_G) {
    for (int64_t jb = s; jb < e; jb += (int64_t)G * U) {
      const int64_t j0 = jb + gl;
      const int64_t rest = e - jb;
      uint64_t k[U];
#pragma unroll
      for (int q = 0; q < U; ++q) {
        k[q] = 0ull;
        if ((int64_t)q * G >= rest) break;
        const int64_t j = j0 + (int64_t)q * G;
        if (j < e) k[q] = RES ? ld_stream_u64(adj.dev + j) : adj.at(j);
#if LM_UB_FILTER
        if (k[q] >= ub) k[q] = 0ull;
#endif
      }
      uint32_t wd[U];
#pragma unroll
      for (int q = 0; q < U; ++q) {
        wd[q] = 0xffffffffu;
        if ((int64_t)q * G >= rest) break;
        if (k[q] > b) wd[q] = probe_word(bits, (uint32_t)k[q]);
      }
#pragma unroll
      for (int q = 0; q < U; ++q) {
        if ((int64_t)q * G >= rest) break;
        const uint32_t v = (uint32_t)k[q];
        if (!((wd[q] >> (v & 31)) & 1u) && k[q] > b) b = k[q];
      }
    }
    return b;
  }
#endif
  // batch loop with a group-uniform trip count (the group votes inside it)
  for (int64_t jb = s; jb < e; jb += (int64_t)G * U) {
    const int64_t j0 = jb + gl;
    uint64_t k[U];
#if LM_IDX32
    if (RES) {
      const int32_t o0 = (int32_t)(jb - s) + gl;
#pragma unroll
      for (int q = 0; q < U; ++q) {
        const int32_t o = o0 + q * G;
        k[q] = o < len32 ? ld_stream_u64(rp + o) : 0ull;
      }
    } else
#endif
    {
#pragma unroll
    for (int q = 0; q < U; ++q) {
      const int64_t j = j0 + (int64_t)q * G;
      k[q] = j < e ? (RES ? ld_stream_u64(adj.dev + j) : adj.at(j)) : 0ull;
#if LM_UB_FILTER
      if (k[q] >= ub) k[q] = 0ull;
#endif
    }
    }
#if LM_PROBE == 3
    if (G >= LM_PROBE3_MIN_G) {
    // Two-phase probe.  Phase 1: every lane probes only its largest candidate; C = the max of
    // the available ones over the reduction group (rmask: the lanes sharing this row, or the
    // warp for CTA rows).  Keys <= max(b, C) cannot be the answer, so phase 2 probes only the
    // keys above it held by lanes whose top candidate was matched -- usually none.  b stays
    // uniform over the reduction group.
    {
      uint64_t mx = 0;
#pragma unroll
#if LM_FRONT_DMAX
      {
        double m = 0.0;
        for (int q = 0; q < U; ++q) m = kd_of(k[q]) > m ? kd_of(k[q]) : m;
        mx = m > kd_of(b) ? ku_of(m) : 0ull;
      }
#elif LM_MAX1
      for (int q = 0; q < U; ++q) mx = umax64(mx, k[q]);
      if (mx <= b) mx = 0;
#else
      for (int q = 0; q < U; ++q) mx = (k[q] > b && k[q] > mx) ? k[q] : mx;
#endif
      bool avail = false;
      if (mx) avail = !((probe_word(bits, (uint32_t)mx) >> ((uint32_t)mx & 31)) & 1u);
      uint64_t c = avail ? mx : 0ull;
      if (G > 1) c = group_max_key(c, rmask);
      const uint64_t bb = c > b ? c : b;
      bool need = false;
      if (mx && !avail) {
#pragma unroll
        for (int q = 0; q < U; ++q) need |= (k[q] > bb && k[q] != mx);
      }
      const bool any = (G > 1) ? (__ballot_sync(rmask, need) & rmask) != 0u : need;
      b = bb;
      if (any) {
        uint32_t wd[U];
#pragma unroll
        for (int q = 0; q < U; ++q)
          wd[q] = (need && k[q] > bb && k[q] != mx) ? probe_word(bits, (uint32_t)k[q]) : 0xffffffffu;
        uint64_t c2 = 0;
#pragma unroll
        for (int q = 0; q < U; ++q) {
          const uint32_t v = (uint32_t)k[q];
          if (!((wd[q] >> (v & 31)) & 1u) && k[q] > c2) c2 = k[q];
        }
        if (G > 1) c2 = group_max_key(c2, rmask);
        b = c2 > b ? c2 : b;
      }
    }
    } else {
      uint32_t wd[U];
#if LM_FRONT_DMAX
      double bd = kd_of(b);
#pragma unroll
      for (int q = 0; q < U; ++q) wd[q] = kd_of(k[q]) > bd ? probe_word(bits, (uint32_t)k[q]) : 0xffffffffu;
#pragma unroll
      for (int q = 0; q < U; ++q) {
        const uint32_t v = (uint32_t)k[q];
        const double kd = kd_of(k[q]);
        bd = (!((wd[q] >> (v & 31)) & 1u) && kd > bd) ? kd : bd;
      }
      b = ku_of(bd);
#else
#pragma unroll
      for (int q = 0; q < U; ++q) wd[q] = k[q] > b ? probe_word(bits, (uint32_t)k[q]) : 0xffffffffu;
#pragma unroll
      for (int q = 0; q < U; ++q) {
        const uint32_t v = (uint32_t)k[q];
        if (!((wd[q] >> (v & 31)) & 1u) && k[q] > b) b = k[q];
      }
#endif
    }
#elif LM_PROBE == 1
    // descending: probe the lane's largest candidate, drop it if matched, repeat
    for (int it = 0; it < U; ++it) {
      uint64_t mx = 0;
#pragma unroll
      for (int q = 0; q < U; ++q) mx = (k[q] > b && k[q] > mx) ? k[q] : mx;
      if (!mx) break;
      const uint32_t v = (uint32_t)mx;
      if (!((probe_word(bits, v) >> (v & 31)) & 1u)) { b = mx; break; }
#pragma unroll
      for (int q = 0; q < U; ++q) k[q] = k[q] == mx ? 0ull : k[q];
    }
#else
#if LM_PROBE == 2
    {
      // the lane's largest candidate first: if available it is the lane's answer for the batch
      uint64_t mx = 0;
#pragma unroll
      for (int q = 0; q < U; ++q) mx = (k[q] > b && k[q] > mx) ? k[q] : mx;
      if (mx) {
        const uint32_t v = (uint32_t)mx;
        if (!((probe_word(bits, v) >> (v & 31)) & 1u)) {
          b = mx;
          continue;
        }
#pragma unroll
        for (int q = 0; q < U; ++q) k[q] = k[q] == mx ? 0ull : k[q];
      }
    }
#endif
    uint32_t wd[U];
#pragma unroll
    for (int q = 0; q < U; ++q) wd[q] = k[q] > b ? probe_word(bits, (uint32_t)k[q]) : 0xffffffffu;
#pragma unroll
    for (int q = 0; q < U; ++q) {
      const uint32_t v = (uint32_t)k[q];
      if (!((wd[q] >> (v & 31)) & 1u) && k[q] > b) b = k[q];
    }
#endif
  }
  return b;
}
// ub: an exclusive upper bound on the available keys of the row (LM_UB_FILTER): the vertex's
// previous pointer, since every key above it was unavailable when it was computed and stays so
// (R3) and the pointer's own target was matched; keys >= ub are neither compared nor probed
template <int G, int U>
__device__ __forceinline__ uint64_t scan_row_available(const AdjView adj,
                                                       const uint32_t* __restrict__ bits,
                                                       int64_t s, int64_t e, int gl,
                                                       unsigned rmask, uint64_t ub = ~0ull) {
#if LM_RES_FAST
  if (e <= adj.R) return scan_row_available_t<G, U, true>(adj, bits, s, e, gl, rmask, ub);
#endif
  return scan_row_available_t<G, U, false>(adj, bits, s, e, gl, rmask, ub);
}

// A7 in-place pruning (opt-in, lmatch_opts.prune) of a row that fits ONE batch
// of the group (deg <= G*U): every key is probed; the group partitions the row in place --
// available entries first (index order), then the dead ones (matched neighbour or zeroed
// self-loop) -- and records live[u] = tag << 16 | #available.  The row stays a permutation of
// itself, so later runs (whose round-1 sweep reads whole rows) are unaffected; later rounds of
// THIS run scan only the live prefix (compact_body).  Dead entries can never become available
// again (available sets only shrink, R3), so the pointer result is unchanged.  Keys
// are read with ld.global.cg: a pruned row may be re-read by another SM in the same
// (persistent) kernel, and the non-coherent L1 path could return the pre-permutation bytes.
template <int G, int U>
__device__ __forceinline__ uint64_t prune_row(const AdjView adj, const uint32_t* __restrict__ bits,
                                              int64_t s, int64_t en, int gl, unsigned gmask,
                                              uint32_t* __restrict__ live, uint32_t tag,
                                              int64_t lu) {
  const int L = (int)(en - s);
  uint64_t* row = adj.ptr(s);
  uint64_t k[U];
#pragma unroll
  for (int q = 0; q < U; ++q) {
    const int r = gl + q * G;
    k[q] = r < L ? __ldcg(reinterpret_cast<const unsigned long long*>(row + r)) : 0ull;
  }
  uint32_t wd[U];
#pragma unroll
  for (int q = 0; q < U; ++q) wd[q] = k[q] ? probe_word(bits, (uint32_t)k[q]) : 0xffffffffu;
  bool sv[U];
  uint64_t b = 0;
#pragma unroll
  for (int q = 0; q < U; ++q) {
    const uint32_t v = (uint32_t)k[q];
    sv[q] = k[q] != 0ull && !((wd[q] >> (v & 31)) & 1u);
    if (sv[q] && k[q] > b) b = k[q];
  }
  if (G > 1) b = group_max_key(b, gmask);
  const int gbase = (threadIdx.x & 31) & ~(G - 1);
  unsigned msk[U];
  int K = 0;
#pragma unroll
  for (int q = 0; q < U; ++q) {
    msk[q] = G > 1 ? (__ballot_sync(gmask, sv[q]) & gmask) >> gbase : (sv[q] ? 1u : 0u);
    K += __popc(msk[q]);
  }
  if (K < L) {
    int cs = 0;  // available entries before batch column q
#pragma unroll
    for (int q = 0; q < U; ++q) {
      const int r = gl + q * G;
      const int rank = cs + __popc(msk[q] & ((1u << gl) - 1u));  // available entries before r
      if (r < L) {
        const int np = sv[q] ? rank : K + (r - rank);
        if (np != r) row[np] = k[q];
      }
      cs += __popc(msk[q]);
    }
    if (gl == 0) live[lu] = (tag << 16) | (uint32_t)K;
  }
  return b;
}

template <int G, int U, bool PRUNE = false>
__device__ __forceinline__ void point_bin_body(const FL list, int64_t cnt,
                                               const int64_t* __restrict__ offs, const AdjView adj,
                                               const uint32_t* __restrict__ bits,
                                               uint64_t* __restrict__ best, int64_t vbase,
                                               int64_t gtid, int64_t gthreads,
                                               uint32_t* __restrict__ live = nullptr,
                                               uint32_t tag = 0) {
  const int lane = threadIdx.x & 31;
  const int gl = lane & (G - 1);
  const unsigned gmask = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
  const int64_t ng = gthreads / G;
#if LM_LIST_PF
  // the group's next list entry is loaded one row ahead, so a row's key loads do not wait for
  // its entry (one dependent DRAM trip less per row)
  ulonglong2 enx = gtid / G < cnt ? list[gtid / G] : make_ulonglong2(0ull, 0ull);
#endif
  for (int64_t i = gtid / G; i < cnt; i += ng) {
#if LM_LIST_PF
    const ulonglong2 e = enx;
    enx = i + ng < cnt ? list[i + ng] : make_ulonglong2(0ull, 0ull);
#else
    const ulonglong2 e = list[i];
#endif
    int64_t s, en;
    row_range(e, offs, vbase, &s, &en);
    uint64_t ub = ~0ull;
#if LM_UB_FILTER
    {
      const uint64_t old = best[(int64_t)(uint32_t)e.x - vbase];
      if (old) ub = old;  // 0: unknown (a pushed vertex's pointer was cleared)
    }
#endif
    uint64_t b;
    if (PRUNE && en - s <= (int64_t)G * U)
      b = prune_row<G, U>(adj, bits, s, en, gl, gmask, live, tag, (int64_t)(uint32_t)e.x - vbase);
    else
      b = group_max_key(scan_row_available<G, U>(adj, bits, s, en, gl, gmask, ub), gmask);
    if (gl == 0) {
      const uint32_t u = (uint32_t)e.x;
      best[u - vbase] = b;
      list.p[i] = make_pair(u, b ? (uint32_t)b : kNoPtr);
    }
  }
}
#ifndef LM_BIN_MINB
#define LM_BIN_MINB 8  // 32-register cap, full occupancy (6 -> 8 with the 16x4 / 32x8 bins: rounds 8.09 -> 7.74 ms)
#endif
template <int G, int U, bool PRUNE = false>
__global__ void __launch_bounds__(256, LM_BIN_MINB) k_point_bin(const FL list, const unsigned long long* cnt_ptr,
                            const int64_t* __restrict__ offs, const AdjView adj,
                            const uint32_t* __restrict__ bits, uint64_t* __restrict__ best,
                            int64_t vbase, uint32_t* __restrict__ live = nullptr,
                            const RoundState* st = nullptr) {
  point_bin_body<G, U, PRUNE>(list, (int64_t)*cnt_ptr, offs, adj, bits, best, vbase,
                              (int64_t)blockIdx.x * blockDim.x + threadIdx.x,
                              (int64_t)gridDim.x * blockDim.x, live, PRUNE ? round_tag(st) : 0u);
}

// Software-pipelined variant for the big host-driven rounds (grid = one resident wave, so every
// group walks many rows): the keys of the NEXT batch (the next batch of the same row, or the
// first batch of the group's next row, whose list entry was prefetched one row earlier) are
// loaded before the bitmap probes of the current batch, so a DRAM round trip and an L2 round
// trip overlap instead of adding up per row.  Same result as point_bin_body (u64 max).
template <int G, int U>
__device__ __forceinline__ void load_batch(const AdjView adj, int64_t j0, int64_t e,
                                           uint64_t (&k)[U]) {
#if LM_RES_FAST
  if (e <= adj.R) {
#pragma unroll
    for (int q = 0; q < U; ++q) {
      const int64_t j = j0 + (int64_t)q * G;
      k[q] = j < e ? ld_stream_u64(adj.dev + j) : 0ull;
    }
    return;
  }
#endif
#pragma unroll
  for (int q = 0; q < U; ++q) {
    const int64_t j = j0 + (int64_t)q * G;
    k[q] = j < e ? adj.at(j) : 0ull;
  }
}
template <int U>
__device__ __forceinline__ uint64_t probe_batch(const uint32_t* __restrict__ bits,
                                                const uint64_t (&k)[U], uint64_t b) {
  uint32_t wd[U];
#if LM_FRONT_DMAX
  double bd = kd_of(b);
#pragma unroll
  for (int q = 0; q < U; ++q) wd[q] = kd_of(k[q]) > bd ? probe_word(bits, (uint32_t)k[q]) : 0xffffffffu;
#pragma unroll
  for (int q = 0; q < U; ++q) {
    const uint32_t v = (uint32_t)k[q];
    const double kd = kd_of(k[q]);
    bd = (!((wd[q] >> (v & 31)) & 1u) && kd > bd) ? kd : bd;
  }
  return ku_of(bd);
#else
#pragma unroll
  for (int q = 0; q < U; ++q) wd[q] = k[q] > b ? probe_word(bits, (uint32_t)k[q]) : 0xffffffffu;
#pragma unroll
  for (int q = 0; q < U; ++q) {
    const uint32_t v = (uint32_t)k[q];
    if (!((wd[q] >> (v & 31)) & 1u) && k[q] > b) b = k[q];
  }
  return b;
#endif
}
// Two-phase probe of one batch (group-uniform b): lanes probe their top candidate; only keys
// above the group's best available top are probed in a second step.
#ifndef LM_PIPE_PROBE3_MIN_G
#define LM_PIPE_PROBE3_MIN_G 1
#endif
#ifndef LM_PIPE_PROBE
#define LM_PIPE_PROBE 0
#endif
template <int G, int U>
__device__ __forceinline__ uint64_t probe_batch2(const uint32_t* __restrict__ bits,
                                                 const uint64_t (&k)[U], uint64_t b,
                                                 unsigned gmask) {
  uint64_t mx = 0;
#pragma unroll
  for (int q = 0; q < U; ++q) mx = (k[q] > b && k[q] > mx) ? k[q] : mx;
  bool avail = false;
  if (mx) avail = !((probe_word(bits, (uint32_t)mx) >> ((uint32_t)mx & 31)) & 1u);
  uint64_t c = avail ? mx : 0ull;
  if (G > 1) c = group_max_key(c, gmask);
  const uint64_t bb = c > b ? c : b;
  bool need = false;
  if (mx && !avail) {
#pragma unroll
    for (int q = 0; q < U; ++q) need |= (k[q] > bb && k[q] != mx);
  }
  const bool any = G > 1 ? (__ballot_sync(gmask, need) & gmask) != 0u : need;
  if (!any) return bb;
  uint32_t wd[U];
#pragma unroll
  for (int q = 0; q < U; ++q)
    wd[q] = (need && k[q] > bb && k[q] != mx) ? probe_word(bits, (uint32_t)k[q]) : 0xffffffffu;
  uint64_t c2 = 0;
#pragma unroll
  for (int q = 0; q < U; ++q) {
    const uint32_t v = (uint32_t)k[q];
    if (!((wd[q] >> (v & 31)) & 1u) && k[q] > c2) c2 = k[q];
  }
  if (G > 1) c2 = group_max_key(c2, gmask);
  return c2 > bb ? c2 : bb;
}

template <int G, int U>
__device__ __forceinline__ void point_pipe_body(const FL list, int64_t cnt,
                                                const int64_t* __restrict__ offs, const AdjView adj,
                                                const uint32_t* __restrict__ bits,
                                                uint64_t* __restrict__ best, int64_t vbase,
                                                int64_t gtid, int64_t gthreads) {
  const int lane = threadIdx.x & 31;
  const int gl = lane & (G - 1);
  const unsigned gmask = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
  const int64_t ng = gthreads / G;
  constexpr int64_t B = (int64_t)G * U;
  int64_t li = gtid / G;  // row of the load stream (group-uniform)
  if (li >= cnt) return;
  ulonglong2 le = list[li];
  ulonglong2 pf = li + ng < cnt ? list[li + ng] : make_ulonglong2(0ull, 0ull);
  int64_t ls, lend;
  row_range(le, offs, vbase, &ls, &lend);
  uint64_t kc[U];
  load_batch<G, U>(adj, ls + gl, lend, kc);
  int64_t ci = li;
  uint32_t cu = (uint32_t)le.x;
  bool clast = ls + B >= lend;
  int64_t ljb = ls + B;  // next batch base of the load row
  uint64_t b = 0;
  for (;;) {
    uint64_t kn[U];
    int64_t ni = -1;
    uint32_t nu = 0;
    bool nlast = false;
    if (ljb < lend) {  // next batch of the same row
      load_batch<G, U>(adj, ljb + gl, lend, kn);
      ni = li;
      nu = (uint32_t)le.x;
      nlast = ljb + B >= lend;
      ljb += B;
    } else if (li + ng < cnt) {  // first batch of the next row
      li += ng;
      le = pf;
      pf = li + ng < cnt ? list[li + ng] : make_ulonglong2(0ull, 0ull);
      row_range(le, offs, vbase, &ls, &lend);
      load_batch<G, U>(adj, ls + gl, lend, kn);
      ni = li;
      nu = (uint32_t)le.x;
      nlast = ls + B >= lend;
      ljb = ls + B;
    }
    // LM_PIPE_PROBE == 3: two-phase probing (probe_batch2, group-uniform b) for groups of at
    // least LM_PIPE_PROBE3_MIN_G lanes; else every candidate of the batch at once
    constexpr bool two_phase = LM_PIPE_PROBE == 3 && G >= LM_PIPE_PROBE3_MIN_G;
    if (two_phase)
      b = probe_batch2<G, U>(bits, kc, b, gmask);
    else
      b = probe_batch<U>(bits, kc, b);
    if (clast) {
      const uint64_t r = (G > 1 && !two_phase) ? group_max_key(b, gmask) : b;
      if (gl == 0) {
        best[cu - vbase] = r;
        list.p[ci] = make_pair(cu, r ? (uint32_t)r : kNoPtr);
      }
      b = 0;
    }
    if (ni < 0) break;
#pragma unroll
    for (int q = 0; q < U; ++q) kc[q] = kn[q];
    ci = ni;
    cu = nu;
    clast = nlast;
  }
}
#ifndef LM_PIPE_MINB
#define LM_PIPE_MINB 1
#endif
template <int G, int U>
__global__ void __launch_bounds__(256, LM_PIPE_MINB)
    k_point_pipe(const FL list, const unsigned long long* cnt_ptr,
                 const int64_t* __restrict__ offs, const AdjView adj,
                 const uint32_t* __restrict__ bits, uint64_t* __restrict__ best, int64_t vbase) {
  point_pipe_body<G, U>(list, (int64_t)*cnt_ptr, offs, adj, bits, best, vbase,
                        (int64_t)blockIdx.x * blockDim.x + threadIdx.x,
                        (int64_t)gridDim.x * blockDim.x);
}

// ---------------------------------------------------------------------------------------------
// Asynchronous-copy variant for the big host-driven rounds.  Each lane keeps a private ring of
// S stages x U keys in shared memory filled with cp.async (LDGSTS, zero-fill past the row end),
// running S-1 (row, batch) items ahead of the bitmap probes, so the bytes in flight per SM no
// longer depend on registers (the register-staged kernels top out near 36 KB in flight per SM,
// ~3 TB/s).  A lane only reads keys it copied itself: cp.async.wait_group is the only sync.
// Layout [stage][q][thread] keeps the 8-byte shared accesses of a warp conflict-free.
__device__ __forceinline__ void cp_async8(void* sdst, const void* gsrc, uint32_t src_bytes) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(smem_u32(sdst)), "l"(gsrc),
               "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
template <int G, int U, int S>
__global__ void __launch_bounds__(256)
    k_point_async(const FL list, const unsigned long long* cnt_ptr,
                  const int64_t* __restrict__ offs, const uint64_t* __restrict__ adj,
                  const uint32_t* __restrict__ bits, uint64_t* __restrict__ best, int64_t vbase) {
  extern __shared__ __align__(16) uint64_t sk[];  // [S][U][256]
  const int tid = threadIdx.x;
  const int lane = tid & 31;
  const int gl = lane & (G - 1);
  const unsigned gmask = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
  const int64_t cnt = (int64_t)*cnt_ptr;
  const int64_t ng = ((int64_t)gridDim.x * blockDim.x) / G;
  constexpr int64_t B = (int64_t)G * U;
  // load stream (group-uniform): current row li, next batch base ljb, row end lend
  int64_t li = ((int64_t)blockIdx.x * blockDim.x + tid) / G;
  bool lvalid = li < cnt;
  int64_t ljb = 0, lend = 0;
  uint32_t lu = 0;
  ulonglong2 pf = make_ulonglong2(0ull, 0ull);
  if (lvalid) {
    const ulonglong2 e = list[li];
    row_range(e, offs, vbase, &ljb, &lend);
    lu = (uint32_t)e.x;
    if (li + ng < cnt) pf = list[li + ng];
  }
  // per-stage tags (registers: every index below is a compile-time constant after unrolling)
  int64_t tci[S];
  uint32_t tu[S];
  bool tlast[S], tval[S];
  auto issue = [&](int st) {
    if (lvalid && ljb >= lend) {  // row done: next row of this group
      li += ng;
      if (li < cnt) {
        const ulonglong2 e = pf;
        pf = li + ng < cnt ? list[li + ng] : make_ulonglong2(0ull, 0ull);
        row_range(e, offs, vbase, &ljb, &lend);
        lu = (uint32_t)e.x;
      } else {
        lvalid = false;
      }
    }
    tval[st] = lvalid;
    if (lvalid) {
#pragma unroll
      for (int q = 0; q < U; ++q) {
        const int64_t j = ljb + gl + (int64_t)q * G;
        const bool in = j < lend;
        cp_async8(&sk[((size_t)st * U + q) * 256 + tid], in ? adj + j : adj, in ? 8u : 0u);
      }
      tci[st] = li;
      tu[st] = lu;
      tlast[st] = ljb + B >= lend;
      ljb += B;
    }
    cp_async_commit();  // also when empty: keeps the group count uniform
  };
#pragma unroll
  for (int st = 0; st < S - 1; ++st) issue(st);
  uint64_t b = 0;
  for (;;) {
#pragma unroll
    for (int st = 0; st < S; ++st) {
      issue((st + S - 1) % S);  // the stage processed in the previous step
      cp_async_wait<S - 1>();   // => stage st has landed
      if (!tval[st]) goto done;
      {
        uint64_t k[U];
#pragma unroll
        for (int q = 0; q < U; ++q) k[q] = sk[((size_t)st * U + q) * 256 + tid];
        b = probe_batch<U>(bits, k, b);
      }
      if (tlast[st]) {
        const uint64_t r = G > 1 ? group_max_key(b, gmask) : b;
        if (gl == 0) {
          best[tu[st] - vbase] = r;
          list.p[tci[st]] = make_pair(tu[st], r ? (uint32_t)r : kNoPtr);
        }
        b = 0;
      }
    }
  }
done:
  cp_async_wait<0>();
}

template <int THREADS, int U>
__device__ __forceinline__ void point_bin_cta_body(const FL list, int64_t cnt,
                                                   const int64_t* __restrict__ offs,
                                                   const AdjView adj,
                                                   const uint32_t* __restrict__ bits,
                                                   uint64_t* __restrict__ best, int64_t vbase,
                                                   int64_t bid, int64_t nblk) {
  __shared__ uint64_t red[THREADS / 32];
  for (int64_t i = bid; i < cnt; i += nblk) {
    const ulonglong2 e = list[i];
    int64_t s, en;
    row_range(e, offs, vbase, &s, &en);
    uint64_t ub = ~0ull;
#if LM_UB_FILTER
    {
      const uint64_t old = best[(int64_t)(uint32_t)e.x - vbase];
      if (old) ub = old;
    }
#endif
    uint64_t b = scan_row_available<THREADS, U>(adj, bits, s, en, threadIdx.x, 0xffffffffu, ub);
    b = group_max_key(b, 0xffffffffu);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = b;
    __syncthreads();
    if (threadIdx.x < 32) {
      uint64_t x = threadIdx.x < THREADS / 32 ? red[threadIdx.x] : 0ull;
      x = group_max_key(x, 0xffffffffu);
      if (threadIdx.x == 0) {
        const uint32_t u = (uint32_t)e.x;
        best[u - vbase] = x;
        list.p[i] = make_pair(u, x ? (uint32_t)x : kNoPtr);
      }
    }
    __syncthreads();
  }
}
template <int THREADS, int U>
__global__ void __launch_bounds__(THREADS)
    k_point_bin_cta(const FL list, const unsigned long long* cnt_ptr,
                    const int64_t* __restrict__ offs, const AdjView adj,
                    const uint32_t* __restrict__ bits, uint64_t* __restrict__ best, int64_t vbase) {
  point_bin_cta_body<THREADS, U>(list, (int64_t)*cnt_ptr, offs, adj, bits, best, vbase, blockIdx.x,
                                 gridDim.x);
}

// =============================================================================================
// A4 match (SETMATES, Alg. 3 L10-13 P:152-155): mutual pointers are locally dominant edges.
// =============================================================================================
// Round 1: every vertex; the warp owning 32 consecutive vertices writes their bitmap word.
// Each warp owns 4 bitmap words per step and issues the 4 random best[ptr u] reads together.
#ifndef LM_MATCHALL_HALF
#define LM_MATCHALL_HALF 1  // round-1 match: mutual pairs checked from their smaller endpoint only
#endif
#ifndef LM_MATCHALL_V
#define LM_MATCHALL_V 4  // bitmap words per warp step (independent best[ptr u] gathers per lane)
#endif
__global__ void k_match_all(const uint64_t* __restrict__ best, int64_t n, uint32_t* bits) {
  constexpr int V = LM_MATCHALL_V;
  const int64_t nwords = (n + 31) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t ws = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t wb = w0; wb < nwords; wb += V * ws) {
    uint64_t b[V], bv[V];
#pragma unroll
    for (int q = 0; q < V; ++q) {
      const int64_t u = ((wb + q * ws) << 5) + lane;
      b[q] = (wb + q * ws < nwords && u < n) ? best[u] : 0ull;
    }
#if LM_MATCHALL_HALF
    // a mutual pair is found by its smaller endpoint only: u reads best[v] only when v > u, so
    // the random gathers (the kernel's cost) halve; that endpoint marks both (bits zeroed by
    // k_reset, so every mark is an atomicOr)
#pragma unroll
    for (int q = 0; q < V; ++q) {
      const int64_t u = ((wb + q * ws) << 5) + lane;
      bv[q] = (b[q] && (int64_t)(uint32_t)b[q] > u) ? best[(uint32_t)b[q]] : 0ull;
    }
#pragma unroll
    for (int q = 0; q < V; ++q) {
      const int64_t wi = wb + q * ws;
      const int64_t u = (wi << 5) + lane;
      const bool mutual = bv[q] != 0 && (uint32_t)bv[q] == (uint32_t)u;
      const unsigned word = __ballot_sync(0xffffffffu, mutual);
      if (lane == 0 && wi < nwords && word) atomicOr(&bits[wi], word);
      if (mutual) {
        const uint32_t v = (uint32_t)b[q];
        atomicOr(&bits[v >> 5], 1u << (v & 31));
      }
    }
#else
#pragma unroll
    for (int q = 0; q < V; ++q) bv[q] = b[q] ? best[(uint32_t)b[q]] : 0ull;
#pragma unroll
    for (int q = 0; q < V; ++q) {
      const int64_t wi = wb + q * ws;
      const int64_t u = (wi << 5) + lane;
      const bool mutual = bv[q] != 0 && (uint32_t)bv[q] == (uint32_t)u;
      const unsigned word = __ballot_sync(0xffffffffu, mutual);
      if (lane == 0 && wi < nwords) bits[wi] = word;
    }
#endif
  }
}

// Rounds >= 2: over the frontier's new pointers (pairs in the bins).  A new mutual pair has at
// least one endpoint that re-pointed this round (R3); that endpoint marks both.
__device__ __forceinline__ void match_bins_body(const Bins& F, const unsigned long long* cntF,
                                                const uint64_t* __restrict__ best, uint32_t* bits,
                                                int64_t tid, int64_t stride) {
#if LM_MATCH_V > 1
  // LM_MATCH_V entries per thread step with their dependent loads batched (the chain
  // entry -> best[ptr] is latency-bound otherwise)
  constexpr int V = LM_MATCH_V;
#pragma unroll
  for (int bb = 0; bb < kBins; ++bb) {
    const int64_t c = (int64_t)cntF[bb];
    for (int64_t i0 = tid; i0 < c; i0 += V * stride) {
      uint64_t p[V], kv[V];
#pragma unroll
      for (int q = 0; q < V; ++q) {
        const int64_t i = i0 + q * stride;
        p[q] = i < c ? F.list[bb].p[i] : ((uint64_t)kNoPtr << 32);
      }
#pragma unroll
      for (int q = 0; q < V; ++q) {
        const uint32_t v = (uint32_t)(p[q] >> 32);
        kv[q] = v != kNoPtr ? best[v] : 0ull;
      }
#pragma unroll
      for (int q = 0; q < V; ++q) {
        const uint32_t u = (uint32_t)p[q], v = (uint32_t)(p[q] >> 32);
        if (kv[q] != 0 && (uint32_t)kv[q] == u) {
          atomicOr(&bits[u >> 5], 1u << (u & 31));
          atomicOr(&bits[v >> 5], 1u << (v & 31));
        }
      }
    }
  }
#else
#pragma unroll
  for (int bb = 0; bb < kBins; ++bb) {
    const int64_t c = (int64_t)cntF[bb];
    for (int64_t i = tid; i < c; i += stride) {
      const uint64_t p = F.list[bb].p[i];
      const uint32_t u = (uint32_t)p, v = (uint32_t)(p >> 32);
      if (v == kNoPtr) continue;
      const uint64_t kv = best[v];
      if (kv != 0 && (uint32_t)kv == u) {
        atomicOr(&bits[u >> 5], 1u << (u & 31));
        atomicOr(&bits[v >> 5], 1u << (v & 31));
      }
    }
  }
#endif
}
__global__ void k_match_bins(Bins F, const unsigned long long* cntF,
                             const uint64_t* __restrict__ best, uint32_t* bits) {
  match_bins_body(F, cntF, best, bits, (int64_t)blockIdx.x * blockDim.x + threadIdx.x,
                  (int64_t)gridDim.x * blockDim.x);
}

// =============================================================================================
// A6 frontier compaction (not in the paper, which rescans every unmatched vertex).
// The live set is kept as pairs (u, ptr u): S_r (pointers unchanged since an earlier round) and
// the frontier bins of round r (fresh pointers).  For each live pair with u still unmatched:
//   ptr u matched   -> u joins frontier bin deg(u) of round r+1 (pointer must be recomputed)
//   ptr u unmatched -> (u, ptr u) joins S_{r+1}
// Round 1 (ALL) derives the pairs from best[] over every vertex.  Inputs are streamed; the random
// accesses are two bitmap bits (L2-resident) and, for frontier members only, deg(u).  Each warp
// owns a chunk of 32*K items: ONE atomicAdd per output list per warp reserves its ranges.
// =============================================================================================
// Set `in` (S and frontier bins) is read (ignored when ALL), set `out` is written.
struct CompactIO {
  const uint64_t* S;
  Bins Fin;
  uint64_t* Sout;
  Bins Fout;
  const unsigned long long* cin;  // counters of the input set (cnt_S .. cnt_F(.,kBins-1) contiguous)
  unsigned long long* cout;       // counters of the output set
  unsigned long long* swept;
  const uint32_t* live;           // A7: live counts (nullptr = pruning off)
  const RoundState* st;
  const int32_t* nzr;             // ALL mode: iterate the non-empty rows only (nullptr = all n)
  const int64_t* noffs = nullptr; // ALL mode with nzr: the non-empty rows' offsets (LM_R1_NOFFS)
  const uint64_t* kc;             // key cache [n][kKC] (nullptr = off)
  uint64_t* best_w;               // key cache: pointers decided by the compaction (= best)
};
__host__ __device__ inline CompactIO compact_io(const RoundArgs& a, int cur) {
  CompactIO io;
  io.S = a.S[cur];
  io.Fin = a.F[cur];
  io.Sout = a.S[cur ^ 1];
  io.Fout = a.F[cur ^ 1];
  io.cin = a.cnt + cnt_S(cur);
  io.cout = a.cnt + cnt_S(cur ^ 1);
  io.swept = a.cnt + kCntSwept;
  io.live = a.live;
  io.st = a.st;
  io.nzr = nullptr;
  io.noffs = nullptr;
  io.kc = a.kc;
  io.best_w = a.best;
  return io;
}

// key cache: the new pointer of frontier vertex u from its cached keys, as Alg. 1 L4 would
// compute it now (the bitmap holds every match up to this round): the first available cached key
// (descending), or "none" when the row has fewer than kKC keys and all are matched (the cache
// holds the whole row).  Returns false when the row must be scanned.
__device__ __forceinline__ bool kc_decide(const uint64_t* __restrict__ kc, const uint32_t* __restrict__ bits,
                                          int64_t lu, uint64_t* key) {
  const ulonglong2* c = reinterpret_cast<const ulonglong2*>(kc + (size_t)lu * kKC);
  uint64_t k[kKC];
#pragma unroll
  for (int h = 0; h < kKC / 2; ++h) {
    const ulonglong2 a = c[h];
    k[2 * h] = a.x;
    k[2 * h + 1] = a.y;
  }
  uint32_t wd[kKC];
#pragma unroll
  for (int q = 0; q < kKC; ++q) wd[q] = k[q] ? bits[(uint32_t)k[q] >> 5] : 0xffffffffu;
#pragma unroll
  for (int q = 0; q < kKC; ++q)
    if (k[q] && !((wd[q] >> ((uint32_t)k[q] & 31)) & 1u)) { *key = k[q]; return true; }
  *key = 0;
  return k[kKC - 1] == 0;
}

// the compaction without the key cache (4 degree bins out; the decided input list is empty)
template <bool ALL, int K>
__device__ __forceinline__ void compact_body_plain(const CompactIO& io, int64_t n,
                                             const uint64_t* __restrict__ best,
                                             const uint32_t* __restrict__ bits,
                                             const int64_t* __restrict__ offs, int64_t vbase,
                                             int64_t bid, int64_t nblk) {
  constexpr int NW = 8, NL = 1 + kDegBins;  // blockDim must be 256
  const uint64_t* __restrict__ S = io.S;
  const unsigned long long* cntS = io.cin;
  const Bins& Fin = io.Fin;
  const unsigned long long* cntFin = io.cin + 1;
  uint64_t* __restrict__ Sout = io.Sout;
  unsigned long long* cntSout = io.cout;
  const Bins& Fout = io.Fout;
  unsigned long long* cntFout = io.cout + 1;
  unsigned long long* swept = io.swept;  // warps per block (blockDim 256), output lists
  __shared__ unsigned wtot[NW][NL];
  __shared__ unsigned long long wbase[NW][NL];
  // virtual concatenation S ++ F_0 ++ F_1 ++ F_2 ++ F_3 (prefix ends p0 < p1 < ... < p4; the
  // decided list F_4 is empty without the key cache)
  const int64_t p0 = ALL ? n : (int64_t)*cntS;
  const int64_t p1 = p0 + (ALL ? 0 : (int64_t)cntFin[0]);
  const int64_t p2 = p1 + (ALL ? 0 : (int64_t)cntFin[1]);
  const int64_t p3 = p2 + (ALL ? 0 : (int64_t)cntFin[2]);
  const int64_t cnt = p3 + (ALL ? 0 : (int64_t)cntFin[3]);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const unsigned lt = lanemask_lt();
  const uint32_t* __restrict__ lcnt = io.live;
  const uint32_t tag = lcnt ? round_tag(io.st) : 0u;
  constexpr int64_t BLK = (int64_t)NW * 32 * K;
  unsigned long long degsum = 0;
  for (int64_t cb = bid * BLK; cb < cnt; cb += nblk * BLK) {
    const int64_t c0 = cb + (int64_t)warp * 32 * K;
    uint32_t sbits = 0, fb0 = 0, fb1 = 0, fb2 = 0, fb3 = 0;
    uint64_t pr[K], rr[K];
    // phase 1: every list element of the chunk (independent loads)
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const int64_t i = c0 + 32 * k + lane;
      uint64_t p = (uint64_t)kNoPtr << 32;
      if (i < cnt) {
        if (ALL) {
          // an empty row never holds a pointer: with the non-empty row list only those are read
          const int64_t r = io.nzr ? (int64_t)io.nzr[i] : i;
          const uint64_t bb = best[r];
          p = make_pair((uint32_t)(r + vbase), bb ? (uint32_t)bb : kNoPtr);
        } else {
          p = i < p0 ? S[i]
              : i < p1 ? Fin.list[0].p[i - p0]
              : i < p2 ? Fin.list[1].p[i - p1]
              : i < p3 ? Fin.list[2].p[i - p2]
                       : Fin.list[3].p[i - p3];
        }
      }
      pr[k] = p;
    }
    // phase 2: matched bits of u and of its pointer (L2-resident bitmap; independent loads)
    uint32_t wu[K], wv[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint32_t u = (uint32_t)pr[k], v = (uint32_t)(pr[k] >> 32);
      const bool ok = v != kNoPtr;
      wu[k] = ok ? bits[u >> 5] : 0xffffffffu;
      wv[k] = ok ? bits[v >> 5] : 0u;
    }
    // phase 3: classify; frontier members fetch their row range (independent loads)
    int64_t os[K], oe[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint32_t u = (uint32_t)pr[k], v = (uint32_t)(pr[k] >> 32);
      const bool live = !((wu[k] >> (u & 31)) & 1u);
      const bool tgt = (wv[k] >> (v & 31)) & 1u;
      if (live && !tgt) sbits |= 1u << k;
      const bool fr = live && tgt;
#if LM_R1_NOFFS
      // round 1 over the non-empty rows: row i's range is noffs[i], noffs[i+1] (item order)
      if (ALL && io.noffs) {
        const int64_t i = c0 + 32 * k + lane;
        os[k] = fr ? io.noffs[i] : 0;
        oe[k] = fr ? io.noffs[i + 1] : -1;
      } else
#endif
      {
        os[k] = fr ? offs[u - vbase] : 0;
        oe[k] = fr ? offs[u - vbase + 1] : -1;
      }
      if (lcnt && fr) {  // A7: a row pruned earlier in this run is scanned over its live prefix
        const uint32_t x = lcnt[u - vbase];
        if ((x >> 16) == tag) oe[k] = os[k] + (int64_t)(x & 0xffffu);
      }
    }
#pragma unroll
    for (int k = 0; k < K; ++k) {
      rr[k] = 0;
      if (oe[k] >= 0) {
        const int64_t d = oe[k] - os[k];
        const int b = bin_of(d);
        const uint32_t m = 1u << k;
        fb0 |= b == 0 ? m : 0u;
        fb1 |= b == 1 ? m : 0u;
        fb2 |= b == 2 ? m : 0u;
        fb3 |= b == 3 ? m : 0u;
        rr[k] = (uint64_t)os[k] | ((uint64_t)(d < (int64_t)kBigDeg ? d : (int64_t)kBigDeg) << 40);
        degsum += (unsigned long long)d;
      }
    }
    // reserve output ranges: warp totals -> block prefix -> ONE atomic per list per block
    {
      const unsigned ts = __reduce_add_sync(0xffffffffu, __popc(sbits));
      const unsigned t0 = __reduce_add_sync(0xffffffffu, __popc(fb0));
      const unsigned t1 = __reduce_add_sync(0xffffffffu, __popc(fb1));
      const unsigned t2 = __reduce_add_sync(0xffffffffu, __popc(fb2));
      const unsigned t3 = __reduce_add_sync(0xffffffffu, __popc(fb3));
      if (lane == 0) {
        wtot[warp][0] = ts; wtot[warp][1] = t0; wtot[warp][2] = t1;
        wtot[warp][3] = t2; wtot[warp][4] = t3;
      }
    }
    __syncthreads();
    if (threadIdx.x < NL) {
      const int q = threadIdx.x;
      unsigned long long tot = 0;
      for (int w = 0; w < NW; ++w) tot += wtot[w][q];
      unsigned long long base = 0;
      if (tot) base = atomicAdd(q == 0 ? cntSout : &cntFout[q - 1], tot);
      for (int w = 0; w < NW; ++w) { wbase[w][q] = base; base += wtot[w][q]; }
    }
    __syncthreads();
    unsigned long long bs = wbase[warp][0], bf0 = wbase[warp][1], bf1 = wbase[warp][2],
                       bf2 = wbase[warp][3], bf3 = wbase[warp][4];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint32_t m = 1u << k;
      const bool ps = sbits & m;
      const unsigned bls = __ballot_sync(0xffffffffu, ps);
      if (ps) Sout[bs + __popc(bls & lt)] = pr[k];
      bs += __popc(bls);
      const ulonglong2 ent = make_ulonglong2(pr[k], rr[k]);
      unsigned bb = __ballot_sync(0xffffffffu, (fb0 & m) != 0);
      if (fb0 & m) Fout.list[0].put(bf0 + __popc(bb & lt), ent);
      bf0 += __popc(bb);
      bb = __ballot_sync(0xffffffffu, (fb1 & m) != 0);
      if (fb1 & m) Fout.list[1].put(bf1 + __popc(bb & lt), ent);
      bf1 += __popc(bb);
      bb = __ballot_sync(0xffffffffu, (fb2 & m) != 0);
      if (fb2 & m) Fout.list[2].put(bf2 + __popc(bb & lt), ent);
      bf2 += __popc(bb);
      bb = __ballot_sync(0xffffffffu, (fb3 & m) != 0);
      if (fb3 & m) Fout.list[3].put(bf3 + __popc(bb & lt), ent);
      bf3 += __popc(bb);
    }
  }
  for (int o = 16; o; o >>= 1) degsum += __shfl_xor_sync(0xffffffffu, degsum, o);
  if (lane == 0 && degsum) atomicAdd(swept, degsum);
}
template <bool ALL, int K, bool KC = false>
__device__ __forceinline__ void compact_body(const CompactIO& io, int64_t n,
                                             const uint64_t* __restrict__ best,
                                             const uint32_t* __restrict__ bits,
                                             const int64_t* __restrict__ offs, int64_t vbase,
                                             int64_t bid, int64_t nblk) {
  constexpr int NW = 8, NL = 1 + kBins;  // blockDim must be 256
  if constexpr (!KC) {
    compact_body_plain<ALL, K>(io, n, best, bits, offs, vbase, bid, nblk);
    return;
  }
  const uint64_t* __restrict__ S = io.S;
  const unsigned long long* cntS = io.cin;
  const Bins& Fin = io.Fin;
  const unsigned long long* cntFin = io.cin + 1;
  uint64_t* __restrict__ Sout = io.Sout;
  unsigned long long* cntSout = io.cout;
  const Bins& Fout = io.Fout;
  unsigned long long* cntFout = io.cout + 1;
  unsigned long long* swept = io.swept;  // warps per block (blockDim 256), output lists
  __shared__ unsigned wtot[NW][NL];
  __shared__ unsigned long long wbase[NW][NL];
  // virtual concatenation S ++ F_0 ++ ... ++ F_{kBins-1} (prefix ends p[0] < p[1] < ...)
  int64_t pe[kBins + 1];
  pe[0] = ALL ? n : (int64_t)*cntS;
#pragma unroll
  for (int q = 0; q < kBins; ++q) pe[q + 1] = pe[q] + (ALL ? 0 : (int64_t)cntFin[q]);
  const int64_t cnt = pe[kBins];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const unsigned lt = lanemask_lt();
  const uint32_t* __restrict__ lcnt = io.live;
  const uint32_t tag = lcnt ? round_tag(io.st) : 0u;
  constexpr int64_t BLK = (int64_t)NW * 32 * K;
  unsigned long long degsum = 0, decided = 0;
  for (int64_t cb = bid * BLK; cb < cnt; cb += nblk * BLK) {
    const int64_t c0 = cb + (int64_t)warp * 32 * K;
    uint32_t sbits = 0, fb[kBins] = {0, 0, 0, 0, 0};
    uint64_t pr[K], rr[K];
    // phase 1: every list element of the chunk (independent loads)
#pragma unroll
    for (int k = 0; k < K; ++k) {
      rr[k] = 0;
      const int64_t i = c0 + 32 * k + lane;
      uint64_t p = (uint64_t)kNoPtr << 32;
      if (i < cnt) {
        if (ALL) {
          // an empty row never holds a pointer: with the non-empty row list only those are read
          const int64_t r = io.nzr ? (int64_t)io.nzr[i] : i;
          const uint64_t bb = best[r];
          p = make_pair((uint32_t)(r + vbase), bb ? (uint32_t)bb : kNoPtr);
        } else {
          p = i < pe[0] ? S[i]
              : i < pe[1] ? Fin.list[0].p[i - pe[0]]
              : i < pe[2] ? Fin.list[1].p[i - pe[1]]
              : i < pe[3] ? Fin.list[2].p[i - pe[2]]
              : i < pe[4] ? Fin.list[3].p[i - pe[3]]
                          : Fin.list[4].p[i - pe[4]];
        }
      }
      pr[k] = p;
    }
    // phase 2: matched bits of u and of its pointer (L2-resident bitmap; independent loads)
    uint32_t wu[K], wv[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint32_t u = (uint32_t)pr[k], v = (uint32_t)(pr[k] >> 32);
      const bool ok = v != kNoPtr;
      wu[k] = ok ? bits[u >> 5] : 0xffffffffu;
      wv[k] = ok ? bits[v >> 5] : 0u;
    }
    // phase 3: classify; frontier members take their pointer from the key cache when it decides
    // it (-> the decided list), else fetch their row range (-> a degree bin)
    uint32_t frm = 0;
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint32_t u = (uint32_t)pr[k], v = (uint32_t)(pr[k] >> 32);
      const bool live = !((wu[k] >> (u & 31)) & 1u);
      const bool tgt = (wv[k] >> (v & 31)) & 1u;
      if (live && !tgt) sbits |= 1u << k;
      if (live && tgt) frm |= 1u << k;
    }
    if (KC) {
#pragma unroll
      for (int k = 0; k < K; ++k) {
        if (!(frm & (1u << k))) continue;
        const uint32_t u = (uint32_t)pr[k];
        uint64_t key;
        if (kc_decide(io.kc, bits, (int64_t)u - vbase, &key)) {
          frm &= ~(1u << k);
          fb[kDecided] |= 1u << k;
          pr[k] = make_pair(u, key ? (uint32_t)key : kNoPtr);
          io.best_w[(int64_t)u - vbase] = key;
        }
      }
    }
    int64_t os[K], oe[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint32_t u = (uint32_t)pr[k];
      const bool fr = (frm >> k) & 1u;
      os[k] = fr ? offs[u - vbase] : 0;
      oe[k] = fr ? offs[u - vbase + 1] : -1;
      if (lcnt && fr) {  // A7: a row pruned earlier in this run is scanned over its live prefix
        const uint32_t x = lcnt[u - vbase];
        if ((x >> 16) == tag) oe[k] = os[k] + (int64_t)(x & 0xffffu);
      }
    }
#pragma unroll
    for (int k = 0; k < K; ++k) {
      if (oe[k] >= 0) {
        const int64_t d = oe[k] - os[k];
        const int b = bin_of(d);
        const uint32_t m = 1u << k;
#pragma unroll
        for (int q = 0; q < kDegBins; ++q) fb[q] |= b == q ? m : 0u;
        rr[k] = (uint64_t)os[k] | ((uint64_t)(d < (int64_t)kBigDeg ? d : (int64_t)kBigDeg) << 40);
        degsum += (unsigned long long)d;
      }
    }
    // without the key cache the decided list stays empty: only the degree bins are written
    constexpr int NOUT = KC ? kBins : kDegBins;
    if (KC) decided += (unsigned long long)__popc(fb[kDecided]);
    // reserve output ranges: warp totals -> block prefix -> ONE atomic per list per block
    {
      const unsigned ts = __reduce_add_sync(0xffffffffu, __popc(sbits));
      if (lane == 0) wtot[warp][0] = ts;
#pragma unroll
      for (int q = 0; q < NOUT; ++q) {
        const unsigned tq = __reduce_add_sync(0xffffffffu, __popc(fb[q]));
        if (lane == 0) wtot[warp][1 + q] = tq;
      }
    }
    __syncthreads();
    if (threadIdx.x < 1 + NOUT) {
      const int q = threadIdx.x;
      unsigned long long tot = 0;
      for (int w = 0; w < NW; ++w) tot += wtot[w][q];
      unsigned long long base = 0;
      if (tot) base = atomicAdd(q == 0 ? cntSout : &cntFout[q - 1], tot);
      for (int w = 0; w < NW; ++w) { wbase[w][q] = base; base += wtot[w][q]; }
    }
    __syncthreads();
    unsigned long long bs = wbase[warp][0], bf[kBins];
#pragma unroll
    for (int q = 0; q < NOUT; ++q) bf[q] = wbase[warp][1 + q];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint32_t m = 1u << k;
      const bool ps = sbits & m;
      const unsigned bls = __ballot_sync(0xffffffffu, ps);
      if (ps) Sout[bs + __popc(bls & lt)] = pr[k];
      bs += __popc(bls);
      const ulonglong2 ent = make_ulonglong2(pr[k], rr[k]);
#pragma unroll
      for (int q = 0; q < NOUT; ++q) {
        const unsigned bb = __ballot_sync(0xffffffffu, (fb[q] & m) != 0);
        if (fb[q] & m) Fout.list[q].put(bf[q] + __popc(bb & lt), ent);
        bf[q] += __popc(bb);
      }
    }
  }
  for (int o = 16; o; o >>= 1) {
    degsum += __shfl_xor_sync(0xffffffffu, degsum, o);
    decided += __shfl_xor_sync(0xffffffffu, decided, o);
  }
  if (lane == 0 && degsum) atomicAdd(swept, degsum);
  if (lane == 0 && decided) atomicAdd(swept + (kCntCache - kCntSwept), decided);
}
template <bool ALL, int K, bool KC = false>
#ifndef LM_COMPACT_MINB
#define LM_COMPACT_MINB 3  // 85-register cap: 36% -> ~50% occupancy, no spills (round-1 compaction -30%)
#endif
__global__ void __launch_bounds__(256, LM_COMPACT_MINB)
    k_compact(CompactIO io, int64_t n, const uint64_t* __restrict__ best,
              const uint32_t* __restrict__ bits, const int64_t* __restrict__ offs, int64_t vbase) {
  compact_body<ALL, K, KC>(io, n, best, bits, offs, vbase, blockIdx.x, gridDim.x);
}

// =============================================================================================
// Round bookkeeping on the device (termination; R6)
// =============================================================================================
__global__ void k_round_init(RoundState* st, long long max_rounds, long long log_cap,
                             long long first_rounds) {
  st->cur = 1;  // round 1's compaction (ALL) writes set 0 = cur ^ 1
  st->cont = 0;
  st->rounds = first_rounds;
  st->max_rounds = max_rounds;
  st->ftot = 0;
  st->log_len = 0;
  st->log_cap = log_cap;
  st->swept_prev = 0;
  st->tag = st->tag >= 0xffffu ? 1u : st->tag + 1u;
  st->push = 0;
}
// After a compaction: the output set becomes current; decide whether another round runs.
// `graph_handle` != 0: running inside a CUDA graph -> set the WHILE node's condition.
#ifndef LM_PUSH_RATIO
#define LM_PUSH_RATIO 8
#endif
constexpr unsigned long long kPushRatio = LM_PUSH_RATIO;
// ... and only once the live list is long enough for its per-round pass to cost more than the
// push step's fixed work (gradient meshes: pull wins at 1024^2 -- 45 vs 57 ms -- push at 2048^2
// and 4096^2 -- 123 vs 135 ms, 222 vs 720 ms)
#ifndef LM_PUSH_MIN_LIVE
#define LM_PUSH_MIN_LIVE (1ull << 20)
#endif
constexpr unsigned long long kPushMinLive = LM_PUSH_MIN_LIVE;
__device__ __forceinline__ int end_round_body(const RoundArgs* __restrict__ ra, long long first_log_rows,
                                              bool push_ok = false) {
  RoundState* st = ra->st;
  const int cur = st->cur ^ 1;
  st->cur = cur;
  unsigned long long nF = 0;
#pragma unroll
  for (int b = 0; b < kBins; ++b) nF += ra->cnt[cnt_F(cur, b)];
  const unsigned long long nS = ra->cnt[cnt_S(cur)];
  const int cont = nF > 0 && st->rounds < st->max_rounds;
  // A6: once the live list is much longer than the frontier (many-round graphs), the next
  // frontier is pushed from the newly matched vertices instead of pulled from the live list
  // (only the persistent kernel runs push rounds; it passes push_ok)
  if (push_ok && ra->N && !st->push && nS + nF > kPushRatio * nF && nS + nF >= ra->push_min_live)
    st->push = 1;
  ra->cnt[kCntN] = 0ull;
  // zero the counters of the set the next compaction writes
#pragma unroll
  for (int q = 0; q < 1 + kBins; ++q) ra->cnt[cnt_S(cur ^ 1) + q] = 0ull;
  if (cont) {
    ++st->rounds;
    st->ftot += (long long)nF;
    const unsigned long long sw = ra->cnt[kCntSwept];
    if (st->log_len < st->log_cap) {
      long long* row = ra->log + 3 * (first_log_rows + st->log_len);
      row[0] = (long long)nF;
      row[1] = (long long)(nS + nF);
      row[2] = (long long)(sw - st->swept_prev);
      ++st->log_len;
    }
    st->swept_prev = sw;
  }
  st->cont = cont;
  return cont;
}
__global__ void k_end_round(const RoundArgs* __restrict__ ra, cudaGraphConditionalHandle handle, int in_graph,
                            long long first_log_rows) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  const int cont = end_round_body(ra, first_log_rows);
  if (in_graph) cudaGraphSetConditional(handle, (unsigned)cont);
}

// ---- A6 push-style frontier (SURVEY 8(a) A6 "push alternative"; not in the paper, whose Alg. 3
// rescans every unmatched vertex).  The pull compaction reads the whole live list every
// round, O(|L| x rounds): quadratic on many-round graphs (a weight gradient along paths).  In a
// push round the match records the vertices it newly matched (N_r, deduplicated by the atomicOr's
// old value), and the next frontier is built from their rows: u joins F_{r+1} iff u is unmatched
// and its pointer is a vertex of N_r -- exactly the pull rule, since a live u's target was
// unmatched when the round began.  Each vertex is matched once, so the whole run pushes O(m)
// entries.  A frontier vertex is claimed by a CAS of its pointer to 0 (its pointer is recomputed
// next round anyway), so repeated (u,v) entries cannot list it twice.
__device__ __forceinline__ void match_push_body(const Bins& F, const unsigned long long* cntF,
                                                const uint64_t* __restrict__ best, uint32_t* bits,
                                                uint32_t* N, unsigned long long* cntN, int64_t tid,
                                                int64_t stride) {
  const int lane = threadIdx.x & 31;
#pragma unroll 1
  for (int bb = 0; bb < kBins; ++bb) {
    const int64_t c = (int64_t)cntF[bb];
    for (int64_t i0 = tid - lane; i0 < c; i0 += stride) {  // warp-uniform trip count
      const int64_t i = i0 + lane;
      const uint64_t p = i < c ? F.list[bb].p[i] : ((uint64_t)kNoPtr << 32);
      const uint32_t u = (uint32_t)p, v = (uint32_t)(p >> 32);
      bool nu = false, nv = false;
      if (v != kNoPtr) {
        const uint64_t kv = best[v];
        if (kv != 0 && (uint32_t)kv == u) {
          const uint32_t mu = 1u << (u & 31), mv = 1u << (v & 31);
          nu = !(atomicOr(&bits[u >> 5], mu) & mu);
          nv = !(atomicOr(&bits[v >> 5], mv) & mv);
        }
      }
      warp_append(nu, (int32_t)u, reinterpret_cast<int32_t*>(N), cntN);
      warp_append(nv, (int32_t)v, reinterpret_cast<int32_t*>(N), cntN);
    }
  }
}
// F_{r+1} from the rows of N_r (a lane per newly matched vertex; its row is short on the graphs
// that reach push mode); appends into the degree bins of the output set
__device__ __forceinline__ void push_body(const uint32_t* __restrict__ N, int64_t nN,
                                          const int64_t* __restrict__ offs, const AdjView adj,
                                          const uint32_t* __restrict__ bits, uint64_t* best,
                                          const Bins& Fout, unsigned long long* cntFout,
                                          unsigned long long* swept, int64_t vbase, int64_t tid,
                                          int64_t stride) {
  unsigned long long degsum = 0;
  for (int64_t i = tid; i < nN; i += stride) {
    const uint32_t v = N[i];
    const int64_t lv = (int64_t)v - vbase;
    for (int64_t j = offs[lv], e = offs[lv + 1]; j < e; ++j) {
      const uint64_t k = adj.at(j);
      const uint32_t u = (uint32_t)k;
      if (k == 0 || bit_test(bits, u)) continue;
      const int64_t lu = (int64_t)u - vbase;
      const uint64_t bu = *reinterpret_cast<volatile const uint64_t*>(best + lu);
      if (bu == 0 || (uint32_t)bu != v) continue;
      if (atomicCAS(reinterpret_cast<unsigned long long*>(best + lu), (unsigned long long)bu, 0ull) != bu)
        continue;
      const int64_t os = offs[lu], d = offs[lu + 1] - os;
      const int b = bin_of(d);
      const unsigned long long pos = atomicAdd(&cntFout[b], 1ull);
      Fout.list[b].put(pos, make_ulonglong2(make_pair(u, v),
                                            (uint64_t)os | ((uint64_t)(d < (int64_t)kBigDeg ? d : (int64_t)kBigDeg) << 40)));
      degsum += (unsigned long long)d;
    }
  }
  for (int o = 16; o; o >>= 1) degsum += __shfl_xor_sync(0xffffffffu, degsum, o);
  if ((threadIdx.x & 31) == 0 && degsum) atomicAdd(swept, degsum);
}

// All rounds >= 2 in ONE cooperative launch (grid = co-resident blocks): pointer phase (every
// degree bin) | grid barrier | match | barrier | compaction | barrier | end of round | barrier.
// No per-round launches or host decisions; the grid barrier's fence also invalidates L1, so
// every phase reads the others' writes.
template <int B0G, int B0U, int B1G, int B1U, int B2G, int B2U, int K, bool PRUNE = false, bool KC = false>
__global__ void __launch_bounds__(256)
    k_rounds_persistent(const RoundArgs* __restrict__ ra, const int64_t* __restrict__ offs, const AdjView adj,
                        uint32_t* bits, uint64_t* best, int64_t n, int64_t vbase) {
  cg::grid_group grid = cg::this_grid();
  const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t gthreads = (int64_t)gridDim.x * blockDim.x;
  for (;;) {
    if (!*reinterpret_cast<volatile int*>(&ra->st->cont)) break;  // uniform after the barrier
    const int cur = *reinterpret_cast<volatile int*>(&ra->st->cur);
    {
      const Bins F = ra->F[cur];
      const unsigned long long* c = ra->cnt + cnt_F(cur, 0);
      const uint32_t tag = PRUNE ? round_tag(ra->st) : 0u;
      point_bin_body<B0G, B0U, PRUNE>(F.list[0], (int64_t)c[0], offs, adj, bits, best, vbase, gtid,
                                      gthreads, ra->live, tag);
      point_bin_body<B1G, B1U, PRUNE>(F.list[1], (int64_t)c[1], offs, adj, bits, best, vbase, gtid,
                                      gthreads, ra->live, tag);
      point_bin_body<B2G, B2U, PRUNE>(F.list[2], (int64_t)c[2], offs, adj, bits, best, vbase, gtid,
                                      gthreads, ra->live, tag);
      point_bin_cta_body<256, 4>(F.list[3], (int64_t)c[3], offs, adj, bits, best, vbase, blockIdx.x,
                                 gridDim.x);
    }
    grid.sync();
    const bool push = *reinterpret_cast<volatile uint32_t*>(&ra->st->push) != 0u;
    if (push)
      match_push_body(ra->F[cur], ra->cnt + cnt_F(cur, 0), best, bits, ra->N, ra->cnt + kCntN, gtid, gthreads);
    else
      match_bins_body(ra->F[cur], ra->cnt + cnt_F(cur, 0), best, bits, gtid, gthreads);
    grid.sync();
    if (push) {
      push_body(ra->N, (int64_t)*reinterpret_cast<volatile unsigned long long*>(ra->cnt + kCntN), offs, adj,
                bits, best, ra->F[cur ^ 1], ra->cnt + cnt_F(cur ^ 1, 0), ra->cnt + kCntSwept, vbase, gtid,
                gthreads);
    } else {
      const CompactIO io = compact_io(*ra, cur);
      compact_body<false, K, KC>(io, n, best, bits, offs, vbase, blockIdx.x, gridDim.x);
    }
    grid.sync();
    if (gtid == 0) {
      if (push) ++ra->cnt[kCntPushRounds];
      end_round_body(ra, 0, !PRUNE);
    }
    grid.sync();
  }
}
__global__ void k_set_cur(RoundState* st, int cur) {
  if (threadIdx.x == 0 && blockIdx.x == 0) st->cur = cur;
}

// =============================================================================================
// Partitioned mode (A3/A5): this rank owns rows [vbase, vend) of a 1-D vertex
// partition; the matched bitmap is replicated; ghost[x] holds, for a remote vertex x,
// the owned vertex x last claimed to point to.  A pointer into u moves off u only after u is
// matched, so a stale ghost is never consulted while u is live (extends Lemma III.1).
// Claims (v | u << 32): "u points to v", sent to owner(v) instead of the paper's
// |V| x 64-bit nccl_AllReduce(pointers) (Alg. 2 L7).
// =============================================================================================
__device__ __forceinline__ int owner_of(const int64_t* __restrict__ bounds, int P, uint32_t v) {
  int lo = 0, hi = P - 1;  // last p with bounds[p] <= v
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (bounds[mid] <= (int64_t)v) lo = mid; else hi = mid - 1;
  }
  return lo;
}
__device__ __forceinline__ uint32_t ptr_of(const uint64_t* __restrict__ best,
                                           const uint32_t* __restrict__ ghost, int64_t vbase,
                                           int64_t vend, uint32_t v) {
  if ((int64_t)v >= vbase && (int64_t)v < vend) {
    const uint64_t k = best[v - vbase];
    return k ? (uint32_t)k : kNoPtr;
  }
  return ghost[v];
}
struct Claims {
  uint64_t* seg;               // P segments of `cap` claims each
  int64_t cap;
  unsigned long long* count;   // [P]
  const int64_t* bounds;       // [P+1]
  int P;
  // peer-memory exchange (lmatch_p2p_*): claims for part d are stored straight into d's inbox
  // segment for this part (dseg[d]) and counted there (dcnt[d]); NULL = local segments above
  uint64_t* const* dseg = nullptr;
  unsigned long long* const* dcnt = nullptr;
};
// warp-collective (all 32 lanes call it): lanes with the same destination share one atomic
__device__ __forceinline__ void claim_append(const Claims& C, bool pred, uint32_t v, uint32_t u) {
  const int d = pred ? owner_of(C.bounds, C.P, v) : -1;
  const unsigned peers = __match_any_sync(0xffffffffu, d);
  if (!pred) return;
  const int lane = threadIdx.x & 31, leader = __ffs(peers) - 1;
  unsigned long long* cnt = C.dcnt ? C.dcnt[d] : &C.count[d];
  uint64_t* seg = C.dseg ? C.dseg[d] : C.seg + (int64_t)d * C.cap;
  unsigned long long base = 0;
  if (lane == leader) base = atomicAdd_system(cnt, (unsigned long long)__popc(peers));
  base = __shfl_sync(peers, base, leader);
  seg[(int64_t)(base + __popc(peers & lanemask_lt()))] = make_pair(v, u);
}
// round 1: every owned vertex whose pointer targets a remote vertex
__global__ void k_claims_all(const uint64_t* __restrict__ best, int64_t n_loc, int64_t vbase,
                             int64_t vend, Claims C) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t n32 = (n_loc + 31) & ~31ll;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n32; i += stride) {
    const uint64_t b = i < n_loc ? best[i] : 0ull;
    const uint32_t v = (uint32_t)b;
    claim_append(C, b != 0 && ((int64_t)v < vbase || (int64_t)v >= vend), v, (uint32_t)(i + vbase));
  }
}
// rounds >= 2: the re-pointed frontier
__global__ void k_claims_bins(Bins F, const unsigned long long* cntF, int64_t vbase, int64_t vend,
                              Claims C) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll
  for (int bb = 0; bb < kBins; ++bb) {
    const int64_t c = (int64_t)cntF[bb];
    const int64_t c32 = (c + 31) & ~31ll;
    for (int64_t i = tid; i < c32; i += stride) {
      const uint64_t p = i < c ? F.list[bb].p[i] : ((uint64_t)kNoPtr << 32);
      const uint32_t u = (uint32_t)p, v = (uint32_t)(p >> 32);
      claim_append(C, v != kNoPtr && ((int64_t)v < vbase || (int64_t)v >= vend), v, u);
    }
  }
}
// received claims (v owned, u remote): record the ghost pointer
__global__ void k_apply_claims(const uint64_t* __restrict__ recv, int64_t nrecv, uint32_t* ghost) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nrecv; i += stride) {
    const uint64_t c = recv[i];
    ghost[(uint32_t)(c >> 32)] = (uint32_t)c;
  }
}
// ... and match them: v (owned) with u (remote) iff ptr v == u
__global__ void k_match_claims(const uint64_t* __restrict__ recv, int64_t nrecv,
                               const uint64_t* __restrict__ best, int64_t vbase, uint32_t* bits) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nrecv; i += stride) {
    const uint64_t c = recv[i];
    const uint32_t v = (uint32_t)c, u = (uint32_t)(c >> 32);
    const uint64_t kv = best[v - vbase];
    if (kv != 0 && (uint32_t)kv == u) atomicOr(&bits[v >> 5], 1u << (v & 31));
  }
}
// ---- peer-memory exchange (lmatch_p2p_*): the inbox holds P segments of `cap` claims, segment
// s written by part s over NVLink / peer memory, with its count in cnt[s] (device-resident, so
// no host round trip decides the grid: the kernels walk every segment).
__global__ void k_apply_inbox(const uint64_t* __restrict__ inbox, int64_t cap,
                              const unsigned long long* __restrict__ cnt, int P, uint32_t* ghost) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int s = 0; s < P; ++s) {
    const int64_t c = (int64_t)cnt[s];
    const uint64_t* seg = inbox + (int64_t)s * cap;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < c; i += stride) {
      const uint64_t x = seg[i];
      ghost[(uint32_t)(x >> 32)] = (uint32_t)x;
    }
  }
}
__global__ void k_match_inbox(const uint64_t* __restrict__ inbox, int64_t cap,
                              unsigned long long* cnt, int P, const uint64_t* __restrict__ best,
                              int64_t vbase, uint32_t* bits) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int s = 0; s < P; ++s) {
    const int64_t c = (int64_t)cnt[s];
    const uint64_t* seg = inbox + (int64_t)s * cap;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < c; i += stride) {
      const uint64_t x = seg[i];
      const uint32_t v = (uint32_t)x, u = (uint32_t)(x >> 32);
      const uint64_t kv = best[v - vbase];
      if (kv != 0 && (uint32_t)kv == u) atomicOr(&bits[v >> 5], 1u << (v & 31));
    }
  }
}
// Push the owned bitmap words that changed since the last push into every peer's replica
// (plain 4-byte stores into peer memory; one owner per word, so no atomics).  Replaces the
// bitmap allgather (nccl_AllReduce(mate), Alg. 2 L9) with n/8 bytes per round at most.
__global__ void k_push_bits(const uint32_t* __restrict__ bits, uint32_t* __restrict__ shadow,
                            int64_t w0, int64_t nw, uint32_t* const* __restrict__ peer_bits,
                            int P, int me) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nw; i += stride) {
    const uint32_t x = bits[w0 + i];
    if (x == shadow[i]) continue;
    shadow[i] = x;
    for (int p = 0; p < P; ++p)
      if (p != me) peer_bits[p][w0 + i] = x;
  }
}
// frontier-size exchange for termination: this part's count into every peer's slot [me]
__global__ void k_push_count(const unsigned long long* __restrict__ cnt, int ncnt,
                             unsigned long long* const* __restrict__ peer_slot, int P) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    unsigned long long t = 0;
    for (int i = 0; i < ncnt; ++i) t += cnt[i];
    for (int p = 0; p < P; ++p) peer_slot[p][0] = t;
  }
}

// ---- library-owned multi-GPU driver (lmatch_create_dist / lmatch_run_dist): a device-side
// barrier over the exchange windows, so no host barrier separates the phases of a round.
// Part `me` stores the barrier's epoch into slot [me] of every peer's flag array with a
// system-scope release (after a system-scope fence: the claims and bitmap words this GPU stored
// into peer memory before the barrier are visible to the peer when it sees the flag), then
// waits until every peer's epoch has arrived in its own array (system-scope acquire).  One
// thread; a peer missing for `timeout_ns` sets *err and returns (the host reports ENCCL) instead
// of hanging the GPU.
__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long global_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__global__ void k_dist_barrier(const unsigned long long* my_flags,
                               unsigned long long* const* __restrict__ peer_flag, int P, int me,
                               unsigned long long epoch, unsigned long long timeout_ns,
                               unsigned* err) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  __threadfence_system();
  for (int p = 0; p < P; ++p)
    if (p != me) st_release_sys(peer_flag[p], epoch);
  const unsigned long long t0 = global_ns();
  for (int q = 0; q < P; ++q) {
    if (q == me) continue;
    while (ld_acquire_sys(my_flags + q) < epoch) {
      if (global_ns() - t0 > timeout_ns) {
        atomicOr(err, 1u);
        return;
      }
      __nanosleep(256);
    }
  }
}
// this part's w(M) share and matched count into every part's result slots [me] (fp64 bits), so
// each part sums the P shares in part order after a barrier (same total on every part)
__global__ void k_push_result(const double* __restrict__ w, const long long* __restrict__ c,
                              unsigned long long* const* __restrict__ peer_w,
                              unsigned long long* const* __restrict__ peer_c, int P) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  const unsigned long long wb = (unsigned long long)__double_as_longlong(*w);
  const unsigned long long cb = (unsigned long long)*c;
  for (int p = 0; p < P; ++p) {
    peer_w[p][0] = wb;
    peer_c[p][0] = cb;
  }
}

// round 1 match over every owned vertex (owned range starts on a 32-vertex boundary)
__global__ void k_match_part_all(const uint64_t* __restrict__ best, int64_t n_loc, int64_t vbase,
                                 int64_t vend, const uint32_t* __restrict__ ghost, uint32_t* bits) {
  const int64_t nwords = (n_loc + 31) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t ws = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t wi = w0; wi < nwords; wi += ws) {
    const int64_t i = (wi << 5) + lane;
    bool mutual = false;
#if LM_MATCHALL_HALF
    // as k_match_all: a pair with both ends in this part is checked from its smaller end, which
    // marks both (atomicOr; the owned words were zeroed by k_reset); a remote target is checked
    // here, its own part marks it
    uint32_t v = 0;
    if (i < n_loc) {
      const uint64_t b = best[i];
      v = (uint32_t)b;
      const bool local = (int64_t)v >= vbase && (int64_t)v < vend;
      if (b && (!local || (int64_t)v > i + vbase))
        mutual = ptr_of(best, ghost, vbase, vend, v) == (uint32_t)(i + vbase);
    }
    const unsigned word = __ballot_sync(0xffffffffu, mutual);
    if (lane == 0 && word) atomicOr(&bits[(vbase >> 5) + wi], word);
    if (mutual && (int64_t)v >= vbase && (int64_t)v < vend) atomicOr(&bits[v >> 5], 1u << (v & 31));
#else
    if (i < n_loc) {
      const uint64_t b = best[i];
      if (b) mutual = ptr_of(best, ghost, vbase, vend, (uint32_t)b) == (uint32_t)(i + vbase);
    }
    const unsigned word = __ballot_sync(0xffffffffu, mutual);
    if (lane == 0) bits[(vbase >> 5) + wi] = word;
#endif
  }
}
// rounds >= 2 match over the re-pointed frontier
__global__ void k_match_part_bins(Bins F, const unsigned long long* cntF,
                                  const uint64_t* __restrict__ best, int64_t vbase, int64_t vend,
                                  const uint32_t* __restrict__ ghost, uint32_t* bits) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  // LM_MATCH_V entries per thread step with their dependent loads batched, as match_bins_body
  constexpr int V = LM_MATCH_V;
#pragma unroll
  for (int bb = 0; bb < kBins; ++bb) {
    const int64_t c = (int64_t)cntF[bb];
    for (int64_t i0 = tid; i0 < c; i0 += V * stride) {
      uint64_t p[V];
      uint32_t pv[V];
#pragma unroll
      for (int q = 0; q < V; ++q) {
        const int64_t i = i0 + q * stride;
        p[q] = i < c ? F.list[bb].p[i] : ((uint64_t)kNoPtr << 32);
      }
#pragma unroll
      for (int q = 0; q < V; ++q) {
        const uint32_t v = (uint32_t)(p[q] >> 32);
        pv[q] = v != kNoPtr ? ptr_of(best, ghost, vbase, vend, v) : kNoPtr;
      }
#pragma unroll
      for (int q = 0; q < V; ++q) {
        const uint32_t u = (uint32_t)p[q], v = (uint32_t)(p[q] >> 32);
        if (v != kNoPtr && pv[q] == u) {
          atomicOr(&bits[u >> 5], 1u << (u & 31));
          if ((int64_t)v >= vbase && (int64_t)v < vend) atomicOr(&bits[v >> 5], 1u << (v & 31));
        }
      }
    }
  }
}

// =============================================================================================
// A10/A9: mate[] materialisation + deterministic fp64 weight / cardinality partial sums
// =============================================================================================
template <int THREADS>
__device__ __forceinline__ void block_sum2(double w, long long c, double* outw, long long* outc) {
  __shared__ double sw[THREADS / 32];
  __shared__ long long sc[THREADS / 32];
  for (int o = 16; o; o >>= 1) {
    w += __shfl_xor_sync(0xffffffffu, w, o);
    c += __shfl_xor_sync(0xffffffffu, c, o);
  }
  if ((threadIdx.x & 31) == 0) { sw[threadIdx.x >> 5] = w; sc[threadIdx.x >> 5] = c; }
  __syncthreads();
  if (threadIdx.x == 0) {
    double tw = 0; long long tc = 0;
    for (int i = 0; i < THREADS / 32; ++i) { tw += sw[i]; tc += sc[i]; }
    *outw = tw; *outc = tc;
  }
}

template <int THREADS>
__global__ void __launch_bounds__(THREADS)
    k_materialize(const uint64_t* __restrict__ best, const uint32_t* __restrict__ bits, int64_t n,
                  int64_t vbase, int32_t* __restrict__ mate, double* pw, long long* pc) {
  // 4 vertices per thread per step with their loads issued together (the per-vertex chain
  // bitmap word -> best[] is latency-bound otherwise); fixed assignment => fixed fp64 order
  constexpr int V = 4;
  double w = 0.0;
  long long c = 0;
  const int64_t stride = (int64_t)gridDim.x * THREADS;
  for (int64_t i0 = (int64_t)blockIdx.x * THREADS + threadIdx.x; i0 < n; i0 += V * stride) {
    uint32_t wd[V];
#pragma unroll
    for (int q = 0; q < V; ++q) {
      const int64_t i = i0 + q * stride;
      wd[q] = i < n ? bits[(uint32_t)(i + vbase) >> 5] : 0u;
    }
    uint64_t k[V];
#pragma unroll
    for (int q = 0; q < V; ++q) {
      const int64_t i = i0 + q * stride;
      const bool mt = i < n && ((wd[q] >> ((uint32_t)(i + vbase) & 31)) & 1u);
      k[q] = mt ? best[i] : ~0ull;
    }
#pragma unroll
    for (int q = 0; q < V; ++q) {
      const int64_t i = i0 + q * stride;
      if (i >= n) break;
      int32_t v = -1;
      if (k[q] != ~0ull) {
        v = (int32_t)(uint32_t)k[q];
        ++c;
        if ((int64_t)v > i + vbase) w += (double)__uint_as_float((uint32_t)(k[q] >> 32));
      }
      mate[i] = v;
    }
  }
  block_sum2<THREADS>(w, c, &pw[blockIdx.x], &pc[blockIdx.x]);
}

// w(M) for an arbitrary mate[]: 8 lanes per vertex search row u for mate[u] (first match).
// err: bit0 = mate out of range / self, bit1 = asymmetric, bit2 = pair not an edge.
template <int THREADS>
__global__ void __launch_bounds__(THREADS)
    k_weight_any(const int32_t* __restrict__ mate, int64_t n, const int64_t* __restrict__ offs,
                 const AdjView adj, double* pw, long long* pc, unsigned* err) {
  const int lane = threadIdx.x & 31, g8 = lane & 7;
  const unsigned gmask = 0xffu << (lane & ~7);
  double w = 0.0;
  long long c = 0;
  const int64_t ng = ((int64_t)gridDim.x * THREADS) >> 3;
  for (int64_t u = ((int64_t)blockIdx.x * THREADS + threadIdx.x) >> 3; u < n; u += ng) {
    const int32_t v = mate[u];
    if (v == -1) continue;
    if (v < -1 || (int64_t)v >= n || (int64_t)v == u) {
      if (g8 == 0) atomicOr(err, 1u);
      continue;
    }
    if (mate[v] != (int32_t)u) {
      if (g8 == 0) atomicOr(err, 2u);
      continue;
    }
    if ((int64_t)v < u) continue;
    uint64_t found = 0;
    for (int64_t j = offs[u] + g8; j < offs[u + 1]; j += 8) {
      const uint64_t k = adj.at(j);
      if (k != 0 && (uint32_t)k == (uint32_t)v) found = k;
    }
    found = group_max_key(found, gmask);
    if (g8 == 0) {
      if (!found) atomicOr(err, 4u);
      else { w += (double)__uint_as_float((uint32_t)(found >> 32)); ++c; }
    }
  }
  block_sum2<THREADS>(w, c, &pw[blockIdx.x], &pc[blockIdx.x]);
}

// Fixed-order (deterministic) sum of the per-block partials: lane l adds partials l, l+32, ...
// in index order, then a fixed butterfly.  Launch <<<1, 32>>>.
__global__ void k_final_sum(const double* pw, const long long* pc, int nb, double* out_w,
                            long long* out_c) {
  const int lane = threadIdx.x & 31;
  double w = 0;
  long long c = 0;
  if (threadIdx.x < 32) {
    for (int i = lane; i < nb; i += 32) { w += pw[i]; c += pc[i]; }
    for (int o = 16; o; o >>= 1) {
      w += __shfl_xor_sync(0xffffffffu, w, o);
      c += __shfl_xor_sync(0xffffffffu, c, o);
    }
    if (lane == 0) { *out_w = w; *out_c = c; }
  }
}

// =============================================================================================
// NEXT-1: out-of-core host-row key cache.  Every row with entries beyond the
// resident prefix ("host row", u >= u_first) keeps its K largest keys in HBM, descending,
// zero-padded.  They are filled in round 1 from the streamed chunks (the round is PCIe-bound,
// so the extra pass over the chunk already in the device ring is free) and used by later rounds:
// if a cached key's neighbour is unmatched, the FIRST such key is the row's maximum available
// key (every larger key of the row is cached and unavailable; available sets only shrink,
// R3), so the frontier entry is redirected to that one cached slot and the host row is not read.
// A row with degree <= K is cached whole, so "no cached key available" means no pointer.  Only
// rows with degree > K whose K cached neighbours are all matched are read zero-copy.
// =============================================================================================
constexpr int kCacheK = 8;

// last row u with offs[u] <= j (the row holding entry j, for 0 <= j < offs[n])
__device__ __forceinline__ int64_t row_of_entry(const int64_t* __restrict__ offs, int64_t n, int64_t j) {
  int64_t lo = 0, hi = n;  // offs[lo] <= j < offs[hi]
  while (hi - lo > 1) {
    const int64_t mid = lo + ((hi - lo) >> 1);
    if (offs[mid] <= j) lo = mid; else hi = mid;
  }
  return lo;
}
// out[k] = row holding entry min(first + k * step, last) for k in [0, cnt)
__global__ void k_rows_of_entries(const int64_t* __restrict__ offs, int64_t n, int64_t first,
                                  int64_t step, int64_t last, int64_t cnt, int64_t* out) {
  const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k < cnt) out[k] = row_of_entry(offs, n, min(first + k * step, last));
}

// Fill / merge the cache of rows [*plo, *phi] from entries [w0, w1) held at base[j - ebase].
// A row starting inside the window overwrites its slots; a row that started before it (spans a
// chunk boundary or the resident/streamed split) merges with the slots written earlier on the
// same stream.  Each warp takes 32 consecutive rows: a row with <= 16 in-window entries is
// reduced by its own lane (register top-K), a longer one by the whole warp (per-lane top-K, then
// K warp-wide pops), and a row with more than kCacheBigRow entries is listed for
// k_cache_fill_big (one CTA per row).
constexpr int64_t kCacheBigRow = 4096;
template <int K>
__device__ __forceinline__ void cache_row_warp(const uint64_t* __restrict__ base, int64_t ebase,
                                               int64_t a, int64_t b, bool merge,
                                               uint64_t* __restrict__ c) {
  const int lane = threadIdx.x & 31;
  uint64_t t[K];
#pragma unroll
  for (int i = 0; i < K; ++i) t[i] = 0ull;
  for (int64_t j = a + lane; j < b; j += 32) topk_insert<K>(t, base[j - ebase]);
  if (merge && lane < K) topk_insert<K>(t, c[lane]);
  const uint64_t mine = warp_topk_pop<K>(t);
  if (lane < K) c[lane] = mine;
}
template <int K>
__global__ void __launch_bounds__(256) k_cache_fill(const uint64_t* __restrict__ base, int64_t ebase,
                                                    int64_t w0, int64_t w1,
                                                    const int64_t* __restrict__ offs,
                                                    const int64_t* __restrict__ plo,
                                                    const int64_t* __restrict__ phi, int64_t u_first,
                                                    uint64_t* __restrict__ cache,
                                                    int64_t* __restrict__ big,
                                                    unsigned long long* __restrict__ nbig) {
  const int lane = threadIdx.x & 31;
  const int64_t ulo = *plo, uhi = *phi;
  const int64_t nrows = uhi - ulo + 1;
  const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r0 = wid * 32; r0 < nrows; r0 += nw * 32) {
    const int64_t u = ulo + r0 + lane;
    int64_t s = 0, a = 0, b = 0;
    if (u <= uhi) {
      s = offs[u];
      a = max(s, w0);
      b = min(offs[u + 1], w1);
    }
    const int64_t len = b > a ? b - a : 0;
    uint64_t* c = cache + (u - u_first) * K;
    if (len > 0 && len <= 16) {
      uint64_t t[K];
#pragma unroll
      for (int i = 0; i < K; ++i) t[i] = 0ull;
      for (int64_t j = a; j < b; ++j) topk_insert<K>(t, base[j - ebase]);
      if (s < w0) {
#pragma unroll
        for (int i = 0; i < K; ++i) topk_insert<K>(t, c[i]);
      }
      ulonglong2* c2 = reinterpret_cast<ulonglong2*>(c);
#pragma unroll
      for (int i = 0; i < K / 2; ++i) c2[i] = make_ulonglong2(t[2 * i], t[2 * i + 1]);
    } else if (len > kCacheBigRow) {
      big[atomicAdd(nbig, 1ull)] = u;
    }
    unsigned mid = __ballot_sync(0xffffffffu, len > 16 && len <= kCacheBigRow);
    while (mid) {
      const int l = __ffs(mid) - 1;
      mid &= mid - 1;
      const int64_t ul = __shfl_sync(0xffffffffu, u, l);
      const int64_t al = __shfl_sync(0xffffffffu, a, l), bl = __shfl_sync(0xffffffffu, b, l);
      const int64_t sl = __shfl_sync(0xffffffffu, s, l);
      cache_row_warp<K>(base, ebase, al, bl, sl < w0, cache + (ul - u_first) * K);
    }
  }
}
// the listed long rows: one CTA per row (per-warp top-K, then warp 0 merges the 8 lists)
template <int K>
__global__ void __launch_bounds__(256) k_cache_fill_big(const uint64_t* __restrict__ base,
                                                        int64_t ebase, int64_t w0, int64_t w1,
                                                        const int64_t* __restrict__ offs,
                                                        const int64_t* __restrict__ big,
                                                        const unsigned long long* __restrict__ nbig,
                                                        int64_t u_first, uint64_t* __restrict__ cache) {
  __shared__ uint64_t cand[8][K];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t nb = (int64_t)*nbig;
  for (int64_t i = blockIdx.x; i < nb; i += gridDim.x) {
    const int64_t u = big[i];
    const int64_t s = offs[u];
    const int64_t a = max(s, w0), b = min(offs[u + 1], w1);
    uint64_t t[K];
#pragma unroll
    for (int q = 0; q < K; ++q) t[q] = 0ull;
    for (int64_t j = a + threadIdx.x; j < b; j += blockDim.x) topk_insert<K>(t, base[j - ebase]);
    uint64_t* c = cache + (u - u_first) * K;
    if (s < w0 && threadIdx.x < K) topk_insert<K>(t, c[threadIdx.x]);
    uint64_t mine = warp_topk_pop<K>(t);
    if (lane < K) cand[warp][lane] = mine;
    __syncthreads();
    if (warp == 0) {
#pragma unroll
      for (int q = 0; q < K; ++q) t[q] = 0ull;
      for (int q = lane; q < 8 * K; q += 32) topk_insert<K>(t, cand[q / K][q % K]);
      mine = warp_topk_pop<K>(t);
      if (lane < K) c[lane] = mine;
    }
    __syncthreads();
  }
}

// Rounds >= 2 (out-of-core): redirect frontier entries of host rows to the cache where it
// decides the pointer.  .y becomes (1 << 40 | M0 + slot) for the first available cached key, or
// an empty range when the whole row is cached and none is available; otherwise the entry keeps
// its host range (read zero-copy).  cnt[0] += rows served by the cache, cnt[1] += host entries
// left to the zero-copy path.
template <int K>
__global__ void k_cache_redirect(Bins F, const unsigned long long* __restrict__ cntF,
                                 const int64_t* __restrict__ offs, const uint64_t* __restrict__ cache,
                                 const uint32_t* __restrict__ bits, int64_t u_first, int64_t M0,
                                 int64_t vbase, unsigned long long* cnt,
                                 uint64_t* __restrict__ rescan = nullptr,
                                 unsigned long long* nrescan = nullptr,
                                 const int64_t* __restrict__ roff = nullptr, int64_t M2 = 0) {
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  unsigned long long served = 0, left = 0, resid = 0;
  for (int bb = 0; bb < kDegBins; ++bb) {
    const int64_t c = (int64_t)cntF[bb];
    for (int64_t i = tid; i < c; i += stride) {
      ulonglong2 e = F.list[bb][i];
      const int64_t u = (int64_t)(uint32_t)e.x - vbase;
      if (u < u_first) continue;
      int64_t s, en;
      row_range(e, offs, vbase, &s, &en);
      const int64_t slot = (u - u_first) * K;
      const ulonglong2* cp = reinterpret_cast<const ulonglong2*>(cache + slot);
      uint64_t k[K];
#pragma unroll
      for (int q = 0; q < K / 2; ++q) {
        const ulonglong2 x = __ldg(cp + q);
        k[2 * q] = x.x;
        k[2 * q + 1] = x.y;
      }
      uint32_t wd[K];
#pragma unroll
      for (int q = 0; q < K; ++q) wd[q] = k[q] ? bits[(uint32_t)k[q] >> 5] : 0xffffffffu;
      int hit = -1;
#pragma unroll
      for (int q = K - 1; q >= 0; --q)
        if (!((wd[q] >> ((uint32_t)k[q] & 31)) & 1u)) hit = q;
      if (hit >= 0) {
        e.y = (1ull << 40) | (uint64_t)(M0 + slot + hit);
      } else if (en - s <= K) {
        e.y = (uint64_t)(M0 + slot);
      } else if (roff && roff[u - u_first] >= 0) {
        // a residual row: its copy in HBM is scanned by the pointer kernels (no host read)
        const int64_t d = en - s;
        e.y = (uint64_t)(M2 + roff[u - u_first]) | ((uint64_t)(d < (int64_t)kBigDeg ? d : (int64_t)kBigDeg) << 40);
        F.list[bb].r[i] = e.y;
        ++resid;
        continue;
      } else {
        left += (unsigned long long)(en - s);
        // refill path: k_host_rescan reads the row once, refills the cache with its K largest
        // available keys and redirects this entry to the first of them
        if (rescan) rescan[atomicAdd(nrescan, 1ull)] = ((uint64_t)bb << 40) | (uint64_t)i;
        continue;
      }
      F.list[bb].r[i] = e.y;
      ++served;
    }
  }
  for (int o = 16; o; o >>= 1) {
    served += __shfl_xor_sync(0xffffffffu, served, o);
    left += __shfl_xor_sync(0xffffffffu, left, o);
    resid += __shfl_xor_sync(0xffffffffu, resid, o);
  }
  if ((threadIdx.x & 31) == 0) {
    if (served) atomicAdd(&cnt[0], served);
    if (left) atomicAdd(&cnt[1], left);
    if (resid) atomicAdd(&cnt[2], resid);
  }
}

// Refill (rounds >= 2, out of core): one warp per listed frontier entry whose cached keys are all
// matched.  The warp reads the host row zero-copy once, keeps the K largest AVAILABLE keys
// (per-lane top-K, then K warp pops) and writes them back as the row's cache: every key of the
// row above the K-th is unavailable now and stays so (R3), so the first available cached key is
// again the row maximum over available neighbours in later rounds.  The entry is redirected to
// the first refilled slot (or to an empty range when nothing is available).
template <int K>
__global__ void __launch_bounds__(256) k_host_rescan(Bins F, const uint64_t* __restrict__ rescan,
                                                     const unsigned long long* __restrict__ nrescan,
                                                     const int64_t* __restrict__ offs, AdjView adj,
                                                     const uint32_t* __restrict__ bits,
                                                     uint64_t* __restrict__ cache, int64_t u_first,
                                                     int64_t M0, int64_t vbase,
                                                     uint64_t* __restrict__ res = nullptr,
                                                     int64_t res_cap = 0,
                                                     unsigned long long* res_used = nullptr,
                                                     int64_t* __restrict__ roff = nullptr) {
  const int lane = threadIdx.x & 31;
  const int64_t c = (int64_t)*nrescan;
  const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t w = wid; w < c; w += nw) {
    const uint64_t r = rescan[w];
    const int bb = (int)(r >> 40);
    const int64_t i = (int64_t)(r & ((1ull << 40) - 1));
    const ulonglong2 e = F.list[bb][i];
    const int64_t u = (int64_t)(uint32_t)e.x - vbase;
    int64_t s, en;
    row_range(e, offs, vbase, &s, &en);
    uint64_t t[K];
#pragma unroll
    for (int q = 0; q < K; ++q) t[q] = 0ull;
    // residual rows (NEXT-1): the row is read over PCIe here anyway, so it is also copied into
    // the HBM residual buffer while space lasts; later rescans of it read HBM instead
    unsigned long long base = ~0ull;
    if (res && lane == 0) {
      const unsigned long long b0 = atomicAdd(res_used, (unsigned long long)(en - s));
      if ((int64_t)b0 + (en - s) <= res_cap) base = b0;
    }
    base = __shfl_sync(0xffffffffu, base, 0);
    for (int64_t j = s + lane; j < en; j += 32) {
      const uint64_t k = adj.at(j);
      if (base != ~0ull) res[base + (j - s)] = k;
      if (k && !bit_test(bits, (uint32_t)k)) topk_insert<K>(t, k);
    }
    if (base != ~0ull && lane == 0) roff[u - u_first] = (int64_t)base;
    const uint64_t mine = warp_topk_pop<K>(t);
    const int64_t slot = (u - u_first) * K;
    if (lane < K) cache[slot + lane] = mine;
    const uint64_t top = __shfl_sync(0xffffffffu, mine, 0);
    if (lane == 0)
      F.list[bb].r[i] = top ? ((1ull << 40) | (uint64_t)(M0 + slot)) : (uint64_t)(M0 + slot);
  }
}

// =============================================================================================
// NEXT-4: the Suitor algorithm (Manne & Halappanavar; the paper's SR-OMP / SR-GPU
// comparison algorithm) under the same strict order, which reaches the same unique
// locally dominant matching without synchronous rounds of mutual checks.
//   suitor[v] = the best proposal v has received: (bits(w(u,v)) << 32) | u  -- v's order over its
//               proposers (R1), so "better proposal" is a u64 compare and acceptance an atomicMax.
//   A vertex u without a standing proposal scans its row for the heaviest neighbour v (its own
//   order, key = bits(w) << 32 | v) whose current suitor is worse than u's offer, and proposes
//   with atomicMax.  A displaced suitor, or a proposer that lost the race, proposes again in the
//   next pass.  When no vertex is left, suitor[] is symmetric: mate[u] = proposer in suitor[u].
// Pass 1 needs no scan: with every suitor[] empty, u's choice is its row maximum, which the
// round-1 sweep already computed into best[u].
// =============================================================================================
constexpr uint64_t kHi32 = 0xffffffff00000000ull;

// u proposes `key` (its chosen neighbour); returns the vertex that must propose again next pass
// (the displaced previous suitor, or u itself when a better proposal got there first), or kNoPtr
__device__ __forceinline__ uint32_t suitor_propose(uint64_t* suitor, uint32_t u, uint64_t key) {
  const uint32_t v = (uint32_t)key;
  const uint64_t p = (key & kHi32) | u;
  const uint64_t old = atomicMax(reinterpret_cast<unsigned long long*>(&suitor[v]),
                                 (unsigned long long)p);
  if (old < p) return old ? (uint32_t)old : kNoPtr;
  return u;
}
// warp-aggregated append of the lanes' `again` vertices (all 32 lanes call it)
__device__ __forceinline__ void suitor_push(uint32_t again, uint32_t* next, unsigned long long* ncnt) {
  const unsigned b = __ballot_sync(0xffffffffu, again != kNoPtr);
  if (!b) return;
  const int lane = threadIdx.x & 31, leader = __ffs(b) - 1;
  unsigned long long base = 0;
  if (lane == leader) base = atomicAdd(ncnt, (unsigned long long)__popc(b));
  base = __shfl_sync(0xffffffffu, base, leader);
  if (again != kNoPtr) next[base + __popc(b & lanemask_lt())] = again;
}

// pass 1: every vertex proposes to its row maximum (best[] from the sweep)
__global__ void k_suitor_first(const uint64_t* __restrict__ best, int64_t n, uint64_t* suitor,
                               uint32_t* next, unsigned long long* ncnt) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t n32 = (n + 31) & ~31ll;
  for (int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; u < n32; u += stride) {
    const uint64_t k = u < n ? best[u] : 0ull;
    suitor_push(k ? suitor_propose(suitor, (uint32_t)u, k) : kNoPtr, next, ncnt);
  }
}

// the best neighbour of u over entries [a, b) whose suitor would accept u
__device__ __forceinline__ uint64_t suitor_best(const uint64_t* __restrict__ adj, int64_t a,
                                                int64_t b, int64_t step, uint32_t u,
                                                const uint64_t* suitor) {
  uint64_t best = 0;
  for (int64_t j = a; j < b; j += step) {
    const uint64_t k = __ldg(adj + j);
    if (k <= best) continue;
    const uint64_t p = (k & kHi32) | u;
    if (p > __ldcg(suitor + (uint32_t)k)) best = k;
  }
  return best;
}

// passes >= 2 over the worklist: a row of <= 32 entries is scanned by its lane, up to
// kSuitorBig entries by the warp, longer rows are listed for k_suitor_scan_big
constexpr int64_t kSuitorBig = 4096;
__global__ void __launch_bounds__(256) k_suitor_scan(const uint32_t* __restrict__ wl,
                                                     const unsigned long long* __restrict__ wcnt,
                                                     const int64_t* __restrict__ offs,
                                                     const uint64_t* __restrict__ adj,
                                                     uint64_t* suitor, uint32_t* next,
                                                     unsigned long long* ncnt, uint32_t* big,
                                                     unsigned long long* nbig,
                                                     unsigned long long* scanned) {
  const int lane = threadIdx.x & 31;
  const int64_t c = (int64_t)*wcnt;
  const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  unsigned long long sc = 0;
  for (int64_t i0 = wid * 32; i0 < c; i0 += nw * 32) {
    const int64_t i = i0 + lane;
    uint32_t u = 0;
    int64_t s = 0, e = 0;
    if (i < c) {
      u = wl[i];
      s = offs[u];
      e = offs[u + 1];
    }
    const int64_t d = e - s;
    uint32_t again = kNoPtr;
    if (d > 0 && d <= 32) {
      sc += (unsigned long long)d;
      const uint64_t b = suitor_best(adj, s, e, 1, u, suitor);
      if (b) again = suitor_propose(suitor, u, b);
    } else if (d > kSuitorBig) {
      big[atomicAdd(nbig, 1ull)] = u;
    }
    suitor_push(again, next, ncnt);
    unsigned mid = __ballot_sync(0xffffffffu, d > 32 && d <= kSuitorBig);
    while (mid) {
      const int l = __ffs(mid) - 1;
      mid &= mid - 1;
      const uint32_t ul = __shfl_sync(0xffffffffu, u, l);
      const int64_t sl = __shfl_sync(0xffffffffu, s, l), el = __shfl_sync(0xffffffffu, e, l);
      if (lane == 0) sc += (unsigned long long)(el - sl);
      const uint64_t b = group_max_key(suitor_best(adj, sl + lane, el, 32, ul, suitor), 0xffffffffu);
      uint32_t ag = kNoPtr;
      if (lane == 0 && b) ag = suitor_propose(suitor, ul, b);
      if (ag != kNoPtr) next[atomicAdd(ncnt, 1ull)] = ag;
    }
  }
  for (int o = 16; o; o >>= 1) sc += __shfl_xor_sync(0xffffffffu, sc, o);
  if (lane == 0 && sc) atomicAdd(scanned, sc);
}

// the listed long rows: one CTA per row
__global__ void __launch_bounds__(256) k_suitor_scan_big(const uint32_t* __restrict__ big,
                                                         const unsigned long long* __restrict__ nbig,
                                                         const int64_t* __restrict__ offs,
                                                         const uint64_t* __restrict__ adj,
                                                         uint64_t* suitor, uint32_t* next,
                                                         unsigned long long* ncnt,
                                                         unsigned long long* scanned) {
  __shared__ uint64_t red[8];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t nb = (int64_t)*nbig;
  for (int64_t i = blockIdx.x; i < nb; i += gridDim.x) {
    const uint32_t u = big[i];
    const int64_t s = offs[u], e = offs[u + 1];
    uint64_t b = group_max_key(suitor_best(adj, s + threadIdx.x, e, blockDim.x, u, suitor),
                               0xffffffffu);
    if (lane == 0) red[warp] = b;
    __syncthreads();
    if (warp == 0) {
      b = group_max_key(lane < 8 ? red[lane] : 0ull, 0xffffffffu);
      if (lane == 0) {
        const uint32_t ag = b ? suitor_propose(suitor, u, b) : kNoPtr;
        if (ag != kNoPtr) next[atomicAdd(ncnt, 1ull)] = ag;
        atomicAdd(scanned, (unsigned long long)(e - s));
      }
    }
    __syncthreads();
  }
}

// mate[] + w(M) from suitor[] (fixed assignment, fixed fp64 order, like k_materialize)
template <int THREADS>
__global__ void __launch_bounds__(THREADS)
    k_suitor_finish(const uint64_t* __restrict__ suitor, int64_t n, int32_t* __restrict__ mate,
                    double* pw, long long* pc) {
  double w = 0.0;
  long long c = 0;
  const int64_t stride = (int64_t)gridDim.x * THREADS;
  for (int64_t i = (int64_t)blockIdx.x * THREADS + threadIdx.x; i < n; i += stride) {
    const uint64_t k = suitor[i];
    int32_t v = -1;
    if (k) {
      v = (int32_t)(uint32_t)k;
      ++c;
      if ((int64_t)v > i) w += (double)__uint_as_float((uint32_t)(k >> 32));
    }
    mate[i] = v;
  }
  block_sum2<THREADS>(w, c, &pw[blockIdx.x], &pc[blockIdx.x]);
}

// ---- hybrid (algorithm 2): the LD iteration hands a long tail over to Suitor.  The vertices it
// matched are final (each mutual pair is in the unique matching M*) and the rest of M* is the
// unique LD matching of the graph without them (an M* edge at an unmatched vertex has an
// unmatched other end), so Suitor on that residual graph completes the same result.  Matched
// vertices get the sentinel suitor ~0, which no proposal exceeds.
__global__ void k_suitor_tail_init(const uint32_t* __restrict__ bits, int64_t n, uint64_t* suitor) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; u < n; u += stride)
    suitor[u] = bit_test(bits, (uint32_t)u) ? ~0ull : 0ull;
}
// worklist = the live vertices: stable pairs S and the frontier bins of the current set
__global__ void k_suitor_tail_list(const uint64_t* __restrict__ S, const unsigned long long* cntS,
                                   Bins F, const unsigned long long* cntF, uint32_t* wl,
                                   unsigned long long* wcnt) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t ns = (int64_t)*cntS;
  for (int64_t i0 = tid - (threadIdx.x & 31); i0 < ns; i0 += stride) {  // warp-uniform trips
    const int64_t i = i0 + (threadIdx.x & 31);
    suitor_push(i < ns ? (uint32_t)S[i] : kNoPtr, wl, wcnt);
  }
  for (int bb = 0; bb < kBins; ++bb) {
    const int64_t c = (int64_t)cntF[bb];
    for (int64_t i0 = tid - (threadIdx.x & 31); i0 < c; i0 += stride) {
      const int64_t i = i0 + (threadIdx.x & 31);
      suitor_push(i < c ? (uint32_t)F.list[bb].p[i] : kNoPtr, wl, wcnt);
    }
  }
}
// mate[] + w(M): LD-matched vertices from best[] (their pointer), the rest from suitor[]
template <int THREADS>
__global__ void __launch_bounds__(THREADS)
    k_hybrid_finish(const uint64_t* __restrict__ best, const uint32_t* __restrict__ bits,
                    const uint64_t* __restrict__ suitor, int64_t n, int32_t* __restrict__ mate,
                    double* pw, long long* pc) {
  double w = 0.0;
  long long c = 0;
  const int64_t stride = (int64_t)gridDim.x * THREADS;
  for (int64_t i = (int64_t)blockIdx.x * THREADS + threadIdx.x; i < n; i += stride) {
    uint64_t k = 0;
    if (bit_test(bits, (uint32_t)i)) k = best[i];
    else {
      const uint64_t sk = suitor[i];
      if (sk != ~0ull) k = sk;
    }
    int32_t v = -1;
    if (k) {
      v = (int32_t)(uint32_t)k;
      ++c;
      if ((int64_t)v > i) w += (double)__uint_as_float((uint32_t)(k >> 32));
    }
    mate[i] = v;
  }
  block_sum2<THREADS>(w, c, &pw[blockIdx.x], &pc[blockIdx.x]);
}


// =============================================================================================
// Sorted adjacency + cursor (algorithm 3).  Every row is sorted once by key,
// descending (the R1 order: weight bits, then neighbour id), so self-loop keys (0) sit at the row
// end.  u's pointer (Alg. 1 L4: the heaviest available neighbour) is then the first entry at
// or after cur[u] whose neighbour is unmatched; matched is permanent, so cur[u] only moves forward
// and the whole run reads each entry at most once (plus one re-check per live vertex per round).
// =============================================================================================
// row-relative int32 segment offsets of rows [r0, r1] for the segmented sort of one chunk
__global__ void k_sc_seg_offsets(const int64_t* __restrict__ offs, int64_t r0, int64_t r1,
                                 int32_t* __restrict__ seg) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t base = offs[r0];
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= r1 - r0; i += stride)
    seg[i] = (int32_t)(offs[r0 + i] - base);
}

// SETPOINTERS with cursors.  Round 1 (L == nullptr): every vertex points at its row's first key
// (nothing is matched yet; a 0 key = self-loops only or an empty row).  Rounds >= 2: the live list
// holds (u, current pointer key) pairs; only u whose target was matched last round change (Alg. 3's
// frontier): cur[u] (row-relative, 0 after round 1) moves past matched neighbours and the
// pair and ptr[u] get the new key (0 when the row ran dry).  A thread walks at most kScSerial (64;
// 2/4/8/16/32/128/512 measured slower or equal)
// entries; rows that need more go to the `big` list (list index) for k_sc_point_warp.
// `reads` counts adjacency entries read.
#ifndef LM_SC_SERIAL
#define LM_SC_SERIAL 64
#endif
#ifndef LM_SC_MINB
#define LM_SC_MINB 8
#endif
constexpr int kScSerial = LM_SC_SERIAL;
__global__ void __launch_bounds__(256, LM_SC_MINB) k_sc_point(ulonglong2* __restrict__ L, const unsigned long long* __restrict__ nL,
                           int64_t n_all, const int64_t* __restrict__ offs,
                           const uint64_t* __restrict__ adj, uint32_t* __restrict__ cur,
                           const uint32_t* __restrict__ bits, uint64_t* __restrict__ ptr,
                           uint32_t* __restrict__ big, unsigned long long* nbig,
                           unsigned long long* reads) {
  const int64_t cnt = L ? (int64_t)*nL : n_all;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  unsigned long long r = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += stride) {
    if (!L) {
      const int64_t a = offs[i];
      uint64_t k = 0;
      if (a < offs[i + 1]) { k = __ldg(adj + a); ++r; }
      ptr[i] = k;
      continue;
    }
    ulonglong2 p = L[i];
    if (!bit_test(bits, (uint32_t)p.y)) continue;  // target still unmatched: pointer unchanged
    const uint32_t u = (uint32_t)p.x;
    const int64_t a = offs[u], e = offs[u + 1];
    int64_t j = a + cur[u] + 1;
    const int64_t stop = j + kScSerial < e ? j + kScSerial : e;
    uint64_t k = 0;
    bool found = false;
    for (; j < stop; ++j) {
      k = __ldg(adj + j);
      ++r;
      if (k == 0ull) { j = e; break; }
      if (!bit_test(bits, (uint32_t)k)) { found = true; break; }
    }
    cur[u] = (uint32_t)(j - a);
    if (!found && j < e) {  // long skip: hand the row to a warp
      big[atomicAdd(nbig, 1ull)] = (uint32_t)i;
      continue;
    }
    if (!found) k = 0ull;
    ptr[u] = k;
    p.y = k;
    L[i] = p;
  }
  for (int o = 16; o; o >>= 1) r += __shfl_xor_sync(0xffffffffu, r, o);
  if ((threadIdx.x & 31) == 0 && r) atomicAdd(reads, r);
}

// the long skips: one warp per listed row scans 32 entries per step from cur[u] and takes the
// first (lowest-index, i.e. heaviest) available key
__global__ void k_sc_point_warp(ulonglong2* __restrict__ L, const uint32_t* __restrict__ big,
                                const unsigned long long* __restrict__ nbig,
                                const int64_t* __restrict__ offs, const uint64_t* __restrict__ adj,
                                uint32_t* __restrict__ cur, const uint32_t* __restrict__ bits,
                                uint64_t* __restrict__ ptr, unsigned long long* reads) {
  const int lane = threadIdx.x & 31;
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t ws = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t cnt = (int64_t)*nbig;
  unsigned long long r = 0;
  for (int64_t w = w0; w < cnt; w += ws) {
    const uint32_t i = big[w];
    ulonglong2 p = L[i];
    const uint32_t u = (uint32_t)p.x;
    const int64_t a = offs[u], e = offs[u + 1];
    uint64_t k = 0;
    int64_t j = a + cur[u];
    for (; j < e; j += 32) {
      const int64_t jj = j + lane;
      const uint64_t kk = jj < e ? __ldg(adj + jj) : 0ull;
      r += jj < e;
      const bool ok = kk != 0ull && !bit_test(bits, (uint32_t)kk);
      const unsigned zb = __ballot_sync(0xffffffffu, jj < e && kk == 0ull);
      const unsigned ob = __ballot_sync(0xffffffffu, ok);
      // keys are descending: a 0 key ends the row's available part
      const unsigned first_zero = zb ? (unsigned)(__ffs(zb) - 1) : 32u;
      if (ob && (unsigned)(__ffs(ob) - 1) < first_zero) {
        const int src = __ffs(ob) - 1;
        k = __shfl_sync(0xffffffffu, kk, src);
        j += src;
        break;
      }
      if (zb) { j = e; break; }
    }
    if (j >= e) { k = 0ull; j = e; }
    if (lane == 0) {
      cur[u] = (uint32_t)(j - a);
      ptr[u] = k;
      p.y = k;
      L[i] = p;
    }
  }
  for (int o = 16; o; o >>= 1) r += __shfl_xor_sync(0xffffffffu, r, o);
  if (lane == 0 && r) atomicAdd(reads, r);
}

// SETMATES (Alg. 1 L6-9): u with ptr[ptr[u]] == u is matched (mate key stored, bit set); a live
// u that is not matched goes to the next list with its pointer; u with no available neighbour
// (key 0) leaves for good.  Round 1 (L == nullptr) reads the pairs (u, ptr[u]) for every u.
// Each thread takes kScItems pairs per block step and the block reserves its output with one
// atomicAdd (per-warp reservations on one counter serialised the kernel).
#ifndef LM_SC_ITEMS
#define LM_SC_ITEMS 4
#endif
constexpr int kScThreads = 256, kScItems = LM_SC_ITEMS;
__global__ void __launch_bounds__(kScThreads)
    k_sc_match(const ulonglong2* __restrict__ L, const unsigned long long* __restrict__ nL,
               int64_t n_all, const uint64_t* __restrict__ ptr, uint32_t* bits,
               uint64_t* __restrict__ matek, ulonglong2* __restrict__ next,
               unsigned long long* ncnt) {
  __shared__ int s_warp[kScThreads / 32];
  __shared__ unsigned long long s_base;
  const int64_t cnt = L ? (int64_t)*nL : n_all;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  constexpr int64_t kStep = (int64_t)kScThreads * kScItems;
  for (int64_t b0 = (int64_t)blockIdx.x * kStep; b0 < cnt; b0 += (int64_t)gridDim.x * kStep) {
    ulonglong2 p[kScItems];
    bool keep[kScItems];
    int mine = 0;
#pragma unroll
    for (int t = 0; t < kScItems; ++t) {
      const int64_t i = b0 + t * kScThreads + threadIdx.x;
      keep[t] = false;
      p[t] = make_ulonglong2(0ull, 0ull);
      if (i < cnt) p[t] = L ? L[i] : make_ulonglong2((unsigned long long)i, ptr[i]);
    }
    uint64_t kv[kScItems];
#pragma unroll
    for (int t = 0; t < kScItems; ++t) kv[t] = p[t].y ? __ldg(ptr + (uint32_t)p[t].y) : 0ull;
#pragma unroll
    for (int t = 0; t < kScItems; ++t) {
      if (!p[t].y) continue;
      const uint32_t u = (uint32_t)p[t].x;
      if ((uint32_t)kv[t] == u && kv[t] != 0ull) {
        matek[u] = p[t].y;
        atomicOr(bits + (u >> 5), 1u << (u & 31));
      } else {
        keep[t] = true;
        ++mine;
      }
    }
    // block-wide exclusive scan of `mine`
    int incl = mine;
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += y;
    }
    if (lane == 31) s_warp[wid] = incl;
    __syncthreads();
    if (threadIdx.x == 0) {
      int tot = 0;
      for (int w = 0; w < kScThreads / 32; ++w) { const int c = s_warp[w]; s_warp[w] = tot; tot += c; }
      s_base = tot ? atomicAdd(ncnt, (unsigned long long)tot) : 0ull;
    }
    __syncthreads();
    unsigned long long o = s_base + s_warp[wid] + (incl - mine);
#pragma unroll
    for (int t = 0; t < kScItems; ++t)
      if (keep[t]) next[o++] = p[t];
    __syncthreads();
  }
}

}  // namespace lm
