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
#include <cuda_runtime.h>

namespace lm {

constexpr int kBins = 4;               // frontier degree bins
constexpr int kBinDeg0 = 8, kBinDeg1 = 128, kBinDeg2 = 4096;  // bins: G = 4, 16, 32 lanes, CTA

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
__global__ void k_symhash(const int64_t* __restrict__ offs, const uint64_t* __restrict__ adj,
                          int64_t n, unsigned long long* acc) {
  const int lane8 = threadIdx.x & 7;
  const int64_t g0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 3;
  const int64_t gs = ((int64_t)gridDim.x * blockDim.x) >> 3;
  uint64_t s = 0;
  for (int64_t u = g0; u < n; u += gs) {
    for (int64_t j = offs[u] + lane8; j < offs[u + 1]; j += 8) {
      const uint64_t k = adj[j];
      const uint64_t v = (uint32_t)k, wb = k >> 32;
      s += mix64(mix64((uint64_t)u * 0x100000001B3ull ^ v) ^ wb) -
           mix64(mix64(v * 0x100000001B3ull ^ (uint64_t)u) ^ wb);
    }
  }
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) atomicAdd(acc, (unsigned long long)s);
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
// per-run reset: matched bitmap, counters, and best[] of the rows the sweep merges with
// atomicMax (rows longer than one piece, or crossing a tile boundary; listed at create time).
// =============================================================================================
__global__ void k_reset(uint32_t* bits, int64_t nwords, uint64_t* best,
                        const int32_t* __restrict__ atomic_rows, int64_t n_atomic,
                        unsigned long long* counters, int ncounters) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (int64_t i = tid; i < nwords; i += stride) bits[i] = 0u;
  for (int64_t i = tid; i < n_atomic; i += stride) best[atomic_rows[i]] = 0ull;
  if (tid < ncounters) counters[tid] = 0ull;
}

// =============================================================================================
// A2 round-1 pointer sweep (SETPOINTERS over all vertices, Alg. 3 L1-9 P:141-151).
//
// Edge-centric tiles: the adjacency is cut into fixed tiles of TILE entries regardless of row
// boundaries, so every CTA streams equal bytes (hub rows and degree-1 rows alike).  A persistent
// CTA keeps STAGES tiles in flight with 1-D TMA bulk copies (cp.async.bulk -> UBLKCP) completing
// on mbarriers: the tile's packed keys, plus the window of its rows' start offsets (low 32 bits)
// and vertex ids.  Per tile, entirely from shared memory:
//   1. classify every row of the window by its in-tile length: short (< 32 entries) rows go to a
//      thread-per-row list; long rows are cut into pieces of <= PIECE entries for a warp each;
//   2. short rows: one thread scans the row;  pieces: a warp scans 32 consecutive keys per step
//      (conflict-free) and reduces with two 32-bit __reduce_max_sync (packed-key max);
//   3. a row wholly inside one unit (tile and piece) is stored; any other row is merged with a
//      global atomicMax on its u64 key (max is order independent => identical to one sequential
//      scan; the row was zeroed by k_reset).
// Self-loops are skipped (simple graph).  No bitmap test: in round 1 nothing is matched.
// =============================================================================================
struct SweepArgs {
  const uint64_t* adj;
  const uint32_t* noffs_lo;  // low 32 bits of each non-empty row's start (+ m)
  const int32_t* nzr;
  const int32_t* tile_nz;
  uint64_t* best;
  int64_t m;
  int64_t ntiles;
};

template <int CONSUMER_WARPS, int STAGES>
struct SweepCfg {
  static constexpr int kTile = 1024;
  static constexpr int kPiece = 256;
  static constexpr int kConsumers = CONSUMER_WARPS;
  static constexpr int kThreads = 32 * (CONSUMER_WARPS + 1);  // warp 0 = TMA producer
  static constexpr int kKeys = kTile + 2;   // u64 slots per stage
  static constexpr int kWin = kTile + 8;    // u32 row starts per stage
  static constexpr int kIds = kTile + 8;    // i32 vertex ids per stage
  static constexpr int kMaxPieces = kTile / 32 + kTile / kPiece + 4;
  static constexpr int kShort = kTile + 8;
  static constexpr size_t kStageBytes = (size_t)kKeys * 8 + (size_t)kWin * 4 + (size_t)kIds * 4;
  static constexpr size_t kSmem = STAGES * kStageBytes + 2 * (size_t)kShort * 2 +
                                  2 * (size_t)kMaxPieces * 8 + 2 * STAGES * 8 + STAGES * 8 + 32;
};

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("{\n .reg .b64 st;\n mbarrier.arrive.shared::cta.b64 st, [%0];\n}\n" ::"r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

template <int CONSUMER_WARPS, int STAGES>
__global__ void __launch_bounds__(32 * (CONSUMER_WARPS + 1)) k_sweep(SweepArgs A) {
  using C = SweepCfg<CONSUMER_WARPS, STAGES>;
  constexpr int TILE = C::kTile, PIECE = C::kPiece, NW = CONSUMER_WARPS, NCT = 32 * NW;
  extern __shared__ __align__(128) unsigned char smem[];
  uint64_t* keys = reinterpret_cast<uint64_t*>(smem);
  uint32_t* win = reinterpret_cast<uint32_t*>(smem + (size_t)STAGES * C::kKeys * 8);
  int32_t* ids = reinterpret_cast<int32_t*>(smem + (size_t)STAGES * (C::kKeys * 8 + C::kWin * 4));
  int16_t* shortl = reinterpret_cast<int16_t*>(smem + (size_t)STAGES * C::kStageBytes);  // [2][kShort]
  int2* pieces = reinterpret_cast<int2*>(shortl + 2 * C::kShort);  // [2][kMaxPieces] (row, a|b<<16)
  uint64_t* full = reinterpret_cast<uint64_t*>(pieces + 2 * C::kMaxPieces);
  uint64_t* empty = full + STAGES;
  int32_t* meta = reinterpret_cast<int32_t*>(empty + STAGES);  // [STAGES][2]
  int32_t* cnt = meta + 2 * STAGES;                              // [3][2]: short, pieces

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid < 6) cnt[tid] = 0;
  if (tid == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], NW);
    }
    fence_mbar_init();
  }
  __syncthreads();

  if (warp == 0) {
    // ---------------- producer: keep STAGES tiles in flight (1-D TMA bulk copies)
    if (lane != 0) return;
    const uint64_t pol = policy_evict_first();
    int64_t t = blockIdx.x;
    int32_t a = 0, bp = 0;
    if (t < A.ntiles) { a = A.tile_nz[t]; bp = A.tile_nz[t + 1]; }
    for (int64_t k = 0; t < A.ntiles; ++k) {
      const int64_t tn = t + gridDim.x;  // prefetch the next tile's row range
      int32_t an = 0, bpn = 0;
      if (tn < A.ntiles) { an = A.tile_nz[tn]; bpn = A.tile_nz[tn + 1]; }
      const int s = (int)(k % STAGES);
      if (k >= STAGES)
        while (!mbar_try_wait(&empty[s], (uint32_t)(((k / STAGES) - 1) & 1))) {
        }
      meta[2 * s] = a;
      meta[2 * s + 1] = bp;
      const int64_t e0 = t * TILE;
      const int64_t len = min((int64_t)TILE, A.m - e0);
      const uint32_t kbytes = (uint32_t)(((len + 1) & ~1ll) * 8);
      const int64_t a4 = a & ~3ll;
      const uint32_t wbytes = (uint32_t)((((int64_t)bp + 2 - a4 + 3) & ~3ll) * 4);
      fence_proxy_async_smem();
      mbar_arrive_expect_tx(&full[s], kbytes + 2 * wbytes);
      tma_bulk_g2s(keys + (size_t)s * C::kKeys, A.adj + e0, kbytes, &full[s], pol);
      tma_bulk_g2s(win + (size_t)s * C::kWin, A.noffs_lo + a4, wbytes, &full[s], pol);
      tma_bulk_g2s(ids + (size_t)s * C::kIds, A.nzr + a4, wbytes, &full[s], pol);
      t = tn; a = an; bp = bpn;
    }
    return;
  }

  // ------------------ consumers (warps 1..NW): one named barrier per tile
  const int ctid = tid - 32, cwarp = warp - 1;
  for (int64_t k = 0;; ++k) {
    const int64_t t = (int64_t)blockIdx.x + k * gridDim.x;
    if (t >= A.ntiles) break;
    const int s = (int)(k % STAGES);
    const int par = (int)(k & 1);
    int32_t* ck = cnt + 2 * (int)(k % 3);
    int16_t* SL = shortl + par * C::kShort;
    int2* PL = pieces + par * C::kMaxPieces;
    while (!mbar_try_wait(&full[s], (uint32_t)((k / STAGES) & 1))) {
    }
    const uint64_t* K = keys + (size_t)s * C::kKeys;
    const uint32_t* W = win + (size_t)s * C::kWin;
    const int32_t* I = ids + (size_t)s * C::kIds;
    const int32_t a = meta[2 * s], bp = meta[2 * s + 1];
    const int lo = a & 3, hi = bp - (a & ~3);
    const int64_t ts = t * TILE;
    const int len = (int)min((int64_t)TILE, A.m - ts);
    const uint32_t ts32 = (uint32_t)ts;
    auto rel = [&](int r) { return (int32_t)(W[r] - ts32); };  // row start relative to tile

    // ---- 1. classify the window's rows by in-tile length
    for (int r0 = lo; r0 <= hi; r0 += NCT) {
      const int r = r0 + ctid;
      int L = 0, ra = 0, rb = 0;
      if (r <= hi) {
        ra = max(rel(r), 0);
        rb = min(rel(r + 1), len);
        L = rb - ra;
      }
      const bool sh = L > 0 && L < 32;
      const unsigned bs = __ballot_sync(0xffffffffu, sh);
      if (bs) {
        int base = 0;
        const int leader = __ffs(bs) - 1;
        if (lane == leader) base = atomicAdd(&ck[0], __popc(bs));
        base = __shfl_sync(0xffffffffu, base, leader);
        if (sh) SL[base + __popc(bs & lanemask_lt())] = (int16_t)r;
      }
      if (L >= 32) {
        const int np = (L + PIECE - 1) / PIECE;
        const int base = atomicAdd(&ck[1], np);
        for (int q = 0; q < np; ++q) {
          const int pa = ra + q * PIECE, pb = min(rb, pa + PIECE);
          PL[base + q] = make_int2(r, pa | (pb << 16));
        }
      }
    }
    named_bar_sync(1, NCT);
    const int nshort = ck[0], npieces = ck[1];
    if (ctid == 0) { int32_t* cz = cnt + 2 * (int)((k + 2) % 3); cz[0] = 0; cz[1] = 0; }
    // ---- 2a. short rows: a thread per row
    for (int i = ctid; i < nshort; i += NCT) {
      const int r = SL[i];
      const int32_t rs = rel(r), re = rel(r + 1);
      const int ja = max(rs, 0), jb = min(re, len);
      const uint32_t vid = (uint32_t)I[r];
      uint64_t b = 0;
      for (int j = ja; j < jb; ++j) {
        const uint64_t key = K[j];
        if ((uint32_t)key != vid && key > b) b = key;
      }
      if (rs >= 0 && re <= len) A.best[vid] = b;
      else if (b) atomicMax(reinterpret_cast<unsigned long long*>(&A.best[vid]), (unsigned long long)b);
    }
    // ---- 2b. pieces of long rows: a warp per piece
    for (int p = cwarp; p < npieces; p += NW) {
      const int2 pc = PL[p];
      const int r = pc.x, pa = pc.y & 0xffff, pb = pc.y >> 16;
      const uint32_t vid = (uint32_t)I[r];
      uint64_t b = 0;
      for (int j = pa + lane; j < pb; j += 32) {
        const uint64_t key = K[j];
        if ((uint32_t)key != vid && key > b) b = key;
      }
      b = group_max_key(b, 0xffffffffu);
      if (lane == 0) {
        const int32_t rs = rel(r), re = rel(r + 1);
        if (rs >= 0 && re <= len && re - rs <= PIECE) A.best[vid] = b;
        else if (b) atomicMax(reinterpret_cast<unsigned long long*>(&A.best[vid]), (unsigned long long)b);
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[s]);  // this warp is done with stage s
  }
}

// rows the sweep merges with atomicMax: degree > PIECE, or crossing a tile boundary
__global__ void k_atomic_rows(const int64_t* __restrict__ noffs, const int32_t* __restrict__ nzr,
                              int64_t n_nz, const int32_t* __restrict__ tile_nz, int64_t ntiles,
                              int64_t tile, int64_t piece, int32_t* out,
                              unsigned long long* count) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t lim = ((n_nz > ntiles ? n_nz : ntiles) + 31) & ~31ll;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < lim; i += stride) {
    const bool longrow = i < n_nz && noffs[i + 1] - noffs[i] > piece;
    warp_append(longrow, longrow ? nzr[i] : 0, out, count);
    bool cross = false;
    int32_t v = 0;
    if (i >= 1 && i < ntiles) {
      const int32_t r = tile_nz[i];
      cross = noffs[r] < i * tile && noffs[r + 1] - noffs[r] <= piece;  // long rows listed above
      v = nzr[r];
    }
    warp_append(cross, v, out, count);
  }
}

__global__ void k_low32(const int64_t* __restrict__ noffs, int64_t cnt, uint32_t* lo) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += stride)
    lo[i] = (uint32_t)noffs[i];
}

// =============================================================================================
// A2 pointer phase on the frontier (rounds >= 2): G lanes per vertex, degree-binned.
// best[u] = max{ adj[j] : j in row(u), col != u, !matched(col) }  (Alg. 3 L5-8).
// =============================================================================================
template <int G>
__global__ void k_point_group(const int32_t* __restrict__ list, const unsigned long long* cnt_ptr,
                              const int64_t* __restrict__ offs, const uint64_t* __restrict__ adj,
                              const uint32_t* __restrict__ bits, uint64_t* __restrict__ best) {
  const int64_t cnt = (int64_t)*cnt_ptr;
  const int lane = threadIdx.x & 31;
  const int gl = lane & (G - 1);
  const unsigned gmask = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
  const int64_t ng = ((int64_t)gridDim.x * blockDim.x) / G;
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / G; i < cnt; i += ng) {
    const uint32_t u = (uint32_t)list[i];
    const int64_t s = offs[u], e = offs[u + 1];
    uint64_t b = 0;
    for (int64_t j = s + gl; j < e; j += G) {
      const uint64_t key = adj[j];
      const uint32_t v = (uint32_t)key;
      if (v != u && key > b && !bit_test(bits, v)) b = key;
    }
    b = group_max_key(b, gmask);
    if (gl == 0) best[u] = b;
  }
}

template <int THREADS>
__global__ void __launch_bounds__(THREADS)
    k_point_cta(const int32_t* __restrict__ list, const unsigned long long* cnt_ptr,
                const int64_t* __restrict__ offs, const uint64_t* __restrict__ adj,
                const uint32_t* __restrict__ bits, uint64_t* __restrict__ best) {
  __shared__ uint64_t red[THREADS / 32];
  const int64_t cnt = (int64_t)*cnt_ptr;
  for (int64_t i = blockIdx.x; i < cnt; i += gridDim.x) {
    const uint32_t u = (uint32_t)list[i];
    const int64_t s = offs[u], e = offs[u + 1];
    uint64_t b = 0;
    for (int64_t j = s + threadIdx.x; j < e; j += THREADS) {
      const uint64_t key = adj[j];
      const uint32_t v = (uint32_t)key;
      if (v != u && key > b && !bit_test(bits, v)) b = key;
    }
    b = group_max_key(b, 0xffffffffu);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = b;
    __syncthreads();
    if (threadIdx.x < 32) {
      uint64_t x = threadIdx.x < THREADS / 32 ? red[threadIdx.x] : 0ull;
      x = group_max_key(x, 0xffffffffu);
      if (threadIdx.x == 0) best[u] = x;
    }
    __syncthreads();
  }
}

// =============================================================================================
// A4 match (SETMATES, Alg. 3 L10-13 P:152-155): mutual pointers are locally dominant edges.
// =============================================================================================
// Round 1: every vertex; the warp owning 32 consecutive vertices writes their bitmap word.
__global__ void k_match_all(const uint64_t* __restrict__ best, int64_t n, uint32_t* bits) {
  const int64_t nwords = (n + 31) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t ws = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t wi = w0; wi < nwords; wi += ws) {
    const int64_t u = (wi << 5) + lane;
    bool mutual = false;
    if (u < n) {
      const uint64_t b = best[u];
      if (b) {
        const uint64_t bv = best[(uint32_t)b];
        mutual = bv != 0 && (uint32_t)bv == (uint32_t)u;
      }
    }
    const unsigned word = __ballot_sync(0xffffffffu, mutual);
    if (lane == 0) bits[wi] = word;
  }
}

// Rounds >= 2: the frontier (all bins).  A new mutual pair has at least one endpoint that
// re-pointed this round (R3); that endpoint marks both.
struct BinLists {
  const int32_t* list[kBins];
};
__global__ void k_match_list(BinLists F, const unsigned long long* cnt,
                             const uint64_t* __restrict__ best, uint32_t* bits) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll
  for (int b = 0; b < kBins; ++b) {
    const int64_t c = (int64_t)cnt[b];
    for (int64_t i = tid; i < c; i += stride) {
      const uint32_t u = (uint32_t)F.list[b][i];
      const uint64_t k = best[u];
      if (!k) continue;
      const uint32_t v = (uint32_t)k;
      const uint64_t kv = best[v];
      if (kv != 0 && (uint32_t)kv == u) {
        atomicOr(&bits[u >> 5], 1u << (u & 31));
        atomicOr(&bits[v >> 5], 1u << (v & 31));
      }
    }
  }
}

// =============================================================================================
// A6 frontier compaction (not in the paper, which rescans every unmatched vertex):
//   L' = { u in L : !matched(u), best[u] != 0 }
//   F' = { u in L' : matched(ptr u) }     binned by degree
// counters layout: [0] |L'|, [1..kBins] |F'_b|, [kBins+1] sum of deg over F'
// Each warp owns a chunk of 32*K items: pass 1 records the predicates in registers and counts,
// ONE atomicAdd per list per warp reserves the output ranges, pass 2 writes -- so the global
// counters see (items / 32K) atomics instead of one per 32 items.
// =============================================================================================
template <bool ALL, int K>
__global__ void k_compact(const int32_t* __restrict__ L, const unsigned long long* Lcnt, int64_t n,
                          const uint64_t* __restrict__ best, const uint32_t* __restrict__ bits,
                          const int64_t* __restrict__ offs, int32_t* Lout, BinLists Fout,
                          unsigned long long* counters) {
  const int64_t cnt = ALL ? n : (int64_t)*Lcnt;
  const int lane = threadIdx.x & 31;
  const int64_t warp0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const unsigned lt = lanemask_lt();
  unsigned long long degsum = 0;
  for (int64_t c0 = warp0 * 32 * K; c0 < cnt; c0 += nwarps * 32 * K) {
    uint32_t live = 0, binb[kBins] = {0, 0, 0, 0};
    uint32_t uu[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const int64_t i = c0 + 32 * k + lane;
      uu[k] = 0;
      if (i < cnt) {
        const uint32_t u = ALL ? (uint32_t)i : (uint32_t)L[i];
        uu[k] = u;
        const uint64_t b = best[u];
        if (b != 0 && !bit_test(bits, u)) {
          live |= 1u << k;
          if (bit_test(bits, (uint32_t)b)) {
            const int64_t d = offs[u + 1] - offs[u];
            binb[bin_of(d)] |= 1u << k;
            degsum += (unsigned long long)d;
          }
        }
      }
    }
    // reserve output ranges: one atomic per list per warp
    unsigned long long base[1 + kBins];
    {
      unsigned tot[1 + kBins];
      tot[0] = __reduce_add_sync(0xffffffffu, __popc(live));
#pragma unroll
      for (int b = 0; b < kBins; ++b) tot[1 + b] = __reduce_add_sync(0xffffffffu, __popc(binb[b]));
#pragma unroll
      for (int q = 0; q < 1 + kBins; ++q) {
        unsigned long long x = 0;
        if (lane == q && tot[q]) x = atomicAdd(&counters[q], (unsigned long long)tot[q]);
        base[q] = __shfl_sync(0xffffffffu, x, q);
      }
    }
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const bool pl = (live >> k) & 1u;
      const unsigned bl = __ballot_sync(0xffffffffu, pl);
      if (pl) Lout[base[0] + __popc(bl & lt)] = (int32_t)uu[k];
      base[0] += __popc(bl);
#pragma unroll
      for (int b = 0; b < kBins; ++b) {
        const bool pb = (binb[b] >> k) & 1u;
        const unsigned bb = __ballot_sync(0xffffffffu, pb);
        if (pb) const_cast<int32_t*>(Fout.list[b])[base[1 + b] + __popc(bb & lt)] = (int32_t)uu[k];
        base[1 + b] += __popc(bb);
      }
    }
  }
  for (int o = 16; o; o >>= 1) degsum += __shfl_xor_sync(0xffffffffu, degsum, o);
  if (lane == 0 && degsum) atomicAdd(&counters[1 + kBins], degsum);
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
                  int32_t* __restrict__ mate, double* pw, long long* pc) {
  double w = 0.0;
  long long c = 0;
  const int64_t stride = (int64_t)gridDim.x * THREADS;
  for (int64_t u = (int64_t)blockIdx.x * THREADS + threadIdx.x; u < n; u += stride) {
    int32_t v = -1;
    if (bit_test(bits, (uint32_t)u)) {
      const uint64_t k = best[u];
      v = (int32_t)(uint32_t)k;
      ++c;
      if ((int64_t)v > u) w += (double)__uint_as_float((uint32_t)(k >> 32));
    }
    mate[u] = v;
  }
  block_sum2<THREADS>(w, c, &pw[blockIdx.x], &pc[blockIdx.x]);
}

// w(M) for an arbitrary mate[]: 8 lanes per vertex search row u for mate[u] (first match).
// err: bit0 = mate out of range / self, bit1 = asymmetric, bit2 = pair not an edge.
template <int THREADS>
__global__ void __launch_bounds__(THREADS)
    k_weight_any(const int32_t* __restrict__ mate, int64_t n, const int64_t* __restrict__ offs,
                 const uint64_t* __restrict__ adj, double* pw, long long* pc, unsigned* err) {
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
      const uint64_t k = adj[j];
      if ((uint32_t)k == (uint32_t)v) found = k;
    }
    found = group_max_key(found, gmask);
    if (g8 == 0) {
      if (!found) atomicOr(err, 4u);
      else { w += (double)__uint_as_float((uint32_t)(found >> 32)); ++c; }
    }
  }
  block_sum2<THREADS>(w, c, &pw[blockIdx.x], &pc[blockIdx.x]);
}

__global__ void k_final_sum(const double* pw, const long long* pc, int nb, double* out_w,
                            long long* out_c) {
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    double w = 0; long long c = 0;
    for (int i = 0; i < nb; ++i) { w += pw[i]; c += pc[i]; }
    *out_w = w; *out_c = c;
  }
}

}  // namespace lm
