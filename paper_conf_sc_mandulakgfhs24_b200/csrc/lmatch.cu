// lmatch.cu -- C ABI (include/lmatch.h) over the sm_100a kernels in kernels.cuh.
//
// Host-side structure:
//   lmatch_create*   A1 ingest: chunked H2D (2 streams, double-buffered staging) + pack/validate,
//                    offsets check, non-empty-row index, sweep tile index.   (untimed)
//   lmatch_run*      reset -> A2 round-1 sweep -> A4 match-all -> A6 compact-all ->
//                    { A2 frontier pointer (per degree bin) -> A4 match -> A6 compact }* ->
//                    A10 mate + A9 weight.  The loop ends when the next frontier is empty
//                    (termination; R6).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <atomic>
#include <climits>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>

#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <time.h>
#include <unistd.h>

#include "../../include/lmatch.h"
#include "kernels.cuh"

#include <cub/device/device_segmented_sort.cuh>


namespace {

thread_local char g_err[512] = "";

void set_err(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof g_err, fmt, ap);
  va_end(ap);
}

#define CK(call)                                                                        \
  do {                                                                                  \
    cudaError_t e_ = (call);                                                            \
    if (e_ != cudaSuccess) {                                                            \
      set_err("%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e_));       \
      return (e_ == cudaErrorMemoryAllocation) ? LMATCH_ENOMEM : LMATCH_ECUDA;          \
    }                                                                                   \
  } while (0)
// every kernel launch of the library is followed by CKL(): it also counts the launch (process-wide,
// lmatch_kernel_launch_count)
static std::atomic<long long> g_launch_count{0};
static thread_local long long t_launch_count = 0;  // this thread's launches (lmatch_run_dist stats)
static inline void count_launches(long long k) {
  g_launch_count.fetch_add(k, std::memory_order_relaxed);
  t_launch_count += k;
}
#define CKL()                                            \
  do {                                                   \
    count_launches(1);                                   \
    CK(cudaGetLastError());                              \
  } while (0)
#define TRY(x)                 \
  do {                         \
    int s_ = (x);              \
    if (s_ != LMATCH_OK) return s_; \
  } while (0)

// Round-1 sweep configurations (tuned on B200), chosen per handle by the
// average degree.  Round 2, after the key max moved to the FP64 pipe, the per-tile TMA issue and
// row-window work became the larger share of the sweep's instructions: for graphs with average
// degree >= LM_SWEEP_DENSE_DEG, 1024-entry tiles, 6 warps per CTA (2 CTAs = 12 warps per SM) and a
// 104-row window measured 2.88 ms against 2.99 ms for 512 / 8 / 72 on R-MAT s26 (ER 1.51 vs
// 1.60 ms); sparse graphs (meshes, road-like) keep 512 / 8 / 72, whose row window holds their
// many short rows (2-D mesh 0.64 vs 0.90 ms, road-like 0.58 vs 0.95 ms with 1024-entry tiles).
#ifndef LM_SWEEP_DENSE_DEG
#define LM_SWEEP_DENSE_DEG 10
#endif
#ifndef LM_SWEEP_S_TILE
#define LM_SWEEP_S_TILE 512
#endif
#ifndef LM_SWEEP_S_WARPS
#define LM_SWEEP_S_WARPS 8
#endif
#ifndef LM_SWEEP_S_WCAP
#define LM_SWEEP_S_WCAP 72
#endif
#ifndef LM_SWEEP_TILE
#define LM_SWEEP_TILE 1024
#endif
#ifndef LM_SWEEP_RING
#define LM_SWEEP_RING 2
#endif
#ifndef LM_SWEEP_WARPS
#define LM_SWEEP_WARPS 6
#endif
#ifndef LM_SWEEP_WCAP
#define LM_SWEEP_WCAP 104
#endif
constexpr int kSweepTile = LM_SWEEP_TILE;    // entries per warp tile
constexpr int kSweepRing = LM_SWEEP_RING;    // TMA stages per warp
constexpr int kSweepWarps = LM_SWEEP_WARPS;  // warps per CTA
constexpr int kSweepWcap = LM_SWEEP_WCAP;    // staged row-window entries per stage
#ifndef LM_SWEEP_IMPL
#define LM_SWEEP_IMPL 1  // 2 = swizzled 2-D TMA + segmented scan; 1 = row-classified 1-D TMA
#endif
#if LM_SWEEP_IMPL == 2
using Sweep = lm::Sweep2DCfg<kSweepTile, kSweepRing, kSweepWarps, kSweepWcap>;
#define SWEEP_KERNEL lm::k_sweep2d<kSweepTile, kSweepRing, kSweepWarps, kSweepWcap>
#else
using Sweep = lm::SweepCfg<kSweepTile, kSweepRing, kSweepWarps, kSweepWcap>;
#define SWEEP_KERNEL lm::k_sweep<kSweepTile, kSweepRing, kSweepWarps, kSweepWcap>
#endif
// the round-1 sweep that also fills the resident key cache (opts.key_cache)
constexpr int kSweepThreads = Sweep::kThreads;
using SweepD = lm::SweepCfg<LM_SWEEP_TILE, LM_SWEEP_RING, LM_SWEEP_WARPS, LM_SWEEP_WCAP>;      // dense
using SweepS = lm::SweepCfg<LM_SWEEP_S_TILE, LM_SWEEP_RING, LM_SWEEP_S_WARPS, LM_SWEEP_S_WCAP>; // sparse
#ifndef LM_COMPACT_K
#define LM_COMPACT_K 8
#endif
constexpr int kCompactK = LM_COMPACT_K;  // items per lane per compaction chunk
#ifndef LM_COMPACT_K1
#define LM_COMPACT_K1 4  // the round-1 compaction (every non-empty row): 4 items per lane measured
#endif               // 0.646 vs 0.665 ms for round-1 match + compaction; later rounds keep 8
constexpr int kCompactK1 = LM_COMPACT_K1;
constexpr long long kLogCap = 1 << 16;  // per-round log rows kept on the device
// hybrid round loop: frontiers up to this size run in the persistent kernel
#ifndef LM_PERSIST_BELOW
#define LM_PERSIST_BELOW (1 << 16)
#endif
constexpr int64_t kPersistentBelow = LM_PERSIST_BELOW;
constexpr int64_t kHandoffRounds = 32;  // hybrid (algorithm 2): LD pointing phases before the Suitor tail
// frontier pointer kernels: lanes per vertex (G) and keys per lane per batch (U), per degree bin
#ifndef LM_B0_G
#define LM_B0_G 1
#define LM_B0_U 8
#endif
// measured at the end of round 1 (R-MAT s26, variants in one call): 32-lane bin U 4 -> 8 and
// 9..64-entry bin 8x8 -> 16x4 lanes x keys: rounds 8.35 -> 8.10 ms (U = 16: 9.08 ms; 4x16: 9.6 ms)
#ifndef LM_B1_G
#define LM_B1_G 16
#define LM_B1_U 4
#endif
#ifndef LM_CACHE_REFILL
#define LM_CACHE_REFILL 1  // out of core: refill a host row's cache when its cached keys run dry
#endif
#ifndef LM_BIN_STREAMS
#define LM_BIN_STREAMS 1  // frontier bins of a round on concurrent side streams (R-MAT s26 rounds 7.64 -> 7.50 ms)
#endif
#ifndef LM_CTA_U
#define LM_CTA_U 16  // keys per thread per batch in the CTA-per-row bin (4 -> 8 -> 16: rounds 7.73 -> 7.64 -> 7.60 ms)
#endif
#ifndef LM_B2_G
#define LM_B2_G 32
#define LM_B2_U 8
#endif

// host-driven rounds: software-pipelined pointer kernels (one resident wave) per bin: bit b of
// LM_PIPE set = bin b uses k_point_pipe<LM_Pb_G, LM_Pb_U>
#ifndef LM_PIPE
#define LM_PIPE 3  // bins 0 and 1 software-pipelined (k_point_pipe<1,8>, <8,4>); round 2, R-MAT s26, one box:
                   // 12.06 -> 11.89 ms against the 16 x 4 bin kernel (4 x 4: 11.89, 4 x 8: 11.95, 2 x 8: 11.97)
#endif
#ifndef LM_P0_G
#define LM_P0_G 1
#define LM_P0_U 8
#endif
#ifndef LM_P1_G
#define LM_P1_G 8
#define LM_P1_U 4
#endif
#ifndef LM_P2_G
#define LM_P2_G 32
#define LM_P2_U 4
#endif
// bit b of LM_ASYNC set = bin b uses k_point_async<LM_Ab_G, LM_Ab_U, LM_ASYNC_S> (resident
// adjacency only; takes precedence over LM_PIPE)
#ifndef LM_ASYNC
#define LM_ASYNC 0
#endif
#ifndef LM_ASYNC_S
#define LM_ASYNC_S 4
#endif
#ifndef LM_A0_G
#define LM_A0_G 1
#define LM_A0_U 8
#endif
#ifndef LM_A1_G
#define LM_A1_G 8
#define LM_A1_U 4
#endif
#ifndef LM_A2_G
#define LM_A2_G 32
#define LM_A2_U 4
#endif
#ifndef LM_PIPE_WAVES
#define LM_PIPE_WAVES 1
#endif
// 1 = the frontier pointer kernels are launched with a persisting L2 access-policy window over
// the matched bitmap (cudaLaunchAttributeAccessPolicyWindow; the device's persisting L2 set-aside
// is sized to the bitmap at create time), so the streamed row keys do not evict it
#ifndef LM_L2_WINDOW
#define LM_L2_WINDOW 0
#endif

constexpr int kFinBlocks = 2368;  // 16 x 148 SMs: fixed => deterministic fp64 summation order
constexpr int kFinThreads = 256;

}  // namespace

struct lmatch_graph {
  int device = 0;
  cudaStream_t stream = nullptr;   // handle stream
  cudaStream_t up[2] = {nullptr, nullptr};
  cudaStream_t bs[3] = {nullptr, nullptr, nullptr};  // side streams for the frontier bins
  cudaEvent_t ev_fork = nullptr, ev_join[3] = {nullptr, nullptr, nullptr};
  int64_t n = 0, m = 0, n_nz = 0, ntiles = 0;  // n, m: this handle's rows and entries
  // partitioned mode (lmatch_create_part): rows [v0, v0 + n) of a graph with n_global vertices
  int64_t v0 = 0, n_global = 0;
  int P = 1;
  int64_t* bounds = nullptr;         // device [P+1]
  uint32_t* ghost = nullptr;         // device [n_global]
  uint64_t* claims = nullptr;        // device [P * claim_cap]
  int64_t claim_cap = 0;
  unsigned long long* claim_cnt = nullptr;    // device [P]
  unsigned long long* h_claim_cnt = nullptr;  // pinned [P]
  int part_round = 0, part_cur = 0;
  std::vector<int64_t> hbounds;      // host copy of the part bounds [P+1]
  // peer-memory exchange (lmatch_p2p_*): window = inbox [P][win_cap] u64 | inbox counts [P] |
  // frontier-size slots [P] | barrier flags [P] | w(M) shares [P] | matched counts [P]; peers
  // store into it (and into `bits`) over NVLink / peer memory
  int p2p = 0, me = 0;
  int64_t win_cap = 0;
  uint64_t* win = nullptr;
  uint32_t* shadow = nullptr;        // owned bitmap words as last pushed to the peers
  uint64_t** d_dseg = nullptr;       // device [P]: my inbox segment in each peer's window
  unsigned long long** d_dcnt = nullptr;  // device [P]: its count
  uint32_t** d_dbits = nullptr;      // device [P]: each peer's bitmap replica
  unsigned long long** d_dnf = nullptr;   // device [P]: my frontier-size slot in each peer
  unsigned long long** d_dflag = nullptr;  // device [P]: my barrier flag in each peer (lmatch_run_dist)
  unsigned long long** d_dresw = nullptr;  // device [P]: my w(M) share slot in each peer
  unsigned long long** d_dresc = nullptr;  // device [P]: my matched-count slot in each peer
  std::vector<uint64_t*> h_dseg;
  std::vector<unsigned long long*> h_dcnt, h_dnf, h_dflag, h_dresw, h_dresc;
  // library-owned multi-GPU driver (lmatch_create_dist): device barrier epoch and error flag
  int dist = 0;
  int dist_local = 0;                // every rank in this process: event barriers (see barrier)
  void* dist_shm = nullptr;          // the rendezvous mapping (kept for in-process barriers)
  size_t dist_shm_bytes = 0;
  cudaEvent_t bev[2] = {nullptr, nullptr};
  unsigned long long epoch = 0;
  unsigned* d_berr = nullptr;
  unsigned long long* h_res6 = nullptr;  // pinned [3P]: frontier sizes, w shares, counts
  std::vector<uint32_t*> h_dbits;
  std::vector<void*> ipc_opened;     // peer allocations opened with cudaIpcOpenMemHandle
  unsigned long long* h_nf = nullptr;  // pinned [P]
  float part_sweep_ms = 0.f;  // (timing=1) last lmatch_part_begin's round-1 sweep
  bool sweep_ms_pending = false;  // its events are recorded, the time not read yet
  bool counts_on_host = false;    // peer-memory round: h_counters holds this set's bin sizes
  bool one_rank_loop = false;     // lmatch_run_dist with P = 1: h_counters is read back after every
                                  // compaction, so match and compaction launches are sized from it
  int validate_level = 1;
  int timing = 0;
  int64_t max_rounds = 0;
  int64_t upload_chunk = 1ll << 25;
  // out-of-core: entries [0, R) resident; [R, m) in pinned mapped host memory, streamed in round 1
  int64_t R = 0;
  int64_t stream_chunk = 1ll << 24;
  int64_t hbm_budget = 0;
  int batches = 0;                   // paper-style batch count (> 1: all streamed)
  int algorithm = 0;                 // 0 = LD pointer iteration, 1 = Suitor (NEXT-4), 3 = sorted+cursor
  int64_t sort_chunk = 1ll << 30;    // algorithm 3: entries per segmented-sort chunk
  // resident key cache (opts.key_cache): the 4 largest keys of every row, filled by the sweep
  int key_cache = 0;
  int kc_attr = 0;
  // A6 push frontier (persistent-kernel rounds; opts.frontier): newly matched vertices [n_nz + 1]
  int push_ok = 1;
  uint32_t* pushN = nullptr;
  int64_t cap_pushN = -1;
  uint64_t* kcache = nullptr;        // the active cache: kc_buf, or nullptr = off for this graph
  uint64_t* kc_buf = nullptr;        // [n + 1][kKC]
  uint64_t* xpart = nullptr;         // [ntiles][2][kKC] partial lists of tile-crossing rows
  int32_t* xrows = nullptr;          // nz index of every tile-crossing row
  unsigned long long* nx = nullptr;  // |xrows|
  int64_t cap_kc_buf = -1, cap_xpart = -1, cap_xrows = -1;
  bool sorted = false;               // algorithm 3: rows sorted by key, descending (NEXT-3)
  float ms_sort = 0.f;               // algorithm 3: device time of the last row sort
  uint32_t* sc_cur = nullptr;        // algorithm 3: per-vertex cursor (row-relative entry index)
  ulonglong2* sc_L[2] = {nullptr, nullptr};  // algorithm 3: live (u, pointer key) pairs
  uint64_t* sc_ptr = nullptr;        // algorithm 3: per-vertex pointer key (0 = none)
  uint64_t* suitor = nullptr;        // Suitor: best proposal received, (w << 32) | proposer
  uint32_t* wl[2] = {nullptr, nullptr};   // Suitor worklists
  uint32_t* wl_big = nullptr;             // Suitor: rows listed for the CTA scan
  unsigned long long* wl_cnt = nullptr;   // [0..1] worklist sizes, [2] big rows, [3] entries scanned
  bool streaming = false;
  uint64_t* host_adj = nullptr;      // pinned, mapped: entries [R, m)
  uint64_t* host_adj_dev = nullptr;  // its device alias
  uint64_t* ring[2] = {nullptr, nullptr};
  cudaStream_t cs = nullptr;         // copy stream for streaming
  // host-row key cache (NEXT-1): rows u >= u_first hold entries >= R; K keys per row in HBM,
  // addressed through AdjView as indices >= M0
  int host_cache = 1;
  uint64_t* cache = nullptr;
  int64_t cap_cache = -1;
  int64_t u_first = 0, M0 = 0, nchunks = 0;
  int64_t* chunk_rows = nullptr;     // device [nchunks + 1]: row holding each chunk's first entry
  int64_t cap_chunk_rows = -1;
  uint64_t* rescan = nullptr;        // device [n_hrows]: frontier entries whose cache ran dry
  unsigned long long* rescan_cnt = nullptr;
  int64_t cap_rescan = -1;
  int64_t* cache_big = nullptr;      // device [1 + cap]: count, then rows listed for the CTA fill
  int64_t cap_cache_big = -1;
  // residual rows (opts.residual_mb): HBM copies of rescanned host rows, roff[u - u_first] = their
  // start in `res` (-1 = not copied), addressed through AdjView as indices >= M2
  int residual_mb = 0;
  uint64_t* res = nullptr;
  int64_t cap_res = -1, M2 = INT64_MAX;
  unsigned long long* res_used = nullptr;
  int64_t* roff = nullptr;
  int64_t cap_roff = -1;
  bool use_cache() const { return streaming && cache != nullptr; }
  cudaEvent_t ev_full[2] = {}, ev_free[2] = {};
  int sweep_grid = 0;
  bool sweep_dense = true;   // round-1 sweep configuration: SweepD (true) or SweepS
  int64_t tile = 1024;       // its entries per tile
  alignas(64) CUtensorMap tmap;  // adjacency as a [ceil(m/16)][16] u64 tensor, 128B swizzle
  int num_sms = 148;
  cudaAccessPolicyWindow bits_window = {};  // LM_L2_WINDOW: the matched bitmap, persisting
  // graph
  int64_t* offs = nullptr;
  uint64_t* adj = nullptr;
  int64_t* noffs = nullptr;
  int32_t* nzr = nullptr;
  int32_t* tile_nz = nullptr;
  uint32_t* noffs_lo = nullptr;
  int32_t* atomic_rows = nullptr;
  int64_t n_atomic = 0;
  // capacities of the buffers sized by the graph's shape (non-empty rows, bins); a reload with a
  // different degree mix grows them and drops the captured CUDA graph
  int64_t cap_noffs = -1, cap_nzr = -1, cap_nlo = -1, cap_S[2] = {-1, -1};
  int64_t cap_bin[2][lm::kBins] = {{-1, -1, -1, -1, -1}, {-1, -1, -1, -1, -1}};   // .p arrays
  int64_t cap_binr[2][lm::kBins] = {{-1, -1, -1, -1, -1}, {-1, -1, -1, -1, -1}};  // .r arrays
  // state
  uint64_t* best = nullptr;
  uint32_t* bits = nullptr;
  uint64_t* S[2] = {nullptr, nullptr};      // stable live pairs (ping-pong)
  lm::Bins F[2] = {};                       // frontier degree bins (ping-pong), pairs
  unsigned long long* counters = nullptr;   // lm::kNumCounters
  unsigned long long* h_counters = nullptr;  // pinned mirror
  double* pw = nullptr;
  long long* pc = nullptr;
  double* res_w = nullptr;
  long long* res_c = nullptr;
  double* h_res = nullptr;  // pinned: [0] = w, [1] = c (as double bits... stored separately)
  long long* h_resc = nullptr;
  int32_t* mate_tmp = nullptr;
  lm::PackErr* perr = nullptr;
  unsigned* werr = nullptr;
  // upload staging
  int32_t* st_col[2] = {nullptr, nullptr};
  float* st_w[2] = {nullptr, nullptr};
  cudaEvent_t ev[8] = {};
  int64_t device_bytes = 0;
  std::vector<int64_t> round_log;  // per round: |F_r|, |L_r|, E(F_r) (directed entries scanned)
  // (timing=1) per-round events of the host-driven rounds >= 2 of the last run (lmatch_round_ms)
  std::vector<cudaEvent_t> rev;
  int64_t n_rev = 0, tail_rounds_from = -1;
  // device-side round loop
  lm::RoundState* rstate = nullptr;
  lm::RoundArgs* d_rargs = nullptr;    // device copy of rargs() (kernels read it by pointer)
  lm::RoundState* h_rstate = nullptr;  // pinned
  long long* rlog = nullptr;           // device [kLogCap][3]
  int round_loop = 0;                  // 0 = CUDA graph, 1 = host-driven
  int prune = 0;                       // A7 in-place pruning (resident, single-graph handles)
  uint32_t* live = nullptr;            // A7 live counts: tag << 16 | count
  cudaGraphExec_t gexec = nullptr;
  cudaGraph_t graph = nullptr;
  cudaStream_t gstream = nullptr;      // stream the graph was captured on (capture needs its own)

  lm::AdjView view() const {
    lm::AdjView v{adj, host_adj_dev - R, R};
    if (use_cache()) { v.cache_off = cache - M0; v.M0 = M0; }
    if (use_cache() && res) { v.res_off = res - M2; v.M2 = M2; }
    return v;
  }
  const lm::RoundArgs* ra() const { return d_rargs; }
  lm::RoundArgs rargs() const {
    lm::RoundArgs a;
    a.S[0] = S[0];
    a.S[1] = S[1];
    a.F[0] = F[0];
    a.F[1] = F[1];
    a.cnt = counters;
    a.st = rstate;
    a.log = rlog;
    a.live = prune ? live : nullptr;
    a.kc = kcache;
    a.best = best;
    a.N = (push_ok && !prune && algorithm != 2) ? pushN : nullptr;
    a.push_min_live = push_ok == 2 ? 0ull : lm::kPushMinLive;
    return a;
  }
};

namespace {

template <class T>
int dmalloc(lmatch_graph* g, T** p, size_t count) {
  size_t bytes = std::max<size_t>(count * sizeof(T), 16);
  cudaError_t e = cudaMalloc(reinterpret_cast<void**>(p), bytes);
  if (e != cudaSuccess) {
    set_err("cudaMalloc(%zu bytes): %s", bytes, cudaGetErrorString(e));
    *p = nullptr;
    return e == cudaErrorMemoryAllocation ? LMATCH_ENOMEM : LMATCH_ECUDA;
  }
  g->device_bytes += (int64_t)bytes;
  return LMATCH_OK;
}

void drop_graph(lmatch_graph* g);

// (re)allocate *p to hold `need` elements unless it already does; contents are not preserved
template <class T>
int ensure(lmatch_graph* g, T** p, int64_t* cap, int64_t need) {
  if (*p && *cap >= need) return LMATCH_OK;
  if (*p) {
    cudaFree(*p);
    g->device_bytes -= (int64_t)std::max<size_t>((size_t)*cap * sizeof(T), 16);
    *p = nullptr;
    drop_graph(g);
  }
  *cap = -1;
  TRY(dmalloc(g, p, (size_t)need));
  *cap = need;
  return LMATCH_OK;
}

void drop_graph(lmatch_graph* g) {
  if (g->gexec) cudaGraphExecDestroy(g->gexec);
  if (g->graph) cudaGraphDestroy(g->graph);
  g->gexec = nullptr;
  g->graph = nullptr;
}

// Rows crossing a sweep-tile boundary merge their per-tile maxima with atomicMax into best[].
// Zeroing those entries before every run is not needed (LM_XROW_RESET = 0): best[] is zeroed at
// create and reload, and every later write stores either 0 or a key of the vertex's own row, so
// the stale entry a run starts from is at most the row maximum and the atomicMax merge still
// yields exactly the row maximum (saves ~60 us of scattered writes per run at R-MAT s26).
#ifndef LM_XROW_RESET
#define LM_XROW_RESET 0
#endif
static int64_t xrow_resets(const lmatch_graph* g) { return LM_XROW_RESET ? g->n_atomic : 0; }

// ---- round-1 sweep launches in the handle's configuration (SweepD or SweepS)
template <class C, bool ZAP, bool KC>
static void sweep_launch_cfg(unsigned grid, cudaStream_t st, const lm::SweepArgs& A) {
  lm::k_sweep<C::kTile, C::kRing, C::kWarps, C::kWin, ZAP, KC><<<grid, C::kThreads, C::kSmem, st>>>(A);
}
template <bool ZAP, bool KC>
static void sweep_launch_any(const lmatch_graph* g, unsigned grid, cudaStream_t st, const lm::SweepArgs& A) {
  if (g->sweep_dense) sweep_launch_cfg<SweepD, ZAP, KC>(grid, st, A);
  else sweep_launch_cfg<SweepS, ZAP, KC>(grid, st, A);
}
static int sweep_warps(const lmatch_graph* g) { return g->sweep_dense ? SweepD::kWarps : SweepS::kWarps; }
// dynamic shared memory opt-in of every sweep instantiation (once per process)
template <class C>
static cudaError_t sweep_attrs_cfg() {
  cudaError_t e = cudaFuncSetAttribute(lm::k_sweep<C::kTile, C::kRing, C::kWarps, C::kWin, false, false>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::kSmem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(lm::k_sweep<C::kTile, C::kRing, C::kWarps, C::kWin, true, false>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::kSmem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(lm::k_sweep<C::kTile, C::kRing, C::kWarps, C::kWin, false, true>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::kSmem);
  return e;
}
static cudaError_t sweep_attrs() {
  cudaError_t e = sweep_attrs_cfg<SweepD>();
  return e == cudaSuccess ? sweep_attrs_cfg<SweepS>() : e;
}
static cudaError_t sweep_occupancy(const lmatch_graph* g, int* occ) {
  return g->sweep_dense
             ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(
                   occ, lm::k_sweep<SweepD::kTile, SweepD::kRing, SweepD::kWarps, SweepD::kWin, false, false>,
                   SweepD::kThreads, SweepD::kSmem)
             : cudaOccupancyMaxActiveBlocksPerMultiprocessor(
                   occ, lm::k_sweep<SweepS::kTile, SweepS::kRing, SweepS::kWarps, SweepS::kWin, false, false>,
                   SweepS::kThreads, SweepS::kSmem);
}

int grid_for(int64_t work, int threads, int max_blocks) {
  int64_t b = (work + threads - 1) / threads;
  if (b < 1) b = 1;
  if (b > max_blocks) b = max_blocks;
  return (int)b;
}

// launch with the bitmap's persisting L2 window (LM_L2_WINDOW), else a plain launch
template <typename... KArgs, typename... Args>
cudaError_t launch_pw(const lmatch_graph* g, void (*k)(KArgs...), unsigned grid, unsigned block,
                      cudaStream_t st, Args... args) {
#if LM_L2_WINDOW
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeAccessPolicyWindow;
  at[0].val.accessPolicyWindow = g->bits_window;
  cfg.attrs = at;
  cfg.numAttrs = g->bits_window.num_bytes > 0 ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, k, args...);
#else
  (void)g;
  k<<<grid, block, 0, st>>>(args...);
  return cudaGetLastError();
#endif
}

int check_args(const void* a, const void* b, const void* c, int64_t n, int64_t m) {
  if (n < 0 || m < 0) { set_err("negative n (%lld) or m (%lld)", (long long)n, (long long)m); return LMATCH_ERANGE; }
  if (n >= (int64_t)1 << 31) { set_err("n = %lld >= 2^31 (vertex ids are int32)", (long long)n); return LMATCH_ERANGE; }
  if (!a || (m > 0 && (!b || !c))) { set_err("NULL input array"); return LMATCH_EINVAL; }
  if (n == 0 && m > 0) { set_err("n == 0 with m > 0"); return LMATCH_EINVAL; }
  return LMATCH_OK;
}

int alloc_all(lmatch_graph* g) {
  const int64_t n = g->n, m = g->m;
#if LM_SWEEP_IMPL == 2
  g->sweep_dense = true;
  g->tile = kSweepTile;
#else
  // dense configuration when the average degree reaches LM_SWEEP_DENSE_DEG (rows per tile stay
  // within its row window); the local part of a partition handle decides for itself
  g->sweep_dense = n > 0 && m >= (int64_t)LM_SWEEP_DENSE_DEG * n;
  g->tile = g->sweep_dense ? SweepD::kTile : SweepS::kTile;
#endif
  const int64_t kTile = g->tile;
  TRY(dmalloc(g, &g->offs, (size_t)n + 1));
  // out-of-core split: keep a prefix of R entries (multiple of the stream chunk) in HBM
  g->R = m;
  if (g->batches > 1 && m > 0) {  // paper-style batches: nothing resident, B streamed batches
    g->stream_chunk = std::max<int64_t>(kTile, (m / g->batches + kTile - 1) / kTile * kTile);
    g->R = 0;
    g->streaming = true;
  } else if (g->hbm_budget > 0 && 8 * m > g->hbm_budget) {
    const int64_t C = std::max<int64_t>(kTile, (g->stream_chunk / kTile) * kTile);
    g->stream_chunk = C;
    g->R = std::max<int64_t>(0, (g->hbm_budget / 8 - 2 * C) / C * C);
    g->R = std::min(g->R, (m / C) * C);
    g->streaming = g->R < m;
  }
  TRY(dmalloc(g, &g->adj, (size_t)g->R + 32));
  // zero the padding past the resident part (tile reads round up to 16 bytes)
  CK(cudaMemsetAsync(g->adj + g->R, 0, 32 * sizeof(uint64_t), g->stream));
  if (g->streaming) {
    const size_t hb = ((size_t)(m - g->R) + 32) * 8;
    CK(cudaHostAlloc(reinterpret_cast<void**>(&g->host_adj), hb, cudaHostAllocMapped));
    std::memset(g->host_adj + (m - g->R), 0, 32 * 8);
    CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&g->host_adj_dev), g->host_adj, 0));
    for (int i = 0; i < 2; ++i) {
      TRY(dmalloc(g, &g->ring[i], (size_t)g->stream_chunk + 32));
      CK(cudaMemsetAsync(g->ring[i], 0, ((size_t)g->stream_chunk + 32) * 8, g->stream));
      CK(cudaEventCreateWithFlags(&g->ev_full[i], cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&g->ev_free[i], cudaEventDisableTiming));
    }
    CK(cudaStreamCreateWithFlags(&g->cs, cudaStreamNonBlocking));
  }
  // per non-empty row buffers (noffs, nzr, noffs_lo, S) are sized in build_index
  g->ntiles = (m + kTile - 1) / kTile;
  TRY(dmalloc(g, &g->tile_nz, (size_t)g->ntiles + 2));
  // a tile-crossing row is listed once per tile boundary it crosses: <= ntiles entries
  TRY(dmalloc(g, &g->atomic_rows, (size_t)g->ntiles + 1));
  TRY(dmalloc(g, &g->best, (size_t)n + 1));
  TRY(dmalloc(g, &g->bits, (size_t)((g->n_global + 31) / 32) + 1));
  TRY(dmalloc(g, &g->counters, lm::kNumCounters));
  TRY(dmalloc(g, &g->rstate, 1));
  CK(cudaMemsetAsync(g->rstate, 0, sizeof(lm::RoundState), g->stream));
  TRY(dmalloc(g, &g->d_rargs, 1));
  TRY(dmalloc(g, &g->rlog, 3 * (size_t)kLogCap + 3));
  CK(cudaHostAlloc(reinterpret_cast<void**>(&g->h_rstate), sizeof(lm::RoundState), cudaHostAllocDefault));
  TRY(dmalloc(g, &g->pw, kFinBlocks));
  TRY(dmalloc(g, &g->pc, kFinBlocks));
  TRY(dmalloc(g, &g->res_w, 1));
  TRY(dmalloc(g, &g->res_c, 1));
  TRY(dmalloc(g, &g->perr, 1));
  TRY(dmalloc(g, &g->werr, 2));
  CK(cudaHostAlloc(reinterpret_cast<void**>(&g->h_counters), lm::kNumCounters * 8, cudaHostAllocDefault));
  CK(cudaHostAlloc(reinterpret_cast<void**>(&g->h_res), 16, cudaHostAllocDefault));
  CK(cudaHostAlloc(reinterpret_cast<void**>(&g->h_resc), 16, cudaHostAllocDefault));
  // best[] = 0 for every vertex: empty rows are never written again (their pointer stays none)
  CK(cudaMemsetAsync(g->best, 0, ((size_t)n + 1) * 8, g->stream));
  return LMATCH_OK;
}

// Sweep index: non-empty rows (noffs, nzr) + tile -> first row.  Also validates offsets.
int build_index(lmatch_graph* g, cudaStream_t st) {
  const int64_t n = g->n, m = g->m;
  if (n == 0) {
    g->n_nz = 0;
    TRY(ensure(g, &g->noffs, &g->cap_noffs, 5));
    TRY(ensure(g, &g->nzr, &g->cap_nzr, 8));
    TRY(ensure(g, &g->noffs_lo, &g->cap_nlo, 9));
    for (int i = 0; i < 2; ++i) TRY(ensure(g, &g->S[i], &g->cap_S[i], 1));
    return LMATCH_OK;
  }
  const int64_t nb = (n + lm::kScanBlock - 1) / lm::kScanBlock;
  int64_t* bs = nullptr;
  int64_t* tot = nullptr;
  TRY(dmalloc(g, &bs, (size_t)nb + 1));
  TRY(dmalloc(g, &tot, 1));
  lm::k_nz_count<<<(unsigned)nb, lm::kScanThreads, 0, st>>>(g->offs, n, bs);
  CKL();
  lm::k_scan_blocksums<<<1, 1024, 0, st>>>(bs, nb, tot);
  CKL();
  int64_t h_tot = 0;
  CK(cudaMemcpyAsync(&h_tot, tot, 8, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  g->n_nz = h_tot;
  // sized by non-empty rows (R-MAT: ~45% of n); the +slack covers the sweep's TMA window reads,
  // which round a tile's row window [a, bp+2) out to 4-entry groups
  TRY(ensure(g, &g->noffs, &g->cap_noffs, h_tot + 5));
  TRY(ensure(g, &g->nzr, &g->cap_nzr, h_tot + 8));
  TRY(ensure(g, &g->noffs_lo, &g->cap_nlo, h_tot + 9));
  for (int i = 0; i < 2; ++i) TRY(ensure(g, &g->S[i], &g->cap_S[i], h_tot + 1));
  lm::k_nz_scatter<<<(unsigned)nb, lm::kScanThreads, 0, st>>>(g->offs, n, bs, g->nzr, g->noffs);
  CKL();
  CK(cudaMemcpyAsync(g->noffs + h_tot, &m, 8, cudaMemcpyHostToDevice, st));
  CK(cudaStreamSynchronize(st));
  if (g->ntiles > 0) {
    lm::k_tile_rows<<<grid_for(g->ntiles + 1, 256, 4096), 256, 0, st>>>(g->noffs, g->n_nz, g->ntiles,
                                                                        g->tile, g->tile_nz);
    CKL();
    lm::k_low32<<<grid_for(g->n_nz + 1, 256, 4096), 256, 0, st>>>(g->noffs, g->n_nz + 1, g->noffs_lo);
    CKL();
    unsigned long long* cnt = nullptr;
    TRY(dmalloc(g, &cnt, 1));
    CK(cudaMemsetAsync(cnt, 0, 8, st));
    lm::k_atomic_rows<<<grid_for(g->ntiles, 256, 4096), 256, 0, st>>>(
        g->noffs, g->nzr, g->tile_nz, g->ntiles, g->tile, g->atomic_rows, cnt);
    CKL();
    unsigned long long h_cnt = 0;
    CK(cudaMemcpyAsync(&h_cnt, cnt, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    g->n_atomic = (int64_t)h_cnt;
    cudaFree(cnt);
    g->device_bytes -= 16;
  }
  CK(cudaStreamSynchronize(st));
  cudaFree(bs);
  cudaFree(tot);
  g->device_bytes -= (int64_t)(nb + 1 + 1) * 8;
  return LMATCH_OK;
}

int check_offsets(lmatch_graph* g, cudaStream_t st) {
  if (g->n == 0) return LMATCH_OK;
  lm::k_check_offsets<<<grid_for(g->n, 256, 8192), 256, 0, st>>>(g->offs, g->n, g->m, g->perr);
  CKL();
  lm::PackErr h{};
  CK(cudaMemcpyAsync(&h, g->perr, sizeof h, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (h.bad_offsets != ULLONG_MAX) {
    set_err("invalid csr_offsets near row %llu (need offsets[0]=0, non-decreasing, offsets[n]=m)",
            h.bad_offsets);
    return LMATCH_EINVAL;
  }
  return LMATCH_OK;
}

int reset_err(lmatch_graph* g, cudaStream_t st) {
  lm::PackErr h{ULLONG_MAX, ULLONG_MAX};
  CK(cudaMemcpyAsync(g->perr, &h, sizeof h, cudaMemcpyHostToDevice, st));
  CK(cudaStreamSynchronize(st));
  return LMATCH_OK;
}

int64_t host_off(lmatch_graph* g, int64_t r, cudaStream_t st, int* err) {
  int64_t v = 0;
  if (cudaMemcpyAsync(&v, g->offs + r, 8, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
      cudaStreamSynchronize(st) != cudaSuccess) *err = 1;
  return v;
}

// Cut rows [0, n) into chunks of at most `cap` entries (a longer row is a chunk of its own):
// cuts[c] .. cuts[c+1]; *maxcnt / *maxrows = the largest chunk's entries / rows.
int row_chunks(lmatch_graph* g, cudaStream_t st, int64_t cap, std::vector<int64_t>* cuts,
               int64_t* maxcnt, int64_t* maxrows) {
  const int64_t n = g->n;
  int err = 0;
  *maxcnt = 0;
  *maxrows = 0;
  cuts->clear();
  const int64_t mtot = host_off(g, n, st, &err);
  for (int64_t r0 = 0; r0 < n;) {
    const int64_t b0 = host_off(g, r0, st, &err);
    int64_t lo = r0 + 1, hi = n;  // largest r1 with offs[r1] - b0 <= cap (at least one row)
    if (mtot - b0 <= cap) lo = n;
    else {
      while (lo < hi) {
        const int64_t mid = lo + (hi - lo + 1) / 2;
        if (host_off(g, mid, st, &err) - b0 <= cap) lo = mid; else hi = mid - 1;
      }
    }
    if (err) { set_err("offset read failed"); return LMATCH_ECUDA; }
    const int64_t cnt = host_off(g, lo, st, &err) - b0;
    if (cnt > INT_MAX) { set_err("row %lld has more than 2^31-1 entries", (long long)r0); return LMATCH_EINVAL; }
    cuts->push_back(r0);
    *maxcnt = std::max(*maxcnt, cnt);
    *maxrows = std::max(*maxrows, lo - r0);
    r0 = lo;
  }
  cuts->push_back(n);
  return err ? LMATCH_ECUDA : LMATCH_OK;
}

// validate_level 2, repeated edges ("duplicate edges with unequal weights" -> EINVAL):
// every row's (neighbour << 32 | weight bits) keys are sorted ascending in scratch memory, chunk by
// chunk, and neighbouring keys of one row with the same neighbour must be equal.  Exact.
constexpr int64_t kDupChunk = 1ll << 27;
int check_duplicates(lmatch_graph* g, cudaStream_t st) {
  if (g->n == 0 || g->m == 0) return LMATCH_OK;
  std::vector<int64_t> cuts;
  int64_t maxcnt = 0, maxrows = 0;
  TRY(row_chunks(g, st, std::min(g->m, std::min(kDupChunk, g->sort_chunk)), &cuts, &maxcnt, &maxrows));
  uint64_t *kin = nullptr, *kout = nullptr;
  int32_t* seg = nullptr;
  unsigned long long* bad = nullptr;
  void* tmp = nullptr;
  size_t tmp_bytes = 0, need = 0;
  int rc = LMATCH_OK;
  auto fail_alloc = [&](const char* what, size_t bytes) {
    cudaGetLastError();
    set_err("validate_level 2: cannot allocate %zu bytes (%s)", bytes, what);
    rc = LMATCH_ENOMEM;
  };
  const size_t kb = (size_t)std::max<int64_t>(maxcnt, 1) * 8;
  if (cudaMalloc(&kin, kb) != cudaSuccess) fail_alloc("row keys", kb);
  if (!rc && cudaMalloc(&kout, kb) != cudaSuccess) fail_alloc("sorted row keys", kb);
  if (!rc && cudaMalloc(&seg, (size_t)(maxrows + 1) * 4) != cudaSuccess) fail_alloc("segments", (size_t)(maxrows + 1) * 4);
  if (!rc && cudaMalloc(&bad, 8) != cudaSuccess) fail_alloc("flag", 8);
  if (!rc && cudaMemsetAsync(bad, 0xff, 8, st) != cudaSuccess) rc = LMATCH_ECUDA;
  int err = 0;
  for (size_t c = 0; rc == LMATCH_OK && c + 1 < cuts.size(); ++c) {
    const int64_t a = cuts[c], b = cuts[c + 1];
    const int64_t base = host_off(g, a, st, &err), cnt = host_off(g, b, st, &err) - base;
    if (err) { set_err("offset read failed"); rc = LMATCH_ECUDA; break; }
    if (cnt == 0) continue;
    lm::k_sc_seg_offsets<<<grid_for(b - a + 1, 256, 65536), 256, 0, st>>>(g->offs, a, b, seg);
    lm::k_dup_keys<<<grid_for(cnt, 256, 65536), 256, 0, st>>>(g->view(), base, cnt, kin);
    if (cudaGetLastError() != cudaSuccess) { set_err("duplicate check launch failed"); rc = LMATCH_ECUDA; break; }
    count_launches(2);
    if (cub::DeviceSegmentedSort::SortKeys(nullptr, need, kin, kout, (int)cnt, (int)(b - a), seg, seg + 1,
                                           st) != cudaSuccess) {
      set_err("duplicate check: sort sizing failed"); rc = LMATCH_ECUDA; break;
    }
    if (need > tmp_bytes) {
      if (tmp) cudaFree(tmp);
      tmp = nullptr;
      tmp_bytes = 0;
      if (cudaMalloc(&tmp, need) != cudaSuccess) { fail_alloc("sort temporary storage", need); break; }
      tmp_bytes = need;
    }
    if (cub::DeviceSegmentedSort::SortKeys(tmp, need, kin, kout, (int)cnt, (int)(b - a), seg, seg + 1,
                                           st) != cudaSuccess) {
      set_err("duplicate check: sort failed"); rc = LMATCH_ECUDA; break;
    }
    lm::k_dup_check<<<grid_for((b - a) * 8, 256, 16384), 256, 0, st>>>(kout, seg, b - a, a, bad);
    if (cudaGetLastError() != cudaSuccess) { set_err("duplicate check launch failed"); rc = LMATCH_ECUDA; break; }
    count_launches(1);
  }
  unsigned long long hbad = ULLONG_MAX;
  if (rc == LMATCH_OK && cudaMemcpyAsync(&hbad, bad, 8, cudaMemcpyDeviceToHost, st) != cudaSuccess) rc = LMATCH_ECUDA;
  const cudaError_t se = cudaStreamSynchronize(st);
  if (tmp) cudaFree(tmp);
  if (seg) cudaFree(seg);
  if (kin) cudaFree(kin);
  if (kout) cudaFree(kout);
  if (bad) cudaFree(bad);
  if (rc != LMATCH_OK) return rc;
  if (se != cudaSuccess) { set_err("duplicate check: %s", cudaGetErrorString(se)); return LMATCH_ECUDA; }
  if (hbad != ULLONG_MAX) {
    set_err("row %llu lists a neighbour twice with unequal weights", hbad);
    return LMATCH_EINVAL;
  }
  return LMATCH_OK;
}

int check_pack(lmatch_graph* g, cudaStream_t st) {
  lm::PackErr h{};
  CK(cudaMemcpyAsync(&h, g->perr, sizeof h, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (h.first_bad != ULLONG_MAX && g->validate_level >= 0) {
    set_err("invalid entry %llu: col out of [0,n) or weight not finite > 0", h.first_bad);
    return LMATCH_EINVAL;
  }
  if (g->validate_level >= 2 && g->n > 0) {
    unsigned long long* acc = nullptr;
    TRY(dmalloc(g, &acc, 1));
    CK(cudaMemsetAsync(acc, 0, 8, st));
    lm::k_symhash<<<grid_for(g->n * 8, 256, 8192), 256, 0, st>>>(g->offs, g->view(), g->n, acc);
    CKL();
    unsigned long long hv = 0;
    CK(cudaMemcpyAsync(&hv, acc, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    cudaFree(acc);
    g->device_bytes -= 16;
    if (hv != 0) {
      set_err("graph is not symmetric: multiset of (u,v,w) differs from (v,u,w)");
      return LMATCH_EINVAL;
    }
    TRY(check_duplicates(g, st));
  }
  return LMATCH_OK;
}

// Host arrays -> device: offsets in one copy; col/w in chunks through two staging buffers on two
// streams so the PCIe copy of chunk k+1 overlaps packing chunk k (LOADBATCH double buffering,
// Alg. 2 L4-5 P:115-116).
int upload_host(lmatch_graph* g, const int64_t* offsets, const int32_t* col, const float* w) {
  const int64_t n = g->n, m = g->m;
  TRY(reset_err(g, g->stream));
  CK(cudaMemcpyAsync(g->offs, offsets, ((size_t)n + 1) * 8, cudaMemcpyHostToDevice, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  if (g->validate_level >= 0) TRY(check_offsets(g, g->stream));
  const int64_t C = g->upload_chunk;
  if (m > 0 && !g->st_col[0]) {
    for (int i = 0; i < 2; ++i) {
      TRY(dmalloc(g, &g->st_col[i], (size_t)std::min(C, m)));
      TRY(dmalloc(g, &g->st_w[i], (size_t)std::min(C, m)));
    }
  }
  for (int64_t base = 0, k = 0; base < m; base += C, ++k) {
    const int64_t cnt = std::min(C, m - base);
    const int i = (int)(k & 1);
    cudaStream_t s = g->up[i];
    CK(cudaMemcpyAsync(g->st_col[i], col + base, (size_t)cnt * 4, cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(g->st_w[i], w + base, (size_t)cnt * 4, cudaMemcpyHostToDevice, s));
    // entries below R go to HBM, the rest to the pinned host copy (written through its alias)
    const int64_t nd = std::max<int64_t>(0, std::min(cnt, g->R - base));
    if (nd > 0) {
      lm::k_pack<<<grid_for(nd, 256, 16384), 256, 0, s>>>(g->st_col[i], g->st_w[i], nd, g->n_global,
                                                          g->adj + base, base, g->perr);
      CKL();
    }
    if (cnt > nd) {
      lm::k_pack<<<grid_for(cnt - nd, 256, 16384), 256, 0, s>>>(
          g->st_col[i] + nd, g->st_w[i] + nd, cnt - nd, g->n_global, g->host_adj_dev + (base + nd - g->R),
          base + nd, g->perr);
      CKL();
    }
  }
  CK(cudaStreamSynchronize(g->up[0]));
  CK(cudaStreamSynchronize(g->up[1]));
  TRY(check_pack(g, g->stream));
  return LMATCH_OK;
}

int upload_device(lmatch_graph* g, const int64_t* d_offsets, const int32_t* d_col,
                  const float* d_w, cudaStream_t st) {
  const int64_t n = g->n, m = g->m;
  TRY(reset_err(g, st));
  CK(cudaMemcpyAsync(g->offs, d_offsets, ((size_t)n + 1) * 8, cudaMemcpyDeviceToDevice, st));
  if (g->validate_level >= 0) TRY(check_offsets(g, st));
  if (m > 0) {
    const int64_t nd = std::min(m, g->R);
    if (nd > 0) {
      lm::k_pack<<<grid_for(nd, 256, 65536), 256, 0, st>>>(d_col, d_w, nd, g->n_global, g->adj, 0, g->perr);
      CKL();
    }
    if (m > nd) {
      lm::k_pack<<<grid_for(m - nd, 256, 65536), 256, 0, st>>>(d_col + nd, d_w + nd, m - nd, g->n_global,
                                                               g->host_adj_dev, nd, g->perr);
      CKL();
    }
  }
  TRY(check_pack(g, st));
  return LMATCH_OK;
}

#if LM_SWEEP_IMPL == 2
int make_tensor_map(lmatch_graph* g) {
  static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  if (!encode) {
    cudaDriverEntryPointQueryResult q;
    void* fn = nullptr;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    if (!fn || q != cudaDriverEntryPointSuccess) {
      set_err("cuTensorMapEncodeTiled unavailable");
      return LMATCH_ECUDA;
    }
    encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  }
  const cuuint64_t dims[2] = {16, (cuuint64_t)((g->m + 15) / 16)};
  const cuuint64_t strides[1] = {128};
  const cuuint32_t box[2] = {16, (cuuint32_t)(kSweepTile / 16)};
  const cuuint32_t es[2] = {1, 1};
  const CUresult r = encode(&g->tmap, CU_TENSOR_MAP_DATA_TYPE_UINT64, 2, g->adj, dims, strides, box,
                            es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_err("cuTensorMapEncodeTiled failed (%d)", (int)r);
    return LMATCH_ECUDA;
  }
  return LMATCH_OK;
}
#endif

// frontier bin lists: bin b can never hold more than the vertices of its degree class
int alloc_bins(lmatch_graph* g, cudaStream_t st) {
  unsigned long long* cnt = nullptr;
  TRY(dmalloc(g, &cnt, lm::kBins));
  CK(cudaMemsetAsync(cnt, 0, 8 * lm::kBins, st));
  if (g->n > 0) {
    lm::k_bin_sizes<<<grid_for(g->n, 256, 4096), 256, 0, st>>>(g->offs, g->n, cnt);
    CKL();
  }
  unsigned long long h[lm::kBins];
  CK(cudaMemcpyAsync(h, cnt, sizeof h, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  cudaFree(cnt);
  g->device_bytes -= 16;
  // A7 pruning moves rows to LOWER bins (live degrees only shrink): bin b must then hold every
  // row whose full degree is in bin b or above
  // the push frontier runs in the persistent kernel only (single graph or a one-rank partition)
  if (g->push_ok && !g->prune && g->algorithm != 2 && g->round_loop != 1 && !g->streaming && g->P == 1)
    TRY(ensure(g, &g->pushN, &g->cap_pushN, g->n_nz + 1));
  // the decided list (key cache only) can hold any non-empty row
  h[lm::kDecided] = 0;
  for (int b = 0; g->kcache && b < lm::kDegBins; ++b) h[lm::kDecided] += h[b];
  if (g->prune)
    for (int b = lm::kDegBins - 2; b >= 0; --b) h[b] += h[b + 1];
  for (int i = 0; i < 2; ++i)
    for (int b = 0; b < lm::kBins; ++b)
    {
      TRY(ensure(g, &g->F[i].list[b].p, &g->cap_bin[i][b], (int64_t)h[b] + 1));
      TRY(ensure(g, &g->F[i].list[b].r, &g->cap_binr[i][b], (int64_t)h[b] + 1));
    }
  const lm::RoundArgs a = g->rargs();
  CK(cudaMemcpy(g->d_rargs, &a, sizeof a, cudaMemcpyHostToDevice));
  return LMATCH_OK;
}

// Out-of-core host-row cache (NEXT-1): chunk k of the streamed part covers entries
// [R + k C, min(R + (k+1) C, m)); chunk_rows[k] = row holding its first entry, chunk_rows[nchunks]
// = row holding entry m - 1.  Host rows are u >= u_first = chunk_rows[0], kCacheK slots each.
int build_cache_index(lmatch_graph* g, cudaStream_t st) {
  if (!g->streaming || !g->host_cache || g->n == 0 || g->m == 0) {
    g->M0 = 0;
    return LMATCH_OK;
  }
  const int64_t C = g->stream_chunk;
  g->nchunks = (g->m - g->R + C - 1) / C;
  TRY(ensure(g, &g->chunk_rows, &g->cap_chunk_rows, g->nchunks + 1));
  lm::k_rows_of_entries<<<grid_for(g->nchunks + 1, 256, 4096), 256, 0, st>>>(
      g->offs, g->n, g->R, C, g->m - 1, g->nchunks + 1, g->chunk_rows);
  CKL();
  int64_t uf = 0;
  CK(cudaMemcpyAsync(&uf, g->chunk_rows, 8, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  g->u_first = uf;
  TRY(ensure(g, &g->cache, &g->cap_cache, (g->n - uf) * lm::kCacheK));
  TRY(ensure(g, &g->rescan, &g->cap_rescan, g->n - uf + 1));
  if (!g->rescan_cnt) TRY(dmalloc(g, &g->rescan_cnt, 1));
  // a window holds at most (entries / kCacheBigRow) rows longer than kCacheBigRow
  TRY(ensure(g, &g->cache_big, &g->cap_cache_big, std::max(C, g->R) / lm::kCacheBigRow + 8));
  g->M0 = g->m + 64;  // past the host part and its padding
  // residual rows: a buffer of up to residual_mb MiB (leaving 1 GiB of free memory), reset per
  // loaded graph; the copies persist across runs on the same graph
  if (g->residual_mb > 0) {
    size_t fr = 0, tot = 0;
    CK(cudaMemGetInfo(&fr, &tot));
    int64_t want = (int64_t)g->residual_mb * (1ll << 20) / 8;
    if (g->res && g->cap_res >= want) want = g->cap_res;
    const int64_t room = ((int64_t)fr - (1ll << 30)) / 8 + (g->res ? g->cap_res : 0);
    want = std::min(want, room);
    if (want > 0) {
      TRY(ensure(g, &g->res, &g->cap_res, want));
      TRY(ensure(g, &g->roff, &g->cap_roff, g->n - uf + 1));
      if (!g->res_used) TRY(dmalloc(g, &g->res_used, 1));
      CK(cudaMemsetAsync(g->res_used, 0, 8, st));
      CK(cudaMemsetAsync(g->roff, 0xff, (size_t)(g->n - uf + 1) * 8, st));
      g->M2 = g->M0 + g->cap_cache;
    }
  }
  return LMATCH_OK;
}

#ifndef LM_MAXL1
#define LM_MAXL1 0  // 1 = prefer the maximum L1 carveout for the frontier pointer kernels
#endif
static int prefer_l1() {
#if LM_MAXL1
  static bool done = false;
  if (done) return LMATCH_OK;
  done = true;
  const int c = cudaSharedmemCarveoutMaxL1;
  CK(cudaFuncSetAttribute(lm::k_point_bin<LM_B1_G, LM_B1_U>, cudaFuncAttributePreferredSharedMemoryCarveout, c));
  CK(cudaFuncSetAttribute(lm::k_point_bin<LM_B2_G, LM_B2_U>, cudaFuncAttributePreferredSharedMemoryCarveout, c));
  CK(cudaFuncSetAttribute(lm::k_point_pipe<LM_P0_G, LM_P0_U>, cudaFuncAttributePreferredSharedMemoryCarveout, c));
  CK(cudaFuncSetAttribute(lm::k_point_bin_cta<256, LM_CTA_U>, cudaFuncAttributePreferredSharedMemoryCarveout, c));
#endif
  return LMATCH_OK;
}

// Resident key cache (opts.key_cache): allocated for resident handles running the LD iteration
// when it fits in free device memory (with 1 GiB to spare); the list of tile-crossing rows it
// merges after the sweep is built here.  Off otherwise (kcache = nullptr).
int setup_key_cache(lmatch_graph* g, cudaStream_t st) {
  const bool want = g->key_cache && !g->streaming && (g->algorithm == 0 || g->algorithm == 2) &&
                    g->n > 0 && g->ntiles > 0 && LM_SWEEP_IMPL == 1;
  g->kcache = nullptr;  // buffers of an earlier graph stay allocated for a later reload
  if (!want) return LMATCH_OK;
  const int64_t need_kc = (g->n + 1) * lm::kKC, need_xp = g->ntiles * 2 * lm::kKC + 8;
  int64_t extra = 0;
  if (!(g->kc_buf && g->cap_kc_buf >= need_kc)) extra += need_kc * 8;
  if (!(g->xpart && g->cap_xpart >= need_xp)) extra += need_xp * 8;
  if (!(g->xrows && g->cap_xrows >= g->ntiles + 1)) extra += (g->ntiles + 1) * 4;
  size_t fr = 0, tot = 0;
  CK(cudaMemGetInfo(&fr, &tot));
  if ((size_t)extra + (1ull << 30) > fr) return LMATCH_OK;
  TRY(ensure(g, &g->kc_buf, &g->cap_kc_buf, need_kc));
  g->kcache = g->kc_buf;
  TRY(ensure(g, &g->xpart, &g->cap_xpart, need_xp));
  TRY(ensure(g, &g->xrows, &g->cap_xrows, g->ntiles + 1));
  if (!g->nx) TRY(dmalloc(g, &g->nx, 1));
  CK(cudaMemsetAsync(g->nx, 0, 8, st));
  lm::k_kc_xrows<<<grid_for((g->n_nz + 31) & ~31ll, 256, 8192), 256, 0, st>>>(g->noffs, g->n_nz, g->tile,
                                                                              g->xrows, g->nx);
  CKL();
  if (!g->kc_attr) {
    CK(sweep_attrs());
    g->kc_attr = 1;
  }
  return LMATCH_OK;
}

int finish_create(lmatch_graph* g, cudaStream_t st) {
  TRY(prefer_l1());
#if LM_L2_WINDOW
  {
    int maxp = 0, maxw = 0;
    CK(cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, g->device));
    CK(cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, g->device));
    const size_t bytes = (size_t)((g->n_global + 31) / 32) * 4;
    if (maxp > 0 && maxw > 0 && bytes > 0) {
      size_t limit = 0;
      CK(cudaDeviceGetLimit(&limit, cudaLimitPersistingL2CacheSize));
      if (limit < std::min(bytes, (size_t)maxp))
        CK(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, std::min(bytes, (size_t)maxp)));
      CK(cudaDeviceGetLimit(&limit, cudaLimitPersistingL2CacheSize));
      g->bits_window.base_ptr = g->bits;
      g->bits_window.num_bytes = std::min(bytes, (size_t)maxw);
      g->bits_window.hitRatio = std::min(1.0f, (float)limit / (float)g->bits_window.num_bytes);
      g->bits_window.hitProp = cudaAccessPropertyPersisting;
      g->bits_window.missProp = cudaAccessPropertyStreaming;
    }
  }
#endif
  if (g->prune && (g->streaming || g->ghost)) g->prune = 0;  // resident single-graph only
  if (g->prune && !g->live) {
    TRY(dmalloc(g, &g->live, (size_t)g->n + 1));
    CK(cudaMemsetAsync(g->live, 0, ((size_t)g->n + 1) * 4, st));
  }
  g->sorted = false;  // (re)loaded adjacency: algorithm 3 sorts it again on the next run
  // best[] = 0 for every vertex: the sweep writes non-empty rows only, so a row that is empty in
  // a reloaded graph must not keep the pointer of the previous graph (Suitor's first pass and the
  // partitioned claims read best[] of every vertex)
  CK(cudaMemsetAsync(g->best, 0, ((size_t)g->n + 1) * 8, st));
  TRY(build_index(g, st));
  TRY(setup_key_cache(g, st));
  TRY(alloc_bins(g, st));
  TRY(build_cache_index(g, st));
  if (g->m > 0) {
    // self-loop keys -> 0: the sweep's tile pass over resident graphs, the row-based
    // kernel over out-of-core ones (rows may live in host memory)
    CK(cudaMemsetAsync(g->werr, 0, 8, st));
    unsigned long long* zc = reinterpret_cast<unsigned long long*>(g->werr);
    if (!g->streaming && g->ntiles > 0) {
      CK(sweep_attrs());
      const int64_t grid = std::max<int64_t>(1, std::min<int64_t>((g->ntiles + sweep_warps(g) - 1) / sweep_warps(g),
                                                                  3 * (int64_t)g->num_sms));
      lm::SweepArgs A{g->adj, g->adj, zc, (uint32_t)g->v0, g->noffs_lo, g->nzr, g->tile_nz, g->best, g->m, 0, g->ntiles};
      sweep_launch_any<true, false>(g, (unsigned)grid, st, A);
      CKL();
    } else {
      lm::k_zap_self_loops<<<grid_for(g->n * 8, 256, 16384), 256, 0, st>>>(g->offs, g->view(), g->n,
                                                                           g->v0, zc);
      CKL();
    }
  }
#if LM_SWEEP_IMPL == 2
  if (g->streaming) { set_err("LM_SWEEP_IMPL=2 does not support out-of-core graphs"); return LMATCH_EINVAL; }
  if (g->ntiles > 0) TRY(make_tensor_map(g));
#endif
  if (g->ntiles > 0) {
    int occ = 0;
#if LM_SWEEP_IMPL == 2
    CK(cudaFuncSetAttribute(SWEEP_KERNEL,
                            cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Sweep::kSmem));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(
        &occ, SWEEP_KERNEL, kSweepThreads, Sweep::kSmem));
#else
    CK(sweep_attrs());
    CK(sweep_occupancy(g, &occ));
#endif
    if (occ < 1) occ = 1;
    g->sweep_grid = (int)std::min<int64_t>((g->ntiles + sweep_warps(g) - 1) / sweep_warps(g),
                                           (int64_t)occ * g->num_sms);
  }
  CK(cudaStreamSynchronize(st));
  return LMATCH_OK;
}

struct PartSpec {
  int64_t v0 = 0, n_global = -1;
  int P = 1;
  const int64_t* bounds = nullptr;  // host [P+1]
};

int create_common(int64_t n, int64_t m, const lmatch_opts* opts, lmatch_graph** out,
                  lmatch_graph** gp, const PartSpec* part = nullptr) {
  lmatch_graph* g = new (std::nothrow) lmatch_graph();
  if (!g) { set_err("host allocation failed"); return LMATCH_ENOMEM; }
  *gp = g;
  g->n = n;
  g->m = m;
  g->n_global = n;
  if (part) {
    g->v0 = part->v0;
    g->n_global = part->n_global;
    g->P = part->P;
    g->hbounds.assign(part->bounds, part->bounds + part->P + 1);
  }
  if (opts) {
    if (opts->use_device) CK(cudaSetDevice(opts->device));
    if (opts->validate_level != 0) g->validate_level = opts->validate_level;
    g->timing = opts->timing;
    g->max_rounds = opts->max_rounds;
    if (opts->upload_chunk > 0) g->upload_chunk = (opts->upload_chunk + 3) & ~3ll;
    g->hbm_budget = opts->hbm_budget_bytes;
    if (opts->stream_chunk > 0) g->stream_chunk = opts->stream_chunk;
    g->round_loop = opts->round_loop;
    g->prune = opts->prune != 0;
    g->host_cache = opts->host_cache >= 0;
    g->batches = opts->batches;
    g->algorithm = opts->algorithm;
    g->key_cache = opts->key_cache > 0;
    g->residual_mb = opts->residual_mb;
    g->push_ok = opts->frontier == 1 ? 0 : (opts->frontier == 2 ? 2 : 1);
    if (opts->sort_chunk_log2 != 0) {
      if (opts->sort_chunk_log2 < 4 || opts->sort_chunk_log2 > 30) {
        set_err("sort_chunk_log2 = %d outside 4..30", opts->sort_chunk_log2);
        return LMATCH_EINVAL;
      }
      g->sort_chunk = 1ll << opts->sort_chunk_log2;
    }
  }
  CK(cudaGetDevice(&g->device));
  CK(cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, g->device));
  // the strict order bounds the pointing phases by n/2 + 1 (R6) -- of the WHOLE graph
  // for a partition handle, whose rounds are the global ones
  if (g->max_rounds <= 0) g->max_rounds = g->n_global / 2 + 2;
  CK(cudaStreamCreateWithFlags(&g->stream, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&g->up[0], cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&g->up[1], cudaStreamNonBlocking));
  if (LM_BIN_STREAMS) {
    for (int i = 0; i < 3; ++i) {
      CK(cudaStreamCreateWithFlags(&g->bs[i], cudaStreamNonBlocking));
      CK(cudaEventCreateWithFlags(&g->ev_join[i], cudaEventDisableTiming));
    }
    CK(cudaEventCreateWithFlags(&g->ev_fork, cudaEventDisableTiming));
  }
  for (auto& e : g->ev) CK(cudaEventCreate(&e));
  TRY(alloc_all(g));
  if (part) {
    TRY(dmalloc(g, &g->bounds, (size_t)g->P + 1));
    CK(cudaMemcpy(g->bounds, part->bounds, ((size_t)g->P + 1) * 8, cudaMemcpyHostToDevice));
    // one part: nothing is remote, so no ghosts and no claims are ever stored (minimal buffers;
    // the handle still counts as a partition handle)
    TRY(dmalloc(g, &g->ghost, g->P > 1 ? (size_t)g->n_global + 1 : 2));
    g->claim_cap = g->P > 1 ? std::max<int64_t>(n, 1) : 1;
    TRY(dmalloc(g, &g->claims, (size_t)g->P * (size_t)g->claim_cap));
    TRY(dmalloc(g, &g->claim_cnt, (size_t)g->P));
    CK(cudaHostAlloc(reinterpret_cast<void**>(&g->h_claim_cnt), (size_t)g->P * 8, cudaHostAllocDefault));
  }
  (void)out;
  return LMATCH_OK;
}

// Round-1 pointer sweep (A2) over every local row: resident tiles, then (out-of-core) the
// streamed chunks through a 2-slot device ring -- the copy of chunk k+1 on the copy stream
// overlaps the sweep of chunk k on the run stream (LOADBATCH double buffering).
int round1_sweep(lmatch_graph* g, cudaStream_t st, int64_t* launches_out, int64_t* sweep_out,
                 int64_t* streamed_out) {
  int64_t launches = 0, sweep_launches = 0, bytes_streamed = 0;
#if LM_SWEEP_IMPL == 2
  lm::Sweep2DArgs A{g->noffs_lo, g->nzr, g->tile_nz, g->best, g->m, g->ntiles};
  SWEEP_KERNEL<<<g->sweep_grid, kSweepThreads, Sweep::kSmem, st>>>(g->tmap, A);
  CKL();
  ++launches;
  ++sweep_launches;
#else
  // resident tiles [0, R/TILE), then the streamed chunks through a 2-slot device ring:
  // the copy of chunk k+1 (copy stream) overlaps the sweep of chunk k (run stream).
  const int64_t rt = g->streaming ? g->R / g->tile : g->ntiles;
  auto sweep_launch = [&](const uint64_t* base, int64_t t0, int64_t t1) -> int {
    const int64_t grid = std::min<int64_t>((t1 - t0 + sweep_warps(g) - 1) / sweep_warps(g), g->sweep_grid);
    lm::SweepArgs A{base, nullptr, nullptr, 0u, g->noffs_lo, g->nzr, g->tile_nz, g->best, g->m, t0, t1};
    if (g->kcache) {
      A.kc = g->kcache;
      A.xpart = g->xpart;
      sweep_launch_any<false, true>(g, (unsigned)std::max<int64_t>(grid, 1), st, A);
    } else {
      sweep_launch_any<false, false>(g, (unsigned)std::max<int64_t>(grid, 1), st, A);
    }
    CKL();
    ++launches;
    ++sweep_launches;
    return LMATCH_OK;
  };
  if (rt > 0) TRY(sweep_launch(g->adj, 0, std::min(rt, g->ntiles)));
  if (g->kcache && rt > 0) {
    // the rows crossing a tile boundary: merge their per-tile top-4 lists (also their pointer)
    lm::k_kc_merge<<<(unsigned)(8 * g->num_sms), 256, 0, st>>>(g->xrows, g->nx, g->noffs, g->nzr, g->xpart,
                                                               g->tile, g->kcache, g->best);
    CKL();
    ++launches;
  }
  // host-row cache fill over entries [w0, w1) held at base[j - ebase], rows [*plo, *phi]
  auto cache_fill = [&](const uint64_t* base, int64_t ebase, int64_t w0, int64_t w1,
                        const int64_t* plo, const int64_t* phi) -> int {
    unsigned long long* nbig = reinterpret_cast<unsigned long long*>(g->cache_big);
    CK(cudaMemsetAsync(nbig, 0, 8, st));
    lm::k_cache_fill<lm::kCacheK><<<(unsigned)(8 * g->num_sms), 256, 0, st>>>(
        base, ebase, w0, w1, g->offs, plo, phi, g->u_first, g->cache, g->cache_big + 1, nbig);
    CKL();
    lm::k_cache_fill_big<lm::kCacheK><<<(unsigned)g->num_sms, 256, 0, st>>>(
        base, ebase, w0, w1, g->offs, g->cache_big + 1, nbig, g->u_first, g->cache);
    CKL();
    launches += 2;
    return LMATCH_OK;
  };
  // the row holding entry R may start in the resident prefix: its resident part first
  if (g->use_cache() && g->R > 0) TRY(cache_fill(g->adj, 0, 0, g->R, g->chunk_rows, g->chunk_rows));
  if (g->streaming) {
    const int64_t C = g->stream_chunk;
    for (int64_t e0 = g->R, k = 0; e0 < g->m; e0 += C, ++k) {
      const int slot = (int)(k & 1);
      const int64_t cnt = std::min(C, g->m - e0);
      if (k >= 2) CK(cudaStreamWaitEvent(g->cs, g->ev_free[slot], 0));
      CK(cudaMemcpyAsync(g->ring[slot], g->host_adj + (e0 - g->R), (size_t)cnt * 8,
                         cudaMemcpyHostToDevice, g->cs));
      CK(cudaEventRecord(g->ev_full[slot], g->cs));
      bytes_streamed += cnt * 8;
      CK(cudaStreamWaitEvent(st, g->ev_full[slot], 0));
      TRY(sweep_launch(g->ring[slot], e0 / g->tile, std::min(g->ntiles, (e0 + cnt + g->tile - 1) / g->tile)));
      if (g->use_cache())
        TRY(cache_fill(g->ring[slot], e0, e0, e0 + cnt, g->chunk_rows + k, g->chunk_rows + k + 1));
      CK(cudaEventRecord(g->ev_free[slot], st));
    }
  }
#endif
  *launches_out += launches;
  *sweep_out += sweep_launches;
  *streamed_out += bytes_streamed;
  return LMATCH_OK;
}

}  // namespace

// ============================================================================ public ABI
extern "C" {

int lmatch_abi_version(void) { return LMATCH_ABI_VERSION; }

int64_t lmatch_kernel_launch_count(void) { return (int64_t)g_launch_count.load(); }
int32_t lmatch_sweep_tile(const lmatch_graph* g) { return g ? (int32_t)g->tile : (int32_t)SweepD::kTile; }

const char* lmatch_strerror(int status) {
  switch (status) {
    case LMATCH_OK: return "ok";
    case LMATCH_EINVAL: return "invalid argument / malformed graph";
    case LMATCH_ERANGE: return "size out of range";
    case LMATCH_ENOMEM: return "out of memory";
    case LMATCH_ECUDA: return "CUDA error";
    case LMATCH_ENCCL: return "NCCL error";
    case LMATCH_ESTATE: return "invalid state";
    case LMATCH_EROUNDS: return "round cap reached before the matching was maximal";
    default: return "unknown status";
  }
}

const char* lmatch_last_error(void) { return g_err; }

void lmatch_destroy(lmatch_graph* g) {
  if (!g) return;
  cudaSetDevice(g->device);
  if (g->stream) cudaStreamSynchronize(g->stream);
  void* dev[] = {g->offs, g->adj, g->noffs, g->nzr, g->tile_nz, g->noffs_lo, g->atomic_rows, g->best,
                 g->bits, g->S[0], g->S[1],
                 g->counters, g->pw, g->pc, g->res_w, g->res_c, g->mate_tmp, g->perr, g->werr,
                 g->st_col[0], g->st_col[1], g->st_w[0], g->st_w[1]};
  for (void* p : dev) if (p) cudaFree(p);
  for (auto& F : g->F)
    for (auto& l : F.list) {
      if (l.p) cudaFree(l.p);
      if (l.r) cudaFree(l.r);
    }
  if (g->h_counters) cudaFreeHost(g->h_counters);
  if (g->host_adj) cudaFreeHost(g->host_adj);
  for (int i = 0; i < 2; ++i) {
    if (g->ring[i]) cudaFree(g->ring[i]);
    if (g->ev_full[i]) cudaEventDestroy(g->ev_full[i]);
    if (g->ev_free[i]) cudaEventDestroy(g->ev_free[i]);
  }
  if (g->cs) cudaStreamDestroy(g->cs);
  if (g->gexec) cudaGraphExecDestroy(g->gexec);
  if (g->graph) cudaGraphDestroy(g->graph);
  if (g->gstream) cudaStreamDestroy(g->gstream);
  if (g->h_rstate) cudaFreeHost(g->h_rstate);
  for (void* p : g->ipc_opened) cudaIpcCloseMemHandle(p);
  if (g->h_nf) cudaFreeHost(g->h_nf);
  if (g->h_res6) cudaFreeHost(g->h_res6);
  if (g->dist_shm) munmap(g->dist_shm, g->dist_shm_bytes);
  for (auto e : g->bev) if (e) cudaEventDestroy(e);
  void* pdev[] = {g->bounds, g->ghost, g->claims, g->claim_cnt, g->rstate, g->rlog, g->d_rargs,
                  g->cache, g->chunk_rows, g->cache_big, g->rescan, g->rescan_cnt, g->live, g->win, g->suitor, g->wl[0],
                  g->wl[1], g->wl_big, g->wl_cnt, g->sc_cur, g->sc_ptr, g->sc_L[0], g->sc_L[1], g->shadow, g->d_dseg, g->d_dcnt,
                  g->d_dbits, g->d_dnf, g->d_dflag, g->d_dresw, g->d_dresc, g->d_berr,
                  g->kc_buf, g->xpart, g->xrows, g->nx, g->res, g->res_used, g->roff, g->pushN};
  for (void* p : pdev) if (p) cudaFree(p);
  if (g->h_claim_cnt) cudaFreeHost(g->h_claim_cnt);
  if (g->h_res) cudaFreeHost(g->h_res);
  if (g->h_resc) cudaFreeHost(g->h_resc);
  for (auto e : g->ev) if (e) cudaEventDestroy(e);
  for (auto e : g->rev) if (e) cudaEventDestroy(e);
  if (g->stream) cudaStreamDestroy(g->stream);
  for (auto s : g->up) if (s) cudaStreamDestroy(s);
  for (auto s : g->bs) if (s) cudaStreamDestroy(s);
  for (auto e : g->ev_join) if (e) cudaEventDestroy(e);
  if (g->ev_fork) cudaEventDestroy(g->ev_fork);
  delete g;
}

int lmatch_create_ex(const int64_t* csr_offsets, const int32_t* col_idx, const float* weights,
                     int64_t n, int64_t m, const lmatch_opts* opts, lmatch_graph** out) {
  if (!out) { set_err("out == NULL"); return LMATCH_EINVAL; }
  *out = nullptr;
  g_err[0] = 0;
  int s = check_args(csr_offsets, col_idx, weights, n, m);
  if (s) return s;
  lmatch_graph* g = nullptr;
  s = create_common(n, m, opts, out, &g);
  if (!s) s = upload_host(g, csr_offsets, col_idx, weights);
  if (!s) s = finish_create(g, g->stream);
  if (s) { lmatch_destroy(g); return s; }
  *out = g;
  return LMATCH_OK;
}

int lmatch_create(const int64_t* csr_offsets, const int32_t* col_idx, const float* weights,
                  int64_t n, int64_t m, lmatch_graph** out) {
  return lmatch_create_ex(csr_offsets, col_idx, weights, n, m, nullptr, out);
}

int lmatch_create_device(const int64_t* d_offsets, const int32_t* d_col, const float* d_weights,
                         int64_t n, int64_t m, const lmatch_opts* opts, void* stream,
                         lmatch_graph** out) {
  if (!out) { set_err("out == NULL"); return LMATCH_EINVAL; }
  *out = nullptr;
  g_err[0] = 0;
  int s = check_args(d_offsets, d_col, d_weights, n, m);
  if (s) return s;
  lmatch_graph* g = nullptr;
  s = create_common(n, m, opts, out, &g);
  cudaStream_t st = stream ? (cudaStream_t)stream : (g ? g->stream : nullptr);
  if (!s) {
    // order the caller's stream (which produced the arrays) before our reads
    cudaError_t e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) { set_err("stream sync: %s", cudaGetErrorString(e)); s = LMATCH_ECUDA; }
  }
  if (!s) s = upload_device(g, d_offsets, d_col, d_weights, st);
  if (!s) s = finish_create(g, st);
  if (s) { lmatch_destroy(g); return s; }
  *out = g;
  return LMATCH_OK;
}

int lmatch_reload(lmatch_graph* g, const int64_t* csr_offsets, const int32_t* col_idx,
                  const float* weights) {
  if (!g) { set_err("NULL handle"); return LMATCH_ESTATE; }
  g_err[0] = 0;
  int s = check_args(csr_offsets, col_idx, weights, g->n, g->m);
  if (s) return s;
  CK(cudaSetDevice(g->device));
  TRY(upload_host(g, csr_offsets, col_idx, weights));
  TRY(finish_create(g, g->stream));
  return LMATCH_OK;
}

int lmatch_round_log(const lmatch_graph* g, int64_t* out, int64_t cap, int64_t* nrounds) {
  if (!g) { set_err("NULL handle"); return LMATCH_ESTATE; }
  const int64_t r = (int64_t)g->round_log.size() / 3;
  if (nrounds) *nrounds = r;
  if (out)
    for (int64_t i = 0; i < std::min<int64_t>(3 * r, 3 * cap); ++i) out[i] = g->round_log[(size_t)i];
  return LMATCH_OK;
}

int lmatch_push_rounds(const lmatch_graph* g, int64_t* push_rounds) {
  if (!g || !push_rounds) { set_err("NULL argument"); return LMATCH_ESTATE; }
  *push_rounds = g->h_counters ? (int64_t)g->h_counters[lm::kCntPushRounds] : 0;
  return LMATCH_OK;
}

int lmatch_round_ms(const lmatch_graph* g, double* ms, int64_t cap, int64_t* nrounds,
                    int64_t* tail_from) {
  if (!g) { set_err("NULL handle"); return LMATCH_ESTATE; }
  const int64_t r = g->n_rev > 1 ? g->n_rev - 1 : 0;
  if (nrounds) *nrounds = r;
  if (tail_from) *tail_from = g->tail_rounds_from;
  for (int64_t i = 0; ms && i < std::min(r, cap); ++i) {
    float x = 0.f;
    CK(cudaEventElapsedTime(&x, g->rev[(size_t)i], g->rev[(size_t)i + 1]));
    ms[i] = x;
  }
  return LMATCH_OK;
}

int lmatch_info(const lmatch_graph* g, int64_t* n, int64_t* m, int64_t* nonempty_rows,
                int64_t* device_bytes) {
  if (!g) { set_err("NULL handle"); return LMATCH_ESTATE; }
  if (n) *n = g->n;
  if (m) *m = g->m;
  if (nonempty_rows) *nonempty_rows = g->n_nz;
  if (device_bytes) *device_bytes = g->device_bytes;
  return LMATCH_OK;
}

// ---- the launch sequence of one run (shared by the host-driven loop and the CUDA graph)
static int seq_prefix(lmatch_graph* g, cudaStream_t st, cudaGraphConditionalHandle h, int in_graph,
                      int64_t* launches, int64_t* sweep_launches, int64_t* bytes_streamed) {
  const int64_t n = g->n;
  const int64_t nwords = (g->n_global + 31) / 32;
  const bool work = g->ntiles > 0 && n > 0;
  lm::k_reset<<<grid_for(std::max(nwords, xrow_resets(g)), 256, 4096), 256, 0, st>>>(
      g->bits, nwords, g->best, g->atomic_rows, xrow_resets(g), g->counters, lm::kNumCounters,
      g->prune ? g->live : nullptr, g->n, g->rstate);
  CKL();
  // hybrid (algorithm 2): the LD iteration stops after kHandoffRounds pointing phases and
  // lmatch_run_device hands the rest to Suitor
  const int64_t rcap = g->algorithm == 2 && !g->streaming ? std::min<int64_t>(g->max_rounds, kHandoffRounds)
                                                          : g->max_rounds;
  lm::k_round_init<<<1, 1, 0, st>>>(g->rstate, rcap, kLogCap, work ? 1 : 0);
  CKL();
  *launches += 2;
  // phase events (inside a graph they become event-record nodes)
  cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
  CK(cudaStreamIsCapturing(st, &cap));
  auto mark = [&](int i) -> int {
    if (g->timing) {
      if (cap == cudaStreamCaptureStatusActive)
        CK(cudaEventRecordWithFlags(g->ev[i], st, cudaEventRecordExternal));
      else
        CK(cudaEventRecord(g->ev[i], st));
    }
    return LMATCH_OK;
  };
  TRY(mark(1));
  if (!work) {
    if (in_graph) {
      lm::k_end_round<<<1, 32, 0, st>>>(g->ra(), h, 1, 0);  // cont = 0
      CKL();
    }
    TRY(mark(2));
    TRY(mark(3));
    return LMATCH_OK;
  }
  // round 1: A2 full sweep (no bitmap test), A4 match-all, A6 compact-all
  TRY(round1_sweep(g, st, launches, sweep_launches, bytes_streamed));
  TRY(mark(2));
  lm::k_match_all<<<grid_for((nwords + LM_MATCHALL_V - 1) / LM_MATCHALL_V * 32, 256, 65536), 256, 0, st>>>(g->best, n, g->bits);
  CKL();
  // round-1 compaction: input set 1 (unused), output set 0; k_end_round makes set 0 current.
  // Items are the non-empty rows (nzr): empty rows never hold a pointer.
  {
    lm::CompactIO io = lm::compact_io(g->rargs(), 1);
    io.nzr = g->nzr;
    io.noffs = g->noffs;
    const unsigned grid = grid_for((g->n_nz + 31) / 32, 8 * kCompactK1, 65536);
    if (g->kcache)
      lm::k_compact<true, kCompactK1, true><<<grid, 256, 0, st>>>(io, g->n_nz, g->best, g->bits, g->offs, g->v0);
    else
      lm::k_compact<true, kCompactK1, false><<<grid, 256, 0, st>>>(io, g->n_nz, g->best, g->bits, g->offs, g->v0);
  }
  CKL();
  lm::k_end_round<<<1, 32, 0, st>>>(g->ra(), h, in_graph, 0);
  CKL();
  *launches += 3;
  TRY(mark(3));
  return LMATCH_OK;
}

// rounds >= 2, host-driven: A2 frontier pointers, A4, A6, end of round, with the current set
// `cur` and its sizes known on the host (grids fit the work; empty bins are skipped).
static int seq_body(lmatch_graph* g, cudaStream_t st, int cur, const int64_t* nFb, int64_t nS,
                    int64_t* launches) {
  const lm::AdjView av = g->view();
  const lm::Bins& Fb = g->F[cur];
  const unsigned long long* cF = g->counters + lm::cnt_F(cur, 0);
  int64_t nF = 0;
  for (int b = 0; b < lm::kBins; ++b) nF += nFb[b];
  if (g->use_cache() && nF > 0) {
    const bool refill = LM_CACHE_REFILL != 0;
    if (refill) CK(cudaMemsetAsync(g->rescan_cnt, 0, 8, st));
    lm::k_cache_redirect<lm::kCacheK><<<grid_for(nF, 256, 65536), 256, 0, st>>>(
        Fb, cF, g->offs, g->cache, g->bits, g->u_first, g->M0, g->v0, g->counters + lm::kCntCache,
        refill ? g->rescan : nullptr, refill ? g->rescan_cnt : nullptr, g->res ? g->roff : nullptr, g->M2);
    CKL();
    ++*launches;
    if (refill) {
      lm::k_host_rescan<lm::kCacheK><<<(unsigned)(8 * g->num_sms), 256, 0, st>>>(
          Fb, g->rescan, g->rescan_cnt, g->offs, g->view(), g->bits, g->cache, g->u_first, g->M0,
          g->v0, g->res, g->cap_res, g->res_used, g->roff);
      CKL();
      ++*launches;
    }
  }
#define PIPE_OR_BIN(b, PG, PU, BG, BU, AG, AU)                                                      \
  if (nFb[b]) {                                                                                   \
    if (g->prune) {                                                                               \
      lm::k_point_bin<BG, BU, true><<<grid_for(nFb[b] * BG, 256, 65536), 256, 0, st>>>(           \
          Fb.list[b], cF + b, g->offs, av, g->bits, g->best, g->v0, g->live, g->rstate);          \
    } else if ((LM_ASYNC & (1 << b)) && !g->streaming) {                                          \
      constexpr size_t smem = (size_t)LM_ASYNC_S * AU * 256 * 8;                                  \
      static int occ = 0;                                                                         \
      if (!occ) {                                                                                 \
        CK(cudaFuncSetAttribute(lm::k_point_async<AG, AU, LM_ASYNC_S>,                            \
                                cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));         \
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, lm::k_point_async<AG, AU, LM_ASYNC_S>, 256, smem)); \
        if (occ < 1) occ = 1;                                                                     \
      }                                                                                           \
      const int64_t wave = (int64_t)occ * g->num_sms;                                             \
      lm::k_point_async<AG, AU, LM_ASYNC_S><<<(unsigned)std::min<int64_t>(wave, (nFb[b] * AG + 255) / 256), 256, smem, st>>>( \
          Fb.list[b], cF + b, g->offs, g->adj, g->bits, g->best, g->v0);                          \
    } else if (LM_PIPE & (1 << b)) {                                                              \
      static int occ = 0;                                                                         \
      if (!occ) {                                                                                 \
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, lm::k_point_pipe<PG, PU>, 256, 0)); \
        if (occ < 1) occ = 1;                                                                     \
      }                                                                                           \
      const int64_t wave = (int64_t)occ * g->num_sms * LM_PIPE_WAVES;                              \
      CK(launch_pw(g, lm::k_point_pipe<PG, PU>, (unsigned)std::min<int64_t>(wave, (nFb[b] * PG + 255) / 256), \
                   256, st, Fb.list[b], cF + b, (const int64_t*)g->offs, av, (const uint32_t*)g->bits, \
                   g->best, g->v0));                                                              \
    } else {                                                                                      \
      CK(launch_pw(g, lm::k_point_bin<BG, BU, false>, (unsigned)grid_for(nFb[b] * BG, 256, 65536), 256, st, \
                   Fb.list[b], cF + b, (const int64_t*)g->offs, av, (const uint32_t*)g->bits, g->best, \
                   g->v0, (uint32_t*)nullptr, (const lm::RoundState*)nullptr));                 \
    }                                                                                             \
    CKL();                                                                                        \
    ++*launches;                                                                                  \
  }
  // the bins of a round are independent (disjoint rows, read-only bitmap): with LM_BIN_STREAMS
  // the 16-lane, 32-lane and CTA bins run on side streams next to the thread bin, so the tail
  // of one kernel overlaps the others; the match waits for all of them
  const int nbusy = (nFb[0] > 0) + (nFb[1] > 0) + (nFb[2] > 0) + (nFb[3] > 0);
  const bool fork = LM_BIN_STREAMS && g->bs[0] && nbusy > 1;
  if (fork) {
    CK(cudaEventRecord(g->ev_fork, st));
    for (int i = 0; i < 3; ++i) CK(cudaStreamWaitEvent(g->bs[i], g->ev_fork, 0));
  }
  {
    cudaStream_t st_main = st;
    {
      cudaStream_t st = fork ? g->bs[0] : st_main;
      PIPE_OR_BIN(1, LM_P1_G, LM_P1_U, LM_B1_G, LM_B1_U, LM_A1_G, LM_A1_U)
    }
    {
      cudaStream_t st = fork ? g->bs[1] : st_main;
      PIPE_OR_BIN(2, LM_P2_G, LM_P2_U, LM_B2_G, LM_B2_U, LM_A2_G, LM_A2_U)
    }
    {
      cudaStream_t st = fork ? g->bs[2] : st_main;
      if (nFb[3]) {
        CK(launch_pw(g, lm::k_point_bin_cta<256, LM_CTA_U>, (unsigned)std::min<int64_t>(nFb[3], 65536), 256, st,
                     Fb.list[3], cF + 3, (const int64_t*)g->offs, av, (const uint32_t*)g->bits, g->best, g->v0));
        CKL();
        ++*launches;
      }
    }
  }
  PIPE_OR_BIN(0, LM_P0_G, LM_P0_U, LM_B0_G, LM_B0_U, LM_A0_G, LM_A0_U)
#undef PIPE_OR_BIN
  if (fork) {
    for (int i = 0; i < 3; ++i) {
      CK(cudaEventRecord(g->ev_join[i], g->bs[i]));
      CK(cudaStreamWaitEvent(st, g->ev_join[i], 0));
    }
  }
  lm::k_match_bins<<<grid_for((nF + LM_MATCH_V - 1) / LM_MATCH_V, 256, 65536), 256, 0, st>>>(Fb, cF, g->best, g->bits);
  CKL();
  {
    const unsigned grid = grid_for((nS + nF + 31) / 32, 8 * kCompactK, 65536);
    const lm::CompactIO io = lm::compact_io(g->rargs(), cur);
    if (g->kcache)
      lm::k_compact<false, kCompactK, true><<<grid, 256, 0, st>>>(io, g->n, g->best, g->bits, g->offs, g->v0);
    else
      lm::k_compact<false, kCompactK, false><<<grid, 256, 0, st>>>(io, g->n, g->best, g->bits, g->offs, g->v0);
  }
  CKL();
  lm::k_end_round<<<1, 32, 0, st>>>(g->ra(), 0, 0, 0);
  CKL();
  *launches += 3;
  return LMATCH_OK;
}

#define PERSISTENT_KERNEL(PR, KC) \
  lm::k_rounds_persistent<LM_B0_G, LM_B0_U, LM_B1_G, LM_B1_U, LM_B2_G, LM_B2_U, kCompactK, PR, KC>

// rounds >= 2 in one cooperative launch (grid = co-resident blocks)
extern "C++" {
template <bool PRUNE, bool KC>
int launch_persistent_t(lmatch_graph* g, cudaStream_t st, int64_t* launches) {
  static int occ = 0;
  if (!occ) {
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, PERSISTENT_KERNEL(PRUNE, KC), 256, 0));
    if (occ < 1) occ = 1;
  }
  const lm::RoundArgs* ra = g->ra();
  const lm::AdjView av = g->view();
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(occ * g->num_sms));
  cfg.blockDim = dim3(256);
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  attr[1].id = cudaLaunchAttributeAccessPolicyWindow;
  attr[1].val.accessPolicyWindow = g->bits_window;
  cfg.attrs = attr;
  cfg.numAttrs = (LM_L2_WINDOW && g->bits_window.num_bytes > 0) ? 2 : 1;
  CK(cudaLaunchKernelEx(&cfg, PERSISTENT_KERNEL(PRUNE, KC), ra, (const int64_t*)g->offs, av, g->bits,
                        g->best, g->n, g->v0));
  count_launches(1);
  ++*launches;
  return LMATCH_OK;
}
}  // extern "C++"
static int launch_persistent(lmatch_graph* g, cudaStream_t st, int64_t* launches) {
  if (g->kcache)
    return g->prune ? launch_persistent_t<true, true>(g, st, launches)
                    : launch_persistent_t<false, true>(g, st, launches);
  return g->prune ? launch_persistent_t<true, false>(g, st, launches)
                  : launch_persistent_t<false, false>(g, st, launches);
}

// Capture reset .. round 1 + the persistent round kernel into one CUDA graph (built once).
static int build_graph_persistent(lmatch_graph* g) {
  if (!g->gstream) CK(cudaStreamCreateWithFlags(&g->gstream, cudaStreamNonBlocking));
  cudaStream_t s = g->gstream;
  int64_t l = 0, sl = 0, bs = 0;
  CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeRelaxed));
  int rc = seq_prefix(g, s, 0, 0, &l, &sl, &bs);
  if (!rc) rc = launch_persistent(g, s, &l);
  cudaGraph_t graph = nullptr;
  const cudaError_t e = cudaStreamEndCapture(s, &graph);
  if (rc) { if (graph) cudaGraphDestroy(graph); return rc; }
  if (e != cudaSuccess) { set_err("end capture: %s", cudaGetErrorString(e)); return LMATCH_ECUDA; }
  g->graph = graph;
  CK(cudaGraphInstantiate(&g->gexec, g->graph, 0));
  return LMATCH_OK;
}

static int ensure_suitor(lmatch_graph* g) {
  if (g->suitor) return LMATCH_OK;
  const int64_t n = g->n;
  TRY(dmalloc(g, &g->suitor, (size_t)n + 1));
  TRY(dmalloc(g, &g->wl[0], (size_t)n + 1));
  TRY(dmalloc(g, &g->wl[1], (size_t)n + 1));
  TRY(dmalloc(g, &g->wl_big, (size_t)(g->m / lm::kSuitorBig) + 2));  // rows longer than kSuitorBig
  TRY(dmalloc(g, &g->wl_cnt, 4));
  return LMATCH_OK;
}

// Suitor passes over the worklist wl[0] (size wl_cnt[0]) until no proposer is left; each pass
// scans the proposers' rows (lane / warp / listed CTA per row) and proposes with atomicMax.
static int suitor_loop(lmatch_graph* g, cudaStream_t st, int64_t* launches, int64_t* passes) {
  int cur = 0;
  unsigned long long* hc = g->h_counters;
  for (;;) {
    CK(cudaMemcpyAsync(hc, g->wl_cnt, 4 * 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    const int64_t c = (int64_t)hc[cur];
    if (c == 0) break;
    if (*passes >= g->max_rounds) {
      set_err("Suitor: %lld proposers left after the pass cap (%lld)", (long long)c, (long long)g->max_rounds);
      return LMATCH_EROUNDS;
    }
    unsigned long long* nc = g->wl_cnt + (cur ^ 1);
    CK(cudaMemsetAsync(nc, 0, 8, st));
    CK(cudaMemsetAsync(g->wl_cnt + 2, 0, 8, st));
    lm::k_suitor_scan<<<grid_for(c, 256, 65536), 256, 0, st>>>(
        g->wl[cur], g->wl_cnt + cur, g->offs, g->adj, g->suitor, g->wl[cur ^ 1], nc, g->wl_big,
        g->wl_cnt + 2, g->wl_cnt + 3);
    CKL();
    lm::k_suitor_scan_big<<<(unsigned)(2 * g->num_sms), 256, 0, st>>>(
        g->wl_big, g->wl_cnt + 2, g->offs, g->adj, g->suitor, g->wl[cur ^ 1], nc, g->wl_cnt + 3);
    CKL();
    *launches += 2;
    ++*passes;
    cur ^= 1;
  }
  // leave the final (empty) list in slot 0 for the next call
  if (cur) CK(cudaMemsetAsync(g->wl_cnt, 0, 2 * 8, st));
  return LMATCH_OK;
}

// Suitor (NEXT-4): reset, the round-1 sweep (pass 1 proposes to every row maximum), then
// host-driven passes over the worklist of proposers without a standing proposal.
static int run_suitor(lmatch_graph* g, int32_t* d_mate, cudaStream_t st, lmatch_stats* stats) {
  const int64_t n = g->n;
  const bool tm = g->timing && stats;
  TRY(ensure_suitor(g));
  int64_t launches = 0, sweep_launches = 0, bytes_streamed = 0, passes = 0;
  if (tm) CK(cudaEventRecord(g->ev[0], st));
  CK(cudaMemsetAsync(g->suitor, 0, ((size_t)n + 1) * 8, st));
  CK(cudaMemsetAsync(g->wl_cnt, 0, 4 * 8, st));
  lm::k_reset<<<grid_for(std::max<int64_t>(xrow_resets(g), 1), 256, 4096), 256, 0, st>>>(
      g->bits, 0, g->best, g->atomic_rows, xrow_resets(g), g->counters, lm::kNumCounters, nullptr, 0,
      g->rstate);
  CKL();
  ++launches;
  if (tm) CK(cudaEventRecord(g->ev[1], st));
  const bool work = g->ntiles > 0 && n > 0;
  if (work) TRY(round1_sweep(g, st, &launches, &sweep_launches, &bytes_streamed));
  if (tm) CK(cudaEventRecord(g->ev[2], st));
  if (work) {
    lm::k_suitor_first<<<grid_for(n, 256, 65536), 256, 0, st>>>(g->best, n, g->suitor, g->wl[0],
                                                                  g->wl_cnt + 0);
    CKL();
    ++launches;
    passes = 1;
  }
  if (tm) CK(cudaEventRecord(g->ev[3], st));
  unsigned long long* hc = g->h_counters;
  if (work) TRY(suitor_loop(g, st, &launches, &passes));
  if (tm) CK(cudaEventRecord(g->ev[4], st));
  if (n > 0) {
    lm::k_suitor_finish<kFinThreads><<<kFinBlocks, kFinThreads, 0, st>>>(g->suitor, n, d_mate, g->pw, g->pc);
    CKL();
    lm::k_final_sum<<<1, 32, 0, st>>>(g->pw, g->pc, kFinBlocks, g->res_w, g->res_c);
    CKL();
    launches += 2;
    CK(cudaMemcpyAsync(g->h_res, g->res_w, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(g->h_resc, g->res_c, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(hc, g->wl_cnt, 4 * 8, cudaMemcpyDeviceToHost, st));
  } else {
    g->h_res[0] = 0.0;
    g->h_resc[0] = 0;
  }
  if (tm) CK(cudaEventRecord(g->ev[5], st));
  CK(cudaStreamSynchronize(st));
  g->round_log.clear();
  if (stats) {
    std::memset(stats, 0, sizeof *stats);
    stats->rounds = passes;
    stats->matched_vertices = g->h_resc[0];
    stats->cardinality = g->h_resc[0] / 2;
    stats->weight = g->h_res[0];
    stats->entries_swept = (work ? g->m : 0) + (n > 0 ? (int64_t)hc[3] : 0);
    stats->sweep_launches = sweep_launches;
    stats->kernel_launches = launches;
    stats->resident_entries = g->R;
    if (tm) {
      float a = 0, b = 0, c = 0, d = 0, e = 0;
      CK(cudaEventElapsedTime(&a, g->ev[0], g->ev[5]));
      CK(cudaEventElapsedTime(&b, g->ev[1], g->ev[2]));
      CK(cudaEventElapsedTime(&c, g->ev[2], g->ev[3]));
      CK(cudaEventElapsedTime(&d, g->ev[3], g->ev[4]));
      CK(cudaEventElapsedTime(&e, g->ev[4], g->ev[5]));
      stats->ms_total = a;
      stats->ms_sweep = b;
      stats->ms_round1_rest = c;
      stats->ms_rounds = d;
      stats->ms_finish = e;
    }
  }
  return LMATCH_OK;
}


// ---- algorithm 3 (NEXT-3): sort every row by key, descending, in place.  Rows are grouped into
// chunks of at most g->sort_chunk entries (cub's segmented sort takes int sizes; a longer row is a
// chunk of its own), each sorted into a scratch buffer sized for the largest chunk and copied back.
// Done once per loaded graph; the time goes to lmatch_stats.ms_sort.
static int sort_rows(lmatch_graph* g, cudaStream_t st) {
  const int64_t n = g->n, m = g->m;
  CK(cudaEventRecord(g->ev[6], st));
  if (m > 0 && n > 0) {
    int err = 0;
    const int64_t cap = std::min<int64_t>(m, g->sort_chunk);
    // cut pass: rows [cuts[c], cuts[c+1]) = the longest run of rows within cap entries (at least
    // one row); the scratch buffer is sized for the largest chunk
    std::vector<int64_t> cuts;
    int64_t maxcnt = 0, maxrows = 0;
    TRY(row_chunks(g, st, cap, &cuts, &maxcnt, &maxrows));
    uint64_t* alt = nullptr;
    int32_t* seg = nullptr;
    void* tmp = nullptr;
    size_t tmp_bytes = 0, need = 0;
    int rc = LMATCH_OK;
    if (cudaMalloc(&alt, (size_t)std::max<int64_t>(maxcnt, 1) * 8) != cudaSuccess) {
      cudaGetLastError();
      set_err("sorted LD: cannot allocate %lld bytes of sort scratch (largest chunk %lld entries)",
              (long long)(std::max<int64_t>(maxcnt, 1) * 8), (long long)maxcnt);
      return LMATCH_ENOMEM;
    }
    if (cudaMalloc(&seg, (size_t)(maxrows + 1) * 4) != cudaSuccess) {
      cudaGetLastError();
      set_err("sorted LD: cannot allocate %lld bytes of segment offsets", (long long)((maxrows + 1) * 4));
      rc = LMATCH_ENOMEM;
    }
    for (size_t c = 0; rc == LMATCH_OK && c + 1 < cuts.size(); ++c) {
      const int64_t a = cuts[c], b = cuts[c + 1];
      const int64_t base = host_off(g, a, st, &err), cnt = host_off(g, b, st, &err) - base;
      if (err) { set_err("offset read failed"); rc = LMATCH_ECUDA; break; }
      if (cnt == 0) continue;
      lm::k_sc_seg_offsets<<<grid_for(b - a + 1, 256, 65536), 256, 0, st>>>(g->offs, a, b, seg);
      if (cudaGetLastError() != cudaSuccess) { set_err("segment offsets launch failed"); rc = LMATCH_ECUDA; break; }
      count_launches(1);
      if (cub::DeviceSegmentedSort::SortKeysDescending(nullptr, need, g->adj + base, alt, (int)cnt,
                                                       (int)(b - a), seg, seg + 1, st) != cudaSuccess) {
        set_err("segmented sort sizing failed"); rc = LMATCH_ECUDA; break;
      }
      if (need > tmp_bytes) {
        if (tmp) cudaFree(tmp);
        tmp = nullptr;
        tmp_bytes = 0;
        if (cudaMalloc(&tmp, need) != cudaSuccess) {
          cudaGetLastError();
          set_err("sorted LD: cannot allocate %zu bytes of sort temporary storage", need);
          rc = LMATCH_ENOMEM;
          break;
        }
        tmp_bytes = need;
      }
      if (cub::DeviceSegmentedSort::SortKeysDescending(tmp, need, g->adj + base, alt, (int)cnt,
                                                       (int)(b - a), seg, seg + 1, st) != cudaSuccess ||
          cudaMemcpyAsync(g->adj + base, alt, (size_t)cnt * 8, cudaMemcpyDeviceToDevice, st) != cudaSuccess) {
        set_err("segmented sort failed"); rc = LMATCH_ECUDA; break;
      }
    }
    const cudaError_t se = cudaStreamSynchronize(st);
    if (tmp) cudaFree(tmp);
    if (seg) cudaFree(seg);
    cudaFree(alt);
    if (rc != LMATCH_OK) return rc;
    if (se != cudaSuccess) { set_err("row sort: %s", cudaGetErrorString(se)); return LMATCH_ECUDA; }
  }
  CK(cudaEventRecord(g->ev[7], st));
  CK(cudaEventSynchronize(g->ev[7]));
  CK(cudaEventElapsedTime(&g->ms_sort, g->ev[6], g->ev[7]));
  g->sorted = true;
  return LMATCH_OK;
}

#ifndef LM_SC_POINT_BPS
#define LM_SC_POINT_BPS 32  // rounds >= 2 point kernel: blocks per SM (4 and 442 measured slower)
#endif
static unsigned sc_grid(const lmatch_graph* g, int64_t work) {
  const int64_t per = (int64_t)lm::kScThreads * lm::kScItems;
  return (unsigned)std::max<int64_t>(1, std::min<int64_t>((work + per - 1) / per, 16ll * g->num_sms));
}

// algorithm 3: round 1 points every vertex at its first available entry, then host-driven rounds
// over the live list (point, match) until it is empty; mate[] and w(M) as for Suitor.
static int run_sorted(lmatch_graph* g, int32_t* d_mate, cudaStream_t st, lmatch_stats* stats) {
  const int64_t n = g->n;
  const bool tm = g->timing && stats;
  bool sorted_now = false;
  if (!g->sorted) { TRY(sort_rows(g, st)); sorted_now = true; }
  TRY(ensure_suitor(g));
  if (!g->sc_cur) {
    TRY(dmalloc(g, &g->sc_cur, (size_t)n + 1));
    TRY(dmalloc(g, &g->sc_ptr, (size_t)n + 1));
    TRY(dmalloc(g, &g->sc_L[0], (size_t)n + 1));
    TRY(dmalloc(g, &g->sc_L[1], (size_t)n + 1));
  }
  int64_t launches = 0, rounds = 0;
  unsigned long long* hc = g->h_counters;
  if (tm) CK(cudaEventRecord(g->ev[0], st));
  CK(cudaMemsetAsync(g->suitor, 0, ((size_t)n + 1) * 8, st));
  CK(cudaMemsetAsync(g->bits, 0, (size_t)((n + 31) / 32) * 4, st));
  CK(cudaMemsetAsync(g->wl_cnt, 0, 4 * 8, st));
  CK(cudaMemsetAsync(g->sc_cur, 0, ((size_t)n + 1) * 4, st));
  if (tm) CK(cudaEventRecord(g->ev[1], st));
  int cur = 0;
  const bool work = g->ntiles > 0 && n > 0;
  if (work) {
    lm::k_sc_point<<<grid_for(n, 256, 65536), 256, 0, st>>>(nullptr, nullptr, n, g->offs, g->adj,
                                                             g->sc_cur, g->bits, g->sc_ptr, nullptr,
                                                             nullptr, g->wl_cnt + 2);
    CKL();
    if (tm) CK(cudaEventRecord(g->ev[2], st));
    lm::k_sc_match<<<sc_grid(g, n), lm::kScThreads, 0, st>>>(nullptr, nullptr, n, g->sc_ptr, g->bits,
                                                             g->suitor, g->sc_L[0], g->wl_cnt + 0);
    CKL();
    launches += 2;
    rounds = 1;
  } else if (tm) {
    CK(cudaEventRecord(g->ev[2], st));
  }
  if (tm) CK(cudaEventRecord(g->ev[3], st));
  for (;;) {
    if (!work) break;
    CK(cudaMemcpyAsync(hc, g->wl_cnt, 4 * 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    const int64_t c = (int64_t)hc[cur];
    if (c == 0) break;
    if (rounds >= g->max_rounds) {
      set_err("sorted LD: %lld vertices still to re-point after the round cap (%lld)", (long long)c,
              (long long)g->max_rounds);
      return LMATCH_EROUNDS;
    }
    CK(cudaMemsetAsync(g->wl_cnt + (cur ^ 1), 0, 8, st));
    CK(cudaMemsetAsync(g->wl_cnt + 3, 0, 8, st));
    lm::k_sc_point<<<grid_for(c, 256, LM_SC_POINT_BPS * g->num_sms), 256, 0, st>>>(g->sc_L[cur], g->wl_cnt + cur, 0, g->offs,
                                                             g->adj, g->sc_cur, g->bits, g->sc_ptr,
                                                             g->wl[0], g->wl_cnt + 3, g->wl_cnt + 2);
    CKL();
    lm::k_sc_point_warp<<<(unsigned)(4 * g->num_sms), 512, 0, st>>>(g->sc_L[cur], g->wl[0], g->wl_cnt + 3,
                                                                    g->offs, g->adj, g->sc_cur, g->bits,
                                                                    g->sc_ptr, g->wl_cnt + 2);
    CKL();
    lm::k_sc_match<<<sc_grid(g, c), lm::kScThreads, 0, st>>>(g->sc_L[cur], g->wl_cnt + cur, 0, g->sc_ptr,
                                                             g->bits, g->suitor, g->sc_L[cur ^ 1],
                                                             g->wl_cnt + (cur ^ 1));
    CKL();
    launches += 3;
    ++rounds;
    cur ^= 1;
  }
  if (tm) CK(cudaEventRecord(g->ev[4], st));
  if (n > 0) {
    lm::k_suitor_finish<kFinThreads><<<kFinBlocks, kFinThreads, 0, st>>>(g->suitor, n, d_mate, g->pw, g->pc);
    CKL();
    lm::k_final_sum<<<1, 32, 0, st>>>(g->pw, g->pc, kFinBlocks, g->res_w, g->res_c);
    CKL();
    launches += 2;
    CK(cudaMemcpyAsync(g->h_res, g->res_w, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(g->h_resc, g->res_c, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(hc, g->wl_cnt, 4 * 8, cudaMemcpyDeviceToHost, st));
  } else {
    g->h_res[0] = 0.0;
    g->h_resc[0] = 0;
  }
  if (tm) CK(cudaEventRecord(g->ev[5], st));
  CK(cudaStreamSynchronize(st));
  g->round_log.clear();
  if (stats) {
    std::memset(stats, 0, sizeof *stats);
    stats->rounds = rounds;
    stats->matched_vertices = g->h_resc[0];
    stats->cardinality = g->h_resc[0] / 2;
    stats->weight = g->h_res[0];
    stats->entries_swept = work ? (int64_t)hc[2] : 0;
    stats->kernel_launches = launches;
    stats->resident_entries = g->R;
    stats->ms_sort = sorted_now ? g->ms_sort : 0.0;
    if (tm) {
      float a = 0, b = 0, c = 0, d = 0, e = 0;
      CK(cudaEventElapsedTime(&a, g->ev[0], g->ev[5]));
      CK(cudaEventElapsedTime(&b, g->ev[1], g->ev[2]));
      CK(cudaEventElapsedTime(&c, g->ev[2], g->ev[3]));
      CK(cudaEventElapsedTime(&d, g->ev[3], g->ev[4]));
      CK(cudaEventElapsedTime(&e, g->ev[4], g->ev[5]));
      stats->ms_total = a;
      stats->ms_sweep = b;
      stats->ms_round1_rest = c;
      stats->ms_rounds = d;
      stats->ms_finish = e;
    }
  }
  return LMATCH_OK;
}

int lmatch_run_device(lmatch_graph* g, int32_t* d_mate, void* stream, lmatch_stats* stats) {
  if (!g) { set_err("NULL handle"); return LMATCH_ESTATE; }
  if (g->algorithm == 1) {
    if (!d_mate && g->n > 0) { set_err("d_mate == NULL"); return LMATCH_EINVAL; }
    if (g->ghost || g->streaming) { set_err("Suitor: resident single-graph handles only"); return LMATCH_EINVAL; }
    g_err[0] = 0;
    CK(cudaSetDevice(g->device));
    return run_suitor(g, d_mate, stream ? (cudaStream_t)stream : g->stream, stats);
  }
  if (g->algorithm == 3) {
    if (!d_mate && g->n > 0) { set_err("d_mate == NULL"); return LMATCH_EINVAL; }
    if (g->ghost || g->streaming) { set_err("sorted LD: resident single-graph handles only"); return LMATCH_EINVAL; }
    g_err[0] = 0;
    CK(cudaSetDevice(g->device));
    return run_sorted(g, d_mate, stream ? (cudaStream_t)stream : g->stream, stats);
  }
  if (!d_mate && g->n > 0) { set_err("d_mate == NULL"); return LMATCH_EINVAL; }
  if (g->ghost) { set_err("partition handle: use the lmatch_part_* calls"); return LMATCH_ESTATE; }
  g_err[0] = 0;
  CK(cudaSetDevice(g->device));
  cudaStream_t st = stream ? (cudaStream_t)stream : g->stream;
  const int64_t n = g->n;
  const bool tm = g->timing && stats;
  // round_loop: 0 = hybrid: host-driven, work-sized launches while the frontier is large, then
  //                 ONE persistent cooperative kernel for the remaining (small) rounds;
  //              1 = host-driven launches for every round;
  //              2 = persistent kernel for every round after round 1;
  //              3 = CUDA graph {round 1, persistent kernel} (no host work per run).
  // the cache redirect runs in the host-driven round body only
  const int mode = g->use_cache() ? 1 : g->round_loop;
  const bool use_graph = mode == 3 && !g->streaming;
  int64_t launches = 0, sweep_launches = 0, bytes_streamed = 0;

  if (tm) CK(cudaEventRecord(g->ev[0], st));
  g->n_rev = 0;
  g->tail_rounds_from = -1;
  if (use_graph) {
    if (!g->gexec) TRY(build_graph_persistent(g));
    CK(cudaGraphLaunch(g->gexec, st));
  } else if (mode == 2) {
    TRY(seq_prefix(g, st, 0, 0, &launches, &sweep_launches, &bytes_streamed));
    if (g->ntiles > 0 && n > 0) TRY(launch_persistent(g, st, &launches));
  } else {
    TRY(seq_prefix(g, st, 0, 0, &launches, &sweep_launches, &bytes_streamed));
    // (timing=1) an event at the start of every host-driven round and at the end of the loop:
    // per-round device times for lmatch_round_ms
    size_t nre = 0;
    auto round_mark = [&]() -> int {
      if (!tm) return LMATCH_OK;
      if (nre == g->rev.size()) {
        cudaEvent_t e;
        CK(cudaEventCreate(&e));
        g->rev.push_back(e);
      }
      CK(cudaEventRecord(g->rev[nre++], st));
      return LMATCH_OK;
    };
    g->tail_rounds_from = -1;
    for (;;) {
      CK(cudaMemcpyAsync(g->h_rstate, g->rstate, sizeof(lm::RoundState), cudaMemcpyDeviceToHost, st));
      CK(cudaMemcpyAsync(g->h_counters, g->counters, lm::kNumCounters * 8, cudaMemcpyDeviceToHost, st));
      CK(cudaStreamSynchronize(st));
      if (!g->h_rstate->cont) break;
      const int cur = g->h_rstate->cur;
      int64_t nFb[lm::kBins], nF = 0;
      for (int b = 0; b < lm::kBins; ++b) { nFb[b] = (int64_t)g->h_counters[lm::cnt_F(cur, b)]; nF += nFb[b]; }
      const int64_t nS = (int64_t)g->h_counters[lm::cnt_S(cur)];
      TRY(round_mark());
      if (mode == 0 && nF <= kPersistentBelow) {  // the tail: every remaining round on the device
        g->tail_rounds_from = (int64_t)nre - 1;
        TRY(launch_persistent(g, st, &launches));
        break;
      }
      TRY(seq_body(g, st, cur, nFb, nS, &launches));
    }
    TRY(round_mark());
    g->n_rev = (int64_t)nre;
  }
  // ---- hybrid: a frontier left after kHandoffRounds phases goes to Suitor on the residual graph
  int64_t tail_passes = 0;
  if (g->algorithm == 2 && !g->streaming && g->ntiles > 0 && n > 0) {
    CK(cudaMemcpyAsync(g->h_rstate, g->rstate, sizeof(lm::RoundState), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(g->h_counters, g->counters, lm::kNumCounters * 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    const int cur = g->h_rstate->cur;
    int64_t nF = 0;
    for (int b = 0; b < lm::kBins; ++b) nF += (int64_t)g->h_counters[lm::cnt_F(cur, b)];
    if (nF > 0) {
      TRY(ensure_suitor(g));
      CK(cudaMemsetAsync(g->wl_cnt, 0, 4 * 8, st));
      lm::k_suitor_tail_init<<<grid_for(n, 256, 65536), 256, 0, st>>>(g->bits, n, g->suitor);
      CKL();
      const int64_t nS = (int64_t)g->h_counters[lm::cnt_S(cur)];
      lm::k_suitor_tail_list<<<grid_for(nS + nF, 256, 65536), 256, 0, st>>>(
          g->S[cur], g->counters + lm::cnt_S(cur), g->F[cur], g->counters + lm::cnt_F(cur, 0),
          g->wl[0], g->wl_cnt);
      CKL();
      launches += 2;
      TRY(suitor_loop(g, st, &launches, &tail_passes));
    }
  }
  if (tm) CK(cudaEventRecord(g->ev[4], st));
  // ---- A10 mate[] + A9 w(M)
  if (n > 0 && tail_passes > 0) {
    lm::k_hybrid_finish<kFinThreads><<<kFinBlocks, kFinThreads, 0, st>>>(g->best, g->bits, g->suitor, n,
                                                                         d_mate, g->pw, g->pc);
    CKL();
    lm::k_final_sum<<<1, 32, 0, st>>>(g->pw, g->pc, kFinBlocks, g->res_w, g->res_c);
    CKL();
    launches += 2;
    CK(cudaMemcpyAsync(g->h_res, g->res_w, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(g->h_resc, g->res_c, 8, cudaMemcpyDeviceToHost, st));
  } else if (n > 0) {
    lm::k_materialize<kFinThreads><<<kFinBlocks, kFinThreads, 0, st>>>(g->best, g->bits, n, g->v0,
                                                                       d_mate, g->pw, g->pc);
    CKL();
    lm::k_final_sum<<<1, 32, 0, st>>>(g->pw, g->pc, kFinBlocks, g->res_w, g->res_c);
    CKL();
    launches += 2;
    CK(cudaMemcpyAsync(g->h_res, g->res_w, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(g->h_resc, g->res_c, 8, cudaMemcpyDeviceToHost, st));
  } else {
    g->h_res[0] = 0.0;
    g->h_resc[0] = 0;
  }
  CK(cudaMemcpyAsync(g->h_rstate, g->rstate, sizeof(lm::RoundState), cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(g->h_counters, g->counters, lm::kNumCounters * 8, cudaMemcpyDeviceToHost, st));
  if (tm) CK(cudaEventRecord(g->ev[5], st));
  CK(cudaStreamSynchronize(st));
  const lm::RoundState rs = *g->h_rstate;
  const int64_t rounds = rs.rounds;
  // a frontier left in the current set means the round cap stopped the iteration (the hybrid's
  // own 32-phase cap hands that frontier to the Suitor tail instead)
  int64_t nF_left = 0;
  if (g->ntiles > 0 && n > 0 && !(g->algorithm == 2 && !g->streaming))
    for (int b = 0; b < lm::kBins; ++b) nF_left += (int64_t)g->h_counters[lm::cnt_F(rs.cur, b)];
  if (use_graph) {  // launches inside the graph
    launches += (rounds > 0 ? 6 : 2) + (rounds > 0 ? 1 : 0);
    sweep_launches = rounds > 0 ? 1 : 0;
  }
  // per-round log: round 1 from the host, later rounds from the device log
  g->round_log.clear();
  if (rounds > 0) {
    g->round_log.insert(g->round_log.end(), {g->n_nz, n, g->m});
    const int64_t rows = std::min<int64_t>(rs.log_len, kLogCap);
    if (rows > 0) {
      std::vector<long long> tmp(3 * (size_t)rows);
      CK(cudaMemcpy(tmp.data(), g->rlog, tmp.size() * 8, cudaMemcpyDeviceToHost));
      for (long long x : tmp) g->round_log.push_back(x);
    }
  }
  if (stats) {
    std::memset(stats, 0, sizeof *stats);
    stats->rounds = rounds;
    stats->matched_vertices = g->h_resc[0];
    stats->cardinality = g->h_resc[0] / 2;
    stats->weight = g->h_res[0];
    stats->entries_swept = 0;
    for (size_t i = 2; i < g->round_log.size(); i += 3) stats->entries_swept += g->round_log[i];
    stats->frontier_total = rs.ftot;
    stats->sweep_launches = sweep_launches;
    stats->kernel_launches = launches;
    stats->bytes_streamed = bytes_streamed;
    stats->resident_entries = g->R;
    stats->tail_passes = tail_passes;
    if (g->kcache) stats->cache_rows = (int64_t)g->h_counters[lm::kCntCache];
    if (g->use_cache()) {
      stats->residual_rows = (int64_t)g->h_counters[lm::kCntCache + 2];
      stats->cache_rows = (int64_t)g->h_counters[lm::kCntCache];
      stats->host_entries_read = (int64_t)g->h_counters[lm::kCntCache + 1];
      stats->cache_bytes = g->cap_cache * 8;
    }
    if (tm) {
      float a = 0, b = 0, c = 0, d = 0, e = 0;
      CK(cudaEventElapsedTime(&a, g->ev[0], g->ev[5]));
      CK(cudaEventElapsedTime(&e, g->ev[4], g->ev[5]));
      CK(cudaEventElapsedTime(&b, g->ev[1], g->ev[2]));
      CK(cudaEventElapsedTime(&c, g->ev[2], g->ev[3]));
      CK(cudaEventElapsedTime(&d, g->ev[3], g->ev[4]));
      stats->ms_total = a;
      stats->ms_sweep = b;
      stats->ms_round1_rest = c;
      stats->ms_rounds = d;
      stats->ms_finish = e;
    }
  }
  if (nF_left > 0) {
    set_err("%lld vertices still to re-point after the round cap (%lld pointing phases)",
            (long long)nF_left, (long long)rounds);
    return LMATCH_EROUNDS;
  }
  return LMATCH_OK;
}

int lmatch_run(lmatch_graph* g, int32_t* mate_out, lmatch_stats* stats) {
  if (!g) { set_err("NULL handle"); return LMATCH_ESTATE; }
  if (!mate_out && g->n > 0) { set_err("mate_out == NULL"); return LMATCH_EINVAL; }
  CK(cudaSetDevice(g->device));
  if (!g->mate_tmp) TRY(dmalloc(g, &g->mate_tmp, (size_t)g->n + 1));
  TRY(lmatch_run_device(g, g->mate_tmp, g->stream, stats));
  if (g->n > 0) {
    CK(cudaMemcpyAsync(mate_out, g->mate_tmp, (size_t)g->n * 4, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaStreamSynchronize(g->stream));
  }
  return LMATCH_OK;
}

int lmatch_weight_device(lmatch_graph* g, const int32_t* d_mate, void* stream, double* out_weight) {
  if (!g) { set_err("NULL handle"); return LMATCH_ESTATE; }
  if (!out_weight || (!d_mate && g->n > 0)) { set_err("NULL argument"); return LMATCH_EINVAL; }
  g_err[0] = 0;
  CK(cudaSetDevice(g->device));
  cudaStream_t st = stream ? (cudaStream_t)stream : g->stream;
  if (g->n == 0) { *out_weight = 0.0; return LMATCH_OK; }
  CK(cudaMemsetAsync(g->werr, 0, 4, st));
  lm::k_weight_any<kFinThreads><<<kFinBlocks, kFinThreads, 0, st>>>(d_mate, g->n, g->offs, g->view(),
                                                                    g->pw, g->pc, g->werr);
  CKL();
  lm::k_final_sum<<<1, 32, 0, st>>>(g->pw, g->pc, kFinBlocks, g->res_w, g->res_c);
  CKL();
  unsigned herr = 0;
  CK(cudaMemcpyAsync(g->h_res, g->res_w, 8, cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(&herr, g->werr, 4, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (herr) {
    set_err("mate[] is not a matching of the graph (%s%s%s)", (herr & 1) ? "id out of range/self " : "",
            (herr & 2) ? "asymmetric " : "", (herr & 4) ? "pair is not an edge" : "");
    return LMATCH_EINVAL;
  }
  *out_weight = g->h_res[0];
  return LMATCH_OK;
}

int lmatch_weight(lmatch_graph* g, const int32_t* mate, double* out_weight) {
  if (!g) { set_err("NULL handle"); return LMATCH_ESTATE; }
  if (!out_weight || (!mate && g->n > 0)) { set_err("NULL argument"); return LMATCH_EINVAL; }
  CK(cudaSetDevice(g->device));
  if (!g->mate_tmp) TRY(dmalloc(g, &g->mate_tmp, (size_t)g->n + 1));
  if (g->n > 0)
    CK(cudaMemcpyAsync(g->mate_tmp, mate, (size_t)g->n * 4, cudaMemcpyHostToDevice, g->stream));
  return lmatch_weight_device(g, g->mate_tmp, g->stream, out_weight);
}

// ------------------------------------------------------------------ partitioned mode (A3/A5)
static int check_part(int64_t n_local, int64_t v_begin, int64_t n_global, int32_t nparts,
                      const int64_t* bounds) {
  if (nparts < 1 || !bounds) { set_err("nparts < 1 or NULL part_bounds"); return LMATCH_EINVAL; }
  if (n_global < 0 || n_global >= ((int64_t)1 << 31)) { set_err("n_global out of range"); return LMATCH_ERANGE; }
  if (bounds[0] != 0 || bounds[nparts] != n_global) { set_err("part_bounds must span [0, n_global]"); return LMATCH_EINVAL; }
  bool found = false;
  for (int p = 0; p < nparts; ++p) {
    if (bounds[p + 1] < bounds[p]) { set_err("part_bounds decrease"); return LMATCH_EINVAL; }
    if (bounds[p] % 32 != 0 && bounds[p] != n_global) { set_err("part_bounds must be multiples of 32"); return LMATCH_EINVAL; }
    if (bounds[p] == v_begin && bounds[p + 1] == v_begin + n_local) found = true;
  }
  if (!found) { set_err("[v_begin, v_begin + n_local) is not a part of part_bounds"); return LMATCH_EINVAL; }
  return LMATCH_OK;
}

int lmatch_create_part(const int64_t* csr_offsets, const int32_t* col_idx, const float* weights,
                       int64_t n_local, int64_t m_local, int64_t v_begin, int64_t n_global,
                       int32_t nparts, const int64_t* part_bounds, const lmatch_opts* opts,
                       lmatch_graph** out) {
  if (!out) { set_err("out == NULL"); return LMATCH_EINVAL; }
  *out = nullptr;
  g_err[0] = 0;
  int s = check_args(csr_offsets, col_idx, weights, n_local, m_local);
  if (!s) s = check_part(n_local, v_begin, n_global, nparts, part_bounds);
  if (s) return s;
  if (opts && opts->validate_level >= 2) { set_err("validate_level 2 is not available per partition"); return LMATCH_EINVAL; }
  PartSpec ps;
  ps.v0 = v_begin; ps.n_global = n_global; ps.P = nparts; ps.bounds = part_bounds;
  lmatch_graph* g = nullptr;
  s = create_common(n_local, m_local, opts, out, &g, &ps);
  if (!s) s = upload_host(g, csr_offsets, col_idx, weights);
  if (!s) s = finish_create(g, g->stream);
  if (s) { lmatch_destroy(g); return s; }
  *out = g;
  return LMATCH_OK;
}

int lmatch_create_part_device(const int64_t* d_offsets, const int32_t* d_col, const float* d_weights,
                              int64_t n_local, int64_t m_local, int64_t v_begin, int64_t n_global,
                              int32_t nparts, const int64_t* part_bounds, const lmatch_opts* opts,
                              void* stream, lmatch_graph** out) {
  if (!out) { set_err("out == NULL"); return LMATCH_EINVAL; }
  *out = nullptr;
  g_err[0] = 0;
  int s = check_args(d_offsets, d_col, d_weights, n_local, m_local);
  if (!s) s = check_part(n_local, v_begin, n_global, nparts, part_bounds);
  if (s) return s;
  if (opts && opts->validate_level >= 2) { set_err("validate_level 2 is not available per partition"); return LMATCH_EINVAL; }
  PartSpec ps;
  ps.v0 = v_begin; ps.n_global = n_global; ps.P = nparts; ps.bounds = part_bounds;
  lmatch_graph* g = nullptr;
  s = create_common(n_local, m_local, opts, out, &g, &ps);
  cudaStream_t st = stream ? (cudaStream_t)stream : (g ? g->stream : nullptr);
  if (!s) {
    cudaError_t e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) { set_err("stream sync: %s", cudaGetErrorString(e)); s = LMATCH_ECUDA; }
  }
  if (!s) s = upload_device(g, d_offsets, d_col, d_weights, st);
  if (!s) s = finish_create(g, st);
  if (s) { lmatch_destroy(g); return s; }
  *out = g;
  return LMATCH_OK;
}

static int part_claims_out(lmatch_graph* g, cudaStream_t st, int64_t* claim_counts) {
  CK(cudaMemcpyAsync(g->h_claim_cnt, g->claim_cnt, (size_t)g->P * 8, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (claim_counts)
    for (int p = 0; p < g->P; ++p) claim_counts[p] = (int64_t)g->h_claim_cnt[p];
  return LMATCH_OK;
}

static lm::Claims part_claims_desc(const lmatch_graph* g) {
  lm::Claims Cl{g->claims, g->claim_cap, g->claim_cnt, g->bounds, g->P};
  if (g->p2p) {
    Cl.dseg = g->d_dseg;
    Cl.dcnt = g->d_dcnt;
  }
  return Cl;
}

static int part_begin_impl(lmatch_graph* g, cudaStream_t st, int64_t* claim_counts) {
  if (g->p2p) CK(cudaMemsetAsync(g->shadow, 0, (size_t)((g->n + 31) / 32 + 1) * 4, st));
  const int64_t nwords = (g->n_global + 31) / 32;
  lm::k_reset<<<grid_for(std::max(nwords, xrow_resets(g)), 256, 4096), 256, 0, st>>>(
      g->bits, nwords, g->best, g->atomic_rows, xrow_resets(g), g->counters, lm::kNumCounters,
      g->prune ? g->live : nullptr, g->n, g->rstate);
  CKL();
  lm::k_round_init<<<1, 1, 0, st>>>(g->rstate, g->max_rounds, kLogCap, 1);
  CKL();
  // one part: nothing is remote, so there are no ghosts and no claims
  if (g->P > 1) CK(cudaMemsetAsync(g->ghost, 0xff, ((size_t)g->n_global + 1) * 4, st));
  CK(cudaMemsetAsync(g->claim_cnt, 0, (size_t)g->P * 8, st));
  int64_t l = 0, sl = 0, bs = 0;
  if (g->timing) CK(cudaEventRecord(g->ev[1], st));
  if (g->ntiles > 0 && g->n > 0) TRY(round1_sweep(g, st, &l, &sl, &bs));
  if (g->timing) CK(cudaEventRecord(g->ev[2], st));
  const lm::Claims Cl = part_claims_desc(g);
  if (g->n > 0 && g->P > 1) {
    lm::k_claims_all<<<grid_for(g->n, 256, 65536), 256, 0, st>>>(g->best, g->n, g->v0,
                                                                   g->v0 + g->n, Cl);
    CKL();
  }
  g->part_round = 1;
  g->round_log.clear();
  g->sweep_ms_pending = g->timing != 0;  // read when the stream next synchronises
  const int rc = g->p2p ? LMATCH_OK : part_claims_out(g, st, claim_counts);
  if (!rc && g->timing && !g->p2p) {
    CK(cudaEventElapsedTime(&g->part_sweep_ms, g->ev[1], g->ev[2]));
    g->sweep_ms_pending = false;
  }
  return rc;
}

int lmatch_part_begin(lmatch_graph* g, void* stream, int64_t* claim_counts) {
  if (!g || !g->ghost) { set_err("not a partition handle"); return LMATCH_ESTATE; }
  if (g->p2p) { set_err("peer-memory handle: use lmatch_p2p_begin"); return LMATCH_ESTATE; }
  g_err[0] = 0;
  CK(cudaSetDevice(g->device));
  return part_begin_impl(g, stream ? (cudaStream_t)stream : g->stream, claim_counts);
}

int lmatch_part_claims(const lmatch_graph* g, uint64_t** seg_ptrs) {
  if (!g || !g->ghost || !seg_ptrs) { set_err("not a partition handle / NULL"); return LMATCH_ESTATE; }
  for (int p = 0; p < g->P; ++p) seg_ptrs[p] = g->claims + (int64_t)p * g->claim_cap;
  return LMATCH_OK;
}

int lmatch_part_apply(lmatch_graph* g, const uint64_t* d_recv, int64_t nrecv, void* stream) {
  if (!g || !g->ghost || g->part_round < 1) { set_err("lmatch_part_apply out of order"); return LMATCH_ESTATE; }
  if (g->p2p) { set_err("peer-memory handle: use lmatch_p2p_match"); return LMATCH_ESTATE; }
  if (nrecv > 0 && !d_recv) { set_err("NULL claims"); return LMATCH_EINVAL; }
  CK(cudaSetDevice(g->device));
  cudaStream_t st = stream ? (cudaStream_t)stream : g->stream;
  if (nrecv > 0) {
    lm::k_apply_claims<<<grid_for(nrecv, 256, 65536), 256, 0, st>>>(d_recv, nrecv, g->ghost);
    CKL();
  }
  if (g->part_round == 1) {
    if (g->n > 0) {
      lm::k_match_part_all<<<grid_for(((g->n + 31) / 32) * 32, 256, 65536), 256, 0, st>>>(
          g->best, g->n, g->v0, g->v0 + g->n, g->ghost, g->bits);
      CKL();
    }
  } else {
    int64_t nF = 0;
    for (int b = 0; b < lm::kBins; ++b) nF += (int64_t)g->h_counters[lm::cnt_F(g->part_cur, b)];
    if (nF > 0) {
      lm::k_match_part_bins<<<grid_for(nF, 256, 65536), 256, 0, st>>>(
          g->F[g->part_cur], g->counters + lm::cnt_F(g->part_cur, 0), g->best, g->v0, g->v0 + g->n,
          g->ghost, g->bits);
      CKL();
    }
  }
  if (nrecv > 0) {
    lm::k_match_claims<<<grid_for(nrecv, 256, 65536), 256, 0, st>>>(d_recv, nrecv, g->best, g->v0,
                                                                      g->bits);
    CKL();
  }
  return LMATCH_OK;
}

int lmatch_part_info(const lmatch_graph* g, int64_t* rounds, double* sweep_ms) {
  if (!g || !g->ghost) { set_err("not a partition handle"); return LMATCH_ESTATE; }
  if (g->sweep_ms_pending) {
    lmatch_graph* gm = const_cast<lmatch_graph*>(g);
    CK(cudaEventSynchronize(g->ev[2]));
    CK(cudaEventElapsedTime(&gm->part_sweep_ms, g->ev[1], g->ev[2]));
    gm->sweep_ms_pending = false;
  }
  if (rounds) *rounds = g->part_round;
  if (sweep_ms) *sweep_ms = g->part_sweep_ms;
  return LMATCH_OK;
}

int lmatch_part_bitmap(lmatch_graph* g, uint32_t** d_bits, int64_t* word_begin, int64_t* nwords_own,
                       int64_t* nwords_total) {
  if (!g) { set_err("NULL handle"); return LMATCH_ESTATE; }
  if (d_bits) *d_bits = g->bits;
  if (word_begin) *word_begin = g->v0 / 32;
  if (nwords_own) *nwords_own = (g->n + 31) / 32;
  if (nwords_total) *nwords_total = (g->n_global + 31) / 32;
  return LMATCH_OK;
}

// the compaction launches of a partition round; the set sizes come from h_counters, or (peer-
// memory rounds, which do not read them back every round) a full resident wave per kernel
static int part_compact_launch(lmatch_graph* g, cudaStream_t st) {
  const int64_t n = g->n;
  // the compaction reads set part_cur (round 1: none) and writes its other set; k_end_round
  // makes that set current (and zeroes the counters the next compaction writes)
  if (g->part_round == 1) {
    if (n > 0) {
      // items are the non-empty rows (nzr): empty rows never hold a pointer
      const unsigned grid = grid_for((g->n_nz + 31) / 32, 8 * kCompactK1, 65536);
      lm::CompactIO io = lm::compact_io(g->rargs(), 1);
      io.nzr = g->nzr;
      io.noffs = g->noffs;
      if (g->kcache)
        lm::k_compact<true, kCompactK1, true><<<grid, 256, 0, st>>>(io, g->n_nz, g->best, g->bits, g->offs, g->v0);
      else
        lm::k_compact<true, kCompactK1, false><<<grid, 256, 0, st>>>(io, g->n_nz, g->best, g->bits, g->offs, g->v0);
      CKL();
    }
    g->part_cur = 0;
    g->round_log.insert(g->round_log.end(), {g->n_nz, n, g->m});
  } else {
    const int cur = g->part_cur;
    const int64_t nS = (int64_t)g->h_counters[lm::cnt_S(cur)];
    int64_t nF = 0;
    for (int b = 0; b < lm::kBins; ++b) nF += (int64_t)g->h_counters[lm::cnt_F(cur, b)];
    if (g->p2p || nS + nF > 0) {
      const unsigned grid = (g->p2p && !g->one_rank_loop) ? (unsigned)(4 * g->num_sms)
                                   : grid_for((nS + nF + 31) / 32, 8 * kCompactK, 65536);
      const lm::CompactIO io = lm::compact_io(g->rargs(), cur);
      if (g->kcache)
        lm::k_compact<false, kCompactK, true><<<grid, 256, 0, st>>>(io, n, g->best, g->bits, g->offs, g->v0);
      else
        lm::k_compact<false, kCompactK, false><<<grid, 256, 0, st>>>(io, n, g->best, g->bits, g->offs, g->v0);
      CKL();
    }
    g->part_cur = cur ^ 1;
  }
  lm::k_end_round<<<1, 32, 0, st>>>(g->ra(), 0, 0, 0);
  CKL();
  return LMATCH_OK;
}

int lmatch_part_compact(lmatch_graph* g, void* stream, int64_t* nF_local) {
  if (!g || !g->ghost || g->part_round < 1) { set_err("lmatch_part_compact out of order"); return LMATCH_ESTATE; }
  CK(cudaSetDevice(g->device));
  cudaStream_t st = stream ? (cudaStream_t)stream : g->stream;
  unsigned long long* C = g->counters;
  TRY(part_compact_launch(g, st));
  CK(cudaMemcpyAsync(g->h_counters, C, lm::kNumCounters * 8, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  int64_t nF = 0;
  for (int b = 0; b < lm::kBins; ++b) nF += (int64_t)g->h_counters[lm::cnt_F(g->part_cur, b)];
  if (nF_local) *nF_local = nF;
  return LMATCH_OK;
}

static int part_point_impl(lmatch_graph* g, cudaStream_t st, int64_t* claim_counts) {
  const int cur = g->part_cur;
  int64_t nFb[lm::kBins], nF = 0;
  for (int b = 0; b < lm::kBins; ++b) { nFb[b] = (int64_t)g->h_counters[lm::cnt_F(cur, b)]; nF += nFb[b]; }
  if (g->p2p && !g->counts_on_host) {
    // peer-memory rounds do not read the bin sizes back: every kernel below loops over the
    // device-resident count, so launch each bin with a full resident wave (an empty bin exits)
    const int64_t wave = 8ll * g->num_sms;
    for (int b = 0; b < lm::kBins; ++b) nFb[b] = wave * 256;
    nF = wave * 256;
  }
  g->counts_on_host = false;
  const lm::AdjView av = g->view();
  const lm::Bins& Fb = g->F[cur];
  const unsigned long long* cF = g->counters + lm::cnt_F(cur, 0);
  if (g->use_cache() && nF > 0) {
    // out-of-core part (per-device batches, NEXT-2): the host-row key cache decides the pointer of
    // host rows where it can, and refills the rows whose cached keys ran dry (as in seq_body)
    const bool refill = LM_CACHE_REFILL != 0;
    if (refill) CK(cudaMemsetAsync(g->rescan_cnt, 0, 8, st));
    lm::k_cache_redirect<lm::kCacheK><<<grid_for(nF, 256, 65536), 256, 0, st>>>(
        Fb, cF, g->offs, g->cache, g->bits, g->u_first, g->M0, g->v0, g->counters + lm::kCntCache,
        refill ? g->rescan : nullptr, refill ? g->rescan_cnt : nullptr, g->res ? g->roff : nullptr, g->M2);
    CKL();
    if (refill) {
      lm::k_host_rescan<lm::kCacheK><<<(unsigned)(8 * g->num_sms), 256, 0, st>>>(
          Fb, g->rescan, g->rescan_cnt, g->offs, g->view(), g->bits, g->cache, g->u_first, g->M0,
          g->v0, g->res, g->cap_res, g->res_used, g->roff);
      CKL();
    }
  }
  if (nFb[0]) {
#if LM_PIPE & 1
    // the software-pipelined thread-per-row kernel, one resident wave (as in the single-graph
    // round loop, seq_body)
    static int occ = 0;
    if (!occ) {
      CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, lm::k_point_pipe<LM_P0_G, LM_P0_U>, 256, 0));
      if (occ < 1) occ = 1;
    }
    const int64_t wave = (int64_t)occ * g->num_sms * LM_PIPE_WAVES;
    lm::k_point_pipe<LM_P0_G, LM_P0_U><<<(unsigned)std::min<int64_t>(wave, (nFb[0] * LM_P0_G + 255) / 256), 256, 0, st>>>(
        Fb.list[0], cF + 0, g->offs, av, g->bits, g->best, g->v0);
#else
    lm::k_point_bin<LM_B0_G, LM_B0_U><<<grid_for(nFb[0] * LM_B0_G, 256, 65536), 256, 0, st>>>(Fb.list[0], cF + 0, g->offs, av, g->bits, g->best, g->v0);
#endif
    CKL();
  }
  if (nFb[1]) {
#if LM_PIPE & 2
    static int occ1 = 0;
    if (!occ1) {
      CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ1, lm::k_point_pipe<LM_P1_G, LM_P1_U>, 256, 0));
      if (occ1 < 1) occ1 = 1;
    }
    const int64_t wave1 = (int64_t)occ1 * g->num_sms * LM_PIPE_WAVES;
    lm::k_point_pipe<LM_P1_G, LM_P1_U><<<(unsigned)std::min<int64_t>(wave1, (nFb[1] * LM_P1_G + 255) / 256), 256, 0, st>>>(
        Fb.list[1], cF + 1, g->offs, av, g->bits, g->best, g->v0);
#else
    lm::k_point_bin<LM_B1_G, LM_B1_U><<<grid_for(nFb[1] * LM_B1_G, 256, 65536), 256, 0, st>>>(Fb.list[1], cF + 1, g->offs, av, g->bits, g->best, g->v0);
#endif
    CKL();
  }
  if (nFb[2]) { lm::k_point_bin<LM_B2_G, LM_B2_U><<<grid_for(nFb[2] * LM_B2_G, 256, 65536), 256, 0, st>>>(Fb.list[2], cF + 2, g->offs, av, g->bits, g->best, g->v0); CKL(); }
  if (nFb[3]) { lm::k_point_bin_cta<256, LM_CTA_U><<<(unsigned)std::min<int64_t>(nFb[3], g->p2p ? 8ll * g->num_sms : 65536), 256, 0, st>>>(Fb.list[3], cF + 3, g->offs, av, g->bits, g->best, g->v0); CKL(); }
  if (!g->p2p) CK(cudaMemsetAsync(g->claim_cnt, 0, (size_t)g->P * 8, st));
  if (nF > 0 && g->P > 1) {
    const lm::Claims Cl = part_claims_desc(g);
    lm::k_claims_bins<<<grid_for(nF, 256, 65536), 256, 0, st>>>(Fb, cF, g->v0, g->v0 + g->n, Cl);
    CKL();
  }
  if (!g->p2p)
    g->round_log.insert(g->round_log.end(), {nF, nF + (int64_t)g->h_counters[lm::cnt_S(cur)],
                                             (int64_t)g->h_counters[lm::kCntSwept]});
  ++g->part_round;
  return g->p2p ? LMATCH_OK : part_claims_out(g, st, claim_counts);
}

int lmatch_part_point(lmatch_graph* g, void* stream, int64_t* claim_counts) {
  if (!g || !g->ghost || g->part_round < 1) { set_err("lmatch_part_point out of order"); return LMATCH_ESTATE; }
  if (g->p2p) { set_err("peer-memory handle: use lmatch_p2p_point"); return LMATCH_ESTATE; }
  CK(cudaSetDevice(g->device));
  return part_point_impl(g, stream ? (cudaStream_t)stream : g->stream, claim_counts);
}

int lmatch_part_finish(lmatch_graph* g, int32_t* d_mate_local, void* stream, double* w_local,
                       int64_t* matched_local) {
  if (!g || !g->ghost) { set_err("not a partition handle"); return LMATCH_ESTATE; }
  CK(cudaSetDevice(g->device));
  cudaStream_t st = stream ? (cudaStream_t)stream : g->stream;
  if (g->n > 0) {
    lm::k_materialize<kFinThreads><<<kFinBlocks, kFinThreads, 0, st>>>(g->best, g->bits, g->n, g->v0,
                                                                       d_mate_local, g->pw, g->pc);
    CKL();
    lm::k_final_sum<<<1, 32, 0, st>>>(g->pw, g->pc, kFinBlocks, g->res_w, g->res_c);
    CKL();
    CK(cudaMemcpyAsync(g->h_res, g->res_w, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(g->h_resc, g->res_c, 8, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
  } else {
    g->h_res[0] = 0.0;
    g->h_resc[0] = 0;
  }
  if (w_local) *w_local = g->h_res[0];
  if (matched_local) *matched_local = g->h_resc[0];
  return LMATCH_OK;
}

int lmatch_part_get_claims(const lmatch_graph* g, int32_t part, uint64_t* d_dst, void* stream) {
  if (!g || !g->ghost || part < 0 || part >= g->P) { set_err("bad handle or part"); return LMATCH_ESTATE; }
  CK(cudaSetDevice(g->device));
  const int64_t c = (int64_t)g->h_claim_cnt[part];
  if (c > 0)
    CK(cudaMemcpyAsync(d_dst, g->claims + (int64_t)part * g->claim_cap, (size_t)c * 8,
                       cudaMemcpyDeviceToDevice, stream ? (cudaStream_t)stream : g->stream));
  return LMATCH_OK;
}

int lmatch_part_get_bits(const lmatch_graph* g, uint32_t* d_dst, void* stream) {
  if (!g || !g->ghost) { set_err("not a partition handle"); return LMATCH_ESTATE; }
  CK(cudaSetDevice(g->device));
  const int64_t nw = (g->n + 31) / 32;
  if (nw > 0)
    CK(cudaMemcpyAsync(d_dst, g->bits + g->v0 / 32, (size_t)nw * 4, cudaMemcpyDeviceToDevice,
                       stream ? (cudaStream_t)stream : g->stream));
  return LMATCH_OK;
}

int lmatch_part_set_bits(lmatch_graph* g, const uint32_t* d_src, int64_t word_begin, int64_t nwords,
                         void* stream) {
  if (!g || !g->ghost) { set_err("not a partition handle"); return LMATCH_ESTATE; }
  if (word_begin < 0 || word_begin + nwords > (g->n_global + 31) / 32) { set_err("word range"); return LMATCH_EINVAL; }
  CK(cudaSetDevice(g->device));
  if (nwords > 0)
    CK(cudaMemcpyAsync(g->bits + word_begin, d_src, (size_t)nwords * 4, cudaMemcpyDeviceToDevice,
                       stream ? (cudaStream_t)stream : g->stream));
  return LMATCH_OK;
}

// ----------------------------------------------------------------- peer-memory exchange (A3/A5)
// The partitioned round with the exchange done by the library's own kernels over peer memory
// (CUDA IPC across processes / GPUs, plain pointers for parts in one process): the claims
// kernels store straight into the owner's inbox, the match step pushes changed owned bitmap
// words into every peer's replica, and the compaction pushes the frontier size into every
// peer's slot.  The caller supplies the barriers between phases (include/lmatch.h).
int lmatch_p2p_enable(lmatch_graph* g, int32_t me) {
  if (!g || !g->ghost) { set_err("not a partition handle"); return LMATCH_ESTATE; }
  if (me < 0 || me >= g->P || g->hbounds.size() != (size_t)g->P + 1 || g->hbounds[me] != g->v0 ||
      g->hbounds[me + 1] != g->v0 + g->n) {
    set_err("part index %d does not own rows [%lld, %lld)", me, (long long)g->v0, (long long)(g->v0 + g->n));
    return LMATCH_EINVAL;
  }
  if (g->p2p) return LMATCH_OK;
  CK(cudaSetDevice(g->device));
  const int P = g->P;
  int64_t cap = 1;  // inbox segment: the largest part (one part receives no claims)
  for (int p = 0; P > 1 && p < P; ++p) cap = std::max(cap, g->hbounds[p + 1] - g->hbounds[p]);
  g->me = me;
  g->win_cap = cap;
  TRY(dmalloc(g, &g->win, (size_t)P * cap + 6 * (size_t)P));
  CK(cudaMemset(g->win + (size_t)P * cap, 0, 6 * (size_t)P * 8));
  TRY(dmalloc(g, &g->shadow, (size_t)(g->n + 31) / 32 + 1));
  TRY(dmalloc(g, &g->d_dseg, (size_t)P));
  TRY(dmalloc(g, &g->d_dcnt, (size_t)P));
  TRY(dmalloc(g, &g->d_dbits, (size_t)P));
  TRY(dmalloc(g, &g->d_dnf, (size_t)P));
  TRY(dmalloc(g, &g->d_dflag, (size_t)P));
  TRY(dmalloc(g, &g->d_dresw, (size_t)P));
  TRY(dmalloc(g, &g->d_dresc, (size_t)P));
  CK(cudaHostAlloc(reinterpret_cast<void**>(&g->h_nf), (size_t)P * 8, cudaHostAllocDefault));
  g->h_dseg.assign(P, nullptr);
  g->h_dcnt.assign(P, nullptr);
  g->h_dnf.assign(P, nullptr);
  g->h_dflag.assign(P, nullptr);
  g->h_dresw.assign(P, nullptr);
  g->h_dresc.assign(P, nullptr);
  g->h_dbits.assign(P, nullptr);
  g->p2p = 1;
  // this part's own entries (its frontier-size slot is written like a peer's)
  return lmatch_p2p_attach_local(g, me, g);
}

static int p2p_set_peer(lmatch_graph* g, int peer, uint64_t* pwin, uint32_t* pbits) {
  const int P = g->P;
  uint64_t* cnt = pwin + (size_t)P * g->win_cap;
  g->h_dseg[peer] = pwin + (size_t)g->me * g->win_cap;
  g->h_dcnt[peer] = reinterpret_cast<unsigned long long*>(cnt) + g->me;
  g->h_dnf[peer] = reinterpret_cast<unsigned long long*>(cnt + P) + g->me;
  g->h_dflag[peer] = reinterpret_cast<unsigned long long*>(cnt + 2 * P) + g->me;
  g->h_dresw[peer] = reinterpret_cast<unsigned long long*>(cnt + 3 * P) + g->me;
  g->h_dresc[peer] = reinterpret_cast<unsigned long long*>(cnt + 4 * P) + g->me;
  g->h_dbits[peer] = pbits;
  CK(cudaMemcpy(g->d_dseg, g->h_dseg.data(), (size_t)P * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(g->d_dcnt, g->h_dcnt.data(), (size_t)P * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(g->d_dnf, g->h_dnf.data(), (size_t)P * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(g->d_dbits, g->h_dbits.data(), (size_t)P * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(g->d_dflag, g->h_dflag.data(), (size_t)P * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(g->d_dresw, g->h_dresw.data(), (size_t)P * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(g->d_dresc, g->h_dresc.data(), (size_t)P * 8, cudaMemcpyHostToDevice));
  return LMATCH_OK;
}

int lmatch_p2p_attach_local(lmatch_graph* g, int32_t peer, lmatch_graph* pg) {
  if (!g || !pg || !g->p2p || !pg->p2p) { set_err("lmatch_p2p_enable both handles first"); return LMATCH_ESTATE; }
  if (peer < 0 || peer >= g->P || pg->me != peer || pg->P != g->P || pg->win_cap != g->win_cap ||
      pg->n_global != g->n_global) {
    set_err("peer handle does not match (part %d)", peer);
    return LMATCH_EINVAL;
  }
  CK(cudaSetDevice(g->device));
  if (pg->device != g->device) {
    const cudaError_t e = cudaDeviceEnablePeerAccess(pg->device, 0);
    if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) {
      set_err("cudaDeviceEnablePeerAccess(%d): %s", pg->device, cudaGetErrorString(e));
      return LMATCH_ECUDA;
    }
    cudaGetLastError();
  }
  return p2p_set_peer(g, peer, pg->win, pg->bits);
}

int lmatch_p2p_export(const lmatch_graph* g, void* handles) {
  if (!g || !g->p2p || !handles) { set_err("lmatch_p2p_enable first / NULL"); return LMATCH_ESTATE; }
  CK(cudaSetDevice(g->device));
  cudaIpcMemHandle_t h[2];
  CK(cudaIpcGetMemHandle(&h[0], g->win));
  CK(cudaIpcGetMemHandle(&h[1], g->bits));
  std::memcpy(handles, h, sizeof h);
  return LMATCH_OK;
}

int lmatch_p2p_attach(lmatch_graph* g, int32_t peer, const void* handles) {
  if (!g || !g->p2p || !handles) { set_err("lmatch_p2p_enable first / NULL"); return LMATCH_ESTATE; }
  if (peer < 0 || peer >= g->P || peer == g->me) { set_err("bad peer %d", peer); return LMATCH_EINVAL; }
  CK(cudaSetDevice(g->device));
  cudaIpcMemHandle_t h[2];
  std::memcpy(h, handles, sizeof h);
  void* pw = nullptr;
  void* pb = nullptr;
  CK(cudaIpcOpenMemHandle(&pw, h[0], cudaIpcMemLazyEnablePeerAccess));
  g->ipc_opened.push_back(pw);
  CK(cudaIpcOpenMemHandle(&pb, h[1], cudaIpcMemLazyEnablePeerAccess));
  g->ipc_opened.push_back(pb);
  return p2p_set_peer(g, peer, static_cast<uint64_t*>(pw), static_cast<uint32_t*>(pb));
}

static int p2p_ready(const lmatch_graph* g) {
  if (!g || !g->p2p) { set_err("not a peer-memory partition handle"); return LMATCH_ESTATE; }
  for (int p = 0; p < g->P; ++p)
    if (!g->h_dbits[p]) { set_err("peer %d not attached", p); return LMATCH_ESTATE; }
  return LMATCH_OK;
}

int lmatch_p2p_begin(lmatch_graph* g, void* stream) {
  TRY(p2p_ready(g));
  g_err[0] = 0;
  CK(cudaSetDevice(g->device));
  return part_begin_impl(g, stream ? (cudaStream_t)stream : g->stream, nullptr);
}

int lmatch_p2p_point(lmatch_graph* g, void* stream) {
  TRY(p2p_ready(g));
  if (g->part_round < 1) { set_err("lmatch_p2p_point out of order"); return LMATCH_ESTATE; }
  CK(cudaSetDevice(g->device));
  return part_point_impl(g, stream ? (cudaStream_t)stream : g->stream, nullptr);
}

int lmatch_p2p_match(lmatch_graph* g, void* stream) {
  TRY(p2p_ready(g));
  if (g->part_round < 1) { set_err("lmatch_p2p_match out of order"); return LMATCH_ESTATE; }
  CK(cudaSetDevice(g->device));
  cudaStream_t st = stream ? (cudaStream_t)stream : g->stream;
  const int P = g->P;
  unsigned long long* icnt = reinterpret_cast<unsigned long long*>(g->win + (size_t)P * g->win_cap);
  const int64_t grid = std::max<int64_t>(1, std::min<int64_t>((g->win_cap + 255) / 256, 4 * g->num_sms));
  // received claims (v owned, u remote): ghost pointers, then the owned mutual checks
  if (P > 1) {
    lm::k_apply_inbox<<<(unsigned)grid, 256, 0, st>>>(g->win, g->win_cap, icnt, P, g->ghost);
    CKL();
  }
  if (g->one_rank_loop) {
    // one part (v0 = 0, no ghosts): the single-graph match kernels, sized from the host counts
    if (g->part_round == 1) {
      const int64_t nwords = (g->n + 31) / 32;
      if (g->n > 0) {
        lm::k_match_all<<<grid_for((nwords + LM_MATCHALL_V - 1) / LM_MATCHALL_V * 32, 256, 65536), 256, 0, st>>>(
            g->best, g->n, g->bits);
        CKL();
      }
    } else {
      int64_t nF = 0;
      for (int b = 0; b < lm::kBins; ++b) nF += (int64_t)g->h_counters[lm::cnt_F(g->part_cur, b)];
      if (nF > 0) {
        lm::k_match_bins<<<grid_for((nF + LM_MATCH_V - 1) / LM_MATCH_V, 256, 65536), 256, 0, st>>>(
            g->F[g->part_cur], g->counters + lm::cnt_F(g->part_cur, 0), g->best, g->bits);
        CKL();
      }
    }
  } else if (g->part_round == 1) {
    if (g->n > 0) {
      lm::k_match_part_all<<<grid_for(((g->n + 31) / 32) * 32, 256, 65536), 256, 0, st>>>(
          g->best, g->n, g->v0, g->v0 + g->n, g->ghost, g->bits);
      CKL();
    }
  } else {
    // the frontier size is device-resident (not read back in peer-memory rounds): one wave
    lm::k_match_part_bins<<<(unsigned)(8 * g->num_sms), 256, 0, st>>>(
        g->F[g->part_cur], g->counters + lm::cnt_F(g->part_cur, 0), g->best, g->v0, g->v0 + g->n,
        g->ghost, g->bits);
    CKL();
  }
  if (P == 1) return LMATCH_OK;  // one part: no inbox, no replicas to update
  lm::k_match_inbox<<<(unsigned)grid, 256, 0, st>>>(g->win, g->win_cap, icnt, P, g->best, g->v0,
                                                     g->bits);
  CKL();
  // the inbox is consumed: its counts are zero again before any peer's next claims phase
  CK(cudaMemsetAsync(icnt, 0, (size_t)P * 8, st));
  const int64_t nw = (g->n + 31) / 32;
  if (nw > 0) {
    lm::k_push_bits<<<grid_for(nw, 256, 4 * g->num_sms), 256, 0, st>>>(g->bits, g->shadow, g->v0 / 32,
                                                                      nw, g->d_dbits, P, g->me);
    CKL();
  }
  return LMATCH_OK;
}

int lmatch_p2p_compact(lmatch_graph* g, void* stream, int64_t* nF_local) {
  TRY(p2p_ready(g));
  cudaStream_t st = stream ? (cudaStream_t)stream : g->stream;
  if (nF_local) {
    TRY(lmatch_part_compact(g, st, nF_local));  // synchronising variant (host needs the size)
  } else {
    CK(cudaSetDevice(g->device));
    TRY(part_compact_launch(g, st));
  }
  lm::k_push_count<<<1, 32, 0, st>>>(g->counters + lm::cnt_F(g->part_cur, 0), lm::kBins, g->d_dnf, g->P);
  CKL();
  return LMATCH_OK;
}

int lmatch_p2p_frontier_total(lmatch_graph* g, void* stream, int64_t* nF_total) {
  TRY(p2p_ready(g));
  if (!nF_total) { set_err("NULL nF_total"); return LMATCH_EINVAL; }
  CK(cudaSetDevice(g->device));
  cudaStream_t st = stream ? (cudaStream_t)stream : g->stream;
  const int P = g->P;
  CK(cudaMemcpyAsync(g->h_nf, g->win + (size_t)P * g->win_cap + P, (size_t)P * 8,
                     cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  int64_t t = 0;
  for (int p = 0; p < P; ++p) t += (int64_t)g->h_nf[p];
  *nF_total = t;
  return LMATCH_OK;
}

int lmatch_p2p_sync(lmatch_graph* g, void* stream) {
  if (!g) { set_err("NULL handle"); return LMATCH_ESTATE; }
  CK(cudaSetDevice(g->device));
  CK(cudaStreamSynchronize(stream ? (cudaStream_t)stream : g->stream));
  return LMATCH_OK;
}


// ------------------------------------------------------------- library-owned multi-GPU driver
// lmatch_partition / lmatch_create_dist / lmatch_run_dist: the 1-D
// edge-balanced partition (binary search on the CSR prefix sums), the peer-memory
// exchange set up by the library itself (the ranks find each other through a POSIX shared-memory
// rendezvous named by an lmatch_dist_id, like an ncclUniqueId), and the whole round loop --
// Alg. 2's per-device loop with the exchange redesigned -- driven by the library,
// with device-side barriers between the phases (no host barrier, one host read per round).
int lmatch_partition(const int64_t* offsets, int64_t n, int32_t nparts, int32_t align,
                     int64_t* bounds) {
  g_err[0] = 0;
  if (!offsets || !bounds) { set_err("NULL offsets or bounds"); return LMATCH_EINVAL; }
  if (n < 0 || n >= ((int64_t)1 << 31)) { set_err("n = %lld out of range", (long long)n); return LMATCH_ERANGE; }
  if (nparts < 1) { set_err("nparts = %d < 1", nparts); return LMATCH_EINVAL; }
  if (align <= 0) align = 32;
  if (offsets[0] != 0) { set_err("offsets[0] != 0"); return LMATCH_EINVAL; }
  const int64_t m = offsets[n];
  if (m < 0) { set_err("offsets[n] < 0"); return LMATCH_EINVAL; }
  bounds[0] = 0;
  for (int p = 1; p < nparts; ++p) {
    // first row whose start reaches p/P of the entries (floor(m p / P) without overflow)
    const int64_t target = (m / nparts) * p + ((m % nparts) * p) / nparts;
    const int64_t v = std::lower_bound(offsets, offsets + n + 1, target) - offsets;
    const int64_t va = std::min<int64_t>(n, (v + align - 1) / align * align);
    bounds[p] = std::max(bounds[p - 1], va);
  }
  bounds[nparts] = n;
  return LMATCH_OK;
}

int lmatch_dist_id_new(lmatch_dist_id* id) {
  if (!id) { set_err("NULL id"); return LMATCH_EINVAL; }
  unsigned long long r = 0;
  const int fd = open("/dev/urandom", O_RDONLY);
  if (fd >= 0) {
    if (read(fd, &r, sizeof r) != (ssize_t)sizeof r) r = 0;
    close(fd);
  }
  struct timespec ts;
  clock_gettime(CLOCK_REALTIME, &ts);
  std::memset(id->bytes, 0, sizeof id->bytes);
  snprintf(id->bytes, sizeof id->bytes, "lmatch-%x-%llx-%llx", (unsigned)getpid(),
           (unsigned long long)ts.tv_sec * 1000000000ull + (unsigned long long)ts.tv_nsec, r);
  return LMATCH_OK;
}

namespace {
// LMATCH_TRACE=1: the multi-GPU driver reports its steps on stderr; =2: it also drains its
// stream after every phase, so a failing phase is named (debugging aids)
int dist_trace_level() {
  static const int lv = [] { const char* e = getenv("LMATCH_TRACE"); return e ? atoi(e) : 0; }();
  return lv;
}
bool dist_trace() { return dist_trace_level() >= 1; }
#define DTRACE(g, ...)                                                                   \
  do {                                                                                   \
    if (dist_trace()) {                                                                  \
      fprintf(stderr, "[lmatch rank %d pid %d] ", (g)->me, (int)getpid());               \
      fprintf(stderr, __VA_ARGS__);                                                      \
      fputc('\n', stderr);                                                               \
    }                                                                                    \
  } while (0)
constexpr uint32_t kShmMagic = 0x4c4d4431u;  // "LMD1"
// how long a rank waits for its peers (rendezvous, barriers): LMATCH_DIST_TIMEOUT_S, default 60 s
unsigned long long dist_timeout_ns() {
  static const unsigned long long t = [] {
    const char* e = getenv("LMATCH_DIST_TIMEOUT_S");
    const long long v = e ? atoll(e) : 0;
    return (unsigned long long)(v > 0 ? v : 60) * 1000000000ull;
  }();
  return t;
}
#define kDistTimeoutNs dist_timeout_ns()
struct DistSlot {
  uint32_t valid;
  int32_t pid;
  int32_t device;
  int32_t nparts;
  int64_t v0, n, n_global, win_cap;
  uint64_t raw_win, raw_bits;   // device pointers, meaningful to a peer in the same process
  unsigned char ipc[128];       // lmatch_p2p_export handles, for peers in other processes
  // in-process barrier (all ranks in one process): the epoch this rank's stream recorded last,
  // and its two barrier events (cudaEvent_t, alternating by epoch parity)
  uint64_t recorded;
  uint64_t ev[2];
};
struct DistShm {
  uint32_t magic;
  int32_t world;
  int32_t attached;
  int32_t pad;
  DistSlot slot[1];
};

int shm_name(const lmatch_dist_id* id, char* out, size_t cap) {
  size_t k = 0;
  out[k++] = '/';
  for (size_t i = 0; i < sizeof id->bytes && id->bytes[i] && k + 1 < cap; ++i) {
    const char c = id->bytes[i];
    if ((c >= 'a' && c <= 'z') || (c >= 'A' && c <= 'Z') || (c >= '0' && c <= '9') || c == '-' || c == '_')
      out[k++] = c;
  }
  out[k] = 0;
  if (k < 8) { set_err("lmatch_dist_id is empty or malformed (use lmatch_dist_id_new)"); return LMATCH_EINVAL; }
  return LMATCH_OK;
}

// every rank publishes its window / bitmap (IPC handles and raw pointers) in the rendezvous,
// waits for all ranks, then attaches each peer: plain pointers within one process (peer access
// enabled across devices), CUDA IPC across processes.  The last rank to attach unlinks it.
int dist_bootstrap(lmatch_graph* g, const lmatch_dist_id* id, int rank, int world) {
  char name[96];
  TRY(shm_name(id, name, sizeof name));
  const size_t bytes = sizeof(DistShm) + (size_t)world * sizeof(DistSlot);
  const int fd = shm_open(name, O_CREAT | O_RDWR, 0600);
  if (fd < 0) { set_err("shm_open(%s) failed", name); return LMATCH_ENCCL; }
  struct stat sb;
  if (fstat(fd, &sb) != 0 || ((size_t)sb.st_size < bytes && ftruncate(fd, (off_t)bytes) != 0)) {
    close(fd);
    set_err("rendezvous %s: cannot size it", name);
    return LMATCH_ENCCL;
  }
  void* mp = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  close(fd);
  if (mp == MAP_FAILED) { set_err("rendezvous %s: mmap failed", name); return LMATCH_ENCCL; }
  DistShm* h = static_cast<DistShm*>(mp);
  int rc = LMATCH_OK;
  DTRACE(g, "rendezvous %s mapped", name);
  uint32_t zero = 0;
  __atomic_compare_exchange_n(&h->magic, &zero, kShmMagic, false, __ATOMIC_ACQ_REL, __ATOMIC_ACQUIRE);
  int32_t w0 = 0;
  __atomic_compare_exchange_n(&h->world, &w0, world, false, __ATOMIC_ACQ_REL, __ATOMIC_ACQUIRE);
  if (__atomic_load_n(&h->magic, __ATOMIC_ACQUIRE) != kShmMagic || __atomic_load_n(&h->world, __ATOMIC_ACQUIRE) != world) {
    set_err("rendezvous %s: world size mismatch (%d here)", name, world);
    rc = LMATCH_EINVAL;
  }
  DistSlot* me = &h->slot[rank];
  if (!rc) {
    if (__atomic_load_n(&me->valid, __ATOMIC_ACQUIRE)) {
      set_err("rendezvous %s: rank %d joined twice", name, rank);
      rc = LMATCH_EINVAL;
    }
  }
  if (!rc) {
    me->pid = (int32_t)getpid();
    me->device = g->device;
    me->nparts = g->P;
    me->v0 = g->v0;
    me->n = g->n;
    me->n_global = g->n_global;
    me->win_cap = g->win_cap;
    me->raw_win = (uint64_t)(uintptr_t)g->win;
    me->raw_bits = (uint64_t)(uintptr_t)g->bits;
    for (int i = 0; i < 2 && !rc; ++i) {
      if (cudaEventCreateWithFlags(&g->bev[i], cudaEventDisableTiming) != cudaSuccess) {
        set_err("cudaEventCreate failed");
        rc = LMATCH_ECUDA;
      }
      me->ev[i] = (uint64_t)(uintptr_t)g->bev[i];
    }
    __atomic_store_n(&me->recorded, 0ull, __ATOMIC_RELAXED);
    rc = lmatch_p2p_export(g, me->ipc);
    if (!rc) __atomic_store_n(&me->valid, 1u, __ATOMIC_RELEASE);
    DTRACE(g, "slot published (rc %d)", rc);
  }
  // wait for every rank
  struct timespec t0, t1;
  clock_gettime(CLOCK_MONOTONIC, &t0);
  for (int q = 0; !rc && q < world; ++q) {
    while (!__atomic_load_n(&h->slot[q].valid, __ATOMIC_ACQUIRE)) {
      clock_gettime(CLOCK_MONOTONIC, &t1);
      if ((t1.tv_sec - t0.tv_sec) * 1000000000ll + (t1.tv_nsec - t0.tv_nsec) > (long long)kDistTimeoutNs) {
        set_err("rendezvous %s: rank %d did not join within %llu s", name, q, kDistTimeoutNs / 1000000000ull);
        rc = LMATCH_ENCCL;
        break;
      }
      usleep(200);
    }
  }
  for (int q = 0; !rc && q < world; ++q) {
    if (q == rank) continue;
    const DistSlot& s = h->slot[q];
    if (s.nparts != g->P || s.n_global != g->n_global || s.win_cap != g->win_cap ||
        s.v0 != g->hbounds[q] || s.v0 + s.n != g->hbounds[q + 1]) {
      set_err("rank %d: partition does not match rank %d's part_bounds / n_global", q, rank);
      rc = LMATCH_EINVAL;
      break;
    }
    if (s.pid == (int32_t)getpid()) {
      if (s.device != g->device) {
        const cudaError_t e = cudaDeviceEnablePeerAccess(s.device, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) {
          set_err("cudaDeviceEnablePeerAccess(%d): %s", s.device, cudaGetErrorString(e));
          rc = LMATCH_ECUDA;
          break;
        }
        cudaGetLastError();
      }
      rc = p2p_set_peer(g, q, reinterpret_cast<uint64_t*>((uintptr_t)s.raw_win),
                        reinterpret_cast<uint32_t*>((uintptr_t)s.raw_bits));
    } else {
      rc = lmatch_p2p_attach(g, q, s.ipc);
    }
  }
  // every rank in this process: keep the mapping for the event barriers
  bool local = true;
  for (int q = 0; q < world; ++q) local = local && h->slot[q].pid == (int32_t)getpid();
  DTRACE(g, "peers attached (rc %d, %s)", rc, local ? "in-process event barriers" : "device flag barriers");
  // the last rank to attach removes the rendezvous; a rank that gave up waiting removes it too
  // (the group cannot complete), so no segment is left behind in /dev/shm
  if (__atomic_add_fetch(&h->attached, 1, __ATOMIC_ACQ_REL) == world || rc == LMATCH_ENCCL) shm_unlink(name);
  if (!rc && local) {
    g->dist_local = 1;
    g->dist_shm = mp;
    g->dist_shm_bytes = bytes;
  } else {
    munmap(mp, bytes);
  }
  return rc;
}

int dist_check(int64_t n_local, int64_t v_begin, int64_t n_global, int32_t rank, int32_t world,
               const int64_t* bounds, const lmatch_dist_id* id, const lmatch_opts* opts) {
  if (world < 1 || rank < 0 || rank >= world) { set_err("rank %d / world %d out of range", rank, world); return LMATCH_EINVAL; }
  if (!id) { set_err("NULL lmatch_dist_id"); return LMATCH_EINVAL; }
  TRY(check_part(n_local, v_begin, n_global, world, bounds));
  if (bounds[rank] != v_begin) { set_err("v_begin is not part_bounds[rank]"); return LMATCH_EINVAL; }
  if (opts && opts->validate_level >= 2) { set_err("validate_level 2 is not available per partition"); return LMATCH_EINVAL; }
  if (opts && opts->algorithm != 0) { set_err("lmatch_run_dist runs the LD iteration (algorithm 0) only"); return LMATCH_EINVAL; }
  return LMATCH_OK;
}

int dist_finish_create(lmatch_graph* g, int rank, int world, const lmatch_dist_id* id) {
  TRY(lmatch_p2p_enable(g, rank));
  TRY(dmalloc(g, &g->d_berr, 1));
  CK(cudaMemset(g->d_berr, 0, 4));
  CK(cudaHostAlloc(reinterpret_cast<void**>(&g->h_res6), (size_t)6 * g->P * 8 + 8, cudaHostAllocDefault));
  if (world > 1) TRY(dist_bootstrap(g, id, rank, world));
  g->dist = 1;
  return LMATCH_OK;
}
}  // namespace

int lmatch_create_dist(const int64_t* csr_offsets, const int32_t* col_idx, const float* weights,
                       int64_t n_local, int64_t m_local, int64_t v_begin, int64_t n_global,
                       int32_t rank, int32_t world, const int64_t* part_bounds,
                       const lmatch_dist_id* id, const lmatch_opts* opts, lmatch_graph** out) {
  if (!out) { set_err("out == NULL"); return LMATCH_EINVAL; }
  *out = nullptr;
  g_err[0] = 0;
  int s = check_args(csr_offsets, col_idx, weights, n_local, m_local);
  if (!s) s = dist_check(n_local, v_begin, n_global, rank, world, part_bounds, id, opts);
  if (s) return s;
  PartSpec ps;
  ps.v0 = v_begin; ps.n_global = n_global; ps.P = world; ps.bounds = part_bounds;
  lmatch_graph* g = nullptr;
  s = create_common(n_local, m_local, opts, out, &g, &ps);
  if (!s) s = upload_host(g, csr_offsets, col_idx, weights);
  if (!s) s = finish_create(g, g->stream);
  if (!s) s = dist_finish_create(g, rank, world, id);
  if (s) { lmatch_destroy(g); return s; }
  *out = g;
  return LMATCH_OK;
}

int lmatch_create_dist_device(const int64_t* d_offsets, const int32_t* d_col, const float* d_weights,
                              int64_t n_local, int64_t m_local, int64_t v_begin, int64_t n_global,
                              int32_t rank, int32_t world, const int64_t* part_bounds,
                              const lmatch_dist_id* id, const lmatch_opts* opts, void* stream,
                              lmatch_graph** out) {
  if (!out) { set_err("out == NULL"); return LMATCH_EINVAL; }
  *out = nullptr;
  g_err[0] = 0;
  int s = check_args(d_offsets, d_col, d_weights, n_local, m_local);
  if (!s) s = dist_check(n_local, v_begin, n_global, rank, world, part_bounds, id, opts);
  if (s) return s;
  PartSpec ps;
  ps.v0 = v_begin; ps.n_global = n_global; ps.P = world; ps.bounds = part_bounds;
  lmatch_graph* g = nullptr;
  s = create_common(n_local, m_local, opts, out, &g, &ps);
  cudaStream_t st = stream ? (cudaStream_t)stream : (g ? g->stream : nullptr);
  if (!s) {
    cudaError_t e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) { set_err("stream sync: %s", cudaGetErrorString(e)); s = LMATCH_ECUDA; }
  }
  if (!s) s = upload_device(g, d_offsets, d_col, d_weights, st);
  if (!s) s = finish_create(g, st);
  if (!s) s = dist_finish_create(g, rank, world, id);
  if (s) { lmatch_destroy(g); return s; }
  *out = g;
  return LMATCH_OK;
}

int lmatch_run_dist_device(lmatch_graph* g, int32_t* d_mate_local, void* stream, lmatch_stats* stats) {
  if (!g || !g->dist) { set_err("not a lmatch_create_dist handle"); return LMATCH_ESTATE; }
  if (!d_mate_local && g->n > 0) { set_err("d_mate_local == NULL"); return LMATCH_EINVAL; }
  g_err[0] = 0;
  CK(cudaSetDevice(g->device));
  cudaStream_t st = stream ? (cudaStream_t)stream : g->stream;
  const int P = g->P;
  const long long l0 = t_launch_count;
  unsigned long long* wslots = reinterpret_cast<unsigned long long*>(g->win + (size_t)P * g->win_cap);
  // wslots: [0,P) inbox counts, [P,2P) frontier sizes, [2P,3P) barrier flags, [3P,4P) w shares,
  // [4P,5P) matched counts
  // Ranks in other processes: a device-side barrier kernel (system-scope flags in the peers'
  // windows).  Ranks all in this process share one CUDA context, where a spinning kernel could be
  // serialised behind another thread's work: each rank records an event on its stream, publishes
  // the epoch in the rendezvous mapping, waits on the host until every rank has recorded it, and
  // makes its stream wait for the peers' events (no stream is drained; two events per rank,
  // alternating by epoch, so a rank one barrier ahead never overwrites a record still needed).
  auto barrier = [&]() -> int {
    if (P == 1) return LMATCH_OK;
    ++g->epoch;
    DTRACE(g, "barrier %llu", g->epoch);
    if (!g->dist_local) {
      lm::k_dist_barrier<<<1, 32, 0, st>>>(wslots + 2 * P, g->d_dflag, P, g->me, g->epoch,
                                           kDistTimeoutNs, g->d_berr);
      CKL();
      return LMATCH_OK;
    }
    DistShm* h = static_cast<DistShm*>(g->dist_shm);
    const int par = (int)(g->epoch & 1);
    CK(cudaEventRecord(g->bev[par], st));
    __atomic_store_n(&h->slot[g->me].recorded, (uint64_t)g->epoch, __ATOMIC_RELEASE);
    struct timespec t0, t1;
    clock_gettime(CLOCK_MONOTONIC, &t0);
    for (int q = 0; q < P; ++q) {
      if (q == g->me) continue;
      while (__atomic_load_n(&h->slot[q].recorded, __ATOMIC_ACQUIRE) < (uint64_t)g->epoch) {
        clock_gettime(CLOCK_MONOTONIC, &t1);
        if ((t1.tv_sec - t0.tv_sec) * 1000000000ll + (t1.tv_nsec - t0.tv_nsec) > (long long)kDistTimeoutNs) {
          set_err("rank %d did not reach barrier %llu within %llu s", q, g->epoch, kDistTimeoutNs / 1000000000ull);
          return LMATCH_ENCCL;
        }
      }
      CK(cudaStreamWaitEvent(st, reinterpret_cast<cudaEvent_t>((uintptr_t)h->slot[q].ev[par]), 0));
    }
    return LMATCH_OK;
  };
  // one host read: the P frontier sizes (and the barrier error flag)
  auto read_slots = [&](int64_t* total) -> int {
    CK(cudaMemcpyAsync(g->h_res6, wslots + P, (size_t)P * 8, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(g->h_res6 + 5 * P, g->d_berr, 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (*reinterpret_cast<unsigned*>(g->h_res6 + 5 * P)) {
      set_err("a peer did not reach a device barrier within %llu s", kDistTimeoutNs / 1000000000ull);
      return LMATCH_ENCCL;
    }
    int64_t t = 0;
    for (int p = 0; p < P; ++p) t += (int64_t)g->h_res6[p];
    *total = t;
    return LMATCH_OK;
  };
  // LMATCH_TRACE=2: also drain the stream after every phase, so a failing phase is named
  auto phase = [&](const char* what) -> int {
    if (dist_trace_level() < 2) return LMATCH_OK;
    const cudaError_t e = cudaStreamSynchronize(st);
    DTRACE(g, "phase %s done: %s", what, cudaGetErrorString(e));
    CK(e);
    return LMATCH_OK;
  };
  if (g->timing && stats) CK(cudaEventRecord(g->ev[0], st));
  CK(cudaMemsetAsync(g->d_berr, 0, 4, st));
  TRY(barrier());  // every part is done with its previous run (inboxes, replicas, slots)
  TRY(phase("barrier"));
  TRY(part_begin_impl(g, st, nullptr));
  TRY(phase("begin"));
  int64_t rounds = 1;
  bool compacted = false, capped = false;
  if (P == 1) {
    // one rank: nothing to exchange, so the round loop is the single-GPU one -- the frontier
    // size read after each compaction sizes the next match, compaction and pointer launches
    // exactly, and the small tail runs in the persistent cooperative kernel (no host round trips)
    g->one_rank_loop = g->v0 == 0 && g->n_global == g->n;
    struct Off {
      lmatch_graph* g;
      ~Off() { g->one_rank_loop = false; }
    } off{g};
    for (;;) {
      TRY(lmatch_p2p_match(g, st));
      TRY(lmatch_p2p_compact(g, st, nullptr));
      CK(cudaMemcpyAsync(g->h_counters, g->counters, lm::kNumCounters * 8, cudaMemcpyDeviceToHost, st));
      CK(cudaStreamSynchronize(st));
      int64_t nF = 0;
      for (int b = 0; b < lm::kBins; ++b) nF += (int64_t)g->h_counters[lm::cnt_F(g->part_cur, b)];
      if (nF == 0) break;
      if (rounds >= g->max_rounds) { capped = true; break; }
      ++rounds;
      if (g->round_loop == 0 && nF <= kPersistentBelow) {
        // k_end_round left the state of the next round in rstate (same cur as part_cur)
        int64_t l = 0;
        TRY(launch_persistent(g, st, &l));
        CK(cudaMemcpyAsync(g->h_rstate, g->rstate, sizeof(lm::RoundState), cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(g->h_counters, g->counters, lm::kNumCounters * 8, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        rounds = g->h_rstate->rounds;  // pointing phases begun, as counted by k_end_round
        int64_t left = 0;
        for (int b = 0; b < lm::kBins; ++b) left += (int64_t)g->h_counters[lm::cnt_F(g->h_rstate->cur, b)];
        capped = left > 0;
        break;
      }
      g->counts_on_host = true;
      TRY(part_point_impl(g, st, nullptr));
    }
  }
  for (; P > 1;) {
    TRY(barrier());  // claims are in the owners' inboxes; frontier sizes in every slot
    if (compacted) {
      int64_t total = 0;
      TRY(read_slots(&total));
      DTRACE(g, "round %lld: global frontier %lld", (long long)rounds, (long long)total);
      if (total == 0) break;
      if (rounds >= g->max_rounds) { capped = true; break; }  // same decision on every part
      ++rounds;
    }
    TRY(phase("barrier"));
    TRY(lmatch_p2p_match(g, st));
    TRY(phase("match"));
    TRY(barrier());  // bitmap replicas complete
    TRY(phase("barrier"));
    TRY(lmatch_p2p_compact(g, st, nullptr));
    TRY(phase("compact"));
    compacted = true;
    TRY(part_point_impl(g, st, nullptr));  // an empty global frontier launches only empty work
    TRY(phase("point"));
  }
  // A10 owned mate[] slice + A9: this part's w(M) share, then every part's shares summed in part
  // order (the same fp64 total on every part)
  if (g->n > 0) {
    lm::k_materialize<kFinThreads><<<kFinBlocks, kFinThreads, 0, st>>>(g->best, g->bits, g->n, g->v0,
                                                                       d_mate_local, g->pw, g->pc);
    CKL();
    lm::k_final_sum<<<1, 32, 0, st>>>(g->pw, g->pc, kFinBlocks, g->res_w, g->res_c);
    CKL();
  } else {
    CK(cudaMemsetAsync(g->res_w, 0, 8, st));
    CK(cudaMemsetAsync(g->res_c, 0, 8, st));
  }
  TRY(phase("finish"));
  lm::k_push_result<<<1, 32, 0, st>>>(g->res_w, g->res_c, g->d_dresw, g->d_dresc, P);
  CKL();
  TRY(phase("push result"));
  TRY(barrier());
  TRY(phase("barrier"));
  CK(cudaMemcpyAsync(g->h_res6 + P, wslots + 3 * P, (size_t)2 * P * 8, cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(g->h_counters, g->counters, lm::kNumCounters * 8, cudaMemcpyDeviceToHost, st));
  int64_t dummy = 0;
  TRY(read_slots(&dummy));  // also synchronises and checks the barrier flag
  if (g->timing && stats) CK(cudaEventRecord(g->ev[5], st));
  double wsum = 0.0;
  int64_t csum = 0;
  for (int p = 0; p < P; ++p) {
    double w;
    std::memcpy(&w, &g->h_res6[P + p], 8);
    wsum += w;
    csum += (int64_t)g->h_res6[2 * P + p];
  }
  if (stats) {
    std::memset(stats, 0, sizeof *stats);
    stats->rounds = rounds;
    stats->matched_vertices = csum;
    stats->cardinality = csum / 2;
    stats->weight = wsum;
    stats->entries_swept = g->m + (int64_t)g->h_counters[lm::kCntSwept];
    stats->kernel_launches = t_launch_count - l0;
    stats->sweep_launches = 1;
    stats->resident_entries = g->R;
    if (g->timing) {
      float a = 0;
      CK(cudaEventSynchronize(g->ev[5]));
      CK(cudaEventElapsedTime(&a, g->ev[0], g->ev[5]));
      stats->ms_total = a;
      double sw = 0;
      TRY(lmatch_part_info(g, nullptr, &sw));
      stats->ms_sweep = sw;
    }
  }
  if (capped) {
    set_err("frontier left after the round cap (%lld pointing phases)", (long long)rounds);
    return LMATCH_EROUNDS;
  }
  return LMATCH_OK;
}

int lmatch_run_dist(lmatch_graph* g, int32_t* mate_local, lmatch_stats* stats) {
  if (!g || !g->dist) { set_err("not a lmatch_create_dist handle"); return LMATCH_ESTATE; }
  if (!mate_local && g->n > 0) { set_err("mate_local == NULL"); return LMATCH_EINVAL; }
  CK(cudaSetDevice(g->device));
  if (!g->mate_tmp) TRY(dmalloc(g, &g->mate_tmp, (size_t)g->n + 1));
  const int rc = lmatch_run_dist_device(g, g->mate_tmp, g->stream, stats);
  if (rc != LMATCH_OK && rc != LMATCH_EROUNDS) return rc;
  if (g->n > 0) {
    CK(cudaMemcpyAsync(mate_local, g->mate_tmp, (size_t)g->n * 4, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaStreamSynchronize(g->stream));
  }
  return rc;
}

}  // extern "C"
