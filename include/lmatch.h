/* lmatch.h -- C ABI of the B200-native pointer-based locally dominant matching library.
 *
 * Computes the 1/2-approximate maximum weight matching of Mandulak et al., "Efficient Weighted
 * Graph Matching on GPUs" (SC'24): the maximal *locally dominant* matching (Def. II.1,
 * PAPER.md:46; Lemma II.1) reached by the pointer-based iteration of Algorithm 1
 * (LD-SEQ) / Algorithms 2-3 (LD-GPU): every round each
 * unmatched vertex points to its heaviest unmatched neighbour, mutually pointing pairs are
 * matched, and matched vertices are retired until no pointer changes.
 *
 * Edge order (R1): the paper's "greater or equal" is made strict: at a
 * vertex u, neighbour v beats v' iff w(u,v) > w(u,v') or (w equal and v > v').  This is the
 * restriction of one global strict order on edges, so the result is the UNIQUE maximal locally
 * dominant matching (= the sequential greedy matching) and is bit-identical for every
 * run, GPU count, tile size and streaming configuration.
 *
 * Graph input (CSR "separate vertex, edge, and value arrays"):
 *   csr_offsets  int64[n+1]  row pointers; offsets[0] = 0, non-decreasing, offsets[n] = m
 *   col_idx      int32[m]    neighbour ids in [0, n); each undirected edge appears in both rows
 *   weights      float32[m]  edge weights, finite and > 0 ("w : E -> R>0");
 *                            w(u,v) must equal w(v,u)
 *   n < 2^31 vertices; m = number of DIRECTED entries (= 2 x undirected edges).
 *   Self-loops are ignored (the paper assumes a simple graph).  Repeated entries
 *   (u,v) with equal weights are harmless.  Rows need not be sorted.
 *
 * Output: mate int32[n]; mate[u] = v if {u,v} is matched, -1 if u is unmatched
 *   (Alg. 1/2 "Output: ... matching in mate array").
 *
 * Errors: every function returns an lmatch_status (0 = OK, < 0 = error).  The library never
 * aborts and no C++ exception crosses this ABI; lmatch_last_error() returns a thread-local
 * human-readable detail of the last failure on the calling thread.
 *
 * Ownership: all input arrays are caller-owned and only read during the call that receives them.
 * The handle owns every device allocation and stream it creates.  One handle must not be used
 * from two threads at once; distinct handles are independent.
 */
#ifndef LMATCH_H_
#define LMATCH_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define LMATCH_ABI_VERSION 4

#if defined(__GNUC__)
#define LMATCH_API __attribute__((visibility("default")))
#else
#define LMATCH_API
#endif

typedef enum lmatch_status {
  LMATCH_OK = 0,
  LMATCH_EINVAL = -1, /* malformed CSR: offsets[0] != 0, decreasing offsets, offsets[n] != m,
                         col out of [0,n), weight NaN/inf/<= 0/-0.0, NULL pointer, or
                         (validate_level 2) an asymmetric graph */
  LMATCH_ERANGE = -2, /* n >= 2^31 or n < 0 or m < 0 */
  LMATCH_ENOMEM = -3, /* device or pinned-host allocation failed */
  LMATCH_ECUDA = -4,  /* CUDA runtime / kernel failure (detail in lmatch_last_error) */
  LMATCH_ENCCL = -5,  /* multi-GPU exchange failure: a rank did not join a lmatch_create_dist
                         rendezvous or reach a device barrier in time, or the rendezvous
                         could not be created */
  LMATCH_ESTATE = -6, /* misuse: NULL handle, size mismatch on reload, ... */
  LMATCH_EROUNDS = -7 /* the round cap (lmatch_opts.max_rounds) stopped the iteration with vertices
                         still to re-point: the contents of the mate output are unspecified.
                         Never returned with the default cap (n/2 + 2 bounds the pointing phases,
                         DESIGN.md R6) */
} lmatch_status;

/* Opaque handle: one graph resident on one GPU (packed adjacency + per-vertex state). */
typedef struct lmatch_graph lmatch_graph;

/* Options for lmatch_create_ex / lmatch_create_device.  Zero-initialise, then set fields;
 * every zero field means "default". */
typedef struct lmatch_opts {
  int32_t device;          /* CUDA device ordinal; default (0 with flag unset) = current device.
                              Set use_device = 1 to honour `device`. */
  int32_t use_device;
  int32_t validate_level;  /* 0 = default (1); 1 = ranges + weights + offsets;
                              2 = also symmetry and repeated edges ("simple undirected
                              graph"; SURVEY 8(b) EINVAL rule): the multiset of (u,v,w) must equal
                              that of (v,u,w) (a 64-bit multiset hash: a false accept needs a
                              hash collision), and a pair (u,v) listed more than once in row u
                              must repeat the same weight (exact: every row is sorted by
                              (v, weight bits) in scratch memory, in chunks of <= 2^27 entries,
                              and neighbouring entries are compared);
                              -1 = skip validation (caller guarantees a valid CSR, including
                              weights finite and > 0: the sweep's key max relies on it) */
  int32_t timing;          /* 1 = record CUDA events per phase into lmatch_stats */
  int64_t max_rounds;      /* 0 = default: n/2 + 2 (the strict order bounds rounds by n/2+1).
                              A smaller cap that stops the iteration with a non-empty frontier
                              makes lmatch_run* return LMATCH_EROUNDS (all algorithms) */
  int64_t upload_chunk;    /* entries per host->device upload chunk (0 = default 2^25) */
  int64_t hbm_budget_bytes;   /* 0 = adjacency fully resident.  Otherwise, if 8*m exceeds it, only a
                                 prefix of the packed adjacency stays in HBM; the rest lives in
                                 library-owned pinned host memory, is streamed through a device
                                 ring in round 1 (LOADBATCH, Alg. 2 L10-12; double
                                 buffering) and read zero-copy by later rounds */
  int64_t stream_chunk;       /* entries per streamed chunk (0 = default 2^24; rounded to the
                                 sweep tile) */
  int32_t round_loop;         /* 0 = default, hybrid: work-sized per-round launches while the
                                 frontier is large, then ONE persistent cooperative kernel runs all
                                 remaining rounds (grid barriers between phases, no host round
                                 trips); 1 = host-driven per-round launches only; 2 = persistent
                                 kernel for every round after round 1; 3 = CUDA graph {round 1,
                                 persistent kernel}.  Out-of-core: 3 behaves as 2. */
  int32_t prune;              /* 1 = A7 in-place pruning (not in the paper): a
                                 frontier row that fits one pointer batch (<= 8 / 64 / 128
                                 entries for the 1/8/32-lane bins) is partitioned in place,
                                 entries with an unmatched neighbour first, and later rounds of
                                 the same run scan only that prefix.  The adjacency stays a
                                 per-row permutation of the input, so the result and later runs
                                 are unchanged.  Ignored for out-of-core and partition handles.
                                 0 = default (off: measured slower on R-MAT) */
  int32_t host_cache;         /* out-of-core only: 0 = default (on), -1 = off.
                                 Every row with entries beyond the resident prefix keeps its 8
                                 largest keys in HBM (64 bytes per such row, allocated on top of
                                 hbm_budget_bytes and reported in lmatch_stats.cache_bytes),
                                 filled in round 1 from the streamed chunks.  Later rounds take
                                 the pointer from the cache when one of the cached neighbours is
                                 unmatched (the first such key is the row maximum over available
                                 neighbours), so only rows whose 8 heaviest neighbours are all
                                 matched are read from host memory.  Same result.  Rounds >= 2
                                 of an out-of-core run with the cache are host-driven launches */
  int32_t batches;            /* paper-style batch count N_i (Alg. 2 L3-5; SURVEY 8(f)
                                 NEXT-2): 0 or 1 = default (resident, or hbm_budget_bytes decides);
                                 B > 1 = nothing resident: the adjacency lives in pinned host
                                 memory as B entry-balanced batches (tile-rounded; a row spanning
                                 two batches is merged with the u64 max) streamed through
                                 the 2-slot device ring in round 1 (2 streams,
                                 double buffering).  Overrides hbm_budget_bytes and
                                 stream_chunk */
  int32_t algorithm;          /* 0 = default: the pointer-based LD iteration (Alg. 1-3).  1 = Suitor
                                 (the paper's SR comparison algorithm,
                                 P:84-86): proposals accepted by a u64 atomicMax on the receiver's
                                 best offer, displaced proposers try again; no synchronous
                                 rounds of mutual checks.  Same unique result under R1 (the
                                 certificate and the oracle decide).  2 = hybrid: the LD
                                 iteration, and if a frontier is left after 32 pointing phases
                                 (many-round graphs, e.g. weight gradients along paths), Suitor on
                                 the graph without the vertices matched so far completes the same
                                 matching (lmatch_stats.tail_passes).  1 and 2: resident
                                 single-graph handles only (1: EINVAL with out-of-core /
                                 partition handles; 2 behaves as 0 there).
                                 3 = sorted adjacency + cursor: the first run
                                 after create/reload sorts every row by key, descending, in place
                                 (the row's entries are permuted, never changed; this time is
                                 lmatch_stats.ms_sort), then each vertex's pointer is the first
                                 entry at or after its cursor whose neighbour is unmatched (Alg. 1
                                 L4).  Same unique result under R1.  Resident single-graph
                                 handles only (EINVAL otherwise).  The sort needs
                                 max(min(m, sort_chunk), longest row) x 8 B of scratch device memory
                                 for the keys, plus cub's temporary storage and 4 B per row of a
                                 chunk for its segment offsets, all freed before the run (ENOMEM,
                                 with the size, when they cannot be allocated) */
  int32_t sort_chunk_log2;    /* algorithm 3: rows are sorted in chunks of at most 2^sort_chunk_log2
                                 entries (a longer row is one chunk of its own); 0 = default (30).
                                 Valid 4..30 (EINVAL otherwise); small values exercise the chunking.
                                 Also caps the chunks of the validate_level-2 duplicate check */
  int32_t key_cache;          /* resident handles, algorithms 0 and 2:
                                 1 = on (when the cache fits in device memory); 0 = default, off
                                 (measured: on R-MAT s26 it saves 1.7 ms of the frontier rounds
                                 but costs the round-1 sweep 6.6 ms).
                                 The round-1 sweep keeps the 4 largest keys of every row (32 bytes
                                 per vertex, plus 64 bytes per sweep tile of scratch); a vertex
                                 whose target was matched then takes the first available cached
                                 key as its new pointer -- Alg. 1's pointer, since every larger key
                                 of the row is cached and matched -- and only rows whose cached
                                 keys are all matched are scanned again.  Same result, same
                                 pointing phases; lmatch_stats.entries_swept counts the rows
                                 actually scanned, cache_rows the pointers the cache decided */
  int32_t residual_mb;        /* out of core with the host-row cache (residual
                                 rows): 0 = default (off); R > 0 = up to R MiB of HBM (on top of
                                 hbm_budget_bytes, capped by free memory) for copies of host rows.
                                 A host row that is rescanned (its 8 cached keys all matched) is
                                 read over PCIe anyway; it is then also copied into this buffer
                                 while space lasts, and later rounds -- and later runs on the same
                                 graph -- scan the HBM copy instead (no extra PCIe traffic).
                                 lmatch_stats.residual_rows counts the rows scanned from it */
  int32_t frontier;           /* A6 next-frontier construction in the persistent-kernel rounds
                                 (round_loop 0, 2, 3): 0 = default, pull (compaction of the live
                                 list) switching to push once the live list is 8x the frontier
                                 and at least 2^20 vertices long (the vertices newly matched in a
                                 round push their row neighbours that pointed at them: O(m) over
                                 the run instead of O(|L| x rounds) -- many-round graphs);
                                 1 = pull only; 2 = push as soon as the live list is 8x the
                                 frontier, whatever its length.  Not with prune or algorithm 2.
                                 Same result and pointing phases */
  int32_t reserved[3];
} lmatch_opts;

/* Filled by lmatch_run / lmatch_run_device when non-NULL. */
typedef struct lmatch_stats {
  int64_t rounds;            /* pointing phases executed (round 1 = full sweep); algorithm 1:
                                Suitor passes (pass 1 = the sweep's row maxima); algorithm 2:
                                LD phases before the handoff (see tail_passes) */
  int64_t matched_vertices;  /* 2 x |M| */
  int64_t cardinality;       /* |M| */
  double weight;             /* w(M) = sum of matched edge weights, fp64 */
  int64_t entries_swept;     /* adjacency entries of the rows scanned over all rounds (rows the
                                out-of-core cache decided are counted with their full degree;
                                host_entries_read has the host part actually read) */
  int64_t frontier_total;    /* sum over rounds >= 2 of |F_r| (vertices re-pointed) */
  double ms_total;           /* (timing=1) lmatch_run_device body, device time */
  double ms_sweep;           /* (timing=1) round-1 pointer sweep kernel alone */
  double ms_rounds;          /* (timing=1) rounds >= 2 (pointer + match + compaction) */
  double ms_round1_rest;     /* (timing=1) round-1 match + compaction */
  double ms_finish;          /* (timing=1) mate materialisation + weight reduction */
  int64_t sweep_launches;    /* kernel launches of the round-1 sweep (1) */
  int64_t kernel_launches;   /* all kernel launches issued by this run */
  int64_t bytes_streamed;    /* host->device adjacency bytes copied by this run (out-of-core) */
  int64_t resident_entries;  /* adjacency entries resident in HBM (= m unless out-of-core) */
  int64_t cache_rows;        /* rounds >= 2: frontier rows whose pointer a key cache decided
                                without scanning the row (out of core: the host-row cache;
                                resident: the key cache, opts.key_cache) */
  int64_t host_entries_read; /* out-of-core: host-resident entries read zero-copy in rounds >= 2 */
  int64_t cache_bytes;       /* out-of-core: device bytes of the host-row cache (0 = none) */
  int64_t tail_passes;       /* algorithm 2: Suitor passes that completed the run after the LD
                                iteration stopped at 32 pointing phases (0 = not needed) */
  double ms_sort;            /* algorithm 3: device time of the row sort this run performed (the
                                first run after create/reload); 0 when the rows were already sorted */
  int64_t residual_rows;     /* out of core, opts.residual_mb: frontier rows of rounds >= 2
                                scanned from their HBM residual copy instead of host memory */
} lmatch_stats;

/* Library / ABI identification.  Returns LMATCH_ABI_VERSION. */
LMATCH_API int lmatch_abi_version(void);
/* Kernels this library has launched in this process so far (all handles; a captured CUDA graph
 * counts its launches once, at capture).  Callers take differences around a region. */
LMATCH_API int64_t lmatch_kernel_launch_count(void);
/* Adjacency entries per round-1 sweep tile of handle g (the configuration follows the average
 * degree; NULL: the dense configuration's tile).  The sweep reads one 4-byte tile index entry per
 * tile: the tile term of its algorithmic bytes, DESIGN.md section 7. */
LMATCH_API int32_t lmatch_sweep_tile(const lmatch_graph* g);

/* Build a handle from HOST CSR arrays (copied to the device in chunks, packed into 64-bit
 * (weight-bits << 32 | neighbour) keys, validated, and indexed for the round-1 sweep).
 * `out` receives the handle (NULL on failure).  Equivalent to lmatch_create_ex(..., NULL, out). */
LMATCH_API int lmatch_create(const int64_t* csr_offsets, const int32_t* col_idx, const float* weights,
                  int64_t n, int64_t m, lmatch_graph** out);

LMATCH_API int lmatch_create_ex(const int64_t* csr_offsets, const int32_t* col_idx, const float* weights,
                     int64_t n, int64_t m, const lmatch_opts* opts, lmatch_graph** out);

/* Same, but the three arrays are DEVICE pointers on the selected device (e.g. torch tensors'
 * data_ptr()).  No host<->device copies; `stream` (cudaStream_t, may be NULL = legacy default)
 * orders the reads of the caller's arrays. */
LMATCH_API int lmatch_create_device(const int64_t* d_offsets, const int32_t* d_col, const float* d_weights,
                         int64_t n, int64_t m, const lmatch_opts* opts, void* stream,
                         lmatch_graph** out);

/* Re-upload a graph with the SAME n and m from host arrays into an existing handle (reuses all
 * device buffers; used for end-to-end timing).  ESTATE if sizes differ. */
LMATCH_API int lmatch_reload(lmatch_graph* g, const int64_t* csr_offsets, const int32_t* col_idx,
                  const float* weights);

/* Compute the matching.  mate_out: HOST int32[n], caller-allocated (pinned memory gives the
 * fastest copy).  stats may be NULL.  Returns after mate_out is complete. */
LMATCH_API int lmatch_run(lmatch_graph* g, int32_t* mate_out, lmatch_stats* stats);

/* Compute the matching into a DEVICE int32[n] buffer on `stream` (cudaStream_t; NULL = the
 * handle's own stream).  Synchronises `stream` before returning (the round loop reads the
 * frontier size each round). */
LMATCH_API int lmatch_run_device(lmatch_graph* g, int32_t* d_mate, void* stream, lmatch_stats* stats);

/* w(M) = sum over pairs {u, mate[u]} of w(u, mate[u]) in fp64, for ANY mate[]
 * (host int32[n]).  EINVAL if mate[] is not a symmetric set of edges of the graph. */
LMATCH_API int lmatch_weight(lmatch_graph* g, const int32_t* mate, double* out_weight);

/* Same with a DEVICE mate buffer, ordered on `stream` (NULL = handle stream); synchronises. */
LMATCH_API int lmatch_weight_device(lmatch_graph* g, const int32_t* d_mate, void* stream,
                         double* out_weight);

/* Graph facts: n, m, non-empty rows, device bytes held by the handle. Any pointer may be NULL. */
LMATCH_API int lmatch_info(const lmatch_graph* g, int64_t* n, int64_t* m, int64_t* nonempty_rows,
                int64_t* device_bytes);

/* Per-round log of the last lmatch_run*: for round r (0-based), out[3r] = |F_r| (vertices whose
 * pointer was computed; round 0 = every non-empty row), out[3r+1] = |L_r| (live vertices scanned
 * by the compaction), out[3r+2] = E(F_r) (adjacency entries scanned).  Writes at most `cap` rounds;
 * *nrounds receives the number of rounds.  (Fig. 8 "edges accessed per iteration".) */
LMATCH_API int lmatch_round_log(const lmatch_graph* g, int64_t* out, int64_t cap, int64_t* nrounds);

/* (timing = 1) Device time of the host-driven rounds >= 2 of the last lmatch_run* on a
 * single-graph handle: ms[i] = round i + 2 (writes at most `cap`), *nrounds = how many were timed.
 * When the default round loop handed the small tail to the persistent kernel, the LAST timed entry
 * is that whole tail and *tail_from = its index (else -1).  0 rounds without timing. */
LMATCH_API int lmatch_round_ms(const lmatch_graph* g, double* ms, int64_t cap, int64_t* nrounds,
                               int64_t* tail_from);

/* Rounds of the last lmatch_run* whose next frontier was pushed (opts.frontier; 0 = all pulled). */
LMATCH_API int lmatch_push_rounds(const lmatch_graph* g, int64_t* push_rounds);

/* ---------------------------------------------------------------------------------------------
 * Partitioned mode (multi-GPU, one process or thread per GPU).
 *
 * The vertex set is cut into nparts contiguous ranges part_bounds[0..nparts] (part_bounds[0] = 0,
 * part_bounds[nparts] = n_global, every bound a multiple of 32), balanced by directed entries
 * (P:96-98).  Each handle owns the rows of one range [v_begin, v_begin + n_local): a local
 * CSR whose col_idx are GLOBAL vertex ids (cut edges appear in both owners' rows).
 *
 * The caller (e.g. paper_conf_sc_mandulakgfhs24_b200/dist.py over torch.distributed) drives the
 * rounds and moves the data between handles:
 *   lmatch_part_begin   -> round-1 pointers + claims         (per destination counts)
 *   [exchange claims: segment p of every handle goes to the owner of part p]
 *   lmatch_part_apply   -> record received claims, match       (mutual pointer check)
 *   [allgather: every handle's owned bitmap words into every handle's bitmap]
 *   lmatch_part_compact -> live set, next frontier             (local frontier size)
 *   [stop when the SUM of frontier sizes over all parts is 0]
 *   lmatch_part_point   -> frontier pointers + claims; then back to the exchange
 *   lmatch_part_finish  -> owned mate[] slice, local w(M) share (edges with mate > u)
 * A claim (v | u << 32) says "remote vertex u points to owned vertex v"; it replaces the paper's
 * |V| x 64-bit nccl_AllReduce(pointers) (Alg. 2 L7), and the bitmap allgather (n/8 bytes)
 * replaces nccl_AllReduce(mate) (Alg. 2 L9).  The result is bit-identical to the
 * single-GPU run for every partition (Lemma III.1).  validate_level 2 is not available
 * per partition (EINVAL: symmetry is a global property).  Out of core works per part as for a
 * single graph (hbm_budget_bytes / batches = the paper's per-device batch count N_i, P:106, P:217;
 * the host-row key cache included).  Calls out of order return ESTATE.
 * ------------------------------------------------------------------------------------------- */
LMATCH_API int lmatch_create_part(const int64_t* csr_offsets, const int32_t* col_idx,
                                  const float* weights, int64_t n_local, int64_t m_local,
                                  int64_t v_begin, int64_t n_global, int32_t nparts,
                                  const int64_t* part_bounds, const lmatch_opts* opts,
                                  lmatch_graph** out);
LMATCH_API int lmatch_create_part_device(const int64_t* d_offsets, const int32_t* d_col,
                                         const float* d_weights, int64_t n_local, int64_t m_local,
                                         int64_t v_begin, int64_t n_global, int32_t nparts,
                                         const int64_t* part_bounds, const lmatch_opts* opts,
                                         void* stream, lmatch_graph** out);
/* Reset + round-1 pointer sweep over the owned rows + claims.  claim_counts: host int64[nparts]
 * (claims destined to each part; the own part's entry is 0).  Synchronises `stream`. */
LMATCH_API int lmatch_part_begin(lmatch_graph* g, void* stream, int64_t* claim_counts);
/* seg_ptrs: host array of nparts DEVICE pointers; segment p holds claim_counts[p] uint64 claims. */
LMATCH_API int lmatch_part_claims(const lmatch_graph* g, uint64_t** seg_ptrs);
/* d_recv: DEVICE uint64[nrecv], all claims whose target this handle owns (any order). */
LMATCH_API int lmatch_part_apply(lmatch_graph* g, const uint64_t* d_recv, int64_t nrecv,
                                 void* stream);
/* The replicated matched bitmap (DEVICE uint32[nwords_total]); this handle writes only words
 * [word_begin, word_begin + nwords_own). */
LMATCH_API int lmatch_part_bitmap(lmatch_graph* g, uint32_t** d_bits, int64_t* word_begin,
                                  int64_t* nwords_own, int64_t* nwords_total);
/* Copy helpers for callers that keep their exchange buffers elsewhere (e.g. torch tensors):
 * claims of segment `part` (claim_counts[part] entries) -> d_dst; owned bitmap words -> d_dst;
 * words [word_begin, word_begin + nwords) of the replicated bitmap <- d_src.  Stream-ordered. */
LMATCH_API int lmatch_part_get_claims(const lmatch_graph* g, int32_t part, uint64_t* d_dst,
                                      void* stream);
LMATCH_API int lmatch_part_get_bits(const lmatch_graph* g, uint32_t* d_dst, void* stream);
LMATCH_API int lmatch_part_set_bits(lmatch_graph* g, const uint32_t* d_src, int64_t word_begin,
                                    int64_t nwords, void* stream);
/* Rounds begun so far in this run; (timing=1) device ms of the last round-1 sweep. */
LMATCH_API int lmatch_part_info(const lmatch_graph* g, int64_t* rounds, double* sweep_ms);
/* Compaction; *nF_local = this part's next frontier size.  Synchronises `stream`. */
LMATCH_API int lmatch_part_compact(lmatch_graph* g, void* stream, int64_t* nF_local);
/* Pointer phase on the frontier + claims (counts as in lmatch_part_begin).  Synchronises. */
LMATCH_API int lmatch_part_point(lmatch_graph* g, void* stream, int64_t* claim_counts);
/* d_mate_local: DEVICE int32[n_local] (global ids, -1 unmatched); *w_local = sum of w over owned
 * u with mate[u] > u (fp64); *matched_local = owned matched vertices.  Synchronises. */
LMATCH_API int lmatch_part_finish(lmatch_graph* g, int32_t* d_mate_local, void* stream,
                                  double* w_local, int64_t* matched_local);

/* ---------------------------------------------------------------------------------------------
 * Peer-memory exchange (the same partitioned round; the library's kernels move the data).
 * Replaces the caller-side all-to-all / allgather / allreduce above with stores into the peers'
 * memory (NVLink 5 / NVSwitch between GPUs; CUDA IPC across processes, plain pointers within one
 * process), fused into the kernels that produce the data:
 *   - the claims kernels store each claim (v | u << 32) straight into the owner's inbox segment
 *     for this part and count it there with a system-scope atomic (replaces the pointer
 *     exchange, Alg. 2 L7);
 *   - the match step pushes every owned bitmap word that changed into every peer's replica
 *     (replaces nccl_AllReduce(mate), Alg. 2 L9);
 *   - the compaction pushes this part's frontier size into every peer's slot (termination,
 *     P:159).
 * Setup, on every part: lmatch_p2p_enable(g, part index) (allocates the exchange window: inbox
 * nparts x max-part-size uint64, counts, slots), then for every other part either
 * lmatch_p2p_attach_local(g, peer, peer_handle) (same process; peer access is enabled when the
 * handles live on different devices) or lmatch_p2p_export on the peer + lmatch_p2p_attach(g, peer,
 * handles) here (another process: 128 bytes = two cudaIpcMemHandle_t, passed by the caller).
 * A round (the caller puts a barrier -- every part's stream drained, e.g. synchronise + a host
 * barrier -- at each "|"):
 *   lmatch_p2p_begin / lmatch_p2p_point | [lmatch_p2p_frontier_total of the previous compaction
 *   -> stop when 0] lmatch_p2p_match | lmatch_p2p_compact, then the next lmatch_p2p_point
 * (the frontier sizes are pushed by the compaction, so they are visible after the next barrier;
 * a pointer phase on an empty frontier launches nothing and sends no claims).
 * and lmatch_part_finish at the end.  Calls are stream-ordered and do not synchronise, except
 * lmatch_p2p_frontier_total (and lmatch_p2p_compact when asked for the local size): one host
 * read per round.  Result: as above,
 * bit-identical to the single-GPU run.  Calls on a handle without enable / with a peer missing
 * return ESTATE; lmatch_part_begin/point/apply on an enabled handle return ESTATE.
 * ------------------------------------------------------------------------------------------- */
LMATCH_API int lmatch_p2p_enable(lmatch_graph* g, int32_t part_index);
LMATCH_API int lmatch_p2p_attach_local(lmatch_graph* g, int32_t peer, lmatch_graph* peer_handle);
/* handles: host buffer of 128 bytes (written by export, read by attach). */
LMATCH_API int lmatch_p2p_export(const lmatch_graph* g, void* handles);
LMATCH_API int lmatch_p2p_attach(lmatch_graph* g, int32_t peer, const void* handles);
LMATCH_API int lmatch_p2p_begin(lmatch_graph* g, void* stream);
LMATCH_API int lmatch_p2p_point(lmatch_graph* g, void* stream);
LMATCH_API int lmatch_p2p_match(lmatch_graph* g, void* stream);
/* Compaction, then this part's frontier size pushed into every peer's slot.  nF_local NULL:
 * stream-ordered, no synchronisation (peer-memory rounds size their launches from the
 * device-resident counts, so nothing is read back); non-NULL: synchronises `stream` and returns
 * this part's next frontier size. */
LMATCH_API int lmatch_p2p_compact(lmatch_graph* g, void* stream, int64_t* nF_local);
/* *nF_total = the sum of every part's pushed frontier size (synchronises `stream`). */
LMATCH_API int lmatch_p2p_frontier_total(lmatch_graph* g, void* stream, int64_t* nF_total);
/* Synchronise `stream` (NULL = the handle's stream): the caller's half of a barrier. */
LMATCH_API int lmatch_p2p_sync(lmatch_graph* g, void* stream);

/* ---------------------------------------------------------------------------------------------
 * Library-owned multi-GPU driver (SURVEY 8(b) lmatch_create_dist, 8(e)).  One process (or one
 * thread) per GPU calls these; the library partitions, sets up the peer-memory exchange above by
 * itself and runs the whole round loop -- Alg. 2's per-device loop with the exchange
 * redesigned (claims into the owners' inboxes instead of nccl_AllReduce(pointers); changed
 * bitmap words instead of nccl_AllReduce(mate); frontier sizes for termination).
 * The phases of a round are separated by DEVICE-side barriers over the exchange windows
 * (system-scope release/acquire flags stored into the peers' memory), so no host barrier is
 * involved; each rank reads one value set per round (the P frontier sizes).
 * ------------------------------------------------------------------------------------------- */

/* Edge-balanced 1-D partition of a CSR ("binary search on the prefix sums"): bounds[0] = 0,
 * bounds[nparts] = n, and for 0 < p < nparts bounds[p] = the first row whose start offset reaches
 * floor(m p / nparts), rounded up to a multiple of `align` (0 = 32: each matched-bitmap word then
 * has one owner) and kept non-decreasing.  csr_offsets: HOST int64[n+1]; bounds: HOST
 * int64[nparts+1], caller-allocated.  Host-only (no CUDA call).  EINVAL on NULL / offsets[0] != 0
 * / nparts < 1; ERANGE on n out of [0, 2^31). */
LMATCH_API int lmatch_partition(const int64_t* csr_offsets, int64_t n, int32_t nparts, int32_t align,
                                int64_t* bounds);

/* Rendezvous name shared by the ranks of one lmatch_create_dist group (like an ncclUniqueId):
 * one rank creates it with lmatch_dist_id_new and sends the 64 bytes to the others (e.g. a
 * torch.distributed broadcast).  The ranks meet in a POSIX shared-memory segment named after it
 * (one node), which the last rank to attach removes.  Host-only. */
typedef struct lmatch_dist_id {
  char bytes[64];
} lmatch_dist_id;
LMATCH_API int lmatch_dist_id_new(lmatch_dist_id* id);

/* Rank `rank` of `world` creates its part: rows [v_begin, v_begin + n_local) of a graph with
 * n_global vertices, given as a HOST local CSR whose col_idx are GLOBAL ids (cut edges appear in
 * both owners' rows); part_bounds: HOST int64[world+1] as lmatch_partition returns (every
 * rank passes the same bounds; v_begin must be part_bounds[rank]).  Blocks until all `world`
 * ranks of `id` have joined (ENCCL after 60 s; environment LMATCH_DIST_TIMEOUT_S overrides the
 * wait here and at the device barriers), then opens every peer's exchange window: plain
 * device pointers for ranks in the same process (peer access enabled across devices), CUDA IPC
 * for other processes.  opts: as for lmatch_create_ex (hbm_budget_bytes / batches stream this
 * rank's rows: the paper's per-device batches N_i), except validate_level 2 and
 * algorithm != 0 (EINVAL).  The returned handle is used with lmatch_run_dist* and
 * lmatch_destroy (and lmatch_info / lmatch_reload); it is a partition handle, so the
 * lmatch_part_* / lmatch_p2p_* calls return ESTATE or act on the same state -- do not mix. */
LMATCH_API int lmatch_create_dist(const int64_t* csr_offsets, const int32_t* col_idx,
                                  const float* weights, int64_t n_local, int64_t m_local,
                                  int64_t v_begin, int64_t n_global, int32_t rank, int32_t world,
                                  const int64_t* part_bounds, const lmatch_dist_id* id,
                                  const lmatch_opts* opts, lmatch_graph** out);
/* Same with the three local arrays on the DEVICE (ordered on `stream`). */
LMATCH_API int lmatch_create_dist_device(const int64_t* d_offsets, const int32_t* d_col,
                                         const float* d_weights, int64_t n_local, int64_t m_local,
                                         int64_t v_begin, int64_t n_global, int32_t rank,
                                         int32_t world, const int64_t* part_bounds,
                                         const lmatch_dist_id* id, const lmatch_opts* opts,
                                         void* stream, lmatch_graph** out);
/* Every rank calls it (collective): the whole matching.  d_mate_local: DEVICE int32[n_local], the
 * owned slice of mate[] (global ids, -1 = unmatched).  stats (optional): rounds = pointing phases,
 * cardinality / matched_vertices / weight = the WHOLE graph's (every rank's share summed in rank
 * order, so every rank gets the same fp64 w(M)), entries_swept / kernel_launches / ms_* = this
 * rank's.  The result is bit-identical to the single-GPU run for every partition (Lemma III.1,
 * P:167-175).  Synchronises `stream` (NULL = the handle's stream).  ENCCL if a peer does not reach
 * a device barrier within 60 s; EROUNDS as for lmatch_run. */
LMATCH_API int lmatch_run_dist_device(lmatch_graph* g, int32_t* d_mate_local, void* stream,
                                      lmatch_stats* stats);
/* Same with a HOST int32[n_local] output. */
LMATCH_API int lmatch_run_dist(lmatch_graph* g, int32_t* mate_local, lmatch_stats* stats);

/* Release everything the handle owns.  NULL-safe. */
LMATCH_API void lmatch_destroy(lmatch_graph* g);

/* Static string for a status code. */
LMATCH_API const char* lmatch_strerror(int status);

/* Thread-local detail of the last error on this thread ("" if none). */
LMATCH_API const char* lmatch_last_error(void);

#ifdef __cplusplus
}
#endif

#endif /* LMATCH_H_ */
