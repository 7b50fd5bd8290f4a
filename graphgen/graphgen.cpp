// graphgen.cpp -- seeded synthetic graph generators shared by the oracle tests
// and the CUDA path's tests/bench.
//
// This module holds NONE of the matching method's arithmetic: it only builds
// symmetric CSR graphs (offsets int64[n+1], col int32[m], w float32[m]) with
// the structure of the paper's workloads ("uniform distribution
// ... three decimal points from [0,1]"; Table I classes):
//   * Erdos-Renyi (GAP-urand-like, uniform degree),
//   * R-MAT / Graph500 Kronecker (GAP-kron-like power law),
//   * 2-D mesh and a road-like thinned mesh (kmer-like low degree).
// Every random choice is a counter-based hash of (seed, index), so the output
// is bit-identical for any OpenMP thread count.  The recipe is in DESIGN.md
// ("Input recipe").
#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <vector>
#include <omp.h>

#include "gg_common.h"

namespace {

inline uint64_t mix64(uint64_t x) { return gg_mix64(x); }
inline uint64_t hash2(uint64_t seed, uint64_t a, uint64_t b) { return gg_hash2(seed, a, b); }

// Builds a symmetric CSR from an edge generator gen(i, &u, &v) -> bool (false = skip),
// i in [0, M).  Self-loops are dropped, rows are sorted ascending and deduplicated.
// col must have capacity >= 2*M.  Returns m (directed entries).
template <class Gen>
int64_t build_csr(int64_t n, int64_t M, Gen gen, int64_t* offsets, int32_t* col) {
  std::vector<std::atomic<int64_t>> cnt(n);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) cnt[i].store(0, std::memory_order_relaxed);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < M; ++i) {
    int64_t u, v;
    if (!gen(i, &u, &v) || u == v) continue;
    cnt[u].fetch_add(1, std::memory_order_relaxed);
    cnt[v].fetch_add(1, std::memory_order_relaxed);
  }
  offsets[0] = 0;
  for (int64_t i = 0; i < n; ++i) offsets[i + 1] = offsets[i] + cnt[i].load(std::memory_order_relaxed);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) cnt[i].store(offsets[i], std::memory_order_relaxed);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < M; ++i) {
    int64_t u, v;
    if (!gen(i, &u, &v) || u == v) continue;
    col[cnt[u].fetch_add(1, std::memory_order_relaxed)] = (int32_t)v;
    col[cnt[v].fetch_add(1, std::memory_order_relaxed)] = (int32_t)u;
  }
  // per-row sort + unique (deterministic regardless of scatter order)
  std::vector<int64_t> ndeg(n);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t r = 0; r < n; ++r) {
    int32_t* b = col + offsets[r];
    int32_t* e = col + offsets[r + 1];
    std::sort(b, e);
    ndeg[r] = std::unique(b, e) - b;
  }
  // sequential in-place compaction (destinations never pass their sources)
  int64_t pos = 0;
  for (int64_t r = 0; r < n; ++r) {
    int64_t s = offsets[r];
    int64_t d = ndeg[r];
    if (pos != s && d) std::memmove(col + pos, col + s, (size_t)d * sizeof(int32_t));
    offsets[r] = pos;
    pos += d;
  }
  offsets[n] = pos;
  return pos;
}

}  // namespace

extern "C" {

uint64_t gg_hash(uint64_t seed, uint64_t a, uint64_t b) { return hash2(seed, a, b); }

int gg_set_threads(int t) { if (t > 0) omp_set_num_threads(t); return omp_get_max_threads(); }

// Erdos-Renyi G(n, M): M = n*avg_degree/2 iid uniform pairs, loops dropped, deduplicated.
int64_t gg_er_csr(int64_t n, double avg_degree, uint64_t seed, int64_t* offsets, int32_t* col,
                  int64_t cap) {
  int64_t M = (int64_t)std::llround((double)n * avg_degree / 2.0);
  if (2 * M > cap) return -1;
  const GGEr er = gg_make_er(n, seed);
  auto gen = [=](int64_t i, int64_t* u, int64_t* v) {
    er.edge(i, u, v);
    return true;
  };
  return build_csr(n, M, gen, offsets, col);
}

int64_t gg_er_max_entries(int64_t n, double avg_degree) {
  return 2 * (int64_t)std::llround((double)n * avg_degree / 2.0);
}

// R-MAT / Graph500 Kronecker: M = edgefactor * 2^scale edges; each level picks a quadrant
// with probabilities (a, b, c, 1-a-b-c) using 16-bit uniforms (4 levels per 64-bit hash);
// vertex ids are relabelled by a seeded bijection so hubs are not clustered at low ids.
int64_t gg_rmat_csr(int scale, int64_t edgefactor, uint64_t seed, double a, double b, double c,
                    int64_t* offsets, int32_t* col, int64_t cap) {
  if (scale < 1 || scale > 31) return -2;
  int64_t n = (int64_t)1 << scale;
  int64_t M = edgefactor * n;
  if (2 * M > cap) return -1;
  const GGRmat rm = gg_make_rmat(scale, seed, a, b, c);
  auto gen = [=](int64_t i, int64_t* u, int64_t* v) {
    rm.edge(i, u, v);
    return true;
  };
  return build_csr(n, M, gen, offsets, col);
}

// side x side open 4-neighbour grid (vertex id = y*side + x).  keep_permille < 1000 keeps each
// grid edge {a,b} iff hash(min,max) mod 1000 < keep_permille ("road-like" thinning).
// Rows come out sorted ascending (up, left, right, down).  Returns m.
int64_t gg_mesh_csr(int64_t side, int keep_permille, uint64_t seed, int64_t* offsets, int32_t* col,
                    int64_t cap) {
  int64_t n = side * side;
  if (4 * n > cap) return -1;
  uint64_t s = mix64(seed ^ 0x3E5u);
  auto keep = [=](int64_t a, int64_t b) -> bool {
    if (keep_permille >= 1000) return true;
    int64_t lo = a < b ? a : b, hi = a < b ? b : a;
    return (int)(hash2(s, (uint64_t)lo, (uint64_t)hi) % 1000u) < keep_permille;
  };
  auto nbrs = [=](int64_t id, int64_t out[4]) {
    int64_t x = id % side, y = id / side;
    int k = 0;
    if (y > 0 && keep(id, id - side)) out[k++] = id - side;
    if (x > 0 && keep(id, id - 1)) out[k++] = id - 1;
    if (x + 1 < side && keep(id, id + 1)) out[k++] = id + 1;
    if (y + 1 < side && keep(id, id + side)) out[k++] = id + side;
    return k;
  };
  std::vector<int64_t> deg(n);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) { int64_t t[4]; deg[i] = nbrs(i, t); }
  offsets[0] = 0;
  for (int64_t i = 0; i < n; ++i) offsets[i + 1] = offsets[i] + deg[i];
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    int64_t t[4];
    int k = nbrs(i, t);
    for (int j = 0; j < k; ++j) col[offsets[i] + j] = (int32_t)t[j];
  }
  return offsets[n];
}

// Edge weights, symmetric by construction (a function of {min(u,v), max(u,v)} only).
//  mode 0: uniform fp32 (1 + H mod 2^24) * 2^-24 in (0, 1]     (default)
//  mode 1: "paper" weights: 3 decimals in {0.001 .. 1.000}    (many ties)
//  mode 2: gradient mesh weights (needs side): ((x+y) + 1e-3*U) / (2*side), U in [0,1)
//          of the larger endpoint; clamped to >= 2^-24   (many-round stress)
//  mode 3: all weights 1.0 (pure tie-break by vertex id)
int gg_weights(const int64_t* offsets, const int32_t* col, int64_t n, uint64_t seed, int mode,
               int64_t side, float* w) {
  const uint64_t ws = gg_mix64(seed ^ 0x77u);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; ++u)
    for (int64_t j = offsets[u]; j < offsets[u + 1]; ++j) w[j] = gg_weight(ws, mode, u, col[j], side);
  return 0;
}

}  // extern "C"
