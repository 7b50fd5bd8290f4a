// oracle.cpp -- TEST INFRASTRUCTURE ONLY.
//
// A plain, slow, obviously-correct CPU statement of what the GPU hot path computes.  Only
// tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may load
// this library.  It shares no code, header, helper or constant with the CUDA path
// (paper_conf_sc_mandulakgfhs24_b200/csrc); neither includes the other.
//
// Citations: "P:N" = /root/reference/PAPER.md line N (section / algorithm in brackets).
//
// What is computed (DESIGN.md "Readings" R1-R4):
//  * The result of the method is the maximal locally dominant matching of G
//    [Def. II.1; Lemma II.1; Alg. 1, P:60-72] under the strict edge order
//        e = {u,v} > f = {x,y}  iff  (w(e), max(u,v), min(u,v)) > (w(f), max(x,y), min(x,y))
//    lexicographically.  At a vertex u this is "heavier weight wins, then larger neighbour id"
//    (BASELINE.json north_star: "a fixed total order on edges (weight, then vertex ids)").
//    Under a strict order that matching is unique and equals the sequential greedy matching
//    that "sorts globally" [P:52] -- DESIGN.md R1 gives the proof.  oracle_greedy() is that
//    definition written out: sort all edges by the order, scan, keep an edge iff both ends free.
//  * oracle_ld_seq() is Algorithm 1 (LD-SEQ) literally: every round every vertex of the
//    remaining graph points to its heaviest remaining neighbour [Alg. 1 L3-4, P:66-67],
//    mutual pairs are matched [L5-7, P:68-70] and all edges incident on matched vertices are
//    removed [L8, P:71 garbled; caption P:56 "remove all edges incident on M"].  It stops when a
//    round adds no edge [P:159].
//  * oracle_ld_frontier() is the same iteration, but a vertex recomputes its pointer only when
//    its current target was matched (the available set only shrinks; R3).  It reports
//    the number of pointing phases the frontier-driven GPU path executes.
//  * oracle_certificate() checks, in O(m), that a given mate[] is exactly that unique matching:
//    mate is a symmetric matching of edges and every non-matching edge has a heavier
//    (in the strict order) matching edge at one of its endpoints (R1(iii)).
//  * oracle_validate() re-implements the input contract of include/lmatch.h.
//
// Weights are fp32 as given; comparisons are exact float comparisons (w > 0 finite).  The
// matched weight w(M) [P:15, P:42] is summed in fp64 with Neumaier compensation.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <vector>
#include <omp.h>

namespace {

double now_s() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

// "e heavier than f" in the strict order (weight, then larger max endpoint, then larger min).
struct Edge {
  float w;
  int32_t hi, lo;
};
inline bool heavier(const Edge& a, const Edge& b) {
  if (a.w != b.w) return a.w > b.w;
  if (a.hi != b.hi) return a.hi > b.hi;
  return a.lo > b.lo;
}

// At vertex u: candidate (weight wa, neighbour a) beats (wb, b) -- the restriction of the
// global order to edges sharing u (R1(i)).
inline bool beats_at(float wa, int64_t a, float wb, int64_t b) {
  if (wa != wb) return wa > wb;
  return a > b;
}

void neumaier_add(double& sum, double& comp, double x) {
  double t = sum + x;
  if (std::fabs(sum) >= std::fabs(x)) comp += (sum - t) + x;
  else comp += (x - t) + sum;
  sum = t;
}

}  // namespace

extern "C" {

// Input contract (include/lmatch.h): 0 = OK, -1 = EINVAL, -2 = ERANGE.  msg receives a reason.
int oracle_validate(const int64_t* offsets, const int32_t* col, const float* w, int64_t n,
                    int64_t m, int level, char* msg, int msglen) {
  auto fail = [&](int code, const char* what, long long a, long long b) {
    if (msg && msglen > 0) snprintf(msg, (size_t)msglen, "%s (%lld, %lld)", what, a, b);
    return code;
  };
  if (n < 0 || m < 0) return fail(-1, "negative size", n, m);
  if (n >= (int64_t)1 << 31) return fail(-2, "n >= 2^31", n, 0);
  if (n == 0) return m == 0 ? 0 : fail(-1, "n == 0 with m > 0", n, m);
  if (offsets[0] != 0) return fail(-1, "offsets[0] != 0", offsets[0], 0);
  for (int64_t u = 0; u < n; ++u)
    if (offsets[u + 1] < offsets[u]) return fail(-1, "offsets decrease at", u, offsets[u + 1]);
  if (offsets[n] != m) return fail(-1, "offsets[n] != m", offsets[n], m);
  for (int64_t j = 0; j < m; ++j) {
    if (col[j] < 0 || col[j] >= n) return fail(-1, "col out of range at", j, col[j]);
    float x = w[j];
    uint32_t bits;
    std::memcpy(&bits, &x, 4);
    if (!(x > 0.0f) || std::isinf(x) || (bits >> 31)) return fail(-1, "weight not finite > 0 at", j, bits);
  }
  if (level >= 2) {
    // symmetric: the multiset {(u, v, w)} equals the multiset {(v, u, w)}; and a repeated (u, v)
    // must repeat its weight.
    struct T { int64_t a, b; uint32_t wb; };
    std::vector<T> fwd, rev;
    fwd.reserve((size_t)m); rev.reserve((size_t)m);
    for (int64_t u = 0; u < n; ++u)
      for (int64_t j = offsets[u]; j < offsets[u + 1]; ++j) {
        uint32_t wb; std::memcpy(&wb, &w[j], 4);
        fwd.push_back({u, col[j], wb});
        rev.push_back({col[j], u, wb});
      }
    auto lt = [](const T& x, const T& y) {
      if (x.a != y.a) return x.a < y.a;
      if (x.b != y.b) return x.b < y.b;
      return x.wb < y.wb;
    };
    std::sort(fwd.begin(), fwd.end(), lt);
    std::sort(rev.begin(), rev.end(), lt);
    for (size_t i = 0; i < fwd.size(); ++i)
      if (fwd[i].a != rev[i].a || fwd[i].b != rev[i].b || fwd[i].wb != rev[i].wb)
        return fail(-1, "graph not symmetric near", fwd[i].a, fwd[i].b);
    for (size_t i = 1; i < fwd.size(); ++i)
      if (fwd[i].a == fwd[i - 1].a && fwd[i].b == fwd[i - 1].b && fwd[i].wb != fwd[i - 1].wb)
        return fail(-1, "duplicate edge with unequal weights", fwd[i].a, fwd[i].b);
  }
  return 0;
}

// Sequential greedy matching = the unique maximal locally dominant matching (R1).
// out_stats[0] = |M|, [1] = w(M) (fp64 Neumaier), [2] = sort seconds, [3] = scan seconds,
// [4] = number of undirected edges sorted.
int oracle_greedy(const int64_t* offsets, const int32_t* col, const float* w, int64_t n,
                  int32_t* mate, double* out_stats) {
  double t0 = now_s();
  std::vector<Edge> E;
  E.reserve((size_t)(offsets[n] / 2 + 1));
  for (int64_t u = 0; u < n; ++u)
    for (int64_t j = offsets[u]; j < offsets[u + 1]; ++j)
      if (u < col[j]) E.push_back({w[j], col[j], (int32_t)u});  // one copy of each edge; no loops
  std::sort(E.begin(), E.end(), heavier);
  double t1 = now_s();
  for (int64_t v = 0; v < n; ++v) mate[v] = -1;
  int64_t card = 0;
  double sum = 0.0, comp = 0.0;
  for (const Edge& e : E) {
    if (mate[e.hi] == -1 && mate[e.lo] == -1) {
      mate[e.hi] = e.lo;
      mate[e.lo] = e.hi;
      ++card;
      neumaier_add(sum, comp, (double)e.w);
    }
  }
  double t2 = now_s();
  if (out_stats) {
    out_stats[0] = (double)card;
    out_stats[1] = sum + comp;
    out_stats[2] = t1 - t0;
    out_stats[3] = t2 - t1;
    out_stats[4] = (double)E.size();
  }
  return 0;
}

// Algorithm 1 (LD-SEQ), literally: full pointing phase over all remaining vertices each round.
// Returns the number of rounds executed, counting the final round that adds nothing [P:159].
int64_t oracle_ld_seq(const int64_t* offsets, const int32_t* col, const float* w, int64_t n,
                      int32_t* mate) {
  std::vector<int64_t> ptr((size_t)n, -1);
  for (int64_t v = 0; v < n; ++v) mate[v] = -1;
  int64_t rounds = 0;
  for (;;) {
    ++rounds;
    // Phase 1: pointing [Alg. 1 L3-4]: heaviest neighbour in the remaining graph.
    for (int64_t v = 0; v < n; ++v) {
      ptr[v] = -1;
      if (mate[v] != -1) continue;
      float bw = 0.0f;
      for (int64_t j = offsets[v]; j < offsets[v + 1]; ++j) {
        int64_t u = col[j];
        if (u == v || mate[u] != -1) continue;
        if (ptr[v] == -1 || beats_at(w[j], u, bw, ptr[v])) { ptr[v] = u; bw = w[j]; }
      }
    }
    // Phase 2: matching [Alg. 1 L5-8]: mutual pointers are locally dominant edges.
    int64_t added = 0;
    for (int64_t v = 0; v < n; ++v) {
      int64_t u = ptr[v];
      if (u > v && ptr[u] == v) { mate[v] = (int32_t)u; mate[u] = (int32_t)v; ++added; }
    }
    if (added == 0) break;
  }
  return rounds;
}

// Frontier-driven Alg. 1: identical matching; a vertex re-points only when its target was
// matched.  Returns the number of pointing phases executed with a non-empty frontier (the GPU
// path's lmatch_stats.rounds).  Also writes per-round frontier sizes into fsize (if non-null,
// capacity fcap).
int64_t oracle_ld_frontier(const int64_t* offsets, const int32_t* col, const float* w, int64_t n,
                           int32_t* mate, int64_t* fsize, int64_t fcap) {
  std::vector<int64_t> ptr((size_t)n, -1);
  std::vector<char> need((size_t)n, 0);
  for (int64_t v = 0; v < n; ++v) { mate[v] = -1; need[v] = offsets[v + 1] > offsets[v]; }
  int64_t phases = 0;
  for (;;) {
    int64_t fs = 0;
    for (int64_t v = 0; v < n; ++v) fs += need[v];
    if (fs == 0) break;
    if (fsize && phases < fcap) fsize[phases] = fs;
    ++phases;
    for (int64_t v = 0; v < n; ++v) {
      if (!need[v]) continue;
      ptr[v] = -1;
      float bw = 0.0f;
      for (int64_t j = offsets[v]; j < offsets[v + 1]; ++j) {
        int64_t u = col[j];
        if (u == v || mate[u] != -1) continue;
        if (ptr[v] == -1 || beats_at(w[j], u, bw, ptr[v])) { ptr[v] = u; bw = w[j]; }
      }
    }
    std::vector<int64_t> newly;
    for (int64_t v = 0; v < n; ++v) {
      if (!need[v]) continue;
      int64_t u = ptr[v];
      if (u >= 0 && mate[v] == -1 && ptr[u] == v) {
        mate[v] = (int32_t)u; mate[u] = (int32_t)v;
        newly.push_back(v); newly.push_back(u);
      }
    }
    for (int64_t v = 0; v < n; ++v) {
      need[v] = 0;
      if (mate[v] != -1 || ptr[v] < 0) continue;
      if (mate[ptr[v]] != -1) need[v] = 1;  // target taken: re-point next phase
    }
  }
  return phases;
}

// Certificate C(M): returns 0 iff mate[] is the unique maximal locally dominant matching.
// Nonzero codes: 1 = mate out of range / self, 2 = not symmetric, 3 = matched pair is not an
// edge, 4 = some edge has no heavier matched edge at either endpoint (bad[0..1] = that edge).
int oracle_certificate(const int64_t* offsets, const int32_t* col, const float* w, int64_t n,
                       const int32_t* mate, int64_t* bad) {
  for (int64_t u = 0; u < n; ++u) {
    int64_t v = mate[u];
    if (v == -1) continue;
    if (v < 0 || v >= n || v == u) { if (bad) { bad[0] = u; bad[1] = v; } return 1; }
    if (mate[v] != u) { if (bad) { bad[0] = u; bad[1] = v; } return 2; }
  }
  std::vector<float> mw((size_t)n, 0.0f);
  std::vector<char> found((size_t)n, 0);
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t u = 0; u < n; ++u) {
    if (mate[u] < 0) continue;
    for (int64_t j = offsets[u]; j < offsets[u + 1]; ++j)
      if (col[j] == mate[u]) { mw[u] = w[j]; found[u] = 1; }
  }
  for (int64_t u = 0; u < n; ++u)
    if (mate[u] >= 0 && !found[u]) { if (bad) { bad[0] = u; bad[1] = mate[u]; } return 3; }
  int code = 0;
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t u = 0; u < n; ++u) {
    for (int64_t j = offsets[u]; j < offsets[u + 1]; ++j) {
      int64_t v = col[j];
      if (v == u || mate[u] == v) continue;
      bool ok = (mate[u] >= 0 && beats_at(mw[u], mate[u], w[j], v)) ||
                (mate[v] >= 0 && beats_at(mw[v], mate[v], w[j], u));
      if (!ok) {
#pragma omp critical
        {
          if (code == 0) { code = 4; if (bad) { bad[0] = u; bad[1] = v; } }
        }
      }
    }
  }
  return code;
}

// w(M) for an arbitrary mate[] (fp64, Neumaier, over u < mate[u]); -1 if a pair is not an edge.
int oracle_weight(const int64_t* offsets, const int32_t* col, const float* w, int64_t n,
                  const int32_t* mate, double* out) {
  double sum = 0.0, comp = 0.0;
  for (int64_t u = 0; u < n; ++u) {
    int64_t v = mate[u];
    if (v <= u) continue;
    bool found = false;
    for (int64_t j = offsets[u]; j < offsets[u + 1]; ++j)
      if (col[j] == v) { neumaier_add(sum, comp, (double)w[j]); found = true; break; }
    if (!found) return -1;
  }
  *out = sum + comp;
  return 0;
}

int oracle_threads(int t) { if (t > 0) omp_set_num_threads(t); return omp_get_max_threads(); }

}  // extern "C"
