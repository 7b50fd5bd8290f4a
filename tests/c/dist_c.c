/* A plain C caller of the library-owned multi-GPU driver (include/lmatch.h): P ranks of one
 * lmatch_create_dist group match one graph end to end -- no Python, no torch, no caller-side
 * exchange or barrier.  Used by tests/test_gpu_dist.py.
 *
 *   dist_c <fork|thread> <P> <out_prefix> [n]
 *
 * The graph (n vertices, default 20000) is a ring plus hashed chords with hashed fp32 weights in
 * (0,1]; it is written to <out_prefix>.offsets/.col/.w (raw little-endian arrays) so the test can
 * run the oracle on it.  The partition comes from lmatch_partition and the rendezvous id from
 * lmatch_dist_id_new (both host-only, so the parent touches no CUDA before fork()).  Each rank
 * builds its local CSR (global column ids), calls lmatch_create_dist + lmatch_run_dist twice and
 * writes its owned mate[] slice into <out_prefix>.mate at offset 4 * v_begin.  "fork" runs the
 * ranks as child processes (CUDA IPC between them), "thread" as threads of one process (plain
 * device pointers).  Afterwards the parent runs the single-graph path (lmatch_create + lmatch_run)
 * and checks that both runs of every rank and the single-graph mate[] are identical.
 * Prints "weight=<w(M)> cardinality=<|M|> rounds=<r>" and exits 0 on success. */
#define _GNU_SOURCE
#include <fcntl.h>
#include <pthread.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/wait.h>
#include <unistd.h>

#include "lmatch.h"

static int64_t N = 20000, M = 0;
static int64_t* offs;
static int32_t* col;
static float* wt;
static int P;
static int64_t* bounds;
static lmatch_dist_id did;
static const char* prefix;

static uint64_t mix(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
static float weight_of(int64_t a, int64_t b) {
  const int64_t lo = a < b ? a : b, hi = a < b ? b : a;
  return (float)(1 + (mix((uint64_t)lo * 1000003ull + (uint64_t)hi) % 1000)) / 1000.0f; /* ties */
}

/* ring u -- u+1, plus chords u -- (u * 7919 + 13) mod N for u % 3 == 0 (duplicates and loops
 * dropped); each row sorted by neighbour */
static int cmp_i32(const void* a, const void* b) {
  const int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
  return (x > y) - (x < y);
}
static void build_graph(void) {
  int64_t* deg = calloc((size_t)N + 1, 8);
  int32_t(*nb)[8] = calloc((size_t)N, sizeof *nb);
  for (int64_t u = 0; u < N; ++u) {
    const int64_t v = (u + 1) % N;
    nb[u][deg[u]++] = (int32_t)v;
    nb[v][deg[v]++] = (int32_t)u;
  }
  for (int64_t u = 0; u < N; u += 3) {
    const int64_t v = (u * 7919 + 13) % N;
    if (v == u) continue;
    int dup = 0;
    for (int k = 0; k < deg[u]; ++k) dup |= nb[u][k] == v;
    if (dup || deg[u] >= 8 || deg[v] >= 8) continue;
    nb[u][deg[u]++] = (int32_t)v;
    nb[v][deg[v]++] = (int32_t)u;
  }
  offs = malloc(((size_t)N + 1) * 8);
  offs[0] = 0;
  for (int64_t u = 0; u < N; ++u) offs[u + 1] = offs[u] + deg[u];
  M = offs[N];
  col = malloc((size_t)M * 4);
  wt = malloc((size_t)M * 4);
  for (int64_t u = 0; u < N; ++u) {
    qsort(nb[u], (size_t)deg[u], 4, cmp_i32);
    for (int k = 0; k < deg[u]; ++k) {
      col[offs[u] + k] = nb[u][k];
      wt[offs[u] + k] = weight_of(u, nb[u][k]);
    }
  }
  free(deg);
  free(nb);
}

static void write_file(const char* suffix, const void* p, size_t bytes) {
  char path[512];
  snprintf(path, sizeof path, "%s.%s", prefix, suffix);
  FILE* f = fopen(path, "wb");
  if (!f || fwrite(p, 1, bytes, f) != bytes) { perror(path); exit(2); }
  fclose(f);
}

struct rank_out { int rc; double w; int64_t card, rounds; };

static struct rank_out rank_main(int r) {
  struct rank_out o = {0, 0.0, 0, 0};
  const int64_t v0 = bounds[r], v1 = bounds[r + 1], nl = v1 - v0;
  const int64_t s0 = offs[v0], ml = offs[v1] - s0;
  int64_t* lo = malloc(((size_t)nl + 1) * 8);
  for (int64_t i = 0; i <= nl; ++i) lo[i] = offs[v0 + i] - s0;
  lmatch_graph* g = NULL;
  o.rc = lmatch_create_dist(lo, col + s0, wt + s0, nl, ml, v0, N, r, P, bounds, &did, NULL, &g);
  if (o.rc) { fprintf(stderr, "rank %d create: %s\n", r, lmatch_last_error()); free(lo); return o; }
  int32_t* mate = malloc(((size_t)nl + 1) * 4);
  int32_t* mate2 = malloc(((size_t)nl + 1) * 4);
  lmatch_stats st, st2;
  o.rc = lmatch_run_dist(g, mate, &st);
  if (!o.rc) o.rc = lmatch_run_dist(g, mate2, &st2);  /* a second run on the same handles */
  if (o.rc) fprintf(stderr, "rank %d run: %s\n", r, lmatch_last_error());
  if (!o.rc && (memcmp(mate, mate2, (size_t)nl * 4) || st.weight != st2.weight || st.rounds != st2.rounds)) {
    fprintf(stderr, "rank %d: second run differs\n", r);
    o.rc = 3;
  }
  if (!o.rc) {
    char path[512];
    snprintf(path, sizeof path, "%s.mate", prefix);
    const int fd = open(path, O_WRONLY);
    if (fd < 0 || pwrite(fd, mate, (size_t)nl * 4, (off_t)(v0 * 4)) != (ssize_t)(nl * 4)) o.rc = 4;
    if (fd >= 0) close(fd);
    o.w = st.weight;
    o.card = st.cardinality;
    o.rounds = st.rounds;
  }
  lmatch_destroy(g);
  free(lo);
  free(mate);
  free(mate2);
  return o;
}

static struct rank_out tout[64];
static void* thread_main(void* arg) {
  const int r = (int)(intptr_t)arg;
  tout[r] = rank_main(r);
  return NULL;
}

int main(int argc, char** argv) {
  if (argc < 4) { fprintf(stderr, "usage: dist_c <fork|thread> <P> <out_prefix> [n]\n"); return 2; }
  const int use_fork = strcmp(argv[1], "fork") == 0;
  P = atoi(argv[2]);
  prefix = argv[3];
  if (argc > 4) N = atoll(argv[4]);
  if (P < 1 || P > 64) return 2;
  build_graph();
  write_file("offsets", offs, ((size_t)N + 1) * 8);
  write_file("col", col, (size_t)M * 4);
  write_file("w", wt, (size_t)M * 4);
  int32_t* none = malloc((size_t)N * 4);
  memset(none, 0x7f, (size_t)N * 4);
  write_file("mate", none, (size_t)N * 4);
  bounds = malloc(((size_t)P + 1) * 8);
  if (lmatch_partition(offs, N, P, 32, bounds) || lmatch_dist_id_new(&did)) {
    fprintf(stderr, "partition/id: %s\n", lmatch_last_error());
    return 2;
  }
  struct rank_out res[64];
  if (use_fork) {
    int pipes[64][2];
    pid_t pid[64];
    for (int r = 0; r < P; ++r) {
      if (pipe(pipes[r])) return 2;
      pid[r] = fork();
      if (pid[r] == 0) {
        struct rank_out o = rank_main(r);
        if (write(pipes[r][1], &o, sizeof o) != (ssize_t)sizeof o) _exit(5);
        _exit(o.rc ? 1 : 0);
      }
    }
    for (int r = 0; r < P; ++r) {
      int stt = 0;
      waitpid(pid[r], &stt, 0);
      if (read(pipes[r][0], &res[r], sizeof res[r]) != (ssize_t)sizeof res[r]) res[r].rc = 6;
    }
  } else {
    pthread_t th[64];
    for (int r = 0; r < P; ++r) pthread_create(&th[r], NULL, thread_main, (void*)(intptr_t)r);
    for (int r = 0; r < P; ++r) pthread_join(th[r], NULL);
    for (int r = 0; r < P; ++r) res[r] = tout[r];
  }
  for (int r = 0; r < P; ++r) {
    if (res[r].rc) { fprintf(stderr, "rank %d failed (%d)\n", r, res[r].rc); return 1; }
    if (res[r].w != res[0].w || res[r].card != res[0].card || res[r].rounds != res[0].rounds) {
      fprintf(stderr, "rank %d reports a different global result\n", r);
      return 1;
    }
  }
  /* the single-graph path on the same graph must give the same mate[] */
  lmatch_graph* g = NULL;
  if (lmatch_create(offs, col, wt, N, M, &g)) { fprintf(stderr, "create: %s\n", lmatch_last_error()); return 1; }
  int32_t* ref = malloc((size_t)N * 4);
  lmatch_stats st;
  if (lmatch_run(g, ref, &st)) { fprintf(stderr, "run: %s\n", lmatch_last_error()); return 1; }
  lmatch_destroy(g);
  char path[512];
  snprintf(path, sizeof path, "%s.mate", prefix);
  FILE* f = fopen(path, "rb");
  int32_t* got = malloc((size_t)N * 4);
  if (!f || fread(got, 4, (size_t)N, f) != (size_t)N) return 1;
  fclose(f);
  if (memcmp(got, ref, (size_t)N * 4)) { fprintf(stderr, "partitioned mate[] differs from the single-GPU run\n"); return 1; }
  if (st.rounds != res[0].rounds || st.cardinality != res[0].card) {
    fprintf(stderr, "rounds/cardinality differ: %lld/%lld vs %lld/%lld\n", (long long)st.rounds,
            (long long)st.cardinality, (long long)res[0].rounds, (long long)res[0].card);
    return 1;
  }
  printf("weight=%.17g cardinality=%lld rounds=%lld single_weight=%.17g\n", res[0].w,
         (long long)res[0].card, (long long)res[0].rounds, st.weight);
  return 0;
}
