// gg_common.h -- counter-based generator primitives shared by graphgen.cpp (host, OpenMP) and
// graphgen_cuda.cu (device), so both produce bit-identical graphs by construction.
// Holds none of the matching method's arithmetic (input generation only).
#pragma once
#include <stdint.h>

#if defined(__CUDACC__)
#define GG_HD __host__ __device__ __forceinline__
#else
#define GG_HD inline
#endif

GG_HD uint64_t gg_mix64(uint64_t x) {  // SplitMix64 finaliser
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
GG_HD uint64_t gg_hash2(uint64_t seed, uint64_t a, uint64_t b) {
  return gg_mix64(gg_mix64(gg_mix64(seed) ^ a) ^ (b * 0xD6E8FEB86659FD93ull));
}
// Uniform integer in [0, n) from a 64-bit hash (multiply-high).
GG_HD uint64_t gg_below(uint64_t h, uint64_t n) {
#if defined(__CUDA_ARCH__)
  return __umul64hi(h, n);
#else
  return (uint64_t)(((unsigned __int128)h * n) >> 64);
#endif
}

// Bijection on [0, 2^s): random relabelling of R-MAT ids without a table.
struct GGPerm {
  int s;
  uint64_t mask, k0, k1, c1, c2;
  GG_HD void init(int s_, uint64_t seed) {
    s = s_;
    mask = (s >= 64) ? ~0ull : ((1ull << s) - 1);
    k0 = gg_mix64(seed ^ 0x1111) & mask;
    k1 = gg_mix64(seed ^ 0x2222) & mask;
    c1 = gg_mix64(seed ^ 0x3333) | 1ull;
    c2 = gg_mix64(seed ^ 0x4444) | 1ull;
  }
  GG_HD uint64_t operator()(uint64_t x) const {
    if (s <= 1) return x ^ (k0 & mask);
    int h = (s + 1) / 2;
    x = (x ^ k0) & mask;
    x = (x * c1) & mask;
    x ^= x >> h;
    x = (x + k1) & mask;
    x = (x * c2) & mask;
    x ^= x >> (s / 2 > 0 ? s / 2 : 1);
    x = (x * c1) & mask;
    x ^= x >> h;
    return x & mask;
  }
};

// R-MAT / Graph500 Kronecker edge i: per level a quadrant with probabilities (a, b, c, d) from a
// 16-bit uniform (4 levels per 64-bit hash), then the seeded relabelling.
struct GGRmat {
  int scale;
  uint32_t tA, tAB, tABC;
  uint64_t s;
  GGPerm perm;
  GG_HD void edge(int64_t i, int64_t* u, int64_t* v) const {
    uint64_t uu = 0, vv = 0, h = 0;
    for (int l = 0; l < scale; ++l) {
      if ((l & 3) == 0) h = gg_hash2(s, (uint64_t)i, (uint64_t)(l >> 2));
      uint32_t r = (uint32_t)(h & 0xFFFFu);
      h >>= 16;
      uint64_t bu, bv;
      if (r < tA) { bu = 0; bv = 0; }
      else if (r < tAB) { bu = 0; bv = 1; }
      else if (r < tABC) { bu = 1; bv = 0; }
      else { bu = 1; bv = 1; }
      uu = (uu << 1) | bu;
      vv = (vv << 1) | bv;
    }
    *u = (int64_t)perm(uu);
    *v = (int64_t)perm(vv);
  }
};

inline GGRmat gg_make_rmat(int scale, uint64_t seed, double a, double b, double c) {
  GGRmat r;
  r.scale = scale;
  // llround equivalents without <cmath> in device-visible code
  r.tA = (uint32_t)(a * 65536.0 + 0.5);
  r.tAB = (uint32_t)((a + b) * 65536.0 + 0.5);
  r.tABC = (uint32_t)((a + b + c) * 65536.0 + 0.5);
  r.s = gg_mix64(seed ^ 0x5A7u);
  r.perm.init(scale, seed ^ 0xBEEFu);
  return r;
}

// Erdos-Renyi pair i: two uniform endpoints in [0, n).
struct GGEr {
  int64_t n;
  uint64_t s;
  GG_HD void edge(int64_t i, int64_t* u, int64_t* v) const {
    *u = (int64_t)gg_below(gg_hash2(s, (uint64_t)i, 0), (uint64_t)n);
    *v = (int64_t)gg_below(gg_hash2(s, (uint64_t)i, 1), (uint64_t)n);
  }
};
inline GGEr gg_make_er(int64_t n, uint64_t seed) {
  GGEr e;
  e.n = n;
  e.s = gg_mix64(seed ^ 0xE7u);
  return e;
}

// Symmetric edge weight (a function of {min, max} only).  Modes: 0 uniform (1+H mod 2^24)*2^-24,
// 1 "paper" 3 decimals, 2 gradient mesh, 3 all ones.  ws = gg_mix64(seed ^ 0x77).
// Compile with FP contraction OFF on both sides (-ffp-contract=off / -fmad=false).
GG_HD float gg_weight(uint64_t ws, int mode, int64_t u, int64_t v, int64_t side) {
  uint64_t lo = (uint64_t)(u < v ? u : v), hi = (uint64_t)(u < v ? v : u);
  uint64_t h = gg_hash2(ws, lo, hi);
  float x;
  switch (mode) {
    case 1: x = (float)((double)(1 + h % 1000u) / 1000.0); break;
    case 2: {
      int64_t bx = (int64_t)hi % side, by = (int64_t)hi / side;
      double U = (double)(h >> 11) * (1.0 / 9007199254740992.0);
      double val = ((double)(bx + by) + 1e-3 * U) / (2.0 * (double)side);
      x = (float)val;
      if (!(x >= 5.9604644775390625e-08f)) x = 5.9604644775390625e-08f;
      break;
    }
    case 3: x = 1.0f; break;
    default: x = (float)(1 + (h & 0xFFFFFFu)) * 5.9604644775390625e-08f; break;
  }
  return x;
}
