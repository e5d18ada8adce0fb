/*
 * graphgen.c — seeded synthetic graph inputs shared by the oracle and the CUDA path.
 *
 * This module holds NONE of CuSha's arithmetic (no shards, windows, compute
 * functions or convergence logic).  It only draws edge lists and per-edge /
 * per-vertex random values with a counter-based generator, so the output is
 * independent of the thread count and identical on every machine.
 *
 * Recipes follow DESIGN.md "Input recipe":
 *   - R-MAT [Chakrabarti et al., cited PAPER.md L469] with Graph500 quadrant
 *     probabilities (a,b,c,d) = (0.57,0.19,0.19,0.05); endpoints >= V rejected,
 *     self-loops and duplicates dropped, exactly E unique edges kept.
 *   - 2D road-like mesh (RoadNet-CA shape, Table 1) with a seeded
 *     fraction of grid bonds kept, stored in both directions.
 *   - A seeded vertex relabelling pi with pi(anchor) = 0 (so vertex 0 stays the
 *     R-MAT top hub / mesh centre and is the traversal source).
 *
 * Counter-based RNG: h(seed, stream, k) = mix64(mix64(seed ^ stream*C) + k*G)
 * where mix64 is the SplitMix64 finaliser.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define GG_OK 0
#define GG_EINVAL -1
#define GG_ENOMEM -2

static inline uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static inline uint64_t ctr_hash(uint64_t seed, uint64_t stream, uint64_t k) {
  return mix64(mix64(seed ^ (stream * 0xD1B54A32D192ED03ull)) + k * 0x9E3779B97F4A7C15ull);
}

/* streams (sub-generators) */
enum { ST_RMAT = 1, ST_PERM = 2, ST_SELECT = 3, ST_MESH = 4, ST_EDGEVAL = 5, ST_VERTVAL = 6 };

uint64_t gg_hash(uint64_t seed, uint64_t stream, uint64_t k) { return ctr_hash(seed, stream, k); }

/* ---------------------------------------------------------------- sorting */
/* Parallel LSD radix sort of 64-bit keys, 16-bit digits; skips digits that are
 * constant across all keys.  tmp must hold n keys. Result ends in keys. */
static void radix_sort_u64(uint64_t* keys, uint64_t* tmp, size_t n) {
  if (n < 2) return;
  int nt = 1;
#ifdef _OPENMP
  nt = omp_get_max_threads();
#endif
  size_t* hist = (size_t*)malloc(sizeof(size_t) * (size_t)nt * 65536);
  uint64_t* src = keys; uint64_t* dst = tmp;
  for (int pass = 0; pass < 4; ++pass) {
    int shift = pass * 16;
    memset(hist, 0, sizeof(size_t) * (size_t)nt * 65536);
#pragma omp parallel num_threads(nt)
    {
      int t = 0;
#ifdef _OPENMP
      t = omp_get_thread_num();
#endif
      size_t lo = n * (size_t)t / nt, hi = n * (size_t)(t + 1) / nt;
      size_t* h = hist + (size_t)t * 65536;
      for (size_t i = lo; i < hi; ++i) h[(src[i] >> shift) & 0xFFFF]++;
    }
    /* skip pass if one digit holds everything */
    int skip = 0;
    for (int d = 0; d < 65536; ++d) {
      size_t c = 0;
      for (int t = 0; t < nt; ++t) c += hist[(size_t)t * 65536 + d];
      if (c == n) { skip = 1; break; }
      if (c) break;
    }
    if (skip) continue;
    size_t run = 0;
    for (int d = 0; d < 65536; ++d)
      for (int t = 0; t < nt; ++t) {
        size_t c = hist[(size_t)t * 65536 + d];
        hist[(size_t)t * 65536 + d] = run;
        run += c;
      }
#pragma omp parallel num_threads(nt)
    {
      int t = 0;
#ifdef _OPENMP
      t = omp_get_thread_num();
#endif
      size_t lo = n * (size_t)t / nt, hi = n * (size_t)(t + 1) / nt;
      size_t* h = hist + (size_t)t * 65536;
      for (size_t i = lo; i < hi; ++i) dst[h[(src[i] >> shift) & 0xFFFF]++] = src[i];
    }
    uint64_t* s = src; src = dst; dst = s;
  }
  if (src != keys) memcpy(keys, src, n * sizeof(uint64_t));
  free(hist);
}

/* remove consecutive duplicates and the sentinel UINT64_MAX; returns count */
static size_t unique_sorted(uint64_t* k, size_t n) {
  size_t m = 0;
  for (size_t i = 0; i < n; ++i) {
    if (k[i] == UINT64_MAX) break; /* sorted: sentinels at the end */
    if (m == 0 || k[m - 1] != k[i]) k[m++] = k[i];
  }
  return m;
}

/* Keep exactly `want` of the `n` keys: those with the smallest
 * ctr_hash(seed, ST_SELECT, key) (ties impossible in practice; broken by key).
 * Order of the kept keys is preserved. */
static int select_subset(uint64_t* k, size_t n, size_t want, uint64_t seed) {
  if (want >= n) return GG_OK;
  size_t* hist = (size_t*)calloc(65536, sizeof(size_t));
  if (!hist) return GG_ENOMEM;
  for (size_t i = 0; i < n; ++i) hist[ctr_hash(seed, ST_SELECT, k[i]) >> 48]++;
  size_t cum = 0; int b = 0;
  for (b = 0; b < 65536; ++b) { if (cum + hist[b] >= want) break; cum += hist[b]; }
  size_t need = want - cum, nb = hist[b];
  free(hist);
  /* collect hashes of bucket b, find the need-th smallest */
  uint64_t* hb = (uint64_t*)malloc(sizeof(uint64_t) * (nb ? nb : 1));
  uint64_t* tb = (uint64_t*)malloc(sizeof(uint64_t) * (nb ? nb : 1));
  if (!hb || !tb) { free(hb); free(tb); return GG_ENOMEM; }
  size_t c = 0;
  for (size_t i = 0; i < n; ++i) {
    uint64_t h = ctr_hash(seed, ST_SELECT, k[i]);
    if ((int)(h >> 48) == b) hb[c++] = h;
  }
  radix_sort_u64(hb, tb, nb);
  uint64_t thr = need ? hb[need - 1] : 0;
  free(hb); free(tb);
  size_t m = 0, took_eq = 0;
  for (size_t i = 0; i < n; ++i) {
    uint64_t h = ctr_hash(seed, ST_SELECT, k[i]);
    int hb16 = (int)(h >> 48);
    int keep = hb16 < b || (hb16 == b && need && h < thr);
    if (!keep && hb16 == b && need && h == thr && took_eq == 0) { keep = 1; took_eq = 1; }
    if (keep) k[m++] = k[i];
  }
  return m == want ? GG_OK : GG_EINVAL;
}

/* ----------------------------------------------------- vertex relabelling */
/* Bijection on [0,n) by a 4-round Feistel network over 2*hb bits with cycle
 * walking; then shifted so that anchor maps to 0. */
typedef struct { uint64_t n, seed, anchor_img; int hb; } perm_t;
static uint64_t feistel(const perm_t* p, uint64_t x) {
  uint64_t mask = (1ull << p->hb) - 1;
  do {
    uint64_t L = x >> p->hb, R = x & mask;
    for (int r = 0; r < 4; ++r) {
      uint64_t F = ctr_hash(p->seed, ST_PERM, (R << 3) | (uint64_t)r) & mask;
      uint64_t nl = R, nr = L ^ F;
      L = nl; R = nr;
    }
    x = (L << p->hb) | R;
  } while (x >= p->n);
  return x;
}
static void perm_init(perm_t* p, uint64_t n, uint64_t seed, uint64_t anchor) {
  p->n = n; p->seed = seed; int bits = 1;
  while ((1ull << bits) < n) ++bits;
  p->hb = (bits + 1) / 2; if (p->hb < 1) p->hb = 1;
  p->anchor_img = 0;
  p->anchor_img = feistel(p, anchor);
}
static inline uint64_t perm_apply(const perm_t* p, uint64_t v) {
  uint64_t y = feistel(p, v);
  return (y + p->n - p->anchor_img) % p->n;
}

int gg_permute_vertex(uint64_t n, uint64_t seed, uint64_t anchor, const uint32_t* in, uint32_t* out, uint64_t cnt) {
  if (n == 0 || anchor >= n) return GG_EINVAL;
  perm_t p; perm_init(&p, n, seed, anchor);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < (int64_t)cnt; ++i) out[i] = (uint32_t)perm_apply(&p, in[i]);
  return GG_OK;
}

/* Finalise: relabel endpoints of keys (src<<32|dst) by pi, sort, write out. */
static int finish_edges(uint64_t* k, uint64_t* tmp, size_t m, uint64_t V, uint64_t seed, int permute,
                        uint64_t anchor, uint32_t* src, uint32_t* dst) {
  if (permute) {
    perm_t p; perm_init(&p, V, seed, anchor);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)m; ++i) {
      uint64_t s = k[i] >> 32, d = k[i] & 0xFFFFFFFFull;
      k[i] = (perm_apply(&p, s) << 32) | perm_apply(&p, d);
    }
    radix_sort_u64(k, tmp, m);
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < (int64_t)m; ++i) { src[i] = (uint32_t)(k[i] >> 32); dst[i] = (uint32_t)k[i]; }
  return GG_OK;
}

/* one R-MAT sample: 16-bit quantised quadrant choice per level */
static inline void rmat_sample(uint64_t seed, uint64_t k, int scale, uint32_t ta, uint32_t tb, uint32_t tc,
                               uint64_t* s_out, uint64_t* d_out) {
  uint64_t s = 0, d = 0, r = 0;
  for (int lvl = 0; lvl < scale; ++lvl) {
    if ((lvl & 3) == 0) r = ctr_hash(seed, ST_RMAT, k * 16 + (uint64_t)(lvl >> 2));
    uint32_t u = (uint32_t)(r & 0xFFFF); r >>= 16;
    int sb = 0, db = 0;
    if (u < ta) { } else if (u < tb) { db = 1; } else if (u < tc) { sb = 1; } else { sb = 1; db = 1; }
    s = (s << 1) | (uint64_t)sb; d = (d << 1) | (uint64_t)db;
  }
  *s_out = s; *d_out = d;
}

/*
 * R-MAT: exactly E unique directed edges (no self-loops) on V vertices.
 * symmetric != 0: E counts undirected pairs; output has 2E directed edges
 * (both directions).  Output sorted by (src, dst).
 */
int gg_rmat(uint64_t V, uint64_t E, uint64_t seed, double a, double b, double c, int symmetric, int permute,
            uint32_t* src, uint32_t* dst) {
  if (V < 2 || V > 0xFFFFFFFFull || E == 0) return GG_EINVAL;
  double maxe = symmetric ? (double)V * (V - 1) / 2.0 : (double)V * (V - 1);
  if ((double)E > 0.5 * maxe) return GG_EINVAL;
  int scale = 0; while ((1ull << scale) < V) ++scale;
  uint32_t ta = (uint32_t)llround(a * 65536.0), tb = (uint32_t)llround((a + b) * 65536.0),
           tc = (uint32_t)llround((a + b + c) * 65536.0);
  size_t M = (size_t)(E + E / 4 + 4096);
  for (int attempt = 0; attempt < 16; ++attempt) {
    uint64_t* k = (uint64_t*)malloc(M * sizeof(uint64_t));
    uint64_t* t = (uint64_t*)malloc(M * sizeof(uint64_t));
    if (!k || !t) { free(k); free(t); return GG_ENOMEM; }
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)M; ++i) {
      uint64_t s, d;
      rmat_sample(seed, (uint64_t)i, scale, ta, tb, tc, &s, &d);
      if (s >= V || d >= V || s == d) { k[i] = UINT64_MAX; continue; }
      if (symmetric && s > d) { uint64_t x = s; s = d; d = x; }
      k[i] = (s << 32) | d;
    }
    radix_sort_u64(k, t, M);
    size_t m = unique_sorted(k, M);
    if (m < E) { free(k); free(t); M = M + M / 2; continue; }
    int rc = select_subset(k, m, E, seed);
    if (rc) { free(k); free(t); return rc; }
    m = E;
    if (symmetric) {
      /* both directions */
      uint64_t* k2 = (uint64_t*)malloc(2 * m * sizeof(uint64_t));
      uint64_t* t2 = (uint64_t*)malloc(2 * m * sizeof(uint64_t));
      if (!k2 || !t2) { free(k); free(t); free(k2); free(t2); return GG_ENOMEM; }
#pragma omp parallel for schedule(static)
      for (int64_t i = 0; i < (int64_t)m; ++i) {
        k2[2 * i] = k[i];
        k2[2 * i + 1] = ((k[i] & 0xFFFFFFFFull) << 32) | (k[i] >> 32);
      }
      free(k); free(t);
      radix_sort_u64(k2, t2, 2 * m);
      rc = finish_edges(k2, t2, 2 * m, V, seed, permute, 0, src, dst);
      free(k2); free(t2);
      return rc;
    }
    rc = finish_edges(k, t, m, V, seed, permute, 0, src, dst);
    free(k); free(t);
    return rc;
  }
  return GG_EINVAL;
}

/*
 * Road-like mesh: vertices laid out row-major on a grid of the given width
 * (last row partial); of the 4-neighbour bonds, exactly `pairs` are kept
 * (the ones with the smallest hash), stored in both directions (2*pairs edges).
 * Relabelled by pi with pi(grid centre) = 0 when permute != 0.
 */
int gg_mesh(uint64_t V, uint64_t width, uint64_t pairs, uint64_t seed, int permute, uint32_t* src, uint32_t* dst) {
  if (V < 4 || width < 2 || width >= V || V > 0xFFFFFFFFull) return GG_EINVAL;
  uint64_t rows = (V + width - 1) / width;
  /* candidate bonds: horizontal (v, v+1) same row; vertical (v, v+width) */
  size_t cap = (size_t)(2 * V);
  uint64_t* k = (uint64_t*)malloc(cap * sizeof(uint64_t));
  uint64_t* t = (uint64_t*)malloc(2 * pairs * sizeof(uint64_t) > cap * sizeof(uint64_t) ? 2 * pairs * sizeof(uint64_t)
                                                                                       : cap * sizeof(uint64_t));
  if (!k || !t) { free(k); free(t); return GG_ENOMEM; }
  size_t m = 0;
  for (uint64_t v = 0; v < V; ++v) {
    uint64_t col = v % width;
    if (col + 1 < width && v + 1 < V) k[m++] = (v << 32) | (v + 1);
    if (v + width < V) k[m++] = (v << 32) | (v + width);
  }
  (void)rows;
  if (pairs > m) { free(k); free(t); return GG_EINVAL; }
  /* select by hash of the bond */
  int rc = select_subset(k, m, pairs, seed ^ 0x6D657368ull);
  if (rc) { free(k); free(t); return rc; }
  uint64_t* k2 = (uint64_t*)malloc(2 * pairs * sizeof(uint64_t));
  if (!k2) { free(k); free(t); return GG_ENOMEM; }
  for (size_t i = 0; i < pairs; ++i) {
    k2[2 * i] = k[i];
    k2[2 * i + 1] = ((k[i] & 0xFFFFFFFFull) << 32) | (k[i] >> 32);
  }
  free(k);
  radix_sort_u64(k2, t, 2 * pairs);
  uint64_t centre = (rows / 2) * width + width / 2;
  if (centre >= V) centre = V / 2;
  rc = finish_edges(k2, t, 2 * pairs, V, seed, permute, centre, src, dst);
  free(k2); free(t);
  return rc;
}

/* Per-edge u32 values in [lo, hi]; symmetric: value depends on the unordered
 * pair {src,dst} so both directions carry the same weight. */
int gg_edge_u32(uint64_t E, const uint32_t* src, const uint32_t* dst, uint64_t seed, uint32_t lo, uint32_t hi,
                int symmetric, uint32_t* out) {
  if (hi < lo) return GG_EINVAL;
  uint64_t span = (uint64_t)hi - lo + 1;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < (int64_t)E; ++i) {
    uint64_t s = src[i], d = dst[i];
    if (symmetric && s > d) { uint64_t x = s; s = d; d = x; }
    out[i] = lo + (uint32_t)(ctr_hash(seed, ST_EDGEVAL, (s << 32) | d) % span);
  }
  return GG_OK;
}

/* uniform float in [lo, hi) from 24 hash bits */
static inline float u01(uint64_t h) { return (float)((h >> 40) * (1.0 / 16777216.0)); }

int gg_edge_f32(uint64_t E, const uint32_t* src, const uint32_t* dst, uint64_t seed, float lo, float hi,
                int symmetric, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < (int64_t)E; ++i) {
    uint64_t s = src[i], d = dst[i];
    if (symmetric && s > d) { uint64_t x = s; s = d; d = x; }
    out[i] = lo + (hi - lo) * u01(ctr_hash(seed, ST_EDGEVAL, (s << 32) | d));
  }
  return GG_OK;
}

int gg_vertex_f32(uint64_t V, uint64_t seed, uint64_t stream, float lo, float hi, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < (int64_t)V; ++i) out[i] = lo + (hi - lo) * u01(ctr_hash(seed, ST_VERTVAL + stream * 16, (uint64_t)i));
  return GG_OK;
}

/* Uniform random simple directed graph (Erdos-Renyi G(V,E)), for window-size tests. */
int gg_uniform(uint64_t V, uint64_t E, uint64_t seed, uint32_t* src, uint32_t* dst) {
  if (V < 2 || (double)E > 0.5 * (double)V * (V - 1)) return GG_EINVAL;
  size_t M = (size_t)(E + E / 4 + 1024);
  for (int attempt = 0; attempt < 16; ++attempt) {
    uint64_t* k = (uint64_t*)malloc(M * sizeof(uint64_t));
    uint64_t* t = (uint64_t*)malloc(M * sizeof(uint64_t));
    if (!k || !t) { free(k); free(t); return GG_ENOMEM; }
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)M; ++i) {
      uint64_t h = ctr_hash(seed, ST_RMAT + 100, (uint64_t)i);
      uint64_t s = (h >> 32) % V, d = (h & 0xFFFFFFFFull) % V;
      k[i] = s == d ? UINT64_MAX : ((s << 32) | d);
    }
    radix_sort_u64(k, t, M);
    size_t m = unique_sorted(k, M);
    if (m < E) { free(k); free(t); M += M / 2; continue; }
    int rc = select_subset(k, m, E, seed);
    if (!rc) rc = finish_edges(k, t, E, V, seed, 0, 0, src, dst);
    free(k); free(t);
    return rc;
  }
  return GG_EINVAL;
}
