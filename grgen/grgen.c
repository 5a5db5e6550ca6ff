/*
 * grgen.c — seeded synthetic graph generators (input recipes of DESIGN.md §3).
 *
 * This module is the ONLY code shared by the CUDA path and the oracle: it
 * produces canonical COO edge lists (src[i] -> dst[i], optional weights) and
 * holds none of the GAS method's arithmetic. Every random draw is a
 * counter-based splitmix64 of (seed, stream, counter), so the output is a pure
 * function of the parameters and independent of the thread count.
 *
 * Shapes follow SURVEY.md §8(d) (BASELINE.json configs 1-5):
 *   - R-MAT / Kronecker (kron_g500-logn*, configs 1, 2, 5)  [PAPER.md L85, L89]
 *   - road-like 2-D lattice (belgium_osm-like, config 3)    [PAPER.md L87]
 *   - web-like power law (uk-2002-like, config 4)           [PAPER.md L91]
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include "grgen.h"

static inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

uint64_t grgen_hash(uint64_t seed, uint64_t stream, uint64_t counter) {
  uint64_t key = mix64(seed * 0x9E3779B97F4A7C15ULL + 0x632BE59BD9B4E019ULL) ^
                 mix64(stream + 0x8CB92BA72F3D8DD7ULL);
  return mix64(key + (counter + 1) * 0x9E3779B97F4A7C15ULL);
}

/* uniform double in [0,1) with 53 bits */
static inline double u01(uint64_t h) { return (double)(h >> 11) * (1.0 / 9007199254740992.0); }
/* uniform double in (0,1] */
static inline double u01_open0(uint64_t h) { return ((double)(h >> 11) + 1.0) * (1.0 / 9007199254740992.0); }

static int clamp_threads(int t) {
  if (t <= 0) t = 1;
  if (t > 256) t = 256;
  return t;
}

/* ------------------------------------------------------------------ R-MAT */
int grgen_rmat(uint32_t scale, uint64_t m, double a, double b, double c, uint64_t seed,
               uint32_t *src, uint32_t *dst, int threads) {
  if (scale == 0 || scale > 32 || !src || !dst) return -1;
  if (a < 0 || b < 0 || c < 0 || a + b + c > 1.0) return -1;
  const double ab = a + b, abc = a + b + c;
  threads = clamp_threads(threads);
  /* one 64-bit draw gives two levels (2 x 32-bit uniforms) */
  const uint32_t draws = (scale + 1) / 2;
#pragma omp parallel for num_threads(threads) schedule(static)
  for (int64_t i = 0; i < (int64_t)m; i++) {
    uint64_t s = 0, d = 0;
    for (uint32_t j = 0; j < draws; j++) {
      uint64_t h = grgen_hash(seed, 1, (uint64_t)i * draws + j);
      for (int k = 0; k < 2; k++) {
        uint32_t level = 2 * j + k;
        if (level >= scale) break;
        double u = (double)((uint32_t)(h >> (32 * k))) * (1.0 / 4294967296.0);
        uint64_t sb, db;
        if (u < a) { sb = 0; db = 0; }
        else if (u < ab) { sb = 0; db = 1; }
        else if (u < abc) { sb = 1; db = 0; }
        else { sb = 1; db = 1; }
        s = (s << 1) | sb;
        d = (d << 1) | db;
      }
    }
    src[i] = (uint32_t)s;
    dst[i] = (uint32_t)d;
  }
  return 0;
}

/* ------------------------------------------------------------- weights */
int grgen_weights(uint64_t m, uint32_t lo, uint32_t hi, uint64_t seed, uint32_t *w, int threads) {
  if (!w || hi < lo) return -1;
  threads = clamp_threads(threads);
  const uint64_t span = (uint64_t)hi - lo + 1;
#pragma omp parallel for num_threads(threads) schedule(static)
  for (int64_t i = 0; i < (int64_t)m; i++) w[i] = lo + (uint32_t)(grgen_hash(seed, 7, (uint64_t)i) % span);
  return 0;
}

/* ------------------------------------------------------------ road grid */
static uint32_t uf_find(uint32_t *p, uint32_t x) {
  while (p[x] != x) {
    p[x] = p[p[x]];
    x = p[x];
  }
  return x;
}

typedef struct {
  uint64_t key;
  uint64_t e;
} keyed_t;

static int cmp_keyed(const void *x, const void *y) {
  const keyed_t *a = (const keyed_t *)x, *b = (const keyed_t *)y;
  if (a->key != b->key) return a->key < b->key ? -1 : 1;
  return a->e < b->e ? -1 : (a->e > b->e);
}

static inline void lattice_edge(uint32_t W, uint32_t H, uint64_t e, uint32_t *x, uint32_t *y) {
  uint64_t nh = (uint64_t)H * (W - 1);
  if (e < nh) {
    uint64_t r = e / (W - 1), c = e % (W - 1);
    *x = (uint32_t)(r * W + c);
    *y = (uint32_t)(r * W + c + 1);
  } else {
    e -= nh;
    uint64_t r = e / W, c = e % W;
    *x = (uint32_t)(r * W + c);
    *y = (uint32_t)((r + 1) * W + c);
  }
}

int64_t grgen_grid(uint32_t W, uint32_t H, double p, uint32_t wmax, uint64_t seed, uint32_t *src,
                   uint32_t *dst, uint32_t *w, uint64_t cap) {
  if (W < 1 || H < 1 || (uint64_t)W * H >= 0xFFFFFFFFULL || wmax < 1) return -1;
  const uint64_t n = (uint64_t)W * H;
  const uint64_t nl = (uint64_t)H * (W - 1) + (uint64_t)(H - 1) * W; /* lattice edges */
  uint8_t *keep = (uint8_t *)calloc(nl ? nl : 1, 1);
  uint32_t *par = (uint32_t *)malloc(sizeof(uint32_t) * n);
  if (!keep || !par) { free(keep); free(par); return -2; }
  for (uint64_t v = 0; v < n; v++) par[v] = (uint32_t)v;
  uint64_t nrest = 0;
  for (uint64_t e = 0; e < nl; e++) {
    if (u01(grgen_hash(seed, 1, e)) < p) {
      keep[e] = 1;
      uint32_t x, y;
      lattice_edge(W, H, e, &x, &y);
      uint32_t rx = uf_find(par, x), ry = uf_find(par, y);
      if (rx != ry) par[rx] = ry;
    } else {
      nrest++;
    }
  }
  /* connectivity repair: non-kept lattice edges in seeded order, added when
   * they join two components (config 3) */
  keyed_t *cand = (keyed_t *)malloc(sizeof(keyed_t) * (nrest ? nrest : 1));
  if (!cand) { free(keep); free(par); return -2; }
  uint64_t k = 0;
  for (uint64_t e = 0; e < nl; e++)
    if (!keep[e]) { cand[k].key = grgen_hash(seed, 2, e); cand[k].e = e; k++; }
  qsort(cand, nrest, sizeof(keyed_t), cmp_keyed);
  for (uint64_t i = 0; i < nrest; i++) {
    uint32_t x, y;
    lattice_edge(W, H, cand[i].e, &x, &y);
    uint32_t rx = uf_find(par, x), ry = uf_find(par, y);
    if (rx != ry) { par[rx] = ry; keep[cand[i].e] = 1; }
  }
  free(cand);
  free(par);
  uint64_t m = 0;
  for (uint64_t e = 0; e < nl; e++) m += keep[e] ? 2 : 0;
  if (src && dst) {
    if (m > cap) { free(keep); return -3; }
    uint64_t j = 0;
    for (uint64_t e = 0; e < nl; e++) {
      if (!keep[e]) continue;
      uint32_t x, y;
      lattice_edge(W, H, e, &x, &y);
      uint32_t wt = 1 + (uint32_t)(grgen_hash(seed, 3, e) % wmax);
      src[j] = x; dst[j] = y; if (w) w[j] = wt; j++;
      src[j] = y; dst[j] = x; if (w) w[j] = wt; j++;
    }
  }
  free(keep);
  return (int64_t)m;
}

/* -------------------------------------------------------------- web-like */
static uint32_t web_degree(uint64_t seed, uint64_t u, double xmin, double zexp, uint32_t dmax) {
  /* discretised Pareto: P(D >= x) ~ x^-(zexp-1)  (Zipf exponent zexp) */
  double U = u01_open0(grgen_hash(seed, 1, u));
  double x = xmin * pow(U, -1.0 / (zexp - 1.0));
  if (x > (double)dmax) x = (double)dmax;
  return (uint32_t)floor(x);
}

static int cmp_u64pair(const void *x, const void *y) {
  const uint64_t *a = (const uint64_t *)x, *b = (const uint64_t *)y;
  if (a[0] != b[0]) return a[0] < b[0] ? -1 : 1;
  return a[1] < b[1] ? -1 : (a[1] > b[1]);
}

int64_t grgen_web(uint64_t n, double xmin, double zexp, uint32_t dmax, double p_local,
                  double geo_p, uint32_t local_cap, double rank_exp, uint64_t seed,
                  uint32_t *src, uint32_t *dst, uint64_t cap, int threads) {
  if (n < 2 || n >= 0xFFFFFFFFULL || zexp <= 1.0 || geo_p <= 0 || geo_p >= 1) return -1;
  threads = clamp_threads(threads);
  uint64_t *off = (uint64_t *)malloc(sizeof(uint64_t) * (n + 1));
  if (!off) return -2;
  off[0] = 0;
  for (uint64_t u = 0; u < n; u++) off[u + 1] = off[u] + web_degree(seed, u, xmin, zexp, dmax);
  const uint64_t total = off[n];
  /* seeded permutation for the global (Chung-Lu by rank) targets */
  uint64_t *pk = (uint64_t *)malloc(sizeof(uint64_t) * 2 * n);
  uint32_t *perm = (uint32_t *)malloc(sizeof(uint32_t) * n);
  uint8_t *selfl = (uint8_t *)malloc(total ? total : 1);
  uint32_t *tgt = (uint32_t *)malloc(sizeof(uint32_t) * (total ? total : 1));
  if (!pk || !perm || !selfl || !tgt) { free(off); free(pk); free(perm); free(selfl); free(tgt); return -2; }
  for (uint64_t v = 0; v < n; v++) { pk[2 * v] = grgen_hash(seed, 3, v); pk[2 * v + 1] = v; }
  qsort(pk, n, 2 * sizeof(uint64_t), cmp_u64pair);
  for (uint64_t r = 0; r < n; r++) perm[r] = (uint32_t)pk[2 * r + 1];
  free(pk);
  const double span = pow((double)n + 1.0, 1.0 - rank_exp) - 1.0;
  const double lq = log(1.0 - geo_p);
#pragma omp parallel for num_threads(threads) schedule(dynamic, 4096)
  for (int64_t u = 0; u < (int64_t)n; u++) {
    for (uint64_t e = off[u]; e < off[u + 1]; e++) {
      uint64_t h = grgen_hash(seed, 4, e);
      uint64_t h2 = grgen_hash(seed, 5, e);
      int64_t t;
      if (u01(h) < p_local) {
        /* local: u +/- Geometric(geo_p) (>=1), capped, wrapped mod n */
        double U = u01_open0(h2);
        uint64_t kk = 1 + (uint64_t)floor(log(U) / lq);
        if (kk > local_cap) kk = local_cap;
        if (h & 1) t = ((int64_t)u + (int64_t)(kk % n)) % (int64_t)n;
        else t = ((int64_t)u - (int64_t)(kk % n) + (int64_t)n) % (int64_t)n;
      } else {
        /* global: rank r with P(r) ~ (r+1)^-rank_exp by inverse CDF, then permuted */
        double U = u01(h2);
        double r = pow(1.0 + U * span, 1.0 / (1.0 - rank_exp)) - 1.0;
        uint64_t ri = (uint64_t)floor(r);
        if (ri >= n) ri = n - 1;
        t = perm[ri];
      }
      tgt[e] = (uint32_t)t;
      selfl[e] = (t == u);
    }
  }
  free(perm);
  uint64_t kept = 0;
  for (uint64_t e = 0; e < total; e++) kept += !selfl[e];
  const uint64_t m = 2 * kept;
  if (src && dst) {
    if (m > cap) { free(off); free(selfl); free(tgt); return -3; }
    uint64_t j = 0;
    for (uint64_t u = 0; u < n; u++)
      for (uint64_t e = off[u]; e < off[u + 1]; e++) {
        if (selfl[e]) continue;
        src[j] = (uint32_t)u; dst[j] = tgt[e]; j++;
        src[j] = tgt[e]; dst[j] = (uint32_t)u; j++;
      }
  }
  free(off);
  free(selfl);
  free(tgt);
  return (int64_t)m;
}
