/* grgen.h — seeded synthetic graph generators (shared input module; no GAS
 * arithmetic). See grgen.c and DESIGN.md §3 for the recipes. All outputs are
 * caller-owned arrays; every function is a pure function of its arguments. */
#ifndef GRGEN_H
#define GRGEN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* counter-based splitmix64 draw for (seed, stream, counter) */
uint64_t grgen_hash(uint64_t seed, uint64_t stream, uint64_t counter);

/* R-MAT with quadrant probabilities a,b,c,(1-a-b-c); vertex ids in [0, 2^scale).
 * Writes m edges; duplicates and self-loops kept. Returns 0, or <0 on bad args. */
int grgen_rmat(uint32_t scale, uint64_t m, double a, double b, double c, uint64_t seed,
               uint32_t *src, uint32_t *dst, int threads);

/* uniform integer weights in [lo, hi] keyed by edge index */
int grgen_weights(uint64_t m, uint32_t lo, uint32_t hi, uint64_t seed, uint32_t *w, int threads);

/* Road-like W x H lattice: keep each lattice edge with probability p, then
 * repair connectivity; both directions stored with weight 1 + hash % wmax.
 * Returns m (edges written or, with src == NULL, the count), or <0. */
int64_t grgen_grid(uint32_t W, uint32_t H, double p, uint32_t wmax, uint64_t seed, uint32_t *src,
                   uint32_t *dst, uint32_t *w, uint64_t cap);

/* Web-like power-law graph, symmetrized (both directions), self-loops dropped.
 * Returns m (written or, with src == NULL, the count), or <0. */
int64_t grgen_web(uint64_t n, double xmin, double zexp, uint32_t dmax, double p_local,
                  double geo_p, uint32_t local_cap, double rank_exp, uint64_t seed,
                  uint32_t *src, uint32_t *dst, uint64_t cap, int threads);

#ifdef __cplusplus
}
#endif
#endif
