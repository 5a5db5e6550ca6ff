/* oracle.h — TEST INFRASTRUCTURE ONLY. A plain, slow, single-threaded CPU GAS
 * engine written from the paper (§2.1, §4.4, §5.2
 * L270, §5.3, Fig. 6). Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load it. It shares
 * no code or headers with the CUDA path (paper_conf_sc_senguptasas15_b200/). */
#ifndef GR_ORACLE_H
#define GR_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum { OR_BFS = 0, OR_SSSP = 1, OR_PAGERANK = 2, OR_CC = 3, OR_WIDEST = 4, OR_PRDELTA = 5, OR_SSSPMSG = 6, OR_HEAT = 7 };
#define OR_HEAT_H0 0x40000000u /* OR_HEAT: heat at the source at initialisation */
#define OR_INF 0xFFFFFFFFu

typedef struct or_graph or_graph;

/* Build the oracle's own CSC (in-edges sorted by (dst, src, w)) and CSR
 * (out-edges sorted by (src, dst, w)) from a COO list. w may be NULL.
 * Returns NULL on bad input (id >= n) or allocation failure. */
or_graph *or_graph_build(uint64_t n, uint64_t m, const uint32_t *src, const uint32_t *dst,
                         const uint32_t *w);
void or_graph_free(or_graph *g);

/* Run one program to termination (or max_iters supersteps; 0 = unlimited).
 * values_out: uint32_t[n] for BFS/SSSP/CC/WIDEST, double[n] for PAGERANK,
 * uint32_t[n] fp32 bit patterns for PRDELTA.
 * OR_PRDELTA: tolerance-driven PageRank (Figs. 16-17,
 * L360-372): A_0 = V; a vertex changes (and only then takes its new rank) when
 * |R_new - R_old| > tolerance / n. Ranks are fp32; the gather is the exact sum
 * of floor(fix(R_u) / n_u) in 2^-62 fixed point, fix(R) = floor(R * 2^62);
 * R_new = fp32(double(floor(((2^20 - q) << 42) / n) + floor(S * q / 2^20)) * 2^-62),
 * q = round(d * 2^20) of the fp32 damping d.
 * OR_WIDEST: single-source widest path (max over paths of the min edge weight),
 * a user GAS program (§4.1) used to check GR_CUSTOM programs.
 * OR_SSSPMSG: SSSP with mutable edge state (the Scatter phase, §2.1
 * L66, §4.4): every edge holds a message, initially INF; after the apply
 * of superstep t and the commit of the new values, every edge (u -> x) with u
 * changed at t gets S = new[u] + w if that is < val[x] (the committed value),
 * else INF; the gather takes the min of the messages on the in-edges. The
 * source is set to 0 and scatters at initialisation.
 * OR_HEAT: heat diffusion with mutable edge state (§2.1 "Heat
 * Simulation"; Scatter L66): temperatures are uint32 heat units, the source
 * starts at OR_HEAT_H0 and everything else at 0; every edge holds the heat
 * its source sends along it, initially 0. The source counts as changed at
 * initialisation and scatters. Superstep t: T_new[x] = sum of the states of
 * x's in-edges (changed iff it differs); after the commit every edge
 * (u -> x) with u changed gets floor(T[u] * (w + 1) / 256). With
 * sum_x (w(u->x) + 1) = 256 for every u (a self-loop carries the heat u
 * keeps) this is the explicit heat step T' = W^T T in fixed point.
 * trace_out (nullable): rows of 4 uint64 per superstep t:
 *   |A_t|, |C_t|, sum_{v in A_t} indeg(v) (0 when gather is eliminated),
 *   sum_{u in C_t} outdeg(u) (0 when FrontierActivate is eliminated).
 * Returns the number of supersteps executed, or <0 on error. */
int64_t or_run(or_graph *g, int algo, uint32_t source, uint32_t max_iters, double damping,
               double tolerance, void *values_out, uint64_t *trace_out, uint64_t trace_cap,
               uint64_t *rows_out);

/* or_run plus the detail columns of the frontier trace:
 * detail_out (nullable): 2 uint64 per superstep t —
 *   active_shards = number of shards [bounds[s], bounds[s+1]) holding a vertex of
 *                   A_t (frontier skipping, §5.2; 0 without bounds),
 *   S_t           = number of distinct sources read by the gather of A_t (0 when
 *                   the gather is eliminated). */
int64_t or_run_detail(or_graph *g, int algo, uint32_t source, uint32_t max_iters, double damping,
                      double tolerance, void *values_out, uint64_t *trace_out, uint64_t trace_cap,
                      uint64_t *rows_out, const uint64_t *shard_bounds, uint32_t num_shards,
                      uint64_t *detail_out);

#ifdef __cplusplus
}
#endif
#endif
