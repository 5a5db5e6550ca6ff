/*
 * graphreduce.h — C ABI of the B200-native sharded Gather-Apply-Scatter (GAS)
 * superstep (GraphReduce, Sengupta et al., SC'15; /root/reference/PAPER.md).
 *
 * The library computes, on one or more B200 GPUs, the GAS model of PAPER.md
 * §2.1 (L62-66): per BSP superstep (L76, L256) a gather over every active
 * vertex's in-edges (gatherMap + gatherReduce, §4.4), an apply per
 * active vertex (L252), and a FrontierActivate over the changed vertices'
 * out-edges (L254, §5.2). The graph is cut into destination-interval
 * shards (§4.2) stored as CSC (in-edges, sorted by destination) and
 * CSR (out-edges, sorted by source) (L208-210). Shards stay resident in HBM or
 * are streamed from pinned host memory (§3.2, §4.3).
 *
 * Conventions (every function):
 *   - returns gr_status; never aborts or exits; on failure the thread-local
 *     message from gr_last_error() says why (CUDA/NCCL error strings included);
 *   - all pointers are HOST pointers unless the field says "device";
 *   - inputs are caller-owned and may be freed as soon as the call returns;
 *     output buffers are caller-owned; a gr_graph is owned by the caller and
 *     released with gr_graph_free();
 *   - one thread at a time per gr_graph handle.
 * Vertex ids are uint32 (n < 2^32 - 1; 0xFFFFFFFF is reserved as INF).
 */
#ifndef GRAPHREDUCE_H
#define GRAPHREDUCE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GR_INF 0xFFFFFFFFu
#define GR_ABI_VERSION 1

typedef enum gr_status {
  GR_OK = 0,
  GR_EINVAL = 1,        /* bad argument: null pointer, id >= n, source >= n, SSSP w/o weights,
                           weight > 255, buffer too small, damping outside (0,1) */
  GR_ENOMEM = 2,        /* device or pinned-host allocation failed */
  GR_ECUDA = 3,         /* CUDA runtime error (message carries cudaGetErrorString) */
  GR_ENCCL = 4,         /* NCCL error (message carries ncclGetErrorString) */
  GR_EUNSUPPORTED = 5,  /* valid request this build cannot serve */
  GR_ESTATE = 6         /* call out of order (e.g. fetch before run) */
} gr_status;

typedef enum gr_format {
  GR_FMT_COO = 0,   /* src[i] -> dst[i], any order, duplicates/self-loops kept (multigraph) */
  GR_FMT_CSR = 1,   /* out-edges of u: col_idx[row_offsets[u] .. row_offsets[u+1]) */
  GR_FMT_SORTED = 2 /* the layout itself, already sorted (single rank; no weights): the in-CSC
                       (in_offsets[n+1] by destination, in_idx = sources, every row ascending) and/or
                       the out-CSR (row_offsets / col_idx, every row ascending) of the same edge
                       multiset. One half alone is accepted for STREAMED graphs (PageRank needs the
                       in-CSC, BFS the out-CSR; other programs fail with GR_EUNSUPPORTED). This is
                       how graphs whose COO does not fit host memory are loaded (cfg5 at scale). */
} gr_format;

/* Programs: the paper's four evaluated algorithms (§6.1). */
typedef enum gr_algo {
  GR_BFS = 0,      /* depth = superstep number (L276); gather eliminated, apply+activate fused */
  GR_SSSP = 1,     /* Bellman-Ford with frontier; "BFS with weighted edges" (L372) */
  GR_PAGERANK = 2, /* L74 (reading R1): R = (1-d)/n + d*sum R_u/outdeg(u); fixed iterations */
  GR_CC = 3,       /* Fig. 6: min-label propagation; input must be symmetric (L290) */
  GR_CUSTOM = 4,   /* program compiled into the library: GR_CUSTOM_PROGRAMS in gr/program.cuh
                      (0: widest path; 1: SSSP by edge messages — mutable edge state written by
                      the Scatter phase, every mode; 2: heat diffusion, §2.1 L68 — the
                      heat flow stored on the edges, fixed-point explicit step, every mode) */
  GR_PAGERANK_DELTA = 5 /* tolerance-driven PageRank (Figs. 16-17): a vertex
                           stays active while |dR| > tolerance/n; exact fixed-point gather, so the
                           frontier is reproducible (gr/program.cuh ProgPRDelta); fp32 rank values */
} gr_algo;

typedef enum gr_mode {
  GR_MODE_AUTO = 0,     /* resident if the shards fit device_budget_bytes, else streamed */
  GR_MODE_RESIDENT = 1, /* every shard copied to HBM once at load */
  GR_MODE_STREAMED = 2  /* shards stay in pinned host memory; copied per superstep, double-buffered */
} gr_mode;

typedef enum gr_loop {
  GR_LOOP_AUTO = 0,       /* persistent loop where supported (single rank, resident), else host */
  GR_LOOP_HOST = 1,       /* host reads the frontier count after every superstep */
  GR_LOOP_DEVICE = 2,     /* CUDA graph with a conditional WHILE node (no host round trip) */
  GR_LOOP_PERSISTENT = 3  /* one cooperative kernel runs every superstep; grid barriers between phases */
} gr_loop;

/* Input graph (caller-owned; the library copies what it needs during load). */
typedef struct gr_edges {
  int32_t fmt;                   /* gr_format */
  uint64_t num_vertices;         /* n */
  uint64_t num_edges;            /* m (directed, stored) */
  const uint32_t *src, *dst;     /* COO: m entries each */
  const uint64_t *row_offsets;   /* CSR: n+1 entries */
  const uint32_t *col_idx;       /* CSR: m entries */
  const uint32_t *weights;       /* nullable; m entries in [0, 255]; required for SSSP */
  const uint64_t *in_offsets;    /* GR_FMT_SORTED: in-CSC offsets (n+1) by destination, or NULL */
  const uint32_t *in_idx;        /* GR_FMT_SORTED: in-CSC sources (m entries + 4 spare when borrowed) */
  const uint32_t *out_degree;    /* GR_FMT_SORTED without an out-CSR: out-degree of every vertex (n),
                                    PageRank's n_j; NULL = counted from in_idx */
} gr_edges;

typedef struct gr_load_opts {
  uint64_t shard_edges;          /* target in+out edges per shard; 0 = auto (Eq. 1-2 rule, K = 2) */
  uint64_t device_budget_bytes;  /* 0 = free device memory minus a reserve; a small value forces streaming */
  int32_t mode;                  /* gr_mode */
  int32_t device;                /* CUDA device ordinal */
  int32_t rank, world;           /* multi-GPU: this rank and the rank count; world <= 1 = single GPU */
  const void *nccl_unique_id;    /* world > 1: 128 bytes from gr_get_unique_id() on rank 0, broadcast */
  int32_t host_threads;          /* shard-builder threads; 0 = all cores */
  int32_t sim_ranks;             /* > 1: emulate this many owner partitions on ONE device (tests) */
  int32_t build;                 /* gr_build: where the shard layout is built */
  int32_t transport;             /* gr_transport: how the ranks of a multi-rank graph exchange */
  int32_t borrow;                /* GR_FMT_SORTED: 1 = use the caller's adjacency arrays in place (no copy;
                                    each needs 4 spare entries after its m used ones); they must stay
                                    valid and unchanged until gr_graph_free (streamed graphs page-lock
                                    them, or use them as they are if the caller already did) */
} gr_load_opts;

typedef enum gr_transport {
  GR_TRANSPORT_NCCL = 0, /* one process per GPU; NCCL (bootstrap: gr_get_unique_id) + cudaIpc peer
                            mappings over NVLink/NVSwitch for the fused exchanges */
  GR_TRANSPORT_SHM = 1   /* one process per rank on ONE node, ranks may share a GPU: host
                            collectives through a POSIX shared-memory segment named after the
                            128-byte id (any bytes, identical on every rank), device data through
                            cross-process cudaIpc mappings; same protocol as NCCL (tests, MPS) */
} gr_transport;

typedef enum gr_build {
  GR_BUILD_AUTO = 0,   /* device for resident single-rank COO inputs, else host */
  GR_BUILD_HOST = 1,   /* multithreaded host builder (always used for streamed / multi-rank graphs) */
  GR_BUILD_DEVICE = 2  /* upload the COO and sort it on the GPU (resident, single rank, COO only) */
} gr_build;

typedef struct gr_run_opts {
  int32_t algo;       /* gr_algo */
  uint32_t source;    /* BFS / SSSP source vertex */
  uint32_t max_iters; /* 0 = PageRank: 30, others: until the frontier is empty */
  float damping;      /* PageRank d; 0 = 0.85 */
  int32_t custom_id;  /* GR_CUSTOM: registered program id */
  int32_t loop;       /* gr_loop */
  void *stream;       /* cudaStream_t to order the run on (device work only); NULL = library stream */
  int32_t profile;    /* 1: time the per-phase kernels with CUDA events (stats.kernel_ms) */
  int32_t direction;  /* gr_direction: how FrontierActivate reaches the out-neighbours of C_t */
  uint32_t pull_div;  /* GR_DIR_AUTO: pull when |C_t| * pull_div > |V|; 0 = library default (16) */
  float tolerance;    /* GR_PAGERANK_DELTA: a vertex changes when |R_new - R_old| > tolerance / n (>= 0) */
  int32_t zero_copy;  /* streamed mode: how a superstep reads the active shards' edges —
                         0 auto (in place over the host link when the frontier's edges are
                         < 1/8 of the active shards' edges, else DMA whole shards into the
                         device slots), 1 always in place, -1 never */
  int32_t trace_detail; /* 1: also record, per superstep, the number of shards holding an active vertex
                           and the number of distinct sources the gather reads (diagnostic: runs the
                           host loop with extra marking kernels; resident single-rank graphs only,
                           else GR_EUNSUPPORTED); fetch with gr_fetch_frontier_trace_detail */
} gr_run_opts;

/* FrontierActivate direction (resident single-rank frontier programs; the
 * activated set and the trace are identical either way — only the cost differs). */
typedef enum gr_direction {
  GR_DIR_AUTO = 0,  /* pull when the changed set is large (|C_t| * pull_div > |V|), else push */
  GR_DIR_PUSH = 1,  /* always expand the out-edges of C_t (stamps + atomics) */
  GR_DIR_PULL = 2,  /* always scan the in-edges of every vertex for a changed source */
  GR_DIR_FUSED = 3  /* programs declaring kPushFused (SSSP, widest path; gr/program.cuh): apply and
                       a push FrontierActivate that carries the gather (atomicGather into a per-vertex
                       accumulator) run as ONE phase per superstep (resident single-rank graphs;
                       measured slower than AUTO on the road grid, so opt-in); other programs
                       and modes treat FUSED as AUTO */
} gr_direction;

typedef struct gr_run_stats {
  uint32_t iterations;       /* supersteps executed */
  double seconds;            /* device time of the run (CUDA events on the run stream) */
  uint64_t edges_gathered;   /* sum over supersteps of sum_{v in A_t} indeg(v) */
  uint64_t edges_scattered;  /* sum over supersteps of sum_{u in C_t} outdeg(u) */
  uint64_t bytes_h2d;        /* streamed shard bytes moved host -> device */
  uint64_t bytes_nvlink;     /* bytes received from peers per rank (allgather) */
  uint64_t bytes_hbm_model;  /* algorithmic (compulsory) HBM bytes */
  uint64_t kernel_launches;  /* library kernel launches issued by this run */
  double kernel_ms[4];       /* profile: [0] gather(+apply), [1] activate/expand, [2] exchange, [3] other */
  uint32_t pull_supersteps;  /* supersteps whose FrontierActivate ran by pull */
  uint32_t zero_copy_phases; /* streamed: gather / activate phases that read edges in place */
  uint64_t bytes_h2d_zero_copy; /* part of bytes_h2d read in place by the kernels (4 B per edge, +1 B weight) */
} gr_run_stats;

typedef struct gr_graph_info {
  uint64_t num_vertices, num_edges;
  uint32_t num_shards;
  int32_t mode;              /* gr_mode actually chosen */
  int32_t rank, world, sim_ranks;
  uint64_t own_lo, own_hi;   /* owned destination range of this rank */
  uint64_t device_bytes;     /* device memory held by the graph */
  uint64_t pinned_bytes;     /* pinned host memory held by the graph */
  int32_t offsets_64bit;     /* 1 if edge offsets are stored as uint64 on the device */
  int32_t has_weights;
  int32_t built_on_device;   /* 1 if the layout was built by the GPU build path (GR_BUILD_DEVICE) */
  int32_t reserved;
} gr_graph_info;

/* One destination-interval shard (Fig. 7, §4.2). */
typedef struct gr_shard_desc {
  uint64_t v_lo, v_hi;       /* vertex interval [v_lo, v_hi) */
  uint64_t in_begin, in_end; /* its in-edges (CSC positions, dst in interval) */
  uint64_t out_begin, out_end; /* its out-edges (CSR positions, src in interval) */
} gr_shard_desc;

typedef struct gr_graph gr_graph;
typedef struct gr_host_graph gr_host_graph;

/* ---- multi-GPU bootstrap -------------------------------------------------- */
/* Rank 0 calls this and broadcasts the 128 bytes (e.g. through a torch process
 * group) to every rank before gr_graph_load. */
gr_status gr_get_unique_id(uint8_t out[128]);

/* ---- load / run / fetch ---------------------------------------------------- */
/* Partition (§4.2), lay out CSC/CSR, and place the shards (resident
 * or pinned-host streamed). With world > 1 every rank passes the SAME edges and
 * keeps only its owned destination range. */
gr_status gr_graph_load(const gr_edges *edges, const gr_load_opts *opts, gr_graph **out);

/* Load from a canonical graph file (memory-mapped, read-only; every rank of a
 * multi-GPU job maps the same file and keeps its owned range — SURVEY §8(b)).
 * Little-endian layout, 32-byte header then the arrays, each 4-byte aligned:
 *   char     magic[8] = "GRGRAPH1"
 *   uint64_t num_vertices, num_edges
 *   uint32_t fmt        (gr_format: 0 COO, 1 CSR by source)
 *   uint32_t flags      (bit 0: weights present)
 *   COO: uint32 src[m], uint32 dst[m]          CSR: uint64 row_offsets[n+1], uint32 col_idx[m]
 *   then, if flags & 1: uint32 weights[m]
 * GR_EINVAL: unreadable file, bad magic/format/flags, or a size that does not
 * match the header; otherwise exactly gr_graph_load's behaviour. The mapping
 * is released before returning. */
gr_status gr_graph_load_file(const char *path, const gr_load_opts *opts, gr_graph **out);

/* Run one program to termination (PAPER.md L62 stages 1-3). Synchronous: returns
 * when the results are on the device. */
gr_status gr_run(gr_graph *g, const gr_run_opts *opts, gr_run_stats *stats);

/* Copy the final vertex values to host_dst: uint32[n] (BFS depth, SSSP distance,
 * CC label; GR_INF = unreached) or float32[n] (PageRank). bytes must be >= 4n.
 * Every rank receives all n values. GR_ESTATE before the first gr_run. */
gr_status gr_fetch_vertex_values(gr_graph *g, void *host_dst, uint64_t bytes);

/* Copy the frontier trace of the last run: 4 uint64 per superstep t:
 * |A_t|, |C_t|, sum_{A_t} indeg (0 if gather eliminated), sum_{C_t} outdeg (0 if
 * FrontierActivate eliminated). *rows = supersteps recorded (<= max_rows). */
gr_status gr_fetch_frontier_trace(gr_graph *g, uint64_t *host_dst, uint64_t max_rows, uint64_t *rows);

/* Detail columns of the last run's trace (it must have run with trace_detail = 1;
 * else GR_ESTATE): 2 uint64 per superstep t — active_shards (shards
 * [v_lo, v_hi) of gr_shard_info holding a vertex of A_t: what frontier skipping
 * moves, §5.2) and S_t (distinct sources read by the gather of A_t;
 * 0 when the gather is eliminated). *rows = supersteps recorded (<= max_rows). */
gr_status gr_fetch_frontier_trace_detail(gr_graph *g, uint64_t *host_dst, uint64_t max_rows, uint64_t *rows);

/* ---- run-time GAS programs (§4.1, Fig. 6) ----
 * Compile a user program at run time and register it. `source` is CUDA C++
 * that defines `struct <struct_name>` (the library places it inside namespace
 * gr, where Ctx, kInitAll & co. and the CUDA intrinsics are visible) with the interface
 * of include/gr/program.cuh: GatherT (4- or 8-byte unsigned), kHasGather,
 * kUsesWeights, kInit (kInitSource / kInitSourceChanged / kInitAll),
 * initValue, identity, gatherMap, gatherReduce (associative + commutative),
 * atomicGather, apply; vertex values are uint32. The library compiles it with
 * NVRTC for the current device together with its own frontier kernels (the
 * same gather / apply / FrontierActivate / persistent BSP loop as the built-in
 * programs) and loads the module; run it with gr_run(algo = GR_CUSTOM,
 * custom_id = *custom_id) on a resident single-GPU graph (persistent loop).
 * Ids start at 1000; programs live until process exit.
 * GR_EINVAL: null argument or empty name; GR_EUNSUPPORTED: libnvrtc /
 * libcuda not loadable; GR_ECUDA: compile or load error — gr_last_error()
 * carries the NVRTC log. Thread-safe. */
gr_status gr_program_compile(const char *source, const char *struct_name, int32_t *custom_id);

gr_status gr_graph_info_get(const gr_graph *g, gr_graph_info *out);
gr_status gr_shard_info(const gr_graph *g, uint32_t shard, gr_shard_desc *out);
void gr_graph_free(gr_graph *g); /* NULL-safe */
const char *gr_last_error(void);  /* thread-local; never NULL */

/* ---- host-only logic (no GPU needed; used by the loader and by CPU tests) --- */
/* Cut [0, n) into P intervals of near-equal weight: weight_prefix[v+1] -
 * weight_prefix[v] is vertex v's weight (in+out degree, §4.2). Writes
 * bounds[0..P] with bounds[0] = 0, bounds[P] = n, non-decreasing. */
gr_status gr_plan_intervals(uint64_t n, const uint64_t *weight_prefix, uint32_t P, uint64_t *bounds);

/* Build the host-side sharded layout (CSC + CSR + shard table) without a GPU. */
gr_status gr_host_build(const gr_edges *edges, const gr_load_opts *opts, gr_host_graph **out);
/* Views into a host build (pointers stay valid until gr_host_free). */
gr_status gr_host_csc(const gr_host_graph *h, const uint64_t **off, const uint32_t **src, const uint8_t **w);
gr_status gr_host_csr(const gr_host_graph *h, const uint64_t **off, const uint32_t **dst, const uint8_t **w);
gr_status gr_host_shards(const gr_host_graph *h, uint32_t *num_shards, const uint64_t **bounds);
void gr_host_free(gr_host_graph *h);

#ifdef __cplusplus
}
#endif
#endif /* GRAPHREDUCE_H */
