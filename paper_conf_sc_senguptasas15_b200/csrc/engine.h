// engine.h — internal state of a loaded graph (the opaque gr_graph).
#pragma once
#include <cmath>
#include <cstring>
#include <cstdlib>
#include <cuda_runtime.h>

#include <map>
#include <string>
#include <utility>
#include <vector>

#include "comm.h"
#include "device_common.cuh"
#include "graphreduce.h"
#include "host_graph.h"

struct gr_graph {
  int device = 0;
  int num_sms = 148;
  cudaStream_t stream = nullptr;
  gr::HostGraph H;               // host layout (pinned payloads in streamed mode)
  int mode = GR_MODE_RESIDENT;
  bool off64 = false;
  uint64_t dev_bytes = 0, pinned_bytes = 0;
  std::vector<void *> allocs;

  // topology (device)
  void *in_off = nullptr, *out_off = nullptr;     // OffT arrays
  uint32_t *in_src = nullptr, *out_dst = nullptr; // resident payloads
  uint8_t *in_w = nullptr;
  uint8_t *out_w = nullptr;                       // CSR weights (built on first fused push run)
  uint32_t *nxt[2] = {nullptr, nullptr};          // fused push accumulators (allocated on first use)
  ulonglong2 *prd_div = nullptr;
  uint32_t *estate = nullptr, *out_eid = nullptr; // mutable edge state (kHasScatter programs; first use)
  // dense edge-segmented gather layout (kDstFreeGather programs; built on the first run that may pull)
  uint32_t *ds_src = nullptr, *ds_flags = nullptr, *ds_row = nullptr, *ds_split = nullptr, *ds_act = nullptr;
  uint8_t *ds_w = nullptr;
  void *ds_acc = nullptr;
  uint32_t ds_tiles = 0, ds_nsplit = 0;
  bool ds_tried = false;
  uint4 *rec_in = nullptr, *rec_out = nullptr;  // vertex records (low-degree graphs; first gather-program run)
  bool rec_tried = false;
  bool stamp_direct = false;  // low-degree graph: activation atomics without the filter read (GR_STAMP_DIRECT)
  double ds_long_frac = -1.0;  // share of in-edges in rows longer than one tile (< 0: not computed)                  // tolerance PageRank divisor table (first GR_PAGERANK_DELTA run)
  uint32_t *hub_in = nullptr, *hub_out = nullptr, *static_hubs = nullptr;
  uint32_t n_static_hubs = 0;
  // hub chunk lists (kChunk edges per CTA work item)
  uint32_t *chkA_h[2] = {nullptr, nullptr}, *chkA_c[2] = {nullptr, nullptr};
  uint32_t *chkC_h = nullptr, *chkC_c = nullptr;
  unsigned long long *hub_acc = nullptr;  // 8-byte slots (GatherT of any program)
  uint32_t *hub_done = nullptr;
  uint32_t *cbits[2] = {nullptr, nullptr};  // changed-set bitmaps (pull activation)
  uint32_t *hub_act = nullptr;
  size_t cbits_words = 0;
  uint32_t *static_chk_h = nullptr, *static_chk_c = nullptr;
  uint32_t n_static_chunks = 0, hub_cap = 0;
  bool dev_built = false;        // layout built on the GPU (device_build.cu)
  bool csr_pending = false;      // device build: out_dst not sorted yet (ensure_csr on first need)
  uint32_t csr_bits = 32;
  uint64_t dev_hubs_in = 0, dev_chunks_in = 0, dev_hubs_out = 0, dev_chunks_out = 0;

  // frontier-program state
  uint32_t *val = nullptr, *stamp = nullptr;
  uint32_t *listA[2] = {nullptr, nullptr}, *listH[2] = {nullptr, nullptr};
  uint32_t *C_v = nullptr, *C_val = nullptr, *CH_v = nullptr, *CH_val = nullptr;
  gr::Ctl *ctl = nullptr;
  gr::Ctl *h_ctl = nullptr;      // pinned mirror
  unsigned long long *trace = nullptr;
  uint32_t trace_cap = 0;
  int grid_frontier = 0;
  bool coop = false;             // cooperative launch available (persistent loop)

  // PageRank state
  uint32_t *d_outdeg = nullptr;
  float *inv_outdeg = nullptr, *contrib[2] = {nullptr, nullptr}, *rank = nullptr;
  uint32_t *carry_row = nullptr, *head_row = nullptr;
  float *carry_val = nullptr, *head_val = nullptr;
  uint32_t pr_tiles = 0;
  uint32_t *tile_row = nullptr;  // merge-path tile starts (resident: [pr_tiles+1]; streamed: per shard)
  uint32_t pr_wtiles = 0;          // warp-granular tiles (kWTile items)
  uint32_t *wtile_row = nullptr;
  int pr_kernel = -1;              // 0 block, 2 warp, 3 warp+hot, 4 warp range, 5 warp range+hot, 6 pipe, 7 seg
  uint8_t *w_is_long = nullptr;    // warp tiles whose head row began > kShortChain tiles earlier
  uint32_t *long_c = nullptr, *long_f = nullptr, n_long = 0;
  int hot_cta = 1024;
  cudaGraphExec_t pr_exec = nullptr;
  uint32_t pr_exec_iters = 0;
  float pr_exec_d = 0.f;
  int pr_exec_prof = -1;
  uint32_t pr_trace_iters = 0;
  // PageRank hot-source path (resident, single rank): shared-memory table of the
  // kHotK highest-out-degree sources, tagged payload pr_src
  int pr_hot = -1;                 // -1 not set up, 0 disabled, 1 enabled
  uint32_t *pr_src = nullptr, *hot_ids = nullptr;
  float *hot_contrib = nullptr;
  uint32_t hot_k = 0, hot_grid = 0;
  size_t hot_smem = 0;
  size_t loop_smem = 0;     // k_pr_seg_loop: hot_smem + (pr_tma) the per-warp TMA staging buffers
  uint32_t tma_off = 0;     // byte offset of that staging in the loop's dynamic shared memory
  bool pr_tma = false;      // item / head-bit streams by TMA bulk copies (GR_PR_TMA)
  // edge-segmented PageRank layout (pr_kernel 7, kernels_pr.cuh k_pr_seg)
  uint32_t *seg_src = nullptr, *seg_flags = nullptr, *seg_row = nullptr, *seg_off = nullptr;
  uint32_t seg_tiles = 0;
  int seg_var = 0;                 // k_pr_seg variant bits (kernels_pr.cuh)
  int pr_loop = 0;                 // 1: all supersteps in one cooperative k_pr_seg_loop launch
  uint32_t *hot_slot = nullptr, *pr_bar = nullptr;
  uint8_t *hot_split = nullptr;
  float *hot_buf[2] = {nullptr, nullptr};
  // source-blocked PageRank layout (pr_kernel 8, k_pr_bseg_loop)
  uint32_t *b_items = nullptr, *b_flags = nullptr, *b_tile_run = nullptr, *b_run_row = nullptr, *b_blk_tile = nullptr;
  float *b_acc = nullptr;
  uint32_t b_nblk = 0, b_nruns = 0, b_tiles = 0, b_S = 0;
  int b_pol = 1;
  uint64_t seg_items = 0;

  // run bookkeeping
  int last_algo = -1;
  uint32_t last_iters = 0;
  uint32_t epoch_next = 1;
  uint64_t trace_rows = 0;
  // detail columns of the trace (gr_run_opts.trace_detail): (active_shards, S_t) per superstep
  unsigned long long *trace_det = nullptr;  // device [2 * trace_cap]
  uint32_t *det_src_bits = nullptr, *det_shard_bits = nullptr;
  uint64_t *d_shard_bounds = nullptr;
  bool last_detail = false;
  std::map<int, std::pair<cudaGraphExec_t, uint64_t>> while_exec;
  cudaEvent_t ev_start = nullptr, ev_stop = nullptr;
  std::vector<cudaEvent_t> prof_ev;

  // streamed mode (stream.cu)
  void *streamer = nullptr;

  // partitioned (multi-GPU / simulated ranks) mode (engine_part.cu)
  gr::Comm *comm = nullptr;
  bool sim = false;
  uint32_t *X_v = nullptr, *X_val = nullptr;  // exchanged changed set
  float *rank_all = nullptr;                  // PageRank fetch assembly
  uint64_t *x_cnt = nullptr;                  // per-superstep (|C_t|, |A_t|) for the count exchange
  // fused frontier exchange: own buffers by parity and every rank's (peer-mapped)
  uint32_t *fx_own_v[2] = {}, *fx_own_val[2] = {};
  uint32_t *fx_v[2][16] = {}, *fx_val[2][16] = {};
  bool fx_ok = false;
  // device-side count exchange of the fused frontier exchange (engine_part.cu): this
  // rank's XCount (cudaMalloc, mapped into every peer), the peers' mappings, and
  // this rank's per-superstep decision (XDev)
  void *xc_own = nullptr, *xc_peer[16] = {}, *xdev = nullptr;
  void **d_xc_peer = nullptr;                 // device copy of xc_peer (the publish kernel's targets)
  unsigned long long *h_xbytes = nullptr;     // pinned: XDev::bytes_in read back without a pageable copy
  bool xc_ok = false;
  // PageRank fused exchange: every other rank's contribution replica (by parity),
  // peer-mapped (cudaIpc, NCCL mode) or same-device (simulated ranks)
  float *pr_peer[2][15] = {};
  uint32_t pr_npeer = 0;
  bool pr_p2p = false;          // the mapping exists (set up at load)
  bool pr_p2p_on = false;       // this run exchanges by peer stores (else NCCL allgatherv)
  // device-side barrier between partitioned supersteps (engine_part.cu k_xbar): every
  // rank's arrival words (cudaMalloc, mapped into every peer) and a sequence counter
  uint32_t *xbar_own = nullptr, *xbar_peer[16] = {}, **d_xbar_peer = nullptr;
  uint32_t xbar_seq = 0;
  bool xbar_ok = false;
  std::vector<void *> plain_allocs;  // cudaMalloc'ed (IPC-exportable) buffers
};

namespace gr {
// --------------------------------------------------------------- Part views
template <class OffT> inline Part<OffT> make_part(gr_graph *g) {
  Part<OffT> P{};
  P.n = (uint32_t)g->H.n;
  P.own_lo = (uint32_t)g->H.own_lo;
  P.own_n = (uint32_t)g->H.own_n();
  P.in_off = (const OffT *)g->in_off;
  P.in_src = g->in_src;
  P.in_w = g->in_w;
  P.prd_div = g->prd_div;
  P.estate = g->estate;
  P.out_eid = g->out_eid;
  P.ds_src = g->ds_src;
  P.ds_w = g->ds_w;
  P.ds_flags = g->ds_flags;
  P.ds_row = g->ds_row;
  P.ds_split = g->ds_split;
  P.ds_acc = g->ds_acc;
  P.ds_act = g->ds_act;
  P.ds_tiles = g->ds_tiles;
  P.ds_nsplit = g->ds_nsplit;
  P.rec_in = g->rec_in;
  P.rec_out = g->rec_out;
  P.stamp_direct = g->stamp_direct ? 1u : 0u;
  P.nxt[0] = g->nxt[0];
  P.nxt[1] = g->nxt[1];
  P.out_w = g->out_w;
  P.out_off = (const OffT *)g->out_off;
  P.out_dst = g->out_dst;
  P.hub_in = g->hub_in;
  P.hub_out = g->hub_out;
  P.val = g->val;
  P.stamp = g->stamp;
  for (int i = 0; i < 2; i++) { P.listA[i] = g->listA[i]; P.listH[i] = g->listH[i]; }
  P.C_v = g->C_v; P.C_val = g->C_val; P.CH_v = g->CH_v; P.CH_val = g->CH_val;
  for (int i = 0; i < 2; i++) { P.chkA_h[i] = g->chkA_h[i]; P.chkA_c[i] = g->chkA_c[i]; }
  P.chkC_h = g->chkC_h; P.chkC_c = g->chkC_c;
  P.hub_acc = g->hub_acc; P.hub_done = g->hub_done;
  P.outdeg = g->d_outdeg;
  P.cbits[0] = g->cbits[0]; P.cbits[1] = g->cbits[1];
  P.hub_act = g->hub_act;
  P.s_hubs = g->static_hubs; P.s_chk_h = g->static_chk_h; P.s_chk_c = g->static_chk_c;
  P.n_s_hubs = g->n_static_hubs; P.n_s_chunks = g->n_static_chunks;
  P.ctl = g->ctl;
  P.trace = g->trace;
  return P;
}

// ProgPRDelta constants (gr/program.cuh), from the fp32 options
inline void prd_setup(Ctl &h, const gr_run_opts *o, uint64_t n) {
  const unsigned long long dq = (unsigned long long)llround((double)o->damping * 1048576.0);
  h.prd_dq = dq;
  h.prd_base = (((1ull << 20) - dq) << 42) / n;
  h.prd_thr = (double)o->tolerance / (double)n;
  const float r0 = (float)((double)((1ull << 62) / n) * 0x1p-62);
  std::memcpy(&h.prd_r0, &r0, 4);
}

gr_status fail(gr_status s, const char *fmt, ...);
// GR_TIMING=1: host wall-clock marks of the load/run phases on stderr
void tmark(const char *what);
const char *last_error();
void clear_error();
gr_status dev_alloc(gr_graph *g, void **p, size_t bytes);
// Stream-ordered allocations from the device's default memory pool. The pool
// keeps freed memory (release threshold = max), so a reload or a temporary
// buffer costs no cudaMalloc/cudaFree (each of which synchronises the device).
void pool_init(int device);
template <class T> inline cudaError_t pmalloc(T **p, size_t bytes, cudaStream_t s) {
  return cudaMallocAsync((void **)p, bytes ? bytes : 16, s);
}
inline void pfree(void *p, cudaStream_t s) {
  if (p) cudaFreeAsync(p, s);
}
gr_status load_device(gr_graph *g);
gr_status device_build(gr_graph *g, const gr_edges *E, uint64_t shard_edges);
gr_status ensure_csr(gr_graph *g);  // device-built graphs: the activation CSR payload, built lazily
gr_status select_hot(gr_graph *g, uint64_t K, uint32_t **hot_ids, uint32_t *hot_k, uint32_t **d_slot);
// partitioned PageRank (engine.cu): kernel/layout selection once per graph, one superstep's launches
gr_status pr_part_prepare(gr_graph *g);
// mutable edge state (kHasScatter programs): CSR->CSC position map, state array, CSR weights
gr_status scatter_setup(gr_graph *g, bool weights);
uint32_t pr_part_iter(gr_graph *g, cudaStream_t s, uint32_t t, uint32_t iters, float d);
gr_status run(gr_graph *g, const gr_run_opts *o, gr_run_stats *st);
gr_status fetch_values(gr_graph *g, void *dst, uint64_t bytes);
gr_status fetch_trace(gr_graph *g, uint64_t *dst, uint64_t max_rows, uint64_t *rows);
gr_status fetch_trace_detail(gr_graph *g, uint64_t *dst, uint64_t max_rows, uint64_t *rows);
void destroy(gr_graph *g);
bool acquire_handles(gr_graph *g);  // stream, events, pinned Ctl (cached per device)
// streamed mode
gr_status stream_setup(gr_graph *g, uint64_t budget);
gr_status run_streamed(gr_graph *g, const gr_run_opts *o, gr_run_stats *st);
void stream_destroy(gr_graph *g);
uint64_t resident_bytes_estimate(const HostGraph &H);
uint64_t static_bytes_estimate(const HostGraph &H);
// partitioned mode
gr_status part_setup(gr_graph *g);
gr_status run_part(gr_graph *g, const gr_run_opts *o, cudaStream_t s, gr_run_stats *st);
gr_status part_fetch_values(gr_graph *g, void *dst, uint64_t bytes);
gr_status part_fetch_trace(gr_graph *g, uint64_t *dst, uint64_t max_rows, uint64_t *rows);
}  // namespace gr
