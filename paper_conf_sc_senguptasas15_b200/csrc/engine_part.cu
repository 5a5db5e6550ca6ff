// engine_part.cu — partitioned (multi-GPU) superstep drivers. SURVEY §8(e).
//
// Rank g owns destinations [own_lo, own_hi) (gr_plan_intervals over in+out
// degree, identical on every rank), their CSC, and an activation CSR holding
// the same edges grouped by source — so FrontierActivate targets only owned
// vertices and no frontier OR-reduction is needed. Vertex values are
// replicated. One exchange per superstep:
//   frontier programs: allgatherv of the changed set (vertex, new value), then
//     every rank commits all of it to its replica and activates its owned
//     out-neighbours;
//   PageRank: allgatherv of the owned contribution slices.
// The loop is host-driven (termination needs the GLOBAL |A_{t+1}|).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <string>
#include <vector>

#include "comm.h"
#include "engine.h"
#include "kernels_frontier.cuh"
#include "kernels_pr.cuh"
#include "prog_desc.h"

namespace gr {

#define PCK(call)                                                                              \
  do {                                                                                         \
    cudaError_t e_ = (call);                                                                   \
    if (e_ != cudaSuccess)                                                                     \
      return fail(e_ == cudaErrorMemoryAllocation ? GR_ENOMEM : GR_ECUDA, "%s: %s (%s:%d)", #call, \
                  cudaGetErrorString(e_), __FILE__, __LINE__);                                 \
  } while (0)
#define XCK(call)                                                      \
  do {                                                                 \
    gr_status s_ = (call);                                             \
    if (s_ != GR_OK) return fail(s_, "exchange failed: %s", #call);    \
  } while (0)

gr_status part_setup(gr_graph *g) {
  gr_status s;
  const uint64_t n = g->H.n;
  if ((s = dev_alloc(g, (void **)&g->X_v, 4 * n)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->X_val, 4 * n)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->rank_all, 4 * n)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->x_cnt, 64)) != GR_OK) return s;
  // frontier exchange buffers by parity (cudaMalloc: exported to the peers), n entries
  // each: rank q's C_t lands at [own_lo_q, own_lo_q + |C_t^q|)
  g->fx_ok = false;
  if (g->comm->world <= 16) {
    bool ok = true;
    for (int b = 0; b < 2 && ok; b++)
      for (uint32_t **arr : {&g->fx_own_v[b], &g->fx_own_val[b]}) {
        if (cudaMalloc((void **)arr, 4 * std::max<uint64_t>(n, 1)) != cudaSuccess) {
          cudaGetLastError();
          return fail(GR_ENOMEM, "frontier exchange buffers");
        }
        g->plain_allocs.push_back(*arr);
        g->dev_bytes += 4 * n;
      }
    for (int b = 0; b < 2 && ok; b++) {
      std::vector<void *> pv, pval;
      gr_status a = g->comm->share_buffer(g->fx_own_v[b], &pv, g->stream);
      gr_status c = a == GR_OK ? g->comm->share_buffer(g->fx_own_val[b], &pval, g->stream) : a;
      if (c == GR_OK) {
        for (int q = 0; q < g->comm->world; q++) {
          g->fx_v[b][q] = static_cast<uint32_t *>(pv[q]);
          g->fx_val[b][q] = static_cast<uint32_t *>(pval[q]);
        }
      } else if (c == GR_EUNSUPPORTED) {
        ok = false;  // agreed by every rank: the allgatherv exchange stays
      } else {
        return fail(c, "frontier exchange buffer mapping failed");
      }
    }
    g->fx_ok = ok;
    // device-side count exchange (same agreed mapping protocol): every rank's
    // (|C_t|, |A_t|) lands in every peer's XCount, flagged by a sequence number
    g->xc_ok = false;
    if (ok) {
      if (cudaMalloc(&g->xc_own, sizeof(XCount)) != cudaSuccess || cudaMemset(g->xc_own, 0, sizeof(XCount)) != cudaSuccess) {
        cudaGetLastError();
        return fail(GR_ENOMEM, "count exchange buffer");
      }
      g->plain_allocs.push_back(g->xc_own);
      gr_status a = dev_alloc(g, &g->xdev, sizeof(XDev));
      if (a != GR_OK) return a;
      XDev x0{};
      for (int q = 0; q < g->comm->world; q++) x0.R.off[q] = (uint32_t)g->H.owners[q];
      x0.R.nr = (uint32_t)g->comm->world;
      if (cudaMemcpy(g->xdev, &x0, sizeof x0, cudaMemcpyHostToDevice) != cudaSuccess)
        return fail(GR_ECUDA, "count exchange init");
      std::vector<void *> pc;
      gr_status c = g->comm->share_buffer(g->xc_own, &pc, g->stream);
      if (c == GR_OK) {
        for (int q = 0; q < g->comm->world; q++) g->xc_peer[q] = pc[q];
        // no pageable copies in the superstep loop: a pageable transfer can wait on the
        // device, where a peer's wait kernel may be spinning on this rank's next publish
        if ((a = dev_alloc(g, (void **)&g->d_xc_peer, sizeof(void *) * 16)) != GR_OK) return a;
        if (cudaMemcpy(g->d_xc_peer, g->xc_peer, sizeof(void *) * 16, cudaMemcpyHostToDevice) != cudaSuccess ||
            cudaMallocHost((void **)&g->h_xbytes, 32) != cudaSuccess)
          return fail(GR_ECUDA, "count exchange setup");
        g->xc_ok = true;
      } else if (c != GR_EUNSUPPORTED) {
        return fail(c, "count exchange mapping failed");
      }
    }
  }
  // device-side superstep barrier (k_xbar): arrival words mapped into every peer
  g->xbar_ok = false;
  if (g->comm->world <= 16) {
    if (cudaMalloc((void **)&g->xbar_own, 64) != cudaSuccess || cudaMemset(g->xbar_own, 0, 64) != cudaSuccess) {
      cudaGetLastError();
      return fail(GR_ENOMEM, "barrier words");
    }
    g->plain_allocs.push_back(g->xbar_own);
    std::vector<void *> pb;
    gr_status c = g->comm->share_buffer(g->xbar_own, &pb, g->stream);
    if (c == GR_OK) {
      gr_status a = dev_alloc(g, (void **)&g->d_xbar_peer, sizeof(void *) * 16);
      if (a != GR_OK) return a;
      for (int q = 0; q < g->comm->world; q++) g->xbar_peer[q] = static_cast<uint32_t *>(pb[q]);
      if (cudaMemcpy(g->d_xbar_peer, g->xbar_peer, sizeof(void *) * 16, cudaMemcpyHostToDevice) != cudaSuccess)
        return fail(GR_ECUDA, "barrier words");
      g->xbar_ok = true;
    } else if (c != GR_EUNSUPPORTED) {
      return fail(c, "barrier word mapping failed");
    }
  }
  // PageRank fused exchange: map every peer's contribution replicas (both
  // parities). Without a mapping (no peer access) PageRank exchanges with NCCL.
  Comm *C = g->comm;
  g->pr_p2p = false;
  g->pr_npeer = 0;
  if (C->world - 1 <= 15 && g->contrib[0] && g->contrib[1]) {
    std::vector<void *> p0, p1;
    // both calls are collective and agree on every rank (comm.h)
    gr_status a = C->share_buffer(g->contrib[0], &p0, g->stream);
    gr_status b = a == GR_OK ? C->share_buffer(g->contrib[1], &p1, g->stream) : a;
    if (b == GR_OK) {
      for (int q = 0; q < C->world; q++) {
        if (q == C->rank) continue;
        g->pr_peer[0][g->pr_npeer] = static_cast<float *>(p0[q]);
        g->pr_peer[1][g->pr_npeer] = static_cast<float *>(p1[q]);
        g->pr_npeer++;
      }
      g->pr_p2p = true;
    } else if (b == GR_EUNSUPPORTED) {
      g->pr_npeer = 0;  // no peer mapping on some rank: every rank exchanges with NCCL
    } else {
      return fail(b, "PageRank replica mapping: exchange failed");
    }
  }
  return GR_OK;
}

static void owner_bytes(const gr_graph *g, uint64_t elem, std::vector<uint64_t> *cnt, std::vector<uint64_t> *dsp) {
  const auto &o = g->H.owners;
  const int W = (int)o.size() - 1;
  cnt->resize(W);
  dsp->resize(W);
  for (int q = 0; q < W; q++) {
    (*cnt)[q] = (o[q + 1] - o[q]) * elem;
    (*dsp)[q] = o[q] * elem;
  }
}

// sum one u64 over ranks
static gr_status global_sum(Comm *c, uint64_t mine, uint64_t *out, cudaStream_t s) {
  std::vector<uint64_t> all(c->world);
  gr_status st = c->allgather_small(&mine, 1, all.data(), s);
  uint64_t t = 0;
  for (uint64_t v : all) t += v;
  *out = t;
  return st;
}

// (|C_t|, |A_t|) of this rank for the count exchange, read where the kernels left them
static __global__ void k_part_counts(const Ctl *ctl, uint64_t *out) {
  out[0] = ctl->cnt_C;
  out[1] = ctl->cnt_act[ctl->iter & 1u];
}

// ---- device-side count exchange (no host synchronisation per superstep) ----
// After the gather of superstep t, k_part_publish stores this rank's
// (|C_t|, |A_t|) into every rank's XCount (peer mappings: NVLink stores across
// GPUs), then raises the slot's sequence number to seq after a system-scope
// fence. k_part_wait (one warp) waits until every rank's seq for t arrived
// — lane q spins on rank q's slot — and decides on the device what the host
// decided before: the rank regions of the fused exchange buffers (XRanges), the
// global |C_t|, and termination (no active vertex on any rank: ctl->stop, the
// same superstep on every rank since every rank sees the same counts). Slots
// are double-buffered by parity: a rank publishes t + 2 only after its wait of
// t + 1, which needs every peer's publish of t + 1, issued after that peer's
// classify of t — so no slot is overwritten while a peer still reads it.
// seq: a number unique to superstep t of this run on every rank (epoch_base + t + 1:
// epochs only grow across runs and advance identically on every rank)
static __global__ void k_part_publish(Ctl *ctl, XCount *const *peers, uint32_t rank, uint32_t world, uint32_t t,
                                      uint32_t seq) {
  const uint32_t q = threadIdx.x;
  if (q >= world || ctl->stop) return;
  const uint32_t par = t & 1u;
  XCount *X = peers[q];
  X->cnt[par][rank][0] = ctl->cnt_C;
  X->cnt[par][rank][1] = ctl->cnt_act[ctl->iter & 1u];
  __threadfence_system();
  *(volatile uint32_t *)&X->seq[par][rank] = seq;
}

constexpr unsigned long long kSpinLimitNs = 60ull * 1000000000ull;  // 60 s without a peer's count
static __global__ void k_part_wait(Ctl *ctl, XCount *mine, XDev *xd, uint32_t rank, uint32_t world, uint32_t t,
                                   uint32_t seq) {
  const uint32_t q = threadIdx.x, par = t & 1u;
  if (ctl->stop) return;  // uniform: every lane reads the same flag
  unsigned long long c = 0, a = 0;
  if (q < world) {
    // a peer that never publishes (it failed, or its process died) must not hang this
    // GPU: after kSpinLimitNs the run stops with XDev::timeout set (the host reports it)
    const unsigned long long t0 = gtimer();
    while (*(volatile uint32_t *)&mine->seq[par][q] != seq) {
      __nanosleep(64);
      if (gtimer() - t0 > kSpinLimitNs) {
        atomicExch(&xd->timeout, ((unsigned long long)q << 32) | seq);
        break;
      }
    }
    __threadfence_system();
    c = *(volatile unsigned long long *)&mine->cnt[par][q][0];
    a = *(volatile unsigned long long *)&mine->cnt[par][q][1];
  }
  // exclusive prefix of |C_q| over ranks (world <= 16 lanes)
  unsigned long long pre = c;
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long y = __shfl_up_sync(0xffffffffu, pre, o);
    if ((int)q >= o) pre += y;
  }
  const unsigned long long tot = __shfl_sync(0xffffffffu, pre, 31);
  unsigned long long act = a;
  for (int o = 16; o > 0; o >>= 1) act += __shfl_xor_sync(0xffffffffu, act, o);
  unsigned long long peer_c = (q < world && q != rank) ? c : 0ull;
  for (int o = 16; o > 0; o >>= 1) peer_c += __shfl_xor_sync(0xffffffffu, peer_c, o);
  if (q < world) xd->R.pre[q] = (uint32_t)(pre - c);  // R.off / R.nr: set at load (owner starts)
  if (q == 0) {
    xd->R.pre[world] = (uint32_t)tot;
    xd->tot = (uint32_t)tot;
    xd->bytes_in += 8ull * peer_c;
    ctl->cnt_C = 0;  // this rank's C list is refilled from the exchanged set by the classify
    if (act == 0 || xd->timeout) ctl->stop = 1u;
  }
}

// Stream-ordered barrier across ranks on the device (no host, no NCCL call):
// lane q stores seq into rank q's arrival word of this rank after a
// system-scope fence (so this rank's earlier kernels' stores, the fused peer
// stores included, are visible first), then waits until rank q's seq arrived
// in this rank's words. seq grows by one per barrier, identically on every rank.
static __global__ void k_xbar(uint32_t *const *peers, uint32_t *mine, uint32_t rank, uint32_t world, uint32_t seq) {
  const uint32_t q = threadIdx.x;
  __threadfence_system();
  if (q < world) *(volatile uint32_t *)(peers[q] + rank) = seq;
  if (q < world) {
    const unsigned long long t0 = gtimer();
    while (*(volatile uint32_t *)(mine + q) < seq && gtimer() - t0 < kSpinLimitNs) __nanosleep(32);
  }
  __threadfence_system();
  __syncwarp();
}

// k_classify with the exchanged set's size and rank regions read from the device
template <class OffT>
__global__ void __launch_bounds__(kBlock) k_classify_dev(const __grid_constant__ Part<OffT> P, const uint32_t *X_v,
                                                         const uint32_t *X_val, const XDev *xd) {
  __shared__ uint32_t sq[kWarpsPerBlock][2][kQueueCap];
  __shared__ uint32_t s_off[kWarpsPerBlock + 1];
  __shared__ XRanges R;
  __shared__ uint32_t s_nx, s_stop;
  if (threadIdx.x == 0) {
    s_stop = *(volatile uint32_t *)&P.ctl->stop;
    s_nx = xd->tot;
    R = xd->R;
  }
  __syncthreads();
  if (s_stop) return;
  const uint32_t nX = s_nx;
  const uint32_t warp = threadIdx.x / 32, lane = lane_id();
  WarpQueue qC{sq[warp][0], sq[warp][1], 0};
  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = gw * 32u; base < nX; base += nw * 32u) {
    const uint32_t i = base + lane;
    const bool valid = i < nX;
    uint32_t at = i;
    if (valid) {
      uint32_t q = 0;
      while (q + 1 < R.nr && R.pre[q + 1] <= i) q++;
      at = R.off[q] + (i - R.pre[q]);
    }
    const uint32_t u = valid ? X_v[at] : 0u, val = valid ? X_val[at] : 0u;
    const bool hub = valid && test_bit(P.hub_out, u);
    if (hub) append_hub_C(P, u, val);
    qC.push(valid && !hub, u, val, P.C_v, P.C_val, &P.ctl->cnt_C);
  }
  qC.block_flush(P.C_v, P.C_val, &P.ctl->cnt_C, s_off);
}

// D: the program's traits and kernels (prog_desc.h) — built-in or run-time compiled
template <class OffT>
gr_status run_frontier_part(gr_graph *g, const gr_run_opts *o, cudaStream_t s, gr_run_stats *st,
                            const ProgDesc &D) {
  constexpr int K = sizeof(OffT) == 8 ? 1 : 0;
#define KL(fn, grid, block, ...)                                   \
  do {                                                             \
    void *a_[] = {__VA_ARGS__};                                    \
    gr_status r_ = klaunch(D, fn, (grid), (block), a_, s);         \
    if (r_ != GR_OK) return r_;                                    \
  } while (0)
  Comm *C = g->comm;
  const bool kScatter = D.scatter;
  if (kScatter) {  // this rank's edges (its CSC and activation CSR) carry the states
    gr_status ss = scatter_setup(g, D.uses_weights);
    if (ss != GR_OK) return ss;
  }
  Part<OffT> P = make_part<OffT>(g);
  uint64_t launches = 0;
  if (g->epoch_next > 0xF0000000u) {
    PCK(cudaMemsetAsync(g->stamp, 0, 4ull * std::max<uint64_t>(g->H.own_n(), 1), s));
    if (g->xc_own) PCK(cudaMemsetAsync(g->xc_own, 0, sizeof(XCount), s));  // sequence numbers restart too
    g->epoch_next = 1;
  }
  Ctl h{};
  h.epoch_base = g->epoch_next;
  h.max_iters = o->max_iters;
  h.trace_cap = g->trace_cap;
  h.source = o->source;
  h.damping = o->damping;
  h.ext_loop = 1;
  h.no_hub_c = 1;
  prd_setup(h, o, g->H.n);
  h.kstart[0] = h.kstart[1] = ~0ull;
  *g->h_ctl = h;  // pinned staging (no pageable transfer while peers' kernels may spin)
  PCK(cudaMemcpyAsync(g->ctl, g->h_ctl, sizeof h, cudaMemcpyHostToDevice, s));
  uint32_t src0 = o->source;
  KL(D.init_values[K], g->num_sms * 4, 256, &P, &src0);
  if (kScatter) {
    uint64_t m_in = g->H.m_in;
    KL(D.init_edges[K], g->num_sms * 8, 256, &P, &m_in);
  }
  {
    void *acc = g->hub_acc;
    unsigned long long cnt = g->hub_cap;
    KL(D.fill, std::min<uint32_t>((g->hub_cap + 255) / 256, 1024) + 1, 256, &acc, &cnt);
  }
  PCK(cudaMemsetAsync(g->hub_done, 0, 4ull * g->hub_cap, s));
  if (D.init == kInitAll && g->n_static_hubs) {
    PCK(cudaMemcpyAsync(g->listH[0], g->static_hubs, 4ull * g->n_static_hubs, cudaMemcpyDeviceToDevice, s));
    PCK(cudaMemcpyAsync(g->chkA_h[0], g->static_chk_h, 4ull * g->n_static_chunks, cudaMemcpyDeviceToDevice, s));
    PCK(cudaMemcpyAsync(g->chkA_c[0], g->static_chk_c, 4ull * g->n_static_chunks, cudaMemcpyDeviceToDevice, s));
  }
  // BFS runs unfused here (apply, exchange, activate), so its A lists are built
  // by the generic activation (hub chunks by in-degree).
  {
    uint32_t nh = (uint32_t)g->n_static_hubs, nc = (uint32_t)g->n_static_chunks;
    KL(D.init_frontier[K], 1, kBlock, &P, &src0, &nh, &nc);
  }
  launches += 3;
  PCK(cudaGetLastError());
  PCK(cudaMemsetAsync(&g->ctl->stop, 0, sizeof(uint32_t), s));  // the host decides termination
  uint32_t t = 0;
  std::vector<uint64_t> cnt(C->world), dsp(C->world), all(2 * C->world);
  const uint32_t grid = g->grid_frontier;
  // One host synchronisation per superstep: after the gather, every rank's
  // (|C_t|, |A_t|) pair is allgathered straight from device memory; it sizes
  // the exchange of C_t and decides termination (no active vertex on any rank:
  // the gather of an empty frontier changed nothing and the run ends at t).
  // Fused exchange (default when every rank mapped every peer's exchange buffers):
  // the gather's C_t appends also land in each rank's buffer of this parity at
  // own_lo + position, so after the count exchange every rank already holds
  // all of C_t — no allgatherv. Parity double buffering: a rank may start the
  // gather of t+1 while a peer still classifies t.
  bool fx = g->fx_ok;
  if (const char *e = getenv("GR_FRONTIER_EXCHANGE")) fx = fx && std::string(e) != "nccl";
  // device-side count exchange (default with the fused exchange): no host
  // synchronisation per superstep; the host enqueues supersteps in batches and
  // reads the stop flag the wait kernels set once per batch
  bool dx = fx && g->xc_ok && C->own_context();
  if (const char *e = getenv("GR_COUNT_EXCHANGE")) dx = dx && std::string(e) != "host";
  if (dx) {
    const uint32_t batch = 8;
    XCount *const *d_peers = reinterpret_cast<XCount *const *>(g->d_xc_peer);
    XDev *xd = static_cast<XDev *>(g->xdev);
    // only pinned / device copies below: a pageable transfer could wait on the device while a
    // peer's wait kernel spins for this rank's next publish
    PCK(cudaMemcpyAsync(g->h_xbytes, &xd->bytes_in, 8, cudaMemcpyDeviceToHost, s));
    // every rank has finished its run setup (allocations, staging copies) before any rank
    // enqueues a wait kernel that spins on its peers: ranks that share a device (simulated,
    // same-GPU processes) must not block in a device-wide synchronisation behind a spinner
    XCK(C->barrier(s));
    P.n_xp = (uint32_t)C->world;
    P.xp_off = (uint32_t)g->H.own_lo;
    for (;;) {
      for (uint32_t b = 0; b < batch && (o->max_iters == 0 || t < o->max_iters); b++, t++) {
        const uint32_t par = t & 1u;
        for (int q = 0; q < C->world; q++) {
          P.xp_v[q] = g->fx_v[par][q];
          P.xp_val[q] = g->fx_val[par][q];
        }
        KL(D.gather_apply_x[K], grid, kBlock, &P);
        const uint32_t seq = h.epoch_base + t + 1;
        k_part_publish<<<1, 32, 0, s>>>(g->ctl, d_peers, (uint32_t)C->rank, (uint32_t)C->world, t, seq);
        k_part_wait<<<1, 32, 0, s>>>(g->ctl, static_cast<XCount *>(g->xc_own), xd, (uint32_t)C->rank,
                                     (uint32_t)C->world, t, seq);
        Part<OffT> Pc = P;
        Pc.n_xp = 0;
        k_classify_dev<OffT><<<grid, kBlock, 0, s>>>(Pc, g->fx_v[par][C->rank], g->fx_val[par][C->rank], xd);
        if (kScatter) {
          k_commit_only<OffT><<<grid, kBlock, 0, s>>>(Pc);
          unsigned long long cond = 0;
          int ug = 0;
          void *a_[] = {&Pc, &cond, &ug};
          gr_status r_ = klaunch(D, D.scatter_activate[K], grid, kBlock, a_, s);
          if (r_ != GR_OK) return r_;
          launches++;
        } else {
          k_activate<OffT><<<grid, kBlock, 0, s>>>(Pc, 0ull, 0);
        }
        launches += 5;
        PCK(cudaGetLastError());
      }
      PCK(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
      PCK(cudaStreamSynchronize(s));
      if (g->h_ctl->stop || (o->max_iters != 0 && t >= o->max_iters)) break;
    }
    PCK(cudaMemcpyAsync(g->h_xbytes + 1, &xd->bytes_in, 8, cudaMemcpyDeviceToHost, s));
    PCK(cudaMemcpyAsync(g->h_xbytes + 2, &xd->timeout, 8, cudaMemcpyDeviceToHost, s));
    PCK(cudaStreamSynchronize(s));
    C->bytes_in += g->h_xbytes[1] - g->h_xbytes[0];
    if (g->h_xbytes[2]) {
      const unsigned long long tv = g->h_xbytes[2];
      PCK(cudaMemsetAsync(&xd->timeout, 0, 8, s));
      return fail(GR_ENCCL, "count exchange: rank %d waited %llu s for rank %u's counts of superstep seq %u "
                  "(peer failed or stalled)", C->rank, kSpinLimitNs / 1000000000ull, (unsigned)(tv >> 32),
                  (unsigned)tv);
    }
    t = g->h_ctl->iter;  // supersteps that ran (the stopped one, if any, did not count)
  }
  while (!dx && (o->max_iters == 0 || t < o->max_iters)) {
    const uint32_t par = t & 1u;
    if (fx) {
      for (int q = 0; q < C->world; q++) {
        P.xp_v[q] = g->fx_v[par][q];
        P.xp_val[q] = g->fx_val[par][q];
      }
      P.n_xp = (uint32_t)C->world;
      P.xp_off = (uint32_t)g->H.own_lo;
    }
    KL(fx ? D.gather_apply_x[K] : D.gather_apply[K], grid, kBlock, &P);
    P.n_xp = 0;
    k_part_counts<<<1, 1, 0, s>>>(g->ctl, g->x_cnt);
    launches += 2;
    XCK(C->allgather_dev(g->x_cnt, 2, all.data(), s));
    uint64_t tot = 0, active = 0;
    for (int q = 0; q < C->world; q++) {
      cnt[q] = 4 * all[2 * q];
      dsp[q] = 4 * tot;
      tot += all[2 * q];
      active += all[2 * q + 1];
    }
    if (active == 0) break;
    // exchange the changed set C_t (vertex, new value)
    XRanges R{};
    const uint32_t *xv = g->X_v, *xval = g->X_val;
    if (fx) {
      uint32_t acc = 0;
      for (int q = 0; q < C->world; q++) {
        R.off[q] = (uint32_t)g->H.owners[q];
        R.pre[q] = acc;
        acc += (uint32_t)all[2 * q];
        if (q != C->rank) C->bytes_in += 8 * all[2 * q];
      }
      R.pre[C->world] = acc;
      R.nr = (uint32_t)C->world;
      xv = g->fx_v[par][C->rank];
      xval = g->fx_val[par][C->rank];
    } else if (tot) {
      XCK(C->allgatherv(g->C_v, g->X_v, cnt, dsp, s));
      XCK(C->allgatherv(g->C_val, g->X_val, cnt, dsp, s));
    }
    PCK(cudaMemsetAsync(&g->ctl->cnt_C, 0, sizeof(uint32_t), s));
    if (tot) k_classify<OffT><<<std::min<uint32_t>(grid, (uint32_t)((tot + kBlock - 1) / kBlock)), kBlock, 0, s>>>(
        P, xv, xval, (uint32_t)tot, R);
    if (kScatter) {
      // commit every rank's C_t first: scatter reads the committed values of its targets
      k_commit_only<OffT><<<grid, kBlock, 0, s>>>(P);
      unsigned long long cond = 0;
      int ug = 0;
      KL(D.scatter_activate[K], grid, kBlock, &P, &cond, &ug);
      launches++;
    } else {
      k_activate<OffT><<<grid, kBlock, 0, s>>>(P, 0ull, 0);
    }
    launches += tot ? 2 : 1;
    PCK(cudaGetLastError());
    t++;
  }
  PCK(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
  PCK(cudaStreamSynchronize(s));
  const Ctl &c = *g->h_ctl;
  uint64_t v[2] = {c.tot_gathered, c.tot_scattered}, av[64];
  XCK(C->allgather_small(v, 2, av, s));
  st->iterations = t;
  st->edges_gathered = st->edges_scattered = 0;
  for (int q = 0; q < C->world; q++) {
    st->edges_gathered += av[2 * q];
    st->edges_scattered += av[2 * q + 1];
  }
  st->kernel_launches += launches;
  st->bytes_nvlink = C->bytes_in;
  g->epoch_next = h.epoch_base + t + 2;
  g->trace_rows = std::min<uint64_t>(t, g->trace_cap);
  st->bytes_hbm_model = (D.uses_weights ? 5 : 4) * c.tot_gathered + 4 * c.tot_scattered;
  return GR_OK;
#undef KL
}

// PageRank over owner partitions. Each rank runs the single-GPU superstep
// kernels (hot-source table + edge-segmented tiles when they apply) over its
// owned rows, reading the full contribution replica. The exchange of the owned
// contribution slices is FUSED into the apply (default): every contribution is
// stored into the local replica and, through the peer mappings, into every
// other rank's replica for superstep t+1, so the slices travel over NVLink
// while the rest of the gather runs; a stream-ordered barrier (one-word NCCL
// allreduce) then orders superstep t+1 after every rank's stores.
// GR_PR_EXCHANGE=nccl (or no peer mapping): allgatherv of the owned slices
// after each superstep instead.
template <class OffT>
gr_status run_pagerank_part(gr_graph *g, const gr_run_opts *o, cudaStream_t s, gr_run_stats *st) {
  Comm *C = g->comm;
  const uint32_t iters = o->max_iters;
  const float d = o->damping;
  const uint32_t lo = (uint32_t)g->H.own_lo;
  std::vector<uint64_t> cnt, dsp;
  owner_bytes(g, 4, &cnt, &dsp);
  gr_status ps = pr_part_prepare(g);
  if (ps != GR_OK) return ps;
  bool p2p = g->pr_p2p;
  if (const char *x = getenv("GR_PR_EXCHANGE")) p2p = p2p && std::string(x) != "nccl";
  g->pr_p2p_on = p2p;
  uint64_t launches = 1;
  k_pr_init<<<g->num_sms * 4, 256, 0, s>>>((uint32_t)g->H.n, g->inv_outdeg, g->contrib[0]);
  // stream-ordered barrier between supersteps: on the device (k_xbar over the
  // mapped arrival words, default) or the communicator's (NCCL allreduce / host)
  bool dbar = g->xbar_ok && C->own_context();
  if (const char *x = getenv("GR_PR_BARRIER")) dbar = dbar && std::string(x) != "comm";
  auto barrier = [&]() -> gr_status {
    if (!dbar) return C->barrier(s);
    k_xbar<<<1, 32, 0, s>>>(g->d_xbar_peer, g->xbar_own, (uint32_t)C->rank, (uint32_t)C->world, ++g->xbar_seq);
    launches++;
    return cudaGetLastError() == cudaSuccess ? GR_OK : GR_ECUDA;
  };
  // every replica is initialised before any rank's first fused store lands in it
  if (p2p) XCK(barrier());
  for (uint32_t t = 0; t < iters; t++) {
    launches += pr_part_iter(g, s, t, iters, d);
    PCK(cudaGetLastError());
    if (t + 1 == iters) break;
    if (p2p) {
      XCK(barrier());
      C->bytes_in += 4 * (g->H.n - g->H.own_n());
    } else {
      float *out = g->contrib[(t + 1) & 1];
      XCK(C->allgatherv(out + lo, out, cnt, dsp, s));  // owned slices -> every replica
    }
  }
  g->pr_p2p_on = false;
  PCK(cudaStreamSynchronize(s));
  st->iterations = iters;
  uint64_t mi = g->H.m_in, tot = 0;
  XCK(global_sum(C, mi, &tot, s));
  st->edges_gathered = (uint64_t)iters * tot;
  st->kernel_launches += launches;
  st->bytes_nvlink = C->bytes_in;
  st->bytes_hbm_model = (uint64_t)iters * (4 * g->H.m_in + 12 * g->H.own_n() + 4 * g->H.n);
  g->trace_rows = iters;
  return GR_OK;
}

// Collective fetches for partitioned graphs.
gr_status part_fetch_values(gr_graph *g, void *dst, uint64_t bytes) {
  const uint64_t n = g->H.n;
  if (g->last_algo == GR_PAGERANK) {
    std::vector<uint64_t> cnt, dsp;
    owner_bytes(g, 4, &cnt, &dsp);
    XCK(g->comm->allgatherv(g->rank, g->rank_all, cnt, dsp, g->stream));
    PCK(cudaStreamSynchronize(g->stream));
    PCK(cudaMemcpyAsync(dst, g->rank_all, 4 * n, cudaMemcpyDeviceToHost, g->stream));
    PCK(cudaStreamSynchronize(g->stream));
  } else {
    PCK(cudaMemcpyAsync(dst, g->val, 4 * n, cudaMemcpyDeviceToHost, g->stream));
    PCK(cudaStreamSynchronize(g->stream));
  }
  (void)bytes;
  return GR_OK;
}

gr_status part_fetch_trace(gr_graph *g, uint64_t *dst, uint64_t max_rows, uint64_t *rows) {
  Comm *C = g->comm;
  const uint64_t r = std::min<uint64_t>(g->trace_rows, max_rows);
  if (g->last_algo == GR_PAGERANK) {
    uint64_t mi = g->H.m_in, tot = 0;
    XCK(global_sum(C, mi, &tot, g->stream));
    for (uint64_t t = 0; t < r; t++) {
      dst[4 * t] = g->H.n;
      dst[4 * t + 1] = g->H.n;
      dst[4 * t + 2] = tot;
      dst[4 * t + 3] = 0;
    }
    *rows = r;
    return GR_OK;
  }
  std::vector<uint64_t> cnt(C->world, 32 * r), dsp(C->world);
  for (int q = 0; q < C->world; q++) dsp[q] = 32 * r * q;
  // local steps first, then one agreed flag: a rank that failed here must not leave the
  // others waiting in the allgatherv (every rank takes the same collective sequence)
  char *base = nullptr;
  uint64_t ok = cudaMalloc((void **)&base, 32 * std::max<uint64_t>(r, 1) * C->world) == cudaSuccess &&
                cudaStreamSynchronize(g->stream) == cudaSuccess &&  // the trace of the last run is complete
                cudaMemcpyAsync(base + 32 * r * C->rank, g->trace, 32 * r, cudaMemcpyDeviceToDevice,
                                g->stream) == cudaSuccess;
  if (!ok) cudaGetLastError();
  std::vector<uint64_t> oks(C->world);
  XCK(C->allgather_small(&ok, 1, oks.data(), g->stream));
  for (int q = 0; q < C->world; q++)
    if (!oks[q]) {
      if (base) cudaFree(base);
      return fail(GR_ECUDA, "trace exchange: rank %d failed locally", q);
    }
  gr_status xs = C->allgatherv(base + 32 * r * C->rank, base, cnt, dsp, g->stream);
  std::vector<uint64_t> all(4 * r * C->world);
  cudaError_t ce = cudaStreamSynchronize(g->stream);
  if (xs == GR_OK && ce == cudaSuccess && r) {
    ce = cudaMemcpyAsync(all.data(), base, 32 * r * C->world, cudaMemcpyDeviceToHost, g->stream);
    if (ce == cudaSuccess) ce = cudaStreamSynchronize(g->stream);
  }
  cudaFree(base);
  if (xs != GR_OK) return fail(xs, "trace exchange failed");
  if (ce != cudaSuccess) return fail(GR_ECUDA, "trace exchange: %s", cudaGetErrorString(ce));
  for (uint64_t i = 0; i < 4 * r; i++) {
    uint64_t sum = 0;
    for (int q = 0; q < C->world; q++) sum += all[q * 4 * r + i];
    dst[i] = sum;
  }
  *rows = r;
  return GR_OK;
}

gr_status run_part(gr_graph *g, const gr_run_opts *o, cudaStream_t s, gr_run_stats *st) {
  gr_status r;
  if (o->algo == GR_PAGERANK) {
    r = g->off64 ? run_pagerank_part<uint64_t>(g, o, s, st) : run_pagerank_part<uint32_t>(g, o, s, st);
  } else {
    ProgDesc D;
    r = prog_desc(o->algo, o->custom_id, &D);
    if (r == GR_OK)
      r = g->off64 ? run_frontier_part<uint64_t>(g, o, s, st, D) : run_frontier_part<uint32_t>(g, o, s, st, D);
  }
  // a rank that fails mid-run (a launch error, a local allocation) aborts the group, so
  // its peers return errors from their next collective instead of waiting forever
  if (r != GR_OK) g->comm->abort_group();
  return r;
}

}  // namespace gr
