// stream.cu — streamed (out-of-core) mode: the H2D shard streamer.
//
// Data Movement Engine of PAPER.md §4.3 redesigned for one B200: the static
// vertex arrays live in HBM (§3.2); each shard's edge payload (CSC
// sources [+ weights] for gather, CSR destinations for FrontierActivate) stays
// in page-locked host memory and is copied with ONE cudaMemcpyAsync per array
// into one of K = 2 device slots (Eq. (1)-(2), L226-240: K = 2) on a dedicated
// copy stream, so the copy of shard s+1 overlaps the kernels of shard s
// (compute-transfer overlap, §3.3). Shards with no active vertex are not
// copied at all (frontier management, §5.2); BFS moves only out-edges and
// PageRank only in-edges (phase elimination, §5.3). The paper's Hyper-Q
// "spray" of many small copies (§5.1) is not used: a shard is one
// contiguous slice per array, which one DMA moves at full link speed.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "engine.h"
#include "kernels_pr.cuh"
#include "kernels_stream.cuh"
#include "prog_desc.h"

namespace gr {

#define SCK(call)                                                                              \
  do {                                                                                         \
    cudaError_t e_ = (call);                                                                   \
    if (e_ != cudaSuccess)                                                                     \
      return fail(e_ == cudaErrorMemoryAllocation ? GR_ENOMEM : GR_ECUDA, "%s: %s (%s:%d)", #call, \
                  cudaGetErrorString(e_), __FILE__, __LINE__);                                 \
  } while (0)

struct Streamer {
  uint32_t P = 0;
  std::vector<uint64_t> in_b, out_b;  // per-shard edge boundaries (P+1)
  std::vector<uint32_t> tile_base;    // PageRank tile offsets per shard (P+1)
  uint64_t slot_edges = 0;
  uint32_t *slot_idx[2] = {nullptr, nullptr};
  uint8_t *slot_w[2] = {nullptr, nullptr};
  cudaStream_t copy_s = nullptr;
  cudaEvent_t copied[2] = {nullptr, nullptr}, freed[2] = {nullptr, nullptr};
  uint64_t uses = 0;
  uint64_t *d_bounds = nullptr;
  uint8_t *d_next = nullptr, *d_changed = nullptr, *h_flags = nullptr;
  uint32_t *cstamp = nullptr;
  uint32_t *d_list = nullptr;
  uint64_t bytes_h2d = 0;
  // zero-copy views of the pinned payloads (device addresses of the mapped host buffers)
  const uint32_t *zc_in = nullptr, *zc_out = nullptr;
  const uint8_t *zc_w = nullptr;
  uint64_t bytes_zc = 0;
  uint32_t zc_phases = 0;
  // mutable edge state (kHasScatter programs): CSC-ordered states and the CSR -> CSC
  // position map in mapped pinned host memory, read and written in place over the link
  uint32_t *h_es = nullptr, *h_eid = nullptr;
  uint32_t *zc_es = nullptr, *zc_eid = nullptr;
  uint8_t *zc_ow = nullptr;
};

// Edge-state layout of a streamed graph (once): the CSR -> CSC position map by a
// stable bucket pass of the CSC positions over their sources (the host CSR is
// ordered (src, dst, w), the CSC (dst, src, w): bucketing the CSC by source in
// order reproduces the CSR order), the state array, the CSR weights mapped.
static gr_status stream_scatter_setup(gr_graph *g, Streamer *S) {
  HostGraph &H = g->H;
  const uint64_t m = H.m_in;
  if (!S->h_es) {
    if (H.out_off.size() != H.n + 1) return fail(GR_EUNSUPPORTED, "streamed edge state needs the host CSR offsets");
    SCK(cudaHostAlloc((void **)&S->h_es, 4 * std::max<uint64_t>(m, 1), cudaHostAllocMapped));
    SCK(cudaHostAlloc((void **)&S->h_eid, 4 * std::max<uint64_t>(m, 1), cudaHostAllocMapped));
    g->pinned_bytes += 8 * m;
    std::vector<uint64_t> pos(H.out_off.begin(), H.out_off.end() - 1);
    const uint32_t *src = H.in_src.as<uint32_t>();
    for (uint64_t e = 0; e < m; e++) S->h_eid[pos[src[e]]++] = (uint32_t)e;
    void *dp = nullptr;
    SCK(cudaHostGetDevicePointer(&dp, S->h_es, 0));
    S->zc_es = (uint32_t *)dp;
    SCK(cudaHostGetDevicePointer(&dp, S->h_eid, 0));
    S->zc_eid = (uint32_t *)dp;
    if (H.out_w.p && H.out_w.bytes && !H.out_w.registered) {
      cudaError_t e = cudaHostRegister(H.out_w.p, H.out_w.bytes, cudaHostRegisterMapped);
      if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(GR_ENOMEM, "cudaHostRegister(out_w): %s", cudaGetErrorString(e));
      }
      H.out_w.registered = true;
      g->pinned_bytes += H.out_w.bytes;
    }
    if (H.out_w.p && H.out_w.bytes) {
      SCK(cudaHostGetDevicePointer(&dp, H.out_w.p, 0));
      S->zc_ow = (uint8_t *)dp;
    }
  }
  // every Part of this run (make_part) carries the mapped views
  g->estate = S->zc_es;
  g->out_eid = S->zc_eid;
  g->out_w = S->zc_ow;
  return GR_OK;
}

// auto mode: read in place when the frontier's edges are < 1/kZcDiv of the
// edges a whole-shard DMA of the active shards would move
constexpr uint64_t kZcDiv = 8;

static Streamer *S_(gr_graph *g) { return static_cast<Streamer *>(g->streamer); }

gr_status stream_setup(gr_graph *g, uint64_t budget) {
  HostGraph &H = g->H;
  auto *S = new Streamer();
  g->streamer = S;
  S->P = H.num_shards();
  S->in_b.resize(S->P + 1);
  S->out_b.resize(S->P + 1);
  S->tile_base.assign(S->P + 1, 0);
  for (uint32_t s = 0; s <= S->P; s++) {
    S->in_b[s] = H.in_off[H.bounds[s] - H.own_lo];
    S->out_b[s] = H.out_off[H.bounds[s]];
  }
  for (uint32_t s = 0; s < S->P; s++) {
    S->slot_edges = std::max(S->slot_edges, std::max(S->in_b[s + 1] - S->in_b[s], S->out_b[s + 1] - S->out_b[s]));
    const uint64_t items = (H.bounds[s + 1] - H.bounds[s]) + (S->in_b[s + 1] - S->in_b[s]);
    S->tile_base[s + 1] = S->tile_base[s] + (uint32_t)((items + kPrTile - 1) / kPrTile);
  }
  const uint64_t slot_bytes = 5 * S->slot_edges + 64;
  if (g->dev_bytes + 2 * slot_bytes > budget)
    return fail(GR_ENOMEM,
                "streamed mode: static vertex arrays (%llu B) + 2 shard slots (2 x %llu B) exceed the device "
                "budget (%llu B); use smaller shards (shard_edges)",
                (unsigned long long)g->dev_bytes, (unsigned long long)slot_bytes, (unsigned long long)budget);
  // page-lock the host payloads for DMA
  for (HostBuf *b : {&H.in_src, &H.out_dst, &H.in_w}) {
    if (!b->p || !b->bytes) continue;
    if (!b->owned) {  // a borrowed buffer the caller already page-locked (cudaHostAlloc / torch pinned): as is
      cudaPointerAttributes pa{};
      if (cudaPointerGetAttributes(&pa, b->p) == cudaSuccess && pa.type == cudaMemoryTypeHost) {
        g->pinned_bytes += b->bytes;
        void *dp = pa.devicePointer;
        if (!dp && cudaHostGetDevicePointer(&dp, b->p, 0) != cudaSuccess) {
          cudaGetLastError();
          return fail(GR_EUNSUPPORTED, "borrowed pinned buffer is not mapped into the device address space");
        }
        if (b == &H.in_src) S->zc_in = (const uint32_t *)dp;
        else if (b == &H.out_dst) S->zc_out = (const uint32_t *)dp;
        else S->zc_w = (const uint8_t *)dp;
        continue;
      }
      cudaGetLastError();
    }
    cudaError_t e = cudaHostRegister(b->p, b->bytes, cudaHostRegisterMapped);
    if (e == cudaErrorHostMemoryAlreadyRegistered && !b->owned) {
      cudaGetLastError();  // registered by the caller in the meantime: used as it is
    } else if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(GR_ENOMEM, "cudaHostRegister(%zu bytes): %s", b->bytes, cudaGetErrorString(e));
    } else {
      b->registered = true;
    }
    g->pinned_bytes += b->bytes;
    void *dp = nullptr;
    SCK(cudaHostGetDevicePointer(&dp, b->p, 0));
    if (b == &H.in_src) S->zc_in = (const uint32_t *)dp;
    else if (b == &H.out_dst) S->zc_out = (const uint32_t *)dp;
    else S->zc_w = (const uint8_t *)dp;
  }
  gr_status st;
  for (int k = 0; k < 2; k++) {
    if ((st = dev_alloc(g, (void **)&S->slot_idx[k], 4 * S->slot_edges + 16)) != GR_OK) return st;
    if (H.has_w && (st = dev_alloc(g, (void **)&S->slot_w[k], S->slot_edges + 16)) != GR_OK) return st;
    SCK(cudaEventCreateWithFlags(&S->copied[k], cudaEventDisableTiming));
    SCK(cudaEventCreateWithFlags(&S->freed[k], cudaEventDisableTiming));
  }
  SCK(cudaStreamCreateWithFlags(&S->copy_s, cudaStreamNonBlocking));
  if ((st = dev_alloc(g, (void **)&S->d_bounds, 8ull * (S->P + 1))) != GR_OK) return st;
  SCK(cudaMemcpyAsync(S->d_bounds, H.bounds.data(), 8ull * (S->P + 1), cudaMemcpyHostToDevice, g->stream));
  if ((st = dev_alloc(g, (void **)&S->d_next, S->P)) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&S->d_changed, S->P)) != GR_OK) return st;
  SCK(cudaMallocHost((void **)&S->h_flags, 2ull * S->P + 16));
  if ((st = dev_alloc(g, (void **)&S->cstamp, 4ull * std::max<uint64_t>(H.own_n(), 1))) != GR_OK) return st;
  SCK(cudaMemsetAsync(S->cstamp, 0, 4ull * std::max<uint64_t>(H.own_n(), 1), g->stream));
  if ((st = dev_alloc(g, (void **)&S->d_list, 4ull * std::max<uint64_t>(H.own_n(), 1))) != GR_OK) return st;
  // PageRank carries per shard
  if (S->tile_base[S->P] > g->pr_tiles) {
    const size_t tb = 4ull * S->tile_base[S->P];
    if ((st = dev_alloc(g, (void **)&g->carry_row, tb)) != GR_OK) return st;
    if ((st = dev_alloc(g, (void **)&g->carry_val, tb)) != GR_OK) return st;
    if ((st = dev_alloc(g, (void **)&g->head_row, tb)) != GR_OK) return st;
    if ((st = dev_alloc(g, (void **)&g->head_val, tb)) != GR_OK) return st;
  }
  // merge-path tile starts per shard (shard s at tile_base[s] + s, tiles_s + 1 entries)
  if ((st = dev_alloc(g, (void **)&g->tile_row, 4ull * (S->tile_base[S->P] + S->P + 1))) != GR_OK) return st;
  for (uint32_t s = 0; s < S->P; s++) {
    const uint64_t r0 = H.bounds[s] - H.own_lo, rows = H.bounds[s + 1] - H.bounds[s];
    const uint32_t tiles = S->tile_base[s + 1] - S->tile_base[s];
    uint32_t *tr = g->tile_row + S->tile_base[s] + s;
    if (g->off64)
      k_pr_tiles<uint64_t><<<(tiles + 256) / 256, 256, 0, g->stream>>>((const uint64_t *)g->in_off + r0, S->in_b[s],
                                                                        (uint32_t)rows, S->in_b[s + 1] - S->in_b[s],
                                                                        tiles, tr);
    else
      k_pr_tiles<uint32_t><<<(tiles + 256) / 256, 256, 0, g->stream>>>((const uint32_t *)g->in_off + r0, S->in_b[s],
                                                                        (uint32_t)rows, S->in_b[s + 1] - S->in_b[s],
                                                                        tiles, tr);
  }
  SCK(cudaGetLastError());
  SCK(cudaStreamSynchronize(g->stream));
  return GR_OK;
}

void stream_destroy(gr_graph *g) {
  Streamer *S = S_(g);
  if (!S) return;
  for (int k = 0; k < 2; k++) {
    if (S->copied[k]) cudaEventDestroy(S->copied[k]);
    if (S->freed[k]) cudaEventDestroy(S->freed[k]);
  }
  if (S->copy_s) cudaStreamDestroy(S->copy_s);
  if (S->h_flags) cudaFreeHost(S->h_flags);
  if (S->h_es) cudaFreeHost(S->h_es);
  if (S->h_eid) cudaFreeHost(S->h_eid);
  if (g->estate == S->zc_es) g->estate = nullptr;
  if (g->out_eid == S->zc_eid) g->out_eid = nullptr;
  if (g->out_w == S->zc_ow) g->out_w = nullptr;
  delete S;
  g->streamer = nullptr;
}

// Copy one shard payload into the next free slot; the compute stream waits for it.
static gr_status stage(gr_graph *g, Streamer *S, cudaStream_t cs, bool in, uint32_t s, bool with_w, int *slot) {
  const int k = (int)(S->uses++ & 1);
  const HostGraph &H = g->H;
  const uint64_t b = in ? S->in_b[s] : S->out_b[s], e = in ? S->in_b[s + 1] : S->out_b[s + 1];
  SCK(cudaStreamWaitEvent(S->copy_s, S->freed[k], 0));
  const uint32_t *src = (in ? H.in_src : H.out_dst).as<uint32_t>() + b;
  if (e > b) SCK(cudaMemcpyAsync(S->slot_idx[k], src, 4 * (e - b), cudaMemcpyHostToDevice, S->copy_s));
  S->bytes_h2d += 4 * (e - b);
  if (with_w && e > b) {
    SCK(cudaMemcpyAsync(S->slot_w[k], H.in_w.as<uint8_t>() + b, e - b, cudaMemcpyHostToDevice, S->copy_s));
    S->bytes_h2d += e - b;
  }
  SCK(cudaEventRecord(S->copied[k], S->copy_s));
  SCK(cudaStreamWaitEvent(cs, S->copied[k], 0));
  *slot = k;
  return GR_OK;
}

// Zero-copy view: the kernels read the whole pinned payload in place (global edge positions).
template <class OffT> static Part<OffT> zc_part(gr_graph *g, Streamer *S, bool in) {
  Part<OffT> P = make_part<OffT>(g);
  if (in) {
    P.in_src = S->zc_in;
    P.in_w = S->zc_w;
  } else {
    P.out_dst = S->zc_out;
  }
  return P;
}

static bool want_zc(const gr_run_opts *o, uint64_t frontier_edges, uint64_t shard_edges) {
  if (o->zero_copy > 0) return true;
  if (o->zero_copy < 0) return false;
  uint64_t div = kZcDiv;
  if (const char *e = getenv("GR_ZC_DIV")) div = strtoull(e, nullptr, 10);
  return div > 0 && frontier_edges * div < shard_edges;
}

template <class OffT> static Part<OffT> slot_part(gr_graph *g, Streamer *S, int k, bool in, uint32_t s) {
  Part<OffT> P = make_part<OffT>(g);
  const uint64_t b = in ? S->in_b[s] : S->out_b[s];
  // shift the slot so global edge positions index it directly (only [b, e) is touched)
  if (in) {
    P.in_src = reinterpret_cast<const uint32_t *>(reinterpret_cast<uintptr_t>(S->slot_idx[k]) - 4 * b);
    if (S->slot_w[k]) P.in_w = reinterpret_cast<const uint8_t *>(reinterpret_cast<uintptr_t>(S->slot_w[k]) - b);
  } else {
    P.out_dst = reinterpret_cast<const uint32_t *>(reinterpret_cast<uintptr_t>(S->slot_idx[k]) - 4 * b);
  }
  return P;
}

static uint32_t grid_for(gr_graph *g, uint64_t items_per_cta_unit) {
  uint64_t want = (items_per_cta_unit + kBlock - 1) / kBlock;
  return (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(want, (uint64_t)g->grid_frontier));
}

// ------------------------------------------------------------- PageRank
template <class OffT>
static gr_status stream_pagerank(gr_graph *g, const gr_run_opts *o, cudaStream_t cs, gr_run_stats *st) {
  Streamer *S = S_(g);
  const HostGraph &H = g->H;
  const uint32_t iters = o->max_iters;
  const float d = o->damping;
  k_pr_init<<<g->num_sms * 4, 256, 0, cs>>>((uint32_t)H.n, g->inv_outdeg, g->contrib[0]);
  uint64_t launches = 1;
  for (uint32_t t = 0; t < iters; t++) {
    for (uint32_t s = 0; s < S->P; s++) {
      const uint64_t r0 = H.bounds[s] - H.own_lo, rows = H.bounds[s + 1] - H.bounds[s];
      const uint64_t me = S->in_b[s + 1] - S->in_b[s];
      if (rows == 0) continue;
      int k = -1;  // PageRank reads every edge: DMA unless zero-copy is forced
      if (o->zero_copy <= 0) {
        gr_status gs = stage(g, S, cs, true, s, false, &k);
        if (gs != GR_OK) return gs;
      } else {
        S->bytes_zc += 4 * me;
      }
      PrArgs<OffT> a{};
      a.n = (uint32_t)H.n;
      a.own_lo = (uint32_t)H.bounds[s];
      a.own_n = (uint32_t)rows;
      a.m_in = me;
      a.e_base = S->in_b[s];
      a.in_off = (const OffT *)g->in_off + r0;
      a.in_src = k >= 0 ? S->slot_idx[k] : S->zc_in + S->in_b[s];
      a.inv_outdeg = g->inv_outdeg;
      a.contrib_in = g->contrib[t & 1];
      a.contrib_out = g->contrib[(t + 1) & 1];
      a.rank = g->rank + r0;
      const uint32_t tb = S->tile_base[s], tiles = S->tile_base[s + 1] - tb;
      a.carry_row = g->carry_row + tb;
      a.carry_val = g->carry_val + tb;
      a.head_row = g->head_row + tb;
      a.head_val = g->head_val + tb;
      a.tile_row = g->tile_row + tb + s;
      a.base = (1.0f - d) / (float)H.n;
      a.d = d;
      a.last = (t + 1 == iters) ? 1 : 0;
      k_pr_gather_apply<OffT><<<tiles, kPrThreads, 0, cs>>>(a);
      k_pr_fixup<OffT><<<(tiles + 255) / 256, 256, 0, cs>>>(a, tiles);
      if (k >= 0) SCK(cudaEventRecord(S->freed[k], cs));
      launches += 2;
    }
  }
  SCK(cudaGetLastError());
  SCK(cudaStreamSynchronize(cs));
  st->iterations = iters;
  if (o->zero_copy > 0) S->zc_phases += iters;
  st->edges_gathered = (uint64_t)iters * H.m_in;
  st->kernel_launches += launches;
  st->bytes_hbm_model = (uint64_t)iters * (4 * H.m_in + 12 * H.own_n() + 4 * H.n);
  g->trace_rows = iters;
  return GR_OK;
}

// ------------------------------------------------------- frontier programs
// D: the program's traits and kernels (prog_desc.h) — built-in or run-time compiled
template <class OffT>
static gr_status stream_frontier(gr_graph *g, const gr_run_opts *o, cudaStream_t cs, gr_run_stats *st,
                                 const ProgDesc &D) {
  constexpr int K = sizeof(OffT) == 8 ? 1 : 0;
#define KL(fn, grid, block, ...)                                   \
  do {                                                             \
    void *a_[] = {__VA_ARGS__};                                    \
    gr_status r_ = klaunch(D, fn[K], (grid), (block), a_, cs);     \
    if (r_ != GR_OK) return r_;                                    \
  } while (0)
  Streamer *S = S_(g);
  const HostGraph &H = g->H;
  const uint32_t P = S->P;
  const bool kScatter = D.scatter;
  if (kScatter) {
    gr_status ss = stream_scatter_setup(g, S);
    if (ss != GR_OK) return ss;
    if (D.uses_weights && !S->zc_ow) return fail(GR_EINVAL, "the program reads edge weights but the graph has none");
  }
  Part<OffT> P0 = make_part<OffT>(g);
  uint64_t launches = 0;
  if (g->epoch_next > 0xF0000000u) {
    SCK(cudaMemsetAsync(g->stamp, 0, 4ull * std::max<uint64_t>(H.own_n(), 1), cs));
    SCK(cudaMemsetAsync(S->cstamp, 0, 4ull * std::max<uint64_t>(H.own_n(), 1), cs));
    g->epoch_next = 1;
  }
  Ctl h{};
  h.epoch_base = g->epoch_next;
  h.max_iters = o->max_iters;
  h.trace_cap = g->trace_cap;
  h.source = o->source;
  h.damping = o->damping;
  prd_setup(h, o, H.n);
  std::vector<uint8_t> act(P, 0);
  std::vector<uint32_t> a0;
  if (D.init == kInitSourceChanged) {
    // A_0 = out-neighbours of the source, read straight from the pinned host CSR
    for (uint64_t e = H.out_off[o->source]; e < H.out_off[o->source + 1]; e++)
      a0.push_back(H.out_dst.as<uint32_t>()[e]);
    std::sort(a0.begin(), a0.end());
    a0.erase(std::unique(a0.begin(), a0.end()), a0.end());
    h.cnt_act[0] = (uint32_t)a0.size();
    h.stop = a0.empty() ? 1u : 0u;
  }
  SCK(cudaMemcpyAsync(g->ctl, &h, sizeof h, cudaMemcpyHostToDevice, cs));
  uint32_t src0 = o->source;
  KL(D.init_values, g->num_sms * 4, 256, &P0, &src0);
  launches++;
  if (kScatter) {  // states in host memory, written in place; the source scatters at init
    uint64_t m_in = H.m_in;
    KL(D.init_edges, g->num_sms * 8, 256, &P0, &m_in);
    launches++;
    if (D.init == kInitSourceChanged) {
      Part<OffT> Pz = zc_part<OffT>(g, S, false);
      KL(D.s_init_scatter, 1, kBlock, &Pz, &src0);
      launches++;
    }
  }
  auto shard_of_host = [&](uint64_t x) {
    return (uint32_t)(std::upper_bound(H.bounds.begin(), H.bounds.end(), x) - H.bounds.begin() - 1);
  };
  if (D.init == kInitSourceChanged) {
    if (!a0.empty()) {
      SCK(cudaMemcpyAsync(S->d_list, a0.data(), 4 * a0.size(), cudaMemcpyHostToDevice, cs));
      k_s_stamp_list<OffT><<<std::max<uint32_t>(1, (uint32_t)std::min<size_t>(1024, (a0.size() + 255) / 256)), 256, 0,
                             cs>>>(P0, S->d_list, (uint32_t)a0.size());
      launches++;
    }
    for (uint32_t x : a0) act[shard_of_host(x)] = 1;
  } else {
    uint32_t z0 = 0, z1 = 0;
    KL(D.init_frontier, 1, kBlock, &P0, &src0, &z0, &z1);
    launches++;
    if (D.init == kInitAll) std::fill(act.begin(), act.end(), 1);
    else act[shard_of_host(o->source)] = 1;
  }
  SCK(cudaGetLastError());
  SCK(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, cs));
  SCK(cudaStreamSynchronize(cs));
  uint8_t *h_changed = S->h_flags, *h_next = S->h_flags + P;
  const double avg_in = H.own_n() ? (double)H.m_in / (double)H.own_n() : 0.0;
  const double avg_out = H.n ? (double)H.m_in / (double)H.n : 0.0;
  const uint64_t wb = D.uses_weights ? 5 : 4;
  // ablation knob (Fig. 15): GR_STREAM_NO_SKIP=1 moves and scans every shard every superstep
  const bool no_skip = getenv("GR_STREAM_NO_SKIP") && getenv("GR_STREAM_NO_SKIP")[0] == '1';
  if (no_skip) std::fill(act.begin(), act.end(), 1);
  while (!g->h_ctl->stop) {
    const uint64_t g0 = g->h_ctl->tot_gathered, s0 = g->h_ctl->tot_scattered;
    SCK(cudaMemsetAsync(S->d_changed, 0, P, cs));
    // gather phase: whole-shard DMA, or in place when A_t's in-edges are few (f1)
    bool zc_g = false;
    if (D.has_gather) {
      uint64_t shard_e = 0;
      for (uint32_t s = 0; s < P; s++)
        if (act[s] || no_skip) shard_e += S->in_b[s + 1] - S->in_b[s];
      const uint32_t nA = g->h_ctl->iter == 0 && g->h_ctl->implicit0 ? (uint32_t)H.own_n()
                                                                       : g->h_ctl->cnt_act[g->h_ctl->iter & 1u];
      zc_g = want_zc(o, (uint64_t)(nA * avg_in), shard_e);
      if (zc_g) S->zc_phases++;
    }
    Part<OffT> Pz_in = zc_part<OffT>(g, S, true);
    if (zc_g) {  // in place: one launch over every shard (stamps select A_t)
      uint32_t v0 = (uint32_t)H.own_lo, v1 = (uint32_t)H.own_hi, all = kAllShards, np = P;
      KL(D.s_gather_apply, grid_for(g, v1 - v0), kBlock, &Pz_in, &v0, &v1, &all, &S->d_changed, &S->cstamp,
         &S->d_bounds, &np);
      launches++;
    }
    for (uint32_t s = 0; s < P && !zc_g; s++) {
      if (!act[s] && !no_skip) continue;  // frontier skipping: no copy, no launch
      uint32_t v0 = (uint32_t)H.bounds[s], v1 = (uint32_t)H.bounds[s + 1];
      if (D.has_gather) {
        int k = -1;
        if (!zc_g) {
          gr_status gs = stage(g, S, cs, true, s, D.uses_weights, &k);
          if (gs != GR_OK) return gs;
        }
        Part<OffT> Pk = zc_g ? Pz_in : slot_part<OffT>(g, S, k, true, s);
        uint32_t sh = s, np = P;
        KL(D.s_gather_apply, grid_for(g, v1 - v0), kBlock, &Pk, &v0, &v1, &sh, &S->d_changed, &S->cstamp,
           &S->d_bounds, &np);
        if (k >= 0) SCK(cudaEventRecord(S->freed[k], cs));
      } else {
        k_s_bfs_apply<OffT><<<grid_for(g, v1 - v0), kBlock, 0, cs>>>(P0, v0, v1, s, S->d_changed, S->cstamp);
      }
      launches++;
    }
    if (D.has_gather) {
      k_s_commit<OffT><<<g->num_sms * 2, 256, 0, cs>>>(P0);
      launches++;
    }
    SCK(cudaMemcpyAsync(h_changed, S->d_changed, P, cudaMemcpyDeviceToHost, cs));
    SCK(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, cs));
    SCK(cudaMemsetAsync(S->d_next, 0, P, cs));
    SCK(cudaStreamSynchronize(cs));
    // FrontierActivate: the same choice over the changed vertices' out-edges
    uint64_t shard_o = 0;
    for (uint32_t s = 0; s < P; s++)
      if (h_changed[s] || no_skip) shard_o += S->out_b[s + 1] - S->out_b[s];
    const bool zc_a = want_zc(o, (uint64_t)((double)g->h_ctl->changed * avg_out), shard_o);
    if (zc_a && shard_o) S->zc_phases++;
    Part<OffT> Pz_out = zc_part<OffT>(g, S, false);
    if (zc_a && shard_o) {  // in place: one launch over every shard (changed stamps select C_t)
      uint32_t u0 = (uint32_t)H.bounds[0], u1 = (uint32_t)H.bounds[P], np = P;
      KL(D.s_activate, grid_for(g, u1 - u0), kBlock, &Pz_out, &u0, &u1, &S->d_bounds, &np, &S->d_next, &S->cstamp);
      launches++;
    }
    for (uint32_t s = 0; s < P && !zc_a; s++) {
      if (!h_changed[s] && !no_skip) continue;
      uint32_t u0 = (uint32_t)H.bounds[s], u1 = (uint32_t)H.bounds[s + 1], np = P;
      int k = -1;
      if (!zc_a) {
        gr_status gs = stage(g, S, cs, false, s, false, &k);
        if (gs != GR_OK) return gs;
      }
      Part<OffT> Pk = zc_a ? Pz_out : slot_part<OffT>(g, S, k, false, s);
      KL(D.s_activate, grid_for(g, u1 - u0), kBlock, &Pk, &u0, &u1, &S->d_bounds, &np, &S->d_next, &S->cstamp);
      if (k >= 0) SCK(cudaEventRecord(S->freed[k], cs));
      launches++;
    }
    k_s_finish<OffT><<<1, kBlock, 0, cs>>>(P0);
    launches++;
    SCK(cudaGetLastError());
    SCK(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, cs));
    SCK(cudaMemcpyAsync(h_next, S->d_next, P, cudaMemcpyDeviceToHost, cs));
    SCK(cudaStreamSynchronize(cs));
    for (uint32_t s = 0; s < P; s++) act[s] = h_next[s];
    // bytes read in place this superstep (exact: the edges the kernels touched)
    if (zc_g) S->bytes_zc += wb * (g->h_ctl->tot_gathered - g0);
    if (zc_a) S->bytes_zc += 4 * (g->h_ctl->tot_scattered - s0);
  }
  const Ctl &c = *g->h_ctl;
  st->iterations = c.iter;
  st->edges_gathered = c.tot_gathered;
  st->edges_scattered = c.tot_scattered;
  st->kernel_launches += launches;
  g->epoch_next = h.epoch_base + c.iter + 2;
  g->trace_rows = std::min<uint64_t>(c.iter, g->trace_cap);
  st->bytes_hbm_model = (D.uses_weights ? 5 : 4) * c.tot_gathered + 4 * c.tot_scattered;
  return GR_OK;
#undef KL
}

gr_status run_streamed(gr_graph *g, const gr_run_opts *o, gr_run_stats *st) {
  Streamer *S = S_(g);
  if (!S) return fail(GR_ESTATE, "streamer not initialised");
  cudaStream_t cs = o->stream ? (cudaStream_t)o->stream : g->stream;
  S->bytes_h2d = 0;
  S->bytes_zc = 0;
  S->zc_phases = 0;
  SCK(cudaEventRecord(g->ev_start, cs));
  gr_status r;
  if (o->algo == GR_PAGERANK) {
    r = g->off64 ? stream_pagerank<uint64_t>(g, o, cs, st) : stream_pagerank<uint32_t>(g, o, cs, st);
  } else {
    ProgDesc D;
    if ((r = prog_desc(o->algo, o->custom_id, &D)) != GR_OK) return r;
    r = g->off64 ? stream_frontier<uint64_t>(g, o, cs, st, D) : stream_frontier<uint32_t>(g, o, cs, st, D);
  }
  if (r != GR_OK) return r;
  SCK(cudaEventRecord(g->ev_stop, cs));
  SCK(cudaEventSynchronize(g->ev_stop));
  float ms = 0;
  SCK(cudaEventElapsedTime(&ms, g->ev_start, g->ev_stop));
  st->seconds = ms * 1e-3;
  st->bytes_h2d = S->bytes_h2d + S->bytes_zc;
  st->bytes_h2d_zero_copy = S->bytes_zc;
  st->zero_copy_phases = S->zc_phases;
  g->last_algo = o->algo;
  g->last_iters = st->iterations;
  return GR_OK;
}

}  // namespace gr
