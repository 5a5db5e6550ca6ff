// engine.cu — the GraphReduce B200 runtime behind include/graphreduce.h.
//
// Data Movement + Compute Engine of PAPER.md §4.3-4.4 redesigned for B200:
//   * resident mode: every shard's CSC/CSR is copied to HBM once at load
//     (static buffers, §3.2); the GPU then runs "one grid spans many
//     shards" — the two-level parallelism of L258 without per-shard launches;
//   * streamed mode (stream.cu): shard payloads stay in pinned host memory and
//     are DMA'd per superstep into K = 2 device slots (Eq. 1-2),
//     skipping shards with no active vertex (§5.2);
//   * the BSP loop (L76, L256) runs on the device as a CUDA graph with a
//     conditional WHILE node (no host round trip per superstep), or on the
//     host (GR_LOOP_HOST).
#include <cuda_runtime.h>

#include <cub/cub.cuh>

#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "engine.h"
#include "jit.h"
#include "kernels_frontier.cuh"
#include "kernels_pr.cuh"

namespace gr {

static thread_local std::string t_err;

gr_status fail(gr_status s, const char *fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  t_err = buf;
  return s;
}

const char *last_error() { return t_err.c_str(); }

void tmark(const char *what) {
  static const bool on = [] {
    const char *e = getenv("GR_TIMING");
    return e && e[0] == '1';
  }();
  if (!on) return;
  static thread_local std::chrono::steady_clock::time_point last = std::chrono::steady_clock::now();
  const auto now = std::chrono::steady_clock::now();
  fprintf(stderr, "[gr timing] %-34s %9.3f ms\n", what, std::chrono::duration<double, std::milli>(now - last).count());
  last = now;
}
void clear_error() { t_err.clear(); }

#define CK(call)                                                                              \
  do {                                                                                        \
    cudaError_t e_ = (call);                                                                  \
    if (e_ != cudaSuccess)                                                                    \
      return fail(e_ == cudaErrorMemoryAllocation ? GR_ENOMEM : GR_ECUDA, "%s: %s (%s:%d)", #call, \
                  cudaGetErrorString(e_), __FILE__, __LINE__);                                \
  } while (0)

void pool_init(int device) {
  static bool done[64] = {};
  if (device < 0 || device >= 64 || done[device]) return;
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
    uint64_t keep = ~0ull;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
  }
  cudaGetLastError();
  done[device] = true;
}

gr_status dev_alloc(gr_graph *g, void **p, size_t bytes) {
  *p = nullptr;
  if (bytes == 0) bytes = 16;
  cudaError_t e = cudaMallocAsync(p, bytes, g->stream);
  if (e != cudaSuccess) {  // give cached pool memory back to the device and retry once
    cudaGetLastError();
    cudaDeviceSynchronize();
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, g->device) == cudaSuccess) cudaMemPoolTrimTo(pool, 0);
    e = cudaMallocAsync(p, bytes, g->stream);
  }
  if (e != cudaSuccess) {
    *p = nullptr;
    cudaGetLastError();
    return fail(GR_ENOMEM, "cudaMalloc(%zu bytes) failed: %s", bytes, cudaGetErrorString(e));
  }
  g->allocs.push_back(*p);
  g->dev_bytes += bytes;
  return GR_OK;
}

// Every setup transfer is ordered on the graph's (non-blocking) stream: a plain
// cudaMemcpy from pageable memory may return before its DMA lands, and
// cudaMemset is asynchronous — neither is ordered with kernels on g->stream.
template <class T> static gr_status upload(gr_graph *g, T **dst, const T *src, size_t count) {
  gr_status s = dev_alloc(g, (void **)dst, count * sizeof(T));
  if (s != GR_OK) return s;
  if (count) {
    CK(cudaMemcpyAsync(*dst, src, count * sizeof(T), cudaMemcpyHostToDevice, g->stream));
    CK(cudaStreamSynchronize(g->stream));  // the host buffer may be freed on return
  }
  return GR_OK;
}

template <class OffT> static gr_status upload_offsets(gr_graph *g, void **dst, const std::vector<uint64_t> &off) {
  if (sizeof(OffT) == 8) return upload(g, (uint64_t **)dst, off.data(), off.size());
  std::vector<uint32_t> o32(off.size());
  for (size_t i = 0; i < off.size(); i++) o32[i] = (uint32_t)off[i];
  return upload(g, (uint32_t **)dst, o32.data(), o32.size());
}

static void build_hub_bits(const std::vector<uint64_t> &off, uint64_t count, std::vector<uint32_t> *bits,
                           std::vector<uint32_t> *list, uint64_t id_base) {
  bits->assign((count + 31) / 32 + 1, 0u);
  for (uint64_t i = 0; i < count; i++)
    if (off[i + 1] - off[i] > kHubDegree) {
      (*bits)[i >> 5] |= 1u << (i & 31);
      if (list) list->push_back((uint32_t)(id_base + i));
    }
}

// ------------------------------------------------------------------- load
gr_status load_device(gr_graph *g) {
  HostGraph &H = g->H;
  const uint64_t n = H.n, own_n = H.own_n(), mi = H.m_in;
  gr_status s;
  uint64_t hubs_in = 0, chunks_in = 0, hubs_out = 0, chunks_out = 0;
  if (g->dev_built) {
    // offsets, payloads, hub bitmaps and static hub chunks already on the device
    hubs_in = g->dev_hubs_in;
    chunks_in = g->dev_chunks_in;
    hubs_out = g->dev_hubs_out;
    chunks_out = g->dev_chunks_out;
  } else {
  g->off64 = (mi >= 0xFFFFFFFFull);
  // static per-vertex metadata (both modes)
  if (g->off64) {
    if ((s = upload_offsets<uint64_t>(g, &g->in_off, H.in_off)) != GR_OK) return s;
    if ((s = upload_offsets<uint64_t>(g, &g->out_off, H.out_off)) != GR_OK) return s;
  } else {
    if ((s = upload_offsets<uint32_t>(g, &g->in_off, H.in_off)) != GR_OK) return s;
    if ((s = upload_offsets<uint32_t>(g, &g->out_off, H.out_off)) != GR_OK) return s;
  }
  std::vector<uint32_t> hb_in, hb_out, hubs;
  build_hub_bits(H.in_off, own_n, &hb_in, &hubs, H.own_lo);
  build_hub_bits(H.out_off, n, &hb_out, nullptr, 0);
  if ((s = upload(g, &g->hub_in, hb_in.data(), hb_in.size())) != GR_OK) return s;
  if ((s = upload(g, &g->hub_out, hb_out.data(), hb_out.size())) != GR_OK) return s;
  g->n_static_hubs = (uint32_t)hubs.size();
  if ((s = upload(g, &g->static_hubs, hubs.data(), hubs.size())) != GR_OK) return s;
  // hub chunk capacities: every hub appears at most once per list
  {
  std::vector<uint32_t> sch_h, sch_c;
  for (uint64_t i = 0; i < own_n; i++) {
    const uint64_t d = H.in_off[i + 1] - H.in_off[i];
    if (d > kHubDegree) {
      const uint64_t nch = (d + kChunk - 1) / kChunk;
      for (uint64_t c = 0; c < nch; c++) { sch_h.push_back((uint32_t)hubs_in); sch_c.push_back((uint32_t)c); }
      hubs_in++;
      chunks_in += nch;
    }
  }
  for (uint64_t u = 0; u < n; u++) {
    const uint64_t d = H.out_off[u + 1] - H.out_off[u];
    if (d > kHubDegree) { hubs_out++; chunks_out += (d + kChunk - 1) / kChunk; }
  }
  g->n_static_chunks = (uint32_t)sch_h.size();
  if ((s = upload(g, &g->static_chk_h, sch_h.data(), sch_h.size())) != GR_OK) return s;
  if ((s = upload(g, &g->static_chk_c, sch_c.data(), sch_c.size())) != GR_OK) return s;
  }
  // edge payloads: resident copies (streamed mode keeps them in pinned host memory)
  if (g->mode == GR_MODE_RESIDENT) {
    if ((s = upload(g, &g->in_src, H.in_src.as<uint32_t>(), mi + 4)) != GR_OK) return s;
    if ((s = upload(g, &g->out_dst, H.out_dst.as<uint32_t>(), mi + 4)) != GR_OK) return s;
    if (H.has_w && (s = upload(g, &g->in_w, H.in_w.as<uint8_t>(), mi + 16)) != GR_OK) return s;
  }
  if ((s = upload(g, &g->d_outdeg, H.outdeg.data(), n)) != GR_OK) return s;
  }
  const uint64_t chk_cap = std::max<uint64_t>(std::max(chunks_in, chunks_out), 1);
  for (int i = 0; i < 2; i++) {
    if ((s = dev_alloc(g, (void **)&g->chkA_h[i], 4 * chk_cap)) != GR_OK) return s;
    if ((s = dev_alloc(g, (void **)&g->chkA_c[i], 4 * chk_cap)) != GR_OK) return s;
  }
  if ((s = dev_alloc(g, (void **)&g->chkC_h, 4 * std::max<uint64_t>(chunks_out, 1))) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->chkC_c, 4 * std::max<uint64_t>(chunks_out, 1))) != GR_OK) return s;
  g->hub_cap = (uint32_t)std::max<uint64_t>(std::max(hubs_in, hubs_out), 1);
  if ((s = dev_alloc(g, (void **)&g->hub_acc, 8ull * g->hub_cap)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->hub_done, 4ull * g->hub_cap)) != GR_OK) return s;
  CK(cudaMemsetAsync(g->hub_done, 0, 4ull * g->hub_cap, g->stream));
  if ((s = dev_alloc(g, (void **)&g->hub_act, 4ull * g->hub_cap)) != GR_OK) return s;
  CK(cudaMemsetAsync(g->hub_act, 0, 4ull * g->hub_cap, g->stream));
  // changed-set bitmaps for pull activation (resident single-rank runs)
  if (g->mode == GR_MODE_RESIDENT && H.owners.size() <= 2) {
    g->cbits_words = cbits_words_n(n);
    for (int i = 0; i < 2; i++)
      if ((s = dev_alloc(g, (void **)&g->cbits[i], 4 * g->cbits_words)) != GR_OK) return s;
  }

  // vertex state (replicated values, owned frontier structures)
  const size_t ow = std::max<uint64_t>(own_n, 1);
  if ((s = dev_alloc(g, (void **)&g->val, 4 * n)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->stamp, 4 * ow)) != GR_OK) return s;
  CK(cudaMemsetAsync(g->stamp, 0, 4 * ow, g->stream));
  for (int i = 0; i < 2; i++) {
    if ((s = dev_alloc(g, (void **)&g->listA[i], 4 * ow)) != GR_OK) return s;
    if ((s = dev_alloc(g, (void **)&g->listH[i], 4 * ow)) != GR_OK) return s;
  }
  // changed lists: owned vertices only, except in partitioned runs where the
  // exchanged changed set of every rank is classified into them
  const size_t cw = H.owners.size() > 2 ? std::max<uint64_t>(n, 1) : ow;
  if ((s = dev_alloc(g, (void **)&g->C_v, 4 * cw)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->C_val, 4 * cw)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->CH_v, 4 * cw)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->CH_val, 4 * cw)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->ctl, sizeof(Ctl))) != GR_OK) return s;
  g->trace_cap = 1u << 20;
  if ((s = dev_alloc(g, (void **)&g->trace, 32ull * g->trace_cap)) != GR_OK) return s;

  // PageRank state
  if ((s = dev_alloc(g, (void **)&g->inv_outdeg, 4 * n)) != GR_OK) return s;
  k_inv_outdeg<<<g->num_sms * 4, 256, 0, g->stream>>>((uint32_t)n, g->d_outdeg, g->inv_outdeg);
  CK(cudaGetLastError());
  for (int i = 0; i < 2; i++) {
    if (H.owners.size() > 2) {
      // partitioned: plain cudaMalloc so the replica can be exported to the peers (cudaIpc)
      CK(cudaMalloc((void **)&g->contrib[i], 4 * std::max<uint64_t>(n, 1)));
      g->plain_allocs.push_back(g->contrib[i]);
      g->dev_bytes += 4 * n;
    } else if ((s = dev_alloc(g, (void **)&g->contrib[i], 4 * n)) != GR_OK) {
      return s;
    }
  }
  if ((s = dev_alloc(g, (void **)&g->rank, 4 * ow)) != GR_OK) return s;
  const uint64_t items = own_n + mi;
  g->pr_tiles = (uint32_t)((items + kPrTile - 1) / kPrTile);
  g->pr_wtiles = (uint32_t)((items + kWTile - 1) / kWTile);
  // head/carry records: one per tile (block/warp kernels) or per persistent warp (range kernels)
  const size_t tb = 4ull * (std::max<uint32_t>(std::max(g->pr_tiles, g->pr_wtiles), 1) + 64ull * g->num_sms);
  if ((s = dev_alloc(g, (void **)&g->carry_row, tb)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->carry_val, tb)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->head_row, tb)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->head_val, tb)) != GR_OK) return s;
  if (g->mode == GR_MODE_RESIDENT) {
    if ((s = dev_alloc(g, (void **)&g->tile_row, 4ull * (g->pr_tiles + 1))) != GR_OK) return s;
    if (g->off64)
      k_pr_tiles<uint64_t><<<(g->pr_tiles + 256) / 256, 256, 0, g->stream>>>(
          (const uint64_t *)g->in_off, 0, (uint32_t)own_n, mi, g->pr_tiles, g->tile_row);
    else
      k_pr_tiles<uint32_t><<<(g->pr_tiles + 256) / 256, 256, 0, g->stream>>>(
          (const uint32_t *)g->in_off, 0, (uint32_t)own_n, mi, g->pr_tiles, g->tile_row);
    if ((s = dev_alloc(g, (void **)&g->wtile_row, 4ull * (g->pr_wtiles + 1))) != GR_OK) return s;
    if ((s = dev_alloc(g, (void **)&g->w_is_long, g->pr_wtiles + 16)) != GR_OK) return s;
    if ((s = dev_alloc(g, (void **)&g->long_c, 4ull * (g->pr_wtiles + 1))) != GR_OK) return s;
    if ((s = dev_alloc(g, (void **)&g->long_f, 4ull * (g->pr_wtiles + 1))) != GR_OK) return s;
    uint32_t *d_nlong = nullptr;
    CK(pmalloc(&d_nlong, 4, g->stream));
    CK(cudaMemsetAsync(d_nlong, 0, 4, g->stream));
    if (g->off64) {
      k_pr_tiles<uint64_t><<<(g->pr_wtiles + 256) / 256, 256, 0, g->stream>>>(
          (const uint64_t *)g->in_off, 0, (uint32_t)own_n, mi, g->pr_wtiles, g->wtile_row, (uint32_t)kWTile);
      k_pr_long_heads<uint64_t><<<(g->pr_wtiles + 255) / 256 + 1, 256, 0, g->stream>>>(
          (const uint64_t *)g->in_off, own_n, mi, g->wtile_row, g->pr_wtiles, kWTile, g->w_is_long, g->long_c,
          g->long_f, d_nlong);
    } else {
      k_pr_tiles<uint32_t><<<(g->pr_wtiles + 256) / 256, 256, 0, g->stream>>>(
          (const uint32_t *)g->in_off, 0, (uint32_t)own_n, mi, g->pr_wtiles, g->wtile_row, (uint32_t)kWTile);
      k_pr_long_heads<uint32_t><<<(g->pr_wtiles + 255) / 256 + 1, 256, 0, g->stream>>>(
          (const uint32_t *)g->in_off, own_n, mi, g->wtile_row, g->pr_wtiles, kWTile, g->w_is_long, g->long_c,
          g->long_f, d_nlong);
    }
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(&g->n_long, d_nlong, 4, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaStreamSynchronize(g->stream));
    pfree(d_nlong, g->stream);
  }
  CK(cudaStreamSynchronize(g->stream));

  // occupancy-derived persistent grid: a multiple of the SM count
  int bps = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_gather_apply<ProgCC, uint32_t>, kBlock, 0));
  g->grid_frontier = g->num_sms * std::max(1, std::min(bps, 8));
  int coop = 0;
  cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, g->device);
  g->coop = coop != 0;
  return GR_OK;
}

// -------------------------------------------------------------- frontier run
// Dense edge-segmented layout (kernels_frontier.cuh dense_seg_phase), once per
// graph: the PageRank seg layout over the CSC without hot tags (items =
// max(indeg, 1) per row, kDsNoSrc for an empty row's item and the padding),
// the weights per item, each tile's first row, and the rows spanning tiles.
template <class OffT>
static __global__ void k_ds_fill_w(const OffT *in_off, uint32_t rows, uint64_t m, const uint8_t *w,
                                   const uint32_t *seg_off, uint8_t *ds_w) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t lo = 0, hi = rows;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if ((uint64_t)in_off[mid] <= e) lo = mid;
      else hi = mid;
    }
    ds_w[seg_off[lo] + (e - (uint64_t)in_off[lo])] = w[e];
  }
}
static __global__ void k_ds_tiles(const uint32_t *seg_off, uint32_t rows, uint32_t tiles, uint32_t *ds_row) {
  for (uint32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < tiles; c += gridDim.x * blockDim.x) {
    const uint64_t i0 = (uint64_t)c * kDsTile;
    uint32_t lo = 0, hi = rows;  // last r with seg_off[r] <= i0
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (seg_off[mid] <= i0) lo = mid;
      else hi = mid;
    }
    ds_row[c] = lo;
  }
}
static __global__ void k_ds_split(const uint32_t *seg_off, uint32_t rows, uint32_t *split, uint32_t *nsplit) {
  for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < rows; r += gridDim.x * blockDim.x)
    if (seg_off[r] / kDsTile != (seg_off[r + 1] - 1) / kDsTile) split[atomicAdd(nsplit, 1u)] = r;
}
// share of the in-edges that sit in rows longer than one tile (the rows the
// vertex path serves least well: warp-cooperative / hub chunks), once per graph
template <class OffT> static gr_status ds_long_fraction(gr_graph *g) {
  const uint32_t rows = (uint32_t)g->H.own_n();
  std::vector<OffT> hoff(rows + 1);
  CK(cudaMemcpyAsync(hoff.data(), g->in_off, sizeof(OffT) * (rows + 1), cudaMemcpyDeviceToHost, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  uint64_t lng = 0;
  for (uint32_t r = 0; r < rows; r++) {
    const uint64_t d = (uint64_t)hoff[r + 1] - (uint64_t)hoff[r];
    if (d > kDsTile) lng += d;
  }
  g->ds_long_frac = g->H.m_in ? (double)lng / (double)g->H.m_in : 0.0;
  return GR_OK;
}

// Vertex records (Part::rec_in / rec_out, kernels_frontier.cuh kRecDeg), once per
// resident single-rank graph whose vertices nearly all have degree <= kRecDeg in
// both directions (road networks, meshes: cfg3): a lane then reads a vertex's
// whole adjacency with one 32-byte sector — one dependent load and two
// requests less per gathered or expanded vertex. GR_REC=0/1 forces.
template <class OffT>
static __global__ void k_rec_count(const OffT *off, uint32_t rows, unsigned long long *n_small) {
  unsigned long long c = 0;
  for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < rows; r += gridDim.x * blockDim.x)
    c += (uint64_t)off[r + 1] - (uint64_t)off[r] <= kRecDeg;
  for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(n_small, c);
}
template <class OffT>
static __global__ void k_rec_fill(const OffT *off, const uint32_t *adj, const uint8_t *w, uint32_t rows, uint4 *rec) {
  for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < rows; r += gridDim.x * blockDim.x) {
    const uint64_t b = (uint64_t)off[r], d = (uint64_t)off[r + 1] - b;
    uint32_t a[kRecDeg] = {0, 0, 0, 0}, w4 = 0;
    for (uint32_t q = 0; q < kRecDeg && q < d; q++) {
      a[q] = adj[b + q];
      if (w) w4 |= (uint32_t)w[b + q] << (8 * q);
    }
    rec[2ull * r] = make_uint4(a[0], a[1], a[2], a[3]);
    rec[2ull * r + 1] = make_uint4(w4, (uint32_t)d, (uint32_t)b, (uint32_t)(b >> 32));
  }
}
// the activation CSR equals the CSC (same offsets, same sorted adjacency): the
// graph is symmetric and a vertex's in-record lists its out-neighbours too
template <class OffT>
static __global__ void k_same_adj(const OffT *a_off, const OffT *b_off, uint32_t rows, const uint32_t *a,
                                  const uint32_t *b, uint64_t m, unsigned long long *diff) {
  unsigned long long c = 0;
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x, nt = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t r = tid; r <= rows; r += nt) c += (uint64_t)a_off[r] != (uint64_t)b_off[r];
  for (uint64_t e = tid; e < m; e += nt) c += a[e] != b[e];
  if (c) atomicAdd(diff, c);
}
template <class OffT> static gr_status rec_setup(gr_graph *g) {
  g->rec_tried = true;
  const uint32_t rows = (uint32_t)g->H.own_n(), n = (uint32_t)g->H.n;
  const char *e = getenv("GR_REC");
  if ((e && atoi(e) == 0) || !rows || !g->in_src || !g->out_dst) return GR_OK;
  cudaStream_t s = g->stream;
  unsigned long long *cnt = nullptr, h[2] = {0, 0};
  CK(cudaMallocAsync(&cnt, sizeof h, s));
  CK(cudaMemsetAsync(cnt, 0, sizeof h, s));
  k_rec_count<OffT><<<g->num_sms * 8, 256, 0, s>>>((const OffT *)g->in_off, rows, cnt);
  k_rec_count<OffT><<<g->num_sms * 8, 256, 0, s>>>((const OffT *)g->out_off, n, cnt + 1);
  CK(cudaMemcpyAsync(h, cnt, sizeof h, cudaMemcpyDeviceToHost, s));
  CK(cudaFreeAsync(cnt, s));
  CK(cudaStreamSynchronize(s));
  if (!(e || (h[0] >= 0.9 * rows && h[1] >= 0.9 * n))) return GR_OK;
  // activation records: measured no gain on cfg3 (the 32-byte out-records double the
  // L2 footprint of the wavefront: gather 214 -> 250 ms, activation 320 -> 297 ms);
  // GR_REC_OUT=1 builds and uses them
  const char *eo = getenv("GR_REC_OUT");
  const bool out = eo && atoi(eo) != 0;
  uint4 *ri = nullptr, *ro = nullptr;
  if (dev_alloc(g, (void **)&ri, 32ull * rows) != GR_OK || (out && dev_alloc(g, (void **)&ro, 32ull * n) != GR_OK))
    return GR_OK;  // records are an accelerator: run without them
  k_rec_fill<OffT><<<g->num_sms * 8, 256, 0, s>>>((const OffT *)g->in_off, g->in_src, g->in_w, rows, ri);
  if (out) k_rec_fill<OffT><<<g->num_sms * 8, 256, 0, s>>>((const OffT *)g->out_off, g->out_dst, nullptr, n, ro);
  CK(cudaGetLastError());
  g->rec_in = ri;
  g->rec_out = ro;
  // symmetric graphs (road networks, meshes, symmetrized inputs) may let the
  // activation read the in-record of the changed vertex (no second record array);
  // measured slower on cfg3 (537 -> 583 ms: the per-lane record batches leave
  // lanes idle where the CSR expansion packs 32 edges per round), so opt-in:
  // GR_REC_SYM=1
  const char *esym = getenv("GR_REC_SYM");
  if (!out && esym && atoi(esym) != 0 && rows == n && g->out_off) {
    unsigned long long *d = nullptr, hd = 1;
    CK(cudaMallocAsync(&d, sizeof hd, s));
    CK(cudaMemsetAsync(d, 0, sizeof hd, s));
    k_same_adj<OffT><<<g->num_sms * 8, 256, 0, s>>>((const OffT *)g->in_off, (const OffT *)g->out_off, rows,
                                                    g->in_src, g->out_dst, g->H.m_in, d);
    CK(cudaMemcpyAsync(&hd, d, sizeof hd, cudaMemcpyDeviceToHost, s));
    CK(cudaFreeAsync(d, s));
    CK(cudaStreamSynchronize(s));
    if (hd == 0) g->rec_out = ri;
  }
  const char *sd = getenv("GR_STAMP_DIRECT");
  g->stamp_direct = sd ? atoi(sd) != 0 : true;
  return GR_OK;
}

template <class OffT> static gr_status ds_setup(gr_graph *g) {
  g->ds_tried = true;
  const HostGraph &H = g->H;
  cudaStream_t s = g->stream;
  const uint32_t rows = (uint32_t)H.own_n();
  const uint64_t m = H.m_in;
  if (rows == 0) return GR_OK;
  const OffT *in_off = (const OffT *)g->in_off;
  // Row placement (host, once per graph): items = max(indeg, 1) per row; a row
  // of at most one tile that would cross a tile boundary starts at the next
  // tile instead (the gap is padding, absorbed by the previous row as identity
  // items), so only rows longer than a tile are split between tiles.
  std::vector<OffT> hoff(rows + 1);
  CK(cudaMemcpyAsync(hoff.data(), in_off, sizeof(OffT) * (rows + 1), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  std::vector<uint32_t> pos(rows + 1);
  uint64_t p = 0;
  for (uint32_t r = 0; r < rows; r++) {
    const uint64_t d = (uint64_t)hoff[r + 1] - (uint64_t)hoff[r];
    const uint64_t L = d ? d : 1;
    if (L <= kDsTile && (p % kDsTile) + L > kDsTile) p = (p + kDsTile - 1) / kDsTile * kDsTile;
    if (p + L + 2 * kDsTile >= 0xFFFFFFFFull) return GR_OK;  // stays on the vertex path
    pos[r] = (uint32_t)p;
    p += L;
  }
  pos[rows] = (uint32_t)p;
  const uint32_t items = (uint32_t)p;
  uint32_t *seg_off = nullptr, *d_n = nullptr;
  CK(pmalloc(&seg_off, 4ull * (rows + 1), s));
  CK(cudaMemcpyAsync(seg_off, pos.data(), 4ull * (rows + 1), cudaMemcpyHostToDevice, s));
  const uint32_t tiles = (items + kDsTile - 1) / kDsTile;
  const uint64_t padded = (uint64_t)tiles * kDsTile;
  gr_status st;
  if ((st = dev_alloc(g, (void **)&g->ds_src, 4 * padded + 16)) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&g->ds_flags, 4ull * (tiles + 2) * 8)) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&g->ds_row, 4ull * (tiles + 1))) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&g->ds_split, 4ull * rows)) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&g->ds_acc, 8ull * rows)) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&g->ds_act, 4ull * (rows / 32 + 2))) != GR_OK) return st;
  CK(cudaMemsetAsync(g->ds_flags, 0, 4ull * (tiles + 2) * 8, s));
  k_fill_u32<<<g->num_sms * 8, 256, 0, s>>>(g->ds_src, kDsNoSrc, padded);  // padding between rows
  k_seg_fill<OffT><<<g->num_sms * 16, 256, 0, s>>>(in_off, rows, m, g->in_src, seg_off, g->ds_src);
  k_seg_rows<OffT><<<g->num_sms * 8, 256, 0, s>>>(in_off, rows, seg_off, g->ds_src, g->ds_flags, kDsNoSrc, padded);
  if (g->in_w) {
    if ((st = dev_alloc(g, (void **)&g->ds_w, padded + 16)) != GR_OK) return st;
    CK(cudaMemsetAsync(g->ds_w, 0, padded + 16, s));
    k_ds_fill_w<OffT><<<g->num_sms * 16, 256, 0, s>>>(in_off, rows, m, g->in_w, seg_off, g->ds_w);
  }
  k_ds_tiles<<<(tiles + 255) / 256, 256, 0, s>>>(seg_off, rows, tiles, g->ds_row);
  CK(pmalloc(&d_n, 4, s));
  CK(cudaMemsetAsync(d_n, 0, 4, s));
  k_ds_split<<<g->num_sms * 8, 256, 0, s>>>(seg_off, rows, g->ds_split, d_n);
  CK(cudaGetLastError());
  uint32_t nsplit = 0;
  CK(cudaMemcpyAsync(&nsplit, d_n, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  pfree(seg_off, s);
  pfree(d_n, s);
  g->ds_tiles = tiles;
  g->ds_nsplit = nsplit;
  return GR_OK;
}

// Tolerance PageRank divisor table: (ceil(2^64 / n_u), n_u); n_u <= 1 keeps m = 0.
static __global__ void k_prd_div(uint64_t n, const uint32_t *outdeg, ulonglong2 *tab) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t d = outdeg[v];
    tab[v] = make_ulonglong2(d >= 2 ? (~0ull) / d + 1ull : 0ull, d);
  }
}

// Fused push state (once per graph): the two accumulator arrays and, for
// weighted programs, the activation CSR's weights. The CSR is the CSC
// transposed by a stable sort of the CSC sources (device build, or the host
// layout sorted the same way), so the same stable sort carrying the CSC
// weights yields them in CSR order.
static gr_status out_w_setup(gr_graph *g);
static gr_status push_setup(gr_graph *g, bool weights) {
  const uint64_t n = g->H.n;
  gr_status st;
  for (int i = 0; i < 2; i++)
    if (!g->nxt[i] && (st = dev_alloc(g, (void **)&g->nxt[i], 4 * std::max<uint64_t>(n, 1))) != GR_OK) return st;
  return weights ? out_w_setup(g) : GR_OK;
}

static __global__ void k_iota_u32(uint32_t *p, uint64_t m) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = (uint32_t)i;
}

// Mutable edge state (kHasScatter programs, once per graph): the CSC position of
// every activation-CSR edge — the same stable sort by source carrying the CSC
// positions — the state array, and the CSR weights when scatter reads them.
gr_status scatter_setup(gr_graph *g, bool weights) {
  const uint64_t n = g->H.n, m = g->H.m_in;
  cudaStream_t s = g->stream;
  gr_status st;
  if (m >= 0xFFFFFFFFull) return fail(GR_EUNSUPPORTED, "edge state: more than 2^32-1 edges");
  if (!g->estate && (st = dev_alloc(g, (void **)&g->estate, 4 * (m + 4))) != GR_OK) return st;
  if (!g->out_eid) {
    if ((st = dev_alloc(g, (void **)&g->out_eid, 4 * (m + 4))) != GR_OK) return st;
    CK(cudaMemsetAsync(g->out_eid + m, 0, 16, s));
    uint32_t bits = 1;
    while ((1ull << bits) < n) bits++;
    uint32_t *kscratch = nullptr, *iota = nullptr;
    void *tmp = nullptr;
    size_t need = 0;
    CK(pmalloc(&kscratch, 4 * std::max<uint64_t>(m, 1), s));
    CK(pmalloc(&iota, 4 * std::max<uint64_t>(m, 1), s));
    k_iota_u32<<<g->num_sms * 8, 256, 0, s>>>(iota, m);
    CK(cub::DeviceRadixSort::SortPairs(nullptr, need, g->in_src, kscratch, iota, g->out_eid, (int64_t)m, 0,
                                       (int)bits, s));
    CK(pmalloc(&tmp, std::max<size_t>(need, 16), s));
    CK(cub::DeviceRadixSort::SortPairs(tmp, need, g->in_src, kscratch, iota, g->out_eid, (int64_t)m, 0, (int)bits,
                                       s));
    pfree(tmp, s);
    pfree(iota, s);
    pfree(kscratch, s);
    CK(cudaStreamSynchronize(s));
  }
  return weights ? out_w_setup(g) : GR_OK;
}

static gr_status out_w_setup(gr_graph *g) {
  const uint64_t n = g->H.n, m = g->H.m_in;
  cudaStream_t s = g->stream;
  gr_status st;
  if (g->out_w) return GR_OK;
  if (!g->in_w) return fail(GR_EINVAL, "the program reads edge weights but the graph has none");
  if ((st = dev_alloc(g, (void **)&g->out_w, m + 16)) != GR_OK) return st;
  CK(cudaMemsetAsync(g->out_w + m, 0, 16, s));
  uint32_t bits = 1;
  while ((1ull << bits) < n) bits++;
  uint32_t *kscratch = nullptr;
  void *tmp = nullptr;
  size_t need = 0;
  CK(pmalloc(&kscratch, 4 * std::max<uint64_t>(m, 1), s));
  CK(cub::DeviceRadixSort::SortPairs(nullptr, need, g->in_src, kscratch, g->in_w, g->out_w, (int64_t)m, 0,
                                     (int)bits, s));
  CK(pmalloc(&tmp, std::max<size_t>(need, 16), s));
  CK(cub::DeviceRadixSort::SortPairs(tmp, need, g->in_src, kscratch, g->in_w, g->out_w, (int64_t)m, 0, (int)bits,
                                     s));
  pfree(tmp, s);
  pfree(kscratch, s);
  CK(cudaStreamSynchronize(s));
  return GR_OK;
}

template <class Prog, class OffT>
static void launch_body(gr_graph *g, cudaStream_t s, unsigned long long cond, int use_graph, uint64_t *launches,
                        bool push) {
  Part<OffT> P = make_part<OffT>(g);
  if (push) {  // fused push superstep: one kernel
    k_push_expand<Prog, OffT><<<g->grid_frontier, kBlock, 0, s>>>(P, cond, use_graph);
    *launches += 1;
    return;
  }
  if constexpr (HasScatter<Prog>::value) {  // gather | commit | scatter + activate
    k_gather_apply<Prog, OffT><<<g->grid_frontier, kBlock, 0, s>>>(P);
    k_commit_only<OffT><<<g->grid_frontier, kBlock, 0, s>>>(P);
    k_scatter_activate<Prog, OffT><<<g->grid_frontier, kBlock, 0, s>>>(P, cond, use_graph);
    *launches += 3;
    return;
  }
  if (Prog::kHasGather) {
    k_gather_apply<Prog, OffT><<<g->grid_frontier, kBlock, 0, s>>>(P);
    k_activate<OffT><<<g->grid_frontier, kBlock, 0, s>>>(P, cond, use_graph);
    *launches += 2;
  } else {
    k_bfs_expand<OffT><<<g->grid_frontier, kBlock, 0, s>>>(P, cond, use_graph);
    *launches += 1;
  }
  if (!Prog::kHasGather && g->cbits[0]) {  // BFS: scan half of a pull superstep (returns at once after a push)
    k_pull<true, OffT><<<g->grid_frontier, kBlock, 0, s>>>(P, cond, use_graph);
    *launches += 1;
  }
}

template <class Prog, class OffT>
static gr_status get_while_graph(gr_graph *g, int key, cudaGraphExec_t *out, uint64_t *per_iter_launches,
                                 bool push) {
  if (push) key += 1000;
  auto it = g->while_exec.find(key);
  if (it != g->while_exec.end()) {
    *out = it->second.first;
    *per_iter_launches = it->second.second;
    return GR_OK;
  }
  cudaGraph_t graph;
  CK(cudaGraphCreate(&graph, 0));
  cudaGraphConditionalHandle h;
  CK(cudaGraphConditionalHandleCreate(&h, graph, 1, cudaGraphCondAssignDefault));
  cudaGraphNodeParams p = {};
  p.type = cudaGraphNodeTypeConditional;
  p.conditional.handle = h;
  p.conditional.type = cudaGraphCondTypeWhile;
  p.conditional.size = 1;
  cudaGraphNode_t node;
  CK(cudaGraphAddNode(&node, graph, nullptr, 0, &p));
  cudaGraph_t body = p.conditional.phGraph_out[0];
  cudaStream_t cs;
  CK(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
  CK(cudaStreamBeginCaptureToGraph(cs, body, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal));
  uint64_t l = 0;
  launch_body<Prog, OffT>(g, cs, (unsigned long long)h, 1, &l, push);
  cudaGraph_t captured = body;
  cudaError_t e = cudaStreamEndCapture(cs, &captured);
  cudaStreamDestroy(cs);
  if (e != cudaSuccess) return fail(GR_ECUDA, "graph capture failed: %s", cudaGetErrorString(e));
  cudaGraphExec_t ex;
  CK(cudaGraphInstantiate(&ex, graph, 0));
  CK(cudaGraphDestroy(graph));
  g->while_exec[key] = {ex, l};
  *out = ex;
  *per_iter_launches = l;
  return GR_OK;
}

// ---- detail columns of the frontier trace (gr_run_opts.trace_detail):
// before superstep t's gather, mark the shard of every vertex of A_t and every
// source its gather reads, then count both sets. A_t is the implicit owned range
// (superstep 0 of kInitAll programs), the vertices with a marked in-neighbour
// (dense supersteps), or the A lists (listA + listH). Diagnostic: host loop only.
// BFS (no gather, apply-only): its A lists hold only the unvisited
// activated vertices, so A_t is recovered from the depths instead — v ∈ A_t iff
// an in-neighbour has depth t-1 (C_{t-1}: the vertices reached at t-1), A_0 = {source}.
template <class OffT>
static __global__ void k_detail_mark(const __grid_constant__ Part<OffT> P, int has_gather, const uint64_t *sb,
                                     uint32_t nsb, uint32_t *src_bits, uint32_t *shard_bits) {
  __shared__ View V;
  load_view(P.ctl, V);
  if (V.stop) return;
  const uint32_t t = V.t, slot = t & 1u;
  const bool bfs = !has_gather;
  const bool implicit = bfs || V.dense || (V.implicit0 && t == 0);
  const uint32_t *bits = P.cbits[slot ^ 1u];
  const uint64_t nA = V.cntA[slot], total = implicit ? (uint64_t)P.own_n : nA + V.cntH[slot];
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t v = implicit ? P.own_lo + (uint32_t)i : (i < nA ? P.listA[slot][i] : P.listH[slot][i - nA]);
    const uint32_t lv = v - P.own_lo;
    const uint64_t b = (uint64_t)P.in_off[lv], e = (uint64_t)P.in_off[lv + 1];
    if (bfs) {
      bool act = t == 0 ? v == V.source : false;
      for (uint64_t k = b; k < e && !act && t > 0; k++) act = ld_cg(P.val + P.in_src[k]) == t - 1;
      if (!act) continue;
    } else if (V.dense) {
      bool act = false;
      for (uint64_t k = b; k < e && !act; k++) act = test_bit_cg(bits, P.in_src[k]);
      if (!act) continue;
    }
    uint32_t lo = 0, hi = nsb;  // shard: last s with sb[s] <= v
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (sb[mid] <= v) lo = mid;
      else hi = mid;
    }
    atomicOr(shard_bits + (lo >> 5), 1u << (lo & 31));
    if (has_gather)
      for (uint64_t k = b; k < e; k++) {
        const uint32_t u = P.in_src[k];
        atomicOr(src_bits + (u >> 5), 1u << (u & 31));
      }
  }
}

static __global__ void k_detail_count(const Ctl *ctl, uint32_t *src_bits, uint64_t src_words, uint32_t *shard_bits,
                                      uint64_t shard_words, unsigned long long *det, uint32_t cap) {
  if (ctl->stop) return;
  unsigned long long a = 0, b = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < src_words; i += (uint64_t)gridDim.x * blockDim.x) {
    b += __popc(src_bits[i]);
    src_bits[i] = 0;
  }
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < shard_words; i += (uint64_t)gridDim.x * blockDim.x) {
    a += __popc(shard_bits[i]);
    shard_bits[i] = 0;
  }
  const uint32_t t = ctl->iter;
  if (t >= cap) return;
  if (a) atomicAdd(det + 2ull * t, a);
  if (b) atomicAdd(det + 2ull * t + 1, b);
}

static gr_status detail_setup(gr_graph *g, cudaStream_t s) {
  gr_status st;
  const uint64_t words = (g->H.n + 31) / 32 + 1, P = g->H.num_shards();
  if (!g->trace_det) {
    if ((st = dev_alloc(g, (void **)&g->trace_det, 16ull * g->trace_cap)) != GR_OK) return st;
    if ((st = dev_alloc(g, (void **)&g->det_src_bits, 4 * words)) != GR_OK) return st;
    if ((st = dev_alloc(g, (void **)&g->det_shard_bits, 4 * (P / 32 + 1))) != GR_OK) return st;
    if ((st = dev_alloc(g, (void **)&g->d_shard_bounds, 8 * (P + 1))) != GR_OK) return st;
    CK(cudaMemcpy(g->d_shard_bounds, g->H.bounds.data(), 8 * (P + 1), cudaMemcpyHostToDevice));
    CK(cudaMemset(g->det_src_bits, 0, 4 * words));
    CK(cudaMemset(g->det_shard_bits, 0, 4 * (P / 32 + 1)));
  }
  CK(cudaMemsetAsync(g->trace_det, 0, 16ull * g->trace_cap, s));
  return GR_OK;
}

template <class OffT>
static gr_status detail_superstep(gr_graph *g, const Part<OffT> &P, bool has_gather, cudaStream_t s) {
  const uint64_t words = (g->H.n + 31) / 32 + 1, np = g->H.num_shards();
  k_detail_mark<OffT><<<g->num_sms * 8, 256, 0, s>>>(P, has_gather ? 1 : 0, g->d_shard_bounds, (uint32_t)np,
                                                    g->det_src_bits, g->det_shard_bits);
  k_detail_count<<<g->num_sms * 2, 256, 0, s>>>(g->ctl, g->det_src_bits, words, g->det_shard_bits, np / 32 + 1,
                                                g->trace_det, g->trace_cap);
  CK(cudaGetLastError());
  return GR_OK;
}

// CTAs per SM of the persistent frontier loop (built-in and run-time programs
// alike): 4; 2 when the owned range has fewer vertices than 4 CTAs per SM have
// threads (cheaper grid barriers: cfg1 BFS 0.392 -> 0.372 ms; SSSP / CC there
// unchanged; cfg3 / cfg4 need 4: 858 vs 783 ms, 20.0 vs 12.3 ms at 2);
// GR_PERSIST_CTAS_PER_SM overrides; never more than the occupancy bps allows.
static uint32_t persistent_grid(const gr_graph *g, int bps) {
  int per_sm = std::min(bps, g->H.own_n() < (uint64_t)g->num_sms * 4 * kBlock ? 2 : 4);
  if (const char *e = getenv("GR_PERSIST_CTAS_PER_SM")) per_sm = std::min(bps, atoi(e));
  return (uint32_t)g->num_sms * (uint32_t)std::max(1, per_sm);
}

template <class Prog, class OffT>
static gr_status run_frontier(gr_graph *g, const gr_run_opts *o, cudaStream_t s, gr_run_stats *st, int key) {
  Part<OffT> P = make_part<OffT>(g);
  uint64_t launches = 0;
  if (g->epoch_next > 0xF0000000u) {
    CK(cudaMemsetAsync(g->stamp, 0, 4ull * std::max<uint64_t>(g->H.own_n(), 1), s));
    g->epoch_next = 1;
  }
  Ctl h{};
  h.epoch_base = g->epoch_next;
  h.max_iters = o->max_iters;
  h.trace_cap = g->trace_cap;
  h.source = o->source;
  h.damping = o->damping;
  h.prof = o->profile ? 1 : 0;
  h.kstart[0] = h.kstart[1] = ~0ull;
  prd_setup(h, o, g->H.n);
  // fused push supersteps (gr/program.cuh kPushFused): direction FUSED, resident, one rank.
  // Not the AUTO choice: on cfg3 (road grid SSSP) one fused phase took 147 us per
  // superstep against 29 + 28 us for the gather / activate pair (profiles/README.md).
  bool push = false;
  if constexpr (PushFused<Prog>::value) {
    push = Prog::kInit == kInitSourceChanged && !g->comm && g->mode == GR_MODE_RESIDENT &&
           o->direction == GR_DIR_FUSED && !o->trace_detail;
    if (const char *e = getenv("GR_PUSH_FUSED")) push = push && atoi(e) != 0;
    if (push) {
      gr_status ps = push_setup(g, Prog::kUsesWeights);
      if (ps != GR_OK) return ps;
      P = make_part<OffT>(g);
      const uint32_t id = Prog::identity_host();
      k_fill<uint32_t><<<g->num_sms * 4, 256, 0, s>>>(g->nxt[0], id, g->H.n);
      k_fill<uint32_t><<<g->num_sms * 4, 256, 0, s>>>(g->nxt[1], id, g->H.n);
      launches += 2;
    }
  }
  h.push = push ? 1u : 0u;
  constexpr bool kScatter = HasScatter<Prog>::value;
  if constexpr (kScatter) {  // mutable edge state: layout once per graph, states reset per run
    gr_status ss = scatter_setup(g, Prog::kUsesWeights);
    if (ss != GR_OK) return ss;
    P = make_part<OffT>(g);
    k_init_edges<Prog, OffT><<<g->num_sms * 8, 256, 0, s>>>(P, g->H.m_in);
    launches++;
  }
  // activation direction (gr_direction); pull needs the bitmaps (resident, one rank);
  // scatter programs always push (the scatter walks the out-edges of C_t)
  const bool may_pull = g->cbits[0] && !push && !kScatter && o->direction != GR_DIR_PUSH;
  bool dseg = false;
  if constexpr (DstFree<Prog>::value) {
    // dense supersteps on edge-segmented tiles: the default for 64-bit gathers
    // and for graphs with >= 25 % of their in-edges in rows longer than a tile
    // (measured on R-MAT: tolerance PageRank 89.8 -> 56.8 ms, CC 4.9 -> 2.8 ms,
    // SSSP 0.89 -> 0.67 ms; the web graph of cfg4 (12 %) stays on the vertex
    // path: 12.3 vs 13.2 ms; profiles/README.md); GR_DENSE_SEG=0/1 forces
    const char *e = getenv("GR_DENSE_SEG");
    const bool ploop = (o->loop == GR_LOOP_AUTO || o->loop == GR_LOOP_PERSISTENT) && g->coop;
    bool want = false;
    if (e) {
      want = atoi(e) != 0;
    } else if (may_pull && ploop) {
      if (sizeof(typename Prog::GatherT) == 8) {
        want = true;
      } else {
        if (g->ds_long_frac < 0) {
          gr_status lf = ds_long_fraction<OffT>(g);
          if (lf != GR_OK) return lf;
        }
        want = g->ds_long_frac >= 0.25;
      }
    }
    if (may_pull && want && ploop && !g->ds_tried) {
      gr_status ds = ds_setup<OffT>(g);
      if (ds != GR_OK) return ds;
    }
    const bool on = may_pull && want && ploop && g->ds_tiles;
    dseg = on;
    if (on) {
      using G = typename Prog::GatherT;
      k_fill<G><<<g->num_sms * 4, 256, 0, s>>>(reinterpret_cast<G *>(g->ds_acc), Prog::identity_host(),
                                              g->H.own_n());
      CK(cudaMemsetAsync(g->ds_act, 0, 4ull * (g->H.own_n() / 32 + 2), s));
      launches++;
    }
    P = make_part<OffT>(g);
    if (!on) P.ds_tiles = 0;
  }
  if (may_pull) {
    uint32_t div = o->pull_div ? o->pull_div : kPullDivDefault;
    if (const char *e = getenv("GR_PULL_DIV")) div = (uint32_t)strtoul(e, nullptr, 10);
    h.pull_div = o->direction == GR_DIR_PULL ? 0xFFFFFFFFu : div;
  }
  *g->h_ctl = h;  // pinned staging: an async copy, not a pageable one (the last run synchronised)
  CK(cudaMemcpyAsync(g->ctl, g->h_ctl, sizeof h, cudaMemcpyHostToDevice, s));
  // values, hub accumulators / done counters and (pull) both changed bitmaps in one launch
  k_init_run<Prog, OffT><<<g->num_sms * 4, 256, 0, s>>>(P, o->source, g->hub_cap, g->cbits_words, may_pull ? 1 : 0);
  launches += 1;
  if (Prog::kInit == kInitAll && g->n_static_hubs) {
    CK(cudaMemcpyAsync(g->listH[0], g->static_hubs, 4ull * g->n_static_hubs, cudaMemcpyDeviceToDevice, s));
    CK(cudaMemcpyAsync(g->chkA_h[0], g->static_chk_h, 4ull * g->n_static_chunks, cudaMemcpyDeviceToDevice, s));
    CK(cudaMemcpyAsync(g->chkA_c[0], g->static_chk_c, 4ull * g->n_static_chunks, cudaMemcpyDeviceToDevice, s));
  }
  k_init_frontier<Prog, OffT><<<1, kBlock, 0, s>>>(P, o->source, g->n_static_hubs, g->n_static_chunks);
  launches++;
  CK(cudaGetLastError());
  const bool detail = o->trace_detail != 0;  // diagnostic: host loop with the detail kernels
  if (detail) {
    gr_status ds = detail_setup(g, s);
    if (ds != GR_OK) return ds;
  }
  const bool persistent = !detail && (o->loop == GR_LOOP_AUTO || o->loop == GR_LOOP_PERSISTENT) && g->coop;
  const bool use_graph = !detail && !persistent && (o->loop == GR_LOOP_DEVICE || o->loop == GR_LOOP_AUTO);
  if (persistent) {
    int bps = 0;
    const void *kf = dseg ? (const void *)k_persistent_ds<Prog, OffT> : (const void *)k_persistent<Prog, OffT>;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, kf, kBlock, 0));
    const uint32_t grid = persistent_grid(g, bps);
    void *args[] = {(void *)&P};
    CK(cudaLaunchCooperativeKernel(kf, dim3(grid), dim3(kBlock), args, 0, s));
    CK(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    launches += 1;
  } else if (use_graph) {
    cudaGraphExec_t ex;
    uint64_t per = 0;
    gr_status gs = get_while_graph<Prog, OffT>(g, key, &ex, &per, push);
    if (gs != GR_OK) return gs;
    CK(cudaGraphLaunch(ex, s));
    CK(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    launches += per * std::max<uint32_t>(g->h_ctl->iter, 1);
  } else {
    for (;;) {
      if (detail) {
        gr_status ds = detail_superstep<OffT>(g, P, Prog::kHasGather, s);
        if (ds != GR_OK) return ds;
      }
      launch_body<Prog, OffT>(g, s, 0, 0, &launches, push);
      CK(cudaGetLastError());
      CK(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
      CK(cudaStreamSynchronize(s));
      if (g->h_ctl->stop) break;
    }
  }
  const Ctl &c = *g->h_ctl;
  if (o->profile) {
    st->kernel_ms[0] += c.kns[0] * 1e-6;
    st->kernel_ms[1] += c.kns[1] * 1e-6;
  }
  st->iterations = c.iter;
  st->pull_supersteps = c.tot_pull;
  st->edges_gathered = c.tot_gathered;
  st->edges_scattered = c.tot_scattered;
  st->kernel_launches += launches;
  g->epoch_next = h.epoch_base + c.iter + 2;
  g->trace_rows = std::min<uint64_t>(c.iter, g->trace_cap);
  // algorithmic bytes: 4 B/in-edge (+1 weight), 12 B per active vertex,
  // 4 B per activated out-edge, 8 B per changed vertex (value commit + offsets)
  const uint64_t sumA = c.tot_A, sumC = c.tot_C;  // accumulated by close_superstep
  const uint64_t wb = Prog::kUsesWeights ? 5 : 4;
  st->bytes_hbm_model = wb * c.tot_gathered + 12 * sumA + 4 * c.tot_scattered + 12 * sumC;
  // fused push: no in-edge walk; per A_t vertex acc + value + offsets (16 B), per
  // pushed edge destination (+ weight), per changed vertex value + offsets (12 B)
  if (push) st->bytes_hbm_model = 16 * sumA + wb * c.tot_scattered + 12 * sumC;
  return GR_OK;
}

// Run-time compiled program (csrc/jit.cu): the same setup
// and persistent BSP loop as run_frontier, with the program's kernels taken
// from its NVRTC module and its static traits read back at compile time.
template <class OffT>
static gr_status run_frontier_jit(gr_graph *g, const gr_run_opts *o, cudaStream_t s, gr_run_stats *st,
                                  const JitProgram *jp) {
  const int k = sizeof(OffT) == 8 ? 1 : 0;
  Part<OffT> P = make_part<OffT>(g);
  uint64_t launches = 0;
  if (g->epoch_next > 0xF0000000u) {
    CK(cudaMemsetAsync(g->stamp, 0, 4ull * std::max<uint64_t>(g->H.own_n(), 1), s));
    g->epoch_next = 1;
  }
  Ctl h{};
  h.epoch_base = g->epoch_next;
  h.max_iters = o->max_iters;
  h.trace_cap = g->trace_cap;
  h.source = o->source;
  h.damping = o->damping;
  h.prof = o->profile ? 1 : 0;
  h.kstart[0] = h.kstart[1] = ~0ull;
  prd_setup(h, o, g->H.n);
  if (jp->scatter) {  // mutable edge state: layout once per graph, states reset per run
    gr_status ss = scatter_setup(g, jp->uses_weights);
    if (ss != GR_OK) return ss;
    P = make_part<OffT>(g);
    uint64_t m_in = g->H.m_in;
    void *args[] = {(void *)&P, (void *)&m_in};
    gr_status r0 = jit_launch(jp->init_edges[k], g->num_sms * 8, 256, args, 0, s, false);
    if (r0 != GR_OK) return r0;
    launches++;
  }
  // scatter programs always push (the scatter walks the out-edges of C_t)
  if (g->cbits[0] && o->direction != GR_DIR_PUSH && !jp->scatter) {
    uint32_t div = o->pull_div ? o->pull_div : kPullDivDefault;
    if (const char *e = getenv("GR_PULL_DIV")) div = (uint32_t)strtoul(e, nullptr, 10);
    h.pull_div = o->direction == GR_DIR_PULL ? 0xFFFFFFFFu : div;
    CK(cudaMemsetAsync(g->cbits[0], 0, 4 * g->cbits_words, s));
    CK(cudaMemsetAsync(g->cbits[1], 0, 4 * g->cbits_words, s));
  }
  *g->h_ctl = h;  // pinned staging: an async copy, not a pageable one (the last run synchronised)
  CK(cudaMemcpyAsync(g->ctl, g->h_ctl, sizeof h, cudaMemcpyHostToDevice, s));
  gr_status r;
  uint32_t src = o->source;
  {
    void *args[] = {(void *)&P, (void *)&src};
    if ((r = jit_launch(jp->init_values[k], g->num_sms * 4, 256, args, 0, s, false)) != GR_OK) return r;
  }
  {
    void *acc = g->hub_acc;
    unsigned long long cnt = g->hub_cap;
    void *args[] = {(void *)&acc, (void *)&cnt};
    if ((r = jit_launch(jp->fill, std::min<uint32_t>((g->hub_cap + 255) / 256, 1024) + 1, 256, args, 0, s, false)) !=
        GR_OK)
      return r;
  }
  CK(cudaMemsetAsync(g->hub_done, 0, 4ull * g->hub_cap, s));
  launches += 2;
  if (jp->init == kInitAll && g->n_static_hubs) {
    CK(cudaMemcpyAsync(g->listH[0], g->static_hubs, 4ull * g->n_static_hubs, cudaMemcpyDeviceToDevice, s));
    CK(cudaMemcpyAsync(g->chkA_h[0], g->static_chk_h, 4ull * g->n_static_chunks, cudaMemcpyDeviceToDevice, s));
    CK(cudaMemcpyAsync(g->chkA_c[0], g->static_chk_c, 4ull * g->n_static_chunks, cudaMemcpyDeviceToDevice, s));
  }
  {
    uint32_t nh = (uint32_t)g->n_static_hubs, nc = (uint32_t)g->n_static_chunks;
    void *args[] = {(void *)&P, (void *)&src, (void *)&nh, (void *)&nc};
    if ((r = jit_launch(jp->init_frontier[k], 1, kBlock, args, 0, s, false)) != GR_OK) return r;
  }
  launches++;
  int bps = 0;
  if ((r = jit_occupancy(jp->persistent[k], kBlock, &bps)) != GR_OK) return r;
  const uint32_t grid = persistent_grid(g, bps);
  {
    void *args[] = {(void *)&P};
    if ((r = jit_launch(jp->persistent[k], grid, kBlock, args, 0, s, true)) != GR_OK) return r;
  }
  CK(cudaMemcpyAsync(g->h_ctl, g->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  launches += 1;
  const Ctl &c = *g->h_ctl;
  if (o->profile) {
    st->kernel_ms[0] += c.kns[0] * 1e-6;
    st->kernel_ms[1] += c.kns[1] * 1e-6;
  }
  st->iterations = c.iter;
  st->pull_supersteps = c.tot_pull;
  st->edges_gathered = c.tot_gathered;
  st->edges_scattered = c.tot_scattered;
  st->kernel_launches += launches;
  g->epoch_next = h.epoch_base + c.iter + 2;
  g->trace_rows = std::min<uint64_t>(c.iter, g->trace_cap);
  const uint64_t sumA = c.tot_A, sumC = c.tot_C;  // accumulated by close_superstep
  const uint64_t wb = jp->uses_weights ? 5 : 4;
  st->bytes_hbm_model = wb * c.tot_gathered + 12 * sumA + 4 * c.tot_scattered + 12 * sumC;
  return GR_OK;
}

// --------------------------------------------------------------- PageRank
template <class OffT> static PrArgs<OffT> pr_args(gr_graph *g, uint32_t t, uint32_t iters, float d) {
  PrArgs<OffT> a{};
  a.n = (uint32_t)g->H.n;
  a.own_lo = (uint32_t)g->H.own_lo;
  a.own_n = (uint32_t)g->H.own_n();
  a.m_in = g->H.m_in;
  a.in_off = (const OffT *)g->in_off;
  a.in_src = g->in_src;
  a.inv_outdeg = g->inv_outdeg;
  a.contrib_in = g->contrib[t & 1];
  a.contrib_out = g->contrib[(t + 1) & 1];
  a.rank = g->rank;
  a.carry_row = g->carry_row;
  a.carry_val = g->carry_val;
  a.head_row = g->head_row;
  a.head_val = g->head_val;
  a.tile_row = g->tile_row;
  a.base = (1.0f - d) / (float)g->H.n;
  a.d = d;
  a.last = (t + 1 == iters) ? 1 : 0;
  if (g->pr_p2p_on && !a.last) {  // fused exchange: the apply also stores into every peer's replica
    static_assert(kMaxPeers == 15, "gr_graph::pr_peer size");
    for (uint32_t q = 0; q < g->pr_npeer; q++) a.peer[q] = g->pr_peer[(t + 1) & 1][q];
    a.npeer = g->pr_npeer;
  }
  return a;
}

// Edge-segmented layout for k_pr_seg (once per graph): item offsets
// seg_off = scan(max(indeg, 1)), the tagged sources placed at their items
// (an empty row's item reads the zero slot), one head bit per item, the first
// row of every 256-item tile and the long fix-up chains.
template <class OffT> static gr_status pr_seg_setup(gr_graph *g) {
  const HostGraph &H = g->H;
  cudaStream_t s = g->stream;
  const uint32_t rows = (uint32_t)H.own_n();
  const OffT *in_off = (const OffT *)g->in_off;
  gr_status st;
  if ((st = dev_alloc(g, (void **)&g->seg_off, 4ull * (rows + 1))) != GR_OK) return st;
  uint32_t *degp = nullptr;
  void *tmp = nullptr;
  size_t need = 0;
  CK(pmalloc(&degp, 4ull * std::max<uint32_t>(rows, 1), s));
  k_seg_deg<OffT><<<g->num_sms * 8, 256, 0, s>>>(in_off, rows, degp);
  CK(cub::DeviceScan::InclusiveSum(nullptr, need, degp, g->seg_off + 1, (int64_t)rows, s));
  CK(pmalloc(&tmp, std::max<size_t>(need, 16), s));
  CK(cub::DeviceScan::InclusiveSum(tmp, need, degp, g->seg_off + 1, (int64_t)rows, s));
  CK(cudaMemsetAsync(g->seg_off, 0, 4, s));
  uint32_t items = 0;
  CK(cudaMemcpyAsync(&items, g->seg_off + rows, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  pfree(degp, s);
  pfree(tmp, s);
  g->seg_items = items;
  g->seg_tiles = (uint32_t)((items + kSegTile - 1) / kSegTile);
  const uint64_t padded = (uint64_t)g->seg_tiles * kSegTile;
  if ((st = dev_alloc(g, (void **)&g->seg_src, 4ull * padded + 16)) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&g->seg_flags, 4ull * (g->seg_tiles + 2) * 8)) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&g->seg_row, 4ull * (g->seg_tiles + 1))) != GR_OK) return st;
  CK(cudaMemsetAsync(g->seg_flags, 0, 4ull * (g->seg_tiles + 2) * 8, s));
  k_seg_fill<OffT><<<g->num_sms * 16, 256, 0, s>>>(in_off, rows, H.m_in, g->pr_src, g->seg_off, g->seg_src);
  k_seg_rows<OffT><<<g->num_sms * 8, 256, 0, s>>>(in_off, rows, g->seg_off, g->seg_src, g->seg_flags,
                                                   kHotTag | g->hot_k, padded);
  uint32_t *d_nlong = nullptr;
  CK(pmalloc(&d_nlong, 4, s));
  CK(cudaMemsetAsync(d_nlong, 0, 4, s));
  k_seg_tiles<<<(g->seg_tiles + 255) / 256, 256, 0, s>>>(g->seg_off, rows, g->seg_tiles, g->seg_row, g->w_is_long,
                                                         g->long_c, g->long_f, d_nlong);
  CK(cudaGetLastError());
  CK(cudaMemcpyAsync(&g->n_long, d_nlong, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  pfree(d_nlong, s);
  return GR_OK;
}

template <class OffT>
using SegKernel = void (*)(const PrArgs<OffT>, const uint32_t *, const uint32_t *, const uint32_t *, const float *,
                           uint32_t, uint32_t);
template <class OffT>
using SegLoopKernel = void (*)(const PrArgs<OffT>, const PrLoop);
// The seg kernels are instantiated for the default variant bits only (the other
// combinations were measured in round 1 and are not built: profiles/README.md)
template <class OffT> static SegLoopKernel<OffT> seg_loop_kernel(int, bool phases = false, bool tma = false) {
  if (tma)
    return phases ? k_pr_seg_loop<OffT, kSegDefaultVar, true, true> : k_pr_seg_loop<OffT, kSegDefaultVar, false, true>;
  return phases ? k_pr_seg_loop<OffT, kSegDefaultVar, true> : k_pr_seg_loop<OffT, kSegDefaultVar, false>;
}
template <class OffT> static SegKernel<OffT> seg_kernel(int) { return k_pr_seg<OffT, kSegDefaultVar>; }

// Source-blocked layout for k_pr_bseg_loop (once per graph):
// stable radix sort of the CSC edges by source block (CSC order kept inside a
// block), each block padded to whole tiles, run heads where a row starts or
// its source block changes, run -> row, first run of every tile.
template <class OffT> static gr_status pr_bseg_setup(gr_graph *g, uint32_t S) {
  const HostGraph &H = g->H;
  cudaStream_t s = g->stream;
  const uint32_t rows = (uint32_t)H.own_n();
  const uint64_t m = H.m_in;
  const OffT *in_off = (const OffT *)g->in_off;
  const uint32_t B = (uint32_t)((H.n + S - 1) / S);
  int end_bit = 1;
  while ((1ull << end_bit) < B) end_bit++;
  uint32_t *k0 = nullptr, *k1 = nullptr, *v0 = nullptr, *v1 = nullptr, *rowbits = nullptr;
  uint64_t *bstart = nullptr, *pstart = nullptr;
  void *tmp = nullptr;
  size_t need = 0;
  auto cleanup = [&] {
    pfree(k0, s); pfree(k1, s); pfree(v0, s); pfree(v1, s); pfree(rowbits, s); pfree(bstart, s); pfree(pstart, s);
    pfree(tmp, s);
  };
  if (pmalloc(&k0, 4 * m, s) != cudaSuccess || pmalloc(&k1, 4 * m, s) != cudaSuccess ||
      pmalloc(&v0, 4 * m, s) != cudaSuccess || pmalloc(&v1, 4 * m, s) != cudaSuccess ||
      pmalloc(&rowbits, 4 * (m / 32 + 2), s) != cudaSuccess || pmalloc(&bstart, 8ull * (B + 1), s) != cudaSuccess ||
      pmalloc(&pstart, 8ull * (B + 1), s) != cudaSuccess) {
    cleanup();
    return fail(GR_ENOMEM, "blocked PageRank layout: allocation failed");
  }
  k_bseg_key<<<g->num_sms * 16, 256, 0, s>>>(g->in_src, m, S, k0, v0);
  cub::DoubleBuffer<uint32_t> kk(k0, k1), vv(v0, v1);
  CK(cub::DeviceRadixSort::SortPairs(nullptr, need, kk, vv, (int64_t)m, 0, end_bit, s));
  if (pmalloc(&tmp, std::max<size_t>(need, 16), s) != cudaSuccess) {
    cleanup();
    return fail(GR_ENOMEM, "blocked PageRank layout: sort temp allocation failed");
  }
  CK(cub::DeviceRadixSort::SortPairs(tmp, need, kk, vv, (int64_t)m, 0, end_bit, s));
  k_bseg_bounds<<<g->num_sms * 16, 256, 0, s>>>(kk.Current(), m, B, bstart);
  std::vector<uint64_t> hb(B + 1), hp(B + 1);
  CK(cudaMemcpyAsync(hb.data(), bstart, 8ull * (B + 1), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  std::vector<uint32_t> hbt(B + 1);
  hp[0] = 0;
  for (uint32_t b = 0; b < B; b++) {
    const uint64_t c = hb[b + 1] - hb[b];
    hp[b + 1] = hp[b] + (c + kSegTile - 1) / kSegTile * kSegTile;
    hbt[b] = (uint32_t)(hp[b] / kSegTile);
  }
  hbt[B] = (uint32_t)(hp[B] / kSegTile);
  const uint64_t P = hp[B];
  if (P + kSegTile >= 0xFFFFFFFFull) {
    cleanup();
    return fail(GR_EUNSUPPORTED, "blocked PageRank layout: %llu items exceed 32-bit item indices",
                (unsigned long long)P);
  }
  CK(cudaMemcpyAsync(pstart, hp.data(), 8ull * (B + 1), cudaMemcpyHostToDevice, s));
  gr_status st;
  if ((st = dev_alloc(g, (void **)&g->b_items, 4 * P + 16)) != GR_OK) { cleanup(); return st; }
  if ((st = dev_alloc(g, (void **)&g->b_flags, 4 * (P / 32 + 16))) != GR_OK) { cleanup(); return st; }
  if ((st = dev_alloc(g, (void **)&g->b_blk_tile, 4ull * (B + 1))) != GR_OK) { cleanup(); return st; }
  if ((st = dev_alloc(g, (void **)&g->b_acc, 4ull * std::max<uint32_t>(rows, 1))) != GR_OK) { cleanup(); return st; }
  CK(cudaMemcpyAsync(g->b_blk_tile, hbt.data(), 4ull * (B + 1), cudaMemcpyHostToDevice, s));
  CK(cudaMemsetAsync(g->b_acc, 0, 4ull * rows, s));
  uint32_t *head = nullptr, *runidx = nullptr;
  if (pmalloc(&head, 4 * P + 4, s) != cudaSuccess || pmalloc(&runidx, 4 * P + 4, s) != cudaSuccess) {
    pfree(head, s); pfree(runidx, s);
    cleanup();
    return fail(GR_ENOMEM, "blocked PageRank layout: head allocation failed");
  }
  k_fill_u32<<<g->num_sms * 8, 256, 0, s>>>(g->b_items, kHotTag | g->hot_k, P);  // padding reads the zero slot
  CK(cudaMemsetAsync(head, 0, 4 * P + 4, s));
  CK(cudaMemsetAsync(rowbits, 0, 4 * (m / 32 + 2), s));
  k_bseg_rowstart<OffT><<<g->num_sms * 8, 256, 0, s>>>(in_off, rows, rowbits);
  k_bseg_place<<<g->num_sms * 16, 256, 0, s>>>(kk.Current(), vv.Current(), m, bstart, pstart, g->in_src, g->pr_src, S,
                                               rowbits, g->b_items, head);
  k_bseg_flags<<<g->num_sms * 8, 256, 0, s>>>(head, P, g->b_flags);
  pfree(tmp, s);
  tmp = nullptr;
  CK(cub::DeviceScan::ExclusiveSum(nullptr, need, head, runidx, (int64_t)P + 1, s));
  CK(pmalloc(&tmp, std::max<size_t>(need, 16), s));
  CK(cub::DeviceScan::ExclusiveSum(tmp, need, head, runidx, (int64_t)P + 1, s));
  uint32_t nruns = 0;
  CK(cudaMemcpyAsync(&nruns, runidx + P, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  uint32_t *run_off = nullptr;
  if ((st = dev_alloc(g, (void **)&g->b_run_row, 4ull * (nruns + 64))) != GR_OK) { pfree(head, s); pfree(runidx, s); cleanup(); return st; }
  CK(pmalloc(&run_off, 4ull * (nruns + 1), s));
  k_bseg_runs<OffT><<<g->num_sms * 16, 256, 0, s>>>(kk.Current(), vv.Current(), m, bstart, pstart, head, runidx,
                                                    in_off, rows, run_off, g->b_run_row);
  const uint32_t Pu = (uint32_t)P;
  CK(cudaMemcpyAsync(run_off + nruns, &Pu, 4, cudaMemcpyHostToDevice, s));
  g->b_tiles = (uint32_t)(P / kSegTile);
  if ((st = dev_alloc(g, (void **)&g->b_tile_run, 4ull * (g->b_tiles + 1))) != GR_OK) { pfree(head, s); pfree(runidx, s); pfree(run_off, s); cleanup(); return st; }
  uint32_t *d_nlong = nullptr;
  CK(pmalloc(&d_nlong, 4, s));
  CK(cudaMemsetAsync(d_nlong, 0, 4, s));
  k_seg_tiles<<<(g->b_tiles + 255) / 256 + 1, 256, 0, s>>>(run_off, nruns, g->b_tiles, g->b_tile_run, g->w_is_long,
                                                            g->long_c, g->long_f, d_nlong);
  CK(cudaGetLastError());
  CK(cudaMemcpyAsync(&g->n_long, d_nlong, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  pfree(d_nlong, s);
  pfree(run_off, s);
  pfree(head, s);
  pfree(runidx, s);
  cleanup();
  g->b_nblk = B;
  g->b_nruns = nruns;
  g->b_S = S;
  return GR_OK;
}

// Hot-source setup (once per graph): pick the K vertices of largest
// out-degree (the sources of the most in-edges), tag them in a PageRank copy
// of the CSC payload, size the persistent grid from the occupancy calculator.
template <class OffT> static gr_status pr_hot_setup(gr_graph *g) {
  g->pr_hot = 0;
  const HostGraph &H = g->H;
  uint64_t hot_min = 1u << 20;  // below ~1M edges the plain warp kernel is as fast
  if (const char *hm = getenv("GR_PR_HOT_MIN_EDGES")) hot_min = strtoull(hm, nullptr, 10);  // tests
  const bool hot_ok = g->mode == GR_MODE_RESIDENT && H.n < 0x80000000ull && H.m_in >= hot_min && H.m_in > 0;
  const bool seg_ok = hot_ok && (uint64_t)H.own_n() + H.m_in + 2 * kSegTile < 0xFFFFFFFFull;
  // source block for the blocked layout: the contributions of one block must stay in L2
  uint64_t block_mb = 64;  // measured on R-MAT s26: 24 MB 4.81, 40 MB 4.52, 64 MB 4.42 ms per superstep
  if (const char *bm = getenv("GR_PR_BLOCK_MB")) block_mb = std::max<uint64_t>(1, strtoull(bm, nullptr, 10));
  uint32_t S = (uint32_t)std::max<uint64_t>(1024, (block_mb << 20) / 4 / 32 * 32);
  if (const char *bv = getenv("GR_PR_BLOCK_V")) S = (uint32_t)std::max<uint64_t>(32, strtoull(bv, nullptr, 10));  // tests
  const bool bseg_ok = seg_ok && !g->comm && H.n > S;
  // kernel (GR_PR_KERNEL = block | warp | warphot | seg | bseg): seg by default, bseg when the
  // contribution array is larger than one L2 block; warphot (hot table, merge-path warp tiles)
  // when the seg layout's 32-bit item indices would overflow, warp for ranks with < 1M
  // in-edges, block (CTA merge-path tiles) when no shared-memory table fits
  g->pr_kernel = bseg_ok ? 8 : seg_ok ? 7 : 3;
  if (const char *k = getenv("GR_PR_KERNEL")) {
    const std::string v(k);
    g->pr_kernel = v == "block" ? 0 : v == "warp" ? 2 : v == "warphot" ? 3 : v == "seg" ? 7 : v == "bseg" ? 8 : 7;
  }
  if (g->pr_kernel == 8 && !seg_ok) g->pr_kernel = hot_ok ? 3 : 2;
  if (g->pr_kernel == 3 && !hot_ok) g->pr_kernel = 2;
  if (g->pr_kernel == 7 && !seg_ok) g->pr_kernel = hot_ok ? 3 : 2;
  if (g->pr_kernel != 3 && g->pr_kernel != 7 && g->pr_kernel != 8) return GR_OK;
  // the seg kernels stage nothing in shared memory: their table can be ~2x larger
  uint64_t K = g->pr_kernel >= 7 ? kSegHotK : kHotK;
  if (const char *hk = getenv("GR_PR_HOTK")) K = std::max<uint64_t>(4, std::min<uint64_t>(strtoull(hk, nullptr, 10), 57344));
  K = std::min<uint64_t>(K, H.n);
  uint32_t *d_slot = nullptr;
  gr_status s;
  if ((s = select_hot(g, K, &g->hot_ids, &g->hot_k, &d_slot)) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->hot_contrib, 4ull * std::max<uint32_t>(g->hot_k, 4))) != GR_OK) return s;
  if ((s = dev_alloc(g, (void **)&g->pr_src, 4 * (H.m_in + 4))) != GR_OK) return s;
  k_pr_tag<<<g->num_sms * 8, 256, 0, g->stream>>>(g->in_src, H.m_in, d_slot, g->pr_src);
  CK(cudaGetLastError());
  CK(cudaStreamSynchronize(g->stream));
  int bps = 0;
  if (g->pr_kernel == 8) {
    if (!g->coop) return fail(GR_EUNSUPPORTED, "blocked PageRank needs cooperative launch");
    if ((s = pr_bseg_setup<OffT>(g, S)) != GR_OK) return s;
    g->hot_cta = 1024;
    g->hot_smem = 4ull * (g->hot_k + 4) + 4ull * 64 * (g->hot_cta / 32);
    g->b_pol = 1;
    if (const char *bp = getenv("GR_PR_BLOCK_POLICY")) g->b_pol = atoi(bp) != 0;
    for (auto kf : {(const void *)k_pr_bseg_loop<OffT, 0>, (const void *)k_pr_bseg_loop<OffT, 1>})
      CK(cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->hot_smem));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_pr_bseg_loop<OffT, 1>, g->hot_cta, g->hot_smem));
    if (bps < 1) return fail(GR_EUNSUPPORTED, "blocked PageRank kernel does not fit on an SM");
    bps = 1;
    g->pr_loop = 1;
  } else if (g->pr_kernel == 7) {
    if ((s = pr_seg_setup<OffT>(g)) != GR_OK) return s;
    g->hot_cta = 1024;
    g->seg_var = kSegDefaultVar;
    // the table plus (kSegBuf) 32 floats per warp; what is left of the SM's 256 KB is L1
    g->hot_smem = 4ull * (g->hot_k + 4) + ((g->seg_var & kSegBuf) ? 4ull * 32 * (g->hot_cta / 32) : 0);
    CK(cudaFuncSetAttribute(seg_kernel<OffT>(g->seg_var), cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)g->hot_smem));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, seg_kernel<OffT>(g->seg_var), g->hot_cta, g->hot_smem));
    // persistent loop: one cooperative launch for all supersteps (GR_PR_LOOP=0: one launch per phase)
    g->pr_loop = g->coop ? 1 : 0;
    if (const char *pl = getenv("GR_PR_LOOP")) g->pr_loop = g->coop && atoi(pl) != 0;
    if (g->comm) g->pr_loop = 0;  // partitioned: one launch per phase, the exchange between supersteps
    if (g->pr_loop) {
      // the item and head-bit streams by TMA bulk copies into two staging buffers per
      // warp (GR_PR_TMA=0: 128-bit loads through L1)
      // measured slower (tiles phase 314 vs 173 us per superstep on cfg2, profiles/README.md):
      // opt-in with GR_PR_TMA=1
      g->pr_tma = false;
      if (const char *e = getenv("GR_PR_TMA")) g->pr_tma = atoi(e) != 0;
      g->tma_off = (uint32_t)((g->hot_smem + 127) / 128 * 128);
      g->loop_smem = g->pr_tma ? g->tma_off + (g->hot_cta / 32) * (2 * kTmaBufBytes + 16) : g->hot_smem;
      int lbps = 0;
      CK(cudaFuncSetAttribute(seg_loop_kernel<OffT>(g->seg_var, false, g->pr_tma),
                              cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->loop_smem));
      CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&lbps, seg_loop_kernel<OffT>(g->seg_var, false, g->pr_tma),
                                                       g->hot_cta, g->loop_smem));
      if (lbps < 1 && g->pr_tma) {  // does not fit next to the table: the load path
        g->pr_tma = false;
        g->loop_smem = g->hot_smem;
        CK(cudaFuncSetAttribute(seg_loop_kernel<OffT>(g->seg_var), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)g->loop_smem));
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&lbps, seg_loop_kernel<OffT>(g->seg_var), g->hot_cta,
                                                         g->loop_smem));
      }
      if (lbps < 1) g->pr_loop = 0;
    }
    if (g->pr_loop) {
      g->hot_slot = d_slot;
      if ((s = dev_alloc(g, (void **)&g->hot_split, g->hot_k + 16)) != GR_OK) return s;
      for (int i = 0; i < 2; i++)
        if ((s = dev_alloc(g, (void **)&g->hot_buf[i], 4ull * (g->hot_k + 4))) != GR_OK) return s;
      if ((s = dev_alloc(g, (void **)&g->pr_bar, 64)) != GR_OK) return s;
      CK(cudaMemsetAsync(g->pr_bar, 0, 64, g->stream));
      k_seg_hot_split<<<(g->hot_k + 255) / 256 + 1, 256, 0, g->stream>>>(g->hot_ids, g->hot_k, g->seg_off,
                                                                         g->hot_split);
      CK(cudaGetLastError());
      CK(cudaStreamSynchronize(g->stream));
    }
  } else {
    g->hot_cta = 1024;
    g->hot_smem = 4ull * g->hot_k + (g->hot_cta / 32) * sizeof(PrWarpSmem);
    CK(cudaFuncSetAttribute(k_pr_warp_hot<OffT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->hot_smem));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, k_pr_warp_hot<OffT>, g->hot_cta, g->hot_smem));
  }
  if (bps < 1) {
    g->pr_kernel = 0;  // shared-memory table does not fit: CTA merge-path kernel
    return GR_OK;
  }
  g->hot_grid = (uint32_t)(g->num_sms * bps);
  g->pr_hot = 1;
  return GR_OK;
}

template <class OffT>
static void pr_launch_iter(gr_graph *g, cudaStream_t s, uint32_t t, uint32_t iters, float d, cudaEvent_t e0,
                           cudaEvent_t e1) {
  PrArgs<OffT> a = pr_args<OffT>(g, t, iters, d);
  const bool warp = g->pr_kernel >= 2;
  if (warp) a.tile_row = g->wtile_row;
  const uint32_t tiles = g->pr_kernel == 7 ? g->seg_tiles : warp ? g->pr_wtiles : g->pr_tiles;
  if (g->pr_hot == 1) {
    k_pr_hot_pack<<<(g->hot_k + 255) / 256, 256, 0, s>>>(a.contrib_in, g->hot_ids, g->hot_contrib, g->hot_k);
    a.in_src = g->pr_src;
  }
  if (e0) cudaEventRecord(e0, s);
  switch (g->pr_kernel) {
    case 0:
      k_pr_gather_apply<OffT><<<std::max<uint32_t>(tiles, 1), kPrThreads, 0, s>>>(a);
      break;
    case 3:
      k_pr_warp_hot<OffT><<<g->hot_grid, g->hot_cta, g->hot_smem, s>>>(a, g->hot_contrib, g->hot_k, tiles);
      break;
    case 7:
      seg_kernel<OffT>(g->seg_var)<<<g->hot_grid, g->hot_cta, g->hot_smem, s>>>(
          a, g->seg_src, g->seg_flags, g->seg_row, g->hot_contrib, g->hot_k, tiles);
      break;
    default:
      k_pr_warp<OffT><<<std::max<uint32_t>((tiles + 7) / 8, 1), 256, 0, s>>>(a, tiles);
  }
  if (e1) cudaEventRecord(e1, s);
  if (warp) {
    k_pr_fixup_short<OffT><<<std::max<uint32_t>((tiles + 255) / 256, 1), 256, 0, s>>>(a, tiles, g->w_is_long);
    if (g->n_long) k_pr_fixup_long<OffT><<<(g->n_long + 7) / 8, 256, 0, s>>>(a, g->long_c, g->long_f, g->n_long);
  }
  else
    k_pr_fixup<OffT><<<std::max<uint32_t>((tiles + 255) / 256, 1), 256, 0, s>>>(a, tiles);
}

// Partitioned PageRank (engine_part.cu): the same per-superstep kernels over the
// rank's owned rows (hot table + edge-segmented tiles when they apply).
gr_status pr_part_prepare(gr_graph *g) {
  if (g->pr_hot >= 0) return GR_OK;
  return g->off64 ? pr_hot_setup<uint64_t>(g) : pr_hot_setup<uint32_t>(g);
}
uint32_t pr_part_iter(gr_graph *g, cudaStream_t s, uint32_t t, uint32_t iters, float d) {
  if (g->off64) pr_launch_iter<uint64_t>(g, s, t, iters, d, nullptr, nullptr);
  else pr_launch_iter<uint32_t>(g, s, t, iters, d, nullptr, nullptr);
  const bool warp = g->pr_kernel >= 2;
  return (g->pr_hot == 1 ? 1u : 0u) + 2u + (warp && g->n_long ? 1u : 0u);
}

template <class OffT>
static gr_status run_pagerank(gr_graph *g, const gr_run_opts *o, cudaStream_t s, gr_run_stats *st) {
  const uint32_t iters = o->max_iters;
  const float d = o->damping;
  const int prof = o->profile ? 1 : 0;
  if (g->pr_hot < 0) {
    tmark("pagerank: before hot setup");
    gr_status hs = pr_hot_setup<OffT>(g);
    if (hs != GR_OK) return hs;
    tmark("pagerank: hot setup");
  }
  if (prof && g->prof_ev.size() < 2 * (size_t)iters + 2) {
    while (g->prof_ev.size() < 2 * (size_t)iters + 2) {
      cudaEvent_t e;
      CK(cudaEventCreate(&e));
      g->prof_ev.push_back(e);
    }
  }
  if (g->pr_kernel == 8) {
    // source-blocked persistent loop (f3): init, first hot-table pack, ONE cooperative launch
    if (!g->hot_buf[0]) {
      for (int i = 0; i < 2; i++) {
        gr_status s2 = dev_alloc(g, (void **)&g->hot_buf[i], 4ull * (g->hot_k + 4));
        if (s2 != GR_OK) return s2;
      }
      gr_status s2 = dev_alloc(g, (void **)&g->pr_bar, 64);
      if (s2 != GR_OK) return s2;
      CK(cudaMemsetAsync(g->pr_bar, 0, 64, s));
    }
    PrArgs<OffT> a = pr_args<OffT>(g, 0, iters, d);
    PrBlk L{};
    L.items = g->b_items;
    L.flags = g->b_flags;
    L.tile_run = g->b_tile_run;
    L.run_row = g->b_run_row;
    L.blk_tile = g->b_blk_tile;
    L.nblk = g->b_nblk;
    L.nruns = g->b_nruns;
    L.num_tiles = g->b_tiles;
    L.iters = iters;
    L.acc = g->b_acc;
    L.hot_ids = g->hot_ids;
    L.hot_buf[0] = g->hot_buf[0];
    L.hot_buf[1] = g->hot_buf[1];
    L.contrib[0] = g->contrib[0];
    L.contrib[1] = g->contrib[1];
    L.is_long = g->w_is_long;
    L.long_c = g->long_c;
    L.long_f = g->long_f;
    L.n_long = g->n_long;
    L.hot_k = g->hot_k;
    L.bar = g->pr_bar;
    k_pr_init<<<g->num_sms * 4, 256, 0, s>>>((uint32_t)g->H.n, g->inv_outdeg, g->contrib[0], g->pr_bar);
    k_pr_hot_pack<<<(g->hot_k + 255) / 256, 256, 0, s>>>(g->contrib[0], g->hot_ids, g->hot_buf[0], g->hot_k);
    if (prof) CK(cudaEventRecord(g->prof_ev[0], s));
    void *args[] = {(void *)&a, (void *)&L};
    const void *kf = g->b_pol ? (const void *)k_pr_bseg_loop<OffT, 1> : (const void *)k_pr_bseg_loop<OffT, 0>;
    CK(cudaLaunchCooperativeKernel(kf, dim3(g->hot_grid), dim3(g->hot_cta), args, g->hot_smem, s));
    if (prof) CK(cudaEventRecord(g->prof_ev[1], s));
    CK(cudaStreamSynchronize(s));
    if (prof) {
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, g->prof_ev[0], g->prof_ev[1]));
      st->kernel_ms[0] += ms;
    }
    st->kernel_launches += 3;
  } else if (g->pr_kernel == 7 && g->pr_loop) {
    // persistent loop: init, pack of the first hot table, ONE cooperative launch for all supersteps
    PrArgs<OffT> a = pr_args<OffT>(g, 0, iters, d);
    PrLoop L{};
    L.seg_src = g->seg_src;
    L.seg_flags = g->seg_flags;
    L.seg_row = g->seg_row;
    L.hot_ids = g->hot_ids;
    L.hot_slot = g->hot_slot;
    L.hot_split = g->hot_split;
    L.hot_buf[0] = g->hot_buf[0];
    L.hot_buf[1] = g->hot_buf[1];
    L.contrib[0] = g->contrib[0];
    L.contrib[1] = g->contrib[1];
    L.is_long = g->w_is_long;
    L.long_c = g->long_c;
    L.long_f = g->long_f;
    L.n_long = g->n_long;
    L.hot_k = g->hot_k;
    L.num_tiles = g->seg_tiles;
    L.iters = iters;
    L.bar = g->pr_bar;
    L.tma_off = g->tma_off;
    // GR_PR_PHASES=1: per-superstep split of the loop (tiles vs fix-ups + pack + barriers),
    // stamped with %globaltimer by CTA 0 after each grid barrier, printed on stderr
    static const bool phases = getenv("GR_PR_PHASES") && atoi(getenv("GR_PR_PHASES")) != 0;
    unsigned long long *d_ts = nullptr;
    if (phases) CK(cudaMallocAsync((void **)&d_ts, 8ull * (2 * iters + 1), s));
    L.ts = d_ts;
    k_pr_init<<<g->num_sms * 4, 256, 0, s>>>((uint32_t)g->H.n, g->inv_outdeg, g->contrib[0], g->pr_bar);
    k_pr_hot_pack<<<(g->hot_k + 255) / 256, 256, 0, s>>>(g->contrib[0], g->hot_ids, g->hot_buf[0], g->hot_k);
    if (prof) CK(cudaEventRecord(g->prof_ev[0], s));
    void *args[] = {(void *)&a, (void *)&L};
    if (phases)
      CK(cudaFuncSetAttribute(seg_loop_kernel<OffT>(g->seg_var, true, g->pr_tma),
                              cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g->loop_smem));
    CK(cudaLaunchCooperativeKernel((const void *)seg_loop_kernel<OffT>(g->seg_var, phases, g->pr_tma),
                                   dim3(g->hot_grid), dim3(g->hot_cta), args, g->loop_smem, s));
    if (prof) CK(cudaEventRecord(g->prof_ev[1], s));
    CK(cudaStreamSynchronize(s));
    if (phases) {
      std::vector<unsigned long long> ts(2 * iters + 1);
      CK(cudaMemcpy(ts.data(), d_ts, 8 * ts.size(), cudaMemcpyDeviceToHost));
      CK(cudaFreeAsync(d_ts, s));
      double p1 = 0, p2 = 0;
      for (uint32_t t = 0; t < iters; t++) {
        p1 += (double)(ts[1 + 2 * t] - ts[2 * t]);
        p2 += (double)(ts[2 + 2 * t] - ts[1 + 2 * t]);
      }
      fprintf(stderr, "[gr] k_pr_seg_loop phases per superstep: tiles %.2f us, fix-ups + pack + barriers %.2f us "
              "(%u supersteps)\n", p1 / iters / 1e3, p2 / iters / 1e3, iters);
    }
    if (prof) {
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, g->prof_ev[0], g->prof_ev[1]));
      st->kernel_ms[0] += ms;
    }
    st->kernel_launches += 3;
  } else if (prof) {
    // direct launches with a CUDA event pair around every gather launch (events
    // recorded inside a captured graph cannot be timed); the host enqueues all
    // 2*iters launches without waiting, so the device runs them back to back
    k_pr_init<<<g->num_sms * 4, 256, 0, s>>>((uint32_t)g->H.n, g->inv_outdeg, g->contrib[0]);
    for (uint32_t t = 0; t < iters; t++)
      pr_launch_iter<OffT>(g, s, t, iters, d, g->prof_ev[2 + 2 * t], g->prof_ev[3 + 2 * t]);
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(s));
    for (uint32_t t = 0; t < iters; t++) {
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, g->prof_ev[2 + 2 * t], g->prof_ev[3 + 2 * t]));
      st->kernel_ms[0] += ms;
    }
  } else {
    // one CUDA graph per (iters, damping): 2 launches per superstep
    if (!g->pr_exec || g->pr_exec_iters != iters || g->pr_exec_d != d) {
      if (g->pr_exec) { cudaGraphExecDestroy(g->pr_exec); g->pr_exec = nullptr; }
      cudaStream_t cs;
      CK(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
      CK(cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal));
      k_pr_init<<<g->num_sms * 4, 256, 0, cs>>>((uint32_t)g->H.n, g->inv_outdeg, g->contrib[0]);
      for (uint32_t t = 0; t < iters; t++) pr_launch_iter<OffT>(g, cs, t, iters, d, nullptr, nullptr);
      cudaGraph_t graph;
      cudaError_t e = cudaStreamEndCapture(cs, &graph);
      cudaStreamDestroy(cs);
      if (e != cudaSuccess) return fail(GR_ECUDA, "PageRank graph capture failed: %s", cudaGetErrorString(e));
      CK(cudaGraphInstantiate(&g->pr_exec, graph, 0));
      CK(cudaGraphDestroy(graph));
      g->pr_exec_iters = iters;
      g->pr_exec_d = d;
    }
    tmark("pagerank: graph ready");
    CK(cudaGraphLaunch(g->pr_exec, s));
    CK(cudaStreamSynchronize(s));
    tmark("pagerank: 30 supersteps");
  }
  st->iterations = iters;
  st->edges_gathered = (uint64_t)iters * g->H.m_in;
  st->edges_scattered = 0;
  const bool loop = (g->pr_kernel == 7 && g->pr_loop) || g->pr_kernel == 8;
  if (!loop) st->kernel_launches += 1 + (g->pr_hot == 1 ? 3ull : 2ull) * iters;
  st->kernel_ms[3] = (double)g->pr_kernel;  // which PageRank gather variant ran (0 block .. 7 seg, 8 blocked seg)
  st->kernel_ms[2] = loop ? 1.0 : 0.0;      // 1: persistent loop (kernel_ms[0] = whole loop)
  st->bytes_hbm_model = (uint64_t)iters * (4 * g->H.m_in + 12 * g->H.own_n() + 4 * g->H.n);
  g->trace_rows = iters;
  return GR_OK;
}

gr_status run(gr_graph *g, const gr_run_opts *oin, gr_run_stats *st) {
  gr_run_opts o = *oin;
  if (o.damping == 0.f) o.damping = 0.85f;
  if (o.algo == GR_PAGERANK && o.max_iters == 0) o.max_iters = 30;
  if ((o.algo == GR_PAGERANK || o.algo == GR_PAGERANK_DELTA) && !(o.damping > 0.f && o.damping < 1.f))
    return fail(GR_EINVAL, "damping must lie in (0, 1)");
  if (o.algo == GR_PAGERANK_DELTA && !(o.tolerance >= 0.f)) return fail(GR_EINVAL, "tolerance must be >= 0");
  if ((o.algo == GR_BFS || o.algo == GR_SSSP) && o.source >= g->H.n)
    return fail(GR_EINVAL, "source %u >= num_vertices %llu", o.source, (unsigned long long)g->H.n);
  if (o.algo == GR_SSSP && !g->H.has_w) return fail(GR_EINVAL, "SSSP needs edge weights");
  if (o.algo < GR_BFS || o.algo > GR_PAGERANK_DELTA) return fail(GR_EINVAL, "unknown algo %d", o.algo);
  if (o.direction < GR_DIR_AUTO || o.direction > GR_DIR_FUSED) return fail(GR_EINVAL, "unknown direction %d", o.direction);
  // one-directional streamed layouts (GR_FMT_SORTED with only one half): PageRank
  // needs the in-CSC alone, BFS the out-CSR alone, every other program both
  if (!g->H.has_in || !g->H.has_out) {
    const bool ok = (o.algo == GR_PAGERANK && g->H.has_in) || (o.algo == GR_BFS && g->H.has_out);
    if (!ok)
      return fail(GR_EUNSUPPORTED, "the graph was loaded with only its %s: algo %d needs %s",
                  g->H.has_in ? "in-CSC" : "out-CSR", o.algo, o.algo == GR_PAGERANK ? "the in-CSC" :
                  o.algo == GR_BFS ? "the out-CSR" : "both directions");
  }
  if (o.trace_detail && (g->mode == GR_MODE_STREAMED || g->comm))
    return fail(GR_EUNSUPPORTED, "trace_detail: resident single-rank graphs only");
  const JitProgram *jp = nullptr;
  if (o.algo == GR_CUSTOM) {
    bool known = false, uses_w = false;
#define GR_X(id, T) if (o.custom_id == id) { known = true; uses_w = T::kUsesWeights; }
    GR_CUSTOM_PROGRAMS(GR_X)
#undef GR_X
    if (!known && (jp = jit_find(o.custom_id))) {
      known = true;
      uses_w = jp->uses_weights;
      if (jp->device != g->device)
        return fail(GR_EINVAL, "run-time program %d was compiled on device %d; the graph lives on device %d "
                    "(compile it with that device current)", o.custom_id, jp->device, g->device);
      // resident single-GPU graphs run the program's persistent BSP loop; streamed and
      // partitioned graphs run their drivers with the program's kernel table (prog_desc.h)
      if (g->mode != GR_MODE_STREAMED && !g->comm) {
        if (!g->coop) return fail(GR_EUNSUPPORTED, "run-time program %d needs cooperative launch", o.custom_id);
        if (o.loop != GR_LOOP_AUTO && o.loop != GR_LOOP_PERSISTENT)
          return fail(GR_EUNSUPPORTED, "run-time program %d: resident graphs run the persistent loop only "
                      "(loop = auto or persistent)", o.custom_id);
      }
    }
    if (!known) return fail(GR_EUNSUPPORTED, "no custom program with id %d is registered", o.custom_id);
    if (uses_w && !g->H.has_w) return fail(GR_EINVAL, "custom program %d needs edge weights", o.custom_id);
    if (o.source >= g->H.n) return fail(GR_EINVAL, "source %u >= num_vertices", o.source);
  }
  if (o.algo == GR_PAGERANK_DELTA && !g->prd_div) {
    // exact divisor table (gr/program.cuh ProgPRDelta::gatherMap), once per graph
    gr_status ds = dev_alloc(g, (void **)&g->prd_div, 16 * std::max<uint64_t>(g->H.n, 1));
    if (ds != GR_OK) return ds;
    k_prd_div<<<g->num_sms * 4, 256, 0, g->stream>>>(g->H.n, g->d_outdeg, g->prd_div);
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(g->stream));
  }
  if (o.algo != GR_PAGERANK) {  // every program but PageRank activates along the out-edges
    gr_status cs = ensure_csr(g);
    if (cs != GR_OK) return cs;
  }
  if (o.algo != GR_PAGERANK && o.algo != GR_BFS && g->mode == GR_MODE_RESIDENT && !g->comm && !g->rec_tried) {
    gr_status rs = g->off64 ? rec_setup<uint64_t>(g) : rec_setup<uint32_t>(g);
    if (rs != GR_OK) return rs;
  }
  if (g->mode == GR_MODE_STREAMED) return run_streamed(g, &o, st);
  cudaStream_t s = o.stream ? (cudaStream_t)o.stream : g->stream;
  CK(cudaEventRecord(g->ev_start, s));
  gr_status r;
  if (g->comm) {
    r = run_part(g, &o, s, st);
    if (r != GR_OK) return r;
    CK(cudaEventRecord(g->ev_stop, s));
    CK(cudaEventSynchronize(g->ev_stop));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, g->ev_start, g->ev_stop));
    st->seconds = ms * 1e-3;
    g->last_algo = o.algo;
    g->last_iters = st->iterations;
    return GR_OK;
  }
  switch (o.algo) {
    case GR_BFS:
      r = g->off64 ? run_frontier<ProgBFS, uint64_t>(g, &o, s, st, 0) : run_frontier<ProgBFS, uint32_t>(g, &o, s, st, 0);
      break;
    case GR_SSSP:
      r = g->off64 ? run_frontier<ProgSSSP, uint64_t>(g, &o, s, st, 1) : run_frontier<ProgSSSP, uint32_t>(g, &o, s, st, 1);
      break;
    case GR_CC:
      r = g->off64 ? run_frontier<ProgCC, uint64_t>(g, &o, s, st, 3) : run_frontier<ProgCC, uint32_t>(g, &o, s, st, 3);
      break;
    case GR_PAGERANK_DELTA:
      r = g->off64 ? run_frontier<ProgPRDelta, uint64_t>(g, &o, s, st, 5)
                   : run_frontier<ProgPRDelta, uint32_t>(g, &o, s, st, 5);
      break;
    case GR_CUSTOM:
      r = GR_EUNSUPPORTED;
      if (jp) r = g->off64 ? run_frontier_jit<uint64_t>(g, &o, s, st, jp) : run_frontier_jit<uint32_t>(g, &o, s, st, jp);
#define GR_X(id, T)                                                                                        \
  if (o.custom_id == id)                                                                                   \
    r = g->off64 ? run_frontier<T, uint64_t>(g, &o, s, st, 16 + id) : run_frontier<T, uint32_t>(g, &o, s, st, 16 + id);
      GR_CUSTOM_PROGRAMS(GR_X)
#undef GR_X
      break;
    default:
      r = g->off64 ? run_pagerank<uint64_t>(g, &o, s, st) : run_pagerank<uint32_t>(g, &o, s, st);
  }
  if (r != GR_OK) return r;
  CK(cudaEventRecord(g->ev_stop, s));
  CK(cudaEventSynchronize(g->ev_stop));
  float ms = 0;
  CK(cudaEventElapsedTime(&ms, g->ev_start, g->ev_stop));
  st->seconds = ms * 1e-3;
  g->last_algo = o.algo;
  g->last_iters = st->iterations;
  g->last_detail = o.trace_detail != 0;
  if (o.algo == GR_PAGERANK) g->pr_trace_iters = o.max_iters;
  return GR_OK;
}

static __global__ void k_count_nonzero(const uint32_t *a, uint64_t n, unsigned long long *out) {
  unsigned long long c = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    c += a[i] != 0;
  for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(out, c);
}

gr_status fetch_trace_detail(gr_graph *g, uint64_t *dst, uint64_t max_rows, uint64_t *rows) {
  if (g->last_algo < 0 || !g->last_detail)
    return fail(GR_ESTATE, "gr_fetch_frontier_trace_detail: the last run did not record the detail columns");
  if (!rows || (max_rows && !dst)) return fail(GR_EINVAL, "null output");
  const uint64_t r = std::min<uint64_t>(g->trace_rows, max_rows);
  if (g->last_algo == GR_PAGERANK) {  // A_t = V: every shard active, every source with an out-edge read
    unsigned long long *d = nullptr, h = 0;
    CK(cudaMallocAsync((void **)&d, 8, g->stream));
    CK(cudaMemsetAsync(d, 0, 8, g->stream));
    k_count_nonzero<<<g->num_sms * 2, 256, 0, g->stream>>>(g->d_outdeg, g->H.n, d);
    CK(cudaMemcpyAsync(&h, d, 8, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaFreeAsync(d, g->stream));
    CK(cudaStreamSynchronize(g->stream));
    for (uint64_t t = 0; t < r; t++) {
      dst[2 * t] = g->H.num_shards();
      dst[2 * t + 1] = h;
    }
  } else if (r) {
    CK(cudaMemcpyAsync(dst, g->trace_det, 16 * r, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaStreamSynchronize(g->stream));
  }
  *rows = r;
  return GR_OK;
}

gr_status fetch_values(gr_graph *g, void *dst, uint64_t bytes) {
  if (g->last_algo < 0) return fail(GR_ESTATE, "gr_fetch_vertex_values before gr_run");
  if (!dst) return fail(GR_EINVAL, "host_dst is NULL");
  const uint64_t n = g->H.n;
  if (bytes < 4 * n) return fail(GR_EINVAL, "buffer of %llu bytes < 4*n = %llu", (unsigned long long)bytes,
                                 (unsigned long long)(4 * n));
  if (g->comm) return part_fetch_values(g, dst, bytes);
  CK(cudaMemcpyAsync(dst, g->last_algo == GR_PAGERANK ? (const void *)g->rank : (const void *)g->val, 4 * n,
                     cudaMemcpyDeviceToHost, g->stream));
  CK(cudaStreamSynchronize(g->stream));
  return GR_OK;
}

gr_status fetch_trace(gr_graph *g, uint64_t *dst, uint64_t max_rows, uint64_t *rows) {
  if (g->last_algo < 0) return fail(GR_ESTATE, "gr_fetch_frontier_trace before gr_run");
  if (!rows || (max_rows && !dst)) return fail(GR_EINVAL, "null output");
  if (g->comm) return part_fetch_trace(g, dst, max_rows, rows);
  const uint64_t r = std::min<uint64_t>(g->trace_rows, max_rows);
  if (g->last_algo == GR_PAGERANK) {
    for (uint64_t t = 0; t < r; t++) {
      dst[4 * t] = g->H.own_n();
      dst[4 * t + 1] = g->H.own_n();
      dst[4 * t + 2] = g->H.m_in;
      dst[4 * t + 3] = 0;
    }
  } else if (r) {
    CK(cudaMemcpyAsync(dst, g->trace, 32 * r, cudaMemcpyDeviceToHost, g->stream));
    CK(cudaStreamSynchronize(g->stream));
  }
  *rows = r;
  return GR_OK;
}

// Per-device cache of the per-graph handles (stream, 4 events, pinned Ctl block):
// a reload takes them back instead of creating them (e2e load path).
namespace {
struct Handles {
  cudaStream_t stream;
  cudaEvent_t ev[4];
  Ctl *h_ctl;
};
std::mutex g_handles_mu;
std::vector<Handles> g_handles[64];
}  // namespace

bool acquire_handles(gr_graph *g) {
  {
    std::lock_guard<std::mutex> lk(g_handles_mu);
    if (g->device >= 0 && g->device < 64 && !g_handles[g->device].empty()) {
      const Handles h = g_handles[g->device].back();
      g_handles[g->device].pop_back();
      g->stream = h.stream;
      g->ev_start = h.ev[0];
      g->ev_stop = h.ev[1];
      g->prof_ev = {h.ev[2], h.ev[3]};
      g->h_ctl = h.h_ctl;
      return true;
    }
  }
  if (cudaStreamCreateWithFlags(&g->stream, cudaStreamNonBlocking) != cudaSuccess ||
      cudaEventCreate(&g->ev_start) != cudaSuccess || cudaEventCreate(&g->ev_stop) != cudaSuccess ||
      cudaMallocHost((void **)&g->h_ctl, sizeof(Ctl)) != cudaSuccess)
    return false;
  for (int i = 0; i < 2; i++) {
    cudaEvent_t e;
    if (cudaEventCreate(&e) != cudaSuccess) return false;
    g->prof_ev.push_back(e);
  }
  return true;
}

static void release_handles(gr_graph *g) {
  if (g->stream && g->ev_start && g->ev_stop && g->h_ctl && g->prof_ev.size() >= 2 && g->device >= 0 &&
      g->device < 64) {
    Handles h{g->stream, {g->ev_start, g->ev_stop, g->prof_ev[0], g->prof_ev[1]}, g->h_ctl};
    for (size_t i = 2; i < g->prof_ev.size(); i++) cudaEventDestroy(g->prof_ev[i]);
    std::lock_guard<std::mutex> lk(g_handles_mu);
    g_handles[g->device].push_back(h);
    return;
  }
  for (auto e : g->prof_ev) cudaEventDestroy(e);
  if (g->ev_start) cudaEventDestroy(g->ev_start);
  if (g->ev_stop) cudaEventDestroy(g->ev_stop);
  if (g->h_ctl) cudaFreeHost(g->h_ctl);
  if (g->stream) cudaStreamDestroy(g->stream);
}

void destroy(gr_graph *g) {
  if (!g) return;
  cudaSetDevice(g->device);
  cudaDeviceSynchronize();
  for (auto &kv : g->while_exec) cudaGraphExecDestroy(kv.second.first);
  if (g->pr_exec) cudaGraphExecDestroy(g->pr_exec);
  stream_destroy(g);
  delete g->comm;
  g->comm = nullptr;
  for (void *p : g->allocs) cudaFreeAsync(p, g->stream);
  for (void *p : g->plain_allocs) cudaFree(p);
  cudaStreamSynchronize(g->stream);
  if (g->h_xbytes) cudaFreeHost(g->h_xbytes);
  release_handles(g);  // stream, events, pinned Ctl back to the device's cache
  delete g;
}

}  // namespace gr
