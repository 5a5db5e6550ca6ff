// device_build.cu — the Shard Creator + Graph Layout Engine on the GPU
// (§4.2) for graphs that are resident in
// HBM. Produces exactly the layout of the host builder (host_graph.cpp): CSC
// sorted by (dst, src, w), CSR sorted by (src, dst), shard intervals of near-
// equal in+out degree — so every later step is unchanged. The host path is
// still used for streamed (out-of-core) and multi-rank graphs.
//
// Sorting uses CUB's LSD radix sort (a library primitive, stable): weights are
// ordered first, then the packed (major, minor) vertex key, which yields the
// (major, minor, w) order. Keys are packed into 2*b bits (b = bits(n)) so only
// the necessary digit passes run.
#include <cuda_runtime.h>

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <algorithm>
#include <vector>

#include "engine.h"

namespace gr {

#define DCK(call)                                                                              \
  do {                                                                                         \
    cudaError_t e_ = (call);                                                                   \
    if (e_ != cudaSuccess)                                                                     \
      return fail(e_ == cudaErrorMemoryAllocation ? GR_ENOMEM : GR_ECUDA, "%s: %s (%s:%d)", #call, \
                  cudaGetErrorString(e_), __FILE__, __LINE__);                                 \
  } while (0)

static __global__ void k_validate_count(const uint32_t *src, const uint32_t *dst, const uint32_t *w, uint64_t m,
                                        uint32_t n, uint32_t *bad, uint32_t *indeg, uint32_t *outdeg) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t s = src[e], d = dst[e];
    uint32_t b = 0;
    if (s >= n || d >= n) b |= 1;
    if (w && w[e] > 255u) b |= 2;
    if (b) {
      atomicOr(bad, b);
      continue;
    }
    atomicAdd(indeg + d, 1u);
    atomicAdd(outdeg + s, 1u);
  }
}

static __global__ void k_pack_keys(const uint32_t *major, const uint32_t *minor, uint64_t m, uint32_t bits,
                                   const uint32_t *perm, uint64_t *keys) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t i = perm ? perm[e] : e;
    keys[e] = ((uint64_t)major[i] << bits) | minor[i];
  }
}

static __global__ void k_iota_w8(const uint32_t *w, uint64_t m, uint8_t *w8, uint32_t *idx) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x) {
    w8[e] = (uint8_t)w[e];
    idx[e] = (uint32_t)e;
  }
}

static __global__ void k_gather_w8(const uint32_t *w, const uint32_t *perm, uint64_t m, uint8_t *out) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x)
    out[e] = (uint8_t)w[perm[e]];
}

static __global__ void k_unpack_minor(const uint64_t *keys, uint64_t m, uint32_t bits, uint32_t *out,
                                      uint32_t *major_out) {
  const uint64_t mask = (bits >= 32) ? 0xFFFFFFFFull : ((1ull << bits) - 1);
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t k = keys[e];
    out[e] = (uint32_t)(k & mask);
    if (major_out) major_out[e] = (uint32_t)(k >> bits);
  }
}

template <class OffT>
static __global__ void k_degree_to_off(const uint32_t *deg, uint64_t n, OffT *off) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v <= n; v += (uint64_t)gridDim.x * blockDim.x)
    off[v] = v < n ? (OffT)deg[v] : (OffT)0;
}

// hub bitmaps (degree > kHubDegree) and the static in-hub chunk list (CC's A_0)
template <class OffT>
static __global__ void k_hubs(const OffT *in_off, const OffT *out_off, uint64_t n, uint32_t *hub_in, uint32_t *hub_out,
                              unsigned long long *counts /* [hubs_in, chunks_in, hubs_out, chunks_out] */) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t di = (uint64_t)in_off[v + 1] - (uint64_t)in_off[v];
    const uint64_t dout = (uint64_t)out_off[v + 1] - (uint64_t)out_off[v];
    if (di > kHubDegree) {
      atomicOr(hub_in + (v >> 5), 1u << (v & 31));
      atomicAdd(counts + 0, 1ull);
      atomicAdd(counts + 1, (unsigned long long)((di + kChunk - 1) / kChunk));
    }
    if (dout > kHubDegree) {
      atomicOr(hub_out + (v >> 5), 1u << (v & 31));
      atomicAdd(counts + 2, 1ull);
      atomicAdd(counts + 3, (unsigned long long)((dout + kChunk - 1) / kChunk));
    }
  }
}

template <class OffT>
static __global__ void k_static_hubs(const OffT *in_off, uint64_t n, uint32_t *hubs, uint32_t *chk_h, uint32_t *chk_c,
                                     uint32_t *cnt /* [hubs, chunks] */) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t di = (uint64_t)in_off[v + 1] - (uint64_t)in_off[v];
    if (di <= kHubDegree) continue;
    const uint32_t pos = atomicAdd(cnt, 1u);
    hubs[pos] = (uint32_t)v;
    const uint32_t nch = (uint32_t)((di + kChunk - 1) / kChunk);
    const uint32_t kb = atomicAdd(cnt + 1, nch);
    for (uint32_t c = 0; c < nch; c++) {
      chk_h[kb + c] = pos;
      chk_c[kb + c] = c;
    }
  }
}

// Shard plan on the device (same rule as gr_plan_intervals over the weight
// prefix in_off[v] + out_off[v]): bound i = first v whose prefix reaches
// 2m*i/P. Writes [bounds | in_off at bounds | out_off at bounds], 3*(P+1).
template <class OffT>
static __global__ void k_plan_bounds(const OffT *in_off, const OffT *out_off, uint64_t n, uint32_t P, uint64_t *out) {
  const uint64_t total = (uint64_t)in_off[n] + (uint64_t)out_off[n];
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i <= P; i += gridDim.x * blockDim.x) {
    uint64_t v;
    if (i == 0) v = 0;
    else if (i == P) v = n;
    else {
      const uint64_t target = (uint64_t)(((unsigned __int128)total * i) / P);
      uint64_t lo = 0, hi = n + 1;  // lower_bound over [0, n]
      while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if ((uint64_t)in_off[mid] + (uint64_t)out_off[mid] < target) lo = mid + 1;
        else hi = mid;
      }
      v = lo > n ? n : lo;
    }
    out[i] = v;
    out[P + 1 + i] = (uint64_t)in_off[v];
    out[2 * (P + 1) + i] = (uint64_t)out_off[v];
  }
}

// one stable (major, minor[, w]) sort; returns sorted minor ids (+ weights)
static gr_status sort_edges(gr_graph *g, const uint32_t *major, const uint32_t *minor, const uint32_t *w, uint64_t m,
                            uint32_t bits, uint32_t *minor_out, uint8_t *w_out, uint32_t *major_out, cudaStream_t s) {
  const int gs = g->num_sms * 8;
  uint64_t *k0 = nullptr, *k1 = nullptr;
  uint32_t *perm0 = nullptr, *perm1 = nullptr;
  uint8_t *w0 = nullptr, *w1 = nullptr;
  void *tmp = nullptr;
  size_t tmp_bytes = 0, need = 0;
  gr_status st = GR_OK;
  auto cleanup = [&] {
    pfree(k0, s); pfree(k1, s); pfree(perm0, s); pfree(perm1, s); pfree(w0, s); pfree(w1, s); pfree(tmp, s);
  };
#define TRY(call)                                                                  \
  do {                                                                             \
    cudaError_t e_ = (call);                                                       \
    if (e_ != cudaSuccess) {                                                       \
      cleanup();                                                                   \
      return fail(e_ == cudaErrorMemoryAllocation ? GR_ENOMEM : GR_ECUDA,          \
                  "device build: %s: %s", #call, cudaGetErrorString(e_));          \
    }                                                                              \
  } while (0)
  const size_t mm = std::max<uint64_t>(m, 1);
  TRY(pmalloc(&k0, 8 * mm, s));
  TRY(pmalloc(&k1, 8 * mm, s));
  const int end_bit = (int)(2 * bits);
  if (w) {
    // pass 1: order by weight (stable), carrying the edge index
    TRY(pmalloc(&w0, mm, s));
    TRY(pmalloc(&w1, mm, s));
    TRY(pmalloc(&perm0, 4 * mm, s));
    TRY(pmalloc(&perm1, 4 * mm, s));
    k_iota_w8<<<gs, 256, 0, s>>>(w, m, w0, perm0);
    cub::DoubleBuffer<uint8_t> kw(w0, w1);
    cub::DoubleBuffer<uint32_t> vp(perm0, perm1);
    TRY(cub::DeviceRadixSort::SortPairs(nullptr, need, kw, vp, (int64_t)m, 0, 8, s));
    tmp_bytes = need;
    TRY(pmalloc(&tmp, std::max<size_t>(tmp_bytes, 16), s));
    TRY(cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, kw, vp, (int64_t)m, 0, 8, s));
    // pass 2: stable order by the packed vertex key, carrying the weight
    k_pack_keys<<<gs, 256, 0, s>>>(major, minor, m, bits, vp.Current(), k0);
    k_gather_w8<<<gs, 256, 0, s>>>(w, vp.Current(), m, w0);
    cub::DoubleBuffer<uint64_t> kk(k0, k1);
    cub::DoubleBuffer<uint8_t> vw(w0, w1);
    TRY(cub::DeviceRadixSort::SortPairs(nullptr, need, kk, vw, (int64_t)m, 0, end_bit, s));
    if (need > tmp_bytes) {
      pfree(tmp, s);
      tmp = nullptr;
      tmp_bytes = need;
      TRY(pmalloc(&tmp, tmp_bytes, s));
    }
    TRY(cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, kk, vw, (int64_t)m, 0, end_bit, s));
    k_unpack_minor<<<gs, 256, 0, s>>>(kk.Current(), m, bits, minor_out, major_out);
    if (w_out) TRY(cudaMemcpyAsync(w_out, vw.Current(), m, cudaMemcpyDeviceToDevice, s));
  } else {
    k_pack_keys<<<gs, 256, 0, s>>>(major, minor, m, bits, nullptr, k0);
    cub::DoubleBuffer<uint64_t> kk(k0, k1);
    TRY(cub::DeviceRadixSort::SortKeys(nullptr, need, kk, (int64_t)m, 0, end_bit, s));
    tmp_bytes = need;
    TRY(pmalloc(&tmp, std::max<size_t>(tmp_bytes, 16), s));
    TRY(cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, kk, (int64_t)m, 0, end_bit, s));
    k_unpack_minor<<<gs, 256, 0, s>>>(kk.Current(), m, bits, minor_out, major_out);
  }
  TRY(cudaStreamSynchronize(s));
  cleanup();
#undef TRY
  return st;
}

template <class OffT>
static gr_status scan_offsets(gr_graph *g, const uint32_t *deg, uint64_t n, OffT *off, cudaStream_t s) {
  k_degree_to_off<OffT><<<g->num_sms * 8, 256, 0, s>>>(deg, n, off);
  size_t need = 0;
  DCK(cub::DeviceScan::ExclusiveSum(nullptr, need, off, off, (int64_t)(n + 1), s));
  void *tmp = nullptr;
  DCK(pmalloc(&tmp, std::max<size_t>(need, 16), s));
  cudaError_t e = cub::DeviceScan::ExclusiveSum(tmp, need, off, off, (int64_t)(n + 1), s);
  cudaStreamSynchronize(s);
  pfree(tmp, s);
  if (e != cudaSuccess) return fail(GR_ECUDA, "device build scan: %s", cudaGetErrorString(e));
  return GR_OK;
}

// destination of every CSC position: the v with in_off[v] <= e < in_off[v+1]
template <class OffT>
static __global__ void k_csc_dst(const OffT *in_off, uint64_t n, uint64_t m, uint32_t *dst) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t lo = 0, hi = n;  // last v with in_off[v] <= e
    while (hi - lo > 1) {
      const uint64_t mid = (lo + hi) >> 1;
      if ((uint64_t)in_off[mid] <= e) lo = mid;
      else hi = mid;
    }
    dst[e] = (uint32_t)lo;
  }
}

// CSR (activation) = transpose of the CSC: a stable sort of the CSC's sources
// (32-bit keys, `bits` wide) carrying the destinations. The CSC is ordered by
// (dst, src, w), so each CSR segment comes out ordered by dst — the host
// builder's layout exactly (tests/test_gpu_parity.py).
template <class OffT> static gr_status build_csr(gr_graph *g) {
  const uint64_t n = g->H.n, m = g->H.m_in;
  cudaStream_t s = g->stream;
  uint32_t *d_dst = nullptr, *kscratch = nullptr;
  void *tmp = nullptr;
  size_t need = 0;
  DCK(pmalloc(&d_dst, 4 * std::max<uint64_t>(m, 1), s));
  DCK(pmalloc(&kscratch, 4 * std::max<uint64_t>(m, 1), s));
  k_csc_dst<OffT><<<g->num_sms * 8, 256, 0, s>>>((const OffT *)g->in_off, n, m, d_dst);
  DCK(cub::DeviceRadixSort::SortPairs(nullptr, need, g->in_src, kscratch, d_dst, g->out_dst, (int64_t)m, 0,
                                      (int)g->csr_bits, s));
  DCK(pmalloc(&tmp, std::max<size_t>(need, 16), s));
  DCK(cub::DeviceRadixSort::SortPairs(tmp, need, g->in_src, kscratch, d_dst, g->out_dst, (int64_t)m, 0,
                                      (int)g->csr_bits, s));
  pfree(tmp, s);
  pfree(kscratch, s);
  pfree(d_dst, s);
  DCK(cudaStreamSynchronize(s));
  g->csr_pending = false;
  tmark("device build: CSR sort (first run that activates)");
  return GR_OK;
}

gr_status ensure_csr(gr_graph *g) {
  if (!g->csr_pending) return GR_OK;
  return g->off64 ? build_csr<uint64_t>(g) : build_csr<uint32_t>(g);
}

template <class OffT>
static gr_status build_typed(gr_graph *g, const uint32_t *d_src, uint32_t *d_dst, const uint32_t *d_w,
                             uint64_t n, uint64_t m, uint32_t *d_indeg, uint32_t *d_outdeg, cudaStream_t s) {
  gr_status st;
  uint32_t bits = 1;
  while ((1ull << bits) < n) bits++;
  // CSC: (dst, src, w)
  if ((st = dev_alloc(g, (void **)&g->in_src, 4 * (m + 4))) != GR_OK) return st;
  DCK(cudaMemsetAsync(g->in_src + m, 0, 16, s));
  if (d_w) {
    if ((st = dev_alloc(g, (void **)&g->in_w, m + 16)) != GR_OK) return st;
    DCK(cudaMemsetAsync(g->in_w + m, 0, 16, s));
  }
  // the CSC sort leaves each edge's destination (in CSC order) in d_dst
  if ((st = sort_edges(g, d_dst, d_src, d_w, m, bits, g->in_src, d_w ? g->in_w : nullptr, d_dst, s)) != GR_OK)
    return st;
  tmark("device build: CSC sort");
  // The activation CSR's payload (out_dst) is built on the first run that needs
  // it (ensure_csr): PageRank eliminates FrontierActivate (L274) and never does,
  // so a load followed by PageRank skips one of the two sorts.
  if ((st = dev_alloc(g, (void **)&g->out_dst, 4 * (m + 4))) != GR_OK) return st;
  DCK(cudaMemsetAsync(g->out_dst + m, 0, 16, s));
  g->csr_pending = true;
  g->csr_bits = bits;
  // offsets
  if ((st = dev_alloc(g, &g->in_off, sizeof(OffT) * (n + 1))) != GR_OK) return st;
  if ((st = dev_alloc(g, &g->out_off, sizeof(OffT) * (n + 1))) != GR_OK) return st;
  if ((st = scan_offsets<OffT>(g, d_indeg, n, (OffT *)g->in_off, s)) != GR_OK) return st;
  if ((st = scan_offsets<OffT>(g, d_outdeg, n, (OffT *)g->out_off, s)) != GR_OK) return st;
  tmark("device build: offsets");
  // hubs
  const size_t words = (n + 31) / 32 + 1;
  if ((st = dev_alloc(g, (void **)&g->hub_in, 4 * words)) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&g->hub_out, 4 * words)) != GR_OK) return st;
  DCK(cudaMemsetAsync(g->hub_in, 0, 4 * words, s));
  DCK(cudaMemsetAsync(g->hub_out, 0, 4 * words, s));
  unsigned long long *d_cnt = nullptr;
  DCK(pmalloc(&d_cnt, 64, s));
  DCK(cudaMemsetAsync(d_cnt, 0, 64, s));
  k_hubs<OffT><<<g->num_sms * 8, 256, 0, s>>>((const OffT *)g->in_off, (const OffT *)g->out_off, n, g->hub_in,
                                                g->hub_out, d_cnt);
  unsigned long long cnt[4];
  DCK(cudaMemcpyAsync(cnt, d_cnt, 32, cudaMemcpyDeviceToHost, s));
  DCK(cudaStreamSynchronize(s));
  g->dev_hubs_in = cnt[0];
  g->dev_chunks_in = cnt[1];
  g->dev_hubs_out = cnt[2];
  g->dev_chunks_out = cnt[3];
  if ((st = dev_alloc(g, (void **)&g->static_hubs, 4 * std::max<uint64_t>(cnt[0], 1))) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&g->static_chk_h, 4 * std::max<uint64_t>(cnt[1], 1))) != GR_OK) return st;
  if ((st = dev_alloc(g, (void **)&g->static_chk_c, 4 * std::max<uint64_t>(cnt[1], 1))) != GR_OK) return st;
  DCK(cudaMemsetAsync(d_cnt, 0, 16, s));
  k_static_hubs<OffT><<<g->num_sms * 8, 256, 0, s>>>((const OffT *)g->in_off, n, g->static_hubs, g->static_chk_h,
                                                       g->static_chk_c, (uint32_t *)d_cnt);
  DCK(cudaStreamSynchronize(s));
  pfree(d_cnt, s);
  g->n_static_hubs = (uint32_t)cnt[0];
  g->n_static_chunks = (uint32_t)cnt[1];
  return GR_OK;
}

// Build the resident layout on the device from a host COO edge list.
gr_status device_build(gr_graph *g, const gr_edges *E, uint64_t shard_edges) {
  HostGraph &H = g->H;
  const uint64_t n = E->num_vertices, m = E->num_edges;
  cudaStream_t s = g->stream;
  uint32_t *d_src = nullptr, *d_dst = nullptr, *d_w = nullptr, *d_indeg = nullptr, *d_outdeg = nullptr,
           *d_bad = nullptr;
  auto cleanup = [&] {
    pfree(d_src, s); pfree(d_dst, s); pfree(d_w, s); pfree(d_indeg, s); pfree(d_bad, s);
  };
  const size_t mm = std::max<uint64_t>(m, 1);
  if (pmalloc(&d_src, 4 * mm, s) != cudaSuccess || pmalloc(&d_dst, 4 * mm, s) != cudaSuccess ||
      (E->weights && pmalloc(&d_w, 4 * mm, s) != cudaSuccess) || pmalloc(&d_indeg, 4 * n, s) != cudaSuccess ||
      pmalloc(&d_bad, 4, s) != cudaSuccess) {
    cudaGetLastError();
    cleanup();
    return fail(GR_ENOMEM, "device build: staging allocation failed");
  }
  gr_status st = dev_alloc(g, (void **)&d_outdeg, 4 * n);  // kept: PageRank out-degrees
  if (st != GR_OK) { cleanup(); return st; }
  cudaMemcpyAsync(d_src, E->src, 4 * m, cudaMemcpyHostToDevice, s);
  cudaMemcpyAsync(d_dst, E->dst, 4 * m, cudaMemcpyHostToDevice, s);
  if (E->weights) cudaMemcpyAsync(d_w, E->weights, 4 * m, cudaMemcpyHostToDevice, s);
  cudaMemsetAsync(d_indeg, 0, 4 * n, s);
  cudaMemsetAsync(d_outdeg, 0, 4 * n, s);
  cudaMemsetAsync(d_bad, 0, 4, s);
  k_validate_count<<<g->num_sms * 8, 256, 0, s>>>(d_src, d_dst, d_w, m, (uint32_t)n, d_bad, d_indeg, d_outdeg);
  uint32_t bad = 0;
  cudaMemcpyAsync(&bad, d_bad, 4, cudaMemcpyDeviceToHost, s);
  cudaError_t ce = cudaStreamSynchronize(s);
  tmark("device build: upload + validate");
  if (ce != cudaSuccess) { cleanup(); return fail(GR_ECUDA, "device build upload: %s", cudaGetErrorString(ce)); }
  if (bad & 1) { cleanup(); return fail(GR_EINVAL, "edge endpoint >= num_vertices"); }
  if (bad & 2) { cleanup(); return fail(GR_EINVAL, "edge weight > 255 (weights are stored as uint8)"); }
  g->off64 = (m >= 0xFFFFFFFFull);
  st = g->off64 ? build_typed<uint64_t>(g, d_src, d_dst, d_w, n, m, d_indeg, d_outdeg, s)
                : build_typed<uint32_t>(g, d_src, d_dst, d_w, n, m, d_indeg, d_outdeg, s);
  if (st != GR_OK) { cleanup(); return st; }
  tmark("device build: sorts + offsets + hubs");
  g->d_outdeg = d_outdeg;
  cleanup();
  // host-side metadata: only the shard plan (bounds and the offsets at them);
  // degrees and offsets stay on the device
  H.n = n;
  H.m_total = m;
  H.own_lo = 0;
  H.own_hi = n;
  H.owners = {0, n};
  H.m_in = m;
  H.has_w = E->weights != nullptr;
  if (shard_edges == 0) shard_edges = uint64_t(1) << 26;
  uint64_t P = (2 * m + shard_edges - 1) / shard_edges;
  P = std::max<uint64_t>(1, std::min<uint64_t>(P, std::min<uint64_t>(65535, n)));
  uint64_t *d_plan = nullptr;
  DCK(pmalloc(&d_plan, 24 * (P + 1), s));
  if (g->off64)
    k_plan_bounds<uint64_t><<<(unsigned)((P + 256) / 256), 256, 0, s>>>((const uint64_t *)g->in_off,
                                                                     (const uint64_t *)g->out_off, n, (uint32_t)P, d_plan);
  else
    k_plan_bounds<uint32_t><<<(unsigned)((P + 256) / 256), 256, 0, s>>>((const uint32_t *)g->in_off,
                                                                     (const uint32_t *)g->out_off, n, (uint32_t)P, d_plan);
  std::vector<uint64_t> plan(3 * (P + 1));
  cudaMemcpyAsync(plan.data(), d_plan, 24 * (P + 1), cudaMemcpyDeviceToHost, s);
  pfree(d_plan, s);
  ce = cudaStreamSynchronize(s);
  if (ce != cudaSuccess) return fail(GR_ECUDA, "device build: %s", cudaGetErrorString(ce));
  H.bounds.assign(plan.begin(), plan.begin() + (P + 1));
  H.bound_in.assign(plan.begin() + (P + 1), plan.begin() + 2 * (P + 1));
  H.bound_out.assign(plan.begin() + 2 * (P + 1), plan.end());
  const gr_status ps = GR_OK;
  tmark("device build: host metadata");
  return ps;
}

}  // namespace gr

namespace gr {

static __global__ void k_desc_key(const uint32_t *outdeg, uint64_t n, uint32_t *key, uint32_t *idx) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    key[v] = ~outdeg[v];  // ascending sort of ~deg = descending degree; stable => ties by ascending id
    idx[v] = (uint32_t)v;
  }
}

static __global__ void k_set_slots(const uint32_t *ids, uint32_t cnt, uint32_t *slot) {
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < cnt; k += gridDim.x * blockDim.x) slot[ids[k]] = k;
}

// The K vertices of largest out-degree (ties: smaller id first), with
// outdeg > 0, selected on the GPU: hot_ids (padded to a multiple of 4 with the
// first id) and a per-vertex slot table (0xFFFFFFFF = not hot).
gr_status select_hot(gr_graph *g, uint64_t K, uint32_t **hot_ids, uint32_t *hot_k, uint32_t **d_slot) {
  const uint64_t n = g->H.n;
  cudaStream_t s = g->stream;
  uint32_t *k0 = nullptr, *k1 = nullptr, *v0 = nullptr, *v1 = nullptr;
  void *tmp = nullptr;
  size_t need = 0;
  auto cleanup = [&] { pfree(k0, s); pfree(k1, s); pfree(v0, s); pfree(v1, s); pfree(tmp, s); };
  if (pmalloc(&k0, 4 * n, s) != cudaSuccess || pmalloc(&k1, 4 * n, s) != cudaSuccess ||
      pmalloc(&v0, 4 * n, s) != cudaSuccess || pmalloc(&v1, 4 * n, s) != cudaSuccess) {
    cleanup();
    return fail(GR_ENOMEM, "hot-set selection: allocation failed");
  }
  k_desc_key<<<g->num_sms * 8, 256, 0, s>>>(g->d_outdeg, n, k0, v0);
  cub::DoubleBuffer<uint32_t> kk(k0, k1), vv(v0, v1);
  cub::DeviceRadixSort::SortPairs(nullptr, need, kk, vv, (int64_t)n, 0, 32, s);
  if (pmalloc(&tmp, std::max<size_t>(need, 16), s) != cudaSuccess) {
    cleanup();
    return fail(GR_ENOMEM, "hot-set selection: temp allocation failed");
  }
  cub::DeviceRadixSort::SortPairs(tmp, need, kk, vv, (int64_t)n, 0, 32, s);
  std::vector<uint32_t> keys(K);
  cudaMemcpyAsync(keys.data(), kk.Current(), 4 * K, cudaMemcpyDeviceToHost, s);
  cudaError_t e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) {
    cleanup();
    return fail(GR_ECUDA, "hot-set selection: %s", cudaGetErrorString(e));
  }
  uint32_t cnt = 0;
  while (cnt < K && ~keys[cnt] > 0) cnt++;  // outdeg > 0
  *hot_k = (cnt + 3) & ~3u;
  gr_status st = dev_alloc(g, (void **)hot_ids, 4ull * std::max<uint32_t>(*hot_k, 4));
  if (st == GR_OK) st = dev_alloc(g, (void **)d_slot, 4 * n);
  if (st != GR_OK) {
    cleanup();
    return st;
  }
  cudaMemcpyAsync(*hot_ids, vv.Current(), 4ull * cnt, cudaMemcpyDeviceToDevice, s);
  for (uint32_t k = cnt; k < *hot_k; k++)  // pad with the first hot id (never tagged)
    cudaMemcpyAsync(*hot_ids + k, vv.Current(), 4, cudaMemcpyDeviceToDevice, s);
  cudaMemsetAsync(*d_slot, 0xFF, 4 * n, s);
  if (cnt) k_set_slots<<<(cnt + 255) / 256, 256, 0, s>>>(*hot_ids, cnt, *d_slot);
  e = cudaStreamSynchronize(s);
  cleanup();
  if (e != cudaSuccess) return fail(GR_ECUDA, "hot-set selection: %s", cudaGetErrorString(e));
  return GR_OK;
}

}  // namespace gr
