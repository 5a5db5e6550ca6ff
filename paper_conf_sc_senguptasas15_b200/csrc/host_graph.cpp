// host_graph.cpp — Shard Creator + Graph Layout Engine (§4.2).
// Multithreaded host build; the result is deterministic (independent of the
// thread count) because every segment is sorted by (neighbour, weight).
#include "host_graph.h"

#include <cuda_runtime_api.h>

#include <algorithm>
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <thread>

namespace gr {

HostBuf::~HostBuf() { release(); }

bool HostBuf::alloc(size_t nbytes) {
  release();
  size_t rounded = ((nbytes ? nbytes : 1) + 4095) & ~size_t(4095);
  p = std::aligned_alloc(4096, rounded);
  if (!p) return false;
  bytes = nbytes;
  return true;
}

void HostBuf::release() {
  if (registered) cudaHostUnregister(p);
  registered = false;
  if (owned) std::free(p);
  owned = true;
  p = nullptr;
  bytes = 0;
}

int default_threads() {
  unsigned h = std::thread::hardware_concurrency();
  return h ? (int)std::min(h, 64u) : 4;
}

// Static split of [0, n) over T threads.
template <class F> static void parallel_for(int T, uint64_t n, F f) {
  if (T <= 1 || n < 65536) {
    f(uint64_t(0), n);
    return;
  }
  std::vector<std::thread> th;
  uint64_t chunk = (n + T - 1) / T;
  for (int t = 0; t < T; t++) {
    uint64_t b = std::min<uint64_t>(n, chunk * t), e = std::min<uint64_t>(n, b + chunk);
    th.emplace_back([=] { f(b, e); });
  }
  for (auto &x : th) x.join();
}

// Dynamic chunks (for skewed per-vertex work such as hub segment sorts).
template <class F> static void parallel_for_dyn(int T, uint64_t n, uint64_t grain, F f) {
  std::atomic<uint64_t> next{0};
  auto body = [&] {
    for (;;) {
      uint64_t b = next.fetch_add(grain);
      if (b >= n) break;
      f(b, std::min(n, b + grain));
    }
  };
  if (T <= 1) {
    body();
    return;
  }
  std::vector<std::thread> th;
  for (int t = 0; t < T; t++) th.emplace_back(body);
  for (auto &x : th) x.join();
}

gr_status plan_owner_ranges(uint64_t n, const uint64_t *prefix, int world,
                            std::vector<uint64_t> *owners) {
  owners->assign(world + 1, 0);
  return gr_plan_intervals(n, prefix, (uint32_t)world, owners->data());
}

// Counting sort of the owned edges into segments keyed by `key` (dst for the
// CSC, src for the activation CSR), then sort each segment by (other, weight).
static void fill_segments(int T, uint64_t m, const uint32_t *key, const uint32_t *other,
                          const uint32_t *w, uint64_t key_lo, uint64_t key_n,
                          const uint32_t *dst_for_owner, uint64_t own_lo, uint64_t own_hi,
                          const std::vector<uint64_t> &off, uint32_t *idx_out, uint8_t *w_out) {
  const uint64_t total = off[key_n];
  std::vector<uint64_t> packed(total ? total : 1);
  std::vector<std::atomic<uint64_t>> cur(key_n ? key_n : 1);
  parallel_for(T, key_n, [&](uint64_t b, uint64_t e) {
    for (uint64_t i = b; i < e; i++) cur[i].store(off[i], std::memory_order_relaxed);
  });
  parallel_for(T, m, [&](uint64_t b, uint64_t e) {
    for (uint64_t i = b; i < e; i++) {
      uint32_t d = dst_for_owner[i];
      if (d < own_lo || d >= own_hi) continue;
      uint64_t k = key[i] - key_lo;
      uint64_t pos = cur[k].fetch_add(1, std::memory_order_relaxed);
      packed[pos] = ((uint64_t)other[i] << 8) | (w ? (w[i] & 0xFFu) : 0u);
    }
  });
  parallel_for_dyn(T, key_n, 4096, [&](uint64_t b, uint64_t e) {
    for (uint64_t v = b; v < e; v++) {
      uint64_t s = off[v], t = off[v + 1];
      if (t - s > 1) std::sort(packed.begin() + s, packed.begin() + t);
    }
  });
  parallel_for(T, total, [&](uint64_t b, uint64_t e) {
    for (uint64_t i = b; i < e; i++) {
      idx_out[i] = (uint32_t)(packed[i] >> 8);
      if (w_out) w_out[i] = (uint8_t)(packed[i] & 0xFF);
    }
  });
}

gr_status build_host_graph(const gr_edges *E, uint64_t shard_edges, int world, int rank,
                           int threads, HostGraph *G, std::string *err) {
  if (!E) { *err = "edges is NULL"; return GR_EINVAL; }
  const uint64_t n = E->num_vertices, m = E->num_edges;
  if (n == 0 || n >= 0xFFFFFFFFull) { *err = "num_vertices must be in [1, 2^32-2]"; return GR_EINVAL; }
  if (world < 1) world = 1;
  if (rank < 0 || rank >= world) { *err = "rank outside [0, world)"; return GR_EINVAL; }
  const int T = threads > 0 ? threads : default_threads();

  // --- canonical COO view
  std::vector<uint32_t> csr_src;
  const uint32_t *src = nullptr, *dst = nullptr;
  if (E->fmt == GR_FMT_COO) {
    if (m && (!E->src || !E->dst)) { *err = "COO src/dst is NULL"; return GR_EINVAL; }
    src = E->src;
    dst = E->dst;
  } else if (E->fmt == GR_FMT_CSR) {
    if (!E->row_offsets || (m && !E->col_idx)) { *err = "CSR arrays are NULL"; return GR_EINVAL; }
    if (E->row_offsets[0] != 0 || E->row_offsets[n] != m) { *err = "CSR row_offsets must span [0, m]"; return GR_EINVAL; }
    for (uint64_t u = 0; u < n; u++)
      if (E->row_offsets[u + 1] < E->row_offsets[u]) { *err = "CSR row_offsets not monotone"; return GR_EINVAL; }
    csr_src.resize(m);
    parallel_for(T, n, [&](uint64_t b, uint64_t e) {
      for (uint64_t u = b; u < e; u++)
        for (uint64_t i = E->row_offsets[u]; i < E->row_offsets[u + 1]; i++) csr_src[i] = (uint32_t)u;
    });
    src = csr_src.data();
    dst = E->col_idx;
  } else {
    *err = "unknown gr_format";
    return GR_EINVAL;
  }
  const uint32_t *w = E->weights;

  // --- validate ids / weights
  std::atomic<int> bad{0};
  parallel_for(T, m, [&](uint64_t b, uint64_t e) {
    int lb = 0;
    for (uint64_t i = b; i < e; i++) {
      if (src[i] >= n || dst[i] >= n) lb |= 1;
      if (w && w[i] > 255u) lb |= 2;
    }
    if (lb) bad.fetch_or(lb);
  });
  if (bad.load() & 1) { *err = "edge endpoint >= num_vertices"; return GR_EINVAL; }
  if (bad.load() & 2) { *err = "edge weight > 255 (weights are stored as uint8)"; return GR_EINVAL; }

  // --- degrees
  std::vector<std::atomic<uint32_t>> indeg(n), outd(n);
  parallel_for(T, n, [&](uint64_t b, uint64_t e) {
    for (uint64_t v = b; v < e; v++) {
      indeg[v].store(0, std::memory_order_relaxed);
      outd[v].store(0, std::memory_order_relaxed);
    }
  });
  parallel_for(T, m, [&](uint64_t b, uint64_t e) {
    for (uint64_t i = b; i < e; i++) {
      indeg[dst[i]].fetch_add(1, std::memory_order_relaxed);
      outd[src[i]].fetch_add(1, std::memory_order_relaxed);
    }
  });
  std::vector<uint64_t> wprefix(n + 1, 0);
  for (uint64_t v = 0; v < n; v++)
    wprefix[v + 1] = wprefix[v] + indeg[v].load(std::memory_order_relaxed) + outd[v].load(std::memory_order_relaxed);

  // --- owner range (multi-GPU: contiguous destination ranges of equal edge weight)
  std::vector<uint64_t> owners;
  gr_status st = plan_owner_ranges(n, wprefix.data(), world, &owners);
  if (st != GR_OK) { *err = "owner planning failed"; return st; }
  G->n = n;
  G->m_total = m;
  G->own_lo = owners[rank];
  G->own_hi = owners[rank + 1];
  G->owners = owners;
  G->has_w = (w != nullptr);
  const uint64_t own_n = G->own_n();

  G->outdeg.resize(n);
  for (uint64_t v = 0; v < n; v++) G->outdeg[v] = outd[v].load(std::memory_order_relaxed);

  // --- CSC offsets over the owned destinations
  G->in_off.assign(own_n + 1, 0);
  for (uint64_t i = 0; i < own_n; i++) G->in_off[i + 1] = G->in_off[i] + indeg[G->own_lo + i].load();
  G->m_in = G->in_off[own_n];
  const uint64_t mi = G->m_in;

  // --- activation CSR offsets (sources over all V, destinations owned)
  G->out_off.assign(n + 1, 0);
  if (world == 1) {
    for (uint64_t v = 0; v < n; v++) G->out_off[v + 1] = G->out_off[v] + G->outdeg[v];
  } else {
    std::vector<std::atomic<uint64_t>> cnt(n);
    parallel_for(T, n, [&](uint64_t b, uint64_t e) {
      for (uint64_t v = b; v < e; v++) cnt[v].store(0, std::memory_order_relaxed);
    });
    parallel_for(T, m, [&](uint64_t b, uint64_t e) {
      for (uint64_t i = b; i < e; i++)
        if (dst[i] >= G->own_lo && dst[i] < G->own_hi) cnt[src[i]].fetch_add(1, std::memory_order_relaxed);
    });
    for (uint64_t v = 0; v < n; v++) G->out_off[v + 1] = G->out_off[v] + cnt[v].load();
  }

  // --- payload arrays (+16 bytes of padding for 128-bit vector loads)
  if (!G->in_src.alloc(4 * mi + 16) || !G->out_dst.alloc(4 * mi + 16) ||
      (G->has_w && (!G->in_w.alloc(mi + 16) || !G->out_w.alloc(mi + 16)))) {
    *err = "host allocation failed";
    return GR_ENOMEM;
  }
  std::memset(G->in_src.as<char>() + 4 * mi, 0, 16);
  std::memset(G->out_dst.as<char>() + 4 * mi, 0, 16);
  if (G->has_w) {
    std::memset(G->in_w.as<char>() + mi, 0, 16);
    std::memset(G->out_w.as<char>() + mi, 0, 16);
  }
  fill_segments(T, m, dst, src, w, G->own_lo, own_n, dst, G->own_lo, G->own_hi, G->in_off,
                G->in_src.as<uint32_t>(), G->has_w ? G->in_w.as<uint8_t>() : nullptr);
  fill_segments(T, m, src, dst, w, 0, n, dst, G->own_lo, G->own_hi, G->out_off,
                G->out_dst.as<uint32_t>(), G->has_w ? G->out_w.as<uint8_t>() : nullptr);

  // --- shards over the owned range (Shard Creator, L208)
  const uint64_t wown = wprefix[G->own_hi] - wprefix[G->own_lo];
  if (shard_edges == 0) shard_edges = uint64_t(1) << 26;
  uint64_t P = (wown + shard_edges - 1) / shard_edges;
  P = std::max<uint64_t>(1, std::min<uint64_t>(P, std::min<uint64_t>(65535, own_n ? own_n : 1)));
  std::vector<uint64_t> local_prefix(own_n + 1);
  for (uint64_t i = 0; i <= own_n; i++) local_prefix[i] = wprefix[G->own_lo + i] - wprefix[G->own_lo];
  G->bounds.assign(P + 1, 0);
  st = gr_plan_intervals(own_n, local_prefix.data(), (uint32_t)P, G->bounds.data());
  if (st != GR_OK) { *err = "interval planning failed"; return st; }
  for (auto &b : G->bounds) b += G->own_lo;
  return GR_OK;
}

// ---- pre-sorted input (GR_FMT_SORTED): the cfg5-scale path where no COO exists
static bool check_adj(int T, uint64_t n, uint64_t m, const uint64_t *off, const uint32_t *adj, std::string *err,
                      const char *what) {
  if (off[0] != 0 || off[n] != m) {
    *err = std::string(what) + ": offsets must span [0, m]";
    return false;
  }
  std::atomic<int> bad{0};
  parallel_for_dyn(T, n, 1 << 16, [&](uint64_t b, uint64_t e) {
    int lb = 0;
    for (uint64_t v = b; v < e && !lb; v++) {
      if (off[v + 1] < off[v]) { lb = 1; break; }
      for (uint64_t i = off[v]; i < off[v + 1]; i++) {
        if (adj[i] >= n) lb |= 2;
        if (i > off[v] && adj[i] < adj[i - 1]) lb |= 4;
      }
    }
    if (lb) bad.fetch_or(lb);
  });
  if (bad.load() & 1) *err = std::string(what) + ": offsets not monotone";
  else if (bad.load() & 2) *err = std::string(what) + ": neighbour id >= num_vertices";
  else if (bad.load() & 4) *err = std::string(what) + ": rows must be sorted ascending (layout R10)";
  return bad.load() == 0;
}

static bool take_adj(HostBuf *dst, const uint32_t *adj, uint64_t m, bool borrow) {
  if (borrow) {  // the caller guarantees 4 spare entries after the m used ones (128-bit loads)
    dst->borrow(adj, 4 * m + 16);
    return true;
  }
  if (!dst->alloc(4 * m + 16)) return false;
  std::memcpy(dst->p, adj, 4 * m);
  std::memset(dst->as<char>() + 4 * m, 0, 16);
  return true;
}

gr_status build_host_sorted(const gr_edges *E, uint64_t shard_edges, bool borrow, int threads, HostGraph *G,
                            std::string *err) {
  const uint64_t n = E->num_vertices, m = E->num_edges;
  if (n == 0 || n >= 0xFFFFFFFFull) { *err = "num_vertices must be in [1, 2^32-2]"; return GR_EINVAL; }
  const bool in = E->in_offsets != nullptr, out = E->row_offsets != nullptr;
  if (!in && !out) { *err = "GR_FMT_SORTED needs in_offsets/in_idx and/or row_offsets/col_idx"; return GR_EINVAL; }
  if ((in && m && !E->in_idx) || (out && m && !E->col_idx)) { *err = "GR_FMT_SORTED: adjacency array is NULL"; return GR_EINVAL; }
  if (E->weights) { *err = "GR_FMT_SORTED carries no weights"; return GR_EINVAL; }
  const int T = threads > 0 ? threads : default_threads();
  if (in && !check_adj(T, n, m, E->in_offsets, E->in_idx, err, "in-CSC")) return GR_EINVAL;
  if (out && !check_adj(T, n, m, E->row_offsets, E->col_idx, err, "out-CSR")) return GR_EINVAL;
  G->n = n;
  G->m_total = m;
  G->own_lo = 0;
  G->own_hi = n;
  G->owners = {0, n};
  G->m_in = m;
  G->has_w = false;
  G->has_in = in;
  G->has_out = out;
  // degrees: from the offsets, from the caller's out_degree, or counted
  G->outdeg.assign(n, 0);
  std::vector<uint32_t> indeg(n, 0);
  if (out) {
    parallel_for(T, n, [&](uint64_t b, uint64_t e) {
      for (uint64_t u = b; u < e; u++) G->outdeg[u] = (uint32_t)(E->row_offsets[u + 1] - E->row_offsets[u]);
    });
  } else if (E->out_degree) {
    std::memcpy(G->outdeg.data(), E->out_degree, 4 * n);
  } else {
    std::vector<std::atomic<uint32_t>> c(n);
    parallel_for(T, n, [&](uint64_t b, uint64_t e) {
      for (uint64_t v = b; v < e; v++) c[v].store(0, std::memory_order_relaxed);
    });
    parallel_for(T, m, [&](uint64_t b, uint64_t e) {
      for (uint64_t i = b; i < e; i++) c[E->in_idx[i]].fetch_add(1, std::memory_order_relaxed);
    });
    for (uint64_t v = 0; v < n; v++) G->outdeg[v] = c[v].load();
  }
  if (in) {
    parallel_for(T, n, [&](uint64_t b, uint64_t e) {
      for (uint64_t v = b; v < e; v++) indeg[v] = (uint32_t)(E->in_offsets[v + 1] - E->in_offsets[v]);
    });
  } else {
    std::vector<std::atomic<uint32_t>> c(n);
    parallel_for(T, n, [&](uint64_t b, uint64_t e) {
      for (uint64_t v = b; v < e; v++) c[v].store(0, std::memory_order_relaxed);
    });
    parallel_for(T, m, [&](uint64_t b, uint64_t e) {
      for (uint64_t i = b; i < e; i++) c[E->col_idx[i]].fetch_add(1, std::memory_order_relaxed);
    });
    for (uint64_t v = 0; v < n; v++) indeg[v] = c[v].load();
  }
  if (in) {
    G->in_off.assign(E->in_offsets, E->in_offsets + n + 1);
    if (!take_adj(&G->in_src, E->in_idx, m, borrow)) { *err = "host allocation failed"; return GR_ENOMEM; }
  } else {
    G->in_off.assign(n + 1, 0);  // offsets only (no edges): zero-degree rows keep the kernels' indexing valid
    for (uint64_t v = 0; v < n; v++) G->in_off[v + 1] = G->in_off[v] + indeg[v];
  }
  if (out) {
    G->out_off.assign(E->row_offsets, E->row_offsets + n + 1);
    if (!take_adj(&G->out_dst, E->col_idx, m, borrow)) { *err = "host allocation failed"; return GR_ENOMEM; }
  } else {
    G->out_off.assign(n + 1, 0);
    for (uint64_t v = 0; v < n; v++) G->out_off[v + 1] = G->out_off[v] + G->outdeg[v];
  }
  // shards (Shard Creator, L208): intervals of near-equal in+out degree
  std::vector<uint64_t> wprefix(n + 1, 0);
  for (uint64_t v = 0; v < n; v++) wprefix[v + 1] = wprefix[v] + indeg[v] + G->outdeg[v];
  if (shard_edges == 0) shard_edges = uint64_t(1) << 26;
  uint64_t P = (wprefix[n] + shard_edges - 1) / shard_edges;
  P = std::max<uint64_t>(1, std::min<uint64_t>(P, std::min<uint64_t>(65535, n)));
  G->bounds.assign(P + 1, 0);
  gr_status st = gr_plan_intervals(n, wprefix.data(), (uint32_t)P, G->bounds.data());
  if (st != GR_OK) { *err = "interval planning failed"; return st; }
  return GR_OK;
}

}  // namespace gr

// ------------------------------------------------------------ C ABI (host-only)
extern "C" gr_status gr_plan_intervals(uint64_t n, const uint64_t *prefix, uint32_t P, uint64_t *bounds) {
  if (!prefix || !bounds || P == 0) return GR_EINVAL;
  const uint64_t total = prefix[n];
  bounds[0] = 0;
  for (uint32_t i = 1; i < P; i++) {
    // first v with prefix[v] >= total * i / P  (128-bit to avoid overflow)
    uint64_t target = (uint64_t)(((unsigned __int128)total * i) / P);
    uint64_t v = (uint64_t)(std::lower_bound(prefix, prefix + n + 1, target) - prefix);
    if (v > n) v = n;
    if (v < bounds[i - 1]) v = bounds[i - 1];
    bounds[i] = v;
  }
  bounds[P] = n;
  return GR_OK;
}
