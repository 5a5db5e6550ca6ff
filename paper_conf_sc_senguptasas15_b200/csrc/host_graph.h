// host_graph.h — host-side sharded layout.
//
// Partition Engine of PAPER.md §4.2 (L200-210): the Shard Creator cuts V into
// P disjoint intervals of near-equal in+out edge count (L208); the Graph Layout
// Engine sorts in-edges by destination (CSC, gather) and out-edges by source
// (CSR, scatter / FrontierActivate) so there is no runtime transposition
// (L208-210). Secondary order inside a segment is (neighbour id, weight), which
// makes the layout a pure function of the edge multiset (R10).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "graphreduce.h"

namespace gr {

// Memory that may later be page-locked for DMA (cudaHostRegister) when the
// graph is streamed; plain page-aligned host memory otherwise.
struct HostBuf {
  void *p = nullptr;
  size_t bytes = 0;
  bool registered = false;
  bool owned = true;   // false: the caller's memory, used in place (GR_FMT_SORTED + borrow)
  void borrow(const void *q, size_t nbytes) {
    release();
    p = const_cast<void *>(q);
    bytes = nbytes;
    owned = false;
  }
  HostBuf() = default;
  HostBuf(const HostBuf &) = delete;
  HostBuf &operator=(const HostBuf &) = delete;
  ~HostBuf();
  bool alloc(size_t nbytes);
  void release();
  template <class T> T *as() const { return static_cast<T *>(p); }
};

struct HostGraph {
  uint64_t n = 0;          // |V|
  uint64_t m_total = 0;    // |E| of the input
  uint64_t own_lo = 0, own_hi = 0;  // owned destination range [own_lo, own_hi)
  std::vector<uint64_t> owners;     // owner range bounds of every rank (world + 1)
  uint64_t m_in = 0;       // in-edges with an owned destination
  bool has_w = false;
  // which halves of the layout exist: a GR_FMT_SORTED input may carry only the
  // in-CSC (PageRank) or only the out-CSR (BFS) of a graph too large for both
  bool has_in = true, has_out = true;
  // CSC over owned destinations: in-edges of v = in_src[in_off[v-own_lo] .. in_off[v-own_lo+1])
  std::vector<uint64_t> in_off;  // own_n + 1
  HostBuf in_src;                // uint32 [m_in] (+ 4 pad entries for 16-byte vector loads)
  HostBuf in_w;                  // uint8  [m_in] (+16 pad) if has_w
  // Activation CSR: edges with an owned destination grouped by source u in [0, n)
  // (== the plain out-edge CSR when one rank owns all of V).
  std::vector<uint64_t> out_off; // n + 1
  HostBuf out_dst;               // uint32 [m_in] (+4 pad)
  HostBuf out_w;                 // uint8 if has_w
  std::vector<uint32_t> outdeg;  // global out-degree of every vertex (PageRank n_j, L74)
  // Shards: intervals [bounds[s], bounds[s+1]) of the owned range
  std::vector<uint64_t> bounds;  // P + 1
  // Device-built graphs keep no host in_off/out_off: the offsets at the shard
  // bounds (in_off[bounds[s]-own_lo], out_off[bounds[s]]) are stored instead.
  std::vector<uint64_t> bound_in, bound_out;
  uint32_t num_shards() const { return bounds.empty() ? 0 : (uint32_t)(bounds.size() - 1); }
  uint64_t own_n() const { return own_hi - own_lo; }
};

// Build the layout. world/rank select the owned destination range (owner ranges
// are themselves gr_plan_intervals over in+out degree, so every rank computes
// the same split). Returns GR_OK or an error with *err filled.
gr_status build_host_graph(const gr_edges *e, uint64_t shard_edges, int world, int rank,
                           int threads, HostGraph *out, std::string *err);

// Layout from a pre-sorted input (GR_FMT_SORTED): the in-CSC and/or out-CSR as
// given (rows sorted ascending, checked), borrowed in place or copied; single rank.
gr_status build_host_sorted(const gr_edges *e, uint64_t shard_edges, bool borrow, int threads, HostGraph *out,
                            std::string *err);

// Owner split of [0, n) for `world` ranks (same on every rank).
gr_status plan_owner_ranges(uint64_t n, const uint64_t *weight_prefix, int world,
                            std::vector<uint64_t> *owners);

int default_threads();

}  // namespace gr
