// api.cu — extern "C" entry points of include/graphreduce.h.
#include <cuda_runtime.h>
#include <nccl.h>

#include <cstring>
#include <cerrno>
#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include "engine.h"
#include "jit.h"

using namespace gr;

struct gr_host_graph {
  HostGraph H;
};

namespace gr {
uint64_t static_bytes_estimate(const HostGraph &H) {
  const uint64_t n = H.n, on = H.own_n(), mi = H.m_in;
  const uint64_t offb = (mi >= 0xFFFFFFFFull) ? 8 : 4;
  const uint64_t tiles = (on + mi) / 2048 + 2;
  return offb * (on + 1) + offb * (n + 1) + n / 8 + on / 8 + 4 * n /*val*/ + 4 * on /*stamp*/ +
         8 * 4 * on /*lists*/ + 4 * n /*outdeg*/ + 12 * n /*inv, contrib x2*/ + 4 * on /*rank*/ + 16 * tiles +
         (32ull << 20) /*trace*/;
}
uint64_t resident_bytes_estimate(const HostGraph &H) {
  return static_bytes_estimate(H) + 8 * (H.m_in + 16) + (H.has_w ? H.m_in + 16 : 0);
}
}  // namespace gr

extern "C" {

const char *gr_last_error(void) { return gr::last_error(); }

gr_status gr_get_unique_id(uint8_t out[128]) {
  clear_error();
  if (!out) return fail(GR_EINVAL, "out is NULL");
  ncclUniqueId id;
  ncclResult_t r = ncclGetUniqueId(&id);
  if (r != ncclSuccess) return fail(GR_ENCCL, "ncclGetUniqueId: %s", ncclGetErrorString(r));
  static_assert(sizeof(id) == 128, "ncclUniqueId is 128 bytes");
  std::memcpy(out, &id, 128);
  return GR_OK;
}

gr_status gr_graph_load(const gr_edges *edges, const gr_load_opts *opts_in, gr_graph **out) {
  clear_error();
  if (!out) return fail(GR_EINVAL, "out is NULL");
  *out = nullptr;
  if (!edges) return fail(GR_EINVAL, "edges is NULL");
  gr_load_opts opts{};
  if (opts_in) opts = *opts_in;
  if (opts.world <= 0) opts.world = 1;
  if (opts.mode < GR_MODE_AUTO || opts.mode > GR_MODE_STREAMED) return fail(GR_EINVAL, "bad mode %d", opts.mode);
  const bool sim = opts.sim_ranks > 1;
  if (sim) opts.world = opts.sim_ranks;
  if (opts.rank < 0 || opts.rank >= opts.world) return fail(GR_EINVAL, "rank %d outside [0, %d)", opts.rank, opts.world);
  if (opts.world > 1 && opts.mode == GR_MODE_STREAMED)
    return fail(GR_EUNSUPPORTED, "streamed mode is single-rank (partition over GPUs to fit HBM instead)");
  if (opts.transport != GR_TRANSPORT_NCCL && opts.transport != GR_TRANSPORT_SHM)
    return fail(GR_EINVAL, "bad transport %d", opts.transport);
  if (opts.world > 1 && !opts.nccl_unique_id)
    return fail(GR_EINVAL, "world > 1 needs nccl_unique_id (simulated ranks: any 128-byte group key)");
  int ndev = 0;
  cudaError_t ce = cudaGetDeviceCount(&ndev);
  if (ce != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return fail(GR_ECUDA, "no CUDA device available (%s)", cudaGetErrorString(ce));
  }
  if (opts.device < 0 || opts.device >= ndev) return fail(GR_EINVAL, "device %d out of range", opts.device);
  if (cudaSetDevice(opts.device) != cudaSuccess) return fail(GR_ECUDA, "cudaSetDevice failed");
  pool_init(opts.device);

  tmark("load: enter");
  gr_graph *g = new gr_graph();
  g->device = opts.device;
  std::string err;
  gr_status s = GR_OK;
  size_t free_b = 0, total_b = 0;
  cudaMemGetInfo(&free_b, &total_b);
  uint64_t budget = opts.device_budget_bytes ? opts.device_budget_bytes
                                             : (free_b > (4ull << 30) ? free_b - (4ull << 30) : free_b / 2);
  // device build: resident, single rank, COO input, and room for the sort buffers (~34 B/edge peak)
  const uint64_t n0 = edges->num_vertices, m0 = edges->num_edges;
  const bool dev_ok = opts.world == 1 && edges->fmt == GR_FMT_COO && opts.mode != GR_MODE_STREAMED && n0 >= 1 &&
                      n0 < 0xFFFFFFFFull && (m0 == 0 || (edges->src && edges->dst)) &&
                      34 * m0 + 64 * n0 + (64ull << 20) <= budget;
  const bool dev_build = opts.build == GR_BUILD_DEVICE || (opts.build == GR_BUILD_AUTO && dev_ok);
  if (opts.build == GR_BUILD_DEVICE && !dev_ok) {
    delete g;
    return fail(GR_EUNSUPPORTED, "device build needs a resident single-rank COO graph that fits the device budget");
  }
  if (edges->fmt == GR_FMT_SORTED) {
    if (opts.world > 1) {
      delete g;
      return fail(GR_EUNSUPPORTED, "GR_FMT_SORTED inputs are single-rank");
    }
    s = build_host_sorted(edges, opts.shard_edges, opts.borrow != 0, opts.host_threads, &g->H, &err);
    if (s == GR_OK && (!g->H.has_in || !g->H.has_out) && opts.mode != GR_MODE_STREAMED) {
      s = GR_EUNSUPPORTED;
      err = "a one-directional layout (only in-CSC or only out-CSR) must be loaded streamed";
    }
    if (s != GR_OK) {
      delete g;
      return fail(s, "%s", err.c_str());
    }
  } else if (!dev_build) {
    s = build_host_graph(edges, opts.shard_edges, opts.world, opts.rank, opts.host_threads, &g->H, &err);
    if (s != GR_OK) {
      delete g;
      return fail(s, "%s", err.c_str());
    }
  }
  cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, g->device);
  // stream, events and the pinned control block: reused from graphs freed earlier on
  // this device (creating them, the pinned allocation above all, costs milliseconds of
  // every load: the e2e path)
  if (!acquire_handles(g)) {
    destroy(g);
    return fail(GR_ECUDA, "stream/event/pinned setup failed");
  }
  tmark("load: host build / setup");
  if (dev_build) {
    g->mode = GR_MODE_RESIDENT;
    g->dev_built = true;
    s = device_build(g, edges, opts.shard_edges);
    tmark("load: device build");
    if (s != GR_OK) {
      std::string keep = gr::last_error();
      destroy(g);
      return fail(s, "%s", keep.c_str());
    }
  } else {
    const uint64_t need = resident_bytes_estimate(g->H);
    if (opts.mode == GR_MODE_AUTO) g->mode = (need <= budget || opts.world > 1) ? GR_MODE_RESIDENT : GR_MODE_STREAMED;
    else g->mode = opts.mode;
  }
  g->sim = sim;
  s = load_device(g);
  tmark("load: load_device");
  if (s == GR_OK && g->mode == GR_MODE_STREAMED) s = stream_setup(g, budget);
  if (s == GR_OK && opts.world > 1) {
    std::string cerr;
    const int transport = sim ? kTransportSim : opts.transport == GR_TRANSPORT_SHM ? kTransportShm : kTransportNccl;
    s = comm_create(opts.world, opts.rank, transport, opts.nccl_unique_id, g->device, &g->comm, &cerr);
    if (s != GR_OK) fail(s, "%s", cerr.c_str());
    if (s == GR_OK) s = part_setup(g);
  }
  if (s != GR_OK) {
    std::string keep = gr::last_error();
    destroy(g);
    return fail(s, "%s", keep.c_str());
  }
  *out = g;
  return GR_OK;
}

gr_status gr_run(gr_graph *g, const gr_run_opts *opts, gr_run_stats *stats) {
  clear_error();
  if (!g || !opts) return fail(GR_EINVAL, "graph or opts is NULL");
  gr_run_stats st{};
  cudaSetDevice(g->device);
  gr_status s = gr::run(g, opts, &st);
  if (stats) *stats = st;
  return s;
}

gr_status gr_fetch_vertex_values(gr_graph *g, void *host_dst, uint64_t bytes) {
  clear_error();
  if (!g) return fail(GR_EINVAL, "graph is NULL");
  cudaSetDevice(g->device);
  return fetch_values(g, host_dst, bytes);
}

gr_status gr_fetch_frontier_trace(gr_graph *g, uint64_t *host_dst, uint64_t max_rows, uint64_t *rows) {
  clear_error();
  if (!g) return fail(GR_EINVAL, "graph is NULL");
  cudaSetDevice(g->device);
  return fetch_trace(g, host_dst, max_rows, rows);
}

gr_status gr_fetch_frontier_trace_detail(gr_graph *g, uint64_t *host_dst, uint64_t max_rows, uint64_t *rows) {
  clear_error();
  if (!g) return fail(GR_EINVAL, "graph is NULL");
  cudaSetDevice(g->device);
  return fetch_trace_detail(g, host_dst, max_rows, rows);
}

gr_status gr_program_compile(const char *source, const char *struct_name, int32_t *custom_id) {
  int id = 0;
  const gr_status s = gr::jit_compile(source, struct_name, &id);
  if (s == GR_OK) *custom_id = id;
  return s;
}

gr_status gr_graph_info_get(const gr_graph *g, gr_graph_info *o) {
  clear_error();
  if (!g || !o) return fail(GR_EINVAL, "null argument");
  std::memset(o, 0, sizeof *o);
  o->num_vertices = g->H.n;
  o->num_edges = g->H.m_total;
  o->num_shards = g->H.num_shards();
  o->mode = g->mode;
  o->rank = g->comm ? g->comm->rank : 0;
  o->world = g->comm ? g->comm->world : 1;
  o->sim_ranks = g->sim ? o->world : 1;
  o->own_lo = g->H.own_lo;
  o->own_hi = g->H.own_hi;
  o->device_bytes = g->dev_bytes;
  o->pinned_bytes = g->pinned_bytes;
  o->offsets_64bit = g->off64 ? 1 : 0;
  o->has_weights = g->H.has_w ? 1 : 0;
  o->built_on_device = g->dev_built ? 1 : 0;
  return GR_OK;
}

static void shard_desc(const HostGraph &H, uint32_t s, gr_shard_desc *o) {
  o->v_lo = H.bounds[s];
  o->v_hi = H.bounds[s + 1];
  if (H.in_off.empty()) {  // device-built: offsets kept only at the bounds
    o->in_begin = H.bound_in[s];
    o->in_end = H.bound_in[s + 1];
    o->out_begin = H.bound_out[s];
    o->out_end = H.bound_out[s + 1];
    return;
  }
  o->in_begin = H.in_off[o->v_lo - H.own_lo];
  o->in_end = H.in_off[o->v_hi - H.own_lo];
  o->out_begin = H.out_off[o->v_lo];
  o->out_end = H.out_off[o->v_hi];
}

gr_status gr_shard_info(const gr_graph *g, uint32_t s, gr_shard_desc *o) {
  clear_error();
  if (!g || !o) return fail(GR_EINVAL, "null argument");
  if (s >= g->H.num_shards()) return fail(GR_EINVAL, "shard %u >= %u", s, g->H.num_shards());
  shard_desc(g->H, s, o);
  return GR_OK;
}

void gr_graph_free(gr_graph *g) { destroy(g); }

gr_status gr_graph_load_file(const char *path, const gr_load_opts *opts, gr_graph **out) {
  clear_error();
  if (!path || !out) return fail(GR_EINVAL, "null argument");
  *out = nullptr;
  const int fd = open(path, O_RDONLY);
  if (fd < 0) return fail(GR_EINVAL, "cannot open %s: %s", path, strerror(errno));
  struct stat sb;
  if (fstat(fd, &sb) != 0 || sb.st_size < 32) {
    close(fd);
    return fail(GR_EINVAL, "%s: not a graph file (size %lld)", path, (long long)sb.st_size);
  }
  const size_t size = (size_t)sb.st_size;
  void *map = mmap(nullptr, size, PROT_READ, MAP_PRIVATE, fd, 0);
  close(fd);
  if (map == MAP_FAILED) return fail(GR_EINVAL, "mmap %s: %s", path, strerror(errno));
  madvise(map, size, MADV_SEQUENTIAL);
  const unsigned char *b = (const unsigned char *)map;
  struct Hdr { char magic[8]; uint64_t n, m; uint32_t fmt, flags; } h;
  std::memcpy(&h, b, sizeof h);
  gr_status st = GR_OK;
  gr_edges e{};
  if (std::memcmp(h.magic, "GRGRAPH1", 8) != 0) st = fail(GR_EINVAL, "%s: bad magic", path);
  else if (h.fmt > GR_FMT_CSR || (h.flags & ~1u)) st = fail(GR_EINVAL, "%s: bad fmt %u / flags %u", path, h.fmt, h.flags);
  else if (h.n >= (1ull << 40) || h.m >= (1ull << 40)) st = fail(GR_EINVAL, "%s: implausible n/m", path);
  else {
    const uint64_t body = h.fmt == GR_FMT_COO ? 8 * h.m : 8 * (h.n + 1) + 4 * h.m;
    const uint64_t need = 32 + body + ((h.flags & 1) ? 4 * h.m : 0);
    if (need != size) st = fail(GR_EINVAL, "%s: size %zu != %llu expected from the header", path, size,
                                (unsigned long long)need);
    else {
      e.fmt = (int32_t)h.fmt;
      e.num_vertices = h.n;
      e.num_edges = h.m;
      const unsigned char *p = b + 32;
      if (h.fmt == GR_FMT_COO) {
        e.src = (const uint32_t *)p;
        e.dst = (const uint32_t *)(p + 4 * h.m);
      } else {
        e.row_offsets = (const uint64_t *)p;
        e.col_idx = (const uint32_t *)(p + 8 * (h.n + 1));
      }
      if (h.flags & 1) e.weights = (const uint32_t *)(b + 32 + body);
    }
  }
  if (st == GR_OK) st = gr_graph_load(&e, opts, out);  // copies everything it keeps
  munmap(map, size);
  return st;
}

gr_status gr_host_build(const gr_edges *edges, const gr_load_opts *opts_in, gr_host_graph **out) {
  clear_error();
  if (!out) return fail(GR_EINVAL, "out is NULL");
  *out = nullptr;
  gr_load_opts opts{};
  if (opts_in) opts = *opts_in;
  if (!edges) return fail(GR_EINVAL, "edges is NULL");
  auto *h = new gr_host_graph();
  std::string err;
  gr_status s = edges->fmt == GR_FMT_SORTED
                    ? build_host_sorted(edges, opts.shard_edges, opts.borrow != 0, opts.host_threads, &h->H, &err)
                    : build_host_graph(edges, opts.shard_edges, opts.world > 0 ? opts.world : 1, opts.rank,
                                       opts.host_threads, &h->H, &err);
  if (s != GR_OK) {
    delete h;
    return fail(s, "%s", err.c_str());
  }
  *out = h;
  return GR_OK;
}

gr_status gr_host_csc(const gr_host_graph *h, const uint64_t **off, const uint32_t **src, const uint8_t **w) {
  if (!h || !off || !src) return fail(GR_EINVAL, "null argument");
  *off = h->H.in_off.data();
  *src = h->H.in_src.as<uint32_t>();
  if (w) *w = h->H.has_w ? h->H.in_w.as<uint8_t>() : nullptr;
  return GR_OK;
}

gr_status gr_host_csr(const gr_host_graph *h, const uint64_t **off, const uint32_t **dst, const uint8_t **w) {
  if (!h || !off || !dst) return fail(GR_EINVAL, "null argument");
  *off = h->H.out_off.data();
  *dst = h->H.out_dst.as<uint32_t>();
  if (w) *w = h->H.has_w ? h->H.out_w.as<uint8_t>() : nullptr;
  return GR_OK;
}

gr_status gr_host_shards(const gr_host_graph *h, uint32_t *num_shards, const uint64_t **bounds) {
  if (!h || !num_shards || !bounds) return fail(GR_EINVAL, "null argument");
  *num_shards = h->H.num_shards();
  *bounds = h->H.bounds.data();
  return GR_OK;
}

void gr_host_free(gr_host_graph *h) { delete h; }

}  // extern "C"
