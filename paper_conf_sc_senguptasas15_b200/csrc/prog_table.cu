// prog_table.cu — the per-program kernel tables of the streamed and the
// partitioned drivers (prog_desc.h). The built-in programs' kernels are
// instantiated here, once; run-time programs get theirs from their NVRTC
// module (jit.cu).
#include "prog_desc.h"

#include "engine.h"
#include "jit.h"
#include "kernels_stream.cuh"

namespace gr {

template <class Prog> static ProgDesc make_desc() {
  ProgDesc d;
  d.has_gather = Prog::kHasGather;
  d.uses_weights = Prog::kUsesWeights;
  d.scatter = HasScatter<Prog>::value;
  d.init = Prog::kInit;
  d.gather_bytes = sizeof(typename Prog::GatherT);
  d.fill = (void *)k_prog_fill<Prog>;
#define GR_K(field, kern)                        \
  d.field[0] = (void *)kern<Prog, uint32_t>;     \
  d.field[1] = (void *)kern<Prog, uint64_t>;
  GR_K(init_values, k_init_values)
  GR_K(init_edges, k_init_edges)
  GR_K(init_frontier, k_init_frontier)
  GR_K(s_init_scatter, k_s_init_scatter)
  GR_K(s_gather_apply, k_s_gather_apply)
  GR_K(s_activate, k_s_activate)
  GR_K(gather_apply, k_gather_apply)
  GR_K(gather_apply_x, k_gather_apply_x)
  GR_K(scatter_activate, k_scatter_activate)
#undef GR_K
  return d;
}

gr_status prog_desc(int algo, int custom_id, ProgDesc *out) {
  switch (algo) {
    case GR_BFS: *out = make_desc<ProgBFS>(); return GR_OK;
    case GR_SSSP: *out = make_desc<ProgSSSP>(); return GR_OK;
    case GR_CC: *out = make_desc<ProgCC>(); return GR_OK;
    case GR_PAGERANK_DELTA: *out = make_desc<ProgPRDelta>(); return GR_OK;
    case GR_CUSTOM: {
#define GR_X(id, T)                    \
  if (custom_id == id) {               \
    *out = make_desc<T>();             \
    return GR_OK;                      \
  }
      GR_CUSTOM_PROGRAMS(GR_X)
#undef GR_X
      if (const JitProgram *jp = jit_find(custom_id)) {
        *out = jp->desc;
        return GR_OK;
      }
      return fail(GR_EUNSUPPORTED, "no custom program with id %d is registered", custom_id);
    }
    default: return fail(GR_EUNSUPPORTED, "algo %d has no frontier program", algo);
  }
}

gr_status klaunch(const ProgDesc &d, void *fn, unsigned grid, unsigned block, void **args, cudaStream_t s) {
  if (d.jit) return jit_launch(fn, grid, block, args, 0, s, false);
  const cudaError_t e = cudaLaunchKernel(fn, dim3(grid), dim3(block), args, 0, s);
  if (e != cudaSuccess) return fail(GR_ECUDA, "kernel launch: %s", cudaGetErrorString(e));
  return GR_OK;
}

}  // namespace gr
