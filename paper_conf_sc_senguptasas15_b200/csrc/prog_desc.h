// prog_desc.h — a GAS program as the host drivers of the streamed and the
// partitioned modes see it: its static traits and the kernels instantiated for
// it — at library build time for the built-in and GR_CUSTOM_PROGRAMS programs
// (prog_table.cu), or at run time by NVRTC for gr_program_compile programs
// (jit.cu, §4.1: the user supplies gatherMap /
// gatherReduce / apply / scatter and the framework instantiates its engine with
// them). One driver then serves both kinds of program.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "graphreduce.h"

namespace gr {

struct ProgDesc {
  bool has_gather = true, uses_weights = false, scatter = false, jit = false;
  int init = 0;               // kInitSource / kInitSourceChanged / kInitAll
  uint32_t gather_bytes = 4;  // sizeof(GatherT)
  int jit_device = -1;        // run-time programs: the device their module was loaded on
  // kernels by offset type: [0] uint32_t, [1] uint64_t (signatures: kernels_frontier.cuh,
  // kernels_stream.cuh). Scatter-only kernels are empty for programs without scatter.
  void *init_values[2] = {}, *init_edges[2] = {}, *init_frontier[2] = {};
  void *s_init_scatter[2] = {}, *s_gather_apply[2] = {}, *s_activate[2] = {};
  void *gather_apply[2] = {}, *gather_apply_x[2] = {}, *scatter_activate[2] = {};
  void *fill = nullptr;       // k_prog_fill<P>(void *p, unsigned long long count): identity()
};

// The descriptor of the program gr_run selects (built-in algo, GR_CUSTOM_PROGRAMS
// id, or a run-time program id); GR_EUNSUPPORTED if none.
gr_status prog_desc(int algo, int custom_id, ProgDesc *out);
// Launch one of the descriptor's kernels (cudaLaunchKernel, or cuLaunchKernel
// for a run-time module) on stream s.
gr_status klaunch(const ProgDesc &d, void *fn, unsigned grid, unsigned block, void **args, cudaStream_t s);

}  // namespace gr
