// jit.h — run-time compiled GAS programs (§4.1
// L196, Fig. 6): NVRTC + driver API glue, loaded with dlopen so the library
// has no link-time dependency on either.
#pragma once
#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>

#include "graphreduce.h"
#include "prog_desc.h"

namespace gr {

struct JitProgram {
  int id = 0;
  uint32_t gather_bytes = 4;   // sizeof(GatherT)
  bool has_gather = true, uses_weights = false, scatter = false;
  int init = 0;                // kInit
  void *mod = nullptr;         // CUmodule
  // [0] OffT = uint32_t, [1] OffT = uint64_t
  void *persistent[2] = {nullptr, nullptr};
  void *init_values[2] = {nullptr, nullptr};
  void *init_frontier[2] = {nullptr, nullptr};
  void *fill = nullptr;        // k_prog_fill<P>(void *acc, uint64_t count): identity()
  void *init_edges[2] = {nullptr, nullptr};  // k_init_edges<P, OffT> (programs with scatter)
  int device = -1;             // the device whose context holds the module
  ProgDesc desc;               // traits + kernel table for the streamed / partitioned drivers
};

gr_status jit_compile(const char *source, const char *name, int *id);
const JitProgram *jit_find(int id);
// cuLaunchKernel / cuLaunchCooperativeKernel on torch's / the graph's stream
gr_status jit_launch(void *fn, unsigned grid, unsigned block, void **args, size_t smem, cudaStream_t s, bool coop);
gr_status jit_occupancy(void *fn, int block, int *blocks_per_sm);

}  // namespace gr
