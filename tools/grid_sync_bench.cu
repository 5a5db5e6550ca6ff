// grid_sync_bench.cu — superstep-floor microbenchmarks on the B200:
// kernel launch latency (stream and CUDA graph) and the software grid barrier
// used by the persistent superstep loop, at several grid sizes.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gsb tools/grid_sync_bench.cu
#include <cuda_runtime.h>

#include <cstdio>

struct Bar {
  unsigned count, gen;
};

__device__ __forceinline__ void grid_sync(Bar *b) {
  __syncthreads();
  if (threadIdx.x == 0) {
    volatile unsigned *gen = &b->gen;
    const unsigned g = *gen;
    __threadfence();
    if (atomicAdd(&b->count, 1u) == gridDim.x - 1) {
      b->count = 0;
      __threadfence();
      atomicAdd(&b->gen, 1u);
    } else {
      while (*gen == g) __nanosleep(32);
    }
    __threadfence();
  }
  __syncthreads();
}

// hierarchical: CTAs of the same group of 16 meet first
__device__ __forceinline__ void grid_sync2(Bar *b, unsigned *grp_cnt) {
  __syncthreads();
  if (threadIdx.x == 0) {
    volatile unsigned *gen = &b->gen;
    const unsigned g = *gen;
    __threadfence();
    const unsigned grp = blockIdx.x >> 4, ngrp = (gridDim.x + 15) >> 4;
    const unsigned gsz = min(16u, gridDim.x - grp * 16u);
    if (atomicAdd(grp_cnt + grp, 1u) == gsz - 1) {
      grp_cnt[grp] = 0;
      __threadfence();
      if (atomicAdd(&b->count, 1u) == ngrp - 1) {
        b->count = 0;
        __threadfence();
        atomicAdd(&b->gen, 1u);
      } else {
        while (*gen == g) {}
      }
    } else {
      while (*gen == g) {}
    }
    __threadfence();
  }
  __syncthreads();
}

__device__ __forceinline__ unsigned ld_acq(const unsigned *p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned atom_add_acqrel(unsigned *p, unsigned x) {
  unsigned v;
  asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "r"(x) : "memory");
  return v;
}
__device__ __forceinline__ void st_rel(unsigned *p, unsigned x) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(x) : "memory");
}
__device__ __forceinline__ void st_relaxed(unsigned *p, unsigned x) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(x) : "memory");
}
// release/acquire: the arrival atom is acq_rel (publishes this CTA's writes,
// sees the others' on the last arrival), the release is a st.release of the new
// generation, waiters spin with ld.acquire; no fence.sc
__device__ __forceinline__ void grid_sync3(Bar *b) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned g = ld_acq(&b->gen);
    if (atom_add_acqrel(&b->count, 1u) == gridDim.x - 1) {
      st_relaxed(&b->count, 0);
      st_rel(&b->gen, g + 1);
    } else {
      while (ld_acq(&b->gen) == g) {}
    }
  }
  __syncthreads();
}
// same, with __nanosleep(32) in the spin
__device__ __forceinline__ void grid_sync4(Bar *b) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned g = ld_acq(&b->gen);
    if (atom_add_acqrel(&b->count, 1u) == gridDim.x - 1) {
      st_relaxed(&b->count, 0);
      st_rel(&b->gen, g + 1);
    } else {
      while (ld_acq(&b->gen) == g) __nanosleep(32);
    }
  }
  __syncthreads();
}
// counter that never resets: arrival k of barrier i returns i*grid + k; waiters
// spin until the counter reaches (i+1)*grid (no separate generation word)
__device__ __forceinline__ void grid_sync5(Bar *b, unsigned i) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned target = (i + 1) * gridDim.x;
    if (atom_add_acqrel(&b->count, 1u) != target - 1)
      while (ld_acq(&b->count) < target) {}
  }
  __syncthreads();
}

__global__ void k_sync(Bar *b, unsigned *grp, int iters, int hier) {
  for (int i = 0; i < iters; i++) {
    if (hier == 1) grid_sync2(b, grp);
    else if (hier == 2) grid_sync3(b);
    else if (hier == 3) grid_sync4(b);
    else if (hier == 4) grid_sync5(b, (unsigned)i);
    else grid_sync(b);
  }
}

__global__ void k_empty() {}

int main() {
  cudaStream_t s;
  cudaStreamCreate(&s);
  cudaEvent_t a, z;
  cudaEventCreate(&a);
  cudaEventCreate(&z);
  float ms;
  // launch latency, back to back
  for (int grid : {1, 592}) {
    for (int i = 0; i < 100; i++) k_empty<<<grid, 256, 0, s>>>();
    cudaEventRecord(a, s);
    for (int i = 0; i < 2000; i++) k_empty<<<grid, 256, 0, s>>>();
    cudaEventRecord(z, s);
    cudaEventSynchronize(z);
    cudaEventElapsedTime(&ms, a, z);
    printf("stream launch grid=%d: %.2f us/kernel\n", grid, ms * 1000 / 2000);
  }
  // graph of 1000 empty kernels
  for (int grid : {1, 592}) {
    cudaGraph_t gph;
    cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
    for (int i = 0; i < 1000; i++) k_empty<<<grid, 256, 0, s>>>();
    cudaStreamEndCapture(s, &gph);
    cudaGraphExec_t ex;
    cudaGraphInstantiate(&ex, gph, 0);
    cudaGraphLaunch(ex, s);
    cudaEventRecord(a, s);
    cudaGraphLaunch(ex, s);
    cudaEventRecord(z, s);
    cudaEventSynchronize(z);
    cudaEventElapsedTime(&ms, a, z);
    printf("graph node grid=%d: %.2f us/kernel\n", grid, ms * 1000 / 1000);
  }
  Bar *b;
  unsigned *grp;
  cudaMalloc(&b, sizeof(Bar));
  cudaMalloc(&grp, 4096);
  const char *names[] = {"", "(hier16)", "(acq_rel)", "(acq_rel+sleep)", "(monotone count)"};
  for (int hier = 0; hier < 5; hier++)
    for (int grid : {148, 296, 592, 1184}) {
      cudaMemset(b, 0, sizeof(Bar));
      cudaMemset(grp, 0, 4096);
      int iters = 2000;
      void *args[] = {&b, &grp, &iters, &hier};
      cudaLaunchCooperativeKernel((void *)k_sync, grid, 256, args, 0, s);
      cudaMemsetAsync(b, 0, sizeof(Bar), s);
      cudaEventRecord(a, s);
      cudaLaunchCooperativeKernel((void *)k_sync, grid, 256, args, 0, s);
      cudaEventRecord(z, s);
      cudaError_t e = cudaEventSynchronize(z);
      cudaEventElapsedTime(&ms, a, z);
      printf("grid_sync%s grid=%d: %.2f us/barrier (%s)\n", names[hier], grid, ms * 1000 / iters,
             cudaGetErrorString(e));
    }
  return 0;
}
