// dsmem_bench.cu — random 4-byte gather throughput on B200 from (0) the CTA's
// own shared memory, (1) distributed shared memory of an 8-CTA cluster, (2)
// global memory resident in L2 (16 MB), (3) global memory beyond L2 (512 MB).
// Decides whether a cluster-shared hot-source table can replace L1/L2 gathers
// in the PageRank kernel (profiles/README.md).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/dsmem tools/dsmem_bench.cu
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>

namespace cg = cooperative_groups;

constexpr int kTable = 16384;  // floats per CTA (64 KB)
constexpr int kIters = 2048;
constexpr int kIlp = 8;

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16;
  x *= 0x7feb352dU;
  x ^= x >> 15;
  x *= 0x846ca68bU;
  x ^= x >> 16;
  return x;
}

template <int kMode>
__global__ void __cluster_dims__(8, 1, 1) __launch_bounds__(1024, 1)
    k_gather(const float *__restrict__ g, uint32_t gmask, float *out) {
  extern __shared__ float tab[];
  for (int i = threadIdx.x; i < kTable; i += blockDim.x) tab[i] = (float)(i & 7);
  cg::cluster_group cl = cg::this_cluster();
  cl.sync();
  float *remote[8];
#pragma unroll
  for (int r = 0; r < 8; r++) remote[r] = cl.map_shared_rank(tab, r);
  uint32_t seed = (blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B9u;
  float acc = 0.f;
  for (int it = 0; it < kIters; it++) {
    float v[kIlp];
#pragma unroll
    for (int q = 0; q < kIlp; q++) {
      const uint32_t h = hash32(seed + it * kIlp + q);
      if (kMode == 0) v[q] = tab[h & (kTable - 1)];
      else if (kMode == 1) v[q] = remote[h >> 29][h & (kTable - 1)];
      else v[q] = __ldg(g + (h & gmask));
    }
#pragma unroll
    for (int q = 0; q < kIlp; q++) acc += v[q];
  }
  cl.sync();  // keep every CTA's table alive until all remote readers are done
  if (acc == 12345.f) out[0] = acc;
}

int main() {
  const size_t big = 512ull << 20;
  float *g, *out;
  cudaMalloc(&g, big);
  cudaMemset(g, 0, big);
  cudaMalloc(&out, 4);
  const int grid = 144, block = 1024;
  const size_t smem = kTable * sizeof(float);
  cudaFuncSetAttribute(k_gather<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(k_gather<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(k_gather<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const char *names[4] = {"local smem", "cluster DSMEM (8 CTAs)", "global, 16 MB (L2)", "global, 512 MB (HBM)"};
  for (int mode = 0; mode < 4; mode++) {
    float best = 1e30f;
    for (int rep = 0; rep < 3; rep++) {
      cudaEventRecord(e0);
      if (mode == 0) k_gather<0><<<grid, block, smem>>>(g, 0, out);
      else if (mode == 1) k_gather<1><<<grid, block, smem>>>(g, 0, out);
      else if (mode == 2) k_gather<2><<<grid, block, smem>>>(g, (16u << 20) / 4 - 1, out);
      else k_gather<2><<<grid, block, smem>>>(g, (uint32_t)(big / 4 - 1), out);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      if (ms < best) best = ms;
    }
    cudaError_t e = cudaGetLastError();
    const double n = (double)grid * block * kIters * kIlp;
    printf("%-26s %8.3f ms  %7.1f G gathers/s  %6.2f per SM per cycle @1.965 GHz  %s\n", names[mode], best,
           n / (best * 1e-3) / 1e9, n / (best * 1e-3) / 144 / 1.965e9, e == cudaSuccess ? "" : cudaGetErrorString(e));
  }
  return 0;
}
