// gather_paths_bench.cu — random 4-byte gathers from an L2-resident 16 MB
// array (the cfg2 PageRank contribution array) through every load path sm_100a
// offers: LDG.CONSTANT (__ldg), plain LDG, LDG with L1::no_allocate, LDG.CG
// (L2 only), texture fetches (TEX pipe), and LDGSTS (cp.async 4 B into shared
// memory). Decides whether the PageRank gather's L1TEX-wavefront bound
// (profiles/README.md: 0.49 gathers per SM per cycle with __ldg) can be moved
// by the instruction choice alone.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/gpaths tools/gather_paths_bench.cu
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

constexpr int kIters = 1024;

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16;
  x *= 0x7feb352dU;
  x ^= x >> 15;
  x *= 0x846ca68bU;
  x ^= x >> 16;
  return x;
}

__device__ __forceinline__ float ld_plain(const float *p) {
  float v;
  asm volatile("ld.global.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ float ld_noalloc(const float *p) {
  float v;
  asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ float ld_cg(const float *p) {
  float v;
  asm volatile("ld.global.cg.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ float ld_lu(const float *p) {
  float v;
  asm volatile("ld.global.nc.L1::evict_first.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}

// kMode: 0 __ldg, 1 plain, 2 nc.no_allocate, 3 cg, 4 tex1Dfetch, 5 cp.async 4B, 6 nc.evict_first,
//        7 __ldg with only lanes 0..15 active (replay cost vs lanes)
template <int kMode, int kIlp>
__global__ void k_gather(const float *__restrict__ g, cudaTextureObject_t tex, uint32_t gmask, float *out) {
  extern __shared__ float stage[];
  uint32_t seed = (blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B9u;
  float acc = 0.f;
  for (int it = 0; it < kIters; it++) {
    float v[kIlp];
    if (kMode == 5) {
#pragma unroll
      for (int q = 0; q < kIlp; q++) {
        const uint32_t h = hash32(seed + it * kIlp + q) & gmask;
        const uint32_t sa = (uint32_t)__cvta_generic_to_shared(stage + q * blockDim.x + threadIdx.x);
        asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(sa), "l"(g + h));
      }
      asm volatile("cp.async.wait_all;" ::: "memory");
#pragma unroll
      for (int q = 0; q < kIlp; q++) v[q] = stage[q * blockDim.x + threadIdx.x];
    } else {
#pragma unroll
      for (int q = 0; q < kIlp; q++) {
        const uint32_t h = hash32(seed + it * kIlp + q) & gmask;
        if (kMode == 0) v[q] = __ldg(g + h);
        else if (kMode == 1) v[q] = ld_plain(g + h);
        else if (kMode == 2) v[q] = ld_noalloc(g + h);
        else if (kMode == 3) v[q] = ld_cg(g + h);
        else if (kMode == 4) v[q] = tex1Dfetch<float>(tex, (int)h);
        else if (kMode == 6) v[q] = ld_lu(g + h);
        else v[q] = (threadIdx.x & 16) ? 0.f : __ldg(g + h);
      }
    }
#pragma unroll
    for (int q = 0; q < kIlp; q++) acc += v[q];
  }
  if (acc == 12345.f) out[0] = acc;
}

// Lane-sharing patterns: the 32 lanes of one load
// instruction form groups of kG lanes; a group reads kG consecutive floats
// spaced kStride floats apart inside ONE randomly chosen 128-byte line
// (kStride 1: the group shares a 32-byte sector when kG <= 8; kStride 8: one
// sector per lane, kG <= 4 sectors of the same line). Counts how the
// 1-request-per-SM-per-cycle limit treats shared sectors and shared lines.
template <int kG, int kStride, int kIlp>
__global__ void k_gather_share(const float *__restrict__ g, uint32_t line_mask, float *out) {
  const uint32_t lane = threadIdx.x & 31, grp = lane / kG, sub = lane % kG;
  uint32_t seed = ((blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 0x9E3779B9u + grp * 0x85EBCA6Bu;
  float acc = 0.f;
  for (int it = 0; it < kIters; it++) {
    float v[kIlp];
#pragma unroll
    for (int q = 0; q < kIlp; q++) {
      const uint32_t line = hash32(seed + it * kIlp + q) & line_mask;
      v[q] = __ldg(g + line * 32u + sub * kStride);
    }
#pragma unroll
    for (int q = 0; q < kIlp; q++) acc += v[q];
  }
  if (acc == 12345.f) out[0] = acc;
}

template <int kG, int kStride>
static void run_share(const char *what, const float *g, uint32_t line_mask, float *out, int sms) {
  const int block = 1024, grid = sms;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float best = 1e30f;
  for (int rep = 0; rep < 4; rep++) {
    cudaEventRecord(e0);
    k_gather_share<kG, kStride, 8><<<grid, block>>>(g, line_mask, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const double instr = (double)grid * (block / 32) * kIters * 8;  // warp load instructions
  const double lanes = instr * 32, lines = instr * (32 / kG);
  const double sectors = kStride == 1 ? instr * (32 / kG) * ((kG + 7) / 8) : instr * 32;
  const double cyc = best * 1e-3 * clk * 1e3 * sms;
  printf("%-44s %8.3f ms  lanes %5.2f  sectors %5.2f  lines %5.2f  per SM per cycle\n", what, best, lanes / cyc,
         sectors / cyc, lines / cyc);
}

template <int kMode, int kIlp>
static void run(const char *name, const float *g, cudaTextureObject_t tex, uint32_t gmask, float *out, int block,
                int ctas_per_sm, int sms) {
  const size_t smem = kMode == 5 ? (size_t)kIlp * block * 4 : 0;
  cudaFuncSetAttribute(k_gather<kMode, kIlp>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  const int grid = sms * ctas_per_sm;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float best = 1e30f;
  for (int rep = 0; rep < 4; rep++) {
    cudaEventRecord(e0);
    k_gather<kMode, kIlp><<<grid, block, smem>>>(g, tex, gmask, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  cudaError_t e = cudaGetLastError();
  double n = (double)grid * block * kIters * kIlp;
  if (kMode == 7) n *= 0.5;  // half the lanes gather
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("%-34s blk %4d x%d/SM ilp %2d  %8.3f ms  %7.1f G gathers/s  %5.2f per SM per cycle @%.3f GHz %s\n", name,
         block, ctas_per_sm, kIlp, best, n / (best * 1e-3) / 1e9, n / (best * 1e-3) / sms / (clk * 1e3), clk / 1e6,
         e == cudaSuccess ? "" : cudaGetErrorString(e));
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t bytes = 16u << 20, bigb = 1024ull << 20;
  float *g, *out, *big;
  cudaMalloc(&g, bytes);
  cudaMemset(g, 0, bytes);
  cudaMalloc(&big, bigb);
  cudaMemset(big, 0, bigb);
  cudaMalloc(&out, 4);
  cudaResourceDesc rd = {};
  rd.resType = cudaResourceTypeLinear;
  rd.res.linear.devPtr = g;
  rd.res.linear.desc = cudaCreateChannelDesc<float>();
  rd.res.linear.sizeInBytes = bytes;
  cudaTextureDesc td = {};
  td.readMode = cudaReadModeElementType;
  cudaTextureObject_t tex = 0;
  cudaCreateTextureObject(&tex, &rd, &td, nullptr);
  const uint32_t mask = (uint32_t)(bytes / 4 - 1);
  printf("random 4-byte gathers over a 16 MB (L2-resident) array, %d SMs\n", sms);
  run<0, 8>("__ldg (LDG.CONSTANT)", g, tex, mask, out, 1024, 1, sms);
  run<0, 16>("__ldg (LDG.CONSTANT)", g, tex, mask, out, 1024, 1, sms);
  run<0, 8>("__ldg (LDG.CONSTANT)", g, tex, mask, out, 256, 8, sms);
  run<0, 16>("__ldg (LDG.CONSTANT)", g, tex, mask, out, 512, 4, sms);
  run<1, 8>("ld.global", g, tex, mask, out, 1024, 1, sms);
  run<2, 8>("ld.global.nc.L1::no_allocate", g, tex, mask, out, 1024, 1, sms);
  run<2, 16>("ld.global.nc.L1::no_allocate", g, tex, mask, out, 512, 4, sms);
  run<3, 8>("ld.global.cg (L2 only)", g, tex, mask, out, 1024, 1, sms);
  run<3, 16>("ld.global.cg (L2 only)", g, tex, mask, out, 512, 4, sms);
  run<6, 8>("ld.global.nc.L1::evict_first", g, tex, mask, out, 1024, 1, sms);
  run<4, 8>("tex1Dfetch (TEX)", g, tex, mask, out, 1024, 1, sms);
  run<4, 16>("tex1Dfetch (TEX)", g, tex, mask, out, 512, 4, sms);
  run<5, 8>("cp.async.ca 4 B -> smem (LDGSTS)", g, tex, mask, out, 1024, 1, sms);
  run<5, 16>("cp.async.ca 4 B -> smem (LDGSTS)", g, tex, mask, out, 512, 2, sms);
  run<7, 8>("__ldg, 16 of 32 lanes active", g, tex, mask, out, 1024, 1, sms);
  printf("L1-resident: random 4-byte gathers over a 32 KB array (hits in L1 after the first touch)\n");
  run<0, 8>("__ldg (LDG.CONSTANT), 32 KB array", g, tex, (32u << 10) / 4 - 1, out, 1024, 1, sms);
  run<1, 8>("ld.global, 32 KB array", g, tex, (32u << 10) / 4 - 1, out, 1024, 1, sms);
  run<0, 8>("__ldg (LDG.CONSTANT), 128 KB array", g, tex, (128u << 10) / 4 - 1, out, 1024, 1, sms);
  printf("lanes sharing sectors / lines of the 16 MB (L2-resident) array (groups of G lanes, one random line each)\n");
  const uint32_t lmask = (uint32_t)(bytes / 128 - 1);
  run_share<1, 1>("G=1  (32 lines, 32 sectors per instr)", g, lmask, out, sms);
  run_share<2, 1>("G=2  same sector (16 lines, 16 sectors)", g, lmask, out, sms);
  run_share<4, 1>("G=4  same sector (8 lines, 8 sectors)", g, lmask, out, sms);
  run_share<8, 1>("G=8  same sector (4 lines, 4 sectors)", g, lmask, out, sms);
  run_share<32, 1>("G=32 one line, 4 sectors", g, lmask, out, sms);
  run_share<2, 8>("G=2  same line, 2 sectors (16 lines, 32 sec)", g, lmask, out, sms);
  run_share<4, 8>("G=4  same line, 4 sectors (8 lines, 32 sec)", g, lmask, out, sms);
  printf("the same over a 32 KB (L1-resident) array\n");
  const uint32_t smask = (uint32_t)((32u << 10) / 128 - 1);
  run_share<1, 1>("L1 G=1  (32 lines per instr)", g, smask, out, sms);
  run_share<4, 8>("L1 G=4  same line, 4 sectors", g, smask, out, sms);
  run_share<8, 1>("L1 G=8  same sector", g, smask, out, sms);
  printf("random 4-byte gathers over a 1 GB (HBM) array\n");
  const uint32_t bmask = (uint32_t)(bigb / 4 - 1);
  run<0, 16>("__ldg (LDG.CONSTANT)", big, tex, bmask, out, 512, 4, sms);
  run<3, 16>("ld.global.cg (L2 only)", big, tex, bmask, out, 512, 4, sms);
  return 0;
}
