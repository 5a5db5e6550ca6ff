// fig4_transfer.cu — B200 re-run of PAPER.md Fig. 4 (L136, L150): moving
// 100,000,000 doubles between host and GPU with (a) explicit H2D copies,
// (b) pinned host memory read in place by the kernel (UVA zero-copy) and
// (c) managed (unified) memory, for sequential and random access by a
// reduction kernel. Each time includes the data movement and the kernel.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/fig4 tools/fig4_transfer.cu
//   tools/fig4 [n]
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>

#define CK(x)                                                                     \
  do {                                                                            \
    cudaError_t e_ = (x);                                                         \
    if (e_ != cudaSuccess) {                                                      \
      fprintf(stderr, "%s: %s (line %d)\n", #x, cudaGetErrorString(e_), __LINE__); \
      exit(1);                                                                    \
    }                                                                             \
  } while (0)

__device__ __forceinline__ unsigned long long mix(unsigned long long x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

// sum of a[i] (sequential) or a[mix(i) % n] (random), n accesses either way
template <bool kRandom>
__global__ void k_sum(const double *a, unsigned long long n, double *out) {
  double s = 0;
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x)
    s += kRandom ? a[mix(i) % n] : a[i];
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) atomicAdd(out, s);
}

int main(int argc, char **argv) {
  const unsigned long long n = argc > 1 ? strtoull(argv[1], nullptr, 10) : 100000000ull;
  const size_t bytes = n * sizeof(double);
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const int grid = sms * 8, block = 256;
  double *h = nullptr, *d = nullptr, *m = nullptr, *out = nullptr;
  CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped));
  for (unsigned long long i = 0; i < n; i++) h[i] = (double)(i % 1000) * 0.5;
  CK(cudaMalloc(&d, bytes));
  CK(cudaMallocManaged(&out, sizeof(double)));
  CK(cudaMallocManaged(&m, bytes));
  double *hd = nullptr;
  CK(cudaHostGetDevicePointer(&hd, h, 0));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  printf("# PAPER.md Fig. 4 on B200: %llu doubles (%.1f MB), %d x %d threads; time includes data movement\n", n,
         bytes / 1e6, grid, block);
  printf("%-10s %-16s %10s %12s\n", "access", "technique", "ms", "GB/s(eff)");
  for (int rnd = 0; rnd < 2; rnd++) {
    for (int tech = 0; tech < 3; tech++) {
      float best = 1e30f;
      for (int rep = 0; rep < 3; rep++) {
        if (tech == 2) {  // fresh managed data resident on the host before every repetition
          CK(cudaMemPrefetchAsync(m, bytes, cudaCpuDeviceId, 0));
          CK(cudaDeviceSynchronize());
          if (rep == 0) memcpy(m, h, bytes);
        }
        *out = 0;
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e0));
        const double *src = hd;
        if (tech == 0) {
          CK(cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice));
          src = d;
        } else if (tech == 2) {
          src = m;
        }
        if (rnd) k_sum<true><<<grid, block>>>(src, n, out);
        else k_sum<false><<<grid, block>>>(src, n, out);
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        CK(cudaGetLastError());
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, e0, e1));
        if (ms < best) best = ms;
      }
      static const char *names[3] = {"explicit_h2d", "pinned_uva", "managed"};
      printf("%-10s %-16s %10.2f %12.2f\n", rnd ? "random" : "sequential", names[tech], best, bytes / (best * 1e-3) / 1e9);
      fflush(stdout);
    }
  }
  return 0;
}
