// grgen_gpu.cu — the R-MAT input of grgen.c generated on a GPU straight into a
// sorted adjacency layout (cfg5 at scale: SURVEY §8(d), PAPER.md L36 — a
// scale-30/31 R-MAT's COO does not fit host memory, so it is never
// materialised). Same draws as grgen_rmat (counter-based splitmix64 of
// (seed, stream 1, edge * draws + j), two 32-bit uniforms per draw, quadrant
// thresholds compared in double), so the edge multiset is exactly grgen.rmat's;
// the output is that multiset sorted by (key, other) with key = dst (in-CSC) or
// src (out-CSR). Input-generation only: holds none of the GAS method.
//
// Multi-pass: pass 0 histograms the keys (and the other endpoint's degrees),
// then each pass regenerates every edge, keeps those whose key falls in the
// pass's key range (ranges sized to a device budget), radix-sorts the packed
// (key << 32 | other) words and copies the others to their final host position.
#include <cub/cub.cuh>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

namespace {

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
uint64_t mix64_h(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

struct RmatP {
  uint64_t key;  // mix64(seed * phi + c0) ^ mix64(stream + c1): the per-(seed, stream) part of grgen_hash
  double a, ab, abc;
  uint32_t scale, draws;
};

__device__ __forceinline__ void rmat_edge(const RmatP &p, uint64_t i, uint32_t &s, uint32_t &d) {
  uint64_t ss = 0, dd = 0;
  for (uint32_t j = 0; j < p.draws; j++) {
    const uint64_t h = mix64(p.key + ((uint64_t)i * p.draws + j + 1) * 0x9E3779B97F4A7C15ULL);
#pragma unroll
    for (int k = 0; k < 2; k++) {
      const uint32_t level = 2 * j + k;
      if (level >= p.scale) break;
      const double u = (double)((uint32_t)(h >> (32 * k))) * (1.0 / 4294967296.0);
      uint64_t sb, db;
      if (u < p.a) { sb = 0; db = 0; }
      else if (u < p.ab) { sb = 0; db = 1; }
      else if (u < p.abc) { sb = 1; db = 0; }
      else { sb = 1; db = 1; }
      ss = (ss << 1) | sb;
      dd = (dd << 1) | db;
    }
  }
  s = (uint32_t)ss;
  d = (uint32_t)dd;
}

__global__ void k_hist(RmatP p, uint64_t m0, uint64_t m1, int by_src, uint32_t *kcnt, uint32_t *ocnt) {
  for (uint64_t i = m0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m1; i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t s, d;
    rmat_edge(p, i, s, d);
    atomicAdd(kcnt + (by_src ? s : d), 1u);
    if (ocnt) atomicAdd(ocnt + (by_src ? d : s), 1u);
  }
}

__global__ void k_collect(RmatP p, uint64_t m0, uint64_t m1, int by_src, uint32_t k0, uint32_t k1,
                          unsigned long long *out, unsigned long long *cnt) {
  for (uint64_t i = m0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m1; i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t s, d;
    rmat_edge(p, i, s, d);
    const uint32_t k = by_src ? s : d, o = by_src ? d : s;
    if (k >= k0 && k < k1) {
      const unsigned long long pos = atomicAdd(cnt, 1ull);
      out[pos] = ((unsigned long long)(k - k0) << 32) | o;
    }
  }
}

__global__ void k_low32(const unsigned long long *in, uint64_t n, uint32_t *out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = (uint32_t)in[i];
}

#define GCK(x)                                                                    \
  do {                                                                            \
    cudaError_t e_ = (x);                                                         \
    if (e_ != cudaSuccess) {                                                      \
      fprintf(stderr, "grgen_gpu: %s: %s\n", #x, cudaGetErrorString(e_));         \
      return -3;                                                                  \
    }                                                                             \
  } while (0)

}  // namespace

extern "C" {

// Sorted adjacency of grgen_rmat(scale, m, a, b, c, seed): by_src = 0 gives the
// in-CSC (off indexed by dst, adj = sources sorted by (dst, src)), 1 the out-CSR
// (by (src, dst)). off: host uint64[n + 1]; adj: host uint32[m]; other_deg
// (nullable): host uint32[n], degree of the other endpoint (out-degree for the
// CSC). budget_bytes: device memory for one pass (0 = 3/4 of the free memory).
// Returns 0, or < 0 on error (bad arguments -1, memory -2, CUDA -3).
int grgen_rmat_sorted_gpu(uint32_t scale, uint64_t m, double a, double b, double c, uint64_t seed, int by_src,
                          int device, uint64_t *off, uint32_t *adj, uint32_t *other_deg, uint64_t budget_bytes) {
  if (scale == 0 || scale > 32 || !off || (m && !adj)) return -1;
  if (a < 0 || b < 0 || c < 0 || a + b + c > 1.0) return -1;
  GCK(cudaSetDevice(device));
  const uint64_t n = 1ull << scale;
  RmatP p;
  p.key = mix64_h(seed * 0x9E3779B97F4A7C15ULL + 0x632BE59BD9B4E019ULL) ^ mix64_h(1 + 0x8CB92BA72F3D8DD7ULL);
  p.a = a;
  p.ab = a + b;
  p.abc = a + b + c;
  p.scale = scale;
  p.draws = (scale + 1) / 2;
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
  const unsigned grid = (unsigned)sms * 8, block = 256;
  // pass 0: degrees
  uint32_t *kcnt = nullptr, *ocnt = nullptr;
  GCK(cudaMalloc(&kcnt, 4 * n));
  GCK(cudaMemset(kcnt, 0, 4 * n));
  if (other_deg) {
    GCK(cudaMalloc(&ocnt, 4 * n));
    GCK(cudaMemset(ocnt, 0, 4 * n));
  }
  k_hist<<<grid, block>>>(p, 0, m, by_src, kcnt, ocnt);
  GCK(cudaGetLastError());
  std::vector<uint32_t> kc(n);
  GCK(cudaMemcpy(kc.data(), kcnt, 4 * n, cudaMemcpyDeviceToHost));
  if (other_deg) GCK(cudaMemcpy(other_deg, ocnt, 4 * n, cudaMemcpyDeviceToHost));
  cudaFree(kcnt);
  if (ocnt) cudaFree(ocnt);
  off[0] = 0;
  for (uint64_t v = 0; v < n; v++) off[v + 1] = off[v] + kc[v];
  if (off[n] != m) return -3;
  // passes over key ranges of at most `cap` edges
  size_t fr = 0, tot = 0;
  GCK(cudaMemGetInfo(&fr, &tot));
  if (!budget_bytes) budget_bytes = fr / 4 * 3;
  uint64_t cap = budget_bytes / 24;  // packed words x2 (sort double buffer) + 4 B out + temp
  if (cap < (1u << 20)) return -2;
  uint64_t maxdeg = 0;
  for (uint64_t v = 0; v < n; v++) maxdeg = kc[v] > maxdeg ? kc[v] : maxdeg;
  if (maxdeg > cap) cap = maxdeg;
  if (cap > 0x7FFFFFFFull) cap = 0x7FFFFFFFull;  // one radix sort call per pass (int item count)
  if (maxdeg > cap) return -2;
  unsigned long long *w0 = nullptr, *w1 = nullptr, *d_cnt = nullptr;
  uint32_t *lo = nullptr;
  const uint64_t need = std::min<uint64_t>(cap, m ? m : 1);
  GCK(cudaMalloc(&w0, 8 * need));
  GCK(cudaMalloc(&w1, 8 * need));
  GCK(cudaMalloc(&lo, 4 * need));
  GCK(cudaMalloc(&d_cnt, 8));
  void *tmp = nullptr;
  size_t tmp_bytes = 0;
  {
    cub::DoubleBuffer<unsigned long long> db(w0, w1);
    cub::DeviceRadixSort::SortKeys(nullptr, tmp_bytes, db, (int)std::min<uint64_t>(need, 0x7FFFFFFFull));
    GCK(cudaMalloc(&tmp, tmp_bytes + 256));
  }
  uint64_t k0 = 0;
  while (k0 < n) {
    uint64_t k1 = k0;
    while (k1 < n && off[k1 + 1] - off[k0] <= need) k1++;
    if (k1 == k0) k1 = k0 + 1;
    const uint64_t cnt = off[k1] - off[k0];
    if (cnt) {
      GCK(cudaMemset(d_cnt, 0, 8));
      k_collect<<<grid, block>>>(p, 0, m, by_src, (uint32_t)k0, (uint32_t)k1, w0, d_cnt);
      GCK(cudaGetLastError());
      // key bits: (k1 - k0 - 1) fits in end_bit - 32 bits
      int kb = 1;
      while ((1ull << kb) < (k1 - k0)) kb++;
      cub::DoubleBuffer<unsigned long long> db(w0, w1);
      GCK(cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, db, (int)cnt, 0, 32 + kb));
      k_low32<<<grid, block>>>(db.Current(), cnt, lo);
      GCK(cudaGetLastError());
      GCK(cudaMemcpy(adj + off[k0], lo, 4 * cnt, cudaMemcpyDeviceToHost));
    }
    k0 = k1;
  }
  cudaFree(w0);
  cudaFree(w1);
  cudaFree(lo);
  cudaFree(d_cnt);
  cudaFree(tmp);
  return 0;
}

}  // extern "C"
