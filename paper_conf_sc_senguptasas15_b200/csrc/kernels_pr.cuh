// kernels_pr.cuh — PageRank superstep (reading R1): all vertices
// active, FrontierActivate eliminated (phase elimination, §5.3).
//
//   gather  (L250-251): acc[v] = sum_{(u->v)} contrib[u],  contrib[u] = R_t(u)/outdeg(u)
//   apply   (L252):     R_{t+1}(v) = (1-d)/n + d*acc[v];  contrib'[v] = R_{t+1}(v)/outdeg(v)
//
// Load balancing (CTA load balancing, L260; merge-path over the CSC offsets,
// K6 in SURVEY §2.3): the merged sequence of row-ends (one per destination) and
// in-edges is cut into tiles of exactly kPrTile items, so hubs and empty rows
// cost the same per item. Each tile stages its offsets and the gathered source
// contributions in shared memory (the random gathers are issued together for
// memory-level parallelism), each thread walks kPrIpt consecutive items, and a
// segmented scan over the threads joins rows split between threads. Rows that
// start in an earlier tile are finished by k_pr_fixup in a fixed order, so the
// fp32 sum order is deterministic run to run.
#pragma once
#include "device_common.cuh"

namespace gr {

constexpr int kPrThreads = 256;
constexpr int kMaxPeers = 15;  // partitioned PageRank: peers written by the fused exchange
constexpr int kPrIpt = 8;
constexpr int kPrTile = kPrThreads * kPrIpt;
constexpr uint32_t kNoRow = 0xFFFFFFFFu;
constexpr int kPrPad = kPrTile / kPrIpt;  // one pad word per kPrIpt items

// Shared-memory index with one pad word per 8 items: thread t walks items
// [8t, 8t+8), so unpadded reads of lanes t and t+4 would hit the same bank
// (8-way conflicts); with the pad, lane t reads bank (9t + q) mod 32 (distinct).
__device__ __forceinline__ uint32_t pr_pad(uint32_t i) { return i + (i >> 3); }

template <class OffT> struct PrArgs {
  uint32_t n, own_lo, own_n; // own_lo/own_n: first global row and row count of this launch
  uint64_t m_in;             // edges of this launch
  uint64_t e_base;           // global edge index of in_src[0] (streamed shard slot; 0 resident)
  const OffT *in_off;        // [own_n + 1] global edge offsets of this launch's rows
  const uint32_t *in_src;    // [m_in]
  const float *inv_outdeg;   // [n]
  const float *contrib_in;   // [n]   contributions of superstep t-1 (read side)
  float *contrib_out;        // [n]   owned slice written
  float *rank;               // [own_n] written on the last iteration
  uint32_t *carry_row;       // [num_tiles]
  float *carry_val;
  uint32_t *head_row;
  float *head_val;
  const uint32_t *tile_row;  // [num_tiles + 1] merge-path row coordinate of each tile start (precomputed)
  float base, d;             // (1-d)/n, d
  int last;                  // 1: write rank instead of contrib_out
  // Partitioned runs, fused exchange: the other ranks' contribution
  // replicas of superstep t+1 (peer-mapped over NVLink, or same-device buffers of
  // simulated ranks). Every owned contribution the apply writes is stored into
  // each of them as well, so the allgather of the owned slices is done by the
  // apply's own stores, row by row, while the gather of other rows continues.
  float *peer[kMaxPeers];
  uint32_t npeer;
};

// contribution of owned vertex v for superstep t+1: the local replica, then every peer's
template <class OffT>
__device__ __forceinline__ void pr_store_contrib(const PrArgs<OffT> &a, uint32_t v, float c) {
  a.contrib_out[v] = c;
  for (uint32_t q = 0; q < a.npeer; q++) a.peer[q][v] = c;
}

template <class OffT>
__device__ __forceinline__ void pr_apply_row(const PrArgs<OffT> &a, uint32_t lrow, float acc) {
  const float R = a.base + a.d * acc;
  const uint32_t v = a.own_lo + lrow;
  if (a.last) a.rank[lrow] = R;
  else pr_store_contrib(a, v, R * __ldg(a.inv_outdeg + v));
}

// Merge-path search over (row ends, edge indices) for diagonal `diag`.
template <class OffT>
__device__ __forceinline__ uint32_t merge_path_rows(const OffT *in_off, uint64_t e_base, uint32_t rows, uint64_t nnz,
                                                    uint64_t diag) {
  uint64_t lo = diag > nnz ? diag - nnz : 0;
  uint64_t hi = diag < rows ? diag : rows;
  while (lo < hi) {
    const uint64_t p = (lo + hi) >> 1;
    if ((uint64_t)in_off[p + 1] - e_base <= diag - p - 1) lo = p + 1;
    else hi = p;
  }
  return (uint32_t)lo;
}

constexpr uint32_t kHotTag = 0x80000000u;  // in the PageRank payload: source is hot, low bits = slot
constexpr int kHotK = 16384;                 // hot sources held in shared memory per CTA (64 KB)

struct PrSmem {
  uint32_t s_end[kPrTile + 1 + kPrPad];  // row ends, local to the tile's first edge (padded)
  float s_val[kPrTile + kPrPad];         // contrib[src] of the tile's edges (padded)
  float s_tot[kPrTile + kPrPad];         // per-row partial totals (padded)
  uint32_t s_crow[kPrThreads];
  float s_cval[kPrThreads];
  uint32_t s_wkey_first[kPrThreads / 32], s_wkey_last[kPrThreads / 32];
  float s_wval_last[kPrThreads / 32];
  uint64_t s_i0, s_i1, s_j0, s_j1, s_rowstart0;
};

// One merge-path tile: stage, walk, join, apply. kHot: sources tagged with
// kHotTag read their contribution from the CTA's shared hot table.
template <class OffT, bool kHot>
__device__ __forceinline__ void pr_tile(const PrArgs<OffT> &a, uint32_t tile, PrSmem &S, const float *s_hot) {
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint64_t total = (uint64_t)a.own_n + a.m_in;
  const uint64_t d0 = (uint64_t)tile * kPrTile;
  const uint64_t d1 = d0 + kPrTile < total ? d0 + kPrTile : total;
  __syncthreads();  // the previous tile's readers are done with S
  if (tid < 2) {
    const uint64_t diag = tid == 0 ? d0 : d1;
    const uint32_t i = __ldg(a.tile_row + tile + tid);  // == merge_path_rows(diag), precomputed
    if (tid == 0) { S.s_i0 = i; S.s_j0 = diag - i; S.s_rowstart0 = (uint64_t)a.in_off[i] - a.e_base; }
    else { S.s_i1 = i; S.s_j1 = diag - i; }
  }
  __syncthreads();
  const uint64_t i0 = S.s_i0, j0 = S.s_j0;
  const uint32_t ni = (uint32_t)(S.s_i1 - i0), nj = (uint32_t)(S.s_j1 - j0);

  // stage row ends (local) and gathered contributions
  for (uint32_t k = tid; k <= ni; k += kPrThreads) {
    const uint64_t r = i0 + k;
    uint64_t e = r < a.own_n ? (uint64_t)a.in_off[r + 1] - a.e_base - j0 : (uint64_t)nj;
    S.s_end[pr_pad(k)] = (uint32_t)(e < nj ? e : nj);
  }
  {
    uint32_t src[kPrIpt];
#pragma unroll
    for (int q = 0; q < kPrIpt; q++) {
      const uint32_t k = tid + q * kPrThreads;
      src[q] = k < nj ? ldg_nc(a.in_src + j0 + k) : 0u;
    }
    float v[kPrIpt];
#pragma unroll
    for (int q = 0; q < kPrIpt; q++) {
      const uint32_t k = tid + q * kPrThreads;
      if (kHot && (src[q] & kHotTag)) v[q] = s_hot[src[q] & ~kHotTag];
      else v[q] = k < nj ? __ldg(a.contrib_in + src[q]) : 0.f;
    }
#pragma unroll
    for (int q = 0; q < kPrIpt; q++) {
      const uint32_t k = tid + q * kPrThreads;
      if (k < nj) S.s_val[pr_pad(k)] = v[q];
    }
  }
  __syncthreads();

  // per-thread merge walk over kPrIpt items
  const uint32_t tile_items = ni + nj;
  const uint32_t dt = min(tid * kPrIpt, tile_items);
  uint32_t lo = dt > nj ? dt - nj : 0, hi = dt < ni ? dt : ni;
  while (lo < hi) {
    const uint32_t p = (lo + hi) >> 1;
    if (S.s_end[pr_pad(p)] <= dt - p - 1) lo = p + 1;
    else hi = p;
  }
  uint32_t i = lo, j = dt - lo;
  float run = 0.f;
  const uint32_t dend = min(dt + kPrIpt, tile_items);
#pragma unroll
  for (int q = 0; q < kPrIpt; q++) {
    if (dt + q < dend) {
      if (j < S.s_end[pr_pad(i)]) { run += S.s_val[pr_pad(j)]; ++j; }
      else { S.s_tot[pr_pad(i)] = run; run = 0.f; ++i; }
    }
  }
  S.s_crow[tid] = i;

  // segmented inclusive scan of the thread carries (keys non-decreasing)
  float x = run;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const float y = __shfl_up_sync(0xffffffffu, x, o);
    const uint32_t ky = __shfl_up_sync(0xffffffffu, i, o);
    if (lane >= (uint32_t)o && ky == i) x += y;
  }
  if (lane == 0) S.s_wkey_first[warp] = i;
  if (lane == 31) { S.s_wkey_last[warp] = i; S.s_wval_last[warp] = x; }
  __syncthreads();
  if (i == S.s_wkey_first[warp]) {
    for (int w = (int)warp - 1; w >= 0; w--) {
      if (S.s_wkey_last[w] != i) break;
      x += S.s_wval_last[w];
      if (S.s_wkey_first[w] != i) break;
    }
  }
  S.s_cval[tid] = x;
  __syncthreads();
  // the last thread of each carry run adds it to the row finished by the next thread
  const bool run_end = (tid == kPrThreads - 1) || (S.s_crow[tid + 1] != i);
  if (run_end && i < ni) S.s_tot[pr_pad(i)] += x;
  __syncthreads();

  // apply the rows whose end lies in this tile (coalesced over destinations)
  const bool head = (ni > 0) && (S.s_rowstart0 < j0);  // row i0 began in an earlier tile
  for (uint32_t k = tid; k < ni; k += kPrThreads) {
    if (k == 0 && head) continue;
    pr_apply_row(a, (uint32_t)(i0 + k), S.s_tot[pr_pad(k)]);
  }
  if (tid == 0) {
    a.head_row[tile] = head ? (uint32_t)i0 : kNoRow;
    a.head_val[tile] = head ? S.s_tot[pr_pad(0)] : 0.f;
    const uint64_t i1 = S.s_i1;
    a.carry_row[tile] = i1 < a.own_n ? (uint32_t)i1 : kNoRow;
    a.carry_val[tile] = S.s_cval[kPrThreads - 1];
  }
}

template <class OffT>
__global__ void __launch_bounds__(kPrThreads, 6) k_pr_gather_apply(const __grid_constant__ PrArgs<OffT> a) {
  __shared__ PrSmem S;
  pr_tile<OffT, false>(a, blockIdx.x, S, nullptr);
}



// ---------------------------------------------------------------------------
// Warp-granular merge path: a tile of kWTile = 256 items belongs to ONE warp
// (8 items per lane). Staging, the merge walk, the segmented join and the
// apply are warp-local (shuffles + __syncwarp), so warps never wait at a CTA
// barrier and every warp's memory phases overlap with its neighbours'.
// Rows spanning warp tiles are finished by k_pr_fixup_warp.
#ifndef GR_WIPT
#define GR_WIPT 8
#endif
constexpr int kWIpt = GR_WIPT;  // items per lane of a warp tile
constexpr int kWTile = 32 * kWIpt;
constexpr int kWPad = kWTile / kWIpt;

struct PrWarpSmem {
  uint32_t s_end[kWTile + 1 + kWPad + 1];
  float s_val[kWTile + kWPad];
  float s_tot[kWTile + kWPad];
};

template <class OffT, bool kHot>
__device__ __forceinline__ void pr_warp_tile(const PrArgs<OffT> &a, uint32_t tile, PrWarpSmem &S,
                                             const float *s_hot) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t total = (uint64_t)a.own_n + a.m_in;
  const uint64_t d0 = (uint64_t)tile * kWTile;
  const uint64_t d1 = d0 + kWTile < total ? d0 + kWTile : total;
  const uint32_t i0 = __ldg(a.tile_row + tile), i1 = __ldg(a.tile_row + tile + 1);
  const uint64_t j0 = d0 - i0;
  const uint32_t ni = i1 - i0, nj = (uint32_t)((d1 - i1) - j0);
  const uint64_t rowstart0 = (uint64_t)a.in_off[i0] - a.e_base;
  __syncwarp();  // the previous tile's readers are done with S
  for (uint32_t k = lane; k <= ni; k += 32) {
    const uint64_t r = (uint64_t)i0 + k;
    const uint64_t e = r < a.own_n ? (uint64_t)a.in_off[r + 1] - a.e_base - j0 : (uint64_t)nj;
    S.s_end[pr_pad(k)] = (uint32_t)(e < nj ? e : nj);
  }
  {
    uint32_t src[kWIpt];
#pragma unroll
    for (int q = 0; q < kWIpt; q++) {
      const uint32_t k = lane + 32u * q;
      src[q] = k < nj ? ldg_nc(a.in_src + j0 + k) : 0u;
    }
    float v[kWIpt];
#pragma unroll
    for (int q = 0; q < kWIpt; q++) {
      const uint32_t k = lane + 32u * q;
      if (kHot && (src[q] & kHotTag)) v[q] = s_hot[src[q] & ~kHotTag];
      else v[q] = k < nj ? __ldg(a.contrib_in + src[q]) : 0.f;
    }
#pragma unroll
    for (int q = 0; q < kWIpt; q++) {
      const uint32_t k = lane + 32u * q;
      if (k < nj) S.s_val[pr_pad(k)] = v[q];
    }
  }
  __syncwarp();
  const uint32_t items = ni + nj;
  const uint32_t dt = min(lane * kWIpt, items);
  uint32_t lo = dt > nj ? dt - nj : 0, hi = dt < ni ? dt : ni;
  while (lo < hi) {
    const uint32_t p = (lo + hi) >> 1;
    if (S.s_end[pr_pad(p)] <= dt - p - 1) lo = p + 1;
    else hi = p;
  }
  uint32_t i = lo, j = dt - lo;
  float run = 0.f;
  const uint32_t dend = min(dt + kWIpt, items);
#pragma unroll
  for (int q = 0; q < kWIpt; q++) {
    if (dt + q < dend) {
      if (j < S.s_end[pr_pad(i)]) { run += S.s_val[pr_pad(j)]; ++j; }
      else { S.s_tot[pr_pad(i)] = run; run = 0.f; ++i; }
    }
  }
  float x = run;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const float y = __shfl_up_sync(0xffffffffu, x, o);
    const uint32_t ky = __shfl_up_sync(0xffffffffu, i, o);
    if (lane >= (uint32_t)o && ky == i) x += y;
  }
  const uint32_t inext = __shfl_down_sync(0xffffffffu, i, 1);
  const float carry = __shfl_sync(0xffffffffu, x, 31);
  __syncwarp();  // every s_tot written by the walk is visible
  const bool run_end = (lane == 31) || (inext != i);
  if (run_end && i < ni) S.s_tot[pr_pad(i)] += x;
  __syncwarp();
  const bool head = (ni > 0) && (rowstart0 < j0);
  for (uint32_t k = lane; k < ni; k += 32) {
    if (k == 0 && head) continue;
    pr_apply_row(a, i0 + k, S.s_tot[pr_pad(k)]);
  }
  if (lane == 0) {
    a.head_row[tile] = head ? i0 : kNoRow;
    a.head_val[tile] = head ? S.s_tot[pr_pad(0)] : 0.f;
    a.carry_row[tile] = i1 < a.own_n ? i1 : kNoRow;
    a.carry_val[tile] = carry;
  }
}

template <class OffT>
__global__ void __launch_bounds__(256) k_pr_warp(const __grid_constant__ PrArgs<OffT> a, uint32_t num_tiles) {
  __shared__ PrWarpSmem S[8];
  const uint32_t w = threadIdx.x >> 5;
  const uint32_t tile = blockIdx.x * 8u + w;
  if (tile < num_tiles) pr_warp_tile<OffT, false>(a, tile, S[w], nullptr);
}

// 1024-thread persistent CTAs: one shared hot table per SM, 32 warp-tile walkers.
template <class OffT>
__global__ void __launch_bounds__(1024, 1) k_pr_warp_hot(const __grid_constant__ PrArgs<OffT> a,
                                                        const float *hot_contrib, uint32_t hot_k,
                                                        uint32_t num_tiles) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  float *s_hot = reinterpret_cast<float *>(smem_raw);
  PrWarpSmem *S = reinterpret_cast<PrWarpSmem *>(smem_raw + 4ull * hot_k);
  for (uint32_t k = threadIdx.x * 4; k < hot_k; k += blockDim.x * 4)
    *reinterpret_cast<float4 *>(s_hot + k) = __ldg(reinterpret_cast<const float4 *>(hot_contrib + k));
  __syncthreads();
  const uint32_t w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  for (uint32_t tile = blockIdx.x * nw + w; tile < num_tiles; tile += gridDim.x * nw)
    pr_warp_tile<OffT, true>(a, tile, S[w], s_hot);
}

// ---------------------------------------------------------------------------
// Edge-segmented warp tiles (`seg`, the default on resident single-GPU runs).
// The PageRank payload is re-laid out once per graph as an item stream in CSC
// order where every destination row owns max(indeg, 1) consecutive items (an
// empty row gets one item reading a zero slot of the hot table), plus one head
// bit per item marking the first item of each row. A warp tile is 256
// consecutive items, lane L owning items 8L..8L+7, loaded with two 128-bit
// loads. Rows are recovered from the head bits (row = first row of the tile +
// heads so far), so there is no merge-path search and no shared-memory
// staging: the per-lane sums run in registers, one segmented shuffle scan over
// the 32 lane tails joins rows split between lanes, and rows split between
// tiles go to the same head/carry fix-up as the other warp kernels. All of the
// shared memory is left to the hot-source table (up to ~56K sources instead of
// 16K next to the staging buffers).
constexpr int kSegIpt = 8;
constexpr int kSegHotK = 32768;  // hot sources of the seg kernel (128 KB of shared memory; measured best of 16K-56K)
constexpr int kSegTile = 32 * kSegIpt;

// Variant bits of k_pr_seg (measured in round 1, profiles/README.md; only kSegDefaultVar is built):
constexpr int kSegBallot = 1;   // segment starts of the lane scan from one ballot (1 shuffle per step, not 3)
constexpr int kSegBuf = 2;      // finished rows through a per-warp buffer: coalesced apply, 1/outdeg preloaded
constexpr int kSegPreFlag = 4;  // head bits loaded one tile ahead
constexpr int kSegStreamNA = 8;  // item/flag/1-outdeg streams loaded with L1::no_allocate (L1 kept for gathers)
constexpr int kSegDefaultVar = kSegBallot;  // measured best of the 16 (profiles/README.md)

template <int kVar> __device__ __forceinline__ uint4 seg_ld4(const uint4 *p) {
  if (kVar & kSegStreamNA) {
    uint4 v;
    asm("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
        : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
  }
  return __ldg(p);
}
template <int kVar> __device__ __forceinline__ uint32_t seg_ld1(const uint32_t *p) {
  if (kVar & kSegStreamNA) {
    uint32_t v;
    asm("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
  }
  return __ldg(p);
}
template <int kVar> __device__ __forceinline__ float seg_ldf(const float *p) {
  if (kVar & kSegStreamNA) {
    float v;
    asm("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
  }
  return __ldg(p);
}

// The contributions of superstep t-1 were written by other CTAs earlier in the same
// (persistent) launch: an ordinary weak load, ordered after those writes by the grid
// barrier's fences — NOT ld.global.nc (the read-only path is defined only for data that
// stays unchanged for the whole kernel). Measured: same rate as __ldg
// (tools/gather_paths_bench.cu: ld.global and LDG.CONSTANT both 1.00 per SM per cycle).
__device__ __forceinline__ float ld_weak_f32(const float *p) {
  float v;
  asm("ld.global.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}

__device__ __forceinline__ float lds_f32(uint32_t saddr) {
  float v;
  asm("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(saddr));
  return v;
}

// TMA bulk copies (cp.async.bulk, non-tensor) into shared memory, completed on
// an mbarrier: the copy engine fetches the item / head-bit streams, so they
// take no slots of the SM's L1->L2 request port (the PageRank floor,
// profiles/pr_floor_r02.md) and no registers while in flight.
__device__ __forceinline__ void mbar_init(uint32_t mbar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(mbar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t mbar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mbar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t mbar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "LAB_WAIT:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra DONE;\n\t"
      "bra LAB_WAIT;\n"
      "DONE:\n\t}" ::"r"(mbar), "r"(parity) : "memory");
}
__device__ __forceinline__ void tma_bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t mbar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(dst), "l"(src), "r"(bytes), "r"(mbar) : "memory");
}
// the generic-proxy reads of a staging buffer are ordered before the next bulk
// copy (async proxy) that overwrites it
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ uint4 lds_v4(uint32_t saddr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(saddr));
  return v;
}
__device__ __forceinline__ uint32_t lds_u32(uint32_t saddr) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(saddr));
  return v;
}
// per-warp staging of one tile: 256 items (1 KB) + its 8 head-bit words and the
// next tile's first word (copied as 48 bytes: bulk sizes are multiples of 16)
constexpr uint32_t kTmaItemBytes = kSegTile * 4;
constexpr uint32_t kTmaFlagBytes = 48;
constexpr uint32_t kTmaBufBytes = kTmaItemBytes + 64;


// contributions of my 8 items: hot sources from the shared table, the rest
// from global memory (L2-resident)
template <int kVar>
__device__ __forceinline__ void seg_gather(const uint4 &s0, const uint4 &s1, const float *s_hot, uint32_t hot_sbase,
                                           const float *__restrict__ contrib, float (&v)[kSegIpt]) {
  const uint32_t src[kSegIpt] = {s0.x, s0.y, s0.z, s0.w, s1.x, s1.y, s1.z, s1.w};
#pragma unroll
  for (int k = 0; k < kSegIpt; k++) {
    v[k] = (src[k] & kHotTag) ? lds_f32(hot_sbase + 4u * (src[k] & ~kHotTag)) : ld_weak_f32(contrib + src[k]);
  }
}

// One tile's reduction and apply from the gathered values v (lane L: items
// 8L..8L+7; b = my head bits, fnext = the item after the tile starts a row).
// No staging of items: each lane sums its items in registers, rows split
// between lanes are joined by one segmented shuffle scan of the lane tails
// (a segment starts at a lane holding a head), and rows split between tiles
// get head/carry records for the fix-up kernels.
template <class OffT, int kVar>
__device__ __forceinline__ void seg_tile(const PrArgs<OffT> &a, uint32_t tile, uint32_t r0, uint32_t b, uint32_t fnext,
                                         float pre_inv, const float (&v)[kSegIpt], float *s_R) {
  const uint32_t lane = threadIdx.x & 31;
  uint32_t bn = __shfl_down_sync(0xffffffffu, b, 1) & 1u;
  if (lane == 31) bn = fnext;
  const uint32_t ends = (b >> 1) | (bn << 7);  // bit k: my item k ends a row
  // lane tail: sum after my last head (all 8 items when I have none)
  float tail = 0.f;
#pragma unroll
  for (int k = 0; k < kSegIpt; k++) {
    if ((b >> k) & 1u) tail = 0.f;
    tail += v[k];
  }
  // inclusive prefix count of heads and segmented inclusive scan of the tails over lanes
  uint32_t cnt = __popc(b);
  float x = tail;
  if (kVar & kSegBallot) {
    const uint32_t hl = __ballot_sync(0xffffffffu, b != 0u) & (0xFFFFFFFFu >> (31 - lane));
    const int seg0 = hl ? 31 - __clz(hl) : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const float y = __shfl_up_sync(0xffffffffu, x, o);
      const uint32_t c = __shfl_up_sync(0xffffffffu, cnt, o);
      if ((int)lane - o >= seg0) x += y;
      if (lane >= (uint32_t)o) cnt += c;
    }
  } else {
    uint32_t hf = b != 0u;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const float y = __shfl_up_sync(0xffffffffu, x, o);
      const uint32_t f = __shfl_up_sync(0xffffffffu, hf, o);
      const uint32_t c = __shfl_up_sync(0xffffffffu, cnt, o);
      if (lane >= (uint32_t)o) {
        if (!hf) x += y;
        hf |= f;
        cnt += c;
      }
    }
  }
  float run = __shfl_up_sync(0xffffffffu, x, 1);
  if (lane == 0) run = 0.f;
  const uint32_t total_heads = __shfl_sync(0xffffffffu, cnt, 31);
  const uint32_t h0 = __shfl_sync(0xffffffffu, b, 0) & 1u;
  uint32_t row = r0 - h0 + (cnt - __popc(b));  // row of the item before my first head
  const bool head_exists = !h0 && (total_heads > 0 || fnext);
  if (lane == 0 && !head_exists) a.head_row[tile] = kNoRow;
#pragma unroll
  for (int k = 0; k < kSegIpt; k++) {
    if ((b >> k) & 1u) { run = 0.f; ++row; }
    run += v[k];
    if (((ends >> k) & 1u) && row < a.own_n) {
      const uint32_t idx = row - r0;
      if (!h0 && idx == 0) {  // row r0 began in an earlier tile: fix-up
        a.head_row[tile] = r0;
        a.head_val[tile] = run;
      } else if ((kVar & kSegBuf) && idx < 32u) {
        s_R[idx] = a.base + a.d * run;
      } else {
        const float R = a.base + a.d * run;
        if (a.last) a.rank[row] = R;
        else pr_store_contrib(a, a.own_lo + row, R * seg_ldf<kVar>(a.inv_outdeg + a.own_lo + row));
      }
    }
  }
  if (lane == 31) {
    const bool open = !fnext && row < a.own_n;
    a.carry_row[tile] = open ? row : kNoRow;
    a.carry_val[tile] = run;
  }
  if (kVar & kSegBuf) {
    __syncwarp();
    // coalesced apply of the finished rows r0 + [first, lastc] among the tile's first 32
    const int first = h0 ? 0 : 1;
    const int lastc = (int)(total_heads - h0) - (fnext ? 0 : 1);
    const uint32_t myrow = r0 + lane;
    if ((int)lane >= first && (int)lane <= lastc && myrow < a.own_n) {
      const float R = s_R[lane];
      if (a.last) a.rank[myrow] = R;
      else pr_store_contrib(a, a.own_lo + myrow, R * pre_inv);
    }
    __syncwarp();
  }
}

template <class OffT, int kVar>
__global__ void __launch_bounds__(1024, 1) k_pr_seg(const __grid_constant__ PrArgs<OffT> a,
                                                   const uint32_t *__restrict__ seg_src,
                                                   const uint32_t *__restrict__ seg_flags,
                                                   const uint32_t *__restrict__ seg_row, const float *hot_contrib,
                                                   uint32_t hot_k, uint32_t num_tiles) {
  extern __shared__ __align__(16) float s_hot[];  // [hot_k + 4] table, then 32 floats per warp
  for (uint32_t k = threadIdx.x * 4; k < hot_k; k += blockDim.x * 4)
    *reinterpret_cast<float4 *>(s_hot + k) = __ldg(reinterpret_cast<const float4 *>(hot_contrib + k));
  if (threadIdx.x < 4) s_hot[hot_k + threadIdx.x] = 0.f;  // the empty rows' item reads slot hot_k
  __syncthreads();
  const uint32_t hot_sbase = (uint32_t)__cvta_generic_to_shared(s_hot);
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  float *s_R = s_hot + hot_k + 4 + 32 * w;
  const uint32_t stride = gridDim.x * nw;
  uint32_t tile = blockIdx.x * nw + w;
  if (tile >= num_tiles) return;
  const uint4 *src4 = reinterpret_cast<const uint4 *>(seg_src) + 2 * lane;
  uint4 s0 = seg_ld4<kVar>(src4 + (uint64_t)tile * (kSegTile / 4));
  uint4 s1 = seg_ld4<kVar>(src4 + (uint64_t)tile * (kSegTile / 4) + 1);
  uint32_t r0 = seg_ld1<kVar>(seg_row + tile);
  uint32_t fw = 0, fnext = 0;
  if (kVar & kSegPreFlag) {
    fw = seg_ld1<kVar>(seg_flags + (uint64_t)tile * 8 + (lane >> 2));
    fnext = seg_ld1<kVar>(seg_flags + (uint64_t)tile * 8 + 8) & 1u;
  }
  for (;;) {
    if (!(kVar & kSegPreFlag)) {  // this tile's head bits, in flight together with the gathers
      fw = seg_ld1<kVar>(seg_flags + (uint64_t)tile * 8 + (lane >> 2));
      fnext = seg_ld1<kVar>(seg_flags + (uint64_t)tile * 8 + 8) & 1u;
    }
    float v[kSegIpt];
    seg_gather<kVar>(s0, s1, s_hot, hot_sbase, a.contrib_in, v);
    float pre_inv = 0.f;
    if (kVar & kSegBuf) {
      const uint32_t prow = r0 + lane;
      pre_inv = (!a.last && prow < a.own_n) ? seg_ldf<kVar>(a.inv_outdeg + a.own_lo + prow) : 0.f;
    }
    const uint32_t b = (fw >> ((lane & 3) * 8)) & 0xFFu;  // bit k: my item k starts a row
    const uint32_t fn = fnext;
    // next tile's items and first row (and head bits)
    const uint32_t ntile = tile + stride;
    uint32_t nr0 = 0;
    if (ntile < num_tiles) {
      s0 = seg_ld4<kVar>(src4 + (uint64_t)ntile * (kSegTile / 4));
      s1 = seg_ld4<kVar>(src4 + (uint64_t)ntile * (kSegTile / 4) + 1);
      nr0 = seg_ld1<kVar>(seg_row + ntile);
      if (kVar & kSegPreFlag) {
        fw = seg_ld1<kVar>(seg_flags + (uint64_t)ntile * 8 + (lane >> 2));
        fnext = seg_ld1<kVar>(seg_flags + (uint64_t)ntile * 8 + 8) & 1u;
      }
    }
    seg_tile<OffT, kVar>(a, tile, r0, b, fn, pre_inv, v, s_R);
    if (ntile >= num_tiles) break;
    tile = ntile;
    r0 = nr0;
  }
}

// --- seg layout builders (once per graph) ---
template <class OffT>
__global__ void k_seg_deg(const OffT *in_off, uint32_t rows, uint32_t *degp) {
  for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < rows; r += gridDim.x * blockDim.x) {
    const uint64_t d = (uint64_t)in_off[r + 1] - (uint64_t)in_off[r];
    degp[r] = d ? (uint32_t)d : 1u;
  }
}

// item of edge e = seg_off[row(e)] + (e - in_off[row(e)]); row(e) by binary search
template <class OffT>
__global__ void k_seg_fill(const OffT *in_off, uint32_t rows, uint64_t m, const uint32_t *pr_src,
                           const uint32_t *seg_off, uint32_t *seg_src) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t lo = 0, hi = rows;  // last r with in_off[r] <= e
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if ((uint64_t)in_off[mid] <= e) lo = mid;
      else hi = mid;
    }
    seg_src[seg_off[lo] + (e - (uint64_t)in_off[lo])] = pr_src[e];
  }
}

template <class OffT>
__global__ void k_seg_rows(const OffT *in_off, uint32_t rows, const uint32_t *seg_off, uint32_t *seg_src,
                           uint32_t *seg_flags, uint32_t zero_tag, uint64_t padded_items) {
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x, nt = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t r = tid; r < rows; r += nt) {
    const uint32_t p = seg_off[r];
    atomicOr(seg_flags + (p >> 5), 1u << (p & 31));
    if (in_off[r + 1] == in_off[r]) seg_src[p] = zero_tag;
  }
  const uint64_t total = seg_off[rows];
  if (tid == 0) atomicOr(seg_flags + (total >> 5), 1u << (total & 31));  // sentinel: ends the last row
  for (uint64_t i = total + tid; i < padded_items; i += nt) seg_src[i] = zero_tag;
}


// Long chains (a head whose row began more than kShortChain tiles earlier) are
// listed once per graph by k_pr_long_heads and finished one warp each by
// k_pr_fixup_long; every other head is finished by one thread (k_pr_fixup_short).
constexpr uint32_t kShortChain = 8;

static __global__ void k_seg_tiles(const uint32_t *seg_off, uint32_t rows, uint32_t num_tiles, uint32_t *seg_row,
                            uint8_t *is_long, uint32_t *long_c, uint32_t *long_f, uint32_t *long_n) {
  for (uint32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < num_tiles; c += gridDim.x * blockDim.x) {
    const uint64_t i0 = (uint64_t)c * kSegTile;
    uint32_t lo = 0, hi = rows;  // last r with seg_off[r] <= i0
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (seg_off[mid] <= i0) lo = mid;
      else hi = mid;
    }
    seg_row[c] = lo;
    const bool h0 = seg_off[lo] == i0;
    const bool ends = (uint64_t)seg_off[lo + 1] <= i0 + kSegTile;
    bool lng = false;
    if (!h0 && ends) {
      const uint32_t f = seg_off[lo] / kSegTile;
      if (c - f > kShortChain) {
        lng = true;
        const uint32_t pos = atomicAdd(long_n, 1u);
        long_c[pos] = c;
        long_f[pos] = f;
      }
    }
    is_long[c] = lng ? 1 : 0;
  }
}

template <class OffT>
__global__ void k_pr_long_heads(const OffT *in_off, uint64_t rows, uint64_t nnz, const uint32_t *tile_row,
                                uint32_t num_tiles, uint32_t tile_items, uint8_t *is_long, uint32_t *long_c,
                                uint32_t *long_f, uint32_t *long_n) {
  const uint64_t total = rows + nnz;
  for (uint32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < num_tiles; c += gridDim.x * blockDim.x) {
    const uint32_t i0 = tile_row[c], i1 = tile_row[c + 1];
    const uint64_t d0 = (uint64_t)c * tile_items;
    const uint64_t j0 = d0 - i0;
    const uint64_t rs = (uint64_t)in_off[i0];
    bool lng = false;
    if (i1 > i0 && rs < j0) {
      // the row's first item sits on merge-path diagonal i0 + rs
      const uint32_t f = (uint32_t)(((uint64_t)i0 + rs) / tile_items);
      if (c - f > kShortChain) {
        lng = true;
        const uint32_t pos = atomicAdd(long_n, 1u);
        long_c[pos] = c;
        long_f[pos] = f;
      }
    }
    is_long[c] = lng ? 1 : 0;
    (void)total;
  }
}

template <class OffT>
__global__ void k_pr_fixup_short(const __grid_constant__ PrArgs<OffT> a, uint32_t num_tiles, const uint8_t *is_long) {
  for (uint32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < num_tiles; c += gridDim.x * blockDim.x) {
    const uint32_t row = a.head_row[c];
    if (row == kNoRow || is_long[c]) continue;
    float acc = a.head_val[c];
    for (int64_t p = (int64_t)c - 1; p >= 0 && a.carry_row[p] == row; p--) acc += a.carry_val[p];
    pr_apply_row(a, row, acc);
  }
}

template <class OffT>
__global__ void k_pr_fixup_long(const __grid_constant__ PrArgs<OffT> a, const uint32_t *long_c, const uint32_t *long_f,
                                uint32_t n_long) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n_long; i += nw) {
    const uint32_t c = long_c[i], f = long_f[i];
    const uint32_t row = a.head_row[c];
    float acc = 0.f;
    for (uint32_t p = f + lane; p < c; p += 32) acc += a.carry_val[p];  // tiles f..c-1 all carry this row
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0 && row != kNoRow) pr_apply_row(a, row, a.head_val[c] + acc);
  }
}

// ---------------------------------------------------------------------------
// Persistent PageRank loop (resident, single GPU; the default with k_pr_seg):
// ONE cooperative launch runs all supersteps. Per superstep t:
//   phase 1  every CTA loads the hot table packed after superstep t-1 and
//            reduces its tiles (seg_tile, as k_pr_seg);
//   barrier
//   phase 2  rows split between tiles are finished from the head/carry
//            records (as k_pr_fixup_short / _long; split hot rows also write
//            their packed slot), and the other hot sources' new contributions
//            are packed for superstep t+1 (as k_pr_hot_pack);
//   barrier.
// Same tiles, same summation order and same values as the per-superstep
// launches; what goes away is 3 launches per superstep.
struct PrLoop {
  const uint32_t *seg_src, *seg_flags, *seg_row;
  uint32_t tma_off;  // kTma: byte offset of the per-warp staging buffers in dynamic shared memory
  const uint32_t *hot_ids, *hot_slot;  // packed slot -> vertex, vertex -> slot (0xFFFFFFFF: not hot)
  const uint8_t *hot_split;            // slot's row is finished by the fix-up phase
  float *hot_buf[2];                   // packed hot contributions, by superstep parity
  float *contrib[2];
  const uint8_t *is_long;
  const uint32_t *long_c, *long_f;
  uint32_t n_long, hot_k, num_tiles, iters;
  uint32_t *bar;                       // [0] arrivals, [1] generation
  unsigned long long *ts;              // GR_PR_PHASES=1: %globaltimer at the loop start and after each barrier
};

// grid barrier of the persistent PageRank loops: bar[0] is the monotone arrival
// counter (zeroed before every launch), `tgt` thread 0's running target
__device__ __forceinline__ void pr_grid_sync(uint32_t *bar, uint32_t &tgt) { grid_barrier(bar, tgt); }

template <class OffT>
__device__ __forceinline__ void pr_apply_fixup(const PrArgs<OffT> &a, const PrLoop &L, float *hot_next, uint32_t lrow,
                                               float acc) {
  const float R = a.base + a.d * acc;
  const uint32_t v = a.own_lo + lrow;
  if (a.last) {
    a.rank[lrow] = R;
  } else {
    const float c = R * __ldg(a.inv_outdeg + v);
    a.contrib_out[v] = c;
    const uint32_t sl = __ldg(L.hot_slot + v);
    if (sl != 0xFFFFFFFFu) hot_next[sl] = c;
  }
}

template <class OffT, int kVar, bool kPhases = false, bool kTma = false>
__global__ void __launch_bounds__(1024, 1) k_pr_seg_loop(const __grid_constant__ PrArgs<OffT> a0,
                                                        const __grid_constant__ PrLoop L) {
  extern __shared__ __align__(16) float s_hot[];
  const uint32_t hot_sbase = (uint32_t)__cvta_generic_to_shared(s_hot);
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  float *s_R = s_hot + L.hot_k + 4 + 32 * w;
  const uint32_t stride = gridDim.x * nw;
  const uint4 *src4 = reinterpret_cast<const uint4 *>(L.seg_src) + 2 * lane;
  const uint64_t gtid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x, gthreads = (uint64_t)gridDim.x * blockDim.x;
  // kTma: two staging buffers per warp (tile i in buffer i & 1), each with its mbarrier;
  // `tph` holds the parity of the next completion of each buffer
  const uint32_t st0 = hot_sbase + L.tma_off + 2u * w * kTmaBufBytes;
  const uint32_t mb0 = hot_sbase + L.tma_off + 2u * nw * kTmaBufBytes + 16u * w;
  uint32_t tph = 0;
  if (kTma) {
    if (lane == 0) {
      mbar_init(mb0, 1);
      mbar_init(mb0 + 8, 1);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
  }
  auto tma_issue = [&](uint32_t tl, uint32_t j) {  // lane 0: tile tl into buffer j
    const uint32_t dst = st0 + j * kTmaBufBytes, mb = mb0 + 8u * j;
    fence_proxy_async_smem();
    mbar_expect_tx(mb, kTmaItemBytes + kTmaFlagBytes);
    tma_bulk_g2s(dst, L.seg_src + (uint64_t)tl * kSegTile, kTmaItemBytes, mb);
    tma_bulk_g2s(dst + kTmaItemBytes, L.seg_flags + (uint64_t)tl * 8, kTmaFlagBytes, mb);
  };
  // kPhases (GR_PR_PHASES=1, a separate instantiation): CTA 0 stamps %globaltimer
  uint32_t bar_tgt = 0;  // grid barrier target (thread 0)
  if (kPhases && blockIdx.x == 0 && threadIdx.x == 0) L.ts[0] = gtimer();
  for (uint32_t t = 0; t < L.iters; t++) {
    PrArgs<OffT> a = a0;
    a.contrib_in = L.contrib[t & 1];
    a.contrib_out = L.contrib[(t + 1) & 1];
    a.last = (t + 1 == L.iters) ? 1 : 0;
    const float *hot_cur = L.hot_buf[t & 1];
    float *hot_next = L.hot_buf[(t + 1) & 1];
    // ---- phase 1: tiles
    for (uint32_t k = threadIdx.x * 4; k < L.hot_k; k += blockDim.x * 4)
      *reinterpret_cast<float4 *>(s_hot + k) = *reinterpret_cast<const float4 *>(hot_cur + k);
    if (threadIdx.x < 4) s_hot[L.hot_k + threadIdx.x] = 0.f;
    __syncthreads();
    uint32_t tile = blockIdx.x * nw + w;
    if (kTma && tile < L.num_tiles) {
      if (lane == 0) tma_issue(tile, 0);
      uint32_t r0 = seg_ld1<kVar>(L.seg_row + tile);
      for (uint32_t j = 0;; j ^= 1u) {
        const uint32_t buf = st0 + j * kTmaBufBytes;
        mbar_wait(mb0 + 8u * j, (tph >> j) & 1u);
        tph ^= 1u << j;
        const uint4 s0 = lds_v4(buf + 32u * lane), s1 = lds_v4(buf + 32u * lane + 16u);
        const uint32_t fw = lds_u32(buf + kTmaItemBytes + 4u * (lane >> 2));
        const uint32_t fnext = lds_u32(buf + kTmaItemBytes + 32u) & 1u;
        float v[kSegIpt];
        seg_gather<kVar>(s0, s1, s_hot, hot_sbase, a.contrib_in, v);
        float pre_inv = 0.f;
        if (kVar & kSegBuf) {
          const uint32_t prow = r0 + lane;
          pre_inv = (!a.last && prow < a.own_n) ? seg_ldf<kVar>(a.inv_outdeg + a.own_lo + prow) : 0.f;
        }
        const uint32_t b = (fw >> ((lane & 3) * 8)) & 0xFFu;
        const uint32_t ntile = tile + stride;
        uint32_t nr0 = 0;
        if (ntile < L.num_tiles) {
          __syncwarp();  // every lane has read the other buffer's previous tile
          if (lane == 0) tma_issue(ntile, j ^ 1u);
          nr0 = seg_ld1<kVar>(L.seg_row + ntile);
        }
        seg_tile<OffT, kVar>(a, tile, r0, b, fnext, pre_inv, v, s_R);
        if (ntile >= L.num_tiles) break;
        tile = ntile;
        r0 = nr0;
      }
    } else if (!kTma && tile < L.num_tiles) {
      uint4 s0 = seg_ld4<kVar>(src4 + (uint64_t)tile * (kSegTile / 4));
      uint4 s1 = seg_ld4<kVar>(src4 + (uint64_t)tile * (kSegTile / 4) + 1);
      uint32_t r0 = seg_ld1<kVar>(L.seg_row + tile);
      for (;;) {
        const uint32_t fw = seg_ld1<kVar>(L.seg_flags + (uint64_t)tile * 8 + (lane >> 2));
        const uint32_t fnext = seg_ld1<kVar>(L.seg_flags + (uint64_t)tile * 8 + 8) & 1u;
        float v[kSegIpt];
        seg_gather<kVar>(s0, s1, s_hot, hot_sbase, a.contrib_in, v);
        float pre_inv = 0.f;
        if (kVar & kSegBuf) {
          const uint32_t prow = r0 + lane;
          pre_inv = (!a.last && prow < a.own_n) ? seg_ldf<kVar>(a.inv_outdeg + a.own_lo + prow) : 0.f;
        }
        const uint32_t b = (fw >> ((lane & 3) * 8)) & 0xFFu;
        const uint32_t ntile = tile + stride;
        uint32_t nr0 = 0;
        if (ntile < L.num_tiles) {
          s0 = seg_ld4<kVar>(src4 + (uint64_t)ntile * (kSegTile / 4));
          s1 = seg_ld4<kVar>(src4 + (uint64_t)ntile * (kSegTile / 4) + 1);
          nr0 = seg_ld1<kVar>(L.seg_row + ntile);
        }
        seg_tile<OffT, kVar>(a, tile, r0, b, fnext, pre_inv, v, s_R);
        if (ntile >= L.num_tiles) break;
        tile = ntile;
        r0 = nr0;
      }
    }
    pr_grid_sync(L.bar, bar_tgt);
    if (kPhases && blockIdx.x == 0 && threadIdx.x == 0) L.ts[1 + 2 * t] = gtimer();
    // ---- phase 2: rows split between tiles, hot-table pack
    for (uint64_t c = gtid; c < L.num_tiles; c += gthreads) {
      const uint32_t row = a.head_row[c];
      if (row == kNoRow || L.is_long[c]) continue;
      float acc = a.head_val[c];
      for (int64_t p = (int64_t)c - 1; p >= 0 && a.carry_row[p] == row; p--) acc += a.carry_val[p];
      pr_apply_fixup(a, L, hot_next, row, acc);
    }
    for (uint64_t i = gtid >> 5; i < L.n_long; i += gthreads >> 5) {
      const uint32_t c = L.long_c[i], f = L.long_f[i];
      const uint32_t row = a.head_row[c];
      float acc = 0.f;
      for (uint32_t p = f + lane; p < c; p += 32) acc += a.carry_val[p];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
      if (lane == 0 && row != kNoRow) pr_apply_fixup(a, L, hot_next, row, a.head_val[c] + acc);
    }
    if (!a.last)
      for (uint64_t k = gtid; k < L.hot_k; k += gthreads)
        if (!L.hot_split[k]) hot_next[k] = a.contrib_out[L.hot_ids[k]];
    pr_grid_sync(L.bar, bar_tgt);
    if (kPhases && blockIdx.x == 0 && threadIdx.x == 0) L.ts[2 + 2 * t] = gtimer();
  }
}

// ---------------------------------------------------------------------------
// Source-blocked PageRank (§4.2 L210 partition hook,
// L352): when the contribution array is much larger than L2 (n·4 B ≫ 126 MB,
// e.g. R-MAT s26+ resident, or cfg5's replicas at G = 8), the sources are cut
// into B blocks of S vertices whose contributions fit in L2, and the item
// stream is re-laid out block-major: block b holds the in-edges with a source
// in block b, in CSC order (by destination). A "run" is the (destination,
// block) slice of a row; runs play the role rows play in k_pr_seg (one head
// bit per run start, tiles of 256 items, each block padded to whole tiles).
// Per superstep the blocks are reduced one after the other, so the random
// gathers of block b hit an L2-resident 4·S-byte slice (cold gathers carry an
// L2 evict_last policy, the streamed items evict_first); each finished run
// adds its partial sum to acc[destination] with one red.global.add — exactly
// one add per (destination, block) per phase, phases ordered by grid
// barriers, so the fp32 sum order is fixed — and an apply phase turns acc
// into ranks / contributions.
struct PrBlk {
  const uint32_t *items, *flags, *tile_run;  // concatenated blocks (each padded to whole tiles)
  const uint32_t *run_row;                   // run -> destination row
  const uint32_t *blk_tile;                  // [nblk + 1] first tile of each block
  uint32_t nblk, nruns, num_tiles, iters;
  float *acc;                                // [n] partial sums (zeroed by the apply phase)
  const uint32_t *hot_ids;
  float *hot_buf[2];
  float *contrib[2];
  const uint8_t *is_long;
  const uint32_t *long_c, *long_f;
  uint32_t n_long, hot_k;
  uint32_t *bar;
};

template <int kPol> __device__ __forceinline__ uint4 bseg_ld4(const uint4 *p, uint64_t pol) {
  if (kPol) {
    uint4 v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0, %1, %2, %3}, [%4], %5;"
        : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol));
    return v;
  }
  return __ldg(p);
}
template <int kPol> __device__ __forceinline__ float bseg_ldc(const float *p, uint64_t pol) {
  if (kPol) {
    float v;
    asm("ld.global.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));  // written in-launch: not .nc
    return v;
  }
  return ld_weak_f32(p);
}

// One block tile: like seg_tile, with runs for rows; finished runs (other than
// the tile's head run) go through the per-warp buffer s_R (64 runs) and are
// added to acc[run_row] by coalesced red.global.add; rr0/rr1 = run_row of the
// tile's first 64 runs, loaded with the gathers.
__device__ __forceinline__ void bseg_tile(const PrBlk &L, uint32_t *head_row, float *head_val, uint32_t *carry_row,
                                          float *carry_val, uint32_t tile, uint32_t j0, uint32_t b, uint32_t fnext,
                                          uint32_t rr0, uint32_t rr1, const float (&v)[kSegIpt], float *s_R) {
  const uint32_t lane = threadIdx.x & 31;
  uint32_t bn = __shfl_down_sync(0xffffffffu, b, 1) & 1u;
  if (lane == 31) bn = fnext;
  const uint32_t ends = (b >> 1) | (bn << 7);
  float tail = 0.f;
#pragma unroll
  for (int k = 0; k < kSegIpt; k++) {
    if ((b >> k) & 1u) tail = 0.f;
    tail += v[k];
  }
  uint32_t cnt = __popc(b);
  float x = tail;
  const uint32_t hl = __ballot_sync(0xffffffffu, b != 0u) & (0xFFFFFFFFu >> (31 - lane));
  const int seg0 = hl ? 31 - __clz(hl) : 0;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const float y = __shfl_up_sync(0xffffffffu, x, o);
    const uint32_t c = __shfl_up_sync(0xffffffffu, cnt, o);
    if ((int)lane - o >= seg0) x += y;
    if (lane >= (uint32_t)o) cnt += c;
  }
  float run = __shfl_up_sync(0xffffffffu, x, 1);
  if (lane == 0) run = 0.f;
  const uint32_t total_heads = __shfl_sync(0xffffffffu, cnt, 31);
  const uint32_t h0 = __shfl_sync(0xffffffffu, b, 0) & 1u;
  uint32_t j = j0 - h0 + (cnt - __popc(b));
  const bool head_exists = !h0 && (total_heads > 0 || fnext);
  if (lane == 0 && !head_exists) head_row[tile] = kNoRow;
#pragma unroll
  for (int k = 0; k < kSegIpt; k++) {
    if ((b >> k) & 1u) { run = 0.f; ++j; }
    run += v[k];
    if (((ends >> k) & 1u) && j < L.nruns) {
      const uint32_t idx = j - j0;
      if (!h0 && idx == 0) {
        head_row[tile] = j0;
        head_val[tile] = run;
      } else if (idx < 64u) {
        s_R[idx] = run;
      } else {
        atomicAdd(L.acc + __ldg(L.run_row + j), run);
      }
    }
  }
  if (lane == 31) {
    const bool open = !fnext && j < L.nruns;
    carry_row[tile] = open ? j : kNoRow;
    carry_val[tile] = run;
  }
  __syncwarp();
  const int first = h0 ? 0 : 1;
  const int lastc = (int)(total_heads - h0) - (fnext ? 0 : 1);
  if ((int)lane >= first && (int)lane <= lastc && j0 + lane < L.nruns) atomicAdd(L.acc + rr0, s_R[lane]);
  if ((int)lane + 32 >= first && (int)lane + 32 <= lastc && j0 + 32 + lane < L.nruns)
    atomicAdd(L.acc + rr1, s_R[32 + lane]);
  __syncwarp();
}

template <class OffT, int kPol>
__global__ void __launch_bounds__(1024, 1) k_pr_bseg_loop(const __grid_constant__ PrArgs<OffT> a0,
                                                         const __grid_constant__ PrBlk L) {
  extern __shared__ __align__(16) float s_hot[];  // [hot_k + 4] table, then 64 floats per warp
  const uint32_t hot_sbase = (uint32_t)__cvta_generic_to_shared(s_hot);
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  float *s_R = s_hot + L.hot_k + 4 + 64 * w;
  const uint32_t gw = blockIdx.x * nw + w, W = gridDim.x * nw;
  const uint4 *src4 = reinterpret_cast<const uint4 *>(L.items) + 2 * lane;
  const uint64_t gtid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x, gthreads = (uint64_t)gridDim.x * blockDim.x;
  uint64_t pol_keep = 0, pol_stream = 0;
  if (kPol) {
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_keep));
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol_stream));
  }
  uint32_t bar_tgt = 0;  // grid barrier target (thread 0)
  for (uint32_t t = 0; t < L.iters; t++) {
    const float *contrib_in = L.contrib[t & 1];
    float *contrib_out = L.contrib[(t + 1) & 1];
    const bool last = t + 1 == L.iters;
    const float *hot_cur = L.hot_buf[t & 1];
    float *hot_next = L.hot_buf[(t + 1) & 1];
    for (uint32_t k = threadIdx.x * 4; k < L.hot_k; k += blockDim.x * 4)
      *reinterpret_cast<float4 *>(s_hot + k) = *reinterpret_cast<const float4 *>(hot_cur + k);
    if (threadIdx.x < 4) s_hot[L.hot_k + threadIdx.x] = 0.f;
    __syncthreads();
    for (uint32_t blk = 0; blk < L.nblk; blk++) {
      const uint32_t t_lo = L.blk_tile[blk], t_hi = L.blk_tile[blk + 1];
      // ---- block phase: its tiles (gathers from the L2-resident source slice)
      uint32_t tile = t_lo + gw;
      if (tile < t_hi) {
        uint4 s0 = bseg_ld4<kPol>(src4 + (uint64_t)tile * (kSegTile / 4), pol_stream);
        uint4 s1 = bseg_ld4<kPol>(src4 + (uint64_t)tile * (kSegTile / 4) + 1, pol_stream);
        uint32_t j0 = __ldg(L.tile_run + tile);
        for (;;) {
          const uint32_t fw = __ldg(L.flags + (uint64_t)tile * 8 + (lane >> 2));
          const uint32_t fnext = __ldg(L.flags + (uint64_t)tile * 8 + 8) & 1u;
          const uint32_t rr0 = j0 + lane < L.nruns ? __ldg(L.run_row + j0 + lane) : 0u;
          const uint32_t rr1 = j0 + 32 + lane < L.nruns ? __ldg(L.run_row + j0 + 32 + lane) : 0u;
          float v[kSegIpt];
          {
            const uint32_t src[kSegIpt] = {s0.x, s0.y, s0.z, s0.w, s1.x, s1.y, s1.z, s1.w};
#pragma unroll
            for (int k = 0; k < kSegIpt; k++)
              v[k] = (src[k] & kHotTag) ? lds_f32(hot_sbase + 4u * (src[k] & ~kHotTag))
                                        : bseg_ldc<kPol>(contrib_in + src[k], pol_keep);
          }
          const uint32_t b = (fw >> ((lane & 3) * 8)) & 0xFFu;
          const uint32_t ntile = tile + W;
          uint32_t nj0 = 0;
          if (ntile < t_hi) {
            s0 = bseg_ld4<kPol>(src4 + (uint64_t)ntile * (kSegTile / 4), pol_stream);
            s1 = bseg_ld4<kPol>(src4 + (uint64_t)ntile * (kSegTile / 4) + 1, pol_stream);
            nj0 = __ldg(L.tile_run + ntile);
          }
          bseg_tile(L, a0.head_row, a0.head_val, a0.carry_row, a0.carry_val, tile, j0, b, fnext, rr0, rr1, v, s_R);
          if (ntile >= t_hi) break;
          tile = ntile;
          j0 = nj0;
        }
      }
      pr_grid_sync(L.bar, bar_tgt);
      // ---- runs split between tiles of this block (fixed order)
      for (uint64_t c = t_lo + gtid; c < t_hi; c += gthreads) {
        const uint32_t jr = a0.head_row[c];
        if (jr == kNoRow || L.is_long[c]) continue;
        float acc = a0.head_val[c];
        for (int64_t p = (int64_t)c - 1; p >= (int64_t)t_lo && a0.carry_row[p] == jr; p--) acc += a0.carry_val[p];
        atomicAdd(L.acc + __ldg(L.run_row + jr), acc);
      }
      for (uint64_t i = gtid >> 5; i < L.n_long; i += gthreads >> 5) {
        const uint32_t c = L.long_c[i], f = L.long_f[i];
        if (c < t_lo || c >= t_hi) continue;
        const uint32_t jr = a0.head_row[c];
        float acc = 0.f;
        for (uint32_t p = f + lane; p < c; p += 32) acc += a0.carry_val[p];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
        if (lane == 0 && jr != kNoRow) atomicAdd(L.acc + __ldg(L.run_row + jr), a0.head_val[c] + acc);
      }
      pr_grid_sync(L.bar, bar_tgt);
    }
    // ---- apply: R = (1-d)/n + d * acc, 4 vertices per 128-bit access, 2 accesses in flight per thread
    {
      const uint64_t n4 = a0.own_n / 4;
      float4 *acc4 = reinterpret_cast<float4 *>(L.acc);
      const float4 *inv4 = reinterpret_cast<const float4 *>(a0.inv_outdeg);
      float4 *out4 = reinterpret_cast<float4 *>(last ? a0.rank : contrib_out);
      auto rank4 = [&](float4 x) {
        return make_float4(a0.base + a0.d * x.x, a0.base + a0.d * x.y, a0.base + a0.d * x.z, a0.base + a0.d * x.w);
      };
      for (uint64_t q0 = gtid; q0 < n4; q0 += 2 * gthreads) {
        float4 x[2], iv[2];
#pragma unroll
        for (int u = 0; u < 2; u++) {
          const uint64_t q = q0 + u * gthreads;
          if (q < n4) {
            x[u] = acc4[q];
            iv[u] = last ? make_float4(1.f, 1.f, 1.f, 1.f) : __ldg(inv4 + q);
          }
        }
#pragma unroll
        for (int u = 0; u < 2; u++) {
          const uint64_t q = q0 + u * gthreads;
          if (q < n4) {
            const float4 R = rank4(x[u]);
            acc4[q] = make_float4(0.f, 0.f, 0.f, 0.f);
            out4[q] = make_float4(R.x * iv[u].x, R.y * iv[u].y, R.z * iv[u].z, R.w * iv[u].w);
          }
        }
      }
      for (uint64_t v = 4 * n4 + gtid; v < a0.own_n; v += gthreads) {
        const float R = a0.base + a0.d * L.acc[v];
        L.acc[v] = 0.f;
        if (last) a0.rank[v] = R;
        else contrib_out[v] = R * __ldg(a0.inv_outdeg + v);
      }
    }
    pr_grid_sync(L.bar, bar_tgt);
    if (!last) {
      for (uint64_t k = gtid; k < L.hot_k; k += gthreads) hot_next[k] = contrib_out[L.hot_ids[k]];
      pr_grid_sync(L.bar, bar_tgt);
    }
  }
}

// --- blocked layout builders (once per graph) ---
static __global__ void k_bseg_key(const uint32_t *in_src, uint64_t m, uint32_t S, uint32_t *key, uint32_t *val) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x) {
    key[e] = in_src[e] / S;
    val[e] = (uint32_t)e;
  }
}
// first sorted position of every block (bstart[B] = m; empty blocks share the next start)
static __global__ void k_bseg_bounds(const uint32_t *skey, uint64_t m, uint32_t B, uint64_t *bstart) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    const int64_t k = skey[i];
    const int64_t kp = i ? (int64_t)skey[i - 1] : -1;
    if (k != kp)
      for (int64_t b = kp + 1; b <= k; b++) bstart[b] = i;
    if (i == m - 1)
      for (int64_t b = k + 1; b <= (int64_t)B; b++) bstart[b] = m;
  }
}
// row-start bits over edge indices: bit in_off[v] for rows with an in-edge
template <class OffT>
__global__ void k_bseg_rowstart(const OffT *in_off, uint32_t rows, uint32_t *bits) {
  for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < rows; v += gridDim.x * blockDim.x) {
    const uint64_t e = in_off[v];
    if ((uint64_t)in_off[v + 1] > e) atomicOr(bits + (e >> 5), 1u << (e & 31));
  }
}
// place sorted edge i at its padded item position; head = run start
static __global__ void k_bseg_place(const uint32_t *skey, const uint32_t *sval, uint64_t m, const uint64_t *bstart,
                                    const uint64_t *pstart, const uint32_t *in_src, const uint32_t *pr_src,
                                    uint32_t S, const uint32_t *rowbits, uint32_t *items, uint32_t *head) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t b = skey[i], e = sval[i];
    const uint64_t pos = pstart[b] + (i - bstart[b]);
    items[pos] = pr_src[e];
    const bool rs = (rowbits[e >> 5] >> (e & 31)) & 1u;
    head[pos] = (rs || in_src[e - 1] / S != b) ? 1 : 0;  // e == 0 is always a row start
  }
}
// heads -> packed bits (+ sentinel at P)
static __global__ void k_bseg_flags(const uint32_t *head, uint64_t P, uint32_t *flags) {
  for (uint64_t wd = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; wd * 32 <= P;
       wd += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t x = 0;
    for (int k = 0; k < 32; k++) {
      const uint64_t i = wd * 32 + k;
      if (i < P ? head[i] != 0 : i == P) x |= 1u << k;
    }
    flags[wd] = x;
  }
}
// runs: run_off[r] = item of the r-th head, run_row[r] = its destination (the edge's row)
template <class OffT>
__global__ void k_bseg_runs(const uint32_t *skey, const uint32_t *sval, uint64_t m, const uint64_t *bstart,
                            const uint64_t *pstart, const uint32_t *head, const uint32_t *runidx, const OffT *in_off,
                            uint32_t rows, uint32_t *run_off, uint32_t *run_row) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t b = skey[i], e = sval[i];
    const uint64_t pos = pstart[b] + (i - bstart[b]);
    if (!head[pos]) continue;
    uint32_t lo = 0, hi = rows;  // last r with in_off[r] <= e
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if ((uint64_t)in_off[mid] <= e) lo = mid;
      else hi = mid;
    }
    const uint32_t r = runidx[pos];
    run_off[r] = (uint32_t)pos;
    run_row[r] = lo;
  }
}

// hot_split[k] = 1 when hot slot k's row spans two or more tiles (finished by the fix-up phase)
static __global__ void k_seg_hot_split(const uint32_t *hot_ids, uint32_t hot_k, const uint32_t *seg_off,
                                       uint8_t *hot_split) {
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < hot_k; k += gridDim.x * blockDim.x) {
    const uint32_t v = hot_ids[k];
    hot_split[k] = (seg_off[v] / kSegTile) != ((seg_off[v + 1] - 1) / kSegTile) ? 1 : 0;
  }
}

// Rows spanning warp tiles: one warp per tile with a head; the preceding
// tiles' carries of the same row are summed 32 at a time (coalesced, ballot
// for the run end) in a fixed order.
template <class OffT>
__global__ void k_pr_fixup_warp(const __grid_constant__ PrArgs<OffT> a, uint32_t num_tiles) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < num_tiles; c += nw) {
    const uint32_t row = a.head_row[c];
    if (row == kNoRow) continue;
    float acc = 0.f;
    for (int64_t base = (int64_t)c - 1; base >= 0; base -= 32) {
      const int64_t p = base - lane;
      const bool ok = p >= 0 && a.carry_row[p] == row;
      const uint32_t mask = __ballot_sync(0xffffffffu, ok);
      const uint32_t run = mask == 0xffffffffu ? 32u : (uint32_t)(__ffs(~mask) - 1);
      if (lane < run) acc += a.carry_val[p];
      if (run < 32) break;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) pr_apply_row(a, row, a.head_val[c] + acc);
  }
}


static __global__ void k_pr_hot_pack(const float *contrib, const uint32_t *hot_ids, float *hot_contrib, uint32_t k) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < k; i += gridDim.x * blockDim.x)
    hot_contrib[i] = contrib[hot_ids[i]];
}

// PageRank payload: in_src with hot sources replaced by kHotTag | slot.
static __global__ void k_pr_tag(const uint32_t *in_src, uint64_t m, const uint32_t *hot_slot, uint32_t *pr_src) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t u = in_src[e];
    const uint32_t sl = hot_slot[u];
    pr_src[e] = sl != 0xFFFFFFFFu ? (kHotTag | sl) : u;
  }
}

// Rows spanning tiles: head partial + the carries of the preceding tiles, in order.
template <class OffT>
__global__ void k_pr_fixup(const __grid_constant__ PrArgs<OffT> a, uint32_t num_tiles) {
  for (uint32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < num_tiles; c += gridDim.x * blockDim.x) {
    const uint32_t row = a.head_row[c];
    if (row == kNoRow) continue;
    float acc = a.head_val[c];
    for (int64_t p = (int64_t)c - 1; p >= 0 && a.carry_row[p] == row; p--) acc += a.carry_val[p];
    pr_apply_row(a, row, acc);
  }
}

// Merge-path coordinates of every tile start (once per graph / shard): tile_row[c]
// = rows consumed before diagonal c * kPrTile (the last entry is the end).
template <class OffT>
__global__ void k_pr_tiles(const OffT *in_off, uint64_t e_base, uint32_t rows, uint64_t nnz, uint32_t num_tiles,
                           uint32_t *tile_row, uint32_t tile_items = kPrTile) {
  const uint64_t total = (uint64_t)rows + nnz;
  for (uint32_t c = blockIdx.x * blockDim.x + threadIdx.x; c <= num_tiles; c += gridDim.x * blockDim.x) {
    uint64_t diag = (uint64_t)c * tile_items;
    if (diag > total) diag = total;
    tile_row[c] = merge_path_rows(in_off, e_base, rows, nnz, diag);
  }
}

// contrib_0[u] = R_0(u) / outdeg(u) with R_0 = 1/n (reading R3); dangling -> 0 (R2).
// (+ zeroes the grid-barrier counter of the persistent loop that follows, if any)
static __global__ void k_pr_init(uint32_t n, const float *inv_outdeg, float *contrib, uint32_t *bar = nullptr) {
  if (bar && blockIdx.x == 0 && threadIdx.x == 0) bar[0] = 0;
  const float r0 = 1.0f / (float)n;
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
    contrib[v] = r0 * inv_outdeg[v];
}

static __global__ void k_inv_outdeg(uint32_t n, const uint32_t *outdeg, float *inv) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t d = outdeg[v];
    inv[v] = d ? 1.0f / (float)d : 0.f;
  }
}

}  // namespace gr
