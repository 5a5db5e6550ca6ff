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
};

template <class OffT>
__device__ __forceinline__ void pr_apply_row(const PrArgs<OffT> &a, uint32_t lrow, float acc) {
  const float R = a.base + a.d * acc;
  const uint32_t v = a.own_lo + lrow;
  if (a.last) a.rank[lrow] = R;
  else a.contrib_out[v] = R * __ldg(a.inv_outdeg + v);
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

// Long chains (a head whose row began more than kShortChain tiles earlier) are
// listed once per graph by k_pr_long_heads and finished one warp each by
// k_pr_fixup_long; every other head is finished by one thread (k_pr_fixup_short).
constexpr uint32_t kShortChain = 8;

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


// ---------------------------------------------------------------------------
// Persistent warp-range kernel: warp w walks the CONTIGUOUS tiles
// [w*T, (w+1)*T) and carries the open row's partial sum in registers from one
// tile to the next, so a row split between two tiles of the same warp is
// finished by that warp. Only rows that cross a warp-range boundary are left to
// k_pr_fixup (one head/carry record per warp range, indexed by the global warp).
constexpr uint32_t kRangeTiles = 8;  // warp tiles per chunk (2048 items)

template <class OffT, bool kHot>
__device__ __forceinline__ void pr_warp_range(const PrArgs<OffT> &a, uint32_t wid, uint32_t t0, uint32_t t1,
                                              PrWarpSmem &S, const float *s_hot) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t total = (uint64_t)a.own_n + a.m_in;
  uint32_t pend_row = kNoRow;  // row whose partial sum is carried into the next tile
  float pend_val = 0.f;
  bool range_head = false;     // pend_row began before this warp's range
  bool head_written = false;
  for (uint32_t tile = t0; tile < t1; tile++) {
    const uint64_t d0 = (uint64_t)tile * kWTile;
    const uint64_t d1 = d0 + kWTile < total ? d0 + kWTile : total;
    const uint32_t i0 = __ldg(a.tile_row + tile), i1 = __ldg(a.tile_row + tile + 1);
    const uint64_t j0 = d0 - i0;
    const uint32_t ni = i1 - i0, nj = (uint32_t)((d1 - i1) - j0);
    const bool started_before = ((uint64_t)a.in_off[i0] - a.e_base) < j0;
    if (tile == t0) {
      pend_row = i0;
      pend_val = 0.f;
      range_head = started_before;
    }
    __syncwarp();
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
    const float cx = __shfl_sync(0xffffffffu, x, 31);  // partial of row i1 inside this tile
    __syncwarp();
    const bool run_end = (lane == 31) || (inext != i);
    if (run_end && i < ni) S.s_tot[pr_pad(i)] += x;
    __syncwarp();
    if (ni > 0) {
      // row i0: add the partial carried from this warp's previous tile
      const float tot0 = S.s_tot[pr_pad(0)] + (started_before && pend_row == i0 ? pend_val : 0.f);
      const bool is_head = started_before && range_head;
      if (lane == 0) {
        if (is_head) {
          a.head_row[wid] = i0;
          a.head_val[wid] = tot0;
        } else {
          pr_apply_row(a, i0, tot0);
        }
      }
      head_written |= is_head;
      for (uint32_t k = 1 + lane; k < ni; k += 32) pr_apply_row(a, i0 + k, S.s_tot[pr_pad(k)]);
      pend_row = i1;
      pend_val = cx;
      range_head = false;
    } else {
      pend_val = (pend_row == i0 ? pend_val : 0.f) + cx;
      pend_row = i0;
    }
  }
  if (lane == 0 && t0 < t1) {
    if (!head_written) a.head_row[wid] = kNoRow;
    a.carry_row[wid] = pend_row < a.own_n ? pend_row : kNoRow;
    a.carry_val[wid] = pend_val;
  } else if (lane == 0) {
    a.head_row[wid] = kNoRow;
    a.carry_row[wid] = kNoRow;
    a.carry_val[wid] = 0.f;
  }
}

template <class OffT, bool kHot>
__global__ void __launch_bounds__(1024, 1) k_pr_warp_range(const __grid_constant__ PrArgs<OffT> a,
                                                          const float *hot_contrib, uint32_t hot_k,
                                                          uint32_t num_tiles) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  float *s_hot = reinterpret_cast<float *>(smem_raw);
  PrWarpSmem *S = reinterpret_cast<PrWarpSmem *>(smem_raw + (kHot ? 4ull * hot_k : 0ull));
  if (kHot) {
    for (uint32_t k = threadIdx.x * 4; k < hot_k; k += blockDim.x * 4)
      *reinterpret_cast<float4 *>(s_hot + k) = __ldg(reinterpret_cast<const float4 *>(hot_contrib + k));
    __syncthreads();
  }
  // interleaved chunks of kRangeTiles contiguous tiles: balanced across warps
  // (hot/cold source mix varies along the graph), carries stay in registers
  // inside a chunk, one head/carry record per chunk for k_pr_fixup
  const uint32_t w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const uint32_t wid = blockIdx.x * nw + w, W = gridDim.x * nw;
  const uint32_t nchunks = (num_tiles + kRangeTiles - 1) / kRangeTiles;
  for (uint32_t c = wid; c < nchunks; c += W) {
    const uint32_t t0 = c * kRangeTiles, t1 = min(t0 + kRangeTiles, num_tiles);
    pr_warp_range<OffT, kHot>(a, c, t0, t1, S[w], s_hot);
  }
}

// hot_contrib[k] = contrib[hot_ids[k]] (after the previous superstep finished)
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
static __global__ void k_pr_init(uint32_t n, const float *inv_outdeg, float *contrib) {
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
