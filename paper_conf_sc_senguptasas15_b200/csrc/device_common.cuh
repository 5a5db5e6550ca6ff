// device_common.cuh — device-side state and warp-level helpers shared by the
// GAS kernels (sm_100a only).
#pragma once
#include <cstdint>

#include <cuda_runtime.h>

namespace gr {

constexpr uint32_t kInf = 0xFFFFFFFFu;
constexpr int kWarp = 32;
constexpr int kBlock = 256;              // threads per CTA for the frontier kernels
constexpr int kWarpsPerBlock = kBlock / kWarp;
constexpr uint32_t kHubDegree = 1024;    // > this degree: hub, split into chunks (K6 CTA load balancing)
constexpr uint32_t kChunk = 4096;        // edges per hub chunk (one CTA each)
constexpr int kQueueCap = 128;           // per-warp staging entries before one global append

// Device control block of one run (superstep bookkeeping).
// Lists are ping-ponged by superstep parity so a captured CUDA graph can loop.
struct Ctl {
  uint32_t iter;          // superstep t
  uint32_t epoch_base;    // stamp epoch of superstep 0 (stamps only grow across runs)
  uint32_t max_iters;     // 0 = unlimited
  uint32_t stop;          // 1 once the frontier is empty / max_iters reached
  uint32_t cnt_A[2];      // non-hub list length of A_t (slot t&1)
  uint32_t cnt_H[2];      // hub list length of A_t
  uint32_t cnt_act[2];    // |A_t| (distinct activated vertices; BFS lists are filtered)
  uint32_t cnt_C;         // non-hub changed entries
  uint32_t cnt_CH;        // hub changed entries
  uint32_t cnt_K[2];      // chunk-list length of the A_t hubs
  uint32_t cnt_KC;        // chunk-list length of the changed hubs
  uint32_t ctr_hub;       // dynamic hub work counter (gather / BFS)
  uint32_t ctr_hub2;      // dynamic hub work counter (activate)
  uint32_t done_blocks;   // (unused; see tick1/tick2)
  uint32_t implicit0;     // superstep 0 list is implicitly the owned range (CC: A_0 = V)
  uint32_t trace_cap;
  uint32_t source;        // BFS / SSSP source (programs may read it through Ctx)
  float damping;
  unsigned long long changed;    // |C_t| of the current superstep
  unsigned long long gathered;   // sum indeg(A_t)
  unsigned long long scattered;  // sum outdeg(C_t)
  unsigned long long tot_gathered, tot_scattered;
  // per-superstep counters spread over kSlots addresses (CTA b adds to slot b % kSlots)
  unsigned long long part_g[64], part_c[64], part_s[64], part_a[64];
  uint32_t tick1[64];     // two-level last-CTA ticket: groups of 32 CTAs
  uint32_t tick2;
  uint32_t ext_loop;      // partitioned runs: the host decides termination (global counts)
  uint32_t bar_count, bar_gen;  // grid barrier of the persistent loop
  uint32_t no_hub_c;      // partitioned runs: changed hubs are classified after the exchange
  unsigned long long prof;               // 1: kernels stamp %globaltimer
  unsigned long long kstart[2], kend[2]; // per-kernel span of the current superstep (ns)
  unsigned long long kns[2];             // accumulated kernel ns: [0] gather+apply, [1] activate / BFS expand
  // Activation direction: pull (scan every owned vertex's in-edges for a
  // changed source) when |changed| * pull_div > own_n; 0 = always push.
  uint32_t pull_div;
  uint32_t pull_pending;  // split-kernel loops: this superstep's pull kernel has work
  uint32_t dirty[2];      // changed-bitmap b holds bits of an earlier pull and must be cleared
  uint32_t tot_pull;      // supersteps that activated by pull
  uint32_t dense;         // superstep `iter` gathers densely (previous activation was by pull)
  uint32_t gate;          // ... reading only the changed sources' values (Selective<> programs)
  uint32_t prd_r0;        // ProgPRDelta constants (Ctx)
  uint32_t push;          // fused push supersteps (gr/program.cuh kPushFused): one phase per superstep
  unsigned long long prd_base, prd_dq;
  double prd_thr;
  unsigned long long tot_A, tot_C;  // sum |A_t|, sum |C_t| over the run (bytes model; no trace read-back)
};

constexpr int kSlots = 64;

// Block-wide sum of a per-thread u64 (all threads call; result valid in thread 0).
__device__ __forceinline__ unsigned long long block_sum_u64(unsigned long long x, unsigned long long *s8) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  __syncthreads();
  if ((threadIdx.x & 31) == 0) s8[threadIdx.x >> 5] = x;
  __syncthreads();
  unsigned long long t = 0;
  if (threadIdx.x == 0)
    for (int i = 0; i < (int)(blockDim.x >> 5); i++) t += s8[i];
  return t;
}

// Per-CTA snapshot of the control block: thread 0 issues every load at once
// (both parities, no load depends on another), the CTA reads shared memory.
// Avoids thousands of warps queueing on the same L2 line with a dependent chain.
struct View {
  uint32_t stop, t, epoch_base, implicit0, no_hub_c, source, prof;
  uint32_t cntA[2], cntK[2], cntH[2], cntC, cntCH, cntKC;
  uint32_t pull_div, pull_pending, dirty[2], dense, push, gate;
  float damping;
  unsigned long long prd_base, prd_dq;
  double prd_thr;
};

__device__ __forceinline__ void load_view(const Ctl *c, View &v) {
  __syncthreads();  // a previous snapshot in the same shared slot is no longer read
  if (threadIdx.x == 0) {
    const volatile Ctl *vc = c;
    const uint32_t a0 = vc->cnt_A[0], a1 = vc->cnt_A[1], k0 = vc->cnt_K[0], k1 = vc->cnt_K[1];
    const uint32_t st = vc->stop, t = vc->iter, eb = vc->epoch_base, im = vc->implicit0, nh = vc->no_hub_c;
    const uint32_t so = vc->source, cc = vc->cnt_C, kc = vc->cnt_KC;
    const float dm = vc->damping;
    const uint32_t pr = (uint32_t)vc->prof;
    const uint32_t h0 = vc->cnt_H[0], h1 = vc->cnt_H[1], ch = vc->cnt_CH;
    const uint32_t pd = vc->pull_div, pp = vc->pull_pending, d0 = vc->dirty[0], d1 = vc->dirty[1], dn = vc->dense;
    v.cntH[0] = h0; v.cntH[1] = h1; v.cntCH = ch;
    v.pull_div = pd; v.pull_pending = pp; v.dirty[0] = d0; v.dirty[1] = d1; v.dense = dn; v.push = vc->push; v.gate = vc->gate;
    v.prd_base = vc->prd_base; v.prd_dq = vc->prd_dq; v.prd_thr = vc->prd_thr;
    v.cntA[0] = a0; v.cntA[1] = a1; v.cntK[0] = k0; v.cntK[1] = k1;
    v.stop = st; v.t = t; v.epoch_base = eb; v.implicit0 = im; v.no_hub_c = nh;
    v.source = so; v.cntC = cc; v.cntKC = kc; v.damping = dm; v.prof = pr;
  }
  __syncthreads();
}

// Software grid barrier of the persistent loops (cooperative launch: every CTA
// is resident). The arrival counter only grows within a launch (zeroed before
// it): barrier k of the launch is passed once it reaches k * gridDim.x, so no
// reset and no separate generation word are needed. The arrival is an acq_rel
// atomic (publishes this CTA's writes: MEMBAR.ALL.GPU, and invalidates L1 on
// return), the wait an ld.acquire spin — no fence.sc. Measured 1.2-1.5 us per
// barrier at 148-592 CTAs against 2.3-3.0 us for a fenced count-and-generation
// barrier (profiles/microbench_r02_grid_sync.txt). `target` is thread 0's
// running k * gridDim.x (start at 0).
__device__ __forceinline__ void grid_barrier(uint32_t *count, uint32_t &target) {
  __syncthreads();
  if (threadIdx.x == 0) {
    target += gridDim.x;
    uint32_t old;
    asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(old) : "l"(count) : "memory");
    if (old != target - 1) {
      for (;;) {
        uint32_t now;
        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(now) : "l"(count) : "memory");
        if ((int32_t)(now - target) >= 0) break;
      }
    }
  }
  __syncthreads();
}

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// device-side kernel timing inside CUDA-graph loops (first block start .. last block end)
__device__ __forceinline__ void prof_begin(Ctl *c, const View &v, int k) {
  if (v.prof && threadIdx.x == 0) atomicMin(&c->kstart[k], gtimer());
}
__device__ __forceinline__ void prof_end(Ctl *c, const View &v, int k) {
  if (v.prof) {
    __syncthreads();
    if (threadIdx.x == 0) atomicMax(&c->kend[k], gtimer());
  }
}

// Device view of one owner partition (single GPU = one partition owning V).
template <class OffT> struct Part {
  uint32_t n;             // |V|
  uint32_t own_lo, own_n; // owned destination range
  const OffT *in_off;     // [own_n + 1]  CSC offsets (local vertex index)
  const uint32_t *in_src; // [m_in]       in-edge sources
  const uint8_t *in_w;    // [m_in]       weights (nullable)
  const OffT *out_off;    // [n + 1]      activation CSR offsets (global source id)
  const uint32_t *out_dst;// [m_in]       owned destinations
  const uint32_t *hub_in; // bitmap over owned vertices: indeg > kHubDegree
  const uint32_t *hub_out;// bitmap over all V: activation outdeg > kHubDegree
  uint32_t *val;          // [n] vertex values (replica of superstep t-1; BSP read side)
  uint32_t *stamp;        // [own_n] activation epoch per owned vertex (dedup)
  uint32_t *listA[2];     // non-hub A lists (owned ids, global)
  uint32_t *listH[2];     // hub A lists
  uint32_t *C_v, *C_val;  // changed list (non-hub)
  uint32_t *CH_v, *CH_val;// changed list (activation hubs)
  uint32_t *chkA_h[2], *chkA_c[2]; // A_t hub chunks: (position in listH, chunk index)
  uint32_t *chkC_h, *chkC_c;       // changed-hub chunks: (position in CH list, chunk index)
  unsigned long long *hub_acc;     // per A-hub position: chunk-combined gather result (GatherT, 8 B slots)
  uint32_t *hub_done;              // per A-hub position: chunks done
  const uint32_t *outdeg;          // out-degree of every vertex (Ctx::outdeg)
  uint32_t *cbits[2];     // changed-set bitmaps over V for pull activation (by superstep parity)
  uint32_t *hub_act;      // per static hub: some chunk saw a marked source (dense gathers)
  const uint32_t *s_hubs, *s_chk_h, *s_chk_c;  // static in-hub list and its chunks (dense gathers)
  const ulonglong2 *prd_div;  // ProgPRDelta divisor table (Ctx::prd_div), or nullptr
  uint32_t *estate;       // [m_in] edge states in CSC order (programs with kHasScatter)
  const uint32_t *out_eid;// [m_in] CSC position of every activation-CSR edge (kHasScatter)
  // dense (pull) supersteps of kDstFreeGather programs: edge-segmented tiles over the
  // CSC (kernels_frontier.cuh dense_seg_phase); ds_tiles == 0: not built
  const uint32_t *ds_src;  // [tiles * 256] CSC sources, kDsNoSrc for an empty row's item and the padding
  const uint8_t *ds_w;     // [tiles * 256] weights per item (weighted graphs)
  const uint32_t *ds_flags;// head bit of the first item of every row (+ a sentinel)
  const uint32_t *ds_row;  // [tiles] row of each tile's first item
  const uint32_t *ds_split;// rows with items in more than one tile
  void *ds_acc;            // [own_n] GatherT slots (8 B) of the split rows, identity between uses
  uint32_t *ds_act;        // [own_n / 32 + 1] active bits of the split rows
  uint32_t ds_tiles, ds_nsplit;
  // vertex records (low-degree graphs, kernels_frontier.cuh kRecDeg): one 32-byte
  // record per vertex holding its first kRecDeg neighbours, their weights, the
  // degree and the CSR/CSC offset, so a lane reads its whole adjacency of degree
  // <= kRecDeg with one sector instead of offsets + sources + weights.
  // rec_in[2 lv]: {src[4]}, rec_in[2 lv + 1]: {w[4] as bytes, deg, beg lo, beg hi} (owned rows);
  // rec_out[2 u]: {dst[4]}, rec_out[2 u + 1]: {0, deg, beg lo, beg hi} (activation CSR). nullptr: off
  const uint4 *rec_in;
  const uint4 *rec_out;
  uint32_t stamp_direct;  // FrontierActivate issues the first-stamper atomic without the filter read
  // partitioned frontier programs, exchange fused into the gather: every rank's
  // changed-set buffers of this superstep's parity (own included), written at
  // xp_off (= own_lo) + list position as the gather appends (WarpQueue mirrors)
  uint32_t *xp_v[16], *xp_val[16];
  uint32_t n_xp, xp_off;
  uint32_t *nxt[2];       // fused push supersteps: per-vertex gather accumulators by parity (GatherT = u32)
  const uint8_t *out_w;   // activation CSR weights (fused push supersteps of weighted programs)
  uint32_t n_s_hubs, n_s_chunks;
  Ctl *ctl;
  unsigned long long *trace; // [trace_cap][4]
};

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__device__ __forceinline__ uint32_t ldg_nc(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ float ldg_na(const float *p) {  // read-only, no L1 allocation, reorderable
  float v;
  asm("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint8_t ldg_nc_u8(const uint8_t *p) {
  uint16_t v;
  asm volatile("ld.global.nc.L1::no_allocate.u8 %0, [%1];" : "=h"(v) : "l"(p));
  return (uint8_t)v;
}

__device__ __forceinline__ uint4 ldg_nc_v4(const uint4 *p) {
  uint4 v;
  asm("ld.global.nc.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}

// L2-coherent read (bypasses L1, so stamps written by other SMs are seen)
__device__ __forceinline__ uint32_t ld_cg(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}

// First-stamper test: a plain L2 read filters the (many) edges that reach an
// already-stamped vertex, so only the first few pay the serialized atomic on a
// popular target's address.
__device__ __forceinline__ bool stamp_first(uint32_t *stamp, uint32_t epoch) {
  return ld_cg(stamp) != epoch && atomicExch(stamp, epoch) != epoch;
}

__device__ __forceinline__ bool test_bit(const uint32_t *bits, uint32_t i) {
  return (__ldg(bits + (i >> 5)) >> (i & 31)) & 1u;
}
// bit test on a bitmap written earlier in the same kernel (L2, not the nc path)
__device__ __forceinline__ bool test_bit_cg(const uint32_t *bits, uint32_t i) {
  return (ld_cg(bits + (i >> 5)) >> (i & 31)) & 1u;
}
// Changed-set bitmaps of dense supersteps: written in an earlier phase, read after
// a grid barrier (whose acquire invalidates L1) or a kernel boundary — an ordinary
// weak, L1-cached load is coherent there (ld.global.cg would send every probe of
// the small bitmap to L2: R-MAT CC 2.43 -> 3.84 ms, tolerance PageRank 56.7 -> 66.9 ms)
__device__ __forceinline__ uint32_t ld_bits(const uint32_t *bits, uint32_t i) { return bits[i >> 5]; }
__device__ __forceinline__ bool test_bit_w(const uint32_t *bits, uint32_t i) { return (ld_bits(bits, i) >> (i & 31)) & 1u; }

// Warp-inclusive scan of a uint32 (all lanes participate).
__device__ __forceinline__ uint32_t warp_incl_scan(uint32_t x) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane_id() >= (uint32_t)o) x += y;
  }
  return x;
}

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}

// Per-warp staging queue: entries are collected in shared memory and appended
// to a global list with ONE atomicAdd per flush (not one per element).
struct WarpQueue {
  uint32_t *s_a;   // [kQueueCap] shared
  uint32_t *s_b;   // [kQueueCap] shared or nullptr (pair lists)
  uint32_t n;      // warp-uniform fill level
  // optional mirrors (partitioned frontier exchange fused into the gather): every
  // flushed entry at list position p is also stored at mir_off + p of each mirror
  uint32_t *const *mir_a = nullptr;
  uint32_t *const *mir_b = nullptr;
  uint32_t n_mir = 0, mir_off = 0;
  __device__ __forceinline__ void mirror(uint32_t pos, uint32_t a, uint32_t b) const {
    for (uint32_t q = 0; q < n_mir; q++) {
      mir_a[q][mir_off + pos] = a;
      mir_b[q][mir_off + pos] = b;
    }
  }
  __device__ void flush(uint32_t *g_a, uint32_t *g_b, uint32_t *g_cnt) {
    __syncwarp();
    if (n == 0) return;
    uint32_t base = 0;
    if (lane_id() == 0) base = atomicAdd(g_cnt, n);
    base = __shfl_sync(0xffffffffu, base, 0);
    for (uint32_t i = lane_id(); i < n; i += 32) {
      g_a[base + i] = s_a[i];
      if (g_b) g_b[base + i] = s_b[i];
      if (n_mir) mirror(base + i, s_a[i], s_b[i]);
    }
    __syncwarp();
    n = 0;
  }
  // Final flush of every warp of the CTA with ONE global atomic (all threads call).
  __device__ void block_flush(uint32_t *g_a, uint32_t *g_b, uint32_t *g_cnt, uint32_t *s_off) {
    const uint32_t w = threadIdx.x >> 5, nw = blockDim.x >> 5;
    __syncthreads();
    if ((threadIdx.x & 31) == 0) s_off[w] = n;
    __syncthreads();
    if (threadIdx.x == 0) {
      uint32_t tot = 0;
      for (uint32_t i = 0; i < nw; i++) { const uint32_t c = s_off[i]; s_off[i] = tot; tot += c; }
      s_off[nw] = tot ? atomicAdd(g_cnt, tot) : 0u;
    }
    __syncthreads();
    const uint32_t base = s_off[nw] + s_off[w];
    for (uint32_t i = threadIdx.x & 31; i < n; i += 32) {
      g_a[base + i] = s_a[i];
      if (g_b) g_b[base + i] = s_b[i];
      if (n_mir) mirror(base + i, s_a[i], s_b[i]);
    }
    __syncwarp();
    n = 0;
  }
  __device__ void push(bool p, uint32_t a, uint32_t b, uint32_t *g_a, uint32_t *g_b, uint32_t *g_cnt) {
    uint32_t mask = __ballot_sync(0xffffffffu, p);
    if (mask == 0) return;
    uint32_t k = __popc(mask);
    if (n + k > (uint32_t)kQueueCap) flush(g_a, g_b, g_cnt);
    if (p) {
      uint32_t pos = n + __popc(mask & lanemask_lt());
      s_a[pos] = a;
      if (s_b) s_b[pos] = b;
    }
    n += k;
    __syncwarp();
  }
};

}  // namespace gr
