// kernels_frontier.cuh — frontier-driven GAS superstep kernels (SSSP, CC, BFS,
// custom programs). SURVEY.md §8(a) rows a2, a4, a5, a6, a7.
//
// One superstep t (§4.4, BSP):
//   k_gather_apply  : for v in A_t: acc = (+) gatherMap(val[u], w) over in-edges
//                     (L250-251), then apply (L252) against val[v]; changed
//                     vertices go to the changed list C_t WITH their new value.
//                     val[] is not written here, so every gather reads the
//                     values of superstep t-1 (BSP, reading R5).
//   k_activate      : commit val[u] = new for u in C_t, then FrontierActivate
//                     (L254, L270): atomically stamp every out-neighbour x with
//                     the epoch of t+1; the first stamper appends x to A_{t+1}.
//                     The last CTA to finish closes the superstep (trace row,
//                     counters, termination, CUDA-graph loop condition).
//   k_bfs_expand    : BFS phase fusion (L276): apply (depth = t) + activate in
//                     one pass over A_t; gather eliminated (L274).
// Load balancing (CTA load balancing from the active list, L270, L352): a warp
// takes 32 list entries; lanes with degree > kPackDeg are processed warp-
// cooperatively one at a time, lanes with degree <= kPackDeg are packed 32 edges per
// round (owner found by a shuffle binary search); vertices with degree >
// kHubDegree live in a separate hub list processed one CTA per vertex.
#pragma once
#include "device_common.cuh"
#include "gr/program.cuh"

namespace gr {

constexpr int kBatch = 4;  // edges in flight per lane per memory phase
#ifndef GR_PACK_DEG  // A/B builds
#define GR_PACK_DEG 128
#endif
// gather lanes whose vertex has at most kPackDeg in-edges have their edges packed
// 32 per round across the warp; larger ones (up to kHubDegree) are walked by the
// whole warp one vertex at a time (128 edges per step). 128 rather than 32: the
// web graph's rows of 33-128 in-edges (14 % of cfg4's edges, ~1.4 per 32-vertex
// group) each cost a whole warp step with most lanes idle.
constexpr uint32_t kPackDeg = GR_PACK_DEG;
// One shared-memory scratch for the staging arrays of every phase of a kernel: the
// phases of the persistent loop are separated by grid barriers (which begin and end
// with __syncthreads), so their per-warp queues and reduction slots are never live
// together. Declared once at namespace scope, it costs the kernel the largest
// phase's footprint (10.3 KB) instead of the sum over its inlined phases (up to 38 KB
// for SSSP), leaving that much more of the SM's 256 KB to L1 — which the random
// gathers hit (GR_NO_SMEM_UNION: per-phase arrays, for A/B).
constexpr uint32_t kSqBytes1 = kWarpsPerBlock * kQueueCap * 4;      // one queue array per warp
constexpr uint32_t kSqBytes2 = 2 * kSqBytes1;                         // two (pair lists)
constexpr uint32_t kPhaseSmemBytes = kSqBytes2 + kWarpsPerBlock * 32 * 8 + kWarpsPerBlock * 8;
__shared__ __align__(16) unsigned char g_phase_smem[kPhaseSmemBytes];
#ifdef GR_NO_SMEM_UNION
#define GR_SQ1(name) __shared__ uint32_t name[kWarpsPerBlock][kQueueCap]
#define GR_SQ2(name) __shared__ uint32_t name[kWarpsPerBlock][2][kQueueCap]
#else
#define GR_SQ1(name) auto &name = *reinterpret_cast<uint32_t(*)[kWarpsPerBlock][kQueueCap]>(g_phase_smem)
#define GR_SQ2(name) auto &name = *reinterpret_cast<uint32_t(*)[kWarpsPerBlock][2][kQueueCap]>(g_phase_smem)
#endif
constexpr uint32_t kRecDeg = 4;  // neighbours held in a vertex record (Part::rec_in / rec_out)
static_assert(kRecDeg == (uint32_t)kBatch, "a record's neighbours form one activation batch");
#ifdef GR_NO_GATE  // A/B build: dense supersteps read every source's value
constexpr bool kGateSelective = false;
#else
constexpr bool kGateSelective = true;
#endif
// how superstep t's FrontierActivate ran (close_superstep)
constexpr int kPush = 0;       // out-edge expansion of C_t with stamps
constexpr int kPullScan = 1;   // BFS: in-edge scan of every vertex for a C_t source -> A_{t+1} list
constexpr int kPullDense = 2;  // gather programs: C_t marked only; superstep t+1 gathers densely

// ----------------------------------------------------------------- helpers
template <class OffT> __device__ __forceinline__ Ctx make_ctx(const Part<OffT> &P, const View &V) {
  Ctx cx;
  cx.iter = V.t;
  cx.n = P.n;
  cx.source = V.source;
  cx.damping = V.damping;
  cx.outdeg = P.outdeg;
  cx.prd_base = V.prd_base;
  cx.prd_dq = V.prd_dq;
  cx.prd_thr = V.prd_thr;
  cx.prd_r0 = 0;
  cx.prd_div = P.prd_div;
  return cx;
}

// gatherMap's edge argument: the mutable edge state (kHasScatter programs; an
// L2-coherent read, the state is rewritten by the previous superstep's
// scatter), else the weight (or 0)
template <class Prog, class OffT>
__device__ __forceinline__ uint32_t edge_w(const Part<OffT> &P, uint64_t e) {
  if constexpr (HasScatter<Prog>::value) return ld_cg(P.estate + e);
  else return Prog::kUsesWeights ? (uint32_t)ldg_nc_u8(P.in_w + e) : 0u;
}

// CSC / CSR position of packed item k owned by lane o, from o's (row start - packed
// offset): one shuffle (two for 64-bit offsets) instead of the start and the offset
template <class OffT>
__device__ __forceinline__ uint64_t packed_pos(uint64_t bx, int o, uint32_t k) {
  if constexpr (sizeof(OffT) == 4) return (uint32_t)(__shfl_sync(0xffffffffu, (uint32_t)bx, o) + k);
  else return __shfl_sync(0xffffffffu, bx, o) + k;
}

template <class Prog>
__device__ __forceinline__ typename Prog::GatherT warp_reduce_prog(typename Prog::GatherT x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x = Prog::gatherReduce(x, __shfl_xor_sync(0xffffffffu, x, o));
  return x;
}


// Gather for up to 32 vertices held one per lane (valid, beg, deg, dval).
// Returns the gatherReduce result of the lane's own vertex. kDense (pull
// supersteps): also sets `act` iff some in-edge source is marked in `bits`
// (the changed set of the previous superstep), i.e. the vertex is in A_t.
template <class Prog, bool kDense, bool kGateT = false, class OffT>
__device__ typename Prog::GatherT gather_warp(const Part<OffT> &P, bool valid, uint64_t beg, uint32_t deg,
                                              uint32_t dval, typename Prog::GatherT *sred, const Ctx &cx,
                                              const uint32_t *bits, bool &act, bool direct = false,
                                              uint4 rs = uint4{}, uint32_t w4 = 0) {
  using G = typename Prog::GatherT;
  const uint32_t lane = lane_id();
  G acc = Prog::identity();
  act = false;
  // dense supersteps of selective programs may read val[u] only for changed sources
  // (Selective<>; chosen per superstep by close_superstep: Ctl::gate)
  constexpr bool kGate = kDense && kGateT && kGateSelective && Selective<Prog>::value;
#ifndef GR_NO_PREFETCH
  // the packed rounds below walk the rows of up to kPackDeg in-edges 32 edges at a
  // time; prefetching each row's first and last line into L1 now turns the source
  // loads of all but the first rounds into L1 hits (one dependent L2 trip less each)
  if (valid && !direct && deg > 0 && deg <= kPackDeg) {
    asm volatile("prefetch.global.L1 [%0];" ::"l"(P.in_src + beg));
    if (deg > 8) asm volatile("prefetch.global.L1 [%0];" ::"l"(P.in_src + beg + deg - 1));
  }
#endif
  // vertex records: a lane whose vertex has degree <= kRecDeg holds its sources
  // (rs) and weights (w4) already and gathers alone, all loads in one phase
  if (direct) {
    const uint32_t us[kRecDeg] = {rs.x, rs.y, rs.z, rs.w};
    uint32_t ew[kRecDeg], vv[kRecDeg], bw[kRecDeg];
    bool a[kRecDeg], h[kRecDeg];
#pragma unroll
    for (uint32_t q = 0; q < kRecDeg; q++) {
      a[q] = q < deg;
      if constexpr (HasScatter<Prog>::value) ew[q] = a[q] ? ld_cg(P.estate + beg + q) : 0u;
      else ew[q] = Prog::kUsesWeights ? (w4 >> (8 * q)) & 0xFFu : 0u;
      if (!kGate) vv[q] = a[q] ? P.val[us[q]] : 0u;
      bw[q] = (kDense && a[q]) ? ld_bits(bits, us[q]) : 0u;
    }
    G r = Prog::identity();
    bool hh = false;
#pragma unroll
    for (uint32_t q = 0; q < kRecDeg; q++) {
      h[q] = kDense && a[q] && ((bw[q] >> (us[q] & 31)) & 1u);
      if (kGate) vv[q] = h[q] ? P.val[us[q]] : 0u;
    }
#pragma unroll
    for (uint32_t q = 0; q < kRecDeg; q++) {
      if (a[q] && (!kGate || h[q])) r = Prog::gatherReduce(r, Prog::gatherMap(dval, vv[q], ew[q], us[q], cx));
      hh |= h[q];
    }
    acc = r;
    act = hh;
  }
  // warp-cooperative: one vertex of degree in (32, kHubDegree] at a time
  uint32_t big = __ballot_sync(0xffffffffu, valid && deg > kPackDeg);
  while (big) {
    const int L = __ffs(big) - 1;
    big &= big - 1;
    const uint64_t b = __shfl_sync(0xffffffffu, beg, L);
    const uint32_t d = __shfl_sync(0xffffffffu, deg, L);
    const uint32_t dv = __shfl_sync(0xffffffffu, dval, L);
    G r = Prog::identity();
    bool hit = false;
    uint32_t k = lane;
    for (; k + 96 < d; k += 128) {  // 4 independent loads in flight per lane
      uint32_t u[4], w[4];
#pragma unroll
      for (int q = 0; q < 4; q++) {
        u[q] = ldg_nc(P.in_src + b + k + 32 * q);
        w[q] = edge_w<Prog>(P, b + k + 32 * q);
      }
      uint32_t v[4], bw[4];
#pragma unroll
      for (int q = 0; q < 4; q++) {
        if (!kGate) v[q] = P.val[u[q]];
        if (kDense) bw[q] = ld_bits(bits, u[q]);
      }
      bool h[4];
#pragma unroll
      for (int q = 0; q < 4; q++) {
        h[q] = kDense && ((bw[q] >> (u[q] & 31)) & 1u);
        if (kGate) v[q] = h[q] ? P.val[u[q]] : 0u;
      }
#pragma unroll
      for (int q = 0; q < 4; q++) {
        if (!kGate || h[q]) r = Prog::gatherReduce(r, Prog::gatherMap(dv, v[q], w[q], u[q], cx));
        hit |= h[q];
      }
    }
    for (; k < d; k += 32) {
      const uint32_t u = ldg_nc(P.in_src + b + k);
      const uint32_t w = edge_w<Prog>(P, b + k);
      const bool h = kDense && test_bit_w(bits, u);
      if (!kGate || h) r = Prog::gatherReduce(r, Prog::gatherMap(dv, P.val[u], w, u, cx));
      hit |= h;
    }
    r = warp_reduce_prog<Prog>(r);
    const bool any = kDense ? (__any_sync(0xffffffffu, hit) != 0) : false;
    if ((int)lane == L) {
      acc = r;
      act = any;
    }
  }
  // fine-grained: pack the edges of all lanes with degree <= kPackDeg, 32 per round;
  // kBatch rounds' loads (sources + weights, then source values) are issued
  // together before their segmented reductions
  const uint32_t sd = (valid && !direct && deg <= kPackDeg) ? deg : 0u;
  const uint32_t incl = warp_incl_scan(sd);
  const uint32_t excl = incl - sd;
  const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
  if (total == 0) return acc;
  sred[lane] = Prog::identity();
  const uint64_t bx = beg - excl;  // CSC position of packed item k of this lane's row: bx + k
  uint32_t hitmask = 0;  // kDense: owner lanes with a marked source (warp-uniform)
  __syncwarp();
  for (uint32_t rb = 0; rb < total; rb += 32u * kBatch) {
    int own[kBatch];
    uint32_t su[kBatch], sw[kBatch], dv[kBatch];
    bool act_q[kBatch];
#pragma unroll
    for (int q = 0; q < kBatch; q++) {
      const uint32_t k = rb + q * 32u + lane;
      int o = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const uint32_t e = __shfl_sync(0xffffffffu, excl, o + step);
        if (e <= k) o += step;
      }
      own[q] = o;
      const uint64_t e = packed_pos<OffT>(bx, o, k);
      dv[q] = DstFree<Prog>::value ? 0u : __shfl_sync(0xffffffffu, dval, o);  // gatherMap ignores it otherwise
      act_q[q] = k < total;
      su[q] = act_q[q] ? ldg_nc(P.in_src + e) : 0u;
      sw[q] = act_q[q] ? edge_w<Prog>(P, e) : 0u;
    }
    uint32_t sv[kBatch], sb[kBatch];
#pragma unroll
    for (int q = 0; q < kBatch; q++) {
      if (!kGate) sv[q] = act_q[q] ? P.val[su[q]] : 0u;
      if (kDense) sb[q] = act_q[q] ? ld_bits(bits, su[q]) : 0u;
    }
    if (kGate) {  // only the changed sources' values: unmarked items map to identity()
#pragma unroll
      for (int q = 0; q < kBatch; q++) {
        act_q[q] = act_q[q] && ((sb[q] >> (su[q] & 31)) & 1u);
        sv[q] = act_q[q] ? P.val[su[q]] : 0u;
      }
    }
#pragma unroll
    for (int q = 0; q < kBatch; q++) {
      if (rb + q * 32u >= total) break;  // warp-uniform
      const int o = own[q];
      if (kDense) {
        const bool h = act_q[q] && ((sb[q] >> (su[q] & 31)) & 1u);
        // owners of hits: OR of (1 << owner) over the warp (one REDUX)
        hitmask |= __reduce_or_sync(0xffffffffu, h ? (1u << o) : 0u);
      }
      G x = act_q[q] ? Prog::gatherMap(dv[q], sv[q], sw[q], su[q], cx) : Prog::identity();
      // segmented inclusive scan keyed by owner lane (owners are non-decreasing)
      const int prev_o = __shfl_up_sync(0xffffffffu, o, 1);
      uint32_t f = (lane == 0 || prev_o != o) ? 1u : 0u;
#pragma unroll
      for (int dd = 1; dd < 32; dd <<= 1) {
        const G y = __shfl_up_sync(0xffffffffu, x, dd);
        const uint32_t g = __shfl_up_sync(0xffffffffu, f, dd);
        if (lane >= (uint32_t)dd) {
          if (!f) x = Prog::gatherReduce(y, x);
          f |= g;
        }
      }
      const int next_o = __shfl_down_sync(0xffffffffu, o, 1);
      if (lane == 31 || next_o != o) sred[o] = Prog::gatherReduce(sred[o], x);
      __syncwarp();
    }
  }
  if (sd > 0) {
    acc = sred[lane];
    if (kDense) act = (hitmask >> lane) & 1u;
  }
  __syncwarp();
  return acc;
}

// Block-wide gather of one hub vertex (chunk). kDense: *act (thread 0) = some
// source in the chunk is marked in `bits`.
template <class Prog, bool kDense, bool kGateT = false, class OffT>
__device__ typename Prog::GatherT gather_block(const Part<OffT> &P, uint64_t beg, uint32_t deg, uint32_t dval,
                                               typename Prog::GatherT *sblk, const Ctx &cx, const uint32_t *bits,
                                               bool *act) {
  using G = typename Prog::GatherT;
  constexpr bool kGate = kDense && kGateT && kGateSelective && Selective<Prog>::value;  // see gather_warp
  G r = Prog::identity();
  bool hit = false;
  uint32_t k = threadIdx.x;
  for (; k + 3 * kBlock < deg; k += 4 * kBlock) {
    uint32_t u[4], w[4];
#pragma unroll
    for (int q = 0; q < 4; q++) {
      u[q] = ldg_nc(P.in_src + beg + k + q * kBlock);
      w[q] = edge_w<Prog>(P, beg + k + q * kBlock);
    }
    uint32_t v[4], bw[4];
#pragma unroll
    for (int q = 0; q < 4; q++) {
      if (!kGate) v[q] = P.val[u[q]];
      if (kDense) bw[q] = ld_bits(bits, u[q]);
    }
    bool h[4];
#pragma unroll
    for (int q = 0; q < 4; q++) {
      h[q] = kDense && ((bw[q] >> (u[q] & 31)) & 1u);
      if (kGate) v[q] = h[q] ? P.val[u[q]] : 0u;
    }
#pragma unroll
    for (int q = 0; q < 4; q++) {
      if (!kGate || h[q]) r = Prog::gatherReduce(r, Prog::gatherMap(dval, v[q], w[q], u[q], cx));
      hit |= h[q];
    }
  }
  for (; k < deg; k += kBlock) {
    const uint32_t u = ldg_nc(P.in_src + beg + k);
    const uint32_t w = edge_w<Prog>(P, beg + k);
    const bool h = kDense && test_bit_w(bits, u);
    if (!kGate || h) r = Prog::gatherReduce(r, Prog::gatherMap(dval, P.val[u], w, u, cx));
    hit |= h;
  }
  if (kDense) {
    const int any = __syncthreads_or(hit ? 1 : 0);
    if (threadIdx.x == 0) *act = any != 0;
  }
  r = warp_reduce_prog<Prog>(r);
  if (lane_id() == 0) sblk[threadIdx.x / 32] = r;
  __syncthreads();
  G t = Prog::identity();
  if (threadIdx.x == 0)
    for (int i = 0; i < kWarpsPerBlock; i++) t = Prog::gatherReduce(t, sblk[i]);
  __syncthreads();
  return t;  // valid in thread 0
}

__device__ __forceinline__ uint32_t chunk_len(uint64_t deg, uint32_t ci) {
  const uint64_t rest = deg - (uint64_t)ci * kChunk;
  return (uint32_t)(rest < kChunk ? rest : kChunk);
}

// Append a hub to the A list of `slot` together with its edge chunks
// (by out-degree for BFS, whose A-phase is the expansion; else by in-degree).
template <bool kByOut, class OffT>
__device__ void append_hub_A(const Part<OffT> &P, uint32_t x, uint32_t slot) {
  Ctl *c = P.ctl;
  const uint32_t pos = atomicAdd(&c->cnt_H[slot], 1u);
  P.listH[slot][pos] = x;
  const uint64_t deg = kByOut ? (uint64_t)P.out_off[x + 1] - (uint64_t)P.out_off[x]
                              : (uint64_t)P.in_off[x - P.own_lo + 1] - (uint64_t)P.in_off[x - P.own_lo];
  const uint32_t nch = (uint32_t)((deg + kChunk - 1) / kChunk);
  const uint32_t kb = atomicAdd(&c->cnt_K[slot], nch);
  for (uint32_t i = 0; i < nch; i++) {
    P.chkA_h[slot][kb + i] = pos;
    P.chkA_c[slot][kb + i] = i;
  }
}

// Append a changed hub (by activation out-degree) with its out-edge chunks.
template <class OffT>
__device__ void append_hub_C(const Part<OffT> &P, uint32_t v, uint32_t nv) {
  Ctl *c = P.ctl;
  const uint32_t pos = atomicAdd(&c->cnt_CH, 1u);
  P.CH_v[pos] = v;
  P.CH_val[pos] = nv;
  const uint64_t deg = (uint64_t)P.out_off[v + 1] - (uint64_t)P.out_off[v];
  const uint32_t nch = (uint32_t)((deg + kChunk - 1) / kChunk);
  const uint32_t kb = atomicAdd(&c->cnt_KC, nch);
  for (uint32_t i = 0; i < nch; i++) {
    P.chkC_h[kb + i] = pos;
    P.chkC_c[kb + i] = i;
  }
}

// FrontierActivate of up to kBatch targets per lane (`act` marks real ones).
// Each memory phase (stamp read, first-stamper atomic, BFS filter read, hub
// bit) is issued for the whole batch before any result is consumed, so a lane
// keeps kBatch independent requests in flight instead of one dependent chain.
// The first stamper of x appends it (BFS: only if still unvisited).
// kPreRead = false (vertex-record lanes: a target of a degree-<=4 source has few
// in-neighbours, so the filter rarely saves an atomic): the atomic is issued at
// once, one dependent L2 round trip less.
template <bool kBfsFilter, class OffT, bool kByOut = kBfsFilter, bool kPreRead = true>
__device__ __forceinline__ uint32_t activate_batch(const Part<OffT> &P, const bool (&act)[kBatch],
                                                   const uint32_t (&x)[kBatch], uint32_t epoch,
                                                   const uint32_t *hub_bits, WarpQueue &qA, uint32_t slot) {
  uint32_t st[kBatch];
  bool hb[kBatch];
#pragma unroll
  for (int q = 0; q < kBatch; q++) {
    st[q] = (act[q] && kPreRead) ? ld_cg(P.stamp + (x[q] - P.own_lo)) : (act[q] ? ~epoch : epoch);
    hb[q] = act[q] && test_bit(hub_bits, kByOut ? x[q] : x[q] - P.own_lo);  // issued with the stamp read
  }
  bool nw[kBatch];
#pragma unroll
  for (int q = 0; q < kBatch; q++) {
    const uint32_t old = (st[q] != epoch) ? atomicExch(P.stamp + (x[q] - P.own_lo), epoch) : epoch;
    nw[q] = old != epoch;
  }
  bool keep[kBatch];
#pragma unroll
  for (int q = 0; q < kBatch; q++) {
    if (kBfsFilter) keep[q] = nw[q] && (*(volatile uint32_t *)(P.val + x[q]) == kInf);
    else keep[q] = nw[q];
  }
  uint32_t cnt = 0;
#pragma unroll
  for (int q = 0; q < kBatch; q++) {
    const bool hub = keep[q] && hb[q];
    if (hub) append_hub_A<kByOut>(P, x[q], slot);
    qA.push(keep[q] && !hub, x[q], 0, P.listA[slot], nullptr, &P.ctl->cnt_A[slot]);
    cnt += __popc(__ballot_sync(0xffffffffu, nw[q]));
  }
  return cnt;
}

// Expand the out-edges of up to 32 source vertices (one per lane, degree <=
// kHubDegree): their edge ranges are concatenated and walked 32*kBatch edges at
// a time; each element finds its source lane by a shuffle binary search over
// the warp's exclusive degree prefix.
template <bool kBfsFilter, class OffT, bool kPreRead = true>
__device__ uint32_t expand_warp(const Part<OffT> &P, bool valid, uint64_t beg, uint32_t deg, uint32_t epoch,
                                const uint32_t *hub_bits, WarpQueue &qA, uint32_t slot) {
  const uint32_t lane = lane_id();
  const uint32_t d = valid ? deg : 0u;
  const uint32_t incl = warp_incl_scan(d);
  const uint32_t excl = incl - d;
  const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
  const uint64_t bx = beg - excl;  // CSR position of packed item k of this lane's row: bx + k
  uint32_t nact = 0;
  for (uint32_t r0 = 0; r0 < total; r0 += 32u * kBatch) {
    bool act[kBatch];
    uint32_t x[kBatch];
#pragma unroll
    for (int q = 0; q < kBatch; q++) {
      const uint32_t k = r0 + q * 32u + lane;
      int o = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const uint32_t e = __shfl_sync(0xffffffffu, excl, o + step);
        if (e <= k) o += step;
      }
      const uint64_t pos = packed_pos<OffT>(bx, o, k);  // a shuffle: every lane, outside the condition
      act[q] = k < total;
      x[q] = act[q] ? ldg_nc(P.out_dst + pos) : 0u;
    }
    nact += activate_batch<kBfsFilter, OffT, kBfsFilter, kPreRead>(P, act, x, epoch, hub_bits, qA, slot);
  }
  return nact;  // warp-uniform
}

// Block-wide expansion of one hub chunk (contiguous out-edges).
template <bool kBfsFilter, class OffT>
__device__ uint32_t expand_block(const Part<OffT> &P, uint64_t beg, uint32_t deg, uint32_t epoch,
                                 const uint32_t *hub_bits, WarpQueue &qA, uint32_t slot) {
  uint32_t nact = 0;
  for (uint32_t r0 = 0; r0 < deg; r0 += kBlock * kBatch) {
    bool act[kBatch];
    uint32_t x[kBatch];
#pragma unroll
    for (int q = 0; q < kBatch; q++) {
      const uint32_t k = r0 + q * kBlock + threadIdx.x;
      act[q] = k < deg;
      x[q] = act[q] ? ldg_nc(P.out_dst + beg + k) : 0u;
    }
    nact += activate_batch<kBfsFilter>(P, act, x, epoch, hub_bits, qA, slot);
  }
  return nact;  // per-warp count
}

// Close superstep t (the whole CTA calls it; thread 0 writes): sum the spread
// counters, write the trace row, reset the per-superstep counters, advance t,
// decide termination and set the CUDA-graph loop condition.
template <class OffT>
__device__ void close_superstep(const Part<OffT> &P, unsigned long long cond_handle, int use_graph, int pulled) {
  __shared__ unsigned long long s_red[4][kWarpsPerBlock];
  __threadfence();
  volatile Ctl *c = P.ctl;
  {
    unsigned long long v[4] = {0, 0, 0, 0};
    if (threadIdx.x < kSlots) {
      const uint32_t i = threadIdx.x;
      v[0] = c->part_g[i]; v[1] = c->part_c[i]; v[2] = c->part_s[i]; v[3] = c->part_a[i];
      c->part_g[i] = 0; c->part_c[i] = 0; c->part_s[i] = 0; c->part_a[i] = 0;
    }
#pragma unroll
    for (int k = 0; k < 4; k++) {
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) v[k] += __shfl_xor_sync(0xffffffffu, v[k], o);
      if (lane_id() == 0) s_red[k][threadIdx.x >> 5] = v[k];
    }
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  unsigned long long sg = 0, sc = 0, ss = 0, sa = 0;
  for (int w = 0; w < kWarpsPerBlock; w++) { sg += s_red[0][w]; sc += s_red[1][w]; ss += s_red[2][w]; sa += s_red[3][w]; }
  // every field read at once (independent loads: one L2 round trip, not one per
  // field — this runs on the critical path of every superstep), then every write
  const uint32_t t = c->iter, act0 = c->cnt_act[0], act1 = c->cnt_act[1], trace_cap = c->trace_cap;
  const uint32_t slot = t & 1u, ns = slot ^ 1u;
  const uint32_t act_ns = slot ? act0 : act1, act_s = slot ? act1 : act0;
  const unsigned long long prof = c->prof, gath0 = c->gathered, chg0 = c->changed, scat0 = c->scattered;
  const unsigned long long totA = c->tot_A, totC = c->tot_C, totG = c->tot_gathered, totS = c->tot_scattered;
  const uint32_t ext_loop = c->ext_loop, max_iters = c->max_iters, tot_pull = c->tot_pull;
  const unsigned long long gath = gath0 + sg, chg = chg0 + sc, scat = scat0 + ss;
  const uint32_t act_next = act_ns + (uint32_t)sa;
  c->cnt_act[ns] = act_next;
  if (t < trace_cap) {
    volatile unsigned long long *row = P.trace + 4ull * t;
    row[0] = act_s;
    row[1] = chg;
    row[2] = gath;
    row[3] = scat;
  }
  if (prof) {
    unsigned long long ks[2], ke[2], kn[2];
    for (int k = 0; k < 2; k++) { ks[k] = c->kstart[k]; ke[k] = c->kend[k]; kn[k] = c->kns[k]; }
    for (int k = 0; k < 2; k++) {
      if (ke[k] > ks[k]) c->kns[k] = kn[k] + (ke[k] - ks[k]);
      c->kstart[k] = ~0ull;
      c->kend[k] = 0;
    }
  }
  c->tot_A = totA + act_s;
  c->tot_C = totC + chg;
  c->tot_gathered = totG + gath;
  c->tot_scattered = totS + scat;
  c->changed = 0;
  c->gathered = 0;
  c->scattered = 0;
  c->cnt_C = 0;
  c->cnt_CH = 0;
  c->cnt_KC = 0;
  c->cnt_K[slot] = 0;
  c->ctr_hub = 0;
  c->ctr_hub2 = 0;
  c->cnt_A[slot] = 0;
  c->cnt_H[slot] = 0;
  c->cnt_act[slot] = 0;
  // changed bitmaps: this superstep's activation cleared bitmap (t+1)&1; a
  // pull left bits in bitmap t&1
  c->dirty[ns] = 0;
  if (pulled) {
    c->dirty[slot] = 1;
    c->tot_pull = tot_pull + 1;
  }
  c->pull_pending = 0;
  // kPullDense: A_{t+1} is found by the dense gather of t+1; it is empty iff
  // C_t has no out-edges
  c->dense = (pulled == kPullDense) ? 1u : 0u;
  // source gating of the dense gather of t+1 (Selective<> programs): it trades a
  // second dependent load for skipping the values of unchanged sources, which
  // pays when fewer than half of the vertices changed (measured: R-MAT CC
  // 2.72 -> 2.42 ms; the web graph's all-changed supersteps 12.2 -> 12.8 ms ungated)
  c->gate = (pulled == kPullDense && 2ull * chg < (unsigned long long)P.own_n) ? 1u : 0u;
  c->iter = t + 1;
  const bool empty = (pulled == kPullDense) ? (scat == 0) : (act_next == 0);
  const bool stop = !ext_loop && (empty || (max_iters != 0 && t + 1 >= max_iters));
  c->stop = stop ? 1u : 0u;
  __threadfence();
#ifndef GR_JIT  // run-time compiled programs (jit.cpp) run only the persistent loop: no conditional graph node
  if (use_graph) cudaGraphSetConditional((cudaGraphConditionalHandle)cond_handle, stop ? 0u : 1u);
#else
  (void)cond_handle;
  (void)use_graph;
#endif
}


// Last CTA of the superstep's final kernel closes superstep t. The ticket is
// two-level (groups of 32 CTAs) so no single address takes one atomic per CTA.
template <class OffT>
__device__ void finish_superstep(const Part<OffT> &P, unsigned long long cond_handle, int use_graph, int pulled) {
  __shared__ bool s_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    Ctl *cc = P.ctl;
    const uint32_t grp = blockIdx.x >> 5, ngrp = (gridDim.x + 31) >> 5;
    const uint32_t gsize = min(32u, gridDim.x - grp * 32u);
    bool last = false;
    if (atomicAdd(&cc->tick1[grp], 1u) == gsize - 1) {
      cc->tick1[grp] = 0;
      __threadfence();
      if (atomicAdd(&cc->tick2, 1u) == ngrp - 1) {
        cc->tick2 = 0;
        last = true;
      }
    }
    s_last = last;
  }
  __syncthreads();
  if (!s_last) return;
  close_superstep(P, cond_handle, use_graph, pulled);
}

// ------------------------------------------------- pull activation (dense)
// When the changed set is a large fraction of V, FrontierActivate by pull:
// commit C_t and mark it in a bitmap, then every owned vertex x scans its
// in-edges for a changed source (early exit) — x is in A_{t+1} iff one exists,
// the same set the push expansion produces (the out-neighbours of C_t), with
// no per-edge atomics. Trace columns are unchanged.
// words of one changed bitmap (a multiple of 4 for 16-byte clears; the host allocates the same)
__host__ __device__ __forceinline__ size_t cbits_words_n(uint64_t n) { return (((n + 31) / 32 + 1) + 3) & ~size_t(3); }
template <class OffT> __device__ __forceinline__ size_t cbits_words(const Part<OffT> &P) { return cbits_words_n(P.n); }

__device__ __forceinline__ bool pull_mode(const View &V, uint32_t own_n, uint32_t frontier) {
  return V.pull_div != 0 && (unsigned long long)frontier * V.pull_div > own_n;
}
__device__ __forceinline__ uint32_t frontier_gather(const View &V) { return V.cntC + V.cntCH; }
__device__ __forceinline__ uint32_t frontier_bfs(const View &V) { return V.cntA[V.t & 1u] + V.cntH[V.t & 1u]; }

// Zero the bitmap the next superstep may pull into (all CTAs; nobody reads it now).
template <class OffT>
__device__ __forceinline__ void clear_dirty(const Part<OffT> &P, const View &V, size_t words) {
  const uint32_t nb = (V.t + 1) & 1u;
  if (!V.dirty[nb]) return;
  uint4 *w = reinterpret_cast<uint4 *>(P.cbits[nb]);
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < words / 4; i += (size_t)gridDim.x * blockDim.x)
    w[i] = make_uint4(0, 0, 0, 0);
}

__device__ __forceinline__ void set_bit(uint32_t *bits, uint32_t u) { atomicOr(bits + (u >> 5), 1u << (u & 31)); }

// Pull mode, gather programs: commit C_t (non-hub and hub entries) and mark it.
template <class OffT>
__device__ __forceinline__ void commit_phase(const Part<OffT> &P, const View &V) {
  uint32_t *bits = P.cbits[V.t & 1u];
  __shared__ unsigned long long s8[kWarpsPerBlock];
  unsigned long long my_s = 0;
  const uint32_t nC = V.cntC, nCH = V.cntCH;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < nC + nCH; i += gridDim.x * blockDim.x) {
    const bool h = i >= nC;
    const uint32_t u = h ? P.CH_v[i - nC] : P.C_v[i];
    P.val[u] = h ? P.CH_val[i - nC] : P.C_val[i];  // BSP commit of superstep t
    set_bit(bits, u);
    my_s += (uint64_t)P.out_off[u + 1] - (uint64_t)P.out_off[u];
  }
  my_s = block_sum_u64(my_s, s8);
  if (threadIdx.x == 0 && my_s) atomicAdd(&P.ctl->part_s[blockIdx.x % kSlots], my_s);
}

// Pull mode, BFS: apply A_t (depth = t, L276; hubs included) and mark C_t.
template <class OffT>
__device__ __forceinline__ void bfs_apply_phase(const Part<OffT> &P, const View &V) {
  const uint32_t t = V.t, slot = t & 1u;
  uint32_t *bits = P.cbits[slot];
  __shared__ unsigned long long s8[kWarpsPerBlock];
  unsigned long long my_s = 0, my_c = 0;
  const uint32_t nA = V.cntA[slot], nH = V.cntH[slot];
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < nA + nH; i += gridDim.x * blockDim.x) {
    const uint32_t v = i < nA ? P.listA[slot][i] : P.listH[slot][i - nA];
    if (P.val[v] == kInf) {
      P.val[v] = t;
      set_bit(bits, v);
      my_c += 1;
      my_s += (uint64_t)P.out_off[v + 1] - (uint64_t)P.out_off[v];
    }
  }
  my_s = block_sum_u64(my_s, s8);
  if (threadIdx.x == 0 && my_s) atomicAdd(&P.ctl->part_s[blockIdx.x % kSlots], my_s);
  my_c = block_sum_u64(my_c, s8);
  if (threadIdx.x == 0 && my_c) atomicAdd(&P.ctl->part_c[blockIdx.x % kSlots], my_c);
}

// Pull mode (BFS): A_{t+1} = owned x with an in-neighbour in C_t. Each lane
// scans its own vertex (kProbe loads in flight, stopping at the first hit);
// vertices of in-degree > kPullLane are scanned by the whole warp, 32 edges
// per step.
// BFS keeps only unvisited vertices in the list (counts every activated one).
constexpr uint32_t kProbe = 4;
constexpr uint32_t kPullLane = 128;  // in-degree up to which a lane scans its vertex alone
constexpr uint32_t kPullDivDefault = 16;  // GR_DIR_AUTO: pull when |C_t| > |V| / 16
template <bool kBfs, class OffT>
__device__ __forceinline__ void pull_phase(const Part<OffT> &P, const View &V) {
  Ctl *ctl = P.ctl;
  const uint32_t t = V.t, ns = (t + 1) & 1u;
  const uint32_t *bits = P.cbits[t & 1u];
  prof_begin(ctl, V, 1);
  GR_SQ1(sq);
  __shared__ uint32_t s_off[kWarpsPerBlock + 1];
  __shared__ unsigned long long s8[kWarpsPerBlock];
  const uint32_t warp = threadIdx.x / 32, lane = lane_id();
  WarpQueue qA{sq[warp], nullptr, 0};
  unsigned long long my_act = 0;
  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = gw * 32u; base < P.own_n; base += nw * 32u) {
    const uint32_t lx = base + lane;
    const bool valid = lx < P.own_n;
    const uint32_t x = P.own_lo + lx;
    uint64_t beg = 0, end = 0;
    if (valid) {
      beg = (uint64_t)P.in_off[lx];
      end = (uint64_t)P.in_off[lx + 1];
    }
    const uint64_t deg = end - beg;
    uint32_t src[kProbe];
#pragma unroll
    for (uint32_t q = 0; q < kProbe; q++) src[q] = (q < deg) ? ldg_nc(P.in_src + beg + q) : 0u;
    bool found = false;
#pragma unroll
    for (uint32_t q = 0; q < kProbe; q++) found |= (q < deg) && test_bit_w(bits, src[q]);
    // moderate degrees: each lane continues its own scan, kProbe loads in flight
    for (uint64_t k = beg + kProbe; !found && deg <= kPullLane && k < end; k += kProbe) {
      uint32_t u[kProbe];
#pragma unroll
      for (uint32_t q = 0; q < kProbe; q++) u[q] = (k + q < end) ? ldg_nc(P.in_src + k + q) : 0u;
#pragma unroll
      for (uint32_t q = 0; q < kProbe; q++) found |= (k + q < end) && test_bit_w(bits, u[q]);
    }
    // large degrees: the whole warp scans one vertex at a time
    uint32_t pend = __ballot_sync(0xffffffffu, !found && deg > kPullLane);
    uint32_t fm = 0;
    while (pend) {
      const int l = __ffs(pend) - 1;
      pend &= pend - 1;
      const uint64_t b = __shfl_sync(0xffffffffu, beg, l) + kProbe, e = __shfl_sync(0xffffffffu, end, l);
      for (uint64_t k = b; k < e; k += 32) {
        const uint64_t kk = k + lane;
        const bool hit = kk < e && test_bit_w(bits, ldg_nc(P.in_src + kk));
        if (__ballot_sync(0xffffffffu, hit)) {
          fm |= 1u << l;
          break;
        }
      }
    }
    found = found || ((fm >> lane) & 1u);
    my_act += __popc(__ballot_sync(0xffffffffu, found));
    const bool keep = found && (!kBfs || *(volatile uint32_t *)(P.val + x) == kInf);
    const bool hub = keep && test_bit(kBfs ? P.hub_out : P.hub_in, kBfs ? x : lx);
    if (hub) append_hub_A<kBfs>(P, x, ns);
    qA.push(keep && !hub, x, 0, P.listA[ns], nullptr, &ctl->cnt_A[ns]);
  }
  qA.block_flush(P.listA[ns], nullptr, &ctl->cnt_A[ns], s_off);
  my_act = block_sum_u64(lane == 0 ? my_act : 0ull, s8);
  if (threadIdx.x == 0 && my_act) atomicAdd(&ctl->part_a[blockIdx.x % kSlots], my_act);
  prof_end(ctl, V, 1);
}

// Split-kernel loops: the pull half of a pull superstep (no-op otherwise).
template <bool kBfs, class OffT>
__global__ void __launch_bounds__(kBlock) k_pull(const __grid_constant__ Part<OffT> P, unsigned long long cond,
                                                 int use_graph) {
  __shared__ View V;
  load_view(P.ctl, V);
  if (V.stop || !V.pull_pending) return;
  pull_phase<kBfs>(P, V);
  finish_superstep(P, cond, use_graph, kPullScan);
}

// ------------------------------------------------------------- kernels
// Gather + apply over A_t (one phase of superstep t). kDense (the previous
// superstep activated by pull): A_t is not materialised — every owned vertex
// is gathered and is active iff one of its in-edge sources is marked in the
// changed bitmap of t-1; only active vertices apply and count in the trace.
template <class Prog, bool kDense, class OffT, bool kMirror = false, bool kGate = false>
__device__ __forceinline__ void gather_phase(const Part<OffT> &P, const View &V) {
  using G = typename Prog::GatherT;
  Ctl *ctl = P.ctl;
  const uint32_t t = V.t;
  const uint32_t slot = t & 1u;
  const Ctx cx = make_ctx(P, V);
  const bool implicit = kDense || (V.implicit0 && t == 0);
  const uint32_t nA = implicit ? P.own_n : V.cntA[slot];
  const uint32_t nK = kDense ? P.n_s_chunks : V.cntK[slot];
  const uint32_t *LA = P.listA[slot];
  const uint32_t *LH = kDense ? P.s_hubs : P.listH[slot];
  const uint32_t *KH = kDense ? P.s_chk_h : P.chkA_h[slot];
  const uint32_t *KC = kDense ? P.s_chk_c : P.chkA_c[slot];
  const uint32_t *bits = P.cbits[slot ^ 1u];  // C_{t-1} (dense only)
  const bool no_hub_c = V.no_hub_c != 0;
  prof_begin(ctl, V, 0);

#ifdef GR_NO_SMEM_UNION
  GR_SQ2(sq);
  __shared__ G sred[kWarpsPerBlock][32];
  __shared__ G sblk[kWarpsPerBlock];
#else
  static_assert(sizeof(G) <= 8, "gather results up to 8 bytes");
  GR_SQ2(sq);
  auto &sred = *reinterpret_cast<G(*)[kWarpsPerBlock][32]>(g_phase_smem + kSqBytes2);
  auto &sblk = *reinterpret_cast<G(*)[kWarpsPerBlock]>(g_phase_smem + kSqBytes2 + kWarpsPerBlock * 32 * 8);
#endif
  __shared__ uint32_t s_h;
  __shared__ bool s_act;
  __shared__ uint32_t s_off[kWarpsPerBlock + 1];
  __shared__ unsigned long long s8[kWarpsPerBlock];
  const uint32_t warp = threadIdx.x / 32, lane = lane_id();
  WarpQueue qC{sq[warp][0], sq[warp][1], 0};
  if constexpr (kMirror) {  // partitioned, fused exchange: C_t also lands in every rank's exchange buffer
    qC.mir_a = P.xp_v;
    qC.mir_b = P.xp_val;
    qC.n_mir = P.n_xp;
    qC.mir_off = P.xp_off;
  }
  unsigned long long my_g = 0, my_c = 0, my_a = 0;

  // Phase 1: non-hub active vertices, 32 per warp, static grid stride
  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = gw * 32u; base < nA; base += nw * 32u) {
    const uint32_t idx = base + lane;
    bool valid = idx < nA;
    uint32_t v = 0;
    if (valid) v = implicit ? P.own_lo + idx : LA[idx];
    const uint32_t lv = v - P.own_lo;
    if (valid && implicit && test_bit(P.hub_in, lv)) valid = false;  // served by the hub chunks
    uint64_t beg = 0;
    uint32_t deg = 0, cur = 0, w4 = 0;
    uint4 rs{};
    bool hubv = false;
    if (valid) {
      if (Prog::kHasGather) {
        if (P.rec_in) {  // vertex record: sources, weights, degree and offset in one sector
          rs = ldg_nc_v4(P.rec_in + 2ull * lv);
          const uint4 r1 = ldg_nc_v4(P.rec_in + 2ull * lv + 1);
          w4 = r1.x;
          deg = r1.y;
          beg = (uint64_t)r1.z | ((uint64_t)r1.w << 32);
        } else {
          beg = (uint64_t)P.in_off[lv];
          deg = (uint32_t)((uint64_t)P.in_off[lv + 1] - beg);
        }
      }
      cur = P.val[v];
      hubv = !no_hub_c && test_bit(P.hub_out, v);  // issued with the offsets, used after apply
    }
    bool hit = false;
    const bool direct = P.rec_in != nullptr && valid && deg <= kRecDeg;
    const G acc = Prog::kHasGather ? gather_warp<Prog, kDense, kGate>(P, valid, beg, deg, cur, sred[warp], cx, bits, hit,
                                                                       direct, rs, w4)
                                   : Prog::identity();
    const bool active = valid && (!kDense || hit);
    bool changed = false;
    uint32_t nv = cur;
    if (active) {
      changed = Prog::apply(&nv, acc, cx);
      my_g += deg;
      my_a += 1;
    }
    const bool hubo = changed && hubv;
    if (hubo) append_hub_C(P, v, nv);
    qC.push(changed && !hubo, v, nv, P.C_v, P.C_val, &ctl->cnt_C);
    my_c += changed ? 1 : 0;
  }
  qC.block_flush(P.C_v, P.C_val, &ctl->cnt_C, s_off);

  // Phase 2: hub chunks (kChunk in-edges each), dynamic over CTAs. Chunk results
  // combine with Prog::atomicGather (exact for min); the last chunk applies.
  for (; nK;) {
    __syncthreads();
    if (threadIdx.x == 0) s_h = atomicAdd(&ctl->ctr_hub, 1u);
    __syncthreads();
    const uint32_t i = s_h;
    if (i >= nK) break;
    const uint32_t hp = KH[i], ci = KC[i];
    const uint32_t v = LH[hp], lv = v - P.own_lo;
    const uint64_t beg = (uint64_t)P.in_off[lv];
    const uint64_t deg = (uint64_t)P.in_off[lv + 1] - beg;
    const uint64_t b = beg + (uint64_t)ci * kChunk;
    const uint32_t len = chunk_len(deg, ci);
    const uint32_t cur = P.val[v];
    if (!Prog::kHasGather && ci != 0) continue;  // no gather: chunk 0 applies
    const G r = Prog::kHasGather ? gather_block<Prog, kDense, kGate>(P, b, len, cur, sblk, cx, bits, &s_act)
                                 : Prog::identity();
    if (threadIdx.x == 0) {
      const uint32_t nch = Prog::kHasGather ? (uint32_t)((deg + kChunk - 1) / kChunk) : 1u;
      bool fin = (nch == 1);
      bool hact = kDense ? s_act : true;
      G acc = r;
      if (!fin) {
        Prog::atomicGather(reinterpret_cast<G *>(P.hub_acc) + hp, r);
        if (kDense && s_act) atomicOr(P.hub_act + hp, 1u);
        __threadfence();
        fin = (atomicAdd(P.hub_done + hp, 1u) == nch - 1);
        if (fin) {
          __threadfence();
          acc = atomicExch(reinterpret_cast<G *>(P.hub_acc) + hp, Prog::identity());
          if (kDense) hact = atomicExch(P.hub_act + hp, 0u) != 0;
          P.hub_done[hp] = 0;
        }
      }
      if (fin && hact) {
        if (Prog::kHasGather) my_g += deg;
        my_a += 1;
        uint32_t nv = cur;
        if (Prog::apply(&nv, acc, cx)) {
          my_c += 1;
          if (!no_hub_c && test_bit(P.hub_out, v)) append_hub_C(P, v, nv);
          else {
            const uint32_t pos = atomicAdd(&ctl->cnt_C, 1u);
            P.C_v[pos] = v;
            P.C_val[pos] = nv;
            if constexpr (kMirror) qC.mirror(pos, v, nv);
          }
        }
      }
    }
  }
  my_g = block_sum_u64(my_g, s8);
  if (threadIdx.x == 0 && my_g) atomicAdd(&ctl->part_g[blockIdx.x % kSlots], my_g);
  my_c = block_sum_u64(my_c, s8);
  if (threadIdx.x == 0 && my_c) atomicAdd(&ctl->part_c[blockIdx.x % kSlots], my_c);
  if (kDense) {  // |A_t| is only known now (one atomic per CTA)
    my_a = block_sum_u64(my_a, s8);
    if (threadIdx.x == 0 && my_a) atomicAdd(&ctl->cnt_act[slot], (uint32_t)my_a);
  }
  prof_end(ctl, V, 0);
}

// dense gather of superstep t: source-gated when the program allows it and the
// changed set of t-1 was small enough (Ctl::gate)
template <class Prog, class OffT>
__device__ __forceinline__ void dense_gather_phase(const Part<OffT> &P, const View &V) {
  if constexpr (kGateSelective && Selective<Prog>::value) {
    if (V.gate) {
      gather_phase<Prog, true, OffT, false, true>(P, V);
      return;
    }
  }
  gather_phase<Prog, true>(P, V);
}

template <class Prog, class OffT>
__global__ void __launch_bounds__(kBlock) k_gather_apply(const __grid_constant__ Part<OffT> P) {
  __shared__ View V;
  load_view(P.ctl, V);
  if (V.stop) return;
  if (V.dense) dense_gather_phase<Prog>(P, V);
  else gather_phase<Prog, false>(P, V);
}

// partitioned runs with the exchange fused into the gather (sparse supersteps only)
template <class Prog, class OffT>
__global__ void __launch_bounds__(kBlock) k_gather_apply_x(const __grid_constant__ Part<OffT> P) {
  __shared__ View V;
  load_view(P.ctl, V);
  if (V.stop) return;
  gather_phase<Prog, false, OffT, true>(P, V);
}

// Commit C_t and FrontierActivate (the other phase of superstep t).
template <class OffT>
__device__ __forceinline__ void activate_phase(const Part<OffT> &P, const View &V) {
  Ctl *ctl = P.ctl;
  const uint32_t t = V.t;
  const uint32_t ns = (t + 1) & 1u;
  const uint32_t epoch = V.epoch_base + t + 1;
  const uint32_t nC = V.cntC;
  const uint32_t nKC = V.cntKC;
  prof_begin(ctl, V, 1);

  GR_SQ1(sq);
  __shared__ uint32_t s_h;
  __shared__ uint32_t s_off[kWarpsPerBlock + 1];
  __shared__ unsigned long long s8[kWarpsPerBlock];
  const uint32_t warp = threadIdx.x / 32, lane = lane_id();
  WarpQueue qA{sq[warp], nullptr, 0};
  unsigned long long my_s = 0, my_act = 0;

  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = gw * 32u; base < nC; base += nw * 32u) {
    const uint32_t idx = base + lane;
    const bool valid = idx < nC;
    uint64_t beg = 0;
    uint32_t deg = 0;
    uint4 rd{};
    if (valid) {
      const uint32_t u = P.C_v[idx];
      P.val[u] = P.C_val[idx];  // BSP commit of superstep t
      if (P.rec_out) {  // vertex record: targets, degree and offset in one sector
        rd = ldg_nc_v4(P.rec_out + 2ull * u);
        const uint4 r1 = ldg_nc_v4(P.rec_out + 2ull * u + 1);
        deg = r1.y;
        beg = (uint64_t)r1.z | ((uint64_t)r1.w << 32);
      } else {
        beg = (uint64_t)P.out_off[u];
        deg = (uint32_t)((uint64_t)P.out_off[u + 1] - beg);
      }
      my_s += deg;
    }
    const bool direct = P.rec_out != nullptr && valid && deg <= kRecDeg;
    if (__any_sync(0xffffffffu, direct)) {  // record lanes: their targets are one activation batch
      const uint32_t x[kBatch] = {rd.x, rd.y, rd.z, rd.w};
      bool a[kBatch];
#pragma unroll
      for (uint32_t q = 0; q < kRecDeg; q++) a[q] = direct && q < deg;
      my_act += activate_batch<false, OffT, false, false>(P, a, x, epoch, P.hub_in, qA, ns);
    }
    // low-degree graphs (Part::stamp_direct): few in-neighbours per target, so the
    // first-stamper filter read rarely saves an atomic — issue the atomic at once
    if (P.stamp_direct) my_act += expand_warp<false, OffT, false>(P, valid && !direct, beg, deg, epoch, P.hub_in, qA, ns);
    else my_act += expand_warp<false>(P, valid && !direct, beg, deg, epoch, P.hub_in, qA, ns);
  }
  // changed hubs: out-edge chunks, dynamic over CTAs
  for (; nKC;) {
    __syncthreads();
    if (threadIdx.x == 0) s_h = atomicAdd(&ctl->ctr_hub2, 1u);
    __syncthreads();
    const uint32_t i = s_h;
    if (i >= nKC) break;
    const uint32_t hp = P.chkC_h[i], ci = P.chkC_c[i];
    const uint32_t u = P.CH_v[hp];
    const uint64_t beg = (uint64_t)P.out_off[u];
    const uint64_t deg = (uint64_t)P.out_off[u + 1] - beg;
    if (threadIdx.x == 0 && ci == 0) {
      P.val[u] = P.CH_val[hp];
      my_s += deg;
    }
    const uint32_t len = chunk_len(deg, ci);
    const uint32_t a = expand_block<false>(P, beg + (uint64_t)ci * kChunk, len, epoch, P.hub_in, qA, ns);
    if (lane == 0) my_act += a;
  }
  qA.block_flush(P.listA[ns], nullptr, &ctl->cnt_A[ns], s_off);
  my_s = block_sum_u64(my_s, s8);
  if (threadIdx.x == 0 && my_s) atomicAdd(&ctl->part_s[blockIdx.x % kSlots], my_s);
  my_act = block_sum_u64(lane == 0 ? my_act : 0ull, s8);
  if (threadIdx.x == 0 && my_act) atomicAdd(&ctl->part_a[blockIdx.x % kSlots], my_act);
  prof_end(ctl, V, 1);
}

template <class OffT>
__global__ void __launch_bounds__(kBlock) k_activate(const __grid_constant__ Part<OffT> P, unsigned long long cond,
                                                     int use_graph) {
  __shared__ View V;
  load_view(P.ctl, V);
  if (V.stop) {
    if (use_graph && blockIdx.x == 0 && threadIdx.x == 0)
      cudaGraphSetConditional((cudaGraphConditionalHandle)cond, 0u);
    return;
  }
  clear_dirty(P, V, cbits_words(P));
  if (pull_mode(V, P.own_n, frontier_gather(V))) {
    commit_phase(P, V);  // superstep t+1 gathers densely
    finish_superstep(P, cond, use_graph, kPullDense);
    return;
  }
  activate_phase(P, V);
  finish_superstep(P, cond, use_graph, kPush);
}

// BFS: apply (depth = t, L276) fused with FrontierActivate; no gather (L274).
template <class OffT>
__device__ __forceinline__ void bfs_phase(const Part<OffT> &P, const View &V) {
  Ctl *ctl = P.ctl;
  const uint32_t t = V.t;
  const uint32_t slot = t & 1u, ns = slot ^ 1u;
  const uint32_t epoch = V.epoch_base + t + 1;
  const uint32_t nA = V.cntA[slot];
  const uint32_t nK = V.cntK[slot];
  const uint32_t *LA = P.listA[slot];
  const uint32_t *LH = P.listH[slot];
  prof_begin(ctl, V, 1);

  GR_SQ1(sq);
  __shared__ uint32_t s_h;
  __shared__ bool s_changed;
  __shared__ uint32_t s_off[kWarpsPerBlock + 1];
  __shared__ unsigned long long s8[kWarpsPerBlock];
  const uint32_t warp = threadIdx.x / 32, lane = lane_id();
  WarpQueue qA{sq[warp], nullptr, 0};
  unsigned long long my_s = 0, my_c = 0, my_act = 0;

  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = gw * 32u; base < nA; base += nw * 32u) {
    const uint32_t idx = base + lane;
    bool changed = false;
    uint64_t beg = 0;
    uint32_t deg = 0;
    if (idx < nA) {
      const uint32_t v = LA[idx];
      if (P.val[v] == kInf) {  // apply: depth = iteration number
        P.val[v] = t;
        changed = true;
        beg = (uint64_t)P.out_off[v];
        deg = (uint32_t)((uint64_t)P.out_off[v + 1] - beg);
        my_s += deg;
        my_c += 1;
      }
    }
    my_act += expand_warp<true>(P, changed, beg, deg, epoch, P.hub_out, qA, ns);
  }
  // hub members of A_t (by out-degree): chunk 0 applies; every chunk expands if
  // the hub's depth is unset or was set in this superstep
  for (; nK;) {
    __syncthreads();
    if (threadIdx.x == 0) s_h = atomicAdd(&ctl->ctr_hub, 1u);
    __syncthreads();
    const uint32_t i = s_h;
    if (i >= nK) break;
    const uint32_t hp = P.chkA_h[slot][i], ci = P.chkA_c[slot][i];
    const uint32_t v = LH[hp];
    const uint64_t beg = (uint64_t)P.out_off[v];
    const uint64_t deg = (uint64_t)P.out_off[v + 1] - beg;
    if (threadIdx.x == 0) {
      if (ci == 0 && P.val[v] == kInf) {
        P.val[v] = t;
        my_c += 1;
        my_s += deg;
      }
      const uint32_t d = *(volatile uint32_t *)(P.val + v);
      s_changed = (d == kInf || d == t);
    }
    __syncthreads();
    if (!s_changed) continue;
    const uint32_t len = chunk_len(deg, ci);
    const uint32_t a = expand_block<true>(P, beg + (uint64_t)ci * kChunk, len, epoch, P.hub_out, qA, ns);
    if (lane == 0) my_act += a;
  }
  qA.block_flush(P.listA[ns], nullptr, &ctl->cnt_A[ns], s_off);
  my_s = block_sum_u64(my_s, s8);
  if (threadIdx.x == 0 && my_s) atomicAdd(&ctl->part_s[blockIdx.x % kSlots], my_s);
  my_c = block_sum_u64(my_c, s8);
  if (threadIdx.x == 0 && my_c) atomicAdd(&ctl->part_c[blockIdx.x % kSlots], my_c);
  my_act = block_sum_u64(lane == 0 ? my_act : 0ull, s8);
  if (threadIdx.x == 0 && my_act) atomicAdd(&ctl->part_a[blockIdx.x % kSlots], my_act);
  prof_end(ctl, V, 1);
}

template <class OffT>
__global__ void __launch_bounds__(kBlock) k_bfs_expand(const __grid_constant__ Part<OffT> P, unsigned long long cond,
                                                       int use_graph) {
  __shared__ View V;
  load_view(P.ctl, V);
  if (V.stop) {
    if (use_graph && blockIdx.x == 0 && threadIdx.x == 0)
      cudaGraphSetConditional((cudaGraphConditionalHandle)cond, 0u);
    return;
  }
  clear_dirty(P, V, cbits_words(P));
  if (pull_mode(V, P.own_n, frontier_bfs(V))) {
    bfs_apply_phase(P, V);
    if (blockIdx.x == 0 && threadIdx.x == 0) P.ctl->pull_pending = 1;
    return;
  }
  bfs_phase(P, V);
  finish_superstep(P, cond, use_graph, kPush);
}

// ------------------------------------------------------ fused push supersteps
// Programs with kPushFused (gr/program.cuh; SSSP, widest path), resident single
// GPU: apply and FrontierActivate run as ONE phase per superstep and the gather
// rides on the activation. For v in A_t: r = acc_t[v] (the atomicGather of the
// pushes of C_{t-1}), apply(&val[v], r); if v changed, every out-edge (v -> x)
// does atomicGather(&acc_{t+1}[x], gatherMap(new[v], w)) and stamps x into
// A_{t+1}. acc is double-buffered by superstep parity and reset when consumed.
// Values, changed sets and the trace equal the BSP gather over all in-edges
// (see program.cuh); Sigma_{A_t} indeg is counted from the offsets. BFS's phase
// fusion (L276) extended to selective monotone gathers: one grid barrier per
// superstep instead of three, and no in-edge walk.
template <class Prog, class OffT>
__device__ __forceinline__ uint32_t push_batch(const Part<OffT> &P, const bool (&act)[kBatch],
                                               const uint32_t (&x)[kBatch], const uint32_t (&gm)[kBatch],
                                               uint32_t *accn, uint32_t epoch, WarpQueue &qA, uint32_t slot) {
#pragma unroll
  for (int q = 0; q < kBatch; q++)  // fire-and-forget (RED): read only after the barrier
    if (act[q] && gm[q] != Prog::identity()) Prog::atomicGather(accn + x[q], gm[q]);
  return activate_batch<false, OffT, true>(P, act, x, epoch, P.hub_out, qA, slot);
}

// Push the out-edges of up to 32 changed vertices (one per lane: vertex u, new
// value nv, edges [beg, beg + deg), deg <= kHubDegree), walked 32*kBatch at a time.
template <class Prog, class OffT>
__device__ uint32_t expand_warp_push(const Part<OffT> &P, bool valid, uint64_t beg, uint32_t deg, uint32_t u,
                                     uint32_t nv, const Ctx &cx, uint32_t *accn, uint32_t epoch, WarpQueue &qA,
                                     uint32_t slot) {
  const uint32_t lane = lane_id();
  const uint32_t d = valid ? deg : 0u;
  const uint32_t incl = warp_incl_scan(d);
  const uint32_t excl = incl - d;
  const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
  uint32_t nact = 0;
  for (uint32_t r0 = 0; r0 < total; r0 += 32u * kBatch) {
    bool act[kBatch];
    uint32_t x[kBatch], gm[kBatch];
#pragma unroll
    for (int q = 0; q < kBatch; q++) {
      const uint32_t k = r0 + q * 32u + lane;
      int o = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const uint32_t e = __shfl_sync(0xffffffffu, excl, o + step);
        if (e <= k) o += step;
      }
      const uint64_t ob = __shfl_sync(0xffffffffu, beg, o);
      const uint32_t oe = __shfl_sync(0xffffffffu, excl, o);
      const uint32_t ov = __shfl_sync(0xffffffffu, nv, o);
      const uint32_t ou = __shfl_sync(0xffffffffu, u, o);
      act[q] = k < total;
      const uint64_t e = ob + (k - oe);
      x[q] = act[q] ? ldg_nc(P.out_dst + e) : 0u;
      const uint32_t w = (act[q] && Prog::kUsesWeights) ? (uint32_t)ldg_nc_u8(P.out_w + e) : 0u;
      gm[q] = act[q] ? Prog::gatherMap(0u, ov, w, ou, cx) : Prog::identity();
    }
    nact += push_batch<Prog>(P, act, x, gm, accn, epoch, qA, slot);
  }
  return nact;  // warp-uniform
}

// Block-wide push of one hub chunk (contiguous out-edges of vertex u, new value nv).
template <class Prog, class OffT>
__device__ uint32_t expand_block_push(const Part<OffT> &P, uint64_t beg, uint32_t deg, uint32_t u, uint32_t nv,
                                      const Ctx &cx, uint32_t *accn, uint32_t epoch, WarpQueue &qA, uint32_t slot) {
  uint32_t nact = 0;
  for (uint32_t r0 = 0; r0 < deg; r0 += kBlock * kBatch) {
    bool act[kBatch];
    uint32_t x[kBatch], gm[kBatch];
#pragma unroll
    for (int q = 0; q < kBatch; q++) {
      const uint32_t k = r0 + q * kBlock + threadIdx.x;
      act[q] = k < deg;
      x[q] = act[q] ? ldg_nc(P.out_dst + beg + k) : 0u;
      const uint32_t w = (act[q] && Prog::kUsesWeights) ? (uint32_t)ldg_nc_u8(P.out_w + beg + k) : 0u;
      gm[q] = act[q] ? Prog::gatherMap(0u, nv, w, u, cx) : Prog::identity();
    }
    nact += push_batch<Prog>(P, act, x, gm, accn, epoch, qA, slot);
  }
  return nact;  // per-warp count
}

template <class Prog, class OffT>
__device__ __forceinline__ void push_phase(const Part<OffT> &P, const View &V) {
  Ctl *ctl = P.ctl;
  const uint32_t t = V.t;
  const uint32_t slot = t & 1u, ns = slot ^ 1u;
  const uint32_t epoch = V.epoch_base + t + 1;
  const uint32_t nA = V.cntA[slot];
  const uint32_t nK = V.cntK[slot];
  const uint32_t *LA = P.listA[slot];
  const uint32_t *LH = P.listH[slot];
  uint32_t *acc = P.nxt[slot], *accn = P.nxt[ns];
  const Ctx cx = make_ctx(P, V);
  prof_begin(ctl, V, 1);

  GR_SQ1(sq);
  __shared__ uint32_t s_h, s_nv;
  __shared__ bool s_changed;
  __shared__ uint32_t s_off[kWarpsPerBlock + 1];
  __shared__ unsigned long long s8[kWarpsPerBlock];
  const uint32_t warp = threadIdx.x / 32, lane = lane_id();
  WarpQueue qA{sq[warp], nullptr, 0};
  unsigned long long my_g = 0, my_s = 0, my_c = 0, my_act = 0;

  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = gw * 32u; base < nA; base += nw * 32u) {
    const uint32_t idx = base + lane;
    bool changed = false;
    uint64_t beg = 0;
    uint32_t deg = 0, v = 0, nv = 0;
    if (idx < nA) {
      v = LA[idx];
      const uint32_t r = acc[v];
      uint32_t cur = P.val[v];
      const uint64_t i0 = (uint64_t)P.in_off[v - P.own_lo], i1 = (uint64_t)P.in_off[v - P.own_lo + 1];  // trace
      acc[v] = Prog::identity();
      my_g += i1 - i0;
      if (Prog::apply(&cur, r, cx)) {
        P.val[v] = cur;
        nv = cur;
        changed = true;
        beg = (uint64_t)P.out_off[v];
        deg = (uint32_t)((uint64_t)P.out_off[v + 1] - beg);
        my_s += deg;
        my_c += 1;
      }
    }
    my_act += expand_warp_push<Prog>(P, changed, beg, deg, v, nv, cx, accn, epoch, qA, ns);
  }
  // A_t hubs (out-degree > kHubDegree), one CTA per out-edge chunk: every chunk
  // applies on a private copy of acc[v] / val[v] (neither changes until all
  // chunks have read them), pushes its chunk if v changes, and the last chunk
  // to read commits (value, accumulator reset, trace counts).
  for (; nK;) {
    __syncthreads();
    if (threadIdx.x == 0) s_h = atomicAdd(&ctl->ctr_hub, 1u);
    __syncthreads();
    const uint32_t i = s_h;
    if (i >= nK) break;
    const uint32_t hp = P.chkA_h[slot][i], ci = P.chkA_c[slot][i];
    const uint32_t v = LH[hp];
    const uint64_t beg = (uint64_t)P.out_off[v];
    const uint64_t deg = (uint64_t)P.out_off[v + 1] - beg;
    if (threadIdx.x == 0) {
      const uint32_t r = *(volatile uint32_t *)(acc + v);
      uint32_t cur = *(volatile uint32_t *)(P.val + v);
      const bool ch = Prog::apply(&cur, r, cx);
      s_changed = ch;
      s_nv = cur;
      __threadfence();
      const uint32_t nch = (uint32_t)((deg + kChunk - 1) / kChunk);
      if (atomicAdd(P.hub_done + hp, 1u) == nch - 1) {
        P.hub_done[hp] = 0;
        acc[v] = Prog::identity();
        if (ch) {
          P.val[v] = cur;
          my_c += 1;
          my_s += deg;
        }
        my_g += (uint64_t)P.in_off[v - P.own_lo + 1] - (uint64_t)P.in_off[v - P.own_lo];
      }
    }
    __syncthreads();
    if (!s_changed) continue;
    const uint32_t a = expand_block_push<Prog>(P, beg + (uint64_t)ci * kChunk, chunk_len(deg, ci), v, s_nv, cx,
                                               accn, epoch, qA, ns);
    if (lane == 0) my_act += a;
  }
  qA.block_flush(P.listA[ns], nullptr, &ctl->cnt_A[ns], s_off);
  my_g = block_sum_u64(my_g, s8);
  if (threadIdx.x == 0 && my_g) atomicAdd(&ctl->part_g[blockIdx.x % kSlots], my_g);
  my_s = block_sum_u64(my_s, s8);
  if (threadIdx.x == 0 && my_s) atomicAdd(&ctl->part_s[blockIdx.x % kSlots], my_s);
  my_c = block_sum_u64(my_c, s8);
  if (threadIdx.x == 0 && my_c) atomicAdd(&ctl->part_c[blockIdx.x % kSlots], my_c);
  my_act = block_sum_u64(lane == 0 ? my_act : 0ull, s8);
  if (threadIdx.x == 0 && my_act) atomicAdd(&ctl->part_a[blockIdx.x % kSlots], my_act);
  prof_end(ctl, V, 1);
}

template <class Prog, class OffT>
__global__ void __launch_bounds__(kBlock) k_push_expand(const __grid_constant__ Part<OffT> P, unsigned long long cond,
                                                        int use_graph) {
  __shared__ View V;
  load_view(P.ctl, V);
  if (V.stop) {
    if (use_graph && blockIdx.x == 0 && threadIdx.x == 0)
      cudaGraphSetConditional((cudaGraphConditionalHandle)cond, 0u);
    return;
  }
  if constexpr (PushFused<Prog>::value) push_phase<Prog>(P, V);
  finish_superstep(P, cond, use_graph, kPush);
}

// ------------------------------------------------------ scatter (edge state)
// Programs with kHasScatter (gr/program.cuh): superstep t commits the new
// values of C_t in its own phase (commit_only_phase), then, after a grid
// barrier, every out-edge (u -> x) of every u in C_t runs
// scatter(new[u], val_t[x], w, &state[csc position]) before FrontierActivate
// (§2.1, §4.4). Each edge has one source, which appears once
// in C_t, so each state is written by exactly one thread per superstep.
template <class OffT>
__device__ __forceinline__ void commit_only_phase(const Part<OffT> &P, const View &V) {
  const uint32_t nC = V.cntC, nCH = V.cntCH;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < nC + nCH; i += gridDim.x * blockDim.x) {
    const bool h = i >= nC;
    const uint32_t u = h ? P.CH_v[i - nC] : P.C_v[i];
    P.val[u] = h ? P.CH_val[i - nC] : P.C_val[i];  // BSP commit of superstep t
  }
}

template <class Prog, class OffT>
__device__ __forceinline__ void scatter_batch(const Part<OffT> &P, const bool (&act)[kBatch],
                                              const uint32_t (&x)[kBatch], const uint32_t (&w)[kBatch],
                                              const uint32_t (&eid)[kBatch], const uint32_t (&sv)[kBatch],
                                              const Ctx &cx) {
  uint32_t dv[kBatch];
#pragma unroll
  for (int q = 0; q < kBatch; q++) dv[q] = act[q] ? ld_cg(P.val + x[q]) : 0u;  // committed values of t
#pragma unroll
  for (int q = 0; q < kBatch; q++)
    if (act[q]) Prog::scatter(sv[q], dv[q], w[q], P.estate + eid[q], cx);
}

template <class Prog, class OffT>
__device__ uint32_t expand_warp_scatter(const Part<OffT> &P, bool valid, uint64_t beg, uint32_t deg, uint32_t nv,
                                        const Ctx &cx, uint32_t epoch, WarpQueue &qA, uint32_t slot) {
  const uint32_t lane = lane_id();
  const uint32_t d = valid ? deg : 0u;
  const uint32_t incl = warp_incl_scan(d);
  const uint32_t excl = incl - d;
  const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
  uint32_t nact = 0;
  for (uint32_t r0 = 0; r0 < total; r0 += 32u * kBatch) {
    bool act[kBatch];
    uint32_t x[kBatch], w[kBatch], eid[kBatch], sv[kBatch];
#pragma unroll
    for (int q = 0; q < kBatch; q++) {
      const uint32_t k = r0 + q * 32u + lane;
      int o = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const uint32_t e = __shfl_sync(0xffffffffu, excl, o + step);
        if (e <= k) o += step;
      }
      const uint64_t ob = __shfl_sync(0xffffffffu, beg, o);
      const uint32_t oe = __shfl_sync(0xffffffffu, excl, o);
      sv[q] = __shfl_sync(0xffffffffu, nv, o);
      act[q] = k < total;
      const uint64_t e = ob + (k - oe);
      x[q] = act[q] ? ldg_nc(P.out_dst + e) : 0u;
      w[q] = (act[q] && Prog::kUsesWeights) ? (uint32_t)ldg_nc_u8(P.out_w + e) : 0u;
      eid[q] = act[q] ? ldg_nc(P.out_eid + e) : 0u;
    }
    scatter_batch<Prog>(P, act, x, w, eid, sv, cx);
    nact += activate_batch<false>(P, act, x, epoch, P.hub_in, qA, slot);
  }
  return nact;  // warp-uniform
}

template <class Prog, class OffT>
__device__ uint32_t expand_block_scatter(const Part<OffT> &P, uint64_t beg, uint32_t deg, uint32_t nv,
                                         const Ctx &cx, uint32_t epoch, WarpQueue &qA, uint32_t slot) {
  uint32_t nact = 0;
  for (uint32_t r0 = 0; r0 < deg; r0 += kBlock * kBatch) {
    bool act[kBatch];
    uint32_t x[kBatch], w[kBatch], eid[kBatch], sv[kBatch];
#pragma unroll
    for (int q = 0; q < kBatch; q++) {
      const uint32_t k = r0 + q * kBlock + threadIdx.x;
      act[q] = k < deg;
      x[q] = act[q] ? ldg_nc(P.out_dst + beg + k) : 0u;
      w[q] = (act[q] && Prog::kUsesWeights) ? (uint32_t)ldg_nc_u8(P.out_w + beg + k) : 0u;
      eid[q] = act[q] ? ldg_nc(P.out_eid + beg + k) : 0u;
      sv[q] = nv;
    }
    scatter_batch<Prog>(P, act, x, w, eid, sv, cx);
    nact += activate_batch<false>(P, act, x, epoch, P.hub_in, qA, slot);
  }
  return nact;  // per-warp count
}

// scatter + FrontierActivate over C_t (values already committed)
template <class Prog, class OffT>
__device__ __forceinline__ void scatter_activate_phase(const Part<OffT> &P, const View &V) {
  Ctl *ctl = P.ctl;
  const uint32_t t = V.t;
  const uint32_t ns = (t + 1) & 1u;
  const uint32_t epoch = V.epoch_base + t + 1;
  const uint32_t nC = V.cntC;
  const uint32_t nKC = V.cntKC;
  const Ctx cx = make_ctx(P, V);
  prof_begin(ctl, V, 1);

  GR_SQ1(sq);
  __shared__ uint32_t s_h;
  __shared__ uint32_t s_off[kWarpsPerBlock + 1];
  __shared__ unsigned long long s8[kWarpsPerBlock];
  const uint32_t warp = threadIdx.x / 32, lane = lane_id();
  WarpQueue qA{sq[warp], nullptr, 0};
  unsigned long long my_s = 0, my_act = 0;

  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = gw * 32u; base < nC; base += nw * 32u) {
    const uint32_t idx = base + lane;
    const bool valid = idx < nC;
    uint64_t beg = 0;
    uint32_t deg = 0, nv = 0;
    if (valid) {
      const uint32_t u = P.C_v[idx];
      nv = P.C_val[idx];
      beg = (uint64_t)P.out_off[u];
      deg = (uint32_t)((uint64_t)P.out_off[u + 1] - beg);
      my_s += deg;
    }
    my_act += expand_warp_scatter<Prog>(P, valid, beg, deg, nv, cx, epoch, qA, ns);
  }
  for (; nKC;) {
    __syncthreads();
    if (threadIdx.x == 0) s_h = atomicAdd(&ctl->ctr_hub2, 1u);
    __syncthreads();
    const uint32_t i = s_h;
    if (i >= nKC) break;
    const uint32_t hp = P.chkC_h[i], ci = P.chkC_c[i];
    const uint32_t u = P.CH_v[hp];
    const uint64_t beg = (uint64_t)P.out_off[u];
    const uint64_t deg = (uint64_t)P.out_off[u + 1] - beg;
    if (threadIdx.x == 0 && ci == 0) my_s += deg;
    const uint32_t a = expand_block_scatter<Prog>(P, beg + (uint64_t)ci * kChunk, chunk_len(deg, ci), P.CH_val[hp],
                                                  cx, epoch, qA, ns);
    if (lane == 0) my_act += a;
  }
  qA.block_flush(P.listA[ns], nullptr, &ctl->cnt_A[ns], s_off);
  my_s = block_sum_u64(my_s, s8);
  if (threadIdx.x == 0 && my_s) atomicAdd(&ctl->part_s[blockIdx.x % kSlots], my_s);
  my_act = block_sum_u64(lane == 0 ? my_act : 0ull, s8);
  if (threadIdx.x == 0 && my_act) atomicAdd(&ctl->part_a[blockIdx.x % kSlots], my_act);
  prof_end(ctl, V, 1);
}

template <class OffT>
__global__ void __launch_bounds__(kBlock) k_commit_only(const __grid_constant__ Part<OffT> P) {
  __shared__ View V;
  load_view(P.ctl, V);
  if (V.stop) return;
  commit_only_phase(P, V);
}

template <class Prog, class OffT>
__global__ void __launch_bounds__(kBlock) k_scatter_activate(const __grid_constant__ Part<OffT> P,
                                                             unsigned long long cond, int use_graph) {
  __shared__ View V;
  load_view(P.ctl, V);
  if (V.stop) {
#ifndef GR_JIT  // run-time programs never run inside a conditional graph node
    if (use_graph && blockIdx.x == 0 && threadIdx.x == 0)
      cudaGraphSetConditional((cudaGraphConditionalHandle)cond, 0u);
#endif
    return;
  }
  if constexpr (HasScatter<Prog>::value) scatter_activate_phase<Prog>(P, V);
  finish_superstep(P, cond, use_graph, kPush);
}

template <class Prog, class OffT>
__global__ void k_init_edges(const __grid_constant__ Part<OffT> P, uint64_t m) {
  if constexpr (HasScatter<Prog>::value) {
    Ctx cx{};
    cx.n = P.n;
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < m; e += (uint64_t)gridDim.x * blockDim.x)
      P.estate[e] = Prog::initEdge(P.in_w ? (uint32_t)P.in_w[e] : 0u, cx);
  }
}

// ------------------------------------------------ dense edge-segmented gather
// Dense (pull) supersteps of kDstFreeGather programs (gr/program.cuh): instead
// of 32 vertices per warp with a shuffle owner search per edge, the CSC is laid
// out as 256-item tiles (one item per in-edge, one empty item per row without
// in-edges, a head bit at each row's first item; the PageRank seg layout
// without hot tags). A warp walks whole tiles: lane L loads items 8L..8L+7 with
// two 128-bit loads, maps them (gatherMap of the source's value; the changed
// bit of the source marks the row active), reduces them in registers and joins
// rows split between lanes with one segmented shuffle scan. Rows that lie in
// one tile apply at once; rows spanning tiles (listed once per graph) combine
// their pieces with atomicGather / atomicOr and apply after a grid barrier
// (dense_split_phase). gatherReduce is associative and commutative (R9), and
// exact for every program with this trait (integer min / max / sum), so the
// result does not depend on the piece order.
constexpr uint32_t kDsIpt = 8;
constexpr uint32_t kDsTile = 32 * kDsIpt;
constexpr uint32_t kDsNoSrc = 0xFFFFFFFFu;

template <class Prog, class OffT>
__device__ __forceinline__ void ds_apply_row(const Part<OffT> &P, uint32_t lv, typename Prog::GatherT acc,
                                             const Ctx &cx, WarpQueue &qC, bool p, unsigned long long &my_g,
                                             unsigned long long &my_c, unsigned long long &my_a, bool no_hub_c) {
  // every lane calls (qC.push is warp-collective); p: this lane applies row lv
  bool changed = false, hubo = false;
  uint32_t v = 0, nv = 0;
  if (p) {
    v = P.own_lo + lv;
    const uint32_t cur = P.val[v];
    my_g += (uint64_t)P.in_off[lv + 1] - (uint64_t)P.in_off[lv];
    my_a += 1;
    nv = cur;
    changed = Prog::apply(&nv, acc, cx);
    if (changed) {
      my_c += 1;
      hubo = !no_hub_c && test_bit(P.hub_out, v);
      if (hubo) append_hub_C(P, v, nv);
    }
  }
  qC.push(changed && !hubo, v, nv, P.C_v, P.C_val, &P.ctl->cnt_C);
}

struct DsSmem {
  unsigned long long s8[kWarpsPerBlock];
  uint32_t sq[kWarpsPerBlock][2][kQueueCap];
  uint32_t s_off[kWarpsPerBlock + 1];
};
__device__ __forceinline__ DsSmem &ds_smem() {
#ifdef GR_NO_SMEM_UNION
  __shared__ DsSmem s;
  return s;
#else
  static_assert(sizeof(DsSmem) <= kPhaseSmemBytes, "dense-tile scratch fits the phase scratch");
  return *reinterpret_cast<DsSmem *>(g_phase_smem);
#endif
}

template <class Prog, bool kGateT, class OffT>
__device__ __forceinline__ void dense_seg_phase(const Part<OffT> &P, const View &V) {
  using G = typename Prog::GatherT;
  Ctl *ctl = P.ctl;
  const uint32_t slot = V.t & 1u;
  const uint32_t *bits = P.cbits[slot ^ 1u];  // C_{t-1}
  const Ctx cx = make_ctx(P, V);
  const bool no_hub_c = V.no_hub_c != 0;
  prof_begin(ctl, V, 0);
  // one shared-memory scratch for both gate variants of this phase (a __shared__ array
  // declared in each template instantiation would be allocated twice per kernel)
  DsSmem &S = ds_smem();
  unsigned long long *s8 = S.s8;
  const uint32_t warp = threadIdx.x / 32, lane = lane_id();
  uint32_t (*sq)[2][kQueueCap] = S.sq;
  uint32_t *s_off = S.s_off;
  WarpQueue qC{sq[warp][0], sq[warp][1], 0};
  unsigned long long my_g = 0, my_c = 0, my_a = 0;
  G *acc_g = reinterpret_cast<G *>(P.ds_acc);
  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t tile = gw; tile < P.ds_tiles; tile += nw) {
    const uint4 *s4 = reinterpret_cast<const uint4 *>(P.ds_src + (uint64_t)tile * kDsTile) + 2 * lane;
    const uint4 s0 = __ldg(s4), s1 = __ldg(s4 + 1);
    const uint32_t fw = __ldg(P.ds_flags + (uint64_t)tile * 8 + (lane >> 2));
    const uint32_t fnext = __ldg(P.ds_flags + (uint64_t)tile * 8 + 8) & 1u;
    const uint32_t r0 = __ldg(P.ds_row + tile);
    const uint32_t src[kDsIpt] = {s0.x, s0.y, s0.z, s0.w, s1.x, s1.y, s1.z, s1.w};
    uint32_t w8[kDsIpt];
    if (Prog::kUsesWeights) {
      const uint2 wv = __ldg(reinterpret_cast<const uint2 *>(P.ds_w + (uint64_t)tile * kDsTile) + lane);
#pragma unroll
      for (int k = 0; k < 4; k++) { w8[k] = (wv.x >> (8 * k)) & 0xFFu; w8[k + 4] = (wv.y >> (8 * k)) & 0xFFu; }
    }
    uint32_t sv[kDsIpt];
    bool sa[kDsIpt];
    constexpr bool kGate = kGateT && kGateSelective && Selective<Prog>::value;  // only the changed sources' values
#pragma unroll
    for (int k = 0; k < kDsIpt; k++) {  // all loads of the 8 items in flight together
      const bool ok = src[k] != kDsNoSrc;
      // values and changed bits were written earlier in this (persistent) launch: coherent
      // loads, not the read-only .nc path (valid only for data read-only during the kernel)
      if (!kGate) sv[k] = ok ? P.val[src[k]] : 0u;
      sa[k] = ok && test_bit_w(bits, src[k]);
    }
    if (kGate) {
#pragma unroll
      for (int k = 0; k < kDsIpt; k++) sv[k] = sa[k] ? P.val[src[k]] : 0u;
    }
    G g[kDsIpt];
#pragma unroll
    for (int k = 0; k < kDsIpt; k++)
      g[k] = (kGate ? sa[k] : src[k] != kDsNoSrc)
                 ? Prog::gatherMap(0u, sv[k], Prog::kUsesWeights ? w8[k] : 0u, src[k], cx)
                 : Prog::identity();
    const uint32_t b = (fw >> ((lane & 3) * 8)) & 0xFFu;  // bit k: my item k starts a row
    uint32_t bn = __shfl_down_sync(0xffffffffu, b, 1) & 1u;
    if (lane == 31) bn = fnext;
    const uint32_t ends = (b >> 1) | (bn << 7);  // bit k: my item k ends a row
    // lane tail (after my last head) and its active flag
    G tail = Prog::identity();
    bool tact = false;
#pragma unroll
    for (int k = 0; k < kDsIpt; k++) {
      if ((b >> k) & 1u) { tail = Prog::identity(); tact = false; }
      tail = Prog::gatherReduce(tail, g[k]);
      tact = tact || sa[k];
    }
    // segmented inclusive scan of the tails over lanes (segments start at lanes with a head)
    uint32_t cnt = __popc(b);
    G x = tail;
    uint32_t xa = tact ? 1u : 0u;
    const uint32_t hl = __ballot_sync(0xffffffffu, b != 0u) & (0xFFFFFFFFu >> (31 - lane));
    const int seg0 = hl ? 31 - __clz(hl) : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const G y = __shfl_up_sync(0xffffffffu, x, o);
      const uint32_t ya = __shfl_up_sync(0xffffffffu, xa, o);
      const uint32_t c = __shfl_up_sync(0xffffffffu, cnt, o);
      if ((int)lane - o >= seg0) { x = Prog::gatherReduce(x, y); xa |= ya; }
      if (lane >= (uint32_t)o) cnt += c;
    }
    G run = __shfl_up_sync(0xffffffffu, x, 1);
    uint32_t ract = __shfl_up_sync(0xffffffffu, xa, 1);
    if (lane == 0) { run = Prog::identity(); ract = 0u; }
    const uint32_t h0 = __shfl_sync(0xffffffffu, b, 0) & 1u;
    uint32_t row = r0 - h0 + (cnt - __popc(b));  // row of the item before my first head
    // walk my items: complete rows apply (collectively, one row per lane per step),
    // pieces of rows spanning tiles go to the split accumulators
    uint32_t done_rows = 0;  // bit k: my item k completes a row that started in this tile
    G done_val[kDsIpt];
    bool done_act[kDsIpt];
#pragma unroll
    for (int k = 0; k < kDsIpt; k++) {
      if ((b >> k) & 1u) { run = Prog::identity(); ract = 0u; ++row; }
      run = Prog::gatherReduce(run, g[k]);
      ract |= sa[k] ? 1u : 0u;
      done_val[k] = run;
      done_act[k] = ract != 0u;
      if (((ends >> k) & 1u) && row < P.own_n) {
        if (!h0 && row == r0) {  // began in an earlier tile: a piece
          Prog::atomicGather(acc_g + row, run);
          if (ract) atomicOr(P.ds_act + (row >> 5), 1u << (row & 31));
        } else {
          done_rows |= 1u << k;
        }
      }
    }
    if (lane == 31 && !fnext && row < P.own_n) {  // the last row continues in the next tile: a piece
      Prog::atomicGather(acc_g + row, run);
      if (ract) atomicOr(P.ds_act + (row >> 5), 1u << (row & 31));
    }
    // apply the complete active rows, each lane its own: the loads of all of them
    // first (one round trip), then the applies, then one warp-queue push per item slot
    uint32_t rr = r0 - h0 + (cnt - __popc(b));
    uint32_t cur[kDsIpt], dg[kDsIpt], vv[kDsIpt];
#pragma unroll
    for (int k = 0; k < kDsIpt; k++) {
      if ((b >> k) & 1u) ++rr;
      vv[k] = P.own_lo + rr;
      const bool p = ((done_rows >> k) & 1u) && done_act[k];
      cur[k] = p ? P.val[vv[k]] : 0u;
      dg[k] = p ? (uint32_t)((uint64_t)P.in_off[rr + 1] - (uint64_t)P.in_off[rr]) : 0u;
    }
    uint32_t chg = 0;
#pragma unroll
    for (int k = 0; k < kDsIpt; k++) {
      if (((done_rows >> k) & 1u) && done_act[k]) {
        my_g += dg[k];
        my_a += 1;
        if (Prog::apply(&cur[k], done_val[k], cx)) {
          my_c += 1;
          if (!no_hub_c && test_bit(P.hub_out, vv[k])) append_hub_C(P, vv[k], cur[k]);
          else chg |= 1u << k;
        }
      }
    }
    if (__any_sync(0xffffffffu, chg != 0u)) {
#pragma unroll
      for (int k = 0; k < kDsIpt; k++) qC.push((chg >> k) & 1u, vv[k], cur[k], P.C_v, P.C_val, &ctl->cnt_C);
    }
  }
  qC.block_flush(P.C_v, P.C_val, &ctl->cnt_C, s_off);
  my_g = block_sum_u64(my_g, s8);
  if (threadIdx.x == 0 && my_g) atomicAdd(&ctl->part_g[blockIdx.x % kSlots], my_g);
  my_c = block_sum_u64(my_c, s8);
  if (threadIdx.x == 0 && my_c) atomicAdd(&ctl->part_c[blockIdx.x % kSlots], my_c);
  my_a = block_sum_u64(my_a, s8);
  if (threadIdx.x == 0 && my_a) atomicAdd(&ctl->cnt_act[slot], (uint32_t)my_a);
  prof_end(ctl, V, 0);
}

// the rows spanning tiles (after a grid barrier): combined pieces apply, slots reset
template <class Prog, class OffT>
__device__ __forceinline__ void dense_split_phase(const Part<OffT> &P, const View &V) {
  using G = typename Prog::GatherT;
  Ctl *ctl = P.ctl;
  const uint32_t slot = V.t & 1u;
  const Ctx cx = make_ctx(P, V);
  const bool no_hub_c = V.no_hub_c != 0;
  GR_SQ2(sq);
  __shared__ uint32_t s_off[kWarpsPerBlock + 1];
  __shared__ unsigned long long s8[kWarpsPerBlock];
  const uint32_t warp = threadIdx.x / 32;
  WarpQueue qC{sq[warp][0], sq[warp][1], 0};
  unsigned long long my_g = 0, my_c = 0, my_a = 0;
  G *acc_g = reinterpret_cast<G *>(P.ds_acc);
  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = gw * 32u; base < P.ds_nsplit; base += nw * 32u) {
    const uint32_t i = base + lane_id();
    bool p = false;
    uint32_t r = 0;
    G acc = Prog::identity();
    if (i < P.ds_nsplit) {
      r = P.ds_split[i];
      acc = acc_g[r];
      acc_g[r] = Prog::identity();
      const uint32_t m = 1u << (r & 31);
      p = (ld_cg(P.ds_act + (r >> 5)) & m) != 0u;
      if (p) atomicAnd(P.ds_act + (r >> 5), ~m);
    }
    ds_apply_row<Prog>(P, r, acc, cx, qC, p, my_g, my_c, my_a, no_hub_c);
  }
  qC.block_flush(P.C_v, P.C_val, &ctl->cnt_C, s_off);
  my_g = block_sum_u64(my_g, s8);
  if (threadIdx.x == 0 && my_g) atomicAdd(&ctl->part_g[blockIdx.x % kSlots], my_g);
  my_c = block_sum_u64(my_c, s8);
  if (threadIdx.x == 0 && my_c) atomicAdd(&ctl->part_c[blockIdx.x % kSlots], my_c);
  my_a = block_sum_u64(my_a, s8);
  if (threadIdx.x == 0 && my_a) atomicAdd(&ctl->cnt_act[slot], (uint32_t)my_a);
}

// Grid barrier of the persistent loop: the monotone arrival counter in the
// control block (zeroed with the rest of it before every run).
__device__ __forceinline__ void grid_sync(Ctl *c, uint32_t &bar) { grid_barrier(&c->bar_count, bar); }

// Persistent device-side BSP loop (one cooperative launch per run): phases are
// separated by grid barriers instead of kernel boundaries, and CTA 0 closes
// each superstep while the others wait — no launch or host round trip per
// superstep (the latency floor of high-diameter graphs, cfg3).
template <class Prog, class OffT, bool kDS>
__device__ __forceinline__ void persistent_body(const Part<OffT> &P) {
  Ctl *ctl = P.ctl;
  __shared__ View V;
  uint32_t bar = 0;  // grid barrier target (thread 0)
  for (;;) {
    load_view(ctl, V);
    if (V.stop) break;
    int pull;
    if constexpr (HasScatter<Prog>::value) {  // gather | commit | scatter + activate (push only)
      gather_phase<Prog, false>(P, V);
      grid_sync(ctl, bar);
      load_view(ctl, V);
      commit_only_phase(P, V);
      grid_sync(ctl, bar);
      scatter_activate_phase<Prog>(P, V);
      grid_sync(ctl, bar);
      if (blockIdx.x == 0) close_superstep(P, 0ull, 0, kPush);
      grid_sync(ctl, bar);
      continue;
    }
    if constexpr (PushFused<Prog>::value) {
      if (V.push) {  // one phase; the last CTA to finish closes the superstep
        push_phase<Prog>(P, V);
        finish_superstep(P, 0ull, 0, kPush);
        grid_sync(ctl, bar);
        continue;
      }
    }
    if (Prog::kHasGather) {
      if (V.dense) {
        if constexpr (kDS && DstFree<Prog>::value) {  // edge-segmented tiles, then the split rows
          if (kGateSelective && Selective<Prog>::value && V.gate) dense_seg_phase<Prog, true>(P, V);
          else dense_seg_phase<Prog, false>(P, V);
          grid_sync(ctl, bar);
          dense_split_phase<Prog>(P, V);
        } else {
          dense_gather_phase<Prog>(P, V);
        }
      } else {
        gather_phase<Prog, false>(P, V);
      }
      grid_sync(ctl, bar);
      load_view(ctl, V);
      clear_dirty(P, V, cbits_words(P));
      pull = pull_mode(V, P.own_n, frontier_gather(V)) ? kPullDense : kPush;
      if (pull) commit_phase(P, V);  // superstep t+1 gathers densely
      else activate_phase(P, V);
    } else {
      clear_dirty(P, V, cbits_words(P));
      pull = pull_mode(V, P.own_n, frontier_bfs(V)) ? kPullScan : kPush;
      if (pull) {
        bfs_apply_phase(P, V);
        grid_sync(ctl, bar);
        pull_phase<true>(P, V);
      } else {
        bfs_phase(P, V);
      }
    }
    grid_sync(ctl, bar);
    if (blockIdx.x == 0) close_superstep(P, 0ull, 0, pull);
    grid_sync(ctl, bar);
  }
}

// 32-bit gathers are compiled for 4 resident CTAs per SM (64 registers): the
// dense CC superstep is occupancy-bound (cfg4: 12.4 ms at 64 registers, 14.6 ms
// when ptxas picked 80 for the same code)
#ifndef GR_PERSIST_CTAS32  // A/B builds: resident CTAs per SM the 32-bit-gather loops are compiled for
#define GR_PERSIST_CTAS32 4
#endif
template <class Prog> struct PersistMinCtas {
  static constexpr int value = sizeof(typename Prog::GatherT) == 4 ? GR_PERSIST_CTAS32 : 3;
};
template <class Prog, class OffT>
__global__ void __launch_bounds__(kBlock, PersistMinCtas<Prog>::value) k_persistent(const __grid_constant__ Part<OffT> P) {
  persistent_body<Prog, OffT, false>(P);
}

#ifndef GR_JIT
// the loop with dense supersteps on edge-segmented tiles (a kernel of its own:
// the tile code's registers would otherwise lower the occupancy of every phase)
template <class Prog, class OffT>
__global__ void __launch_bounds__(kBlock, 3) k_persistent_ds(const __grid_constant__ Part<OffT> P) {
  persistent_body<Prog, OffT, DstFree<Prog>::value>(P);
}
#endif


// Regions of the exchange buffer holding each rank's C_t (fused exchange): rank q's
// entries at [off[q], off[q] + pre[q+1] - pre[q]); nr == 0: one contiguous list
struct XRanges {
  uint32_t off[16], pre[17];
  uint32_t nr;
};
// device-side count exchange of partitioned runs (engine_part.cu): every rank's
// (|C_t|, |A_t|) by superstep parity, with a per-slot sequence number (t + 1)
struct XCount {
  unsigned long long cnt[2][16][2];
  uint32_t seq[2][16];
};
// this rank's decision after the count exchange of superstep t
struct XDev {
  XRanges R;
  uint32_t tot;                 // global |C_t|
  unsigned long long bytes_in;  // changed-set bytes received from peers (stats)
  unsigned long long timeout;   // (rank << 32 | seq) of a count that never arrived (0: none)
};

// Partitioned runs: split the exchanged changed set (every rank's C_t) into
// the local non-hub list and the local changed-hub chunks (hub-ness depends on
// this rank's activation CSR).
template <class OffT>
__global__ void __launch_bounds__(kBlock) k_classify(const __grid_constant__ Part<OffT> P, const uint32_t *X_v,
                                                     const uint32_t *X_val, uint32_t nX, const XRanges R) {
  GR_SQ2(sq);
  __shared__ uint32_t s_off[kWarpsPerBlock + 1];
  const uint32_t warp = threadIdx.x / 32, lane = lane_id();
  WarpQueue qC{sq[warp][0], sq[warp][1], 0};
  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = gw * 32u; base < nX; base += nw * 32u) {
    const uint32_t i = base + lane;
    const bool valid = i < nX;
    uint32_t at = i;  // fused exchange: entry i of the concatenation of the rank regions
    if (valid && R.nr) {
      uint32_t q = 0;
      while (q + 1 < R.nr && R.pre[q + 1] <= i) q++;
      at = R.off[q] + (i - R.pre[q]);
    }
    const uint32_t u = valid ? X_v[at] : 0u, val = valid ? X_val[at] : 0u;
    const bool hub = valid && test_bit(P.hub_out, u);
    if (hub) append_hub_C(P, u, val);
    qC.push(valid && !hub, u, val, P.C_v, P.C_val, &P.ctl->cnt_C);
  }
  qC.block_flush(P.C_v, P.C_val, &P.ctl->cnt_C, s_off);
}

// ----------------------------------------------------------- initialisation
template <class Prog, class OffT>
__global__ void k_init_values(const __grid_constant__ Part<OffT> P, uint32_t source) {
  Ctx cx{};
  cx.n = P.n;
  cx.source = source;
  cx.prd_r0 = P.ctl->prd_r0;
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < P.n; v += (uint64_t)gridDim.x * blockDim.x)
    P.val[v] = Prog::initValue((uint32_t)v, cx);
}

// All per-run resets of a resident frontier run in one launch (small graphs are
// bound by the launches before the persistent loop): initial values, the hub
// accumulators (identity) and done counters, and (pull) both changed bitmaps.
template <class Prog, class OffT>
__global__ void k_init_run(const __grid_constant__ Part<OffT> P, uint32_t source, uint64_t hub_cap,
                           uint64_t cbits_words, int zero_cbits) {
  using G = typename Prog::GatherT;
  Ctx cx{};
  cx.n = P.n;
  cx.source = source;
  cx.prd_r0 = P.ctl->prd_r0;
  const uint64_t i0 = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x, st = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t v = i0; v < P.n; v += st) P.val[v] = Prog::initValue((uint32_t)v, cx);
  G *ha = reinterpret_cast<G *>(P.hub_acc);
  for (uint64_t i = i0; i < hub_cap; i += st) {
    ha[i] = Prog::identity();
    P.hub_done[i] = 0u;
  }
  if (zero_cbits)
    for (uint64_t i = i0; i < cbits_words; i += st) {
      P.cbits[0][i] = 0u;
      P.cbits[1][i] = 0u;
    }
}

template <class T> __global__ void k_fill(T *p, T value, uint64_t count) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = value;
}

// identity() into a gather accumulator array of the program's GatherT (hub slots)
template <class Prog> __global__ void k_prog_fill(void *p, unsigned long long count) {
  typename Prog::GatherT *a = reinterpret_cast<typename Prog::GatherT *>(p);
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < count;
       i += (unsigned long long)gridDim.x * blockDim.x)
    a[i] = Prog::identity();
}

static __global__ void k_fill_u32(uint32_t *p, uint32_t value, uint64_t count) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = value;
}

// Stage 1 (L62): the starting frontier A_0. One CTA. kInitAll expects listH[0]
// and the chunk list of slot 0 pre-filled with the static in-hub list.
template <class Prog, class OffT>
__global__ void __launch_bounds__(kBlock) k_init_frontier(const __grid_constant__ Part<OffT> P, uint32_t source,
                                                          uint32_t n_static_hubs, uint32_t n_static_chunks) {
  Ctl *ctl = P.ctl;
  const uint32_t epoch0 = ctl->epoch_base;
  const bool owned = source >= P.own_lo && source < P.own_lo + P.own_n;
  if (Prog::kInit == kInitAll) {
    if (threadIdx.x == 0) {
      ctl->implicit0 = 1;
      ctl->cnt_A[0] = P.own_n;
      ctl->cnt_H[0] = n_static_hubs;
      ctl->cnt_K[0] = n_static_chunks;
      ctl->cnt_act[0] = P.own_n;
      ctl->stop = (P.own_n == 0);
    }
    return;
  }
  if (Prog::kInit == kInitSource) {
    if (threadIdx.x == 0) {
      if (owned) {
        P.stamp[source - P.own_lo] = epoch0;
        const bool hub = test_bit(Prog::kHasGather ? P.hub_in : P.hub_out,
                                  Prog::kHasGather ? source - P.own_lo : source);
        if (hub) append_hub_A<!Prog::kHasGather>(P, source, 0);
        else { P.listA[0][0] = source; ctl->cnt_A[0] = 1; }
        ctl->cnt_act[0] = 1;
      }
      ctl->stop = owned ? 0u : 1u;
    }
    return;
  }
  // kInitSourceChanged: the source is "changed" at initialisation; A_0 = out-neighbours.
  __shared__ uint32_t sq[kWarpsPerBlock][kQueueCap];
  const uint32_t warp = threadIdx.x / 32;
  WarpQueue qA{sq[warp], nullptr, 0};
  const uint64_t beg = (uint64_t)P.out_off[source];
  const uint32_t deg = (uint32_t)((uint64_t)P.out_off[source + 1] - beg);
  uint32_t a;
  if constexpr (HasScatter<Prog>::value) {  // the source changed at init: it scatters
    Ctx cx{};
    cx.n = P.n;
    cx.source = source;
    cx.outdeg = P.outdeg;
    a = expand_block_scatter<Prog>(P, beg, deg, P.val[source], cx, epoch0, qA, 0);
  } else if constexpr (PushFused<Prog>::value) {
    if (ctl->push) {  // fused push supersteps: the source's value is pushed into acc_0
      Ctx cx{};
      cx.n = P.n;
      cx.source = source;
      cx.outdeg = P.outdeg;
      a = expand_block_push<Prog>(P, beg, deg, source, P.val[source], cx, P.nxt[0], epoch0, qA, 0);
    } else {
      a = expand_block<false>(P, beg, deg, epoch0, P.hub_in, qA, 0);
    }
  } else {
    a = expand_block<false>(P, beg, deg, epoch0, P.hub_in, qA, 0);
  }
  qA.flush(P.listA[0], nullptr, &ctl->cnt_A[0]);
  if (lane_id() == 0 && a) atomicAdd(&ctl->cnt_act[0], a);
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    ctl->stop = (*(volatile uint32_t *)&ctl->cnt_act[0] == 0) ? 1u : 0u;
  }
}

}  // namespace gr
