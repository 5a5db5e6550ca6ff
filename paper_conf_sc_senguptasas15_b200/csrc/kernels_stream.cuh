// kernels_stream.cuh — per-shard kernels of the streamed (out-of-core) mode.
// shards whose edges exceed HBM stay in pinned
// host memory (§3.2) and are copied per superstep into one of
// K = 2 device slots (Eq. 1-2). A shard is copied only when it holds an
// active vertex (gather) or a changed vertex (FrontierActivate) — the frontier
// skipping of §5.2 L270. The kernels scan the shard's vertex interval and test
// the per-vertex epoch stamps, so no list has to be bucketed by shard.
#pragma once
#include "kernels_frontier.cuh"

namespace gr {

// shard containing vertex x: last s with bounds[s] <= x
__device__ __forceinline__ uint32_t shard_of(const uint64_t *bounds, uint32_t P, uint32_t x) {
  uint32_t lo = 0, hi = P;  // invariant: bounds[lo] <= x < bounds[hi]
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (__ldg(bounds + mid) <= x) lo = mid;
    else hi = mid;
  }
  return lo;
}

// Gather + apply over the active vertices of one shard [v0, v1); in-edges in a slot.
// shard == kAllShards: one launch over every shard's interval (zero-copy
// phases); changed flags are then set per vertex through `bounds`.
constexpr uint32_t kAllShards = 0xFFFFFFFFu;
template <class Prog, class OffT>
__global__ void __launch_bounds__(kBlock) k_s_gather_apply(const __grid_constant__ Part<OffT> P, uint32_t v0,
                                                           uint32_t v1, uint32_t shard, uint8_t *changed_flags,
                                                           uint32_t *cstamp, const uint64_t *bounds,
                                                           uint32_t nshards) {
  using G = typename Prog::GatherT;
  Ctl *ctl = P.ctl;
  __shared__ View V;
  load_view(ctl, V);
  const uint32_t t = V.t;
  const Ctx cx = make_ctx(P, V);
  const bool implicit = V.implicit0 && t == 0;
  const uint32_t epoch_t = V.epoch_base + t;
  __shared__ uint32_t sq[kWarpsPerBlock][2][kQueueCap];
  __shared__ G sred[kWarpsPerBlock][32];
  __shared__ int s_any;
  if (threadIdx.x == 0) s_any = 0;
  __syncthreads();
  const uint32_t warp = threadIdx.x / 32, lane = lane_id();
  WarpQueue qC{sq[warp][0], sq[warp][1], 0};
  unsigned long long my_g = 0, my_c = 0;
  const uint32_t gw = blockIdx.x * kWarpsPerBlock + warp, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = v0 + gw * 32u; base < v1; base += nw * 32u) {
    const uint32_t v = base + lane;
    bool valid = v < v1;
    const uint32_t lv = v - P.own_lo;
    if (valid && !implicit) valid = (P.stamp[lv] == epoch_t);
    uint64_t beg = 0;
    uint32_t deg = 0, cur = 0;
    if (valid) {
      beg = (uint64_t)P.in_off[lv];
      deg = (uint32_t)((uint64_t)P.in_off[lv + 1] - beg);
      cur = P.val[v];
    }
    bool unused;
    const G acc = gather_warp<Prog, false>(P, valid, beg, deg, cur, sred[warp], cx, nullptr, unused);
    bool changed = false;
    uint32_t nv = cur;
    if (valid) {
      changed = Prog::apply(&nv, acc, cx);
      my_g += deg;
      if (changed) {
        cstamp[lv] = epoch_t;
        if (shard == kAllShards) changed_flags[shard_of(bounds, nshards, v)] = 1;
      }
    }
    qC.push(changed, v, nv, P.C_v, P.C_val, &ctl->cnt_C);
    my_c += changed ? 1 : 0;
  }
  qC.flush(P.C_v, P.C_val, &ctl->cnt_C);
  my_g = warp_sum_u64(my_g);
  my_c = warp_sum_u64(my_c);
  if (lane == 0) {
    if (my_g) atomicAdd(&ctl->gathered, my_g);
    if (my_c) { atomicAdd(&ctl->changed, my_c); s_any = 1; }
  }
  __syncthreads();
  if (threadIdx.x == 0 && s_any && shard != kAllShards) changed_flags[shard] = 1;
}

// BSP commit of superstep t: val[u] = new for u in C_t.
template <class OffT> __global__ void k_s_commit(const __grid_constant__ Part<OffT> P) {
  const uint32_t nC = P.ctl->cnt_C;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < nC; i += gridDim.x * blockDim.x)
    P.val[P.C_v[i]] = P.C_val[i];
}

// BFS apply over the active vertices of one shard (no edges needed, so no copy):
// depth = t for unvisited members of A_t (L276). Streamed mode keeps apply and
// FrontierActivate as separate passes because A_t membership lives in the
// stamps that the activation of superstep t overwrites.
template <class OffT>
__global__ void k_s_bfs_apply(const __grid_constant__ Part<OffT> P, uint32_t v0, uint32_t v1, uint32_t shard,
                              uint8_t *changed_flags, uint32_t *cstamp) {
  Ctl *ctl = P.ctl;
  const uint32_t t = ctl->iter, epoch_t = ctl->epoch_base + t;
  __shared__ int s_any;
  if (threadIdx.x == 0) s_any = 0;
  __syncthreads();
  unsigned long long my_c = 0;
  for (uint32_t v = v0 + blockIdx.x * blockDim.x + threadIdx.x; v < v1; v += gridDim.x * blockDim.x) {
    const uint32_t lv = v - P.own_lo;
    if (P.stamp[lv] == epoch_t && P.val[v] == kInf) {
      P.val[v] = t;
      cstamp[lv] = epoch_t;
      my_c += 1;
    }
  }
  my_c = warp_sum_u64(my_c);
  if (lane_id() == 0 && my_c) { atomicAdd(&ctl->changed, my_c); s_any = 1; }
  __syncthreads();
  if (threadIdx.x == 0 && s_any) changed_flags[shard] = 1;
}

// FrontierActivate for the changed vertices of one shard (out-edges in a slot).
// kHasScatter programs first run scatter on every expanded edge (values are
// committed by k_s_commit; the edge states live in mapped host memory and
// are updated in place over the host link, P.estate / P.out_eid / P.out_w).
template <class Prog, class OffT>
__global__ void __launch_bounds__(kBlock) k_s_activate(const __grid_constant__ Part<OffT> P, uint32_t u0,
                                                       uint32_t u1, const uint64_t *bounds, uint32_t nshards,
                                                       uint8_t *next_flags, const uint32_t *cstamp) {
  Ctl *ctl = P.ctl;
  const uint32_t t = ctl->iter;
  const uint32_t epoch_t = ctl->epoch_base + t, epoch_n = epoch_t + 1;
  const uint32_t warp_lane = lane_id();
  Ctx cx{};
  cx.iter = t;
  cx.n = P.n;
  cx.source = ctl->source;
  cx.outdeg = P.outdeg;
  unsigned long long my_s = 0, my_act = 0;
  const uint32_t gw = blockIdx.x * kWarpsPerBlock + threadIdx.x / 32, nw = gridDim.x * kWarpsPerBlock;
  for (uint32_t base = u0 + gw * 32u; base < u1; base += nw * 32u) {
    const uint32_t u = base + warp_lane;
    const bool valid = u < u1 && cstamp[u - P.own_lo] == epoch_t;
    uint64_t beg = 0;
    uint32_t deg = 0, uval = 0;
    if (valid) {
      beg = (uint64_t)P.out_off[u];
      deg = (uint32_t)((uint64_t)P.out_off[u + 1] - beg);
      my_s += deg;
      if constexpr (HasScatter<Prog>::value) uval = P.val[u];  // committed value of t
    }
    // expand: stamp targets with epoch t+1; first stamper flags the target's shard
    uint32_t big = __ballot_sync(0xffffffffu, valid && deg > 32);
    auto act_one = [&](bool act, uint32_t x, uint64_t e, uint32_t sv) {
      if constexpr (HasScatter<Prog>::value) {
        if (act) {
          const uint32_t w = Prog::kUsesWeights ? (uint32_t)P.out_w[e] : 0u;
          Prog::scatter(sv, ld_cg(P.val + x), w, P.estate + P.out_eid[e], cx);
        }
      } else {
        (void)e;
        (void)sv;
      }
      bool newly = false;
      if (act) newly = stamp_first(P.stamp + (x - P.own_lo), epoch_n);
      if (newly) next_flags[shard_of(bounds, nshards, x)] = 1;
      return (uint32_t)__popc(__ballot_sync(0xffffffffu, newly));
    };
    while (big) {
      const int L = __ffs(big) - 1;
      big &= big - 1;
      const uint64_t b = __shfl_sync(0xffffffffu, beg, L);
      const uint32_t d = __shfl_sync(0xffffffffu, deg, L);
      const uint32_t sv = __shfl_sync(0xffffffffu, uval, L);
      for (uint32_t r0 = 0; r0 < d; r0 += 32) {
        const uint32_t k = r0 + warp_lane;
        const bool a = k < d;
        my_act += act_one(a, a ? ldg_nc(P.out_dst + b + k) : 0u, b + k, sv);
      }
    }
    const uint32_t sd = (valid && deg <= 32) ? deg : 0u;
    const uint32_t incl = warp_incl_scan(sd), excl = incl - sd;
    const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
    for (uint32_t r0 = 0; r0 < total; r0 += 32) {
      const uint32_t k = r0 + warp_lane;
      int o = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const uint32_t e = __shfl_sync(0xffffffffu, excl, o + step);
        if (e <= k) o += step;
      }
      const uint64_t ob = __shfl_sync(0xffffffffu, beg, o);
      const uint32_t oe = __shfl_sync(0xffffffffu, excl, o);
      const uint32_t sv = __shfl_sync(0xffffffffu, uval, o);
      const bool a = k < total;
      my_act += act_one(a, a ? ldg_nc(P.out_dst + ob + (k - oe)) : 0u, ob + (k - oe), sv);
    }
  }
  my_s = warp_sum_u64(my_s);
  if (warp_lane == 0) {
    if (my_s) atomicAdd(&ctl->scattered, my_s);
    if (my_act) atomicAdd(&ctl->cnt_act[(t + 1) & 1u], (uint32_t)my_act);
  }
}

// Close the superstep (one CTA): the same bookkeeping as the resident path.
template <class OffT> __global__ void k_s_finish(const __grid_constant__ Part<OffT> P) {
  finish_superstep(P, 0ull, 0, kPush);
}

// kHasScatter programs whose source changes at init: it scatters over its out-edges.
template <class Prog, class OffT>
__global__ void k_s_init_scatter(const __grid_constant__ Part<OffT> P, uint32_t source) {
  if constexpr (HasScatter<Prog>::value) {
    Ctx cx{};
    cx.n = P.n;
    cx.source = source;
    cx.outdeg = P.outdeg;
    const uint64_t b = (uint64_t)P.out_off[source], e1 = (uint64_t)P.out_off[source + 1];
    const uint32_t sv = P.val[source];
    for (uint64_t e = b + threadIdx.x; e < e1; e += blockDim.x) {
      const uint32_t x = P.out_dst[e];
      const uint32_t w = Prog::kUsesWeights ? (uint32_t)P.out_w[e] : 0u;
      Prog::scatter(sv, P.val[x], w, P.estate + P.out_eid[e], cx);
    }
  }
}

// Stamp a host-computed starting frontier (SSSP: out-neighbours of the source).
template <class OffT>
__global__ void k_s_stamp_list(const __grid_constant__ Part<OffT> P, const uint32_t *list, uint32_t k) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < k; i += gridDim.x * blockDim.x)
    P.stamp[list[i] - P.own_lo] = P.ctl->epoch_base;
}

}  // namespace gr
