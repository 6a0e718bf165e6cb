// aggregate.cu — vertex-centric GCN aggregation for sm_100a (north_star; P:L72,
// L195, L322).  One kernel family serves the forward (in-CSR) and the backward
// (out-CSR, the exact transpose):
//
//   out[r,:] = scale_row[r] · Σ_{j ∈ row r} scale_col[col[j]] · in[col[j],:] + bias
//
// Work list: the snapshot's schedule (graph.cuh) lists the rows in node_ids
// order (degree-descending presort) as work items of <= 64 edges
// (hub rows are cut into 64-edge chunks).  Three decompositions
// (stg_aggregate_set_strategy; DESIGN.md §Aggregation has the measurements):
//
//  2 (default, W <= 128 per launch) k_agg_stream: a warp takes 32 items
//    at a time from a work queue, scans their edge counts and walks their
//    concatenated edge lists in 32-edge batches, gathering D neighbour rows at
//    once ACROSS row boundaries (lane c holds float4 column c of a row), with
//    the next batch's column ids and the next group's descriptors in flight;
//    hub chunks leave partial sums that k_agg_hubs adds in fixed order.
//  1 k_agg_items: a warp serves 32/G rows at once (feature-adaptive lane
//    groups, the paper's FA-TGA) with a three-stage prefetch across
//    items (descriptor i+2, first column batch of i+1, gathers of i); the last
//    chunk of a hub row to finish sums the chunk partials (atomic ticket).
//  0 k_aggregate: the same lane groups without the schedule prefetch; also the
//    path for caller-built views without a schedule.
//
// Every fp32 chain is <= 64 terms (one accumulator per <= 64-edge item; hub
// partials are summed in blocks of 16 then in a fixed order), there are no
// float atomics, and every result is deterministic run to run (reading C20).
#include <map>
#include <mutex>

#include "graph.cuh"

namespace stg {
namespace {

constexpr int kAggThreads = 256;

struct AggArgs {
  int32_t R;
  const int32_t* rowptr;
  const int32_t* col;
  const int32_t* ids;
  const int32_t* sched;
  const float* srow;
  const float* scol;
  const float* bias;
  int32_t W;  // columns of this launch
  const float* x;
  int64_t ldx;
  float* y;
  int64_t ldy;
  float* partials;  // [chunks][W]
  int32_t* counters;
};

template <int VEC> struct VecT;
template <> struct VecT<4> { using T = float4; };
template <> struct VecT<1> { using T = float; };

__device__ __forceinline__ float4 ldg_v(const float4* p) { return __ldg(p); }
__device__ __forceinline__ float ldg_v(const float* p) { return __ldg(p); }
__device__ __forceinline__ float4 ldcg_v(const float4* p) { return __ldcg(p); }
__device__ __forceinline__ float ldcg_v(const float* p) { return __ldcg(p); }
__device__ __forceinline__ void zero(float4& a) { a = make_float4(0.f, 0.f, 0.f, 0.f); }
__device__ __forceinline__ void zero(float& a) { a = 0.f; }
__device__ __forceinline__ void fma_v(float4& a, float s, const float4& b) {
  a.x = fmaf(s, b.x, a.x); a.y = fmaf(s, b.y, a.y); a.z = fmaf(s, b.z, a.z); a.w = fmaf(s, b.w, a.w);
}
__device__ __forceinline__ void fma_v(float& a, float s, const float& b) { a = fmaf(s, b, a); }
__device__ __forceinline__ void add_v(float4& a, const float4& b) { a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w; }
// Packed fp32x2 adds / fmas (FADD2 / FFMA2, sm_100): two IEEE round-to-nearest
// operations per instruction, bit-identical to the scalar ones.
__device__ __forceinline__ void add2_v(float4& a, const float4& b) {
  unsigned long long a0, a1;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(a0) : "l"(*reinterpret_cast<const unsigned long long*>(&a.x)),
      "l"(*reinterpret_cast<const unsigned long long*>(&b.x)));
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(a1) : "l"(*reinterpret_cast<const unsigned long long*>(&a.z)),
      "l"(*reinterpret_cast<const unsigned long long*>(&b.z)));
  *reinterpret_cast<unsigned long long*>(&a.x) = a0;
  *reinterpret_cast<unsigned long long*>(&a.z) = a1;
}
__device__ __forceinline__ void fma2_v(float4& a, float s, const float4& b) {
  const float2 ss = make_float2(s, s);
  unsigned long long a0, a1;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(a0) : "l"(*reinterpret_cast<const unsigned long long*>(&ss)),
      "l"(*reinterpret_cast<const unsigned long long*>(&b.x)), "l"(*reinterpret_cast<const unsigned long long*>(&a.x)));
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(a1) : "l"(*reinterpret_cast<const unsigned long long*>(&ss)),
      "l"(*reinterpret_cast<const unsigned long long*>(&b.z)), "l"(*reinterpret_cast<const unsigned long long*>(&a.z)));
  *reinterpret_cast<unsigned long long*>(&a.x) = a0;
  *reinterpret_cast<unsigned long long*>(&a.z) = a1;
}
__device__ __forceinline__ void add_v(float& a, const float& b) { a += b; }
__device__ __forceinline__ float4 scale_bias(float s, const float4& a, const float* bias, int c0) {
  float4 r;
  r.x = s * a.x; r.y = s * a.y; r.z = s * a.z; r.w = s * a.w;
  if (bias) { r.x += bias[c0]; r.y += bias[c0 + 1]; r.z += bias[c0 + 2]; r.w += bias[c0 + 3]; }
  return r;
}
__device__ __forceinline__ float scale_bias(float s, const float& a, const float* bias, int c0) {
  float r = s * a;
  if (bias) r += bias[c0];
  return r;
}

template <int VEC, int G, int VPL, int U, bool SCOL>
__global__ void __launch_bounds__(kAggThreads) k_aggregate(const AggArgs a) {
  using VT = typename VecT<VEC>::T;
  constexpr int NG = 32 / G;                  // row groups per warp
  constexpr int IPL = U > G ? U / G : 1;       // column indices per lane per batch
  constexpr int B = G * IPL;                   // edges per batch (multiple of U)
  static_assert(B % U == 0, "batch must be a multiple of U");
  const unsigned FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const int gi = lane / G, gl = lane % G;
  const int32_t n_hub = a.sched ? a.sched[0] : 0;
  const int32_t n_chunks = a.sched ? a.sched[1] : 0;
  const int32_t* cptr = a.sched ? a.sched + a.sched[2] : nullptr;
  const int64_t total = (int64_t)n_chunks + (a.R - n_hub);
  const int64_t warp_id = ((int64_t)blockIdx.x * kAggThreads + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * kAggThreads) >> 5;

  for (int64_t base = warp_id * NG; base < total; base += nwarps * NG) {
    const int64_t item = base + gi;
    const bool valid = item < total;
    int32_t v = 0, beg = 0, end = 0, hub = -1;
    if (valid) {
      if (item < n_chunks) {
        int32_t lo = 0, hi = n_hub;           // largest h with cptr[h] <= item
        while (lo < hi) {
          int32_t mid = (lo + hi + 1) >> 1;
          if (cptr[mid] <= item) lo = mid; else hi = mid - 1;
        }
        hub = lo;
        v = a.ids[lo];
        int32_t rb = a.rowptr[v], re = a.rowptr[v + 1];
        beg = rb + (int32_t)(item - cptr[lo]) * kHubChunk;
        end = min(beg + kHubChunk, re);
      } else {
        int64_t li = n_hub + (item - n_chunks);
        v = a.ids ? a.ids[li] : (int32_t)li;
        beg = a.rowptr[v];
        end = a.rowptr[v + 1];
      }
    }
    const int32_t n = end - beg;
    const int32_t nmax = __reduce_max_sync(FULL, n);

    VT acc[U][VPL];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int c = 0; c < VPL; ++c) zero(acc[u][c]);

    for (int32_t e0 = 0; e0 < nmax; e0 += B) {
      int32_t idx[IPL];
      float sc[IPL];
#pragma unroll
      for (int q = 0; q < IPL; ++q) {
        int32_t e = e0 + q * G + gl;
        idx[q] = e < n ? __ldg(a.col + beg + e) : -1;
        sc[q] = (SCOL && idx[q] >= 0) ? __ldg(a.scol + idx[q]) : 1.0f;
      }
#pragma unroll
      for (int k = 0; k < B; k += U) {
        VT val[U][VPL];
        float ss[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int j = k + u;
          const int src = gi * G + (j % G);
          const int32_t uu = __shfl_sync(FULL, idx[j / G], src);
          ss[u] = SCOL ? __shfl_sync(FULL, sc[j / G], src) : 1.0f;
          const VT* xr = reinterpret_cast<const VT*>(a.x + (int64_t)(uu < 0 ? 0 : uu) * a.ldx);
#pragma unroll
          for (int c = 0; c < VPL; ++c) {
            const int cv = c * G + gl;
            if (uu >= 0 && cv * VEC < a.W) val[u][c] = ldg_v(xr + cv);
            else zero(val[u][c]);
          }
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int c = 0; c < VPL; ++c) {
            if (SCOL) fma_v(acc[u][c], ss[u], val[u][c]);
            else add_v(acc[u][c], val[u][c]);
          }
      }
    }
    // pairwise combine of the U accumulators
#pragma unroll
    for (int w = 1; w < U; w <<= 1)
#pragma unroll
      for (int u = 0; u < U; u += 2 * w)
#pragma unroll
        for (int c = 0; c < VPL; ++c) add_v(acc[u][c], acc[u + w][c]);

    const bool hubitem = valid && hub >= 0;
    if (valid && !hubitem) {
      const float s = a.srow ? a.srow[v] : 1.0f;
      VT* yr = reinterpret_cast<VT*>(a.y + (int64_t)v * a.ldy);
#pragma unroll
      for (int c = 0; c < VPL; ++c) {
        const int cv = c * G + gl;
        if (cv * VEC < a.W) yr[cv] = scale_bias(s, acc[0][c], a.bias, cv * VEC);
      }
    }
    if (hubitem) {
      VT* pr = reinterpret_cast<VT*>(a.partials + item * (int64_t)a.W);
#pragma unroll
      for (int c = 0; c < VPL; ++c) {
        const int cv = c * G + gl;
        if (cv * VEC < a.W) pr[cv] = acc[0][c];
      }
      __threadfence();
    }
    __syncwarp();
    int32_t ticket = 0;
    if (hubitem && gl == 0) ticket = atomicAdd(a.counters + hub, 1);
    ticket = __shfl_sync(FULL, ticket, gi * G);
    const bool last = hubitem && ticket == (cptr[hub + 1] - cptr[hub]) - 1;
    if (last) {
      __threadfence();
      const int32_t cb = cptr[hub], ce = cptr[hub + 1];
      VT tot[VPL];
#pragma unroll
      for (int c = 0; c < VPL; ++c) zero(tot[c]);
      for (int32_t c0 = cb; c0 < ce; c0 += 16) {      // two-level fixed-order sum
        VT blk[VPL];
#pragma unroll
        for (int c = 0; c < VPL; ++c) zero(blk[c]);
        const int32_t c1 = min(c0 + 16, ce);
        for (int32_t ch = c0; ch < c1; ++ch) {
          const VT* pr = reinterpret_cast<const VT*>(a.partials + (int64_t)ch * a.W);
#pragma unroll
          for (int c = 0; c < VPL; ++c) {
            const int cv = c * G + gl;
            if (cv * VEC < a.W) add_v(blk[c], ldcg_v(pr + cv));
          }
        }
#pragma unroll
        for (int c = 0; c < VPL; ++c) add_v(tot[c], blk[c]);
      }
      const float s = a.srow ? a.srow[v] : 1.0f;
      VT* yr = reinterpret_cast<VT*>(a.y + (int64_t)v * a.ldy);
#pragma unroll
      for (int c = 0; c < VPL; ++c) {
        const int cv = c * G + gl;
        if (cv * VEC < a.W) yr[cv] = scale_bias(s, tot[c], a.bias, cv * VEC);
      }
      if (gl == 0) a.counters[hub] = 0;             // self-reset for the next call
    }
  }
}


// ---------------------------------------------------------------------------
// Arguments of the schedule-driven kernels (strategies 1 and 2).
struct Agg2Args {
  const int32_t* sched;
  const int32_t* col;
  const float* srow;
  const float* scol;
  const float* bias;
  int32_t W;
  const float* x;
  int64_t ldx;
  float* y;
  int64_t ldy;
  float* partials;
  int32_t* counters;
  int32_t upad;     // a valid column id for the padding gathers past the stream end
  int32_t hgrp;     // edge stream: hub-chunk items per work group (<= 32)
  int32_t lgrp;     // edge stream: light-row items per work group (<= 32)
  // column chunks run side by side (blockIdx.y = chunk): chunk k covers columns
  // [k·wsplit, min((k+1)·wsplit, wtotal)) and its hub partials start at k·pstride
  int32_t wsplit, wtotal;
  int64_t pstride;
  // sharded mode (stg_gcn_aggregate_peer): source row u lives in block k with
  // pbnd[k] <= u < pbnd[k+1] (pbnd[k] = INT_MAX past the last block), at
  // pbase[k] + u·ldx (the block base shifted back by pbnd[k] rows)
  const float* pbase[STG_MAX_PEERS];
  int32_t pbnd[STG_MAX_PEERS];
  // edge weights (stg_gcn_aggregate_weighted): the weight of
  // the edge at CSR position e is ew[eid ? eid[e] : e] (ew in in-CSR order, the
  // shared edge labels P:L197; the out-CSR reaches it through out_eid).  Only the
  // SCOL instantiation reads them.
  const float* ew;
  const int32_t* eid;
};

// Strategy 1: software-pipelined degree-ordered items.  A warp serves 32/G
// items at once (G lanes × VPL float4 per row) and runs a three-stage pipeline
// across its items: item i+2's descriptor and item i+1's first column batch
// are loaded while item i's neighbour rows are gathered; inside an item the
// next column batch is loaded while the current one is gathered.
template <int G, int VPL, int BT, bool SCOL>
__global__ void __launch_bounds__(kAggThreads, 4) k_agg_items(const Agg2Args a) {
  constexpr int NG = 32 / G;
  static_assert(BT <= G && G % BT == 0, "BT must divide G");
  const unsigned FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31, gi = lane / G, gl = lane % G;
  const int64_t total = a.sched[3];
  const int32_t* cptr = a.sched + a.sched[2];
  const int4* items = reinterpret_cast<const int4*>(a.sched + kSchedHdr);
  const int64_t warp_id = ((int64_t)blockIdx.x * kAggThreads + threadIdx.x) >> 5;
  const int64_t stride = (((int64_t)gridDim.x * kAggThreads) >> 5) * NG;
  const int nv = a.W >> 2;
  const float4 z4 = make_float4(0.f, 0.f, 0.f, 0.f);

  int64_t item = warp_id * NG + gi;
  int4 m0 = item < total ? __ldcs(items + item) : make_int4(0, 0, 0, -2);
  int4 m1 = item + stride < total ? __ldcs(items + item + stride) : make_int4(0, 0, 0, -2);
  int32_t idx0 = gl < m0.z ? __ldcs(a.col + m0.y + gl) : -1;
  float s0 = (a.srow && m0.w > -2) ? __ldg(a.srow + m0.x) : 1.0f;

  for (int64_t base = warp_id * NG; base < total; base += stride, item += stride) {
    // stage 1: descriptor of item i+2; stage 2: first column batch (+ row scale) of item i+1
    const int64_t i2 = item + 2 * stride;
    const int4 m2 = i2 < total ? __ldcs(items + i2) : make_int4(0, 0, 0, -2);
    const int32_t idx1 = gl < m1.z ? __ldcs(a.col + m1.y + gl) : -1;
    const float s1 = (a.srow && m1.w > -2) ? __ldg(a.srow + m1.x) : 1.0f;
    // stage 3: gather item i
    const int32_t n = m0.z;
    const int32_t nmax = __reduce_max_sync(FULL, n);
    float4 acc[VPL];
#pragma unroll
    for (int c = 0; c < VPL; ++c) acc[c] = z4;
    int32_t cur = idx0;
    for (int32_t e0 = 0; e0 < nmax; e0 += G) {
      const int32_t en = e0 + G + gl;
      const int32_t nxt = en < n ? __ldcs(a.col + m0.y + en) : -1;
      const float sc = (SCOL && cur >= 0) ? __ldg(a.scol + cur) : 1.0f;
      const int32_t jn = nmax - e0;             // warp-uniform
#pragma unroll
      for (int j0 = 0; j0 < G; j0 += BT) {
        if (j0 < jn) {
          float4 val[BT][VPL];
          float ss[BT];
#pragma unroll
          for (int b = 0; b < BT; ++b) {
            const int32_t uf = __shfl_sync(FULL, cur, gi * G + j0 + b);
            ss[b] = SCOL ? __shfl_sync(FULL, sc, gi * G + j0 + b) : 1.0f;
            const bool ok = uf >= 0;
            const float4* xr = reinterpret_cast<const float4*>(a.x + (int64_t)(ok ? uf : 0) * a.ldx);
#pragma unroll
            for (int c = 0; c < VPL; ++c) {
              const int cv = c * G + gl;
              val[b][c] = (ok && cv < nv) ? __ldg(xr + cv) : z4;
            }
          }
#pragma unroll
          for (int b = 0; b < BT; ++b)
#pragma unroll
            for (int c = 0; c < VPL; ++c) {
              if (SCOL) fma_v(acc[c], ss[b], val[b][c]);
              else add_v(acc[c], val[b][c]);
            }
        }
      }
      cur = nxt;
    }
    const bool valid = m0.w > -2;
    const int32_t hub = m0.w;
    const int32_t v = m0.x;
    if (valid && hub < 0) {
      float4* yr = reinterpret_cast<float4*>(a.y + (int64_t)v * a.ldy);
#pragma unroll
      for (int c = 0; c < VPL; ++c) {
        const int cv = c * G + gl;
        if (cv < nv) __stcs(yr + cv, scale_bias(s0, acc[c], a.bias, cv * 4));
      }
    }
    const bool hubitem = valid && hub >= 0;
    if (hubitem) {
      float4* pr = reinterpret_cast<float4*>(a.partials + item * (int64_t)a.W);
#pragma unroll
      for (int c = 0; c < VPL; ++c) {
        const int cv = c * G + gl;
        if (cv < nv) pr[cv] = acc[c];
      }
      __threadfence();
    }
    __syncwarp();
    if (__any_sync(FULL, hubitem)) {
      int32_t ticket = 0;
      if (hubitem && gl == 0) ticket = atomicAdd(a.counters + hub, 1);
      ticket = __shfl_sync(FULL, ticket, gi * G);
      const bool last = hubitem && ticket == (cptr[hub + 1] - cptr[hub]) - 1;
      if (last) {
        __threadfence();
        const int32_t cb = cptr[hub], ce = cptr[hub + 1];
        float4 tot[VPL];
#pragma unroll
        for (int c = 0; c < VPL; ++c) tot[c] = z4;
        for (int32_t q0 = cb; q0 < ce; q0 += 16) {      // two-level fixed-order sum
          float4 blk[VPL];
#pragma unroll
          for (int c = 0; c < VPL; ++c) blk[c] = z4;
          const int32_t q1 = min(q0 + 16, ce);
          for (int32_t q = q0; q < q1; ++q) {
            const float4* pr = reinterpret_cast<const float4*>(a.partials + (int64_t)q * a.W);
#pragma unroll
            for (int c = 0; c < VPL; ++c) {
              const int cv = c * G + gl;
              if (cv < nv) add_v(blk[c], __ldcg(pr + cv));
            }
          }
#pragma unroll
          for (int c = 0; c < VPL; ++c) add_v(tot[c], blk[c]);
        }
        float4* yr = reinterpret_cast<float4*>(a.y + (int64_t)v * a.ldy);
#pragma unroll
        for (int c = 0; c < VPL; ++c) {
          const int cv = c * G + gl;
          if (cv < nv) __stcs(yr + cv, scale_bias(s0, tot[c], a.bias, cv * 4));
        }
        if (gl == 0) a.counters[hub] = 0;             // self-reset for the next call
      }
    }
    m0 = m1; m1 = m2; idx0 = idx1; s0 = s1;
  }
}

// ---------------------------------------------------------------------------
// Strategy 2: edge stream over groups of 32 work items (16 < W/4 <= 32 float4
// per launch).  A warp claims the next group of 32 consecutive schedule items
// from a global queue (largest first: hub chunks lead the schedule), scans
// their edge counts and walks the concatenated edge list in batches of 32
// positions: lane l resolves position b·32+l to (item, column id) by a 5-step
// binary search over the scan (shared memory), and the warp gathers D
// neighbour rows at a time (lane c holds float4 column c of the row)
// REGARDLESS of item boundaries, so short rows do not serialise on latency.
// The next batch's column ids and the next group's descriptors (cp.async into
// shared memory) are in flight while the current batch is gathered.  An item's
// sum is flushed when the stream crosses into the next item: light rows are
// written (s_v·Σ + bias), hub chunks store their partial for k_agg_hubs.
// Hub rows of k_agg_stream: every chunk item stored its partial sum (unscaled) at
// partials[item].  One CTA per hub row (grid-stride over the hub rows, which
// lead node_ids: largest first): warp w sums chunk blocks w, w+8, ... (16
// chunk partials per block, loaded together, added in chunk order) into
// shared memory, then a fixed pairwise tree over the blocks gives the row sum
// (deterministic: the tree shape depends only on the chunk count), written as
// y[v] = s_v·Σ + bias.  Rows with more than 64 blocks run in rounds of 64.
constexpr int kHubBlk = 16, kHubRound = 64;
constexpr int kHubGroup = 8;     // hub-chunk items per edge-stream work group (at most)
__global__ void __launch_bounds__(256) k_agg_hubs(const Agg2Args a, const int32_t* __restrict__ ids) {
  __shared__ float4 blk[kHubRound][32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int32_t n_hub = a.sched[0];
  const int32_t* cptr = a.sched + a.sched[2];
  const float4 z4 = make_float4(0.f, 0.f, 0.f, 0.f);
  const int c0y = blockIdx.y * a.wsplit;                       // this launch's column chunk
  const int Wl = min(a.wsplit, a.wtotal - c0y);
  float* const ybase = a.y + c0y;
  const float* const bbase = a.bias ? a.bias + c0y : nullptr;
  const float* const pbase = a.partials + (int64_t)blockIdx.y * a.pstride;
  const int nv = Wl >> 2;
  const int c = lane < nv ? lane : nv - 1;
  // big hubs (more than one block of chunks) lead the schedule: n_big = first h
  // with cptr[h+1] - cptr[h] <= kHubBlk (chunk counts are non-increasing)
  int32_t lo = 0, hi = n_hub;
  while (lo < hi) {
    const int32_t mid = (lo + hi) >> 1;
    if (cptr[mid + 1] - cptr[mid] > kHubBlk) lo = mid + 1; else hi = mid;
  }
  const int32_t n_big = lo;
  // (1) big hubs: one CTA each, blocks of 16 chunk partials per warp, fixed tree
  for (int32_t h = blockIdx.x; h < n_big; h += gridDim.x) {
    const int32_t cb = cptr[h], ce = cptr[h + 1], v = ids[h];
    const int32_t nblk = (ce - cb + kHubBlk - 1) / kHubBlk;
    float4 tot = z4;
    for (int32_t r0 = 0; r0 < nblk; r0 += kHubRound) {
      const int nr = min(kHubRound, nblk - r0);
      for (int b = warp; b < nr; b += 8) {
        const int32_t q0 = cb + (r0 + b) * kHubBlk, q1 = min(q0 + kHubBlk, ce);
        float4 p[kHubBlk];
#pragma unroll
        for (int i = 0; i < kHubBlk; ++i)
          p[i] = q0 + i < q1 ? __ldcg(reinterpret_cast<const float4*>(pbase + (int64_t)(q0 + i) * Wl) + c) : z4;
        float4 sb = p[0];
#pragma unroll
        for (int i = 1; i < kHubBlk; ++i) add_v(sb, p[i]);
        blk[b][lane] = sb;
      }
      __syncthreads();
      for (int st = 1; st < nr; st <<= 1) {            // fixed pairwise tree over the blocks
        for (int e = threadIdx.x; e < nr * 32; e += 256) {
          const int b = e >> 5, l = e & 31;
          if ((b % (2 * st)) == 0 && b + st < nr) add_v(blk[b][l], blk[b + st][l]);
        }
        __syncthreads();
      }
      if (warp == 0) add_v(tot, blk[0][lane]);
      __syncthreads();
    }
    if (warp == 0 && lane < nv) {
      const float sv = a.srow ? a.srow[v] : 1.0f;
      __stcs(reinterpret_cast<float4*>(ybase + (int64_t)v * a.ldy) + lane, scale_bias(sv, tot, bbase, 4 * lane));
    }
  }
  // (2) hubs of <= 16 chunks: one warp each, all chunk partials loaded together
  const int64_t nw = (int64_t)gridDim.x * 8;
  for (int64_t h = n_big + (int64_t)blockIdx.x * 8 + warp; h < n_hub; h += nw) {
    const int32_t cb = cptr[h], ce = cptr[h + 1], v = ids[h];
    float4 p[kHubBlk];
#pragma unroll
    for (int i = 0; i < kHubBlk; ++i)
      p[i] = cb + i < ce ? __ldcg(reinterpret_cast<const float4*>(pbase + (int64_t)(cb + i) * Wl) + c) : z4;
    float4 sb = p[0];
#pragma unroll
    for (int i = 1; i < kHubBlk; ++i) add_v(sb, p[i]);
    if (lane < nv) {
      const float sv = a.srow ? a.srow[v] : 1.0f;
      __stcs(reinterpret_cast<float4*>(ybase + (int64_t)v * a.ldy) + lane, scale_bias(sv, sb, bbase, 4 * lane));
    }
  }
}

template <int D, int MINB, bool SCOL, bool PEER>
__global__ void __launch_bounds__(kAggThreads, MINB) k_agg_stream(const Agg2Args a, uint32_t* __restrict__ queue) {
  constexpr int NW = kAggThreads / 32;
  __shared__ __align__(16) int4 s_items[NW][2][32];
  __shared__ int32_t s_excl[NW][32], s_v[NW][32], s_beg[NW][32], s_hub[NW][32];
  __shared__ const float* s_pbase[STG_MAX_PEERS];
  __shared__ int32_t s_pbnd[STG_MAX_PEERS];
  const unsigned FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (PEER) {
    if (threadIdx.x < STG_MAX_PEERS) {
      s_pbase[threadIdx.x] = a.pbase[threadIdx.x];
      s_pbnd[threadIdx.x] = a.pbnd[threadIdx.x];
    }
    __syncthreads();
  }
  const int64_t total = a.sched[3];
  const int4* items = reinterpret_cast<const int4*>(a.sched + kSchedHdr);
  // Work groups: hub chunks (<= 64 edges each) a.hgrp per group; then the light
  // rows (degree order) in three tiers — n > kTierB: 4 per group, n > kTierC: 16,
  // the rest a.lgrp (host-chosen so that small graphs still spread over many
  // warps) — so no warp walks a long group of the heaviest light rows while
  // others idle (<= 256 edges per group outside the hubs).
  const int64_t n_chunks = a.sched[1];
  const int64_t tb = a.sched[4], tc = a.sched[5];
  const int64_t hg = a.hgrp, lg = a.lgrp;
  constexpr int64_t ga = 4, gb = 16;
  const int64_t nhg = (n_chunks + hg - 1) / hg;
  const int64_t nga = nhg + (tb - n_chunks + ga - 1) / ga;          // groups before tier B
  const int64_t ngb = nga + (tc - tb + gb - 1) / gb;                // groups before tier C
  const uint32_t ngroups = (uint32_t)(ngb + (total - tc + lg - 1) / lg);
  auto gbase = [&](int64_t g) {
    return g < nhg ? g * hg : (g < nga ? n_chunks + (g - nhg) * ga : (g < ngb ? tb + (g - nga) * gb : tc + (g - ngb) * lg));
  };
  auto gend = [&](int64_t g) {
    return g < nhg ? min((g + 1) * hg, n_chunks)
                   : (g < nga ? min(gbase(g) + ga, tb) : (g < ngb ? min(gbase(g) + gb, tc) : min(gbase(g) + lg, total)));
  };
  const int c0y = blockIdx.y * a.wsplit;                       // this launch's column chunk
  const int Wl = min(a.wsplit, a.wtotal - c0y);
  float* const ybase = a.y + c0y;
  const float* const bbase = a.bias ? a.bias + c0y : nullptr;
  float* const pbase = a.partials + (int64_t)blockIdx.y * a.pstride;
  queue += blockIdx.y;
  const int nv = Wl >> 2;
  const bool lane_on = lane < nv;
  const int lanec = lane_on ? lane : nv - 1;
  const float4* xl = reinterpret_cast<const float4*>(a.x + c0y) + lanec;
  const uint32_t ld4 = (uint32_t)(a.ldx >> 2);
  // sharded mode: the float4 offset of source row u's column chunk in its owner's
  // block (resolved once per edge by the lane that loads the column id)
  auto peer_row = [&](int32_t u) -> unsigned long long {
    int k = 0;
#pragma unroll
    for (int i = 1; i < STG_MAX_PEERS; ++i) k += (u >= s_pbnd[i]) ? 1 : 0;
    return reinterpret_cast<unsigned long long>(reinterpret_cast<const float4*>(s_pbase[k] + c0y) +
                                                (size_t)(uint32_t)u * ld4);
  };
  int32_t* ex = s_excl[w];
  auto fetch = [&](uint32_t g, int buf) {         // cp.async the 32 descriptors of group g
    const int64_t it = gbase(g) + lane;
    const uint32_t dst = (uint32_t)__cvta_generic_to_shared(&s_items[w][buf][lane]);
    const int4* src = items + (it < total ? it : 0);
    const int bytes = (g < ngroups && it < gend(g)) ? 16 : 0;
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(dst), "l"(src), "r"(bytes) : "memory");
    asm volatile("cp.async.commit_group;\n" ::: "memory");
  };
  uint32_t grp = 0;
  if (lane == 0) grp = atomicAdd(queue, 1u);
  grp = __shfl_sync(FULL, grp, 0);
  int buf = 0;
  fetch(grp, 0);
  while (grp < ngroups) {
    const uint32_t g_cur = grp;
    if (lane == 0) grp = atomicAdd(queue, 1u);         // claim + prefetch the next group
    grp = __shfl_sync(FULL, grp, 0);
    fetch(grp, buf ^ 1);
    asm volatile("cp.async.wait_group 1;\n" ::: "memory");
    __syncwarp();
    int4 m = s_items[w][buf][lane];
    buf ^= 1;
    const int64_t ib = gbase(g_cur);
    if (ib + lane >= gend(g_cur)) m = make_int4(0, 0, 0, -2);
    const int32_t nl = m.w > -2 ? m.z : 0;
    int32_t incl = nl;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t t = __shfl_up_sync(FULL, incl, o);
      if (lane >= o) incl += t;
    }
    const int32_t N = __shfl_sync(FULL, incl, 31);
    ex[lane] = incl - nl;
    s_v[w][lane] = m.x;
    s_beg[w][lane] = m.y;
    s_hub[w][lane] = m.w;
    const float sl = (a.srow && m.w > -2) ? __ldg(a.srow + m.x) : 1.0f;
    const unsigned zmask = __ballot_sync(FULL, m.w > -2 && nl == 0);
    __syncwarp();
    for (unsigned zm = zmask; zm; zm &= zm - 1) {      // rows without edges: y = bias
      const int32_t vz = s_v[w][__ffs(zm) - 1];
      if (lane_on)
        __stcs(reinterpret_cast<float4*>(ybase + (int64_t)vz * a.ldy) + lane,
               scale_bias(0.f, make_float4(0.f, 0.f, 0.f, 0.f), bbase, 4 * lane));
    }
    auto resolve = [&](int32_t pos, int32_t& u, int32_t& k, int32_t& e) {
      int32_t lo = 0;
#pragma unroll
      for (int st = 16; st >= 1; st >>= 1)
        if (lo + st <= 31 && ex[lo + st] <= pos) lo += st;
      k = lo;
      e = s_beg[w][lo] + (pos - ex[lo]);
      u = pos < N ? __ldcs(a.col + e) : a.upad;
    };
    auto flush = [&](int c, const float4& sum) {
      const float sv = __shfl_sync(FULL, sl, c);
      const int32_t hub = s_hub[w][c];
      if (lane_on) {
        if (hub < 0)
          __stcs(reinterpret_cast<float4*>(ybase + (int64_t)s_v[w][c] * a.ldy) + lane, scale_bias(sv, sum, bbase, 4 * lane));
        else
          reinterpret_cast<float4*>(pbase + (ib + c) * Wl)[lane] = sum;
      }
    };
    int32_t u0, k0, e0;
    resolve(lane, u0, k0, e0);
    int cur = -1;
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int32_t b0 = 0; b0 < N; b0 += 32) {
      const int32_t nb = min(32, N - b0);
      // item boundaries of this batch: bit j = edge j starts a new item.  The
      // first position past the stream end is a boundary to the dummy item -1,
      // so a partial last step needs no per-edge bounds checks.
      const int32_t kp = __shfl_up_sync(FULL, k0, 1);
      const int32_t kc = lane < nb ? k0 : -1;
      const uint32_t bm = __ballot_sync(FULL, lane <= nb && (lane == 0 ? kc != cur : (lane == nb || kc != kp)));
      float sc = 1.0f;
      if (SCOL && lane < nb) {
        sc = a.scol ? __ldg(a.scol + u0) : 1.0f;
        if (a.ew) sc *= __ldg(a.ew + (a.eid ? __ldg(a.eid + e0) : e0));
      }
      const int32_t uc = u0;
      const unsigned long long ua = PEER ? peer_row(u0) : 0ull;
      if (b0 + 32 < N) resolve(b0 + 32 + lane, u0, k0, e0);  // next batch in flight
      for (int32_t j0 = 0; j0 < nb; j0 += D) {
        float4 v[D];
#pragma unroll
        for (int d = 0; d < D; ++d) {
          if (PEER) {          // NVLink peer (or local) load from the owner's block
            const unsigned long long r = __shfl_sync(FULL, ua, (j0 + d) & 31);
            v[d] = __ldg(reinterpret_cast<const float4*>(r) + lanec);
          } else {
            const uint32_t u = (uint32_t)__shfl_sync(FULL, uc, (j0 + d) & 31);
            v[d] = __ldg(xl + (size_t)u * ld4);
          }
        }
        const uint32_t mseg = (bm >> (j0 & 31)) & (D >= 32 ? 0xffffffffu : ((1u << D) - 1u));
        if (mseg == 0) {                                // warp-uniform: no item starts in this group
#pragma unroll
          for (int d = 0; d < D; ++d) {
            if (SCOL) fma2_v(acc, __shfl_sync(FULL, sc, (j0 + d) & 31), v[d]);
            else add2_v(acc, v[d]);
          }
          continue;
        }
#pragma unroll
        for (int d = 0; d < D; ++d) {
          const float sj = SCOL ? __shfl_sync(FULL, sc, (j0 + d) & 31) : 1.0f;
          if ((mseg >> d) & 1u) {
            if (cur >= 0) flush(cur, acc);
            cur = __shfl_sync(FULL, kc, (j0 + d) & 31);
            if (SCOL) { acc = make_float4(0.f, 0.f, 0.f, 0.f); fma2_v(acc, sj, v[d]); }
            else acc = v[d];
          } else {
            if (SCOL) fma2_v(acc, sj, v[d]);
            else add2_v(acc, v[d]);
          }
        }
      }
    }
    if (cur >= 0) flush(cur, acc);
    __syncwarp();
  }
  asm volatile("cp.async.wait_group 0;\n" ::: "memory");
}

// Weighted GCN normalisation (PyG gcn_norm with edge weights, reading C21 / NEXT-4):
// deg_w[v] = Σ_{j ∈ in-row v} ew[j], norm[v] = deg_w^-1/2 (0 if deg_w <= 0).  One
// warp per row; lane-strided fp64 partial sums and a fixed shuffle tree, so the
// fp32 result is the correctly rounded norm of a (nearly) exact sum, run to run.
__global__ void __launch_bounds__(256) k_weighted_norm(const int32_t* __restrict__ rowptr, int32_t R,
                                                       const float* __restrict__ ew, float* __restrict__ norm) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t v = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < R; v += nw) {
    const int32_t b = rowptr[v], e = rowptr[v + 1];
    double acc = 0.0;
    for (int32_t j = b + lane; j < e; j += 32) acc += (double)__ldg(ew + j);
#pragma unroll
    for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) norm[v] = acc > 0.0 ? (float)(1.0 / sqrt(acc)) : 0.0f;
  }
}

using ItemsFn = void (*)(const Agg2Args);
template <int G, int VPL, bool SCOL>
ItemsFn pick_items_vpl() {
  return k_agg_items<G, VPL, (G >= 4 ? 4 : G), SCOL>;
}
template <int G, bool SCOL>
ItemsFn pick_items_g(int vpl) {
  switch (vpl) {
    case 1: return pick_items_vpl<G, 1, SCOL>();
    case 2: return pick_items_vpl<G, 2, SCOL>();
    case 3: return pick_items_vpl<G, 3, SCOL>();
    default: return pick_items_vpl<G, 4, SCOL>();
  }
}
template <bool SCOL>
ItemsFn pick_items(int g, int vpl) {
  switch (g) {
    case 1: return pick_items_g<1, SCOL>(vpl);
    case 2: return pick_items_g<2, SCOL>(vpl);
    case 4: return pick_items_g<4, SCOL>(vpl);
    case 8: return pick_items_g<8, SCOL>(vpl);
    case 16: return pick_items_g<16, SCOL>(vpl);
    default: return pick_items_g<32, SCOL>(vpl);
  }
}

using StreamFn = void (*)(const Agg2Args, uint32_t*);
StreamFn pick_stream(int d, int minb, bool scol) {
#define STG_STREAM(DD, MB) \
  if (d == DD && minb == MB) return scol ? k_agg_stream<DD, MB, true, false> : k_agg_stream<DD, MB, false, false>;
  STG_STREAM(4, 6) STG_STREAM(8, 4) STG_STREAM(16, 2) STG_STREAM(16, 3)
#undef STG_STREAM
  return scol ? k_agg_stream<16, 3, true, false> : k_agg_stream<16, 3, false, false>;
}
StreamFn pick_stream_peer(bool scol) {
  return scol ? k_agg_stream<16, 3, true, true> : k_agg_stream<16, 3, false, true>;
}

using KernelFn = void (*)(const AggArgs);

template <int VEC, int G, bool SCOL>
KernelFn pick_vpl(int vpl) {
  switch (vpl) {
    case 1: return k_aggregate<VEC, G, 1, 4, SCOL>;
    case 2: return k_aggregate<VEC, G, 2, 4, SCOL>;
    case 3: return k_aggregate<VEC, G, 3, 2, SCOL>;
    default: return k_aggregate<VEC, G, 4, 2, SCOL>;
  }
}

template <int VEC, bool SCOL>
KernelFn pick_g(int g, int vpl) {
  switch (g) {
    case 1: return pick_vpl<VEC, 1, SCOL>(vpl);
    case 2: return pick_vpl<VEC, 2, SCOL>(vpl);
    case 4: return pick_vpl<VEC, 4, SCOL>(vpl);
    case 8: return pick_vpl<VEC, 8, SCOL>(vpl);
    case 16: return pick_vpl<VEC, 16, SCOL>(vpl);
    default: return pick_vpl<VEC, 32, SCOL>(vpl);
  }
}

KernelFn pick(int vec, int g, int vpl, bool scol) {
  if (vec == 4) return scol ? pick_g<4, true>(g, vpl) : pick_g<4, false>(g, vpl);
  return scol ? pick_g<1, true>(g, vpl) : pick_g<1, false>(g, vpl);
}

int max_blocks_for(KernelFn fn) {
  static std::mutex mu;
  static std::map<KernelFn, int> cache;
  std::lock_guard<std::mutex> lk(mu);
  auto it = cache.find(fn);
  if (it != cache.end()) return it->second;
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kAggThreads, 0) != cudaSuccess || per_sm < 1) {
    cudaGetLastError();
    per_sm = 1;
  }
  int b = per_sm * num_sms();
  cache[fn] = b;
  return b;
}

}  // namespace

// Work decomposition (stg_aggregate_set_strategy) and strategy-2 tunables.
static int g_strategy = 2;
struct AggTune {
  // rows in flight per warp and min resident blocks per SM (register budget) of the
  // stream kernel: with the light-row tiers balancing the groups, 48 warps x 4 rows beat
  // 24 x 16 (C5 W = 96: 0.443 vs 0.477 ms; W = 64: 0.357 vs 0.418 ms)
  int d = 4;
  int minb = 6;
  // stream kernel for wmin < W_launch <= 128: it beats the row items at every width
  // on C5 (scripts/agg_width_probe.py: W = 16 0.353 vs 0.452 ms, 32 0.364 vs 0.561, 64 0.392 vs 0.756)
  int wmin = 0;
};
static AggTune g_tune;

static int occupancy_grid(const void* fn) {
  static std::mutex mu;
  static std::map<const void*, int> cache;
  std::lock_guard<std::mutex> lk(mu);
  auto it = cache.find(fn);
  if (it != cache.end()) return it->second;
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kAggThreads, 0) != cudaSuccess || per_sm < 1) {
    cudaGetLastError();
    per_sm = 1;
  }
  return cache[fn] = per_sm * num_sms();
}

// lane-group size G and float4 per lane for nv float4 columns (vpl_max float4 per lane)
static void lane_groups(int nv, int vpl_max, int* g, int* vpl) {
  int gg = 1;
  while (gg < 32 && gg * vpl_max < nv) gg <<= 1;
  *g = gg;
  *vpl = (nv + gg - 1) / gg;
}

// Sharded mode (stg_gcn_aggregate_peer): the source rows come from the owners'
// blocks of `peers` (in / ldin are ignored); only the edge-stream kernel serves it.
stg_status aggregate_launch(const stg_csr_view* gv, int backward, int32_t W, const float* in, int64_t ldin,
                            float* out, int64_t ldout, const float* srow, const float* scol, const float* bias,
                            cudaStream_t s, const stg_peer_rows* peers, const float* ew) {
  if (!gv) return fail(STG_ERR_INVALID_ARG, "aggregate: view is NULL");
  if (ew && backward && !gv->out_eid)
    return fail(STG_ERR_INVALID_ARG, "aggregate_weighted: the backward needs the edge labels (STG_EDGE_IDS)");
  if (W < 1) return fail(STG_ERR_INVALID_ARG, "aggregate: W=%d < 1", W);
  int32_t peer_pad = 0;
  if (peers) {
    if (backward) return fail(STG_ERR_INVALID_ARG, "aggregate_peer: forward direction only");
    if (peers->world < 1 || peers->world > STG_MAX_PEERS || !peers->bounds || !peers->blocks)
      return fail(STG_ERR_INVALID_ARG, "aggregate_peer: world must be in [1,%d] with bounds and blocks", STG_MAX_PEERS);
    if (W % 4 || W > 512 || peers->ld < W || peers->ld % 4)
      return fail(STG_ERR_INVALID_ARG, "aggregate_peer: need W %% 4 == 0, W <= 512, ld >= W, ld %% 4 == 0");
    const int32_t* bd = peers->bounds;
    if (bd[0] != 0 || bd[peers->world] != gv->num_nodes)
      return fail(STG_ERR_INVALID_ARG, "aggregate_peer: bounds must span [0, V=%d)", gv->num_nodes);
    peer_pad = -1;
    for (int k = 0; k < peers->world; ++k) {
      if (bd[k + 1] < bd[k]) return fail(STG_ERR_INVALID_ARG, "aggregate_peer: bounds decrease at %d", k);
      if (bd[k + 1] > bd[k]) {
        if (!peers->blocks[k] || (uintptr_t)peers->blocks[k] % 16)
          return fail(STG_ERR_INVALID_ARG, "aggregate_peer: block %d is NULL or not 16-byte aligned", k);
        if (peer_pad < 0) peer_pad = bd[k];
      }
    }
    if (peer_pad < 0) peer_pad = 0;
    if (!gv->in_sched || !gv->in_ids || !gv->workspace)
      return fail(STG_ERR_INVALID_ARG, "aggregate_peer: the view lacks the library schedule");
    in = peers->blocks[0] ? peers->blocks[0] : reinterpret_cast<const float*>(16);   // alignment checks only
    ldin = peers->ld;
  }
  if (ldin < W || ldout < W) return fail(STG_ERR_INVALID_ARG, "aggregate: leading dimension < W");
  const int32_t R = backward ? gv->num_nodes : gv->row_end - gv->row_begin;
  if (R <= 0) return STG_OK;                     // an empty row block: nothing to write
  if (!in || !out) return fail(STG_ERR_INVALID_ARG, "aggregate: NULL input/output");
  AggArgs a{};
  a.R = R;
  a.rowptr = backward ? gv->out_rowptr : gv->in_rowptr;
  a.col = backward ? gv->out_col : gv->in_col;
  a.ids = backward ? gv->out_ids : gv->in_ids;
  a.sched = backward ? gv->out_sched : gv->in_sched;
  if (!a.rowptr || (gv->num_edges > 0 && !a.col))
    return fail(STG_ERR_INVALID_ARG, "aggregate: view lacks the %s CSR", backward ? "backward" : "forward");
  if (a.sched && (!a.ids || !gv->workspace)) a.sched = nullptr;
  // Sharded views (row block [rb, re)): destination-indexed arrays are local
  // rows (forward: out, scale_row; backward: in, scale_col), everything else is
  // global.  Work items carry global vertex ids, so the local arrays are
  // addressed through bases shifted by -rb rows (the view's in_rowptr is the
  // local suffix of the global row pointer).
  const int64_t rb = gv->row_begin;
  if (rb != 0 && a.ids) {
    if (!backward) {
      a.rowptr -= rb;
      out -= rb * ldout;
      if (srow) srow -= rb;
    } else {
      in -= rb * ldin;
      if (scol) scol -= rb;
    }
  }
  a.srow = srow;
  a.scol = scol;
  a.bias = bias;
  const bool vec4 = (W % 4 == 0) && (ldin % 4 == 0) && (ldout % 4 == 0) &&
                    ((uintptr_t)in % 16 == 0) && ((uintptr_t)out % 16 == 0);
  // column split: launches of <= 512 columns (strategies 0/1) or <= 128 (strategy 2)
  const int32_t cmax = vec4 ? 512 : 128;
  // hub chunks: <= E/64 full chunks plus one partial chunk per hub row (<= sched_cap(E) hub rows)
  const int64_t chunks_bound = a.sched ? (gv->num_edges / kHubChunk) + sched_cap(gv->num_edges) + 2 : 0;
  AggScratch* ws = gv->workspace ? static_cast<AggWs*>(gv->workspace)->get(s) : nullptr;
  if (a.sched) {
    STG_TRY(ws->partials.alloc((size_t)chunks_bound * std::min(W, cmax) + 4, s));
    const int64_t ncnt = sched_cap(gv->num_edges) + 1;
    if (ws->counters_n < ncnt) {
      STG_TRY(ws->counters.alloc(ncnt, s));
      STG_CUDA(cudaMemsetAsync(ws->counters.p, 0, sizeof(int32_t) * ncnt, s));
      ws->counters_n = ncnt;
    }
    a.partials = ws->partials.p;
    a.counters = ws->counters.p;
  }
  const int64_t items_bound = (int64_t)R + chunks_bound + 1;
  ProfScope prof(backward ? PH_AGG_BWD : PH_AGG_FWD, s);

  // strategy 2: edge stream, in near-equal column chunks of <= 128 columns
  const int nsplit = (int)ceil_div(W, 128);
  const int32_t wsplit = (int32_t)(ceil_div(ceil_div(W, 4), nsplit) * 4);
  if (peers && !(vec4 && a.sched && wsplit <= 128))
    return fail(STG_ERR_INVALID_ARG, "aggregate_peer: output must be 16-byte aligned with ldout %% 4 == 0");
  if (ew && !(vec4 && a.sched && wsplit <= 128))
    return fail(STG_ERR_INVALID_ARG, "aggregate_weighted: needs W %% 4 == 0, W <= 512, 16-byte aligned rows "
                "and a library view (schedule)");
  // below ~1M edges a single-launch-width aggregation is latency-bound and the
  // pipelined row items (strategy 1) finish first (measured at W = 96: C4 0.024 vs
  // 0.036 ms, C2 0.016 vs 0.030 ms); wide (column-chunked) launches keep the stream
  const bool small_narrow = gv->num_edges < (int64_t(1) << 20) && nsplit == 1;
  if (peers || ew ||
      (vec4 && g_strategy == 2 && a.sched && wsplit > 4 * (g_tune.wmin / 4) && wsplit <= 128 && !small_narrow)) {
    STG_TRY(ws->queue.alloc(nsplit, s));
    STG_CUDA(cudaMemsetAsync(ws->queue.p, 0, sizeof(uint32_t) * nsplit, s));
    const int64_t pstride = chunks_bound * wsplit;               // the column chunks run concurrently
    STG_TRY(ws->partials.alloc((size_t)(pstride * nsplit) + 4, s));
    const bool per_edge = scol != nullptr || ew != nullptr;
    const StreamFn fn = peers ? pick_stream_peer(per_edge) : pick_stream(g_tune.d, g_tune.minb, per_edge);
    // group sizes: ~max(256, E / (8 warps x #SM)) edges per group (all 32-item light
    // groups at C5 scale; small graphs get small groups, hence many warps)
    const int64_t target = std::max<int64_t>(256, gv->num_edges / (8 * (int64_t)num_sms()));
    const int64_t avg = std::max<int64_t>(1, gv->num_edges / std::max<int32_t>(1, R));
    int hgrp = kHubGroup, lgrp = 32;
    while (hgrp > 2 && (int64_t)hgrp * kHubChunk > target) hgrp >>= 1;
    while (lgrp > 4 && (int64_t)lgrp * avg > 2 * target) lgrp >>= 1;
    const int64_t ngroups = ceil_div(chunks_bound, hgrp) + ceil_div(R, 4) + 3;       // bound on work groups
    const int64_t blocks = std::min<int64_t>(occupancy_grid((const void*)fn), ceil_div(ngroups, 8) + 1);
    const int32_t* hids = backward ? gv->out_ids : gv->in_ids;
    Agg2Args b{};
    b.sched = a.sched; b.col = a.col; b.srow = srow; b.scol = scol;
    b.partials = ws->partials.p; b.counters = a.counters;
    b.W = wsplit; b.x = in; b.ldx = ldin; b.y = out; b.ldy = ldout;
    b.bias = bias;
    b.upad = (backward && a.ids) ? (int32_t)rb : 0;     // row 0 of a shifted input is not a valid row
    b.hgrp = hgrp; b.lgrp = lgrp;
    b.wsplit = wsplit; b.wtotal = W; b.pstride = pstride;
    b.ew = ew;
    b.eid = (ew && backward) ? gv->out_eid : nullptr;
    for (int k = 0; k < STG_MAX_PEERS; ++k) {
      b.pbnd[k] = INT32_MAX;
      b.pbase[k] = nullptr;
    }
    if (peers) {
      b.upad = peer_pad;
      for (int k = 0; k < peers->world; ++k) {
        b.pbnd[k] = k == 0 ? 0 : peers->bounds[k];
        // block k base shifted back by bounds[k] rows: row u is at pbase[k] + u·ld
        b.pbase[k] = reinterpret_cast<const float*>(reinterpret_cast<uintptr_t>(peers->blocks[k]) -
                                                    (uintptr_t)((int64_t)peers->bounds[k] * peers->ld * 4));
      }
      // empty blocks: never selected (rows of an empty block k belong to the next
      // non-empty block, pbnd is non-decreasing so the count skips them)
    }
    // one launch for all column chunks (gridDim.y): the chunks of a wide W (e.g. a
    // sequence-batched S·3H) walk the graph side by side instead of one after another
    const int64_t bx = nsplit > 1 ? std::max<int64_t>(1, std::min<int64_t>(blocks, ceil_div(occupancy_grid(
                                                                               (const void*)fn), nsplit)))
                                  : blocks;
    fn<<<dim3((unsigned)bx, (unsigned)nsplit), kAggThreads, 0, s>>>(b, ws->queue.p);
    k_agg_hubs<<<dim3((unsigned)std::max(1, 4 * num_sms() / nsplit), (unsigned)nsplit), 256, 0, s>>>(b, hids);
    count_launch(2);
    return check_launch("aggregate_stream");
  }
  // strategy 1: pipelined items
  if (vec4 && g_strategy >= 1 && a.sched) {
    for (int32_t c0 = 0; c0 < W; c0 += cmax) {
      const int32_t wl = std::min(cmax, W - c0);
      int g, vpl;
      lane_groups(wl / 4, 2, &g, &vpl);
      Agg2Args b{};
      b.sched = a.sched; b.col = a.col; b.srow = srow; b.scol = scol;
      b.partials = a.partials; b.counters = a.counters;
      b.W = wl; b.x = in + c0; b.ldx = ldin; b.y = out + c0; b.ldy = ldout;
      b.bias = bias ? bias + c0 : nullptr;
      const ItemsFn fn = scol ? pick_items<true>(g, vpl) : pick_items<false>(g, vpl);
      const int64_t blocks = std::max<int64_t>(
          1, std::min<int64_t>(occupancy_grid((const void*)fn), ceil_div(items_bound, (kAggThreads / 32) * (32 / g))));
      fn<<<(unsigned)blocks, kAggThreads, 0, s>>>(b);
      count_launch();
    }
    return check_launch("aggregate_items");
  }
  // strategy 0: row items with register gathers (any width / alignment, any view)
  for (int32_t c0 = 0; c0 < W; c0 += cmax) {
    const int32_t wl = std::min(cmax, W - c0);
    int g, vpl;
    lane_groups(vec4 ? wl / 4 : wl, 4, &g, &vpl);
    a.W = wl;
    a.x = in + c0;
    a.ldx = ldin;
    a.y = out + c0;
    a.ldy = ldout;
    a.bias = bias ? bias + c0 : nullptr;
    const KernelFn fn = pick(vec4 ? 4 : 1, g, vpl, scol != nullptr);
    const int64_t blocks = std::max<int64_t>(
        1, std::min<int64_t>(max_blocks_for(fn), ceil_div(items_bound, (kAggThreads / 32) * (32 / g))));
    fn<<<(unsigned)blocks, kAggThreads, 0, s>>>(a);
    count_launch();
  }
  return check_launch("aggregate");
}

}  // namespace stg

extern "C" {

stg_status stg_gcn_aggregate_fwd(const stg_csr_view* g, int32_t W, const float* x, int64_t ldx, float* y,
                                 int64_t ldy, stg_stream_t stream) {
  if (!g) return stg::fail(STG_ERR_INVALID_ARG, "stg_gcn_aggregate_fwd: view is NULL");
  return stg::aggregate_launch(g, 0, W, x, ldx, y, ldy, g->norm_dst ? g->norm_dst + g->row_begin : nullptr,
                               g->norm_src, nullptr, (cudaStream_t)stream);
}

stg_status stg_gcn_aggregate_bwd(const stg_csr_view* g, int32_t W, const float* gy, int64_t ldgy, float* gx,
                                 int64_t ldgx, stg_stream_t stream) {
  if (!g) return stg::fail(STG_ERR_INVALID_ARG, "stg_gcn_aggregate_bwd: view is NULL");
  return stg::aggregate_launch(g, 1, W, gy, ldgy, gx, ldgx, g->norm_src,
                               g->norm_dst ? g->norm_dst + g->row_begin : nullptr, nullptr, (cudaStream_t)stream);
}

stg_status stg_gcn_aggregate_peer(const stg_csr_view* g, int32_t W, const stg_peer_rows* x, float* out,
                                  int64_t ldout, const float* scale_row, const float* scale_col, const float* bias,
                                  stg_stream_t stream) {
  if (!x) return stg::fail(STG_ERR_INVALID_ARG, "stg_gcn_aggregate_peer: row table is NULL");
  return stg::aggregate_launch(g, 0, W, nullptr, 0, out, ldout, scale_row, scale_col, bias, (cudaStream_t)stream, x);
}

stg_status stg_gcn_aggregate_weighted(const stg_csr_view* g, int32_t backward, int32_t W, const float* ew,
                                      const float* in, int64_t ldin, float* out, int64_t ldout,
                                      const float* scale_row, const float* scale_col, const float* bias,
                                      stg_stream_t stream) {
  if (!g) return stg::fail(STG_ERR_INVALID_ARG, "stg_gcn_aggregate_weighted: view is NULL");
  if (!ew && g->num_edges > 0) return stg::fail(STG_ERR_INVALID_ARG, "stg_gcn_aggregate_weighted: ew is NULL");
  return stg::aggregate_launch(g, backward, W, in, ldin, out, ldout, scale_row, scale_col, bias, (cudaStream_t)stream,
                               nullptr, ew ? ew : nullptr);
}

stg_status stg_gcn_weighted_norm(const stg_csr_view* g, const float* ew, float* norm, stg_stream_t stream) {
  using stg::fail;
  if (!g || !norm || (!ew && g->num_edges > 0)) return fail(STG_ERR_INVALID_ARG, "stg_gcn_weighted_norm: NULL argument");
  if (!g->in_rowptr) return fail(STG_ERR_INVALID_ARG, "stg_gcn_weighted_norm: view lacks the forward CSR");
  const int32_t R = g->row_end - g->row_begin;
  if (R <= 0) return STG_OK;
  const unsigned blocks = (unsigned)std::min<int64_t>(stg::ceil_div(R, 8), (int64_t)stg::num_sms() * 16);
  stg::k_weighted_norm<<<blocks, 256, 0, (cudaStream_t)stream>>>(g->in_rowptr, R, ew, norm);
  stg::count_launch();
  return stg::check_launch("stg_gcn_weighted_norm");
}

stg_status stg_aggregate_set_strategy(int32_t strategy) {
  if (strategy < 0 || strategy > 2) return stg::fail(STG_ERR_INVALID_ARG, "stg_aggregate_set_strategy: %d", strategy);
  stg::g_strategy = strategy;
  return STG_OK;
}

stg_status stg_aggregate_set_param(int32_t key, int64_t value) {
  switch (key) {
    case 0:
      if (value != 4 && value != 8 && value != 16) break;
      stg::g_tune.d = (int)value;
      return STG_OK;
    case 1:
      if (value < 2 || value > 6) break;
      stg::g_tune.minb = (int)value;
      return STG_OK;
    case 2:
      if (value != 0 && value != 8 && value != 16 && value != 32 && value != 64) break;
      stg::g_tune.wmin = (int)value;
      return STG_OK;

    default:
      break;
  }
  return stg::fail(STG_ERR_INVALID_ARG, "stg_aggregate_set_param: key %d value %lld", key, (long long)value);
}

stg_status stg_gcn_aggregate_ex(const stg_csr_view* g, int32_t backward, int32_t W, const float* in, int64_t ldin,
                                float* out, int64_t ldout, const float* scale_row, const float* scale_col,
                                const float* bias, stg_stream_t stream) {
  return stg::aggregate_launch(g, backward, W, in, ldin, out, ldout, scale_row, scale_col, bias,
                               (cudaStream_t)stream);
}

}  // extern "C"
