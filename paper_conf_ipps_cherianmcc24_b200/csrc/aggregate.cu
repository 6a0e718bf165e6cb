// aggregate.cu — vertex-centric GCN aggregation for sm_100a (north_star; P:L72,
// L195, L322).  One kernel serves the forward (in-CSR) and the backward
// (out-CSR, the exact transpose):
//
//   out[r,:] = scale_row[r] · Σ_{j ∈ row r} scale_col[col[j]] · in[col[j],:] + bias
//
// Design:
//  * feature-adaptive thread groups (the paper's FA-TGA): a row is
//    owned by a group of G lanes; each lane holds VPL 128-bit vectors of the
//    row (G·VPL·4 >= W), so a 32-lane warp works on 32/G rows at once;
//  * rows are taken in node_ids order (degree-descending presort)
//    so the rows sharing a warp have similar degrees;
//  * rows with more than kHubChunk edges are split into fixed chunks of
//    kHubChunk edges (hub items first); the last chunk to finish sums the
//    chunk partials in a fixed order — deterministic, no float atomics;
//  * column indices are loaded coalesced, one per lane, and broadcast with
//    __shfl_sync; feature rows are gathered with 128-bit ld.global.nc;
//  * U independent accumulators per vector bound every sequential fp32 chain
//    to <= 64 terms (reading C19/C20 error bound).
//  * persistent grid of (#SMs × resident blocks), grid-stride over work items.
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
  const int32_t* cptr = a.sched ? a.sched + 2 : nullptr;
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
// Asynchronous-gather variant (float4 path, W <= 128): per warp a double-
// buffered ring of 32 row slots in shared memory.  For each batch the warp
// loads the 32 column indices (one per lane, coalesced), then issues the row
// copies as 16-byte cp.async (LDGSTS, no register destinations) for batch b+1
// while it consumes batch b from shared memory.  Slot s belongs to group
// s / G (the G lanes that own one row item); accumulation order per row is the
// same fixed edge order as k_aggregate, so results are deterministic.
template <int G, int VPL, int U, bool SCOL>
__global__ void __launch_bounds__(kAggThreads) k_aggregate_async(const AggArgs a, int warps_per_block) {
  constexpr int NG = 32 / G;                 // row items per warp
  constexpr int EPG = G;                     // slots (edges) per item per batch
  const unsigned FULL = 0xffffffffu;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  if (wib >= warps_per_block) return;
  const int gi = lane / G, gl = lane % G;
  const int W = a.W, nv = W / 4;             // row length in float4
  const int slot_bytes = W * 4;
  unsigned char* wbase = smem_raw + (size_t)wib * (2 * 32 * slot_bytes + 2 * 32 * 4);
  unsigned char* buf[2] = {wbase, wbase + 32 * slot_bytes};
  float* scs[2] = {reinterpret_cast<float*>(wbase + 2 * 32 * slot_bytes),
                   reinterpret_cast<float*>(wbase + 2 * 32 * slot_bytes) + 32};
  const int32_t n_hub = a.sched ? a.sched[0] : 0;
  const int32_t n_chunks = a.sched ? a.sched[1] : 0;
  const int32_t* cptr = a.sched ? a.sched + 2 : nullptr;
  const int64_t total = (int64_t)n_chunks + (a.R - n_hub);
  const int64_t warp_id = (int64_t)blockIdx.x * warps_per_block + wib;
  const int64_t nwarps = (int64_t)gridDim.x * warps_per_block;

  for (int64_t base = warp_id * NG; base < total; base += nwarps * NG) {
    const int64_t item = base + gi;
    const bool valid = item < total;
    int32_t v = 0, beg = 0, end = 0, hub = -1;
    if (valid) {
      if (item < n_chunks) {
        int32_t lo = 0, hi = n_hub;
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
    const int nb = (nmax + EPG - 1) / EPG;
    // lane s describes slot s: group s / EPG, edge (b·EPG + s % EPG) of that group
    const int sg = lane / EPG, se = lane % EPG;
    const int32_t s_beg = __shfl_sync(FULL, beg, sg * G);
    const int32_t s_n = __shfl_sync(FULL, n, sg * G);

    auto issue = [&](int b, int which) {
      const int e = b * EPG + se;
      const int32_t u = e < s_n ? __ldg(a.col + s_beg + e) : -1;
      if (SCOL) scs[which][lane] = u >= 0 ? __ldg(a.scol + u) : 0.0f;
      const uint32_t dst0 = (uint32_t)__cvta_generic_to_shared(buf[which]);
      for (int p = lane; p < 32 * nv; p += 32) {
        const int slot = p / nv, ch = p - slot * nv;
        const int32_t us = __shfl_sync(FULL, u, slot);
        if (us >= 0) {
          const float* src = a.x + (int64_t)us * a.ldx + 4 * ch;
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(dst0 + (uint32_t)(slot * slot_bytes + 16 * ch)),
                       "l"(src)
                       : "memory");
        }
      }
      asm volatile("cp.async.commit_group;\n" ::: "memory");
    };

    float4 acc[U][VPL];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int c = 0; c < VPL; ++c) acc[u][c] = make_float4(0.f, 0.f, 0.f, 0.f);

    if (nb > 0) issue(0, 0);
    for (int b = 0; b < nb; ++b) {
      if (b + 1 < nb) {
        issue(b + 1, (b + 1) & 1);
        asm volatile("cp.async.wait_group 1;\n" ::: "memory");
      } else {
        asm volatile("cp.async.wait_group 0;\n" ::: "memory");
      }
      __syncwarp();
      const unsigned char* bb = buf[b & 1];
      const float* sc = scs[b & 1];
#pragma unroll
      for (int e = 0; e < EPG; ++e) {
        if (b * EPG + e < n) {
          const int slot = gi * EPG + e;
          const float4* row = reinterpret_cast<const float4*>(bb + slot * slot_bytes);
          const float ssc = SCOL ? sc[slot] : 1.0f;
#pragma unroll
          for (int c = 0; c < VPL; ++c) {
            const int cv = c * G + gl;
            if (cv < nv) {
              const float4 xv = row[cv];
              if (SCOL) fma_v(acc[e % U][c], ssc, xv);
              else add_v(acc[e % U][c], xv);
            }
          }
        }
      }
      __syncwarp();
    }
#pragma unroll
    for (int w = 1; w < U; w <<= 1)
#pragma unroll
      for (int u = 0; u < U; u += 2 * w)
#pragma unroll
        for (int c = 0; c < VPL; ++c) add_v(acc[u][c], acc[u + w][c]);

    const bool hubitem = valid && hub >= 0;
    if (valid && !hubitem) {
      const float s = a.srow ? a.srow[v] : 1.0f;
      float4* yr = reinterpret_cast<float4*>(a.y + (int64_t)v * a.ldy);
#pragma unroll
      for (int c = 0; c < VPL; ++c) {
        const int cv = c * G + gl;
        if (cv < nv) yr[cv] = scale_bias(s, acc[0][c], a.bias, cv * 4);
      }
    }
    if (hubitem) {
      float4* pr = reinterpret_cast<float4*>(a.partials + item * (int64_t)W);
#pragma unroll
      for (int c = 0; c < VPL; ++c) {
        const int cv = c * G + gl;
        if (cv < nv) pr[cv] = acc[0][c];
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
      float4 tot[VPL];
#pragma unroll
      for (int c = 0; c < VPL; ++c) tot[c] = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int32_t c0 = cb; c0 < ce; c0 += 16) {
        float4 blk[VPL];
#pragma unroll
        for (int c = 0; c < VPL; ++c) blk[c] = make_float4(0.f, 0.f, 0.f, 0.f);
        const int32_t c1 = min(c0 + 16, ce);
        for (int32_t ch = c0; ch < c1; ++ch) {
          const float4* pr = reinterpret_cast<const float4*>(a.partials + (int64_t)ch * W);
#pragma unroll
          for (int c = 0; c < VPL; ++c) {
            const int cv = c * G + gl;
            if (cv < nv) add_v(blk[c], __ldcg(pr + cv));
          }
        }
#pragma unroll
        for (int c = 0; c < VPL; ++c) add_v(tot[c], blk[c]);
      }
      const float s = a.srow ? a.srow[v] : 1.0f;
      float4* yr = reinterpret_cast<float4*>(a.y + (int64_t)v * a.ldy);
#pragma unroll
      for (int c = 0; c < VPL; ++c) {
        const int cv = c * G + gl;
        if (cv < nv) yr[cv] = scale_bias(s, tot[c], a.bias, cv * 4);
      }
      if (gl == 0) a.counters[hub] = 0;
    }
  }
}

using AsyncFn = void (*)(const AggArgs, int);

template <int G, bool SCOL>
AsyncFn pick_async_vpl(int vpl) {
  switch (vpl) {
    case 1: return k_aggregate_async<G, 1, 4, SCOL>;
    case 2: return k_aggregate_async<G, 2, 4, SCOL>;
    case 3: return k_aggregate_async<G, 3, 2, SCOL>;
    default: return k_aggregate_async<G, 4, 2, SCOL>;
  }
}
template <bool SCOL>
AsyncFn pick_async_g(int g, int vpl) {
  switch (g) {
    case 1: return pick_async_vpl<1, SCOL>(vpl);
    case 2: return pick_async_vpl<2, SCOL>(vpl);
    case 4: return pick_async_vpl<4, SCOL>(vpl);
    case 8: return pick_async_vpl<8, SCOL>(vpl);
    case 16: return pick_async_vpl<16, SCOL>(vpl);
    default: return pick_async_vpl<32, SCOL>(vpl);
  }
}

// ---------------------------------------------------------------------------
// Edge-parallel ("merge-path") variant for W <= 128 float4 rows: warp w streams
// the contiguous edge chunks c = w, w + nwarps, ... of kEdgeChunk edges.  Column
// and row ids are read 32 at a time (coalesced) and broadcast; 8 feature-row
// gathers are in flight per lane; a row is flushed when the row id changes.
// Rows fully inside a chunk are written directly; a row split across chunks
// [c_a, c_b] leaves one partial per chunk (slot 2c_a+1, then 2c for c > c_a) and
// the last chunk to finish (atomic ticket per row, self-resetting) sums them in
// chunk order.  Two accumulators alternate on edge parity: every fp32 chain is
// <= 64 terms, results are deterministic, no float atomics.
constexpr int kEdgeChunk = 128;

struct EdgeArgs {
  int32_t R;
  int64_t E;
  const int32_t* rowptr;
  const int32_t* col;
  const int32_t* row;
  const float* srow;
  const float* scol;
  const float* bias;
  int32_t W;
  const float* x;
  int64_t ldx;
  float* y;
  int64_t ldy;
  float* partials;   // [2 * nchunks][W]
  int32_t* counters; // [R]
};

__device__ __forceinline__ void edge_write_row(const EdgeArgs& a, int32_t r, float4 v, int lane, int nv) {
  if (lane < nv) {
    const float s = a.srow ? a.srow[r] : 1.0f;
    reinterpret_cast<float4*>(a.y + (int64_t)r * a.ldy)[lane] = scale_bias(s, v, a.bias, 4 * lane);
  }
}

template <bool SCOL>
__global__ void __launch_bounds__(kAggThreads) k_agg_edges(const EdgeArgs a) {
  constexpr int U = 8;
  const unsigned FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const int nv = a.W / 4;
  const int64_t nchunks = (a.E + kEdgeChunk - 1) / kEdgeChunk;
  const int64_t warp_id = ((int64_t)blockIdx.x * kAggThreads + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * kAggThreads) >> 5;
  const float4 z4 = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int64_t c = warp_id; c < nchunks; c += nwarps) {
    const int64_t e0 = c * kEdgeChunk, e1 = (a.E < e0 + kEdgeChunk) ? a.E : e0 + kEdgeChunk;
    const int32_t r_first = a.row[e0], r_last = a.row[e1 - 1];
    const bool start_open = e0 > a.rowptr[r_first];
    const bool end_open = e1 < a.rowptr[r_last + 1];
    // empty rows in the gap before this chunk (and after the last chunk)
    {
      const int32_t gap0 = c == 0 ? 0 : a.row[e0 - 1] + 1;
      for (int32_t r = gap0; r < r_first; ++r) edge_write_row(a, r, z4, lane, nv);
      if (c == nchunks - 1)
        for (int32_t r = r_last + 1; r < a.R; ++r) edge_write_row(a, r, z4, lane, nv);
    }
    int32_t cur = r_first;
    float4 acc0 = z4, acc1 = z4;
    auto flush = [&](int32_t r) {
      float4 v = acc0;
      add_v(v, acc1);
      const bool open_s = (r == r_first) && start_open, open_e = (r == r_last) && end_open;
      if (!open_s && !open_e) {
        edge_write_row(a, r, v, lane, nv);
        return;
      }
      const int64_t slot = open_s ? 2 * c : 2 * c + 1;
      if (lane < nv) reinterpret_cast<float4*>(a.partials + slot * a.W)[lane] = v;
      __threadfence();
      __syncwarp();
      const int64_t rb = a.rowptr[r], re = a.rowptr[r + 1];
      const int64_t ca = rb / kEdgeChunk, cb = (re - 1) / kEdgeChunk;
      int32_t ticket = 0;
      if (lane == 0) ticket = atomicAdd(a.counters + r, 1);
      ticket = __shfl_sync(FULL, ticket, 0);
      if (ticket == (int32_t)(cb - ca)) {       // last chunk of row r to finish
        __threadfence();
        float4 tot = z4;
        for (int64_t q0 = ca; q0 <= cb; q0 += 16) {
          float4 blk = z4;
          const int64_t q1 = (q0 + 16 < cb + 1) ? q0 + 16 : cb + 1;
          for (int64_t q = q0; q < q1; ++q) {
            const int64_t sl = q == ca ? 2 * q + 1 : 2 * q;
            if (lane < nv) add_v(blk, __ldcg(reinterpret_cast<const float4*>(a.partials + sl * a.W) + lane));
          }
          add_v(tot, blk);
        }
        edge_write_row(a, r, tot, lane, nv);
        if (lane == 0) a.counters[r] = 0;
      }
    };
    for (int64_t base = e0; base < e1; base += 32) {
      const int n = (int)((e1 - base) < 32 ? (e1 - base) : 32);
      const int32_t my_col = lane < n ? __ldg(a.col + base + lane) : 0;
      const int32_t my_row = lane < n ? __ldg(a.row + base + lane) : cur;
      const float my_sc = (SCOL && lane < n) ? __ldg(a.scol + my_col) : 1.0f;
      for (int j0 = 0; j0 < n; j0 += U) {
        float4 xv[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int32_t cj = __shfl_sync(FULL, my_col, j0 + u);
          xv[u] = (j0 + u < n && lane < nv) ? __ldg(reinterpret_cast<const float4*>(a.x + (int64_t)cj * a.ldx) + lane)
                                            : z4;
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (j0 + u >= n) break;
          const int32_t rj = __shfl_sync(FULL, my_row, j0 + u);
          const float sj = SCOL ? __shfl_sync(FULL, my_sc, j0 + u) : 1.0f;
          if (rj != cur) {
            flush(cur);
            for (int32_t r = cur + 1; r < rj; ++r) edge_write_row(a, r, z4, lane, nv);
            cur = rj;
            acc0 = z4;
            acc1 = z4;
          }
          if (((base + j0 + u) & 1) == 0) {
            if (SCOL) fma_v(acc0, sj, xv[u]); else add_v(acc0, xv[u]);
          } else {
            if (SCOL) fma_v(acc1, sj, xv[u]); else add_v(acc1, xv[u]);
          }
        }
      }
    }
    flush(cur);
  }
}

// TMA-gather edge-parallel kernel (strategy 2): per warp two 32-slot row
// buffers in shared memory; for every 32-edge batch each lane issues ONE bulk
// copy (cp.async.bulk, the whole W·4-byte feature row) that completes on the
// buffer's mbarrier (expect_tx).  The next batch (possibly of the next chunk)
// is issued before the current one is consumed, so a warp keeps up to 64 rows
// in flight without register destinations.  Accumulation order and the chunk /
// split-row logic are those of k_agg_edges.
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t mbar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(mbar)
               : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t mbar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(mbar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait_parity(uint32_t mbar, uint32_t phase) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "W_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra D_%=;\n\t"
      "bra W_%=;\n"
      "D_%=:\n\t}\n" ::"r"(mbar),
      "r"(phase)
      : "memory");
}

template <bool SCOL>
__global__ void __launch_bounds__(kAggThreads) k_agg_edges_tma(const EdgeArgs a, int warps_per_block) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  __shared__ __align__(8) uint64_t mbars[kAggThreads / 32][2];
  const unsigned FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  if (wib >= warps_per_block) return;
  const int nv = a.W / 4;
  const uint32_t rowb = (uint32_t)a.W * 4;
  unsigned char* wbuf = smem_raw + (size_t)wib * 2 * 32 * rowb;
  const uint32_t sbuf0 = (uint32_t)__cvta_generic_to_shared(wbuf);
  const uint32_t mb0 = (uint32_t)__cvta_generic_to_shared(&mbars[wib][0]);
  const uint32_t mb1 = (uint32_t)__cvta_generic_to_shared(&mbars[wib][1]);
  if (lane == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(mb0) : "memory");
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(mb1) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncwarp();
  const int64_t nchunks = (a.E + kEdgeChunk - 1) / kEdgeChunk;
  const int64_t warp_id = (int64_t)blockIdx.x * warps_per_block + wib;
  const int64_t nwarps = (int64_t)gridDim.x * warps_per_block;
  const float4 z4 = make_float4(0.f, 0.f, 0.f, 0.f);
  uint32_t phase0 = 0, phase1 = 0;
  // batch stream: (chunk c, edge base) in order; issue(k) fills buffer k & 1
  int32_t q_row0 = 0, q_row1 = 0, q_n0 = 0, q_n1 = 0;   // per-buffer batch metadata (no local arrays)
  float q_sc0 = 1.f, q_sc1 = 1.f;
  auto issue = [&](int64_t c, int64_t base, int which) {
    const int64_t e1 = (a.E < c * kEdgeChunk + kEdgeChunk) ? a.E : c * kEdgeChunk + kEdgeChunk;
    const int n = (int)((e1 - base) < 32 ? (e1 - base) : 32);
    int32_t u = 0, rw = 0;
    float sc = 1.0f;
    if (lane < n) {
      u = __ldg(a.col + base + lane);
      rw = __ldg(a.row + base + lane);
      sc = SCOL ? __ldg(a.scol + u) : 1.0f;
    }
    if (which) { q_row1 = rw; q_sc1 = sc; q_n1 = n; } else { q_row0 = rw; q_sc0 = sc; q_n0 = n; }
    const uint32_t mb = which ? mb1 : mb0;
    if (lane == 0) mbar_expect_tx(mb, (uint32_t)n * rowb);
    __syncwarp();
    if (lane < n) bulk_g2s(sbuf0 + (uint32_t)which * 32 * rowb + (uint32_t)lane * rowb, a.x + (int64_t)u * a.ldx, rowb, mb);
  };
  int64_t c = warp_id;
  if (c >= nchunks) return;
  int which = 0;
  issue(c, c * kEdgeChunk, 0);
  for (; c < nchunks; c += nwarps) {
    const int64_t e0 = c * kEdgeChunk, e1 = (a.E < e0 + kEdgeChunk) ? a.E : e0 + kEdgeChunk;
    const int32_t r_first = a.row[e0], r_last = a.row[e1 - 1];
    const bool start_open = e0 > a.rowptr[r_first];
    const bool end_open = e1 < a.rowptr[r_last + 1];
    {
      const int32_t gap0 = c == 0 ? 0 : a.row[e0 - 1] + 1;
      for (int32_t r = gap0; r < r_first; ++r) edge_write_row(a, r, z4, lane, nv);
      if (c == nchunks - 1)
        for (int32_t r = r_last + 1; r < a.R; ++r) edge_write_row(a, r, z4, lane, nv);
    }
    int32_t cur = r_first;
    float4 acc0 = z4, acc1 = z4;
    auto flush = [&](int32_t r) {
      float4 v = acc0;
      add_v(v, acc1);
      const bool open_s = (r == r_first) && start_open, open_e = (r == r_last) && end_open;
      if (!open_s && !open_e) {
        edge_write_row(a, r, v, lane, nv);
        return;
      }
      const int64_t slot = open_s ? 2 * c : 2 * c + 1;
      if (lane < nv) reinterpret_cast<float4*>(a.partials + slot * a.W)[lane] = v;
      __threadfence();
      __syncwarp();
      const int64_t rb = a.rowptr[r], re = a.rowptr[r + 1];
      const int64_t ca = rb / kEdgeChunk, cb = (re - 1) / kEdgeChunk;
      int32_t ticket = 0;
      if (lane == 0) ticket = atomicAdd(a.counters + r, 1);
      ticket = __shfl_sync(FULL, ticket, 0);
      if (ticket == (int32_t)(cb - ca)) {
        __threadfence();
        float4 tot = z4;
        for (int64_t q0 = ca; q0 <= cb; q0 += 16) {
          float4 blk = z4;
          const int64_t q1 = (q0 + 16 < cb + 1) ? q0 + 16 : cb + 1;
          for (int64_t q = q0; q < q1; ++q) {
            const int64_t sl = q == ca ? 2 * q + 1 : 2 * q;
            if (lane < nv) add_v(blk, __ldcg(reinterpret_cast<const float4*>(a.partials + sl * a.W) + lane));
          }
          add_v(tot, blk);
        }
        edge_write_row(a, r, tot, lane, nv);
        if (lane == 0) a.counters[r] = 0;
      }
    };
    for (int64_t base = e0; base < e1; base += 32) {
      // prefetch the next batch of the stream (this chunk or the next chunk of this warp)
      const int nxt = which ^ 1;
      if (base + 32 < e1) issue(c, base + 32, nxt);
      else if (c + nwarps < nchunks) issue(c + nwarps, (c + nwarps) * kEdgeChunk, nxt);
      mbar_wait_parity(which ? mb1 : mb0, which ? phase1 : phase0);
      if (which) phase1 ^= 1u; else phase0 ^= 1u;
      const unsigned char* bb = wbuf + (size_t)which * 32 * rowb;
      const int n = which ? q_n1 : q_n0;
      const int32_t my_row = which ? q_row1 : q_row0;
      const float my_sc = which ? q_sc1 : q_sc0;
      for (int j = 0; j < n; ++j) {
        const int32_t rj = __shfl_sync(FULL, my_row, j);
        const float sj = SCOL ? __shfl_sync(FULL, my_sc, j) : 1.0f;
        if (rj != cur) {
          flush(cur);
          for (int32_t r = cur + 1; r < rj; ++r) edge_write_row(a, r, z4, lane, nv);
          cur = rj;
          acc0 = z4;
          acc1 = z4;
        }
        if (lane < nv) {
          const float4 xv = reinterpret_cast<const float4*>(bb + (size_t)j * rowb)[lane];
          if (((base + j) & 1) == 0) {
            if (SCOL) fma_v(acc0, sj, xv); else add_v(acc0, xv);
          } else {
            if (SCOL) fma_v(acc1, sj, xv); else add_v(acc1, xv);
          }
        }
      }
      __syncwarp();     // every lane is done reading this buffer before it is refilled
      which = nxt;
    }
    flush(cur);
  }
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

// Gather strategy switch (1 = cp.async shared-memory ring; 0 = register gathers).
static int g_agg_async = 0;   // measured fastest on C5

// Launch plan: vector width, group size, vectors per lane for W columns.
struct AggPlan {
  int vec, g, vpl, wmax;
};
static AggPlan plan_for(int32_t W, bool vec4) {
  AggPlan p;
  p.vec = vec4 ? 4 : 1;
  int nv = W / p.vec;
  if (nv > 128) nv = 128;                 // column-split into 128-vector launches
  int g = 1;
  while (g < 32 && g * 4 < nv) g <<= 1;
  p.g = g;
  p.vpl = (nv + g - 1) / g;
  p.wmax = 128 * p.vec;
  return p;
}

stg_status aggregate_launch(const stg_csr_view* gv, int backward, int32_t W, const float* in, int64_t ldin,
                            float* out, int64_t ldout, const float* srow, const float* scol, const float* bias,
                            cudaStream_t s) {
  if (!gv) return fail(STG_ERR_INVALID_ARG, "aggregate: view is NULL");
  if (W < 1) return fail(STG_ERR_INVALID_ARG, "aggregate: W=%d < 1", W);
  if (ldin < W || ldout < W) return fail(STG_ERR_INVALID_ARG, "aggregate: leading dimension < W");
  if (!in || !out) return fail(STG_ERR_INVALID_ARG, "aggregate: NULL input/output");
  const int32_t R = backward ? gv->num_nodes : gv->row_end - gv->row_begin;
  if (R <= 0) return STG_OK;
  AggArgs a{};
  a.R = R;
  a.rowptr = backward ? gv->out_rowptr : gv->in_rowptr;
  a.col = backward ? gv->out_col : gv->in_col;
  a.ids = backward ? gv->out_ids : gv->in_ids;
  a.sched = backward ? gv->out_sched : gv->in_sched;
  if (!a.rowptr || (gv->num_edges > 0 && !a.col))
    return fail(STG_ERR_INVALID_ARG, "aggregate: view lacks the %s CSR", backward ? "backward" : "forward");
  if (a.sched && (!a.ids || !gv->workspace)) a.sched = nullptr;
  a.srow = srow;
  a.scol = scol;
  a.bias = bias;
  const bool vec4 = (W % 4 == 0) && (ldin % 4 == 0) && (ldout % 4 == 0) &&
                    ((uintptr_t)in % 16 == 0) && ((uintptr_t)out % 16 == 0);
  const AggPlan p0 = plan_for(W, vec4);
  const int64_t chunks_bound = a.sched ? 2 * (gv->num_edges / kHubChunk) + 2 : 0;
  AggWs* ws = static_cast<AggWs*>(gv->workspace);
  if (a.sched) {
    const int32_t wl = W < p0.wmax ? W : p0.wmax;
    STG_TRY(ws->partials.alloc((size_t)chunks_bound * wl + 4, s));   // >= the async path's 128-column chunks
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
  // edge-parallel path: float4 rows, 16 <= float4-per-row chunks (W in [64, 128] per launch), COO rows known
  const int32_t* rowarr = backward ? gv->out_row : gv->in_row;
  if (vec4 && g_agg_async == 2 && W >= 64 && rowarr && gv->num_edges > 0 && gv->workspace) {
    const int64_t E = gv->num_edges;
    const int64_t nchunks = (E + kEdgeChunk - 1) / kEdgeChunk;
    STG_TRY(ws->epartials.alloc((size_t)2 * nchunks * 128 + 4, s));
    if (ws->ecounters_n < R) {
      STG_TRY(ws->ecounters.alloc(R, s));
      STG_CUDA(cudaMemsetAsync(ws->ecounters.p, 0, sizeof(int32_t) * R, s));
      ws->ecounters_n = R;
    }
    EdgeArgs ea{};
    ea.R = R; ea.E = E; ea.rowptr = a.rowptr; ea.col = a.col; ea.row = rowarr;
    ea.srow = srow; ea.scol = scol;
    ea.partials = ws->epartials.p; ea.counters = ws->ecounters.p;
    for (int32_t c0 = 0; c0 < W; c0 += 128) {
      const int32_t wl = (W - c0) < 128 ? (W - c0) : 128;
      ea.W = wl; ea.x = in + c0; ea.ldx = ldin; ea.y = out + c0; ea.ldy = ldout;
      ea.bias = bias ? bias + c0 : nullptr;
      auto fn = scol ? k_agg_edges_tma<true> : k_agg_edges_tma<false>;
      const size_t per_warp = (size_t)2 * 32 * wl * 4;
      int wpb = (int)std::min<size_t>(kAggThreads / 32, (size_t)(200 * 1024) / per_warp);
      if (wpb < 1) wpb = 1;
      const size_t smem = per_warp * wpb;
      {
        static std::mutex mu;
        std::lock_guard<std::mutex> lk(mu);
        static size_t attr[2] = {0, 0};
        if (attr[scol ? 1 : 0] < smem) {
          STG_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
          attr[scol ? 1 : 0] = smem;
        }
      }
      int per_sm = 0;
      if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kAggThreads, smem) != cudaSuccess || per_sm < 1) {
        cudaGetLastError();
        per_sm = 1;
      }
      int64_t blocks = ceil_div(nchunks, wpb);
      const int64_t mb = (int64_t)per_sm * num_sms();
      if (blocks > mb) blocks = mb;
      fn<<<(unsigned)blocks, kAggThreads, smem, s>>>(ea, wpb);
      count_launch();
    }
    return check_launch("aggregate_edges");
  }
  const bool use_async = vec4 && g_agg_async == 1;
  const int wmax = use_async ? 128 : p0.wmax;
  for (int32_t c0 = 0; c0 < W; c0 += wmax) {
    const int32_t wl = (W - c0) < wmax ? (W - c0) : wmax;
    const AggPlan p = plan_for(wl, vec4);
    a.W = wl;
    a.x = in + c0;
    a.ldx = ldin;
    a.y = out + c0;
    a.ldy = ldout;
    a.bias = bias ? bias + c0 : nullptr;
    const int rows_per_warp = 32 / p.g;
    const int U = p.vpl <= 2 ? 4 : 2;
    if (use_async && p.g >= U) {
      AsyncFn fn = scol ? pick_async_g<true>(p.g, p.vpl) : pick_async_g<false>(p.g, p.vpl);
      const size_t per_warp = (size_t)2 * 32 * wl * 4 + 2 * 32 * 4;
      int wpb = (int)std::min<size_t>(8, (size_t)(200 * 1024) / per_warp);
      if (wpb < 1) wpb = 1;
      const size_t smem = per_warp * wpb;
      static std::mutex mu;
      {
        std::lock_guard<std::mutex> lk(mu);
        static std::map<AsyncFn, size_t> attr;
        if (attr[fn] < smem) {
          STG_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
          attr[fn] = smem;
        }
      }
      int per_sm = 0;
      if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kAggThreads, smem) != cudaSuccess || per_sm < 1) {
        cudaGetLastError();
        per_sm = 1;
      }
      int64_t blocks = ceil_div(items_bound, (int64_t)wpb * rows_per_warp);
      const int64_t mb = (int64_t)per_sm * num_sms();
      if (blocks > mb) blocks = mb;
      if (blocks < 1) blocks = 1;
      fn<<<(unsigned)blocks, kAggThreads, smem, s>>>(a, wpb);
    } else {
      KernelFn fn = pick(p.vec, p.g, p.vpl, scol != nullptr);
      const int rows_per_block = (kAggThreads / 32) * rows_per_warp;
      int64_t blocks = ceil_div(items_bound, rows_per_block);
      const int64_t mb = max_blocks_for(fn);
      if (blocks > mb) blocks = mb;
      if (blocks < 1) blocks = 1;
      fn<<<(unsigned)blocks, kAggThreads, 0, s>>>(a);
    }
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
  return stg::aggregate_launch(g, 1, W, gy, ldgy, gx, ldgx, g->norm_src, g->norm_dst, nullptr,
                               (cudaStream_t)stream);
}

stg_status stg_aggregate_set_strategy(int32_t strategy) {
  if (strategy < 0 || strategy > 2) return stg::fail(STG_ERR_INVALID_ARG, "stg_aggregate_set_strategy: %d", strategy);
  stg::g_agg_async = strategy;
  return STG_OK;
}

stg_status stg_gcn_aggregate_ex(const stg_csr_view* g, int32_t backward, int32_t W, const float* in, int64_t ldin,
                                float* out, int64_t ldout, const float* scale_row, const float* scale_col,
                                const float* bias, stg_stream_t stream) {
  return stg::aggregate_launch(g, backward, W, in, ldin, out, ldout, scale_row, scale_col, bias,
                               (cudaStream_t)stream);
}

}  // extern "C"
