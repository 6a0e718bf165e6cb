// agg_locality_probe.cu — microbenchmark (not part of libstg): the C5 in-CSR
// aggregation's memory pattern (gather x[col[e]] rows of W = 96 fp32 in CSR
// order, one 384-byte output row written per destination) under different
// source-row layouts and L1/L2 eviction hints.  The question it answers: can
// the L2 keep the hot (high out-degree) source rows, and does that cut DRAM
// bytes and time?  The driver (agg_locality_probe.py) relabels the sources
// hot-first (rank in out-degree order) and times each variant; ncu supplies
// the DRAM bytes.
//
// hint: 0 = plain __ldg
//       1 = u <  K: L2 evict_last (createpolicy), u >= K: L1 no_allocate + L2 evict_first
//       2 = u >= K: L1 no_allocate + L2 evict_first only
//       3 = u <  K: L2 evict_last only
//       4 = like 1, plus L1 evict_last for the hot rows
#include <cuda_runtime.h>
#include <cstdint>

__device__ __forceinline__ float4 ld_plain(const float4* p) { return __ldg(p); }
__device__ __forceinline__ float4 ld_pol(const float4* p, uint64_t pol) {
  float4 v;
  asm volatile("ld.global.nc.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ float4 ld_pol_na(const float4* p, uint64_t pol) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ float4 ld_pol_l1el(const float4* p, uint64_t pol) {
  float4 v;
  asm volatile("ld.global.nc.L1::evict_last.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
  return v;
}

// Each warp walks a contiguous chunk of CH edges (edges of consecutive rows);
// lane j of a 32-edge batch loads (col, row) of edge j; D rows in flight; the
// running sum is written (streaming store) whenever the row changes.
__device__ __forceinline__ void st_pol(float4* p, float4 v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1,%2,%3,%4}, %5;" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z),
               "f"(v.w), "l"(pol) : "memory");
}

// STORE: 0 = no output rows (one float4 per lane at the end), 1 = st.global.cs,
// 2 = st.global with an L2 evict_first policy, 3 = plain st.global
template <int D, int HINT, int STORE = 1>
__global__ void __launch_bounds__(256) k_probe(const float4* __restrict__ x, const int32_t* __restrict__ col,
                                               const int32_t* __restrict__ row, int64_t E, int32_t K, int64_t CH,
                                               float4* __restrict__ y) {
  const int lane = threadIdx.x & 31;
  const int lc = lane < 24 ? lane : 23;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  uint64_t pf = 0, pl = 0;
  if (HINT) {
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pf));
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pl));
  }
  float4 sink = make_float4(0.f, 0.f, 0.f, 0.f);
  auto put = [&](int32_t r, const float4& v) {
    if (lane >= 24) return;
    float4* q = y + (int64_t)r * 24 + lane;
    if (STORE == 0) { sink.x += v.x; sink.y += v.y; sink.z += v.z; sink.w += v.w; }
    else if (STORE == 1) __stcs(q, v);
    else if (STORE == 2) st_pol(q, v, pf);
    else *q = v;
  };
  if (STORE == 2 && !HINT) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pf));
  for (int64_t c0 = warp * CH; c0 < E; c0 += nw * CH) {
    const int64_t c1 = c0 + CH < E ? c0 + CH : E;
    int32_t cur = -1;
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int64_t b0 = c0; b0 < c1; b0 += 32) {
      const int64_t e = b0 + lane;
      const int32_t mu = e < c1 ? __ldcs(col + e) : -1;
      const int32_t mr = e < c1 ? __ldcs(row + e) : -1;
      const int nb = (int)(c1 - b0 < 32 ? c1 - b0 : 32);
      for (int j0 = 0; j0 < nb; j0 += D) {
        float4 v[D];
        int32_t rr[D];
#pragma unroll
        for (int d = 0; d < D; ++d) {
          const int32_t u = __shfl_sync(0xffffffffu, mu, (j0 + d) & 31);
          rr[d] = __shfl_sync(0xffffffffu, mr, (j0 + d) & 31);
          if (u < 0) { v[d] = make_float4(0.f, 0.f, 0.f, 0.f); continue; }
          const float4* p = x + (int64_t)u * 24 + lc;
          if (HINT == 0) v[d] = ld_plain(p);
          else if (HINT == 1) v[d] = u < K ? ld_pol(p, pl) : ld_pol_na(p, pf);
          else if (HINT == 2) v[d] = u < K ? ld_plain(p) : ld_pol_na(p, pf);
          else if (HINT == 3) v[d] = u < K ? ld_pol(p, pl) : ld_plain(p);
          else v[d] = u < K ? ld_pol_l1el(p, pl) : ld_pol_na(p, pf);
        }
#pragma unroll
        for (int d = 0; d < D; ++d) {
          if (rr[d] < 0) continue;
          if (rr[d] != cur) {
            if (cur >= 0) put(cur, acc);
            cur = rr[d];
            acc = v[d];
          } else {
            acc.x += v[d].x; acc.y += v[d].y; acc.z += v[d].z; acc.w += v[d].w;
          }
        }
      }
    }
    if (cur >= 0) put(cur, acc);
  }
  if (STORE == 0 && lane < 24) y[((int64_t)blockIdx.x * blockDim.x + threadIdx.x) % 24] = sink;
}

template <int HINT>
static void launch(int D, const float4* x, const int32_t* col, const int32_t* row, int64_t E, int32_t K, int64_t CH,
                   float4* y, int blocks, cudaStream_t s) {
  switch (D) {
    case 2: k_probe<2, HINT><<<blocks, 256, 0, s>>>(x, col, row, E, K, CH, y); break;
    case 4: k_probe<4, HINT><<<blocks, 256, 0, s>>>(x, col, row, E, K, CH, y); break;
    default: k_probe<8, HINT><<<blocks, 256, 0, s>>>(x, col, row, E, K, CH, y); break;
  }
}

extern "C" int probe_run(int hint, int D, const void* x, const int32_t* col, const int32_t* row, int64_t E,
                         int32_t K, int64_t CH, void* y, int blocks, void* stream) {
  const float4* xx = (const float4*)x;
  float4* yy = (float4*)y;
  cudaStream_t s = (cudaStream_t)stream;
  switch (hint) {
    case 0: launch<0>(D, xx, col, row, E, K, CH, yy, blocks, s); break;
    case 1: launch<1>(D, xx, col, row, E, K, CH, yy, blocks, s); break;
    case 2: launch<2>(D, xx, col, row, E, K, CH, yy, blocks, s); break;
    case 3: launch<3>(D, xx, col, row, E, K, CH, yy, blocks, s); break;
    default: launch<4>(D, xx, col, row, E, K, CH, yy, blocks, s); break;
  }
  return (int)cudaGetLastError();
}

extern "C" int probe_store_run(int store, const void* x, const int32_t* col, const int32_t* row, int64_t E,
                               int64_t CH, void* y, int blocks, void* stream) {
  const float4* xx = (const float4*)x;
  float4* yy = (float4*)y;
  cudaStream_t s = (cudaStream_t)stream;
  cudaGetLastError();
  switch (store) {
    case 0: k_probe<4, 0, 0><<<blocks, 256, 0, s>>>(xx, col, row, E, 0, CH, yy); break;
    case 1: k_probe<4, 0, 1><<<blocks, 256, 0, s>>>(xx, col, row, E, 0, CH, yy); break;
    case 2: k_probe<4, 0, 2><<<blocks, 256, 0, s>>>(xx, col, row, E, 0, CH, yy); break;
    default: k_probe<4, 0, 3><<<blocks, 256, 0, s>>>(xx, col, row, E, 0, CH, yy); break;
  }
  return (int)cudaGetLastError();
}

extern "C" int set_persist(void* stream, const void* base, size_t win_bytes, float hit_ratio, size_t limit) {
  cudaStream_t s = (cudaStream_t)stream;
  cudaError_t e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, limit);
  if (e != cudaSuccess) return 1000 + (int)e;
  cudaStreamAttrValue v = {};
  v.accessPolicyWindow.base_ptr = const_cast<void*>(base);
  v.accessPolicyWindow.num_bytes = win_bytes;
  v.accessPolicyWindow.hitRatio = hit_ratio;
  v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
  v.accessPolicyWindow.missProp = cudaAccessPropertyNormal;
  e = cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v);
  if (e != cudaSuccess) return 2000 + (int)e;
  if (win_bytes == 0) cudaCtxResetPersistingL2Cache();
  return 0;
}
