// gather_bench.cu — microbenchmark of the raw row-gather ceiling on B200 (not
// part of libstg).  Sums rows x[idx[i]] (row = W fp32) into one float4 per
// lane, with D independent rows in flight per warp; 24/32-lane row mapping
// for W = 96.  Reports nothing itself: the python driver times it.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC
#include <cuda_runtime.h>
#include <cstdint>

template <int D, int NV>
__global__ void __launch_bounds__(256) k_gather(const float4* __restrict__ x, const int32_t* __restrict__ idx,
                                                int64_t n, float4* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int64_t base = warp * 32; base < n; base += nw * 32) {
    const int32_t my = base + lane < n ? __ldg(idx + base + lane) : -1;
#pragma unroll 1
    for (int j0 = 0; j0 < 32; j0 += D) {
      float4 v[D];
#pragma unroll
      for (int d = 0; d < D; ++d) {
        const int32_t u = __shfl_sync(0xffffffffu, my, j0 + d);
        v[d] = (u >= 0 && lane < NV) ? __ldg(x + (int64_t)u * NV + lane) : make_float4(0.f, 0.f, 0.f, 0.f);
      }
#pragma unroll
      for (int d = 0; d < D; ++d) {
        acc.x += v[d].x; acc.y += v[d].y; acc.z += v[d].z; acc.w += v[d].w;
      }
    }
  }
  if (lane < NV) out[((int64_t)blockIdx.x * blockDim.x + threadIdx.x)] = acc;
}

extern "C" int gather_run(int D, const void* x, const int32_t* idx, int64_t n, void* out, int blocks) {
  const float4* xx = (const float4*)x;
  float4* o = (float4*)out;
  switch (D) {
    case 1: k_gather<1, 24><<<blocks, 256>>>(xx, idx, n, o); break;
    case 2: k_gather<2, 24><<<blocks, 256>>>(xx, idx, n, o); break;
    case 4: k_gather<4, 24><<<blocks, 256>>>(xx, idx, n, o); break;
    case 8: k_gather<8, 24><<<blocks, 256>>>(xx, idx, n, o); break;
    case 16: k_gather<16, 24><<<blocks, 256>>>(xx, idx, n, o); break;
    default: return -1;
  }
  return (int)cudaGetLastError();
}

// Store-pattern probe: V rows of 96 fp32 written by a grid of `blocks` x `threads`.
// mode 0: thread-per-row (each thread writes its row's 24 float4);
// mode 1: warp-coalesced (lane l writes float4 l of a row, 24 lanes active);
// mode 2: thread-per-row through a per-warp shared stage + TMA bulk store per row.
__global__ void __launch_bounds__(128) k_store(int mode, float4* __restrict__ y, int64_t V) {
  extern __shared__ __align__(16) float4 stage_raw[];
  float4 (*stage)[32 * 25] = reinterpret_cast<float4 (*)[32 * 25]>(stage_raw);
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
  const float4 val = make_float4(1.f, 2.f, 3.f, (float)threadIdx.x);
  if (mode == 0) {
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < V; r += nthr)
#pragma unroll
      for (int c = 0; c < 24; ++c) y[r * 24 + c] = val;
  } else if (mode == 1) {
    const int64_t nw = nthr / 32;
    for (int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / 32; r < V; r += nw)
      if (lane < 24) y[r * 24 + lane] = val;
  } else {
    for (int64_t r0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x - lane); r0 < V; r0 += nthr) {
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      __syncwarp();
#pragma unroll
      for (int c = 0; c < 24; ++c) stage[w][lane * 25 + c] = val;
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      const int64_t r = r0 + lane;
      if (r < V) {
        const uint32_t src = (uint32_t)__cvta_generic_to_shared(&stage[w][lane * 25]);
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], 384;" ::"l"(y + r * 24), "r"(src)
                     : "memory");
      }
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
}

extern "C" int store_run(int mode, void* y, int64_t V, int blocks, int threads) {
  const int smem = 4 * 32 * 25 * 16;
  cudaFuncSetAttribute(k_store, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k_store<<<blocks, threads, smem>>>(mode, (float4*)y, V);
  return (int)cudaGetLastError();
}

// Feature-sliced gather probe: x stored as [S][V][SW] (slice-major) or as the
// plain row-major [V][S*SW]; one pass per slice gathers the SW-float piece of
// every indexed row (SW/4 lanes per row, 32/(SW/4) rows per warp instruction,
// D instructions in flight).  Slice-major makes each pass's working set V*SW*4 B.
template <int SW, int D>
__global__ void __launch_bounds__(256) k_gather_sliced(const float4* __restrict__ x, const int32_t* __restrict__ idx,
                                                       int64_t n, int64_t V, int slice, int S, int slice_major,
                                                       float4* __restrict__ out) {
  constexpr int LPR = SW / 4;          // lanes per row
  constexpr int RPI = 32 / LPR;        // rows per instruction
  const int lane = threadIdx.x & 31;
  const int sub = lane / LPR, q = lane % LPR;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const float4* xs = slice_major ? x + (int64_t)slice * V * LPR : x + (int64_t)slice * LPR;
  const int64_t rstride = slice_major ? LPR : (int64_t)S * LPR;
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int64_t base = warp * 32; base < n; base += nw * 32) {
    const int32_t my = base + lane < n ? __ldg(idx + base + lane) : -1;
#pragma unroll
    for (int j0 = 0; j0 < 32; j0 += RPI * D) {
      float4 v[D];
#pragma unroll
      for (int d = 0; d < D; ++d) {
        const int32_t u = __shfl_sync(0xffffffffu, my, j0 + d * RPI + sub);
        v[d] = u >= 0 ? __ldg(xs + (int64_t)u * rstride + q) : make_float4(0.f, 0.f, 0.f, 0.f);
      }
#pragma unroll
      for (int d = 0; d < D; ++d) {
        acc.x += v[d].x; acc.y += v[d].y; acc.z += v[d].z; acc.w += v[d].w;
      }
    }
  }
  out[((int64_t)blockIdx.x * blockDim.x + threadIdx.x)] = acc;
}

extern "C" int gather_sliced_run(int SW, int D, const void* x, const int32_t* idx, int64_t n, int64_t V, int S,
                                 int slice_major, void* out, int blocks) {
  const float4* xx = (const float4*)x;
  float4* o = (float4*)out;
  for (int s = 0; s < S; ++s) {
#define GS(sw, d) if (SW == sw && D == d) k_gather_sliced<sw, d><<<blocks, 256>>>(xx, idx, n, V, s, S, slice_major, o)
    GS(8, 1); GS(8, 2); GS(8, 4); GS(8, 8);
    GS(16, 1); GS(16, 2); GS(16, 4); GS(16, 8);
    GS(32, 1); GS(32, 2); GS(32, 4);
#undef GS
  }
  return (int)cudaGetLastError();
}

// L2 persistence probe: the same row gather on a caller stream, optionally
// with an access-policy window (persisting) over the first `win_bytes` of x.
extern "C" int gather_run_stream(int D, const void* x, const int32_t* idx, int64_t n, void* out, int blocks,
                                 void* stream) {
  cudaStream_t s = (cudaStream_t)stream;
  const float4* xx = (const float4*)x;
  float4* o = (float4*)out;
  switch (D) {
    case 2: k_gather<2, 24><<<blocks, 256, 0, s>>>(xx, idx, n, o); break;
    case 4: k_gather<4, 24><<<blocks, 256, 0, s>>>(xx, idx, n, o); break;
    case 8: k_gather<8, 24><<<blocks, 256, 0, s>>>(xx, idx, n, o); break;
    default: return -1;
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
  v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
  e = cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v);
  if (e != cudaSuccess) return 2000 + (int)e;
  if (win_bytes == 0) cudaCtxResetPersistingL2Cache();
  return 0;
}

extern "C" size_t max_persist() {
  int dev = 0, v = 0, w = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&v, cudaDevAttrMaxPersistingL2CacheSize, dev);
  cudaDeviceGetAttribute(&w, cudaDevAttrMaxAccessPolicyWindowSize, dev);
  return ((size_t)v << 32) | (size_t)(unsigned)w;
}
