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
