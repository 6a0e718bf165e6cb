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
