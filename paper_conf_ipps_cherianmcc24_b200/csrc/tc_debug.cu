// tc_debug.cu — diagnostic tcgen05 3xTF32 GEMM used by the GPU tests to pin
// the descriptor / layout / TMEM conventions of tc.cuh against a plain product.
//   mode 0: C[M,N] = A[M,K] · B[K,N]            (K-major A and B, M = 128·tiles)
//   mode 1: C[128,N] = Xᵀ·Y, X[R,128], Y[R,N]    (MN-major views, R = 128·tiles,
//           accumulated across tiles in TMEM — the reduction form of dW / dL)
#include "common.cuh"
#include "tc.cuh"

namespace stg {
namespace {

// Stage rows [0,128) × cols [0,F) of a row-major array (leading dim ld) as the
// transposed K-major operand [F × 128] (hi/lo), via tc::stage_rows_T.
__device__ void stage_transposed(unsigned char* hi, unsigned char* lo, const float* src, int F, int ld) {
  tc::stage_rows_T(hi, lo, src, ld, 128, F, 0, 0, 32);
}

__global__ void __launch_bounds__(128) k_tc_debug(int mode, int M, int N, int K, int R, const float* __restrict__ A,
                                                  const float* __restrict__ B, float* __restrict__ C) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t mbar;
  __shared__ uint32_t tslot;
  const int Kt = mode == 0 ? K : 32;            // K extent of a stored tile (32 rows for mode 1)
  const int Mrows = 128;
  unsigned char* a_hi = sm;
  const int pf = mode == 0 ? 4 : 5;              // mode 1 tiles use the padded transposed layout
  unsigned char* a_lo = a_hi + Mrows * Kt * pf;
  const int Kb = mode == 0 ? K : 32;             // mode 0: B stored [N × K]; mode 1: Yᵀ tile [N × 32]
  const int Nr = N;
  unsigned char* b_hi = a_lo + Mrows * Kt * pf;
  unsigned char* b_lo = b_hi + Nr * Kb * pf;
  const int warp = threadIdx.x >> 5;
  uint32_t ncols = 32;
  while ((int)ncols < N) ncols <<= 1;
  if (warp == 0) tc::tmem_alloc(&tslot, ncols);
  if (threadIdx.x == 0) {
    tc::mbar_init(&mbar, 1);
    tc::fence_mbar_init();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  uint32_t phase = 0;
  const int tiles = mode == 0 ? 1 : R / 32;
  const int row0 = mode == 0 ? blockIdx.x * 128 : 0;
  for (int tile = 0; tile < tiles; ++tile) {
    // ---- stage operands
    if (mode == 0) {
      for (int e = threadIdx.x; e < 128 * (K / 4); e += 128) {
        const int rl = e & 7, j = (e >> 3) % (K / 4), rg = e / (8 * (K / 4));
        const int r = rg * 8 + rl;
        float4 v = *reinterpret_cast<const float4*>(A + (int64_t)(row0 + r) * K + 4 * j);
        tc::st_split4(a_hi, a_lo, r, j, K, v);
      }
      for (int e = threadIdx.x; e < N * K; e += 128) {   // B[k][n] -> K-major [n][k]
        const int n = e / K, k = e % K;
        const float v = B[(int64_t)k * N + n];
        const float h = tc::tf32_hi(v);
        *reinterpret_cast<float*>(b_hi + tc::kmaj_off(n, k, K)) = h;
        *reinterpret_cast<float*>(b_lo + tc::kmaj_off(n, k, K)) = v - h;
      }
    } else {
      // transposed K-major staging: A' = X tileᵀ [128 feats × 32 rows], B' = Y tileᵀ [N × 32 rows]
      const int r0 = tile * 32;
      stage_transposed(a_hi, a_lo, A + (int64_t)r0 * 128, 128, 128);
      stage_transposed(b_hi, b_lo, B + (int64_t)r0 * N, N, N);
    }
    tc::fence_proxy_async();
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    if (threadIdx.x == 0) {
      if (mode == 0) {
        tc::mma_3xtf32_kmajor(tm, tc::smem_u32(a_hi), tc::smem_u32(a_lo), tc::smem_u32(b_hi), tc::smem_u32(b_lo), K,
                              tc::idesc_tf32(128, N, 0, 0), false);
      } else {
        const uint32_t sb = tc::sbo_t(32), idesc = tc::idesc_tf32(128, N, 0, 0);
        for (int k = 0; k < 32; k += 8) {
          const uint32_t o = (uint32_t)(k / 4) * tc::kLboT;
          const uint32_t acc = (tile > 0 || k > 0) ? 1u : 0u;
          tc::mma_tf32(tm, tc::desc(tc::smem_u32(a_lo) + o, tc::kLboT, sb), tc::desc(tc::smem_u32(b_hi) + o, tc::kLboT, sb), idesc, acc);
          tc::mma_tf32(tm, tc::desc(tc::smem_u32(a_hi) + o, tc::kLboT, sb), tc::desc(tc::smem_u32(b_lo) + o, tc::kLboT, sb), idesc, 1u);
          tc::mma_tf32(tm, tc::desc(tc::smem_u32(a_hi) + o, tc::kLboT, sb), tc::desc(tc::smem_u32(b_hi) + o, tc::kLboT, sb), idesc, 1u);
        }
      }
      tc::commit(&mbar);
    }
    tc::mbar_wait(&mbar, phase);
    phase ^= 1;
    tc::fence_after();
    __syncthreads();   // smem operands may be overwritten by the next tile
  }
  // ---- epilogue: TMEM -> registers -> global
  const int r = warp * 32 + (threadIdx.x & 31);
  for (int c = 0; c < N; c += 8) {
    float v[8];
    tc::tmem_ld8(tm + ((uint32_t)(warp * 32) << 16) + (uint32_t)c, v);
    tc::tmem_wait_ld();
#pragma unroll
    for (int i = 0; i < 8; ++i) C[(int64_t)(row0 + r) * N + c + i] = v[i];
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 0) tc::tmem_free(tm, ncols);
  (void)M;
}

}  // namespace
}  // namespace stg

extern "C" stg_status stg_debug_tc_gemm(int32_t mode, int32_t M, int32_t N, int32_t K, int32_t R, const float* A,
                                        const float* B, float* C, stg_stream_t stream) {
  using namespace stg;
  if (N % 16 || N < 16 || N > 256) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: N=%d", N);
  if (mode == 0 && (M % 128 || K % 8 || K < 8 || K > 256)) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: M/K");
  if (mode == 1 && (R % 32 || R < 32)) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: R");
  const int Kt = mode == 0 ? K : 32, Kb = mode == 0 ? K : 32, Nr = N;
  const int pf = mode == 0 ? 4 : 5;
  const size_t smem = (size_t)2 * 128 * Kt * pf + (size_t)2 * Nr * Kb * pf;
  if (smem > 200 * 1024) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: tile too large");
  STG_CUDA(cudaFuncSetAttribute(k_tc_debug, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int grid = mode == 0 ? M / 128 : 1;
  k_tc_debug<<<grid, 128, smem, (cudaStream_t)stream>>>(mode, M, N, K, R, A, B, C);
  count_launch();
  return check_launch("stg_debug_tc_gemm");
}
