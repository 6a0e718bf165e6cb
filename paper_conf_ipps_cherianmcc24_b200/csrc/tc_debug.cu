// tc_debug.cu — diagnostic tcgen05 3xTF32 GEMM used by the GPU tests to pin
// the descriptor / layout / TMEM conventions of tc.cuh against a plain product.
//   mode 0: C[M,N] = A[M,K] · B[K,N]            (K-major A and B, M = 128·tiles)
//   mode 1: C[128,N] = Xᵀ·Y, X[R,128], Y[R,N]    (MN-major views, R = 128·tiles,
//           accumulated across tiles in TMEM — the reduction form of dW / dL)
//   mode 2: as mode 0 with the A operand (hi/lo) written to TENSOR MEMORY by
//           the threads (tcgen05.st, thread = row) and read by the MMA from there
//   mode 3: ONE tf32 MMA on unsplit fp32 operands (A raw · B raw): the test
//           compares it with truncated and rounded tf32 products to pin the
//           hardware's fp32 -> tf32 input conversion
//   mode 4: as mode 1 (Xᵀ·Y, X[R,128], Y[R,N]) with both operands loaded by 2-D
//           TMA boxes (128 rows x 32 fp32) in the MN-major SWIZZLE_128B_BASE32B
//           layout (k_tc_debug_mn: no transposition by threads; hi = raw)
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
  const int Kt = mode != 1 ? K : 32;            // K extent of a stored tile (32 rows for mode 1)
  const int Mrows = 128;
  unsigned char* a_hi = sm;
  const int pf = mode != 1 ? 4 : 5;              // mode 1 tiles use the padded transposed layout
  unsigned char* a_lo = a_hi + Mrows * Kt * pf;
  const int Kb = mode != 1 ? K : 32;             // modes 0/2/3: B stored [N × K]; mode 1: Yᵀ tile [N × 32]
  const int Nr = N;
  unsigned char* b_hi = a_lo + Mrows * Kt * pf;
  unsigned char* b_lo = b_hi + Nr * Kb * pf;
  const int warp = threadIdx.x >> 5;
  uint32_t ncols = 32;
  while ((int)ncols < N) ncols <<= 1;
  if (mode == 2) ncols = 512;                     // [0,256) accumulator, [256, 256+2K) A hi/lo
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
  const int tiles = mode != 1 ? 1 : R / 32;
  const int row0 = mode != 1 ? blockIdx.x * 128 : 0;
  for (int tile = 0; tile < tiles; ++tile) {
    // ---- stage operands
    if (mode == 2) {
      const int r = threadIdx.x;                      // thread = row = TMEM lane (warp w -> lanes 32w..)
      for (int k0 = 0; k0 < K; k0 += 8) {
        float hv[8], lv[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const float v = A[(int64_t)(row0 + r) * K + k0 + i];
          hv[i] = tc::tf32_hi(v);
          lv[i] = v - hv[i];
        }
        tc::tmem_st8(tm + ((uint32_t)(warp * 32) << 16) + (uint32_t)(256 + k0), hv);
        tc::tmem_st8(tm + ((uint32_t)(warp * 32) << 16) + (uint32_t)(256 + K + k0), lv);
      }
      tc::tmem_wait_st();
    }
    if (mode == 0 || mode == 2 || mode == 3) {
      for (int e = threadIdx.x; mode != 2 && e < 128 * (K / 4); e += 128) {
        const int rl = e & 7, j = (e >> 3) % (K / 4), rg = e / (8 * (K / 4));
        const int r = rg * 8 + rl;
        float4 v = *reinterpret_cast<const float4*>(A + (int64_t)(row0 + r) * K + 4 * j);
        if (mode == 3) {            // raw fp32 as the "hi" operand
          const uint32_t off = (uint32_t)((r & 7) * 16 + (r >> 3) * (K / 4) * 128 + j * 128);
          *reinterpret_cast<float4*>(a_hi + off) = v;
        } else {
          tc::st_split4(a_hi, a_lo, r, j, K, v);
        }
      }
      for (int e = threadIdx.x; e < N * K; e += 128) {   // B[k][n] -> K-major [n][k]
        const int n = e / K, k = e % K;
        const float v = B[(int64_t)k * N + n];
        const float h = mode == 3 ? v : tc::tf32_hi(v);
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
      } else if (mode == 3) {
        const uint32_t idesc = tc::idesc_tf32(128, N, 0, 0), sbo = (uint32_t)(K / 4) * 128;
        for (int k = 0; k < K; k += 8) {
          const uint32_t off = (uint32_t)(k / 4) * 128;
          tc::mma_tf32(tm, tc::desc(tc::smem_u32(a_hi) + off, 128, sbo), tc::desc(tc::smem_u32(b_hi) + off, 128, sbo),
                       idesc, k > 0 ? 1u : 0u);
        }
      } else if (mode == 2) {
        const uint32_t idesc = tc::idesc_tf32(128, N, 0, 0), sbo = (uint32_t)(K / 4) * 128;
        for (int k = 0; k < K; k += 8) {
          const uint32_t off = (uint32_t)(k / 4) * 128;
          const uint64_t bh = tc::desc(tc::smem_u32(b_hi) + off, 128, sbo), bl = tc::desc(tc::smem_u32(b_lo) + off, 128, sbo);
          tc::mma_tf32_ts(tm, tm + 256 + K + k, bh, idesc, k > 0 ? 1u : 0u);   // A_lo·B_hi
          tc::mma_tf32_ts(tm, tm + 256 + k, bl, idesc, 1u);                    // A_hi·B_lo
          tc::mma_tf32_ts(tm, tm + 256 + k, bh, idesc, 1u);                    // A_hi·B_hi
        }
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

// mode 4: D[128 x N] += Xᵀ Y over R rows in 128-row tiles, A/B MN-major (TMA).
__global__ void __launch_bounds__(128) k_tc_debug_mn(int N, int R, const __grid_constant__ CUtensorMap tmX,
                                                     const __grid_constant__ CUtensorMap tmY, float* __restrict__ C) {
  extern __shared__ unsigned char sm_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(sm_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full, mbar;
  __shared__ uint32_t tslot;
  constexpr int BOX = 128 * 32 * 4;
  const int nby = N / 32;
  unsigned char* xh = sm;                       // 4 boxes
  unsigned char* xl = sm + 4 * BOX;
  unsigned char* yh = sm + 8 * BOX;             // nby boxes
  unsigned char* yl = yh + nby * BOX;
  const int warp = threadIdx.x >> 5;
  uint32_t ncols = 32;
  while ((int)ncols < N) ncols <<= 1;
  if (warp == 0) tc::tmem_alloc(&tslot, ncols);
  if (threadIdx.x == 0) { tc::mbar_init(&full, 1); tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  const uint32_t idesc = tc::idesc_tf32(128, N, 1, 1);
  for (int t = 0; t < R / 128; ++t) {
    if (threadIdx.x == 0) {
      tc::mbar_expect_tx(&full, (uint32_t)(4 + nby) * BOX);
      for (int k = 0; k < 4; ++k) tc::tma_load_2d(xh + k * BOX, &tmX, 32 * k, 128 * t, &full);
      for (int k = 0; k < nby; ++k) tc::tma_load_2d(yh + k * BOX, &tmY, 32 * k, 128 * t, &full);
    }
    tc::mbar_wait(&full, t & 1);
    // lo = raw - trunc(raw), elementwise over the (identically laid out) boxes
    for (int e = threadIdx.x; e < (4 + nby) * BOX / 16; e += 128) {
      const int which = e < 4 * BOX / 16 ? 0 : 1;
      const int o = which ? e - 4 * BOX / 16 : e;
      const float4 v = reinterpret_cast<const float4*>(which ? yh : xh)[o];
      reinterpret_cast<float4*>(which ? yl : xl)[o] =
          make_float4(v.x - tc::tf32_hi(v.x), v.y - tc::tf32_hi(v.y), v.z - tc::tf32_hi(v.z), v.w - tc::tf32_hi(v.w));
    }
    tc::fence_proxy_async();
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    if (threadIdx.x == 0) {
      for (int k = 0; k < 128; k += 8) {               // 8 K-rows (1024 B) per MMA
        const uint32_t o = (uint32_t)k * 128;
        const uint64_t ah = tc::desc_mn_sw128_32b(tc::smem_u32(xh) + o, BOX), al = tc::desc_mn_sw128_32b(tc::smem_u32(xl) + o, BOX);
        const uint64_t bh = tc::desc_mn_sw128_32b(tc::smem_u32(yh) + o, BOX), bl = tc::desc_mn_sw128_32b(tc::smem_u32(yl) + o, BOX);
        tc::mma_tf32(tm, al, bh, idesc, (t > 0 || k > 0) ? 1u : 0u);
        tc::mma_tf32(tm, ah, bl, idesc, 1u);
        tc::mma_tf32(tm, ah, bh, idesc, 1u);
      }
      tc::commit(&mbar);
    }
    tc::mbar_wait(&mbar, t & 1);
    tc::fence_after();
    __syncthreads();
  }
  const int r = warp * 32 + (threadIdx.x & 31);
  for (int c = 0; c < N; c += 8) {
    float v[8];
    tc::tmem_ld8(tm + ((uint32_t)(warp * 32) << 16) + (uint32_t)c, v);
    tc::tmem_wait_ld();
#pragma unroll
    for (int i = 0; i < 8; ++i) C[(int64_t)r * N + c + i] = v[i];
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 0) tc::tmem_free(tm, ncols);
}

}  // namespace
}  // namespace stg

extern "C" stg_status stg_debug_tc_gemm(int32_t mode, int32_t M, int32_t N, int32_t K, int32_t R, const float* A,
                                        const float* B, float* C, stg_stream_t stream) {
  using namespace stg;
  if (N % 16 || N < 16 || N > 256) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: N=%d", N);
  if (mode < 0 || mode > 4) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: mode=%d", mode);
  if (mode == 4) {
    if (R % 128 || N % 32) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: mode 4 needs R %% 128 == 0, N %% 32 == 0");
    CUtensorMap tx, ty;
    STG_TRY(make_tmap_f32(&tx, A, (uint64_t)R, 128, 128, 32, 128, true));
    STG_TRY(make_tmap_f32(&ty, B, (uint64_t)R, (uint64_t)N, (uint64_t)N, 32, 128, true));
    const size_t smem = (size_t)2 * (4 + N / 32) * 128 * 32 * 4 + 1024;
    STG_CUDA(cudaFuncSetAttribute(k_tc_debug_mn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    k_tc_debug_mn<<<1, 128, smem, (cudaStream_t)stream>>>(N, R, tx, ty, C);
    count_launch();
    return check_launch("stg_debug_tc_gemm mode 4");
  }
  if (mode != 1 && (M % 128 || K % 8 || K < 8 || K > 256)) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: M/K");
  if (mode == 2 && K > 128) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: K > 128 for TMEM A");
  if (mode == 1 && (R % 32 || R < 32)) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: R");
  const int Kt = mode != 1 ? K : 32, Kb = mode != 1 ? K : 32, Nr = N;
  const int pf = mode != 1 ? 4 : 5;
  const size_t smem = (size_t)2 * 128 * Kt * pf + (size_t)2 * Nr * Kb * pf;
  if (smem > 200 * 1024) return fail(STG_ERR_INVALID_ARG, "stg_debug_tc_gemm: tile too large");
  STG_CUDA(cudaFuncSetAttribute(k_tc_debug, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int grid = mode != 1 ? M / 128 : 1;
  k_tc_debug<<<grid, 128, smem, (cudaStream_t)stream>>>(mode, M, N, K, R, A, B, C);
  count_launch();
  return check_launch("stg_debug_tc_gemm");
}
