// tc_tgcn.cu — the TGCN dense contractions on 5th-gen tensor cores (tcgen05,
// 3xTF32 for fp32-class accuracy, accumulators in TMEM).  Each kernel is a
// persistent loop over 128-row tiles (one row per thread in the epilogue):
//
//   k_tc_xw_pipe  P' = diag(n_src)·X·W                  (K = F, N = 3H; k_tc_xw for 64 < F <= 128)
//   k_tc_gru_fwd2 a_z = [C_z|H]·L_z, a_r = [C_r|H]·L_r   (MMA, K = 2H, N = H each)
//                 Z, R = σ(·+l);  RH = R⊙H
//                 a_h = [C_h|RH]·L_h → Ĥ = tanh, H' = Z⊙H + (1−Z)⊙Ĥ
//   k_tc_gru_bwd2 recompute a_z, a_r, a_h (as above), then
//                 [dC_h|dRH] = da_h·L_hᵀ, [dC_z|dH_z] = da_z·L_zᵀ, [dC_r|dH_r] = da_r·L_rᵀ
//                 (MMA, K = H, N = 2H each) and the elementwise chain rule;
//                 writes dC' = n_dst⊙dC, dH_prev, and da = [da_z|da_r|da_h], RH
//                 for the parameter-gradient reduction
//   k_tc_atb2     D = Σ_rows A[r,:]ᵀ·B[r,:] with A, B loaded by TMA in the MN-major
//                 layout (K = rows), per-CTA partials, fixed-order reduction → dW, dL, dl.
//
// The equations are those of SURVEY §8(c) (readings C13-C15).
#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>
#include <vector>

#include "common.cuh"
#include "tc.cuh"

namespace stg {
namespace {

constexpr int kTcThreads = 128;

__device__ __forceinline__ float sigm(float a) { return 1.0f / (1.0f + expf(-a)); }

__device__ __forceinline__ void sync_mma_operands() {
  tc::fence_proxy_async();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
}

__device__ __forceinline__ void wait_mma(uint64_t* mbar, uint32_t& phase) {
  tc::mbar_wait(mbar, phase);
  phase ^= 1u;
  tc::fence_after();
}

// Chained 3xTF32 MMAs over a list of K segments of 8-column steps:
// segment s contributes A columns [a_k0, a_k0 + len) and B columns [b_k0, b_k0 + len).
__device__ __forceinline__ void mma_seg(uint32_t d, uint32_t ahi, uint32_t alo, int a_K, int a_k0, uint32_t bhi,
                                        uint32_t blo, int b_K, int b_k0, int len, uint32_t idesc, bool first) {
  const uint32_t sa = (uint32_t)(a_K / 4) * 128, sb = (uint32_t)(b_K / 4) * 128;
  for (int k = 0; k < len; k += 8) {
    const uint32_t oa = (uint32_t)((a_k0 + k) / 4) * 128, ob = (uint32_t)((b_k0 + k) / 4) * 128;
    const uint32_t acc = (first && k == 0) ? 0u : 1u;
    tc::mma_tf32(d, tc::desc(alo + oa, 128, sa), tc::desc(bhi + ob, 128, sb), idesc, acc);
    tc::mma_tf32(d, tc::desc(ahi + oa, 128, sa), tc::desc(blo + ob, 128, sb), idesc, 1u);
    tc::mma_tf32(d, tc::desc(ahi + oa, 128, sa), tc::desc(bhi + ob, 128, sb), idesc, 1u);
  }
}

// A warp can only touch its TMEM lane quarter (warp % 4): lanes 32·(w%4) + lane.
// 3xTF32 chain over two TRANSPOSED tiles (padded layout, K = RK rows).
__device__ __forceinline__ void mma_T(uint32_t d, uint32_t ahi, uint32_t alo, uint32_t bhi, uint32_t blo, int RK,
                                      uint32_t idesc, bool first) {
  const uint32_t sb = tc::sbo_t(RK);
  for (int k = 0; k < RK; k += 8) {
    const uint32_t o = (uint32_t)(k / 4) * tc::kLboT;
    const uint32_t acc = (first && k == 0) ? 0u : 1u;
    tc::mma_tf32(d, tc::desc(alo + o, tc::kLboT, sb), tc::desc(bhi + o, tc::kLboT, sb), idesc, acc);
    tc::mma_tf32(d, tc::desc(ahi + o, tc::kLboT, sb), tc::desc(blo + o, tc::kLboT, sb), idesc, 1u);
    tc::mma_tf32(d, tc::desc(ahi + o, tc::kLboT, sb), tc::desc(bhi + o, tc::kLboT, sb), idesc, 1u);
  }
}

__device__ __forceinline__ uint32_t tmem_row(uint32_t base, int col) {
  return base + ((uint32_t)(((threadIdx.x >> 5) & 3) * 32) << 16) + (uint32_t)col;
}

template <int N>
__device__ __forceinline__ void tmem_row_load(uint32_t base, int col, float (&v)[N]) {
  static_assert(N % 8 == 0, "N % 8");
#pragma unroll
  for (int c = 0; c + 16 <= N; c += 16) {
    float t[16];
    tc::tmem_ld16(tmem_row(base, col + c), t);
#pragma unroll
    for (int i = 0; i < 16; ++i) v[c + i] = t[i];
  }
  if (N % 16) {
    float t[8];
    tc::tmem_ld8(tmem_row(base, col + (N / 16) * 16), t);
#pragma unroll
    for (int i = 0; i < 8; ++i) v[(N / 16) * 16 + i] = t[i];
  }
  tc::tmem_wait_ld();
}

// ------------------------------------------------------------------ X·W
// smem: B = Wᵀ [N × Kp] (hi, lo), A = X tile [128 × Kp] (hi, lo).
template <int N>
__global__ void __launch_bounds__(kTcThreads) k_tc_xw(int V, int F, int Kp, const float* __restrict__ X,
                                                      const float* __restrict__ W, const float* __restrict__ rs,
                                                      float* __restrict__ P) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ uint64_t mbar;
  __shared__ uint32_t tslot;
  unsigned char* bhi = sm;
  unsigned char* blo = bhi + N * Kp * 4;
  unsigned char* ahi = blo + N * Kp * 4;
  unsigned char* alo = ahi + 128 * Kp * 4;
  constexpr uint32_t NC = N <= 32 ? 32 : (N <= 64 ? 64 : (N <= 128 ? 128 : 256));
  tc::stage_weight_T(bhi, blo, W, F, N, Kp, N);
  for (int i = threadIdx.x; i < 128 * Kp; i += kTcThreads) {      // zero the K padding once
    reinterpret_cast<float*>(ahi)[i] = 0.f;
    reinterpret_cast<float*>(alo)[i] = 0.f;
  }
  if ((threadIdx.x >> 5) == 0) tc::tmem_alloc(&tslot, NC);
  if (threadIdx.x == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  uint32_t phase = 0;
  const uint32_t idesc = tc::idesc_tf32(128, N, 0, 0);
  const int ntiles = (V + 127) / 128;
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int r0 = tile * 128;
    tc::stage_rows(ahi, alo, X + (int64_t)r0 * F, F, V - r0, 128, F, 0, 0, Kp);
    sync_mma_operands();
    if (threadIdx.x == 0) {
      mma_seg(tm, tc::smem_u32(ahi), tc::smem_u32(alo), Kp, 0, tc::smem_u32(bhi), tc::smem_u32(blo), Kp, 0, Kp, idesc,
              true);
      tc::commit(&mbar);
    }
    wait_mma(&mbar, phase);
    const int row = r0 + threadIdx.x;
    float v[N];
    tmem_row_load<N>(tm, 0, v);
    if (row < V) {
      const float s = rs ? rs[row] : 1.0f;
      float4* out = reinterpret_cast<float4*>(P + (int64_t)row * N);
#pragma unroll
      for (int c = 0; c < N / 4; ++c) out[c] = make_float4(s * v[4 * c], s * v[4 * c + 1], s * v[4 * c + 2], s * v[4 * c + 3]);
    }
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
  }
  tc::fence_before();
  __syncthreads();
  if ((threadIdx.x >> 5) == 0) tc::tmem_free(tm, NC);
}

// ------------------------------------------------------------------ X·W, pipelined
// Warp-specialised persistent kernel (13 warps):
//   warps 4-11 producers, two groups of 4 warps taking alternate tiles: each
//              group stages its tile (3xTF32 hi/lo split) into its own slot of
//              a 2-slot shared-memory ring and arrives full[slot]; the group's
//              next tile is loaded into registers before it waits for the
//              slot to free up, so two tiles of loads are in flight per SM;
//   warp  12   one lane issues the tcgen05 MMAs of a tile into one of two TMEM
//              accumulators and commits empty[slot] and tfull[acc];
//   warps 0-3  epilogue: thread = tile row = TMEM lane, tcgen05.ld, release
//              the accumulator (tempty[acc]), scale by n_src, and store P'
//              through a per-warp shared stage so that lanes write consecutive
//              16-byte chunks (a thread-per-row store pattern is capped at
//              ~2.5 TB/s, scripts/store_bench.py).
constexpr int kXwThreads = 416;
constexpr int kXwStages = 2;

template <int N>
__global__ void __launch_bounds__(kXwThreads, 1) k_tc_xw_pipe(int V, int F, int Kp, const float* __restrict__ X,
                                                              const float* __restrict__ W,
                                                              const float* __restrict__ rs, float* __restrict__ P,
                                                              int rs_div,
                                                              const __grid_constant__ CUtensorMap tmP,
                                                              const float* __restrict__ bias) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ uint64_t full[kXwStages], empty[kXwStages], tfull[2], tempty[2];
  __shared__ uint32_t tslot;
  constexpr uint32_t NC = N <= 32 ? 32 : (N <= 64 ? 64 : (N <= 128 ? 128 : 256));
  constexpr int NQ = N / 4;
  const int ABYTES = 128 * Kp * 4;
  unsigned char* bhi = sm;
  unsigned char* blo = bhi + N * Kp * 4;
  unsigned char* abase = blo + N * Kp * 4;
  auto ahi = [&](int st) { return abase + (size_t)st * 2 * ABYTES; };
  auto alo = [&](int st) { return abase + (size_t)st * 2 * ABYTES + ABYTES; };
  float4* ostage = reinterpret_cast<float4*>(abase + (size_t)kXwStages * 2 * ABYTES);   // 4 warps x 32 rows
  const int warp = threadIdx.x >> 5;
  tc::stage_weight_T(bhi, blo, W, F, N, Kp, N);
  for (int i = threadIdx.x; i < kXwStages * 2 * 128 * Kp; i += blockDim.x)   // zero the K padding once
    reinterpret_cast<float*>(abase)[i] = 0.f;
  if (warp == 12) tc::tmem_alloc(&tslot, 2 * NC);
  if (threadIdx.x == 0) {
    for (int st = 0; st < kXwStages; ++st) { tc::mbar_init(&full[st], 128); tc::mbar_init(&empty[st], 1); }
    for (int b = 0; b < 2; ++b) { tc::mbar_init(&tfull[b], 1); tc::mbar_init(&tempty[b], 128); }
    tc::fence_mbar_init();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  const int ntiles = (V + 127) / 128;
  if (warp >= 4 && warp < 12) {                      // ---- producers (group = slot)
    // a 128 x F (F <= 64) tile = at most 16 float4 per producer thread
    const int grp = (warp - 4) >> 2, tid = threadIdx.x - 128 - 128 * grp;
    float4 v[16];
    int tile = blockIdx.x + grp * gridDim.x;
    if (tile < ntiles) tc::grp_load<16>(v, X + (int64_t)tile * 128 * F, F, V - tile * 128, 128, F, 0, tid, 128);
    for (int k = 0; tile < ntiles; tile += 2 * gridDim.x, ++k) {
      if (k > 0) tc::mbar_wait(&empty[grp], (k - 1) & 1);
      tc::grp_store<16>(v, ahi(grp), alo(grp), 128, F, 0, Kp, tid, 128);
      tc::fence_proxy_async();
      tc::mbar_arrive(&full[grp]);
      const int nt = tile + 2 * gridDim.x;
      if (nt < ntiles) tc::grp_load<16>(v, X + (int64_t)nt * 128 * F, F, V - nt * 128, 128, F, 0, tid, 128);
    }
  } else if (warp == 12) {                           // ---- MMA issuer
    if ((threadIdx.x & 31) == 0) {
      const uint32_t idesc = tc::idesc_tf32(128, N, 0, 0);
      int i = 0;
      for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++i) {
        const int st = i & 1, k = i >> 1;            // tile i lives in slot i % 2, accumulator i % 2
        tc::mbar_wait(&full[st], k & 1);
        if (k > 0) tc::mbar_wait(&tempty[st], (k - 1) & 1);
        tc::fence_after();
        mma_seg(tm + st * NC, tc::smem_u32(ahi(st)), tc::smem_u32(alo(st)), Kp, 0, tc::smem_u32(bhi),
                  tc::smem_u32(blo), Kp, 0, Kp, idesc, true);
        tc::commit(&empty[st]);
        tc::commit(&tfull[st]);
      }
    }
  } else if (warp < 4) {                             // ---- epilogue, TMA box stores
    unsigned char* obuf = reinterpret_cast<unsigned char*>(
        (reinterpret_cast<uintptr_t>(abase + (size_t)kXwStages * 2 * ABYTES) + 1023) & ~uintptr_t(1023)) + warp * 4096;
    int oslot = 0;
    int i = 0;
    for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++i) {
      const int b = i & 1, kb = i >> 1;
      const int row = tile * 128 + threadIdx.x;
      const float sc = (rs && row < V) ? __ldg(rs + row / rs_div) : 1.0f;
      tc::mbar_wait(&tfull[b], kb & 1);
      tc::fence_after();
      const int wr0 = tile * 128 + warp * 32;
#pragma unroll
      for (int c0 = 0; c0 < N; c0 += 16) {               // TMEM -> registers -> swizzled box -> TMA store
        float v[16];
        tmem_row_load<16>(tm + b * NC, c0, v);
        if (c0 + 16 >= N) {                               // accumulator b fully read: release it early
          tc::fence_before();
          tc::mbar_arrive(&tempty[b]);
        }
        if (bias) {                                       // C = (ÂX)·W + b (aggregate-first order, NEXT-1)
#pragma unroll
          for (int j = 0; j < 16; ++j) v[j] = __fadd_rn(__fmul_rn(v[j], sc), __ldg(bias + c0 + j));
          tc::warp_box_store<16>(obuf, oslot, v, 1.0f, &tmP, c0, wr0);
        } else {
          tc::warp_box_store<16>(obuf, oslot, v, sc, &tmP, c0, wr0);
        }
      }
    }
    if ((threadIdx.x & 31) == 0) tc::bulk_wait_all();  // output boxes written before the CTA exits
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 12) tc::tmem_free(tm, 2 * NC);
}

// ------------------------------------------------------------------ GRU shared pieces
// Weight operands (K-major [N × K], hi/lo):
//   Bz [H × 2H]: (j, k<H) = L_z¹[k][j], (j, H+k) = L_z²[k][j]   (likewise Br, Bh)
//   Lz, Lr, Lh as stored [2H × H] are directly the K-major operands of the
//   backward products da_g·L_gᵀ (rows n = output feature, k = j).
template <int H>
struct GruSmem {
  static constexpr int BG = H * 2 * H * 4;                // bytes of one [H × 2H] (or [2H × H]) tile
  static constexpr int A1 = 128 * 3 * H * 4;              // A tile [128 × 3H]
};

template <int H>
__device__ __forceinline__ void stage_gate_weights(unsigned char* hi, unsigned char* lo, const float* __restrict__ Lg) {
  // Lg: [2H][H] row-major; target (j, k) with k in [0, 2H): Lg[k][j]
  tc::stage_weight_T(hi, lo, Lg, 2 * H, H, 2 * H, H);
}

template <int H>
__device__ __forceinline__ void stage_plain(unsigned char* hi, unsigned char* lo, const float* __restrict__ Lg) {
  // Lg [2H][H] row-major is already K-major as [N = 2H rows × K = H]
  for (int e = threadIdx.x; e < 2 * H * H; e += blockDim.x) {
    const int n = e / H, k = e % H;
    const float v = Lg[e];
    const float h = tc::tf32_hi(v);
    *reinterpret_cast<float*>(hi + tc::kmaj_off(n, k, H)) = h;
    *reinterpret_cast<float*>(lo + tc::kmaj_off(n, k, H)) = v - h;
  }
}

// A1 = [C_z | C_r | H] (width 3H); the z and r gates are K-segment chains over it.
template <int H>
__device__ __forceinline__ void issue_zr(uint32_t tm, unsigned char* ahi, unsigned char* alo, unsigned char* bz_hi,
                                         unsigned char* bz_lo, unsigned char* br_hi, unsigned char* br_lo) {
  const uint32_t idesc = tc::idesc_tf32(128, H, 0, 0);
  const uint32_t a_h = tc::smem_u32(ahi), a_l = tc::smem_u32(alo);
  // z: [C_z | H] · Bz
  mma_seg(tm + 0, a_h, a_l, 3 * H, 0, tc::smem_u32(bz_hi), tc::smem_u32(bz_lo), 2 * H, 0, H, idesc, true);
  mma_seg(tm + 0, a_h, a_l, 3 * H, 2 * H, tc::smem_u32(bz_hi), tc::smem_u32(bz_lo), 2 * H, H, H, idesc, false);
  // r: [C_r | H] · Br
  mma_seg(tm + H, a_h, a_l, 3 * H, H, tc::smem_u32(br_hi), tc::smem_u32(br_lo), 2 * H, 0, H, idesc, true);
  mma_seg(tm + H, a_h, a_l, 3 * H, 2 * H, tc::smem_u32(br_hi), tc::smem_u32(br_lo), 2 * H, H, H, idesc, false);
}

// ------------------------------------------------------------------ GRU forward
// 256 threads: thread t owns tile row (w % 4)·32 + lane (its TMEM lane) and the
// column half (w / 4) of every H-wide quantity.  All GRU epilogue math is
// column-local; the column mixing happens in the MMAs.
constexpr int kGruThreads = 256;

// ------------------------------------------------------------------ GRU forward, v2
// One persistent CTA per SM, 8 warps; thread = (tile row = TMEM lane, column
// half).  Inputs arrive by 2-D TMA tensor loads (boxes of 128 rows x 32 fp32,
// 128-byte swizzle, so the row-per-lane reads below are bank-conflict-free)
// into a double-buffered raw tile; tile i+2 is requested as soon as tile i
// has been moved into tensor memory.  The MMA A operands live in TENSOR
// MEMORY (tcgen05.mma ... [a_tmem]): the hardware reads fp32 as tf32 by
// truncation (pinned by tests/test_gpu_tc.py), so hi = the raw value and only
// lo = x - trunc(x) is computed.  TMEM columns (units of H):
//   [0,3H) [C_z|C_r|H] hi, [3H,6H) lo, [6H,7H) C_h hi, [7H,8H) lo,
//   [8H,9H) acc z, [9H,10H) acc r, [10H,11H) RH hi, [11H,12H) lo, [12H,13H) acc h.
// H' leaves through a per-warp shared stage (coalesced 64-byte row segments).
constexpr int kBox = 128 * 32 * 4;       // one TMA box: 128 rows x 32 fp32 (16 KB)

template <int H>
struct GruF2 {
  static constexpr int H3 = 3 * H, HH = H / 2, NQ = HH / 4;
  static constexpr int NBC = (H3 + 31) / 32, NBH = (H + 31) / 32;   // boxes per C / H tile
  static constexpr int RAW = (NBC + NBH) * kBox;
  static constexpr int BG = H * 2 * H * 4;
  static constexpr int OBUF = 2 * 32 * HH * 4;                     // per-warp output box buffers
  static constexpr int WOFF = 2 * RAW;                              // weights after the raw buffers
  static constexpr int SMEM = WOFF + 6 * BG + 8 * OBUF + 1024;      // + alignment slack
  static constexpr uint32_t TCOLS = 13 * H <= 256 ? 256 : 512;
};

// 3xTF32 chain with A in tensor memory (columns a_hi.., a_lo..) and B in smem.
__device__ __forceinline__ void mma_ts_seg(uint32_t d, uint32_t a_hi, uint32_t a_lo, uint32_t bhi, uint32_t blo,
                                           int b_K, int b_k0, int len, uint32_t idesc, bool first) {
  const uint32_t sb = (uint32_t)(b_K / 4) * 128;
  for (int k = 0; k < len; k += 8) {
    const uint32_t ob = (uint32_t)((b_k0 + k) / 4) * 128;
    const uint64_t dh = tc::desc(bhi + ob, 128, sb), dl = tc::desc(blo + ob, 128, sb);
    tc::mma_tf32_ts(d, a_lo + k, dh, idesc, (first && k == 0) ? 0u : 1u);
    tc::mma_tf32_ts(d, a_hi + k, dl, idesc, 1u);
    tc::mma_tf32_ts(d, a_hi + k, dh, idesc, 1u);
  }
}

// HH fp32 values (columns col..col+HH of row r) of a raw tile made of 128x32
// swizzled boxes -> TMEM (hi = raw, lo = raw - trunc(raw)) at columns (t_hi, t_lo)
template <int HH>
__device__ __forceinline__ void raw_to_tmem(const unsigned char* tile, int r, int col, uint32_t t_hi, uint32_t t_lo,
                                            float (&v)[HH]) {
  const unsigned char* box = tile + (col / 32) * kBox;
  const int c16 = (col % 32) / 4;
#pragma unroll
  for (int q = 0; q < HH / 4; ++q) {
    const float4 x = tc::lds128(tc::smem_u32(box) + tc::swz128(r, c16 + q));
    v[4 * q] = x.x; v[4 * q + 1] = x.y; v[4 * q + 2] = x.z; v[4 * q + 3] = x.w;
  }
  float lo[HH];
#pragma unroll
  for (int j = 0; j < HH; ++j) lo[j] = v[j] - tc::tf32_hi(v[j]);
  if constexpr (HH == 16) {
    tc::tmem_st16(t_hi, v);
    tc::tmem_st16(t_lo, lo);
  } else {
    static_assert(HH == 8, "HH");
    tc::tmem_st8(t_hi, v);
    tc::tmem_st8(t_lo, lo);
  }
}

template <int H, bool HEAD>
__global__ void __launch_bounds__(256, 1) k_tc_gru_fwd2(int V, const __grid_constant__ CUtensorMap tmC,
                                                        const __grid_constant__ CUtensorMap tmH,
                                                        const float* __restrict__ L, const float* __restrict__ l,
                                                        const __grid_constant__ CUtensorMap tmHn,
                                                        const HeadArgs hd) {
  using G = GruF2<H>;
  constexpr int HH = G::HH, NQ = G::NQ;
  __shared__ float s_dot[2][128];
  __shared__ uint32_t s_mk[2][128];
  __shared__ float s_red[8][HH + 1];
  __shared__ double s_l[8];
  extern __shared__ unsigned char sm_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(sm_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[2], mma_bar;
  __shared__ uint32_t tslot;
  // [Bz; Br] hi and lo are each one contiguous N = 2H operand (the z and r gates' H parts
  // run as one N = 2H product into the adjacent accumulators z | r)
  unsigned char* bz_hi = sm + G::WOFF;  unsigned char* br_hi = bz_hi + G::BG;
  unsigned char* bz_lo = br_hi + G::BG; unsigned char* br_lo = bz_lo + G::BG;
  unsigned char* bh_hi = br_lo + G::BG; unsigned char* bh_lo = bh_hi + G::BG;
  auto rawC = [&](int b) { return sm + (size_t)b * G::RAW; };
  auto rawH = [&](int b) { return sm + (size_t)b * G::RAW + G::NBC * kBox; };
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, q = warp & 3, hf = warp >> 2;
  const int lr = q * 32 + lane, c0 = hf * HH;
  unsigned char* obuf = bh_lo + G::BG + warp * G::OBUF;          // this warp's two output box buffers
  int oslot = 0;
  const int LG = 2 * H * H;
  stage_gate_weights<H>(bz_hi, bz_lo, L);
  stage_gate_weights<H>(br_hi, br_lo, L + LG);
  stage_gate_weights<H>(bh_hi, bh_lo, L + 2 * LG);
  if (warp == 0) tc::tmem_alloc(&tslot, G::TCOLS);
  if (threadIdx.x == 0) {
    tc::mbar_init(&full[0], 1); tc::mbar_init(&full[1], 1); tc::mbar_init(&mma_bar, 1);
    tc::fence_mbar_init();
  }
  tc::fence_proxy_async();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  const uint32_t tq = tm + ((uint32_t)(q * 32) << 16);   // this thread's TMEM lane quarter
  const int ntiles = (V + 127) / 128;
  float lz[HH], lrr[HH], lh[HH];
#pragma unroll
  for (int j = 0; j < HH; ++j) { lz[j] = l[c0 + j]; lrr[j] = l[H + c0 + j]; lh[j] = l[2 * H + c0 + j]; }
  // fused surrogate head (HEAD): per-thread partials of Σ e², Σ g·ReLU(H'), Σ g
  float wo[HEAD ? HH : 1], gw[HEAD ? HH : 1];
  float bo = 0.f, gb = 0.f;
  double lacc = 0.0;
  if (HEAD) {
#pragma unroll
    for (int j = 0; j < HH; ++j) { wo[j] = hd.w_o[c0 + j]; gw[j] = 0.f; }
    bo = hd.b_o[0];
  }
  auto issue = [&](int tile, int b) {                   // (thread 0) TMA boxes of tile into raw buffer b
    if (tile >= ntiles) return;
    tc::mbar_expect_tx(&full[b], (uint32_t)(G::NBC + G::NBH) * kBox);
#pragma unroll
    for (int k = 0; k < G::NBC; ++k) tc::tma_load_2d(rawC(b) + k * kBox, &tmC, 32 * k, tile * 128, &full[b]);
    tc::tma_load_2d(rawH(b), &tmH, 0, tile * 128, &full[b]);
  };
  if (threadIdx.x == 0) {
    issue(blockIdx.x, 0);
    issue(blockIdx.x + gridDim.x, 1);
  }
  const uint32_t idesc = tc::idesc_tf32(128, H, 0, 0), idesc2 = tc::idesc_tf32(128, 2 * H, 0, 0);
  uint32_t mph = 0;
  int i = 0;
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++i) {
    const int b = i & 1, r0 = tile * 128;
    const float yv = (HEAD && r0 + lr < V) ? __ldg(hd.y + r0 + lr) : 0.f;   // issued before the waits
    tc::mbar_wait(&full[b], (i >> 1) & 1);
    // raw tile -> tensor-memory A operands; this thread's half of H stays in registers
    float h[HH];
    {
      float t[HH];
      raw_to_tmem<HH>(rawC(b), lr, c0, tq + c0, tq + 3 * H + c0, t);                    // C_z
      raw_to_tmem<HH>(rawC(b), lr, H + c0, tq + H + c0, tq + 4 * H + c0, t);            // C_r
      raw_to_tmem<HH>(rawC(b), lr, 2 * H + c0, tq + 6 * H + c0, tq + 7 * H + c0, t);    // C_h
      raw_to_tmem<HH>(rawH(b), lr, c0, tq + 2 * H + c0, tq + 5 * H + c0, h);            // H
    }
    tc::tmem_wait_st();
    tc::fence_before();
    __syncthreads();
    if (threadIdx.x == 0) {
      tc::fence_after();
      const uint32_t zh = tc::smem_u32(bz_hi), zl = tc::smem_u32(bz_lo), rh_ = tc::smem_u32(br_hi), rl = tc::smem_u32(br_lo);
      mma_ts_seg(tm + 8 * H, tm + 0, tm + 3 * H, zh, zl, 2 * H, 0, H, idesc, true);          // z: C_z part
      mma_ts_seg(tm + 9 * H, tm + H, tm + 4 * H, rh_, rl, 2 * H, 0, H, idesc, true);         // r: C_r part
      mma_ts_seg(tm + 8 * H, tm + 2 * H, tm + 5 * H, zh, zl, 2 * H, H, H, idesc2, false);    // z | r: H part
      tc::commit(&mma_bar);
      issue(tile + 2 * gridDim.x, b);                  // raw buffer b is free
    }
    tc::mbar_wait(&mma_bar, mph);
    mph ^= 1;
    tc::fence_after();
    float z[HH];
    {
      float az[HH], ar[HH], rh[HH], lo[HH];
      tmem_row_load<HH>(tm + 8 * H, c0, az);
      tmem_row_load<HH>(tm + 9 * H, c0, ar);
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        z[j] = sigm(az[j] + lz[j]);
        rh[j] = sigm(ar[j] + lrr[j]) * h[j];
        lo[j] = rh[j] - tc::tf32_hi(rh[j]);
      }
      if constexpr (HH == 16) { tc::tmem_st16(tq + 10 * H + c0, rh); tc::tmem_st16(tq + 11 * H + c0, lo); }
      else { tc::tmem_st8(tq + 10 * H + c0, rh); tc::tmem_st8(tq + 11 * H + c0, lo); }
    }
    tc::tmem_wait_st();
    tc::fence_before();
    __syncthreads();
    if (threadIdx.x == 0) {
      tc::fence_after();
      const uint32_t hh_ = tc::smem_u32(bh_hi), hl = tc::smem_u32(bh_lo);
      mma_ts_seg(tm + 12 * H, tm + 6 * H, tm + 7 * H, hh_, hl, 2 * H, 0, H, idesc, true);    // h: C_h part
      mma_ts_seg(tm + 12 * H, tm + 10 * H, tm + 11 * H, hh_, hl, 2 * H, H, H, idesc, false); //    RH part
      tc::commit(&mma_bar);
    }
    tc::mbar_wait(&mma_bar, mph);
    mph ^= 1;
    tc::fence_after();
    {
      float ah[HH], o[HH];
      tmem_row_load<HH>(tm + 12 * H, c0, ah);
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        const float hh = tanhf(ah[j] + lh[j]);
        o[j] = z[j] * h[j] + (1.0f - z[j]) * hh;
      }
      tc::warp_box_store<HH>(obuf, oslot, o, 1.0f, &tmHn, c0, r0 + q * 32);    // H'
      if (HEAD) {        // ŷ = ReLU(H')·w_o + b_o, e = ŷ − y, g = 2e / V_total (the head's dℓ/dŷ)
        float dot = 0.f;
        uint32_t mk = 0;
#pragma unroll
        for (int j = 0; j < HH; ++j) {
          dot = fmaf(fmaxf(o[j], 0.f), wo[j], dot);
          mk |= (o[j] > 0.f ? 1u : 0u) << j;
        }
        s_dot[hf][lr] = dot;
        s_mk[hf][lr] = mk << c0;
        __syncthreads();
        const int row = r0 + lr;
        if (row < V) {
          const float e = (s_dot[0][lr] + s_dot[1][lr] + bo) - yv;
          const float g = 2.0f * e * hd.inv_v;
          if (hf == 0) {
            lacc += (double)e * (double)e;
            gb += g;
            hd.hg[row] = make_float2(g, __uint_as_float(s_mk[0][lr] | s_mk[1][lr]));
          }
#pragma unroll
          for (int j = 0; j < HH; ++j) gw[j] = fmaf(g, fmaxf(o[j], 0.f), gw[j]);
        }
        __syncthreads();                               // s_dot / s_mk reused by the next tile
      }
    }
    tc::fence_before();
  }
  if (lane == 0) tc::bulk_wait_all();                // output boxes written before the CTA exits
  if (HEAD) {        // fixed-order CTA partials: lanes (xor tree), then the 4 row-quarter warps in order
#pragma unroll
    for (int o = 16; o; o >>= 1) {
#pragma unroll
      for (int j = 0; j < HH; ++j) gw[j] += __shfl_xor_sync(0xffffffffu, gw[j], o);
      gb += __shfl_xor_sync(0xffffffffu, gb, o);
      lacc += __shfl_xor_sync(0xffffffffu, lacc, o);
    }
    if (lane == 0) {
#pragma unroll
      for (int j = 0; j < HH; ++j) s_red[warp][j] = gw[j];
      s_red[warp][HH] = gb;
      s_l[warp] = lacc;
    }
    __syncthreads();
    if (threadIdx.x <= H) {
      const int k = threadIdx.x;
      float t = 0.f;
      if (k < H) {
        const int h2 = k / HH, jj = k % HH;
        for (int qq = 0; qq < 4; ++qq) t += s_red[h2 * 4 + qq][jj];
      } else {
        for (int qq = 0; qq < 4; ++qq) t += s_red[qq][HH];      // hf == 0 warps carry Σ g
      }
      hd.gpart[(int64_t)blockIdx.x * (H + 1) + k] = t;
    }
    if (threadIdx.x == 0) {
      double t = 0.0;
      for (int qq = 0; qq < 4; ++qq) t += s_l[qq];
      hd.lpart[blockIdx.x] = t;
    }
  }
  __syncthreads();
  if (warp == 0) tc::tmem_free(tm, G::TCOLS);
}


// ------------------------------------------------------------------ GRU backward, v2
// Same data path as k_tc_gru_fwd2 (TMA boxes -> swizzled raw tile -> tensor
// memory A operands; single raw buffer: the next tile is requested as soon as
// the current one is in TMEM, so its loads overlap the four MMA phases):
//   P1 z, r  (recompute, [C_z|H]·L_z, [C_r|H]·L_r)      P2 h ([C_h|RH]·L_h)
//   P3 [dC_h|dRH] = da_h·L_hᵀ, [dC_z|dH_z] = da_z·L_zᵀ  P4 [dC_r|dH_r] = da_r·L_rᵀ
// TMEM columns (units of H): P1/P2 as in k_tc_gru_fwd2; afterwards
//   [0,H) da_h hi, [H,2H) lo, [2H,3H) da_z hi, [3H,4H) lo, [4H,6H) acc P3h,
//   [6H,8H) acc P3z, [10H,11H) da_r hi, [11H,12H) lo, [8H,10H) acc P4.
// Outputs dC' = n_dst ⊙ dC, dH_prev, da = [da_z|da_r|da_h], RH leave through
// the per-warp shared stage (coalesced 64-byte row segments).
template <int H>
struct GruB2 {
  static constexpr int H3 = 3 * H, HH = H / 2, NQ = HH / 4;
  static constexpr int NBC = (H3 + 31) / 32, NBH = (H + 31) / 32;
  static constexpr int RAW = (NBC + 2 * NBH) * kBox;                // C, H, G
  static constexpr int BG = H * 2 * H * 4;
  static constexpr int OBUF = 2 * 32 * HH * 4;                     // per-warp output box buffers
  static constexpr int WOFF = RAW;
  static constexpr int SMEM = WOFF + 12 * BG + 8 * OBUF + 1024;
  static constexpr uint32_t TCOLS = 13 * H <= 256 ? 256 : 512;
};

template <int HH>
__device__ __forceinline__ void tmem_st_split(uint32_t t_hi, uint32_t t_lo, const float (&v)[HH]) {
  float lo[HH];
#pragma unroll
  for (int j = 0; j < HH; ++j) lo[j] = v[j] - tc::tf32_hi(v[j]);
  if constexpr (HH == 16) {
    tc::tmem_st16(t_hi, v);
    tc::tmem_st16(t_lo, lo);
  } else {
    tc::tmem_st8(t_hi, v);
    tc::tmem_st8(t_lo, lo);
  }
}

// stage this thread's HH values (times s) as its row of the warp stage and flush to dst
template <int HH>
__device__ __forceinline__ void stage_flush(float4* stage, const float (&v)[HH], float s, float* dst, int64_t ld,
                                            int row0, int nvalid) {
  constexpr int NQ = HH / 4;
  float4* srow = stage + (threadIdx.x & 31) * tc::kStagePitch<NQ>;
#pragma unroll
  for (int qq = 0; qq < NQ; ++qq)
    srow[qq] = make_float4(s * v[4 * qq], s * v[4 * qq + 1], s * v[4 * qq + 2], s * v[4 * qq + 3]);
  tc::flush_stage_rows<NQ>(stage, dst, ld, row0, nvalid);
}

template <int H, bool HEADG>
__global__ void __launch_bounds__(256, 1) k_tc_gru_bwd2(int V, const __grid_constant__ CUtensorMap tmC,
                                                        const __grid_constant__ CUtensorMap tmH,
                                                        const __grid_constant__ CUtensorMap tmG,
                                                        const float* __restrict__ L, const float* __restrict__ l,
                                                        const float* __restrict__ ndst,
                                                        const __grid_constant__ CUtensorMap tmDC,
                                                        const __grid_constant__ CUtensorMap tmDH,
                                                        const __grid_constant__ CUtensorMap tmDA,
                                                        const __grid_constant__ CUtensorMap tmRH,
                                                        const float2* __restrict__ hg, const float* __restrict__ w_o) {
  using G = GruB2<H>;
  constexpr int H3 = G::H3, HH = G::HH;
  extern __shared__ unsigned char sm_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(sm_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full, mma_bar;
  __shared__ uint32_t tslot;
  unsigned char* w0 = sm + G::WOFF;
  unsigned char* bz_hi = w0;              unsigned char* br_hi = w0 + 1 * G::BG;   // [Bz; Br] contiguous (as fwd2)
  unsigned char* bz_lo = w0 + 2 * G::BG;  unsigned char* br_lo = w0 + 3 * G::BG;
  unsigned char* bh_hi = w0 + 4 * G::BG;  unsigned char* bh_lo = w0 + 5 * G::BG;
  unsigned char* lz_hi = w0 + 6 * G::BG;  unsigned char* lz_lo = w0 + 7 * G::BG;
  unsigned char* lr_hi = w0 + 8 * G::BG;  unsigned char* lr_lo = w0 + 9 * G::BG;
  unsigned char* lh_hi = w0 + 10 * G::BG; unsigned char* lh_lo = w0 + 11 * G::BG;
  unsigned char* rawC = sm;
  unsigned char* rawH = sm + G::NBC * kBox;
  unsigned char* rawG = sm + (G::NBC + G::NBH) * kBox;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, q = warp & 3, hf = warp >> 2;
  const int lr = q * 32 + lane, c0 = hf * HH;
  unsigned char* obuf = w0 + 12 * G::BG + warp * G::OBUF;       // this warp's two output box buffers
  int oslot = 0;
  __shared__ float s_l[3 * H];                                   // gate biases
  for (int e = threadIdx.x; e < 3 * H; e += blockDim.x) s_l[e] = l[e];
  const int LG = 2 * H * H;
  stage_gate_weights<H>(bz_hi, bz_lo, L);
  stage_gate_weights<H>(br_hi, br_lo, L + LG);
  stage_gate_weights<H>(bh_hi, bh_lo, L + 2 * LG);
  stage_plain<H>(lz_hi, lz_lo, L);
  stage_plain<H>(lr_hi, lr_lo, L + LG);
  stage_plain<H>(lh_hi, lh_lo, L + 2 * LG);
  if (warp == 0) tc::tmem_alloc(&tslot, G::TCOLS);
  if (threadIdx.x == 0) {
    tc::mbar_init(&full, 1); tc::mbar_init(&mma_bar, 1);
    tc::fence_mbar_init();
  }
  tc::fence_proxy_async();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  const uint32_t tq = tm + ((uint32_t)(q * 32) << 16);
  const int ntiles = (V + 127) / 128;
  auto issue = [&](int tile) {                          // (thread 0) TMA boxes of tile into the raw buffer
    if (tile >= ntiles) return;
    tc::mbar_expect_tx(&full, (uint32_t)(G::NBC + 2 * G::NBH) * kBox);
#pragma unroll
    for (int k = 0; k < G::NBC; ++k) tc::tma_load_2d(rawC + k * kBox, &tmC, 32 * k, tile * 128, &full);
    tc::tma_load_2d(rawH, &tmH, 0, tile * 128, &full);
    tc::tma_load_2d(rawG, &tmG, 0, tile * 128, &full);
  };
  if (threadIdx.x == 0) issue(blockIdx.x);
  const uint32_t id_h = tc::idesc_tf32(128, H, 0, 0), id_2h = tc::idesc_tf32(128, 2 * H, 0, 0);
  auto mma_wait = [&](uint32_t& ph) {
    tc::mbar_wait(&mma_bar, ph);
    ph ^= 1;
    tc::fence_after();
  };
  auto sync_tmem = [&]() {                              // thread-written TMEM visible to the MMA issuer
    tc::tmem_wait_st();
    tc::fence_before();
    __syncthreads();
  };
  uint32_t mph = 0;
  int i = 0;
  float wog[HEADG ? HH : 1];                           // this thread's columns of w_o (head gradient)
#pragma unroll
  for (int j = 0; j < (HEADG ? HH : 1); ++j) wog[j] = HEADG ? __ldg(w_o + c0 + j) : 0.f;
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++i) {
    const int r0 = tile * 128, wr0 = r0 + q * 32;
    const int row = r0 + lr;
    const float nd = row < V ? (ndst ? __ldg(ndst + row) : 1.0f) : 0.f;   // (NULL: dC unscaled, aggregate-first)
    const float2 hv = (HEADG && row < V) ? __ldg(hg + row) : make_float2(0.f, 0.f);   // issued before the waits
    tc::mbar_wait(&full, i & 1);
    float h[HH], g[HH];
    {
      float t[HH];
      raw_to_tmem<HH>(rawC, lr, c0, tq + c0, tq + 3 * H + c0, t);                    // C_z
      raw_to_tmem<HH>(rawC, lr, H + c0, tq + H + c0, tq + 4 * H + c0, t);            // C_r
      raw_to_tmem<HH>(rawC, lr, 2 * H + c0, tq + 6 * H + c0, tq + 7 * H + c0, t);    // C_h
      raw_to_tmem<HH>(rawH, lr, c0, tq + 2 * H + c0, tq + 5 * H + c0, h);            // H
      const unsigned char* box = rawG + (c0 / 32) * kBox;
#pragma unroll
      for (int qq = 0; qq < HH / 4; ++qq) {
        const float4 x = tc::lds128(tc::smem_u32(box) + tc::swz128(lr, (c0 % 32) / 4 + qq));
        g[4 * qq] = x.x; g[4 * qq + 1] = x.y; g[4 * qq + 2] = x.z; g[4 * qq + 3] = x.w;
      }
      if (HEADG && row < V) {            // G = dH from step t+1 + the head's g·w_o ⊙ [H' > 0]
        const uint32_t mk = __float_as_uint(hv.y) >> c0;
#pragma unroll
        for (int j = 0; j < HH; ++j)
          if ((mk >> j) & 1u) g[j] = __fadd_rn(g[j], __fmul_rn(hv.x, wog[j]));
      }
    }
    sync_tmem();
    if (threadIdx.x == 0) {                             // P1; then request the next tile
      tc::fence_after();
      const uint32_t zh = tc::smem_u32(bz_hi), zl = tc::smem_u32(bz_lo), rh_ = tc::smem_u32(br_hi), rl = tc::smem_u32(br_lo);
      mma_ts_seg(tm + 8 * H, tm + 0, tm + 3 * H, zh, zl, 2 * H, 0, H, id_h, true);          // z: C_z part
      mma_ts_seg(tm + 9 * H, tm + H, tm + 4 * H, rh_, rl, 2 * H, 0, H, id_h, true);         // r: C_r part
      mma_ts_seg(tm + 8 * H, tm + 2 * H, tm + 5 * H, zh, zl, 2 * H, H, H, id_2h, false);    // z | r: H part
      tc::commit(&mma_bar);
      issue(tile + gridDim.x);
    }
    mma_wait(mph);
    float z[HH], r[HH];
    {
      float az[HH], ar[HH], rh[HH];
      tmem_row_load<HH>(tm + 8 * H, c0, az);
      tmem_row_load<HH>(tm + 9 * H, c0, ar);
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        z[j] = sigm(az[j] + s_l[c0 + j]);
        r[j] = sigm(ar[j] + s_l[H + c0 + j]);
        rh[j] = r[j] * h[j];
      }
      tmem_st_split<HH>(tq + 10 * H + c0, tq + 11 * H + c0, rh);
      sync_tmem();
      if (threadIdx.x == 0) {                           // P2
        tc::fence_after();
        const uint32_t hh_ = tc::smem_u32(bh_hi), hl = tc::smem_u32(bh_lo);
        mma_ts_seg(tm + 12 * H, tm + 6 * H, tm + 7 * H, hh_, hl, 2 * H, 0, H, id_h, true);
        mma_ts_seg(tm + 12 * H, tm + 10 * H, tm + 11 * H, hh_, hl, 2 * H, H, H, id_h, false);
        tc::commit(&mma_bar);
      }
      tc::warp_box_store<HH>(obuf, oslot, rh, 1.0f, &tmRH, c0, wr0);       // RH (for dL_h²), overlaps P2
    }
    mma_wait(mph);
    float dh[HH];
    {
      float ah[HH], dah[HH], daz[HH];
      tmem_row_load<HH>(tm + 12 * H, c0, ah);
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        const float hh = tanhf(ah[j] + s_l[2 * H + c0 + j]);
        const float dZ = g[j] * (h[j] - hh), dHh = g[j] * (1.0f - z[j]);
        dah[j] = dHh * (1.0f - hh * hh);
        daz[j] = dZ * z[j] * (1.0f - z[j]);
        dh[j] = g[j] * z[j];
      }
      // P1/P2 operands are consumed: reuse [0,4H) for da_h, da_z
      tmem_st_split<HH>(tq + c0, tq + H + c0, dah);
      tmem_st_split<HH>(tq + 2 * H + c0, tq + 3 * H + c0, daz);
      sync_tmem();
      if (threadIdx.x == 0) {                           // P3
        tc::fence_after();
        mma_ts_seg(tm + 4 * H, tm + 0, tm + H, tc::smem_u32(lh_hi), tc::smem_u32(lh_lo), H, 0, H, id_2h, true);
        mma_ts_seg(tm + 6 * H, tm + 2 * H, tm + 3 * H, tc::smem_u32(lz_hi), tc::smem_u32(lz_lo), H, 0, H, id_2h, true);
        tc::commit(&mma_bar);
      }
      tc::warp_box_store<HH>(obuf, oslot, daz, 1.0f, &tmDA, c0, wr0);      // da_z
      tc::warp_box_store<HH>(obuf, oslot, dah, 1.0f, &tmDA, 2 * H + c0, wr0);   // da_h
    }
    mma_wait(mph);
    {
      float dch[HH], drh[HH], dar[HH];
      tmem_row_load<HH>(tm + 4 * H, c0, dch);          // dC_h
      tmem_row_load<HH>(tm + 5 * H, c0, drh);          // dRH
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        dh[j] += drh[j] * r[j];
        dar[j] = drh[j] * h[j] * r[j] * (1.0f - r[j]);
      }
      tmem_st_split<HH>(tq + 10 * H + c0, tq + 11 * H + c0, dar);
      sync_tmem();
      if (threadIdx.x == 0) {                           // P4
        tc::fence_after();
        mma_ts_seg(tm + 8 * H, tm + 10 * H, tm + 11 * H, tc::smem_u32(lr_hi), tc::smem_u32(lr_lo), H, 0, H, id_2h, true);
        tc::commit(&mma_bar);
      }
      tc::warp_box_store<HH>(obuf, oslot, dch, nd, &tmDC, 2 * H + c0, wr0);     // dC'_h
      tc::warp_box_store<HH>(obuf, oslot, dar, 1.0f, &tmDA, H + c0, wr0);  // da_r
      float dcz[HH], dhz[HH];
      tmem_row_load<HH>(tm + 6 * H, c0, dcz);          // dC_z
      tmem_row_load<HH>(tm + 7 * H, c0, dhz);          // dH_z
#pragma unroll
      for (int j = 0; j < HH; ++j) dh[j] += dhz[j];
      tc::warp_box_store<HH>(obuf, oslot, dcz, nd, &tmDC, c0, wr0);        // dC'_z
    }
    mma_wait(mph);
    {
      float dcr[HH], dhr[HH];
      tmem_row_load<HH>(tm + 8 * H, c0, dcr);          // dC_r
      tmem_row_load<HH>(tm + 9 * H, c0, dhr);          // dH_r
#pragma unroll
      for (int j = 0; j < HH; ++j) dh[j] += dhr[j];
      tc::warp_box_store<HH>(obuf, oslot, dcr, nd, &tmDC, H + c0, wr0);    // dC'_r
      tc::warp_box_store<HH>(obuf, oslot, dh, 1.0f, &tmDH, c0, wr0);       // dH_prev
    }
    tc::fence_before();
    __syncthreads();                                   // TMEM / stage reuse by the next tile
  }
  if (lane == 0) tc::bulk_wait_all();                // output boxes written before the CTA exits
  if (warp == 0) tc::tmem_free(tm, G::TCOLS);
}

// ------------------------------------------------------------------ Σ_rows Aᵀ·B, v2 (TMA, MN-major)
// D_a[128 x N] = Σ_r A_a[r,:]ᵀ B[r,:] for one or two A operands, both operands
// loaded by 2-D TMA boxes (RT rows x 32 fp32) straight into the UMMA MN-major
// SWIZZLE_128B_BASE32B layout (K = rows; pinned by tests/test_gpu_tc.py mode 4):
// no transposition by threads; hi = the raw fp32 (hardware truncation) and
// lo = x - trunc(x) is computed in place, elementwise, by 4 converter warps.
// A stage is a row of box slots [A slots | B slots]; A operand a covers 4
// consecutive slots from a_first[a] (M = 128 features, one 32-feature chunk per
// slot): slots past an operand's real boxes hold the following boxes, so the
// corresponding D rows are garbage that is never read (rows are independent).
// A slot is a TMA box or the static "ones" box (1.0 in feature 0 of every row:
// the Σ_rows term of dl).  Warp 0 issues the TMA, warp 1 the MMAs, warps 2-5
// convert and run the epilogue.  The raw (hi) boxes sit in an S-stage TMA ring;
// lo is written into a separate 2-slot ring (a tile is converted just before its
// MMAs), so the shared memory goes to loads in flight rather than to lo copies.  Each CTA accumulates its tiles (grid-stride, fixed) in TMEM and
// writes its partial; k_tc_sum_parts adds the partials in a fixed order.
struct AtbSpec2 {
  int V;
  int na;                 // 1 or 2 A operands
  int a_first[2];         // first slot of each A operand
  int nsa;                // A slots in a stage (<= 8)
  int src_map[8];         // A slot source: tensor map 0..3, or -2 = ones box
  int src_col[8];
  int nb;                 // B boxes (N = 32 nb), from map b_map at columns 32 k
  int b_map;
  float* part;            // [gridDim][na][128][N]
};

template <int NB, int RT, int S, int L = 2>
__global__ void __launch_bounds__(192, 1) k_tc_atb2(const __grid_constant__ CUtensorMap m0,
                                                    const __grid_constant__ CUtensorMap m1,
                                                    const __grid_constant__ CUtensorMap m2,
                                                    const __grid_constant__ CUtensorMap m3,
                                                    const __grid_constant__ CUtensorMap m_ones, const AtbSpec2 sp) {
  constexpr int N = 32 * NB;
  constexpr int BOX = RT * 32 * 4;
  extern __shared__ unsigned char sm_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(sm_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[S], empty[S], conv[L], lfree[L], done, init_bar;
  __shared__ uint32_t tslot;
  const int na = sp.na, nsa = sp.nsa;
  const int nbox = nsa + NB;                       // box slots per stage
  const size_t half = (size_t)nbox * BOX;          // one stage (hi ring) or one lo slot
  auto hi = [&](int st, int bx) { return sm + (size_t)st * half + (size_t)bx * BOX; };
  auto lo = [&](int ls, int bx) { return sm + (size_t)(S + ls) * half + (size_t)bx * BOX; };
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  auto map_of = [&](int m) -> const CUtensorMap* { return m == 0 ? &m0 : (m == 1 ? &m1 : (m == 2 ? &m2 : &m3)); };
  for (size_t e = threadIdx.x; e < (size_t)(S + L) * half / 16; e += blockDim.x)   // lo of the ones box stays 0
    reinterpret_cast<float4*>(sm)[e] = make_float4(0.f, 0.f, 0.f, 0.f);
  const uint32_t tcols = na * N <= 128 ? 128 : 256;
  if (warp == 1) tc::tmem_alloc(&tslot, tcols);
  if (threadIdx.x == 0) {
    for (int st = 0; st < S; ++st) { tc::mbar_init(&full[st], 1); tc::mbar_init(&empty[st], 1); }
    for (int ls = 0; ls < L; ++ls) { tc::mbar_init(&conv[ls], 128); tc::mbar_init(&lfree[ls], 1); }
    tc::mbar_init(&done, 1); tc::mbar_init(&init_bar, 1);
    tc::fence_mbar_init();
  }
  tc::fence_proxy_async();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  int n_ones = 0;
  uint32_t ones_mask = 0;
  for (int k = 0; k < nsa; ++k)
    if (sp.src_map[k] < 0) { n_ones += sp.src_map[k] == -2; ones_mask |= 1u << k; }
  if (n_ones) {                                      // the ones box (hardware swizzle) into each stage
    if (threadIdx.x == 0) {
      tc::mbar_expect_tx(&init_bar, (uint32_t)(n_ones * S * BOX));
      for (int st = 0; st < S; ++st)
        for (int k = 0; k < nsa; ++k)
          if (sp.src_map[k] == -2) tc::tma_load_2d(hi(st, k), &m_ones, 0, 0, &init_bar);
    }
    tc::mbar_wait(&init_bar, 0);
  }
  const uint32_t tm = tslot;
  const int ntiles = (sp.V + RT - 1) / RT;
  int my_tiles = 0;
  for (int t = blockIdx.x; t < ntiles; t += gridDim.x) ++my_tiles;
  if (warp == 0) {                                   // ---- TMA producer
    if (lane == 0) {
      int bytes = NB * BOX;
      for (int k = 0; k < nsa; ++k) bytes += sp.src_map[k] >= 0 ? BOX : 0;
      for (int i = 0; i < my_tiles; ++i) {
        const int st = i % S, kk = i / S, r0 = (blockIdx.x + i * gridDim.x) * RT;
        if (kk > 0) tc::mbar_wait(&empty[st], (kk - 1) & 1);
        tc::mbar_expect_tx(&full[st], (uint32_t)bytes);
        for (int k = 0; k < nsa; ++k)
          if (sp.src_map[k] >= 0) tc::tma_load_2d(hi(st, k), map_of(sp.src_map[k]), sp.src_col[k], r0, &full[st]);
        for (int k = 0; k < NB; ++k) tc::tma_load_2d(hi(st, nsa + k), map_of(sp.b_map), 32 * k, r0, &full[st]);
      }
    }
  } else if (warp == 1) {                            // ---- MMA issuer
    if (lane == 0) {
      const uint32_t idesc = tc::idesc_tf32(128, N, 1, 1);
      for (int i = 0; i < my_tiles; ++i) {
        const int st = i % S, ls = i % L;
        tc::mbar_wait(&conv[ls], (i / L) & 1);
        tc::fence_after();
        const uint32_t bh = tc::smem_u32(hi(st, nsa)), bl = tc::smem_u32(lo(ls, nsa));
        for (int a = 0; a < na; ++a) {
          const uint32_t ah = tc::smem_u32(hi(st, sp.a_first[a])), al = tc::smem_u32(lo(ls, sp.a_first[a]));
          for (int k = 0; k < RT; k += 8) {                // 8 K-rows (1024 B) per MMA
            const uint32_t o = (uint32_t)k * 128;
            const uint64_t dah = tc::desc_mn_sw128_32b(ah + o, BOX), dal = tc::desc_mn_sw128_32b(al + o, BOX);
            const uint64_t dbh = tc::desc_mn_sw128_32b(bh + o, BOX), dbl = tc::desc_mn_sw128_32b(bl + o, BOX);
            const uint32_t d = tm + a * N;
            tc::mma_tf32(d, dal, dbh, idesc, (i > 0 || k > 0) ? 1u : 0u);
            tc::mma_tf32(d, dah, dbl, idesc, 1u);
            tc::mma_tf32(d, dah, dbh, idesc, 1u);
          }
        }
        tc::commit(&empty[st]);
        tc::commit(&lfree[ls]);
      }
      tc::commit(&done);
    }
  } else {                                           // ---- converters (warps 2-5), then epilogue
    const int ct = threadIdx.x - 64;
    for (int i = 0; i < my_tiles; ++i) {
      const int st = i % S, ls = i % L;
      tc::mbar_wait(&full[st], (i / S) & 1);
      if (i >= L) tc::mbar_wait(&lfree[ls], ((i / L) - 1) & 1);   // MMAs of tile i-L done with slot ls
      // the stage's boxes are contiguous: 8 shared loads in flight per thread, then the lo stores
      const uint32_t hb = tc::smem_u32(hi(st, 0)), lb = tc::smem_u32(lo(ls, 0));
      constexpr int B4 = BOX / 16;                    // float4 per box
      for (int e0 = ct; e0 < nbox * B4; e0 += 8 * 128) {
        float4 v[8];
#pragma unroll
        for (int j = 0; j < 8; ++j)
          if (e0 + 128 * j < nbox * B4) v[j] = tc::lds128(hb + 16u * (uint32_t)(e0 + 128 * j));
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int e = e0 + 128 * j;
          if (e < nbox * B4 && !((ones_mask >> (e / B4)) & 1u))   // ones box: lo stays 0
            tc::sts128(lb + 16u * (uint32_t)e,
                       make_float4(v[j].x - tc::tf32_hi(v[j].x), v[j].y - tc::tf32_hi(v[j].y),
                                   v[j].z - tc::tf32_hi(v[j].z), v[j].w - tc::tf32_hi(v[j].w)));
        }
      }
      tc::fence_proxy_async();
      tc::mbar_arrive(&conv[ls]);
    }
    // epilogue: this warp reads TMEM lane quarter warp % 4
    tc::mbar_wait(&done, 0);
    tc::fence_after();
    const int q = warp & 3, row = q * 32 + lane;
    float* out = sp.part + (size_t)blockIdx.x * na * 128 * N;
    for (int c = 0; c < na * N; c += 8) {
      float v[8];
      if (my_tiles == 0) {
#pragma unroll
        for (int e = 0; e < 8; ++e) v[e] = 0.f;
      } else {
        tc::tmem_ld8(tm + ((uint32_t)(q * 32) << 16) + (uint32_t)c, v);
        tc::tmem_wait_ld();
      }
      const int a = c / N, cc = c % N;
#pragma unroll
      for (int e = 0; e < 8; ++e) out[(size_t)a * 128 * N + (size_t)row * N + cc + e] = v[e];
    }
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 1) tc::tmem_free(tm, tcols);
}

// ------------------------------------------------------------------ dL, gate-blocked (H = 32)
// Only the gate-diagonal blocks of Σ_rows [C|H]ᵀ·da are parameter gradients:
//   D_g = Σ_rows [C_g | H_g' | ones]ᵀ · da_g,   H_z' = H_r' = H, H_h' = RH,
// rows 0..H-1 → dL_g¹, rows H..2H-1 → dL_g², row 2H → dl_g (the ones feature).
// Three M = 128, N = 32 products per tile instead of two M = 128, N = 96 ones
// (half the 3xTF32 tensor work, TMEM 96 columns).  Each A operand is 4 box slots
// LBO apart in the stage (slots 0..10, BOX bytes each):
//   0 C_z  1 C_r  2 H  3 ones  4 ones  5 C_h  6 RH  7 ones  8 da_z  9 da_r  10 da_h
//   A_z = slots 0, 2, 4, 6 (LBO 2 boxes)   A_r = 1, 2, 3, 4   A_h = 5, 6, 7, 8
// (the 4th chunk of each is another operand: D rows 96..127, never read).  The
// ones boxes are static (hi = 1.0 in feature 0, lo = 0); warp 0 issues the TMA,
// warp 1 the MMAs, warps 2-5 convert (lo = x − trunc x) and run the epilogue.
constexpr int kDl3Slots = 11;
template <int RT, int S, int L>
__global__ void __launch_bounds__(192, 1) k_tc_dl3(const __grid_constant__ CUtensorMap mC,
                                                   const __grid_constant__ CUtensorMap mH,
                                                   const __grid_constant__ CUtensorMap mRH,
                                                   const __grid_constant__ CUtensorMap mDA,
                                                   const __grid_constant__ CUtensorMap m_ones, int V,
                                                   float* __restrict__ part) {
  constexpr int BOX = RT * 32 * 4;
  constexpr int NS = kDl3Slots;
  constexpr uint32_t ONES = (1u << 3) | (1u << 4) | (1u << 7);
  extern __shared__ unsigned char sm_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(sm_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[S], empty[S], conv[L], lfree[L], done, init_bar;
  __shared__ uint32_t tslot;
  constexpr size_t half = (size_t)NS * BOX;          // one stage (hi ring) or one lo slot
  auto hi = [&](int st, int bx) { return sm + (size_t)st * half + (size_t)bx * BOX; };
  auto lo = [&](int ls, int bx) { return sm + (size_t)(S + ls) * half + (size_t)bx * BOX; };
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (size_t e = threadIdx.x; e < (size_t)(S + L) * half / 16; e += blockDim.x)   // lo of the ones boxes stays 0
    reinterpret_cast<float4*>(sm)[e] = make_float4(0.f, 0.f, 0.f, 0.f);
  if (warp == 1) tc::tmem_alloc(&tslot, 128);
  if (threadIdx.x == 0) {
    for (int st = 0; st < S; ++st) { tc::mbar_init(&full[st], 1); tc::mbar_init(&empty[st], 1); }
    for (int ls = 0; ls < L; ++ls) { tc::mbar_init(&conv[ls], 128); tc::mbar_init(&lfree[ls], 1); }
    tc::mbar_init(&done, 1); tc::mbar_init(&init_bar, 1);
    tc::fence_mbar_init();
  }
  tc::fence_proxy_async();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  if (threadIdx.x == 0) {                            // the static ones boxes of every stage
    tc::mbar_expect_tx(&init_bar, (uint32_t)(3 * S * BOX));
    for (int st = 0; st < S; ++st)
      for (int k = 0; k < NS; ++k)
        if ((ONES >> k) & 1u) tc::tma_load_2d(hi(st, k), &m_ones, 0, 0, &init_bar);
  }
  tc::mbar_wait(&init_bar, 0);
  const uint32_t tm = tslot;
  const int ntiles = (V + RT - 1) / RT;
  int my_tiles = 0;
  for (int t = blockIdx.x; t < ntiles; t += gridDim.x) ++my_tiles;
  if (warp == 0) {                                   // ---- TMA producer
    if (lane == 0) {
      for (int i = 0; i < my_tiles; ++i) {
        const int st = i % S, kk = i / S, r0 = (blockIdx.x + i * gridDim.x) * RT;
        if (kk > 0) tc::mbar_wait(&empty[st], (kk - 1) & 1);
        tc::mbar_expect_tx(&full[st], (uint32_t)(8 * BOX));
        tc::tma_load_2d(hi(st, 0), &mC, 0, r0, &full[st]);
        tc::tma_load_2d(hi(st, 1), &mC, 32, r0, &full[st]);
        tc::tma_load_2d(hi(st, 5), &mC, 64, r0, &full[st]);
        tc::tma_load_2d(hi(st, 2), &mH, 0, r0, &full[st]);
        tc::tma_load_2d(hi(st, 6), &mRH, 0, r0, &full[st]);
        tc::tma_load_2d(hi(st, 8), &mDA, 0, r0, &full[st]);
        tc::tma_load_2d(hi(st, 9), &mDA, 32, r0, &full[st]);
        tc::tma_load_2d(hi(st, 10), &mDA, 64, r0, &full[st]);
      }
    }
  } else if (warp == 1) {                            // ---- MMA issuer
    if (lane == 0) {
      const uint32_t idesc = tc::idesc_tf32(128, 32, 1, 1);
      const int a_slot[3] = {0, 1, 5}, b_slot[3] = {8, 9, 10};
      const uint32_t lbo[3] = {2u * BOX, (uint32_t)BOX, (uint32_t)BOX};
      for (int i = 0; i < my_tiles; ++i) {
        const int st = i % S, ls = i % L;
        tc::mbar_wait(&conv[ls], (i / L) & 1);
        tc::fence_after();
#pragma unroll
        for (int g = 0; g < 3; ++g) {
          const uint32_t ah = tc::smem_u32(hi(st, a_slot[g])), al = tc::smem_u32(lo(ls, a_slot[g]));
          const uint32_t bh = tc::smem_u32(hi(st, b_slot[g])), bl = tc::smem_u32(lo(ls, b_slot[g]));
          const uint32_t d = tm + 32 * g;
          for (int k = 0; k < RT; k += 8) {              // 8 K-rows (1024 B) per MMA
            const uint32_t o = (uint32_t)k * 128;
            const uint64_t dah = tc::desc_mn_sw128_32b(ah + o, lbo[g]), dal = tc::desc_mn_sw128_32b(al + o, lbo[g]);
            const uint64_t dbh = tc::desc_mn_sw128_32b(bh + o, BOX), dbl = tc::desc_mn_sw128_32b(bl + o, BOX);
            tc::mma_tf32(d, dal, dbh, idesc, (i > 0 || k > 0) ? 1u : 0u);
            tc::mma_tf32(d, dah, dbl, idesc, 1u);
            tc::mma_tf32(d, dah, dbh, idesc, 1u);
          }
        }
        tc::commit(&empty[st]);
        tc::commit(&lfree[ls]);
      }
      tc::commit(&done);
    }
  } else {                                           // ---- converters (warps 2-5), then epilogue
    const int ct = threadIdx.x - 64;
    for (int i = 0; i < my_tiles; ++i) {
      const int st = i % S, ls = i % L;
      tc::mbar_wait(&full[st], (i / S) & 1);
      if (i >= L) tc::mbar_wait(&lfree[ls], ((i / L) - 1) & 1);   // MMAs of tile i-L done with slot ls
      const uint32_t hb = tc::smem_u32(hi(st, 0)), lb = tc::smem_u32(lo(ls, 0));
      constexpr int B4 = BOX / 16;                    // float4 per box
      for (int e0 = ct; e0 < NS * B4; e0 += 8 * 128) {
        float4 v[8];
#pragma unroll
        for (int j = 0; j < 8; ++j)
          if (e0 + 128 * j < NS * B4) v[j] = tc::lds128(hb + 16u * (uint32_t)(e0 + 128 * j));
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int e = e0 + 128 * j;
          if (e < NS * B4 && !((ONES >> (e / B4)) & 1u))
            tc::sts128(lb + 16u * (uint32_t)e,
                       make_float4(v[j].x - tc::tf32_hi(v[j].x), v[j].y - tc::tf32_hi(v[j].y),
                                   v[j].z - tc::tf32_hi(v[j].z), v[j].w - tc::tf32_hi(v[j].w)));
        }
      }
      tc::fence_proxy_async();
      tc::mbar_arrive(&conv[ls]);
    }
    // epilogue: rows 0..2H of each gate's D (lane quarter warp % 4), part[cta][g][row][32]
    tc::mbar_wait(&done, 0);
    tc::fence_after();
    const int q = warp & 3, row = q * 32 + lane;
    float* out = part + (size_t)blockIdx.x * 3 * 65 * 32;
    for (int c = 0; c < 96; c += 8) {
      float v[8];
      if (my_tiles == 0 || q > 2) {
#pragma unroll
        for (int e = 0; e < 8; ++e) v[e] = 0.f;
      } else {
        tc::tmem_ld8(tm + ((uint32_t)(q * 32) << 16) + (uint32_t)c, v);
        tc::tmem_wait_ld();
      }
      const int g = c / 32, cc = c % 32;
      if (row <= 64) {
#pragma unroll
        for (int e = 0; e < 8; ++e) out[((size_t)g * 65 + row) * 32 + cc + e] = v[e];
      }
    }
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 1) tc::tmem_free(tm, 128);
}

// dL / dl / db from the gate blocks tot[g][row][j] (rows 0..2H-1: [C_g | H_g'], row 2H: ones)
__global__ void k_dl3_scatter(const float* __restrict__ tot, const float* __restrict__ L, float* __restrict__ dL,
                              float* __restrict__ dl, float* __restrict__ db) {
  constexpr int H = 32, LG = 2 * H * H;
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < 6 * H * H + 6 * H; e += gridDim.x * blockDim.x) {
    if (e < 6 * H * H) {
      const int g = e / LG, rem = e % LG, i = rem / H, j = rem % H;
      dL[e] += tot[((size_t)g * 65 + i) * 32 + j];
    } else if (e < 6 * H * H + 3 * H) {
      const int c = e - 6 * H * H, g = c / H, j = c % H;
      dl[c] += tot[((size_t)g * 65 + 64) * 32 + j];
    } else {
      const int c = e - 6 * H * H - 3 * H, g = c / H, i = c % H;      // db_g = dl_g · L_g¹ᵀ
      const float* Lg = L + (int64_t)g * LG;
      float s = 0.f;
      for (int j = 0; j < H; ++j) s = fmaf(tot[((size_t)g * 65 + 64) * 32 + j], Lg[i * H + j], s);
      db[c] += s;
    }
  }
}

// Fixed-order sum of the per-CTA partials: tot[e] = Σ_b part[b][e] (blocks of 16).
__global__ void k_tc_sum_parts(const float* __restrict__ part, int nb, int n, float* __restrict__ tot) {
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < n; e += gridDim.x * blockDim.x) {
    float t = 0.f;
    for (int b0 = 0; b0 < nb; b0 += 16) {
      float blk = 0.f;
      const int b1 = min(b0 + 16, nb);
      for (int b = b0; b < b1; ++b) blk += part[(int64_t)b * n + e];
      t += blk;
    }
    tot[e] = t;
  }
}

// The same sum in the same order, parallel over the 16-partial groups: a block owns 32
// consecutive elements; warp y forms the group sums j = y, y+8, ... (coalesced rows of
// 32), then lane row 0 adds them in group order — bit-identical to k_tc_sum_parts.
constexpr int kSumMaxGroups = 64;                  // nb <= 1024
__global__ void __launch_bounds__(256) k_tc_sum_parts2(const float* __restrict__ part, int nb, int n,
                                                       float* __restrict__ tot) {
  __shared__ float blk[kSumMaxGroups][33];
  const int x = threadIdx.x & 31, y = threadIdx.x >> 5;
  const int e = blockIdx.x * 32 + x;
  const int ng = (nb + 15) / 16;
  for (int j = y; j < ng; j += 8) {
    float b = 0.f;
    if (e < n) {
      const int b0 = 16 * j, b1 = min(b0 + 16, nb);
      float v[16];
#pragma unroll
      for (int k = 0; k < 16; ++k) v[k] = (b0 + k < b1) ? __ldg(part + (int64_t)(b0 + k) * n + e) : 0.f;
#pragma unroll
      for (int k = 0; k < 16; ++k)
        if (b0 + k < b1) b += v[k];
    }
    blk[j][x] = b;
  }
  __syncthreads();
  if (y == 0 && e < n) {
    float t = 0.f;
    for (int j = 0; j < ng; ++j) t += blk[j][x];
    tot[e] = t;
  }
}

// Scatter the dL / dl / db pieces out of tot = [D1 (128 × ldd) | D2 (128 × ldd)]
// (row = A feature, column = da feature: da_z | da_r | da_h, ldd >= 3H):
//   D1 rows: C_z | C_r | C_h (rows 0..3H) | H (rows hoff..hoff+H),
//   D2 rows: RH (rows 0..H) | ones (row orow).
__global__ void k_dl_scatter(int H, int hoff, int orow, int ldd, const float* __restrict__ tot,
                             const float* __restrict__ L, float* __restrict__ dL, float* __restrict__ dl,
                             float* __restrict__ db) {
  const int LG = 2 * H * H;
  const float* D1 = tot;
  const float* D2 = tot + 128 * ldd;
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < 6 * H * H + 6 * H; e += gridDim.x * blockDim.x) {
    if (e < 6 * H * H) {
      const int g = e / LG, rem = e % LG, i = rem / H, j = rem % H;
      float v;
      if (i < H) v = D1[(g * H + i) * ldd + g * H + j];                // C_gᵀ da_g
      else if (g < 2) v = D1[(hoff + i - H) * ldd + g * H + j];       // Hᵀ da_z, Hᵀ da_r
      else v = D2[(i - H) * ldd + 2 * H + j];                         // RHᵀ da_h
      dL[e] += v;
    } else if (e < 6 * H * H + 3 * H) {
      const int c = e - 6 * H * H;
      dl[c] += D2[orow * ldd + c];                                    // ones row: Σ_rows da
    } else {
      const int c = e - 6 * H * H - 3 * H, g = c / H, i = c % H;      // db_g = dl_g · L_g¹ᵀ
      const float* Lg = L + (int64_t)g * LG;
      float s = 0.f;
      for (int j = 0; j < H; ++j) s = fmaf(D2[orow * ldd + g * H + j], Lg[i * H + j], s);
      db[c] += s;
    }
  }
}

// dW[f][c] += tot[c][f]  (tot = D = dPᵀ·X, [128 × Np])
__global__ void k_dw_scatter(int F, int N3, int Np, const float* __restrict__ tot, float* __restrict__ dW) {
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < F * N3; e += gridDim.x * blockDim.x) {
    const int f = e / N3, c = e % N3;
    dW[e] += tot[c * Np + f];
  }
}

// ------------------------------------------------------------------ sequence-batched GRU (NEXT-1)
// Static graphs: C_t = Â(X_t W) + b does not depend on H, so a whole sequence's
// aggregations run as ONE width-S·3H SpMM and the GRU recurrence, being
// row-local, runs for all S timestamps inside one persistent kernel: a CTA
// walks t = 0..S-1 (forward) or S-1..0 (backward) for each of its row tiles,
// carrying H (forward) / dH (backward) in registers.  Layouts: C_all, dC'_all,
// da_all [V][S][3H]; Hp_all [V][S][H] (slot t = H_{t-1}); RH_all [V][S][H];
// H_seq [S][V][H] (the API's); Y_all [V][S].  The MSE head is fused: the
// forward accumulates the loss, the backward the head gradient (G = dℓ_t/dH_t
// + dH from t+1) and dw_o, db_o — per-CTA partials, reduced in a fixed order.
template <int H>
__device__ __forceinline__ float row_dot_relu(const float (&hv)[H / 2], const float* __restrict__ w, int c0) {
  float d = 0.f;
#pragma unroll
  for (int j = 0; j < H / 2; ++j) d = fmaf(fmaxf(hv[j], 0.f), w[c0 + j], d);
  return d;
}

template <int H>
__global__ void __launch_bounds__(256, 1) k_tc_gru_seq_fwd(int V, int S, const __grid_constant__ CUtensorMap tmC,
                                                           const __grid_constant__ CUtensorMap tmH0,
                                                           const float* __restrict__ L, const float* __restrict__ l,
                                                           const __grid_constant__ CUtensorMap tmHseq,
                                                           const __grid_constant__ CUtensorMap tmHp,
                                                           const float* __restrict__ Yall,
                                                           const float* __restrict__ w_o,
                                                           const float* __restrict__ b_o, double* __restrict__ lpart) {
  using G = GruF2<H>;
  constexpr int HH = G::HH, H3 = 3 * H;
  constexpr int RAWC = G::NBC * kBox;                     // one C_t tile; two buffers, then H0, weights, obuf
  extern __shared__ unsigned char sm_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(sm_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[2], h0bar, mma_bar;
  __shared__ uint32_t tslot;
  __shared__ float s_dot[2][128];
  __shared__ double s_loss[8];
  unsigned char* rawH0 = sm + 2 * RAWC;
  unsigned char* bz_hi = rawH0 + kBox;  unsigned char* bz_lo = bz_hi + G::BG;
  unsigned char* br_hi = bz_lo + G::BG; unsigned char* br_lo = br_hi + G::BG;
  unsigned char* bh_hi = br_lo + G::BG; unsigned char* bh_lo = bh_hi + G::BG;
  auto rawC = [&](int b) { return sm + (size_t)b * RAWC; };
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, q = warp & 3, hf = warp >> 2;
  const int lr = q * 32 + lane, c0 = hf * HH;
  unsigned char* obuf = bh_lo + G::BG + warp * G::OBUF;
  int oslot = 0;
  const int LG = 2 * H * H;
  stage_gate_weights<H>(bz_hi, bz_lo, L);
  stage_gate_weights<H>(br_hi, br_lo, L + LG);
  stage_gate_weights<H>(bh_hi, bh_lo, L + 2 * LG);
  if (warp == 0) tc::tmem_alloc(&tslot, G::TCOLS);
  if (threadIdx.x == 0) {
    tc::mbar_init(&full[0], 1); tc::mbar_init(&full[1], 1); tc::mbar_init(&h0bar, 1); tc::mbar_init(&mma_bar, 1);
    tc::fence_mbar_init();
  }
  tc::fence_proxy_async();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  const uint32_t tq = tm + ((uint32_t)(q * 32) << 16);
  const int ntiles = (V + 127) / 128;
  float lz[HH], lrr[HH], lh[HH], wo[HH];
#pragma unroll
  for (int j = 0; j < HH; ++j) {
    lz[j] = l[c0 + j]; lrr[j] = l[H + c0 + j]; lh[j] = l[2 * H + c0 + j]; wo[j] = w_o[c0 + j];
  }
  const float bo = b_o[0];
  int my_tiles = 0;
  for (int tl = blockIdx.x; tl < ntiles; tl += gridDim.x) ++my_tiles;
  const int nitems = my_tiles * S;                         // item i = (tile i / S, t = i % S)
  auto issue = [&](int i) {                                 // (thread 0) C_t boxes of item i (+ H0 at t = 0)
    if (i >= nitems) return;
    const int b = i & 1, tile = blockIdx.x + (i / S) * gridDim.x, t = i % S;
    tc::mbar_expect_tx(&full[b], (uint32_t)G::NBC * kBox);
#pragma unroll
    for (int k = 0; k < G::NBC; ++k) tc::tma_load_2d(rawC(b) + k * kBox, &tmC, t * H3 + 32 * k, tile * 128, &full[b]);
  };
  auto issue_h0 = [&](int i) {                              // (thread 0) H0 box of the tile of item i
    if (i >= nitems) return;
    const int tile = blockIdx.x + (i / S) * gridDim.x;
    tc::mbar_expect_tx(&h0bar, (uint32_t)kBox);
    tc::tma_load_2d(rawH0, &tmH0, 0, tile * 128, &h0bar);
  };
  if (threadIdx.x == 0) { issue(0); issue(1); issue_h0(0); }
  const uint32_t idesc = tc::idesc_tf32(128, H, 0, 0);
  uint32_t mph = 0, h0ph = 0;
  double lacc = 0.0;
  float h[HH];
  for (int i = 0; i < nitems; ++i) {
    const int b = i & 1, tile = blockIdx.x + (i / S) * gridDim.x, t = i % S, r0 = tile * 128;
    const int row = r0 + lr;
    tc::mbar_wait(&full[b], (i >> 1) & 1);
    {
      float tt[HH];
      raw_to_tmem<HH>(rawC(b), lr, c0, tq + c0, tq + 3 * H + c0, tt);                    // C_z
      raw_to_tmem<HH>(rawC(b), lr, H + c0, tq + H + c0, tq + 4 * H + c0, tt);            // C_r
      raw_to_tmem<HH>(rawC(b), lr, 2 * H + c0, tq + 6 * H + c0, tq + 7 * H + c0, tt);    // C_h
      if (t == 0) {                                                                      // H_{-1} = H0
        tc::mbar_wait(&h0bar, h0ph);
        h0ph ^= 1;
        raw_to_tmem<HH>(rawH0, lr, c0, tq + 2 * H + c0, tq + 5 * H + c0, h);
      } else {                                                                           // H_{t-1} from registers
        tmem_st_split<HH>(tq + 2 * H + c0, tq + 5 * H + c0, h);
      }
    }
    tc::warp_box_store<HH>(obuf, oslot, h, 1.0f, &tmHp, t * H + c0, r0 + q * 32);          // Hp_all slot t
    tc::tmem_wait_st();
    tc::fence_before();
    __syncthreads();
    if (threadIdx.x == 0) {
      tc::fence_after();
      const uint32_t zh = tc::smem_u32(bz_hi), zl = tc::smem_u32(bz_lo), rh_ = tc::smem_u32(br_hi), rl = tc::smem_u32(br_lo);
      mma_ts_seg(tm + 8 * H, tm + 0, tm + 3 * H, zh, zl, 2 * H, 0, H, idesc, true);
      mma_ts_seg(tm + 8 * H, tm + 2 * H, tm + 5 * H, zh, zl, 2 * H, H, H, idesc, false);
      mma_ts_seg(tm + 9 * H, tm + H, tm + 4 * H, rh_, rl, 2 * H, 0, H, idesc, true);
      mma_ts_seg(tm + 9 * H, tm + 2 * H, tm + 5 * H, rh_, rl, 2 * H, H, H, idesc, false);
      tc::commit(&mma_bar);
      issue(i + 2);                                       // raw buffer b is in TMEM
      if (t == 0) issue_h0(i + S);                        // the next tile's H0 (rawH0 consumed)
    }
    tc::mbar_wait(&mma_bar, mph);
    mph ^= 1;
    tc::fence_after();
    float z[HH];
    {
      float az[HH], ar[HH], rh[HH], lo[HH];
      tmem_row_load<HH>(tm + 8 * H, c0, az);
      tmem_row_load<HH>(tm + 9 * H, c0, ar);
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        z[j] = sigm(az[j] + lz[j]);
        rh[j] = sigm(ar[j] + lrr[j]) * h[j];
        lo[j] = rh[j] - tc::tf32_hi(rh[j]);
      }
      if constexpr (HH == 16) { tc::tmem_st16(tq + 10 * H + c0, rh); tc::tmem_st16(tq + 11 * H + c0, lo); }
      else { tc::tmem_st8(tq + 10 * H + c0, rh); tc::tmem_st8(tq + 11 * H + c0, lo); }
    }
    tc::tmem_wait_st();
    tc::fence_before();
    __syncthreads();
    if (threadIdx.x == 0) {
      tc::fence_after();
      const uint32_t hh_ = tc::smem_u32(bh_hi), hl = tc::smem_u32(bh_lo);
      mma_ts_seg(tm + 12 * H, tm + 6 * H, tm + 7 * H, hh_, hl, 2 * H, 0, H, idesc, true);
      mma_ts_seg(tm + 12 * H, tm + 10 * H, tm + 11 * H, hh_, hl, 2 * H, H, H, idesc, false);
      tc::commit(&mma_bar);
    }
    tc::mbar_wait(&mma_bar, mph);
    mph ^= 1;
    tc::fence_after();
    {
      float ah[HH];
      tmem_row_load<HH>(tm + 12 * H, c0, ah);
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        const float hh = tanhf(ah[j] + lh[j]);
        h[j] = z[j] * h[j] + (1.0f - z[j]) * hh;          // H_t
      }
    }
    tc::warp_box_store3<HH>(obuf, oslot, h, &tmHseq, c0, r0 + q * 32, t);                // H_seq[t]
    // fused head, forward: loss += (Σ_k ReLU(H_t)·w_o + b_o − y_t)² over the tile's rows
    s_dot[hf][lr] = row_dot_relu<H>(h, wo, 0);
    tc::fence_before();
    __syncthreads();
    if (hf == 0 && row < V) {
      const float e = (s_dot[0][lr] + s_dot[1][lr] + bo) - Yall[(int64_t)row * S + t];
      lacc += (double)e * (double)e;
    }
  }
  // per-CTA loss partial (fixed order: lanes, then warps)
#pragma unroll
  for (int o = 16; o; o >>= 1) lacc += __shfl_xor_sync(0xffffffffu, lacc, o);
  if (lane == 0) s_loss[warp] = lacc;
  if (lane == 0) tc::bulk_wait_all();
  __syncthreads();
  if (threadIdx.x == 0) {
    double tot = 0.0;
    for (int w = 0; w < 8; ++w) tot += s_loss[w];
    lpart[blockIdx.x] = tot;
  }
  if (warp == 0) tc::tmem_free(tm, G::TCOLS);
}

template <int H>
__global__ void __launch_bounds__(256, 1) k_tc_gru_seq_bwd(int V, int S, const __grid_constant__ CUtensorMap tmC,
                                                           const __grid_constant__ CUtensorMap tmHp,
                                                           const __grid_constant__ CUtensorMap tmHs,
                                                           const float* __restrict__ L, const float* __restrict__ l,
                                                           const float* __restrict__ ndst,
                                                           const float* __restrict__ Yall,
                                                           const float* __restrict__ w_o,
                                                           const float* __restrict__ b_o, float inv_vn,
                                                           const __grid_constant__ CUtensorMap tmDC,
                                                           const __grid_constant__ CUtensorMap tmDA,
                                                           const __grid_constant__ CUtensorMap tmRH,
                                                           float* __restrict__ gpart) {
  using G = GruB2<H>;
  constexpr int H3 = G::H3, HH = G::HH;
  extern __shared__ unsigned char sm_raw[];
  unsigned char* sm = reinterpret_cast<unsigned char*>((reinterpret_cast<uintptr_t>(sm_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full, mma_bar;
  __shared__ uint32_t tslot;
  __shared__ float s_l[3 * H];
  __shared__ float s_dot[2][128];
  __shared__ float s_g[4][H + 1];
  unsigned char* w0 = sm + G::WOFF;
  unsigned char* bz_hi = w0;              unsigned char* br_hi = w0 + 1 * G::BG;   // [Bz; Br] contiguous (as fwd2)
  unsigned char* bz_lo = w0 + 2 * G::BG;  unsigned char* br_lo = w0 + 3 * G::BG;
  unsigned char* bh_hi = w0 + 4 * G::BG;  unsigned char* bh_lo = w0 + 5 * G::BG;
  unsigned char* lz_hi = w0 + 6 * G::BG;  unsigned char* lz_lo = w0 + 7 * G::BG;
  unsigned char* lr_hi = w0 + 8 * G::BG;  unsigned char* lr_lo = w0 + 9 * G::BG;
  unsigned char* lh_hi = w0 + 10 * G::BG; unsigned char* lh_lo = w0 + 11 * G::BG;
  unsigned char* rawC = sm;
  unsigned char* rawH = sm + G::NBC * kBox;                 // H_{t-1}
  unsigned char* rawT = sm + (G::NBC + G::NBH) * kBox;      // H_t (the head's input)
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, q = warp & 3, hf = warp >> 2;
  const int lr = q * 32 + lane, c0 = hf * HH;
  unsigned char* obuf = w0 + 12 * G::BG + warp * G::OBUF;
  int oslot = 0;
  for (int e = threadIdx.x; e < 3 * H; e += blockDim.x) s_l[e] = l[e];
  const int LG = 2 * H * H;
  stage_gate_weights<H>(bz_hi, bz_lo, L);
  stage_gate_weights<H>(br_hi, br_lo, L + LG);
  stage_gate_weights<H>(bh_hi, bh_lo, L + 2 * LG);
  stage_plain<H>(lz_hi, lz_lo, L);
  stage_plain<H>(lr_hi, lr_lo, L + LG);
  stage_plain<H>(lh_hi, lh_lo, L + 2 * LG);
  if (warp == 0) tc::tmem_alloc(&tslot, G::TCOLS);
  if (threadIdx.x == 0) {
    tc::mbar_init(&full, 1); tc::mbar_init(&mma_bar, 1);
    tc::fence_mbar_init();
  }
  tc::fence_proxy_async();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  const uint32_t tq = tm + ((uint32_t)(q * 32) << 16);
  const int ntiles = (V + 127) / 128;
  float wo[HH];
#pragma unroll
  for (int j = 0; j < HH; ++j) wo[j] = w_o[c0 + j];
  const float bo = b_o[0];
  int my_tiles = 0;
  for (int tl = blockIdx.x; tl < ntiles; tl += gridDim.x) ++my_tiles;
  const int nitems = my_tiles * S;                         // item i = (tile i / S, t = S-1 - i % S)
  auto issue = [&](int i) {
    if (i >= nitems) return;
    const int tile = blockIdx.x + (i / S) * gridDim.x, t = S - 1 - i % S;
    tc::mbar_expect_tx(&full, (uint32_t)(G::NBC + 2 * G::NBH) * kBox);
#pragma unroll
    for (int k = 0; k < G::NBC; ++k) tc::tma_load_2d(rawC + k * kBox, &tmC, t * H3 + 32 * k, tile * 128, &full);
    tc::tma_load_2d(rawH, &tmHp, t * H, tile * 128, &full);
    tc::tma_load_2d(rawT, &tmHs, 0, t * V + tile * 128, &full);   // H_seq as [S·V, H]: rows past V are
                                                                    // the next plane's, unused (gs = 0 there)
  };
  if (threadIdx.x == 0) issue(0);
  const uint32_t id_h = tc::idesc_tf32(128, H, 0, 0), id_2h = tc::idesc_tf32(128, 2 * H, 0, 0);
  auto mma_wait = [&](uint32_t& ph) {
    tc::mbar_wait(&mma_bar, ph);
    ph ^= 1;
    tc::fence_after();
  };
  auto sync_tmem = [&]() {
    tc::tmem_wait_st();
    tc::fence_before();
    __syncthreads();
  };
  uint32_t mph = 0;
  float dh[HH];                                             // dℓ/dH_t flowing back from t+1
  float gw[HH], gb = 0.f;                                   // head gradient partials (dw_o, db_o)
#pragma unroll
  for (int j = 0; j < HH; ++j) gw[j] = 0.f;
  for (int i = 0; i < nitems; ++i) {
    const int tile = blockIdx.x + (i / S) * gridDim.x, t = S - 1 - i % S;
    const int r0 = tile * 128, wr0 = r0 + q * 32, row = r0 + lr;
    if (t == S - 1) {
#pragma unroll
      for (int j = 0; j < HH; ++j) dh[j] = 0.f;
    }
    const float nd = row < V ? (ndst ? __ldg(ndst + row) : 1.0f) : 0.f;   // (NULL: dC unscaled, aggregate-first)
    tc::mbar_wait(&full, i & 1);
    float h[HH], g[HH];
    {
      float tt[HH], ht[HH];
      raw_to_tmem<HH>(rawC, lr, c0, tq + c0, tq + 3 * H + c0, tt);                    // C_z
      raw_to_tmem<HH>(rawC, lr, H + c0, tq + H + c0, tq + 4 * H + c0, tt);            // C_r
      raw_to_tmem<HH>(rawC, lr, 2 * H + c0, tq + 6 * H + c0, tq + 7 * H + c0, tt);    // C_h
      raw_to_tmem<HH>(rawH, lr, c0, tq + 2 * H + c0, tq + 5 * H + c0, h);            // H_{t-1}
      const unsigned char* box = rawT + (c0 / 32) * kBox;
#pragma unroll
      for (int qq = 0; qq < HH / 4; ++qq) {
        const float4 x = tc::lds128(tc::smem_u32(box) + tc::swz128(lr, (c0 % 32) / 4 + qq));
        ht[4 * qq] = x.x; ht[4 * qq + 1] = x.y; ht[4 * qq + 2] = x.z; ht[4 * qq + 3] = x.w;
      }
      // fused head, backward: gs = 2(ŷ − y)/V_total;  G = gs·w_o⊙[H_t > 0] + dH(t+1)
      s_dot[hf][lr] = row_dot_relu<H>(ht, wo, 0);
      sync_tmem();
      const float yv = row < V ? Yall[(int64_t)row * S + t] : 0.f;
      const float e = (s_dot[0][lr] + s_dot[1][lr] + bo) - yv;
      const float gs = row < V ? 2.0f * e * inv_vn : 0.f;
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        const float r = fmaxf(ht[j], 0.f);
        g[j] = (ht[j] > 0.f ? gs * wo[j] : 0.f) + dh[j];
        gw[j] = fmaf(gs, r, gw[j]);
      }
      if (hf == 0) gb += gs;
    }
    if (threadIdx.x == 0) {                             // P1; then request the next item
      tc::fence_after();
      const uint32_t zh = tc::smem_u32(bz_hi), zl = tc::smem_u32(bz_lo), rh_ = tc::smem_u32(br_hi), rl = tc::smem_u32(br_lo);
      mma_ts_seg(tm + 8 * H, tm + 0, tm + 3 * H, zh, zl, 2 * H, 0, H, id_h, true);
      mma_ts_seg(tm + 8 * H, tm + 2 * H, tm + 5 * H, zh, zl, 2 * H, H, H, id_h, false);
      mma_ts_seg(tm + 9 * H, tm + H, tm + 4 * H, rh_, rl, 2 * H, 0, H, id_h, true);
      mma_ts_seg(tm + 9 * H, tm + 2 * H, tm + 5 * H, rh_, rl, 2 * H, H, H, id_h, false);
      tc::commit(&mma_bar);
      issue(i + 1);
    }
    mma_wait(mph);
    float z[HH], r[HH];
    {
      float az[HH], ar[HH], rh[HH];
      tmem_row_load<HH>(tm + 8 * H, c0, az);
      tmem_row_load<HH>(tm + 9 * H, c0, ar);
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        z[j] = sigm(az[j] + s_l[c0 + j]);
        r[j] = sigm(ar[j] + s_l[H + c0 + j]);
        rh[j] = r[j] * h[j];
      }
      tmem_st_split<HH>(tq + 10 * H + c0, tq + 11 * H + c0, rh);
      sync_tmem();
      if (threadIdx.x == 0) {                           // P2
        tc::fence_after();
        const uint32_t hh_ = tc::smem_u32(bh_hi), hl = tc::smem_u32(bh_lo);
        mma_ts_seg(tm + 12 * H, tm + 6 * H, tm + 7 * H, hh_, hl, 2 * H, 0, H, id_h, true);
        mma_ts_seg(tm + 12 * H, tm + 10 * H, tm + 11 * H, hh_, hl, 2 * H, H, H, id_h, false);
        tc::commit(&mma_bar);
      }
      tc::warp_box_store<HH>(obuf, oslot, rh, 1.0f, &tmRH, t * H + c0, wr0);          // RH_t
    }
    mma_wait(mph);
    float dhn[HH];
    {
      float ah[HH], dah[HH], daz[HH];
      tmem_row_load<HH>(tm + 12 * H, c0, ah);
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        const float hh = tanhf(ah[j] + s_l[2 * H + c0 + j]);
        const float dZ = g[j] * (h[j] - hh), dHh = g[j] * (1.0f - z[j]);
        dah[j] = dHh * (1.0f - hh * hh);
        daz[j] = dZ * z[j] * (1.0f - z[j]);
        dhn[j] = g[j] * z[j];
      }
      tmem_st_split<HH>(tq + c0, tq + H + c0, dah);
      tmem_st_split<HH>(tq + 2 * H + c0, tq + 3 * H + c0, daz);
      sync_tmem();
      if (threadIdx.x == 0) {                           // P3
        tc::fence_after();
        mma_ts_seg(tm + 4 * H, tm + 0, tm + H, tc::smem_u32(lh_hi), tc::smem_u32(lh_lo), H, 0, H, id_2h, true);
        mma_ts_seg(tm + 6 * H, tm + 2 * H, tm + 3 * H, tc::smem_u32(lz_hi), tc::smem_u32(lz_lo), H, 0, H, id_2h, true);
        tc::commit(&mma_bar);
      }
      tc::warp_box_store<HH>(obuf, oslot, daz, 1.0f, &tmDA, t * H3 + c0, wr0);         // da_z
      tc::warp_box_store<HH>(obuf, oslot, dah, 1.0f, &tmDA, t * H3 + 2 * H + c0, wr0); // da_h
    }
    mma_wait(mph);
    {
      float dch[HH], drh[HH], dar[HH];
      tmem_row_load<HH>(tm + 4 * H, c0, dch);
      tmem_row_load<HH>(tm + 5 * H, c0, drh);
#pragma unroll
      for (int j = 0; j < HH; ++j) {
        dhn[j] += drh[j] * r[j];
        dar[j] = drh[j] * h[j] * r[j] * (1.0f - r[j]);
      }
      tmem_st_split<HH>(tq + 10 * H + c0, tq + 11 * H + c0, dar);
      sync_tmem();
      if (threadIdx.x == 0) {                           // P4
        tc::fence_after();
        mma_ts_seg(tm + 8 * H, tm + 10 * H, tm + 11 * H, tc::smem_u32(lr_hi), tc::smem_u32(lr_lo), H, 0, H, id_2h, true);
        tc::commit(&mma_bar);
      }
      tc::warp_box_store<HH>(obuf, oslot, dch, nd, &tmDC, t * H3 + 2 * H + c0, wr0);   // dC'_h
      tc::warp_box_store<HH>(obuf, oslot, dar, 1.0f, &tmDA, t * H3 + H + c0, wr0);     // da_r
      float dcz[HH], dhz[HH];
      tmem_row_load<HH>(tm + 6 * H, c0, dcz);
      tmem_row_load<HH>(tm + 7 * H, c0, dhz);
#pragma unroll
      for (int j = 0; j < HH; ++j) dhn[j] += dhz[j];
      tc::warp_box_store<HH>(obuf, oslot, dcz, nd, &tmDC, t * H3 + c0, wr0);          // dC'_z
    }
    mma_wait(mph);
    {
      float dcr[HH], dhr[HH];
      tmem_row_load<HH>(tm + 8 * H, c0, dcr);
      tmem_row_load<HH>(tm + 9 * H, c0, dhr);
#pragma unroll
      for (int j = 0; j < HH; ++j) dh[j] = dhn[j] + dhr[j];                           // dℓ/dH_{t-1}
      tc::warp_box_store<HH>(obuf, oslot, dcr, nd, &tmDC, t * H3 + H + c0, wr0);      // dC'_r
    }
    tc::fence_before();
    __syncthreads();
  }
  // head-gradient partials of this CTA: rows (lanes, then the 4 lane quarters) in a fixed order
#pragma unroll
  for (int j = 0; j < HH; ++j) {
#pragma unroll
    for (int o = 16; o; o >>= 1) gw[j] += __shfl_xor_sync(0xffffffffu, gw[j], o);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) gb += __shfl_xor_sync(0xffffffffu, gb, o);
  for (int qq = 0; qq < 4; ++qq) {
    if (q == qq && lane == 0) {
#pragma unroll
      for (int j = 0; j < HH; ++j) s_g[qq][c0 + j] = gw[j];
      if (hf == 0) s_g[qq][H] = gb;
    }
  }
  if (lane == 0) tc::bulk_wait_all();
  __syncthreads();
  for (int k = threadIdx.x; k <= H; k += blockDim.x)
    gpart[(int64_t)blockIdx.x * (H + 1) + k] = ((s_g[0][k] + s_g[1][k]) + s_g[2][k]) + s_g[3][k];
  if (warp == 0) tc::tmem_free(tm, G::TCOLS);
}

// fixed-order sum of the per-CTA partials of the fused head: loss (double, ÷ V_total),
// dw_o [H], db_o [1]
__global__ void k_seq_head_reduce(int nb, int H, const double* __restrict__ lpart, const float* __restrict__ gpart,
                                  double inv_vn, float* __restrict__ loss, float* __restrict__ dw_o,
                                  float* __restrict__ db_o) {
  const int k = threadIdx.x;
  if (lpart && k == 0 && loss) {
    double t = 0.0;
    for (int b = 0; b < nb; ++b) t += lpart[b];
    *loss += (float)(t * inv_vn);
  }
  if (gpart && k <= H) {
    float t = 0.f;
    for (int b = 0; b < nb; ++b) t += gpart[(int64_t)b * (H + 1) + k];
    if (k < H) { if (dw_o) dw_o[k] += t; }
    else if (db_o) db_o[0] += t;
  }
}

template <class K>
int occupancy_blocks(K fn, size_t smem, int threads = kTcThreads) {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, threads, smem) != cudaSuccess || per_sm < 1) {
    cudaGetLastError();
    per_sm = 1;
  }
  return per_sm * num_sms();
}

template <class K>
stg_status prep(K fn, size_t smem) {
  STG_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  return STG_OK;
}

}  // namespace

// ------------------------------------------------------------------ host side
bool tc_supported(int F, int H) { return (H == 16 || H == 32) && F % 4 == 0 && F <= 128 && F >= 4; }
// part for tc_dw / tc_dl: tc_atb_max_blocks() · 2 · 128 · 128 floats; tot: 2 · 128 · 128

stg_status tc_xw(int V, int F, int H, const float* X, const float* W, const float* rs, float* P, cudaStream_t s,
                 int rs_div, const float* bias) {
  const int N = 3 * H, Kp = (F + 7) / 8 * 8;
  const int ntiles = (V + 127) / 128;
  if (Kp <= 64) {                     // pipelined kernel (2-stage ring of 128 x Kp tiles + output stage)
    const size_t smem = (size_t)2 * N * Kp * 4 + (size_t)kXwStages * 2 * 128 * Kp * 4 +
                        std::max<size_t>((size_t)128 * (N / 4 + 1 + ((N / 4) & 1)) * 16, 4 * 4096 + 1024);
    const int nb = std::min(ntiles, num_sms());
    CUtensorMap tmP;
    STG_TRY(make_tmap_f32_store(&tmP, P, (uint64_t)V, (uint64_t)N, (uint64_t)N, 16, 32));
    if (H == 32) {
      STG_TRY(prep(k_tc_xw_pipe<96>, smem));
      k_tc_xw_pipe<96><<<nb, kXwThreads, smem, s>>>(V, F, Kp, X, W, rs, P, rs_div, tmP, bias);
    } else {
      STG_TRY(prep(k_tc_xw_pipe<48>, smem));
      k_tc_xw_pipe<48><<<nb, kXwThreads, smem, s>>>(V, F, Kp, X, W, rs, P, rs_div, tmP, bias);
    }
  } else {                            // 64 < F <= 128: one tile per CTA at a time
    if (rs_div != 1) return fail(STG_ERR_INVALID_ARG, "tc_xw: row-scale divisor needs F <= 64");
    if (bias) return fail(STG_ERR_INVALID_ARG, "tc_xw: a bias needs F <= 64");
    const size_t smem = (size_t)2 * N * Kp * 4 + (size_t)2 * 128 * Kp * 4;
    if (H == 32) {
      STG_TRY(prep(k_tc_xw<96>, smem));
      const int nb = std::min(ntiles, occupancy_blocks(k_tc_xw<96>, smem));
      k_tc_xw<96><<<nb, kTcThreads, smem, s>>>(V, F, Kp, X, W, rs, P);
    } else {
      STG_TRY(prep(k_tc_xw<48>, smem));
      const int nb = std::min(ntiles, occupancy_blocks(k_tc_xw<48>, smem));
      k_tc_xw<48><<<nb, kTcThreads, smem, s>>>(V, F, Kp, X, W, rs, P);
    }
  }
  count_launch();
  return check_launch("tc_xw");
}

int tc_gru_blocks(int V) { return std::max(1, std::min((V + 127) / 128, num_sms())); }

stg_status tc_gru_fwd(int V, int H, const float* C, const float* Hp, const float* L, const float* l, float* Hn,
                      cudaStream_t s, const HeadArgs* head) {
  const int ntiles = (V + 127) / 128;
  const int nb = std::min(ntiles, num_sms());
  CUtensorMap tmC, tmH, tmHn;
  STG_TRY(make_tmap_f32(&tmC, C, (uint64_t)V, 3 * H, 3 * H, 32, 128));
  STG_TRY(make_tmap_f32(&tmH, Hp, (uint64_t)V, H, H, 32, 128));
  STG_TRY(make_tmap_f32_store(&tmHn, Hn, (uint64_t)V, H, H, (uint32_t)H / 2, 32));
  if (head) {                                      // fused surrogate head
    if (H == 32) {
      STG_TRY(prep(k_tc_gru_fwd2<32, true>, GruF2<32>::SMEM));
      k_tc_gru_fwd2<32, true><<<nb, 256, GruF2<32>::SMEM, s>>>(V, tmC, tmH, L, l, tmHn, *head);
    } else {
      STG_TRY(prep(k_tc_gru_fwd2<16, true>, GruF2<16>::SMEM));
      k_tc_gru_fwd2<16, true><<<nb, 256, GruF2<16>::SMEM, s>>>(V, tmC, tmH, L, l, tmHn, *head);
    }
  } else if (H == 32) {
    STG_TRY(prep(k_tc_gru_fwd2<32, false>, GruF2<32>::SMEM));
    k_tc_gru_fwd2<32, false><<<nb, 256, GruF2<32>::SMEM, s>>>(V, tmC, tmH, L, l, tmHn, HeadArgs{});
  } else {
    STG_TRY(prep(k_tc_gru_fwd2<16, false>, GruF2<16>::SMEM));
    k_tc_gru_fwd2<16, false><<<nb, 256, GruF2<16>::SMEM, s>>>(V, tmC, tmH, L, l, tmHn, HeadArgs{});
  }
  count_launch();
  return check_launch("tc_gru_fwd");
}

stg_status tc_gru_bwd(int V, int H, const float* C, const float* Hp, const float* G, const float* L, const float* l,
                      const float* ndst, float* dCs, float* dHp, float* da, float* RH, cudaStream_t s,
                      const float2* hg, const float* w_o) {
  const int ntiles = (V + 127) / 128;
  const int nb = std::min(ntiles, num_sms());
  CUtensorMap tmC, tmH, tmG, tmDC, tmDH, tmDA, tmRH;
  STG_TRY(make_tmap_f32(&tmC, C, (uint64_t)V, 3 * H, 3 * H, 32, 128));
  STG_TRY(make_tmap_f32(&tmH, Hp, (uint64_t)V, H, H, 32, 128));
  STG_TRY(make_tmap_f32(&tmG, G, (uint64_t)V, H, H, 32, 128));
  const uint32_t hh = (uint32_t)H / 2;                  // output boxes: 32 rows x H/2 columns per warp
  STG_TRY(make_tmap_f32_store(&tmDC, dCs, (uint64_t)V, 3 * H, 3 * H, hh, 32));
  STG_TRY(make_tmap_f32_store(&tmDH, dHp, (uint64_t)V, H, H, hh, 32));
  STG_TRY(make_tmap_f32_store(&tmDA, da, (uint64_t)V, 3 * H, 3 * H, hh, 32));
  STG_TRY(make_tmap_f32_store(&tmRH, RH, (uint64_t)V, H, H, hh, 32));
#define STG_GRU_BWD(HV, HD)                                                                                  \
  do {                                                                                                       \
    STG_TRY(prep(k_tc_gru_bwd2<HV, HD>, GruB2<HV>::SMEM));                                                    \
    k_tc_gru_bwd2<HV, HD><<<nb, 256, GruB2<HV>::SMEM, s>>>(V, tmC, tmH, tmG, L, l, ndst, tmDC, tmDH, tmDA, tmRH, \
                                                           hg, w_o);                                          \
  } while (0)
  if (H == 32) {
    if (hg) STG_GRU_BWD(32, true); else STG_GRU_BWD(32, false);
  } else {
    if (hg) STG_GRU_BWD(16, true); else STG_GRU_BWD(16, false);
  }
#undef STG_GRU_BWD
  count_launch();
  return check_launch("tc_gru_bwd");
}

int tc_atb_max_blocks() { return 2 * num_sms(); }   // k_tc_atb2 may run 2 CTAs per SM

template <int NB, int RT, int S, int L = 2>
static stg_status atb2_launch(const CUtensorMap* m, const CUtensorMap& ones, const AtbSpec2& sp, int* nb_out,
                              cudaStream_t s, int ctas_per_sm = 1) {
  const int nbox = sp.nsa + NB;
  const size_t smem = (size_t)(S + L) * nbox * RT * 32 * 4 + 1024;   // S hi stages + L lo slots
  STG_CUDA(cudaFuncSetAttribute(k_tc_atb2<NB, RT, S, L>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int ntiles = (sp.V + RT - 1) / RT;
  const int nb = std::max(1, std::min(ntiles, ctas_per_sm * num_sms()));
  k_tc_atb2<NB, RT, S, L><<<nb, 192, smem, s>>>(m[0], m[1], m[2], m[3], ones, sp);
  count_launch();
  *nb_out = nb;
  return check_launch("tc_atb2");
}

// 32-row tiles; as many ring stages (4, 3 or 2) as fit in shared memory
constexpr int kAtbRT = 32;     // rows per ring stage of the Σ AᵀB reductions (16 rows: dL 17.4 -> 23.4 ms, dW 10.2 -> 13.9 ms per C5 epoch)

template <int NB>
static stg_status atb2_stages(const CUtensorMap* m, const CUtensorMap& ones, const AtbSpec2& sp, int* nb,
                              cudaStream_t s) {
  constexpr int RT = kAtbRT;
  const size_t stage = (size_t)(sp.nsa + NB) * RT * 32 * 4;   // one hi stage = one lo slot
  static const size_t cap = [] {                    // ring budget (experiments: STG_ATB_SMEM_KB)
    const char* v = getenv("STG_ATB_SMEM_KB");
    return (size_t)(v ? atoi(v) : 220) * 1024;
  }();
  static const int two = [] {                      // 2 CTAs per SM when 3 hi stages fit twice
    const char* v = getenv("STG_ATB_CTAS");
    return v ? atoi(v) == 2 : 1;
  }();
  static const int l1 = [] {                       // 2 CTAs x (2 hi stages + 1 lo slot): dL 19.0 -> 20.1 ms, off
    const char* v = getenv("STG_ATB_L1");
    return v ? atoi(v) : 0;
  }();
  if (two && 5 * stage <= 108 * 1024) return atb2_launch<NB, RT, 3>(m, ones, sp, nb, s, 2);
  if (two && l1 && 3 * stage <= 108 * 1024) return atb2_launch<NB, RT, 2, 1>(m, ones, sp, nb, s, 2);
  // measured on C5: deeper rings than 4 hi stages did not help (dW 10.9 ms/epoch at 4, 12.9 at 8)
  if (6 * stage <= cap) return atb2_launch<NB, RT, 4>(m, ones, sp, nb, s);
  if (5 * stage <= cap) return atb2_launch<NB, RT, 3>(m, ones, sp, nb, s);
  return atb2_launch<NB, RT, 2>(m, ones, sp, nb, s);
}

static stg_status atb2_dispatch(int NB, const CUtensorMap* m, const CUtensorMap& ones, const AtbSpec2& spec, int* nb,
                                cudaStream_t s) {
  // an M = 128 A operand spans 4 consecutive box slots from a_first: pad the stage with
  // empty slots (src_map -1: never loaded, hi and lo stay 0) until they exist
  AtbSpec2 sp = spec;
  while (sp.nsa + NB < sp.a_first[sp.na - 1] + 4 && sp.nsa < 8) sp.src_map[sp.nsa++] = -1;
  if (sp.nsa + NB < sp.a_first[sp.na - 1] + 4) return fail(STG_ERR_INVALID_ARG, "atb2: %d A slots", sp.nsa);
  switch (NB) {
    case 1: return atb2_stages<1>(m, ones, sp, nb, s);
    case 2: return atb2_stages<2>(m, ones, sp, nb, s);
    case 3: return atb2_stages<3>(m, ones, sp, nb, s);
    case 4: return atb2_stages<4>(m, ones, sp, nb, s);
    default: return fail(STG_ERR_INVALID_ARG, "atb2: %d B boxes", NB);
  }
}

// the [RT x 32] "ones" tile (1.0 in column 0): the Σ_rows feature of dl.  A
// statically initialised device global (one instance per device's module), so
// no allocation or copy happens at run time (safe inside stream capture, on any
// device, from any thread).
constexpr int kOnesMaxRT = 64;
__device__ __align__(128) float g_ones_tile[kOnesMaxRT][32] = {{1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}, {1.f}};

static stg_status ones_map(CUtensorMap* out, int RT, cudaStream_t s) {
  (void)s;
  if (RT > kOnesMaxRT) return fail(STG_ERR_INVALID_ARG, "ones tile: %d rows > %d", RT, kOnesMaxRT);
  void* d = nullptr;
  STG_CUDA(cudaGetSymbolAddress(&d, g_ones_tile));
  return make_tmap_f32(out, static_cast<const float*>(d), RT, 32, 32, 32, RT, true);
}

// dW[f][c] += Σ_v X[v,f]·dP[v,c]  via D = dPᵀ·X  (M = 128 features of dP, N = 32·ceil(F/32)).
// part: tc_atb_max_blocks() · 2 · 128 · 128 floats; tot: 2 · 128 · 128 floats.
stg_status tc_dw(int V, int F, int H, const float* X, const float* dP, float* part, float* tot, float* dW,
                 cudaStream_t s) {
  const int H3 = 3 * H, NB = (F + 31) / 32, N = 32 * NB, NA = (H3 + 31) / 32;
  CUtensorMap m[4], ones;
  STG_TRY(make_tmap_f32(&m[0], dP, (uint64_t)V, H3, H3, 32, kAtbRT, true));
  STG_TRY(make_tmap_f32(&m[1], X, (uint64_t)V, F, F, 32, kAtbRT, true));
  m[2] = m[0]; m[3] = m[0];
  STG_TRY(ones_map(&ones, kAtbRT, s));
  AtbSpec2 sp{};
  sp.V = V; sp.na = 1; sp.a_first[0] = 0; sp.nsa = NA; sp.nb = NB; sp.b_map = 1; sp.part = part;
  for (int k = 0; k < NA; ++k) { sp.src_map[k] = 0; sp.src_col[k] = 32 * k; }
  int nb = 0;
  STG_TRY(atb2_dispatch(NB, m, ones, sp, &nb, s));
  const int n = 128 * N;
  if (nb <= 16 * kSumMaxGroups) k_tc_sum_parts2<<<(n + 31) / 32, 256, 0, s>>>(part, nb, n, tot);
  else k_tc_sum_parts<<<(n + 255) / 256, 256, 0, s>>>(part, nb, n, tot);
  k_dw_scatter<<<(F * H3 + 255) / 256, 256, 0, s>>>(F, H3, N, tot, dW);
  count_launch(2);
  return check_launch("tc_dw");
}

// dL, dl, db from C, H, RH, da (see k_tc_gru_bwd2) with ONE reduction kernel:
//   D1 = [C_z|C_r|C_h | H]ᵀ·da  (C in feature boxes 0.., H at feature 32·ceil(3H/32)),
//   D2 = [RH | ones]ᵀ·da        (RH features 0..H, the ones feature at 32).
static stg_status tc_dl3(int V, const float* C, const float* Hp, const float* RH, const float* da, float* part,
                         float* tot, float* dL, float* dl, float* db, const float* L, cudaStream_t s) {
  constexpr int H = 32, RT = kAtbRT, S = 3, Ls = 2;
  CUtensorMap mC, mH, mRH, mDA, ones;
  STG_TRY(make_tmap_f32(&mC, C, (uint64_t)V, 3 * H, 3 * H, 32, RT, true));
  STG_TRY(make_tmap_f32(&mH, Hp, (uint64_t)V, H, H, 32, RT, true));
  STG_TRY(make_tmap_f32(&mRH, RH, (uint64_t)V, H, H, 32, RT, true));
  STG_TRY(make_tmap_f32(&mDA, da, (uint64_t)V, 3 * H, 3 * H, 32, RT, true));
  STG_TRY(ones_map(&ones, RT, s));
  const size_t smem = (size_t)(S + Ls) * kDl3Slots * RT * 32 * 4 + 1024;
  STG_CUDA(cudaFuncSetAttribute(k_tc_dl3<RT, S, Ls>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int ntiles = (V + RT - 1) / RT;
  const int nb = std::max(1, std::min(ntiles, num_sms()));
  k_tc_dl3<RT, S, Ls><<<nb, 192, smem, s>>>(mC, mH, mRH, mDA, ones, V, part);
  const int n = 3 * 65 * 32;
  k_tc_sum_parts2<<<(n + 31) / 32, 256, 0, s>>>(part, nb, n, tot);
  k_dl3_scatter<<<(6 * H * H + 6 * H + 255) / 256, 256, 0, s>>>(tot, L, dL, dl, db);
  count_launch(3);
  return check_launch("tc_dl3");
}

stg_status tc_dl(int V, int H, const float* C, const float* Hp, const float* RH, const float* da, float* part,
                 float* tot, float* dL, float* dl, float* db, const float* L, cudaStream_t s) {
  static const int gate_blocked = [] {               // (A/B switch: STG_DL3=0 restores the full products)
    const char* v = getenv("STG_DL3");
    return v ? atoi(v) : 1;
  }();
  if (H == 32 && gate_blocked) return tc_dl3(V, C, Hp, RH, da, part, tot, dL, dl, db, L, s);
  const int H3 = 3 * H, NBC = (H3 + 31) / 32;
  CUtensorMap m[4], ones;
  STG_TRY(make_tmap_f32(&m[0], C, (uint64_t)V, H3, H3, 32, kAtbRT, true));
  STG_TRY(make_tmap_f32(&m[1], Hp, (uint64_t)V, H, H, 32, kAtbRT, true));
  STG_TRY(make_tmap_f32(&m[2], RH, (uint64_t)V, H, H, 32, kAtbRT, true));
  STG_TRY(make_tmap_f32(&m[3], da, (uint64_t)V, H3, H3, 32, kAtbRT, true));
  STG_TRY(ones_map(&ones, kAtbRT, s));
  // slots: C boxes | H | RH | ones | da boxes;  A1 = [C.. | H] (H at feature 32·NBC), A2 = [RH | ones]
  AtbSpec2 sp{};
  sp.V = V; sp.na = 2; sp.nb = NBC; sp.b_map = 3; sp.part = part;
  int k = 0;
  for (; k < NBC; ++k) { sp.src_map[k] = 0; sp.src_col[k] = 32 * k; }
  sp.src_map[k] = 1; sp.src_col[k] = 0; ++k;
  sp.a_first[0] = 0;
  sp.a_first[1] = k;
  sp.src_map[k] = 2; sp.src_col[k] = 0; ++k;
  sp.src_map[k] = -2; sp.src_col[k] = 0; ++k;
  sp.nsa = k;
  int nb = 0;
  STG_TRY(atb2_dispatch(NBC, m, ones, sp, &nb, s));
  const int N = 32 * NBC, n = 2 * 128 * N;
  if (nb <= 16 * kSumMaxGroups) k_tc_sum_parts2<<<(n + 31) / 32, 256, 0, s>>>(part, nb, n, tot);
  else k_tc_sum_parts<<<(n + 255) / 256, 256, 0, s>>>(part, nb, n, tot);
  k_dl_scatter<<<(6 * H * H + 6 * H + 255) / 256, 256, 0, s>>>(H, N, 32, N, tot, L, dL, dl, db);
  count_launch(2);
  return check_launch("tc_dl");
}

}  // namespace stg

namespace stg {

// ---- sequence-batched GRU launchers (NEXT-1; layouts in the kernels' comment)
// ---- sequence GRU for small graphs (V <= kSmallMaxV): fp32 SIMT, a CTA owns RB rows
// (the recurrence is row-local) and stages its rows' whole-sequence inputs in shared
// memory once.  A 128-row tcgen05 tile would be mostly padding for C1 (V = 20), and
// each of its MMA phases is a full round trip; here a timestep is a few block-wide
// phases of 2H-term dot products.  Same outputs, layouts and fused head as the
// tcgen05 kernels; per-CTA head partials (nb = number of CTAs).
constexpr int kSmallT = 512, kSmallMaxV = 4096;

// block-wide copy of n floats (n % 4 == 0, 16-byte aligned) with several loads in flight
__device__ __forceinline__ void stage_f4(float* __restrict__ dst, const float* __restrict__ src, int n) {
  const float4* s4 = reinterpret_cast<const float4*>(src);
  float4* d4 = reinterpret_cast<float4*>(dst);
  const int n4 = n >> 2;
  int e = threadIdx.x;
  for (; e + 3 * kSmallT < n4; e += 4 * kSmallT) {
    const float4 a = __ldg(s4 + e), b = __ldg(s4 + e + kSmallT), c = __ldg(s4 + e + 2 * kSmallT),
                 d = __ldg(s4 + e + 3 * kSmallT);
    d4[e] = a; d4[e + kSmallT] = b; d4[e + 2 * kSmallT] = c; d4[e + 3 * kSmallT] = d;
  }
  for (; e < n4; e += kSmallT) d4[e] = __ldg(s4 + e);
}

template <int H>
__global__ void __launch_bounds__(kSmallT) k_seq_fwd_small(int V, int S, int RB, const float* __restrict__ C_all,
                                                           const float* __restrict__ H0, const float* __restrict__ L,
                                                           const float* __restrict__ l, float* __restrict__ H_seq,
                                                           float* __restrict__ Hp_all, const float* __restrict__ Yall,
                                                           const float* __restrict__ w_o,
                                                           const float* __restrict__ b_o, double* __restrict__ lpart) {
  extern __shared__ float sm[];
  const int r0 = blockIdx.x * RB, Vl = min(RB, V - r0);
  const int VH = Vl * H, H3 = 3 * H, LG = 2 * H * H;
  float* sL = sm;                  // [3][2H][H]
  float* sh = sL + 3 * LG;         // H_{t-1} [Vl][H]
  float* sz = sh + RB * H;         // z
  float* srh = sz + RB * H;        // r ⊙ h
  float* sn = srh + RB * H;        // H_t
  float* sC = sn + RB * H;         // this CTA's rows of C_all [Vl][S][3H]
  __shared__ double sloss[kSmallT];
  __shared__ float sl[3 * H], swo[H];
  float* sY = sC + (size_t)RB * S * H3;      // [Vl][S]
  stage_f4(sC, C_all + (int64_t)r0 * S * H3, Vl * S * H3);
  for (int e = threadIdx.x; e < Vl * S; e += kSmallT) sY[e] = Yall[(int64_t)r0 * S + e];
  for (int e = threadIdx.x; e < 3 * H; e += kSmallT) sl[e] = l[e];
  for (int e = threadIdx.x; e < H; e += kSmallT) swo[e] = w_o[e];
  stage_f4(sL, L, 3 * LG);
  stage_f4(sh, H0 + (int64_t)r0 * H, VH);
  for (int v = threadIdx.x; v < Vl; v += kSmallT) sloss[v] = 0.0;
  const float* Lz = sL; const float* Lr = sL + LG; const float* Lh = sL + 2 * LG;
  const float bo = b_o[0];
  __syncthreads();
  for (int t = 0; t < S; ++t) {
    for (int e = threadIdx.x; e < VH; e += kSmallT) {          // z, r⊙h; Hp_all slot t = H_{t-1}
      const int v = e / H, j = e % H;
      const float* c = sC + ((int64_t)v * S + t) * H3;
      const float* hv = sh + v * H;
      float az = sl[j], ar = sl[H + j];
#pragma unroll
      for (int i = 0; i < H; ++i) {
        az = fmaf(c[i], Lz[i * H + j], az);
        ar = fmaf(c[H + i], Lr[i * H + j], ar);
      }
#pragma unroll
      for (int i = 0; i < H; ++i) {
        az = fmaf(hv[i], Lz[(H + i) * H + j], az);
        ar = fmaf(hv[i], Lr[(H + i) * H + j], ar);
      }
      sz[e] = 1.0f / (1.0f + expf(-az));
      srh[e] = hv[j] / (1.0f + expf(-ar));
      Hp_all[((int64_t)(r0 + v) * S + t) * H + j] = hv[j];
    }
    __syncthreads();
    for (int e = threadIdx.x; e < VH; e += kSmallT) {          // candidate, H_t
      const int v = e / H, j = e % H;
      const float* c = sC + ((int64_t)v * S + t) * H3 + 2 * H;
      float ah = sl[2 * H + j];
#pragma unroll
      for (int i = 0; i < H; ++i) ah = fmaf(c[i], Lh[i * H + j], ah);
#pragma unroll
      for (int i = 0; i < H; ++i) ah = fmaf(srh[v * H + i], Lh[(H + i) * H + j], ah);
      const float z = sz[e], hh = tanhf(ah);
      const float hn = z * sh[e] + (1.0f - z) * hh;
      sn[e] = hn;
      H_seq[((int64_t)t * V + r0 + v) * H + j] = hn;
    }
    __syncthreads();
    for (int v = threadIdx.x; v < Vl; v += kSmallT) {           // fused head: loss of row v at t
      float d = 0.f;
#pragma unroll
      for (int j = 0; j < H; ++j) d = fmaf(fmaxf(sn[v * H + j], 0.f), swo[j], d);
      const float e = (d + bo) - sY[v * S + t];
      sloss[v] += (double)e * (double)e;
    }
    for (int e = threadIdx.x; e < VH; e += kSmallT) sh[e] = sn[e];
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    double tot = 0.0;
    for (int v = 0; v < Vl; ++v) tot += sloss[v];
    lpart[blockIdx.x] = tot;
  }
}

template <int H>
__global__ void __launch_bounds__(kSmallT) k_seq_bwd_small(int V, int S, int RB, const float* __restrict__ C_all,
                                                           const float* __restrict__ Hp_all,
                                                           const float* __restrict__ H_seq,
                                                           const float* __restrict__ L, const float* __restrict__ l,
                                                           const float* __restrict__ ndst,
                                                           const float* __restrict__ Yall,
                                                           const float* __restrict__ w_o,
                                                           const float* __restrict__ b_o, float inv_vn,
                                                           float* __restrict__ dC_all, float* __restrict__ da_all,
                                                           float* __restrict__ RH_all, float* __restrict__ gpart) {
  extern __shared__ float sm[];
  const int r0 = blockIdx.x * RB, Vl = min(RB, V - r0);
  const int VH = Vl * H, H3 = 3 * H, LG = 2 * H * H, RH = RB * H;
  float* sL = sm;                  // [3][2H][H]
  float* sdh = sL + 3 * LG;        // dℓ/dH_t flowing back from t+1
  float* sg = sdh + RH;            // G
  float* sz = sg + RH;
  float* sr = sz + RH;
  float* srh = sr + RH;
  float* sdaz = srh + RH;
  float* sdah = sdaz + RH;
  float* sdar = sdah + RH;
  float* sdhn = sdar + RH;
  float* sC = sdhn + RH;                     // [Vl][S][3H]
  float* sHp = sC + (size_t)RB * S * H3;     // [Vl][S][H]
  float* sHs = sHp + (size_t)RB * S * H;     // [S][Vl][H]
  __shared__ float sgs[kSmallT];
  __shared__ float sgw[65];
  __shared__ float sl[3 * H], swo[H], snd[kSmallT];
  float* sY = sHs + (size_t)RB * S * H;      // [Vl][S]
  for (int e = threadIdx.x; e < Vl * S; e += kSmallT) sY[e] = Yall[(int64_t)r0 * S + e];
  for (int e = threadIdx.x; e < 3 * H; e += kSmallT) sl[e] = l[e];
  for (int e = threadIdx.x; e < H; e += kSmallT) swo[e] = w_o[e];
  for (int v = threadIdx.x; v < Vl; v += kSmallT) snd[v] = ndst[r0 + v];
  stage_f4(sC, C_all + (int64_t)r0 * S * H3, Vl * S * H3);
  stage_f4(sHp, Hp_all + (int64_t)r0 * S * H, Vl * S * H);
  for (int t = 0; t < S; ++t) stage_f4(sHs + (size_t)t * VH, H_seq + ((int64_t)t * V + r0) * H, VH);
  stage_f4(sL, L, 3 * LG);
  for (int e = threadIdx.x; e < VH; e += kSmallT) sdh[e] = 0.f;
  for (int j = threadIdx.x; j <= H; j += kSmallT) sgw[j] = 0.f;
  const float* Lz = sL; const float* Lr = sL + LG; const float* Lh = sL + 2 * LG;
  const float bo = b_o[0];
  __syncthreads();
  for (int t = S - 1; t >= 0; --t) {
    for (int v = threadIdx.x; v < Vl; v += kSmallT) {           // head gradient scale of row v
      const float* ht = sHs + ((int64_t)t * Vl + v) * H;
      float d = 0.f;
#pragma unroll
      for (int j = 0; j < H; ++j) d = fmaf(fmaxf(ht[j], 0.f), swo[j], d);
      sgs[v] = 2.0f * ((d + bo) - sY[v * S + t]) * inv_vn;
    }
    __syncthreads();
    if (threadIdx.x <= H) {                                     // dw_o, db_o partials (rows in order)
      const int j = threadIdx.x;
      float acc = sgw[j];
      for (int v = 0; v < Vl; ++v)
        acc += j < H ? sgs[v] * fmaxf(sHs[((int64_t)t * Vl + v) * H + j], 0.f) : sgs[v];
      sgw[j] = acc;
    }
    for (int e = threadIdx.x; e < VH; e += kSmallT) {          // G, z, r, r⊙h
      const int v = e / H, j = e % H;
      const float ht = sHs[((int64_t)t * Vl + v) * H + j];
      sg[e] = (ht > 0.f ? sgs[v] * swo[j] : 0.f) + sdh[e];
      const float* c = sC + ((int64_t)v * S + t) * H3;
      const float* hv = sHp + ((int64_t)v * S + t) * H;
      float az = sl[j], ar = sl[H + j];
#pragma unroll
      for (int i = 0; i < H; ++i) {
        az = fmaf(c[i], Lz[i * H + j], az);
        ar = fmaf(c[H + i], Lr[i * H + j], ar);
      }
#pragma unroll
      for (int i = 0; i < H; ++i) {
        az = fmaf(hv[i], Lz[(H + i) * H + j], az);
        ar = fmaf(hv[i], Lr[(H + i) * H + j], ar);
      }
      const float z = 1.0f / (1.0f + expf(-az)), r = 1.0f / (1.0f + expf(-ar));
      sz[e] = z;
      sr[e] = r;
      srh[e] = r * hv[j];
      RH_all[((int64_t)(r0 + v) * S + t) * H + j] = r * hv[j];
    }
    __syncthreads();
    for (int e = threadIdx.x; e < VH; e += kSmallT) {          // candidate; da_z, da_h
      const int v = e / H, j = e % H;
      const float* c = sC + ((int64_t)v * S + t) * H3 + 2 * H;
      float ah = sl[2 * H + j];
#pragma unroll
      for (int i = 0; i < H; ++i) ah = fmaf(c[i], Lh[i * H + j], ah);
#pragma unroll
      for (int i = 0; i < H; ++i) ah = fmaf(srh[v * H + i], Lh[(H + i) * H + j], ah);
      const float hh = tanhf(ah), g = sg[e], z = sz[e];
      const float h = sHp[((int64_t)v * S + t) * H + j];
      const float dZ = g * (h - hh), dHh = g * (1.0f - z);
      const float dah = dHh * (1.0f - hh * hh), daz = dZ * z * (1.0f - z);
      sdah[e] = dah;
      sdaz[e] = daz;
      sdhn[e] = g * z;
      float* da = da_all + ((int64_t)(r0 + v) * S + t) * H3;
      da[j] = daz;
      da[2 * H + j] = dah;
    }
    __syncthreads();
    for (int e = threadIdx.x; e < VH; e += kSmallT) {          // dC_h, d(r⊙h) -> da_r; dC_z, dH_z
      const int v = e / H, i = e % H;
      float dch = 0.f, drh = 0.f, dcz = 0.f, dhz = 0.f;
#pragma unroll
      for (int j = 0; j < H; ++j) {
        const float a = sdah[v * H + j], b = sdaz[v * H + j];
        dch = fmaf(a, Lh[i * H + j], dch);
        drh = fmaf(a, Lh[(H + i) * H + j], drh);
        dcz = fmaf(b, Lz[i * H + j], dcz);
        dhz = fmaf(b, Lz[(H + i) * H + j], dhz);
      }
      const float r = sr[e], h = sHp[((int64_t)v * S + t) * H + i];
      const float dar = drh * h * r * (1.0f - r);
      sdar[e] = dar;
      sdhn[e] += drh * r + dhz;
      const float nd = snd[v];
      float* dc = dC_all + ((int64_t)(r0 + v) * S + t) * H3;
      dc[i] = nd * dcz;
      dc[2 * H + i] = nd * dch;
      da_all[((int64_t)(r0 + v) * S + t) * H3 + H + i] = dar;
    }
    __syncthreads();
    for (int e = threadIdx.x; e < VH; e += kSmallT) {          // dC_r, dH_r; dℓ/dH_{t-1}
      const int v = e / H, i = e % H;
      float dcr = 0.f, dhr = 0.f;
#pragma unroll
      for (int j = 0; j < H; ++j) {
        const float a = sdar[v * H + j];
        dcr = fmaf(a, Lr[i * H + j], dcr);
        dhr = fmaf(a, Lr[(H + i) * H + j], dhr);
      }
      dC_all[((int64_t)(r0 + v) * S + t) * H3 + H + i] = snd[v] * dcr;
      sdh[e] = sdhn[e] + dhr;
    }
    __syncthreads();
  }
  for (int j = threadIdx.x; j <= H; j += kSmallT) gpart[(int64_t)blockIdx.x * (H + 1) + j] = sgw[j];
}

static size_t small_fwd_smem(int RB, int S, int H) {
  return sizeof(float) * (6 * (size_t)H * H + 4 * (size_t)RB * H + (size_t)RB * S * (3 * H + 1));
}
static size_t small_bwd_smem(int RB, int S, int H) {
  return sizeof(float) * (6 * (size_t)H * H + 9 * (size_t)RB * H + (size_t)RB * S * (5 * H + 1));
}
// Rows per CTA of the small-graph path (0 = use the tcgen05 kernels).  A timestep is a
// latency chain of block-wide phases, so the rows are spread over one wave of CTAs with
// as few rows per CTA as that allows (at least 64/H, about two warps of (row, column)
// work).  Measured per epoch: C1 (V = 20) 4 rows 4.6 ms vs 20 rows 6.1 ms vs tcgen05
// 7.1 ms; C3 (V = 319) 4 rows 364 ms, 2 rows 404 ms, tcgen05 505 ms; C2 (V = 1068) 8 rows
// 19.3 ms vs tcgen05 21.7 ms, 2 rows (534 CTAs) 24.8 ms.  Beyond one wave of at most
// kSmallT/H rows per CTA (or the shared-memory budget) the tcgen05 tiles take over.
static int small_rows(int V, int S, int H) {
  if (V > kSmallMaxV || (H != 16 && H != 32)) return 0;
  static const int forced = [] {                   // experiments: STG_SMALL_RB=rows per CTA
    const char* e = getenv("STG_SMALL_RB");
    return e ? atoi(e) : 0;
  }();
  int rb = forced > 0 ? forced : std::max(64 / H, (V + num_sms() - 1) / num_sms());
  if (rb * H > kSmallT || small_bwd_smem(rb, S, H) > 200 * 1024) return 0;
  return rb >= V ? V : rb;
}

stg_status tc_gru_seq_fwd(int V, int S, int H, const float* C_all, const float* H0, const float* L, const float* l,
                          float* H_seq, float* Hp_all, const float* Y_all, const float* w_o, const float* b_o,
                          double* lpart, int* nb_out, cudaStream_t s) {
  if (const int rb = small_rows(V, S, H)) {
    const size_t smem = small_fwd_smem(rb, S, H);
    const int nb = (V + rb - 1) / rb;
    if (H == 32) {
      STG_TRY(prep(k_seq_fwd_small<32>, smem));
      k_seq_fwd_small<32><<<nb, kSmallT, smem, s>>>(V, S, rb, C_all, H0, L, l, H_seq, Hp_all, Y_all, w_o, b_o, lpart);
    } else {
      STG_TRY(prep(k_seq_fwd_small<16>, smem));
      k_seq_fwd_small<16><<<nb, kSmallT, smem, s>>>(V, S, rb, C_all, H0, L, l, H_seq, Hp_all, Y_all, w_o, b_o, lpart);
    }
    count_launch();
    *nb_out = nb;
    return check_launch("seq_fwd_small");
  }
  const int ntiles = (V + 127) / 128;
  const int nb = std::min(ntiles, num_sms());
  const uint32_t hh = (uint32_t)H / 2;
  CUtensorMap tmC, tmH0, tmHs, tmHp;
  STG_TRY(make_tmap_f32(&tmC, C_all, (uint64_t)V, (uint64_t)S * 3 * H, (uint64_t)S * 3 * H, 32, 128));
  STG_TRY(make_tmap_f32(&tmH0, H0, (uint64_t)V, H, H, 32, 128));
  STG_TRY(make_tmap_f32_store3(&tmHs, H_seq, (uint64_t)S, (uint64_t)V, H, hh, 32));
  STG_TRY(make_tmap_f32_store(&tmHp, Hp_all, (uint64_t)V, (uint64_t)S * H, (uint64_t)S * H, hh, 32));
  if (H == 32) {
    using G = GruF2<32>;
    const size_t smem = 2 * G::NBC * kBox + kBox + 6 * G::BG + 8 * G::OBUF + 1024;
    STG_TRY(prep(k_tc_gru_seq_fwd<32>, smem));
    k_tc_gru_seq_fwd<32><<<nb, 256, smem, s>>>(V, S, tmC, tmH0, L, l, tmHs, tmHp, Y_all, w_o, b_o, lpart);
  } else {
    using G = GruF2<16>;
    const size_t smem = 2 * G::NBC * kBox + kBox + 6 * G::BG + 8 * G::OBUF + 1024;
    STG_TRY(prep(k_tc_gru_seq_fwd<16>, smem));
    k_tc_gru_seq_fwd<16><<<nb, 256, smem, s>>>(V, S, tmC, tmH0, L, l, tmHs, tmHp, Y_all, w_o, b_o, lpart);
  }
  count_launch();
  *nb_out = nb;
  return check_launch("tc_gru_seq_fwd");
}

stg_status tc_gru_seq_bwd(int V, int S, int H, const float* C_all, const float* Hp_all, const float* H_seq,
                          const float* L, const float* l, const float* ndst, const float* Y_all, const float* w_o,
                          const float* b_o, float inv_vn, float* dC_all, float* da_all, float* RH_all, float* gpart,
                          int* nb_out, cudaStream_t s) {
  if (const int rb = small_rows(V, S, H)) {
    const size_t smem = small_bwd_smem(rb, S, H);
    const int nb = (V + rb - 1) / rb;
    if (H == 32) {
      STG_TRY(prep(k_seq_bwd_small<32>, smem));
      k_seq_bwd_small<32><<<nb, kSmallT, smem, s>>>(V, S, rb, C_all, Hp_all, H_seq, L, l, ndst, Y_all, w_o, b_o,
                                                    inv_vn, dC_all, da_all, RH_all, gpart);
    } else {
      STG_TRY(prep(k_seq_bwd_small<16>, smem));
      k_seq_bwd_small<16><<<nb, kSmallT, smem, s>>>(V, S, rb, C_all, Hp_all, H_seq, L, l, ndst, Y_all, w_o, b_o,
                                                    inv_vn, dC_all, da_all, RH_all, gpart);
    }
    count_launch();
    *nb_out = nb;
    return check_launch("seq_bwd_small");
  }
  const int ntiles = (V + 127) / 128;
  const int nb = std::min(ntiles, num_sms());
  const uint32_t hh = (uint32_t)H / 2;
  const uint64_t H3S = (uint64_t)S * 3 * H;
  CUtensorMap tmC, tmHp, tmHs, tmDC, tmDA, tmRH;
  STG_TRY(make_tmap_f32(&tmC, C_all, (uint64_t)V, H3S, H3S, 32, 128));
  STG_TRY(make_tmap_f32(&tmHp, Hp_all, (uint64_t)V, (uint64_t)S * H, (uint64_t)S * H, 32, 128));
  STG_TRY(make_tmap_f32(&tmHs, H_seq, (uint64_t)S * V, H, H, 32, 128));
  STG_TRY(make_tmap_f32_store(&tmDC, dC_all, (uint64_t)V, H3S, H3S, hh, 32));
  STG_TRY(make_tmap_f32_store(&tmDA, da_all, (uint64_t)V, H3S, H3S, hh, 32));
  STG_TRY(make_tmap_f32_store(&tmRH, RH_all, (uint64_t)V, (uint64_t)S * H, (uint64_t)S * H, hh, 32));
  if (H == 32) {
    STG_TRY(prep(k_tc_gru_seq_bwd<32>, GruB2<32>::SMEM));
    k_tc_gru_seq_bwd<32><<<nb, 256, GruB2<32>::SMEM, s>>>(V, S, tmC, tmHp, tmHs, L, l, ndst, Y_all, w_o, b_o, inv_vn,
                                                          tmDC, tmDA, tmRH, gpart);
  } else {
    STG_TRY(prep(k_tc_gru_seq_bwd<16>, GruB2<16>::SMEM));
    k_tc_gru_seq_bwd<16><<<nb, 256, GruB2<16>::SMEM, s>>>(V, S, tmC, tmHp, tmHs, L, l, ndst, Y_all, w_o, b_o, inv_vn,
                                                          tmDC, tmDA, tmRH, gpart);
  }
  count_launch();
  *nb_out = nb;
  return check_launch("tc_gru_seq_bwd");
}

stg_status tc_seq_head_reduce(int nb, int H, const double* lpart, const float* gpart, double inv_vn, float* loss,
                              float* dw_o, float* db_o, cudaStream_t s) {
  k_seq_head_reduce<<<1, 128, 0, s>>>(nb, H, lpart, gpart, inv_vn, loss, dw_o, db_o);
  count_launch();
  return check_launch("tc_seq_head_reduce");
}

}  // namespace stg

// Diagnostic entry point (tests only): the fixed-order partial sum of the Σ AᵀB
// reductions in either implementation (0 = serial per element, 1 = parallel over
// the 16-partial groups, nb <= 1024), so a test can check that they agree bit for bit.
extern "C" stg_status stg_debug_sum_parts(const float* part, int32_t nb, int32_t n, float* tot, int32_t variant,
                                          stg_stream_t stream) {
  using namespace stg;
  if (!part || !tot || nb < 1 || n < 1) return fail(STG_ERR_INVALID_ARG, "stg_debug_sum_parts: nb=%d n=%d", nb, n);
  cudaStream_t s = (cudaStream_t)stream;
  if (variant == 1) {
    if (nb > 16 * kSumMaxGroups) return fail(STG_ERR_INVALID_ARG, "stg_debug_sum_parts: nb=%d > %d", nb, 16 * kSumMaxGroups);
    k_tc_sum_parts2<<<(n + 31) / 32, 256, 0, s>>>(part, nb, n, tot);
  } else if (variant == 0) {
    k_tc_sum_parts<<<(n + 255) / 256, 256, 0, s>>>(part, nb, n, tot);
  } else {
    return fail(STG_ERR_INVALID_ARG, "stg_debug_sum_parts: variant %d", variant);
  }
  count_launch();
  return check_launch("stg_debug_sum_parts");
}

// ------------------------------------------------------------------ NEXT-2 dense parts on tcgen05
// The original T-GCN cell's convolutions multiply a row
// concatenation [A1 | A2] by a small weight slice:
//   out[r, :] (+)= rs[r] · [A1[r, :K1] | A2[r, :K2]] · W,  W(k, n) = W[k·sk + n·sn]
// (the forward [X, H]·W_g / [X, r⊙H]·W_c, the backward dY·W[F:, :]ᵀ), and reduce
//   grad[k, n] += Σ_r [A1 | A2][r, k] · B[r, n]
// (dW_g, dW_c) — both 3xTF32 on the tensor cores like the TGCN's X·W and Σ AᵀB.
namespace stg {
namespace {

// one 128-row tile per CTA at a time; B = Wᵀ [N × Kp] and the A tile [128 × Kp]
// (both hi / lo, K-major) in shared memory; accumulator in TMEM; thread = row.
template <int N>
__global__ void __launch_bounds__(kTcThreads) k_tc_catmm(int V, const float* __restrict__ A1, int K1, int64_t ld1,
                                                         const float* __restrict__ A2, int K2, int64_t ld2, int Kp,
                                                         const float* __restrict__ W, int64_t sk, int64_t sn,
                                                         const float* __restrict__ rs, float* __restrict__ out,
                                                         int64_t ldo, int accumulate) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ uint64_t mbar;
  __shared__ uint32_t tslot;
  unsigned char* bhi = sm;
  unsigned char* blo = bhi + N * Kp * 4;
  unsigned char* ahi = blo + N * Kp * 4;
  unsigned char* alo = ahi + 128 * Kp * 4;
  constexpr uint32_t NC = N <= 32 ? 32 : (N <= 64 ? 64 : 128);
  const int K = K1 + K2;
  for (int e = threadIdx.x; e < N * Kp; e += blockDim.x) {            // B = Wᵀ (strided slice), zero past K
    const int n = e / Kp, k = e % Kp;
    const float v = k < K ? W[(int64_t)k * sk + (int64_t)n * sn] : 0.0f;
    const float h = tc::tf32_hi(v);
    *reinterpret_cast<float*>(bhi + tc::kmaj_off(n, k, Kp)) = h;
    *reinterpret_cast<float*>(blo + tc::kmaj_off(n, k, Kp)) = v - h;
  }
  for (int i = threadIdx.x; i < 128 * Kp; i += kTcThreads) {          // zero the K padding once
    reinterpret_cast<float*>(ahi)[i] = 0.f;
    reinterpret_cast<float*>(alo)[i] = 0.f;
  }
  if ((threadIdx.x >> 5) == 0) tc::tmem_alloc(&tslot, NC);
  if (threadIdx.x == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  uint32_t phase = 0;
  const uint32_t idesc = tc::idesc_tf32(128, N, 0, 0);
  const int ntiles = (V + 127) / 128;
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int r0 = tile * 128;
    tc::stage_rows(ahi, alo, A1 + (int64_t)r0 * ld1, ld1, V - r0, 128, K1, 0, 0, Kp);
    if (K2 > 0) tc::stage_rows(ahi, alo, A2 + (int64_t)r0 * ld2, ld2, V - r0, 128, K2, 0, K1, Kp);
    sync_mma_operands();
    if (threadIdx.x == 0) {
      mma_seg(tm, tc::smem_u32(ahi), tc::smem_u32(alo), Kp, 0, tc::smem_u32(bhi), tc::smem_u32(blo), Kp, 0, Kp, idesc,
              true);
      tc::commit(&mbar);
    }
    wait_mma(&mbar, phase);
    const int row = r0 + threadIdx.x;
    float v[N];
    tmem_row_load<N>(tm, 0, v);
    if (row < V) {
      const float s = rs ? rs[row] : 1.0f;
      float4* o = reinterpret_cast<float4*>(out + (int64_t)row * ldo);
#pragma unroll
      for (int c = 0; c < N / 4; ++c) {
        float4 r = make_float4(s * v[4 * c], s * v[4 * c + 1], s * v[4 * c + 2], s * v[4 * c + 3]);
        if (accumulate) {
          const float4 q = o[c];
          r.x += q.x; r.y += q.y; r.z += q.z; r.w += q.w;
        }
        o[c] = r;
      }
    }
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
  }
  tc::fence_before();
  __syncthreads();
  if ((threadIdx.x >> 5) == 0) tc::tmem_free(tm, NC);
}

// A 128-row tile of [A1 | A2] (K1 + K2 <= 128 columns, K1 % 4 == 0) as float4 chunks
// of the concatenated row, nthr threads, at most 16 chunks per thread: load into
// registers, then split into hi / lo at K-major column 4j.  Rows >= nvalid are 0.
__device__ __forceinline__ void cat_load(float4 (&v)[16], const float* __restrict__ A1, int64_t ld1, int K1,
                                         const float* __restrict__ A2, int64_t ld2, int K2, int nvalid, int tid,
                                         int nthr) {
  const int lane = tid & 31, warp = tid >> 5, nw = nthr >> 5;
  const int nj = (K1 + K2) / 4, njb = (nj + 3) / 4, total = 16 * njb, j1 = K1 / 4;
#pragma unroll
  for (int i = 0; i < 16; ++i) {
    const int it = warp + i * nw;
    const int r = (it % 16) * 8 + (lane & 7);
    const int j = (it / 16) * 4 + (lane >> 3);
    v[i] = make_float4(0.f, 0.f, 0.f, 0.f);
    if (it < total && j < nj && r < nvalid)
      v[i] = __ldg(reinterpret_cast<const float4*>(j < j1 ? A1 + (int64_t)r * ld1 + 4 * j
                                                          : A2 + (int64_t)r * ld2 + 4 * (j - j1)));
  }
}
__device__ __forceinline__ void cat_store(const float4 (&v)[16], unsigned char* hi, unsigned char* lo, int K, int Kp,
                                          int tid, int nthr) {
  const int lane = tid & 31, warp = tid >> 5, nw = nthr >> 5;
  const int nj = K / 4, njb = (nj + 3) / 4, total = 16 * njb;
#pragma unroll
  for (int i = 0; i < 16; ++i) {
    const int it = warp + i * nw;
    const int r = (it % 16) * 8 + (lane & 7);
    const int j = (it / 16) * 4 + (lane >> 3);
    if (it < total && j < nj) tc::st_split4(hi, lo, r, j, Kp, v[i]);
  }
}

// The same product, warp-specialised like k_tc_xw_pipe:
//   warps 4-11  producers: NST groups of 256/NST threads (NST = ring slots, 2 when
//               shared memory allows, else 1) take alternate tiles; a group holds its
//               next tile in registers while it waits for its slot, then splits it;
//   warp 12     one lane issues the 3xTF32 MMAs into one of two TMEM accumulators;
//   warps 0-3   epilogue: tcgen05.ld, row scale, per-warp TMA box store, or a TMA
//               reduce-add into out when accumulating.
template <int N, int NST>
__global__ void __launch_bounds__(kXwThreads, 1) k_tc_catmm_pipe(int V, const float* __restrict__ A1, int K1,
                                                                 int64_t ld1, const float* __restrict__ A2, int K2,
                                                                 int64_t ld2, int Kp,
                                                                 const float* __restrict__ W, int64_t sk, int64_t sn,
                                                                 const float* __restrict__ rs,
                                                                 const __grid_constant__ CUtensorMap tmO,
                                                                 int accumulate) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ uint64_t full[NST], empty[NST], tfull[2], tempty[2];
  __shared__ uint32_t tslot;
  constexpr uint32_t NC = N <= 32 ? 32 : 64;
  constexpr int NT = 256 / NST;                      // producer threads per group
  const int ABYTES = 128 * Kp * 4;
  unsigned char* bhi = sm;
  unsigned char* blo = bhi + N * Kp * 4;
  unsigned char* abase = blo + N * Kp * 4;
  auto ahi = [&](int st) { return abase + (size_t)st * 2 * ABYTES; };
  auto alo = [&](int st) { return abase + (size_t)st * 2 * ABYTES + ABYTES; };
  const int warp = threadIdx.x >> 5;
  const int K = K1 + K2;
  for (int e = threadIdx.x; e < N * Kp; e += blockDim.x) {            // B = Wᵀ (strided slice), zero past K
    const int n = e / Kp, k = e % Kp;
    const float v = k < K ? W[(int64_t)k * sk + (int64_t)n * sn] : 0.0f;
    const float h = tc::tf32_hi(v);
    *reinterpret_cast<float*>(bhi + tc::kmaj_off(n, k, Kp)) = h;
    *reinterpret_cast<float*>(blo + tc::kmaj_off(n, k, Kp)) = v - h;
  }
  for (int i = threadIdx.x; i < NST * 2 * 128 * Kp; i += blockDim.x)   // zero the K padding once
    reinterpret_cast<float*>(abase)[i] = 0.f;
  if (warp == 12) tc::tmem_alloc(&tslot, 2 * NC);
  if (threadIdx.x == 0) {
    for (int st = 0; st < NST; ++st) { tc::mbar_init(&full[st], NT); tc::mbar_init(&empty[st], 1); }
    for (int b = 0; b < 2; ++b) { tc::mbar_init(&tfull[b], 1); tc::mbar_init(&tempty[b], 128); }
    tc::fence_mbar_init();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  const int ntiles = (V + 127) / 128;
  if (warp >= 4 && warp < 12) {                      // ---- producers (group = slot)
    const int grp = (warp - 4) / (NT / 32), tid = threadIdx.x - 128 - NT * grp;
    float4 v[16];
    int tile = blockIdx.x + grp * gridDim.x;
    auto load = [&](int t) {
      cat_load(v, A1 + (int64_t)t * 128 * ld1, ld1, K1, A2 + (int64_t)t * 128 * ld2, ld2, K2, V - t * 128, tid, NT);
    };
    if (tile < ntiles) load(tile);
    for (int k = 0; tile < ntiles; tile += NST * gridDim.x, ++k) {
      if (k > 0) tc::mbar_wait(&empty[grp], (k - 1) & 1);
      cat_store(v, ahi(grp), alo(grp), K, Kp, tid, NT);
      tc::fence_proxy_async();
      tc::mbar_arrive(&full[grp]);
      const int nt = tile + NST * gridDim.x;
      if (nt < ntiles) load(nt);
    }
  } else if (warp == 12) {                           // ---- MMA issuer
    if ((threadIdx.x & 31) == 0) {
      const uint32_t idesc = tc::idesc_tf32(128, N, 0, 0);
      int i = 0;
      for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++i) {
        const int st = i % NST, ks = i / NST;        // tile i: ring slot i % NST, accumulator i % 2
        const int b = i & 1, kb = i >> 1;
        tc::mbar_wait(&full[st], ks & 1);
        if (kb > 0) tc::mbar_wait(&tempty[b], (kb - 1) & 1);
        tc::fence_after();
        mma_seg(tm + b * NC, tc::smem_u32(ahi(st)), tc::smem_u32(alo(st)), Kp, 0, tc::smem_u32(bhi),
                tc::smem_u32(blo), Kp, 0, Kp, idesc, true);
        tc::commit(&empty[st]);
        tc::commit(&tfull[b]);
      }
    }
  } else if (warp < 4) {                             // ---- epilogue, TMA box stores / reduce-adds
    unsigned char* obuf = reinterpret_cast<unsigned char*>(
        (reinterpret_cast<uintptr_t>(abase + (size_t)NST * 2 * ABYTES) + 1023) & ~uintptr_t(1023)) + warp * 4096;
    int oslot = 0;
    int i = 0;
    for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++i) {
      const int b = i & 1, kb = i >> 1;
      const int row = tile * 128 + threadIdx.x;
      const float sc = (rs && row < V) ? __ldg(rs + row) : 1.0f;
      tc::mbar_wait(&tfull[b], kb & 1);
      tc::fence_after();
      const int wr0 = tile * 128 + warp * 32;
#pragma unroll
      for (int c0 = 0; c0 < N; c0 += 16) {
        float v[16];
        tmem_row_load<16>(tm + b * NC, c0, v);
        if (c0 + 16 >= N) {                          // accumulator b fully read: release it early
          tc::fence_before();
          tc::mbar_arrive(&tempty[b]);
        }
        if (accumulate) tc::warp_box_store<16, true>(obuf, oslot, v, sc, &tmO, c0, wr0);
        else tc::warp_box_store<16>(obuf, oslot, v, sc, &tmO, c0, wr0);
      }
    }
    if ((threadIdx.x & 31) == 0) tc::bulk_wait_all();  // output boxes written before the CTA exits
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 12) tc::tmem_free(tm, 2 * NC);
}

// grad[k][n] += tot[row(k)][n]; rows 0..K1 hold A1's features, A2's start at hoff
__global__ void k_cat_scatter(int K1, int K2, int N, int hoff, int Np, const float* __restrict__ tot,
                              float* __restrict__ grad) {
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < (K1 + K2) * N; e += gridDim.x * blockDim.x) {
    const int k = e / N, n = e % N;
    const int m = k < K1 ? k : hoff + (k - K1);
    grad[e] += tot[(int64_t)m * Np + n];
  }
}

}  // namespace

bool tc_cat_supported(int K1, int K2, int N) {
  return (N == 16 || N == 32 || N == 64) && K1 % 4 == 0 && K2 % 4 == 0 && K1 >= 4 && K1 + K2 <= 128 &&
         32 * ((K1 + 31) / 32) + 32 * ((K2 + 31) / 32) <= 128;
}

stg_status tc_catmm(int V, const float* A1, int K1, int64_t ld1, const float* A2, int K2, int64_t ld2, const float* W,
                    int64_t sk, int64_t sn, int N, const float* rs, float* out, int64_t ldo, bool accumulate,
                    cudaStream_t s) {
  if (V <= 0) return STG_OK;
  const int Kp = (K1 + K2 + 7) / 8 * 8;
  const int ntiles = (V + 127) / 128;
  if (K1 + K2 <= 128 && N % 16 == 0 && ((uintptr_t)out) % 16 == 0) {   // warp-specialised pipeline
    const auto need = [&](int nst) { return (size_t)2 * N * Kp * 4 + (size_t)nst * 2 * 128 * Kp * 4 + 1024 + 4 * 4096; };
    const int nst = need(2) <= 227 * 1024 ? 2 : (need(1) <= 227 * 1024 ? 1 : 0);
    if (nst) {
      const size_t smem = need(nst);
      CUtensorMap tmO;
      STG_TRY(make_tmap_f32_store(&tmO, out, (uint64_t)V, (uint64_t)N, (uint64_t)ldo, 16, 32));
      const int nb = std::min(ntiles, num_sms());
#define STG_CATMM_PIPE(NN, NS)                                                                                   \
  do {                                                                                                           \
    STG_TRY(prep(k_tc_catmm_pipe<NN, NS>, smem));                                                                \
    k_tc_catmm_pipe<NN, NS><<<nb, kXwThreads, smem, s>>>(V, A1, K1, ld1, A2, K2, ld2, Kp, W, sk, sn, rs, tmO,    \
                                                         accumulate ? 1 : 0);                                    \
  } while (0)
      if (nst == 2) {
        if (N == 16) STG_CATMM_PIPE(16, 2);
        else if (N == 32) STG_CATMM_PIPE(32, 2);
        else STG_CATMM_PIPE(64, 2);
      } else {
        if (N == 16) STG_CATMM_PIPE(16, 1);
        else if (N == 32) STG_CATMM_PIPE(32, 1);
        else STG_CATMM_PIPE(64, 1);
      }
#undef STG_CATMM_PIPE
      count_launch();
      return check_launch("tc_catmm_pipe");
    }
  }
  const size_t smem = (size_t)2 * N * Kp * 4 + (size_t)2 * 128 * Kp * 4;
#define STG_CATMM(NN)                                                                                           \
  do {                                                                                                          \
    STG_TRY(prep(k_tc_catmm<NN>, smem));                                                                        \
    const int nb = std::min(ntiles, occupancy_blocks(k_tc_catmm<NN>, smem));                                    \
    k_tc_catmm<NN><<<nb, kTcThreads, smem, s>>>(V, A1, K1, ld1, A2, K2, ld2, Kp, W, sk, sn, rs, out, ldo,        \
                                                accumulate ? 1 : 0);                                            \
  } while (0)
  if (N == 16) STG_CATMM(16);
  else if (N == 32) STG_CATMM(32);
  else if (N == 64) STG_CATMM(64);
  else return fail(STG_ERR_INVALID_ARG, "tc_catmm: N=%d", N);
#undef STG_CATMM
  count_launch();
  return check_launch("tc_catmm");
}

// grad[K1+K2][N] += [A1 | A2]ᵀ · B  (A1 [V, K1], A2 [V, K2], B [V, N], row-major, contiguous)
stg_status tc_atb_cat(int V, const float* A1, int K1, const float* A2, int K2, const float* B, int N, float* part,
                      float* tot, float* grad, cudaStream_t s) {
  if (V <= 0) return STG_OK;
  const int NB = (N + 31) / 32, Np = 32 * NB, n1 = (K1 + 31) / 32, n2 = K2 > 0 ? (K2 + 31) / 32 : 0;
  CUtensorMap m[4], ones;
  STG_TRY(make_tmap_f32(&m[0], A1, (uint64_t)V, K1, K1, 32, kAtbRT, true));
  if (K2 > 0) STG_TRY(make_tmap_f32(&m[1], A2, (uint64_t)V, K2, K2, 32, kAtbRT, true));
  else m[1] = m[0];
  STG_TRY(make_tmap_f32(&m[2], B, (uint64_t)V, N, N, 32, kAtbRT, true));
  m[3] = m[0];
  STG_TRY(ones_map(&ones, kAtbRT, s));
  AtbSpec2 sp{};
  sp.V = V; sp.na = 1; sp.a_first[0] = 0; sp.nsa = n1 + n2; sp.nb = NB; sp.b_map = 2; sp.part = part;
  for (int k = 0; k < n1; ++k) { sp.src_map[k] = 0; sp.src_col[k] = 32 * k; }
  for (int k = 0; k < n2; ++k) { sp.src_map[n1 + k] = 1; sp.src_col[n1 + k] = 32 * k; }
  int nb = 0;
  STG_TRY(atb2_dispatch(NB, m, ones, sp, &nb, s));
  const int n = 128 * Np;
  if (nb <= 16 * kSumMaxGroups) k_tc_sum_parts2<<<(n + 31) / 32, 256, 0, s>>>(part, nb, n, tot);
  else k_tc_sum_parts<<<(n + 255) / 256, 256, 0, s>>>(part, nb, n, tot);
  k_cat_scatter<<<((K1 + K2) * N + 255) / 256, 256, 0, s>>>(K1, K2, N, 32 * n1, Np, tot, grad);
  count_launch(2);
  return check_launch("tc_atb_cat");
}

}  // namespace stg
