// tc_tgcn.cu — the TGCN dense contractions on 5th-gen tensor cores (tcgen05,
// 3xTF32 for fp32-class accuracy, accumulators in TMEM).  Each kernel is a
// persistent loop over 128-row tiles (one row per thread in the epilogue):
//
//   k_tc_xw      P' = diag(n_src)·X·W                  (K = F, N = 3H)
//   k_tc_gru_fwd a_z = [C_z|H]·L_z, a_r = [C_r|H]·L_r   (MMA, K = 2H, N = H each)
//                Z, R = σ(·+l);  RH = R⊙H  staged in smem
//                a_h = [C_h|RH]·L_h → Ĥ = tanh, H' = Z⊙H + (1−Z)⊙Ĥ
//   k_tc_gru_bwd recompute a_z, a_r, a_h (as above), then
//                [dC_h|dRH] = da_h·L_hᵀ, [dC_z|dH_z] = da_z·L_zᵀ, [dC_r|dH_r] = da_r·L_rᵀ
//                (MMA, K = H, N = 2H each) and the elementwise chain rule;
//                writes dC' = n_dst⊙dC, dH_prev, and da = [da_z|da_r|da_h], RH
//                for the parameter-gradient reduction
//   k_tc_atb     D = Σ_rows A[r,:]ᵀ·B[r,:] with A, B staged transposed (K = rows),
//                per-CTA partials, fixed-order reduction → dW, dL, dl.
//
// The equations are those of SURVEY §8(c) (readings C13-C15).
#include <algorithm>
#include <map>
#include <mutex>

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

__device__ __forceinline__ uint32_t tmem_row(uint32_t base, int col) {
  return base + ((uint32_t)((threadIdx.x >> 5) * 32) << 16) + (uint32_t)col;
}

template <int N>
__device__ __forceinline__ void tmem_row_load(uint32_t base, int col, float (&v)[N]) {
  static_assert(N % 16 == 0, "N % 16");
#pragma unroll
  for (int c = 0; c < N; c += 16) {
    float t[16];
    tc::tmem_ld16(tmem_row(base, col + c), t);
#pragma unroll
    for (int i = 0; i < 16; ++i) v[c + i] = t[i];
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
  for (int e = threadIdx.x; e < 2 * H * H; e += kTcThreads) {
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

// Writes RH (row-local, into columns [H, 2H) of the width-2H A2 tile).
template <int H>
__device__ __forceinline__ void stage_row_vec(unsigned char* hi, unsigned char* lo, int r, int k0, int K,
                                              const float* v) {
#pragma unroll
  for (int q = 0; q < H / 4; ++q)
    tc::st_split4(hi, lo, r, k0 / 4 + q, K, make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]));
}

// ------------------------------------------------------------------ GRU forward
template <int H>
__global__ void __launch_bounds__(kTcThreads, 1) k_tc_gru_fwd(int V, const float* __restrict__ C,
                                                              const float* __restrict__ Hp,
                                                              const float* __restrict__ L,
                                                              const float* __restrict__ l, float* __restrict__ Hn) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ uint64_t mbar;
  __shared__ uint32_t tslot;
  constexpr int BG = GruSmem<H>::BG, A1 = GruSmem<H>::A1, H3 = 3 * H;
  unsigned char* bz_hi = sm;               unsigned char* bz_lo = bz_hi + BG;
  unsigned char* br_hi = bz_lo + BG;       unsigned char* br_lo = br_hi + BG;
  unsigned char* bh_hi = br_lo + BG;       unsigned char* bh_lo = bh_hi + BG;
  unsigned char* ahi = bh_lo + BG;         unsigned char* alo = ahi + A1;
  const int LG = 2 * H * H;
  stage_gate_weights<H>(bz_hi, bz_lo, L);
  stage_gate_weights<H>(br_hi, br_lo, L + LG);
  stage_gate_weights<H>(bh_hi, bh_lo, L + 2 * LG);
  if ((threadIdx.x >> 5) == 0) tc::tmem_alloc(&tslot, 128);
  if (threadIdx.x == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  uint32_t phase = 0;
  const int ntiles = (V + 127) / 128;
  const int t = threadIdx.x;
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int r0 = tile * 128, nv = V - r0, row = r0 + t;
    // A1 = [C_z | C_r | H]
    tc::stage_rows(ahi, alo, C + (int64_t)r0 * H3, H3, nv, 128, 2 * H, 0, 0, H3);
    tc::stage_rows(ahi, alo, Hp + (int64_t)r0 * H, H, nv, 128, H, 0, 2 * H, H3);
    sync_mma_operands();
    if (t == 0) {
      issue_zr<H>(tm, ahi, alo, bz_hi, bz_lo, br_hi, br_lo);
      tc::commit(&mbar);
    }
    wait_mma(&mbar, phase);
    float z[H], rh[H], h[H];
    {
      float a[2 * H];
      tmem_row_load<2 * H>(tm, 0, a);
#pragma unroll
      for (int j = 0; j < H; ++j) h[j] = 0.f;
      if (row < V) {
        const float4* hp = reinterpret_cast<const float4*>(Hp + (int64_t)row * H);
#pragma unroll
        for (int q = 0; q < H / 4; ++q) {
          float4 x = __ldg(hp + q);
          h[4 * q] = x.x; h[4 * q + 1] = x.y; h[4 * q + 2] = x.z; h[4 * q + 3] = x.w;
        }
      }
#pragma unroll
      for (int j = 0; j < H; ++j) {
        z[j] = sigm(a[j] + __ldg(l + j));
        rh[j] = sigm(a[H + j] + __ldg(l + H + j)) * h[j];
      }
    }
    // A2 = [C_h | RH] (width 2H) reuses the A1 storage (MMA on A1 has completed)
    tc::stage_rows(ahi, alo, C + (int64_t)r0 * H3, H3, nv, 128, H, 2 * H, 0, 2 * H);
    stage_row_vec<H>(ahi, alo, t, H, 2 * H, rh);
    sync_mma_operands();
    if (t == 0) {
      const uint32_t idesc = tc::idesc_tf32(128, H, 0, 0);
      mma_seg(tm + 2 * H, tc::smem_u32(ahi), tc::smem_u32(alo), 2 * H, 0, tc::smem_u32(bh_hi), tc::smem_u32(bh_lo),
              2 * H, 0, 2 * H, idesc, true);
      tc::commit(&mbar);
    }
    wait_mma(&mbar, phase);
    {
      float a[H];
      tmem_row_load<H>(tm, 2 * H, a);
      if (row < V) {
        float4* out = reinterpret_cast<float4*>(Hn + (int64_t)row * H);
#pragma unroll
        for (int q = 0; q < H / 4; ++q) {
          float o[4];
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const int j = 4 * q + i;
            const float hh = tanhf(a[j] + __ldg(l + 2 * H + j));
            o[i] = z[j] * h[j] + (1.0f - z[j]) * hh;
          }
          out[q] = make_float4(o[0], o[1], o[2], o[3]);
        }
      }
    }
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
  }
  tc::fence_before();
  __syncthreads();
  if ((threadIdx.x >> 5) == 0) tc::tmem_free(tm, 128);
}

// ------------------------------------------------------------------ GRU backward
template <int H>
__global__ void __launch_bounds__(kTcThreads, 1) k_tc_gru_bwd(int V, const float* __restrict__ C,
                                                              const float* __restrict__ Hp,
                                                              const float* __restrict__ G,
                                                              const float* __restrict__ L,
                                                              const float* __restrict__ l,
                                                              const float* __restrict__ ndst,
                                                              float* __restrict__ dCs, float* __restrict__ dHp,
                                                              float* __restrict__ da, float* __restrict__ RHo) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ uint64_t mbar;
  __shared__ uint32_t tslot;
  constexpr int BG = GruSmem<H>::BG, A1 = GruSmem<H>::A1, H3 = 3 * H;
  unsigned char* bz_hi = sm;               unsigned char* bz_lo = bz_hi + BG;
  unsigned char* br_hi = bz_lo + BG;       unsigned char* br_lo = br_hi + BG;
  unsigned char* bh_hi = br_lo + BG;       unsigned char* bh_lo = bh_hi + BG;
  unsigned char* lz_hi = bh_lo + BG;       unsigned char* lz_lo = lz_hi + BG;
  unsigned char* lr_hi = lz_lo + BG;       unsigned char* lr_lo = lr_hi + BG;
  unsigned char* lh_hi = lr_lo + BG;       unsigned char* lh_lo = lh_hi + BG;
  unsigned char* ahi = lh_lo + BG;         unsigned char* alo = ahi + A1;
  const int LG = 2 * H * H;
  stage_gate_weights<H>(bz_hi, bz_lo, L);
  stage_gate_weights<H>(br_hi, br_lo, L + LG);
  stage_gate_weights<H>(bh_hi, bh_lo, L + 2 * LG);
  stage_plain<H>(lz_hi, lz_lo, L);
  stage_plain<H>(lr_hi, lr_lo, L + LG);
  stage_plain<H>(lh_hi, lh_lo, L + 2 * LG);
  // TMEM columns: Dz [0,H), Dr [H,2H), Dh [2H,3H), D3 [4H,6H), D4z [6H,8H), D4r [8H,10H)
  constexpr uint32_t NC = 10 * H <= 256 ? 256 : 512;
  if ((threadIdx.x >> 5) == 0) tc::tmem_alloc(&tslot, NC);
  if (threadIdx.x == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  uint32_t phase = 0;
  const int ntiles = (V + 127) / 128;
  const int t = threadIdx.x;
  const uint32_t id_h = tc::idesc_tf32(128, H, 0, 0), id_2h = tc::idesc_tf32(128, 2 * H, 0, 0);
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int r0 = tile * 128, nv = V - r0, row = r0 + t;
    const bool ok = row < V;
    tc::stage_rows(ahi, alo, C + (int64_t)r0 * H3, H3, nv, 128, 2 * H, 0, 0, H3);
    tc::stage_rows(ahi, alo, Hp + (int64_t)r0 * H, H, nv, 128, H, 0, 2 * H, H3);
    sync_mma_operands();
    if (t == 0) {
      issue_zr<H>(tm, ahi, alo, bz_hi, bz_lo, br_hi, br_lo);
      tc::commit(&mbar);
    }
    wait_mma(&mbar, phase);
    float z[H], r[H], h[H], dh[H];
    {
      float a[2 * H];
      tmem_row_load<2 * H>(tm, 0, a);
#pragma unroll
      for (int j = 0; j < H; ++j) h[j] = 0.f;
      if (ok) {
        const float4* hp = reinterpret_cast<const float4*>(Hp + (int64_t)row * H);
#pragma unroll
        for (int q = 0; q < H / 4; ++q) {
          float4 x = __ldg(hp + q);
          h[4 * q] = x.x; h[4 * q + 1] = x.y; h[4 * q + 2] = x.z; h[4 * q + 3] = x.w;
        }
      }
#pragma unroll
      for (int j = 0; j < H; ++j) {
        z[j] = sigm(a[j] + __ldg(l + j));
        r[j] = sigm(a[H + j] + __ldg(l + H + j));
        dh[j] = r[j] * h[j];                        // RH for now
      }
    }
    tc::stage_rows(ahi, alo, C + (int64_t)r0 * H3, H3, nv, 128, H, 2 * H, 0, 2 * H);
    stage_row_vec<H>(ahi, alo, t, H, 2 * H, dh);
    if (ok) {
      float4* o = reinterpret_cast<float4*>(RHo + (int64_t)row * H);
#pragma unroll
      for (int q = 0; q < H / 4; ++q) o[q] = make_float4(dh[4 * q], dh[4 * q + 1], dh[4 * q + 2], dh[4 * q + 3]);
    }
    sync_mma_operands();
    if (t == 0) {
      mma_seg(tm + 2 * H, tc::smem_u32(ahi), tc::smem_u32(alo), 2 * H, 0, tc::smem_u32(bh_hi), tc::smem_u32(bh_lo),
              2 * H, 0, 2 * H, id_h, true);
      tc::commit(&mbar);
    }
    wait_mma(&mbar, phase);
    // A3 = da_h [128 × H] (K = H), A4z = da_z, A4r = da_r placed after it
    unsigned char* a3h = ahi;                      unsigned char* a3l = alo;
    unsigned char* a4zh = ahi + 128 * H * 4;       unsigned char* a4zl = alo + 128 * H * 4;
    unsigned char* a4rh = ahi + 2 * 128 * H * 4;   unsigned char* a4rl = alo + 2 * 128 * H * 4;
    {
      float a[H], g[H], dah[H], daz[H];
      tmem_row_load<H>(tm, 2 * H, a);
#pragma unroll
      for (int j = 0; j < H; ++j) g[j] = 0.f;
      if (ok) {
        const float4* gp = reinterpret_cast<const float4*>(G + (int64_t)row * H);
#pragma unroll
        for (int q = 0; q < H / 4; ++q) {
          float4 x = __ldg(gp + q);
          g[4 * q] = x.x; g[4 * q + 1] = x.y; g[4 * q + 2] = x.z; g[4 * q + 3] = x.w;
        }
      }
#pragma unroll
      for (int j = 0; j < H; ++j) {
        const float hh = tanhf(a[j] + __ldg(l + 2 * H + j));
        const float dZ = g[j] * (h[j] - hh), dHh = g[j] * (1.0f - z[j]);
        dah[j] = dHh * (1.0f - hh * hh);
        daz[j] = dZ * z[j] * (1.0f - z[j]);
        dh[j] = g[j] * z[j];
      }
      stage_row_vec<H>(a3h, a3l, t, 0, H, dah);
      stage_row_vec<H>(a4zh, a4zl, t, 0, H, daz);
      if (ok) {
        float4* oa = reinterpret_cast<float4*>(da + (int64_t)row * H3);
#pragma unroll
        for (int q = 0; q < H / 4; ++q) {
          oa[q] = make_float4(daz[4 * q], daz[4 * q + 1], daz[4 * q + 2], daz[4 * q + 3]);
          oa[H / 2 + q] = make_float4(dah[4 * q], dah[4 * q + 1], dah[4 * q + 2], dah[4 * q + 3]);
        }
      }
    }
    sync_mma_operands();
    if (t == 0) {
      mma_seg(tm + 4 * H, tc::smem_u32(a3h), tc::smem_u32(a3l), H, 0, tc::smem_u32(lh_hi), tc::smem_u32(lh_lo), H, 0,
              H, id_2h, true);
      mma_seg(tm + 6 * H, tc::smem_u32(a4zh), tc::smem_u32(a4zl), H, 0, tc::smem_u32(lz_hi), tc::smem_u32(lz_lo), H,
              0, H, id_2h, true);
      tc::commit(&mbar);
    }
    wait_mma(&mbar, phase);
    const float nd = ok ? ndst[row] : 0.f;
    {
      float a[2 * H], dar[H];
      tmem_row_load<2 * H>(tm, 4 * H, a);              // [dC_h | dRH]
      if (ok) {
        float4* o = reinterpret_cast<float4*>(dCs + (int64_t)row * H3 + 2 * H);
#pragma unroll
        for (int q = 0; q < H / 4; ++q)
          o[q] = make_float4(nd * a[4 * q], nd * a[4 * q + 1], nd * a[4 * q + 2], nd * a[4 * q + 3]);
      }
#pragma unroll
      for (int j = 0; j < H; ++j) {
        const float dRH = a[H + j];
        dh[j] += dRH * r[j];
        dar[j] = dRH * h[j] * r[j] * (1.0f - r[j]);
      }
      stage_row_vec<H>(a4rh, a4rl, t, 0, H, dar);
      if (ok) {
        float4* oa = reinterpret_cast<float4*>(da + (int64_t)row * H3 + H);
#pragma unroll
        for (int q = 0; q < H / 4; ++q) oa[q] = make_float4(dar[4 * q], dar[4 * q + 1], dar[4 * q + 2], dar[4 * q + 3]);
      }
    }
    sync_mma_operands();
    if (t == 0) {
      mma_seg(tm + 8 * H, tc::smem_u32(a4rh), tc::smem_u32(a4rl), H, 0, tc::smem_u32(lr_hi), tc::smem_u32(lr_lo), H,
              0, H, id_2h, true);
      tc::commit(&mbar);
    }
    wait_mma(&mbar, phase);
#pragma unroll
    for (int half = 0; half < 2; ++half) {               // [dC_z | dH_z], then [dC_r | dH_r]
      float a[2 * H];
      tmem_row_load<2 * H>(tm, (6 + 2 * half) * H, a);
      if (ok) {
        float4* o = reinterpret_cast<float4*>(dCs + (int64_t)row * H3 + half * H);
#pragma unroll
        for (int q = 0; q < H / 4; ++q)
          o[q] = make_float4(nd * a[4 * q], nd * a[4 * q + 1], nd * a[4 * q + 2], nd * a[4 * q + 3]);
      }
#pragma unroll
      for (int j = 0; j < H; ++j) dh[j] += a[H + j];
    }
    if (ok) {
      float4* od = reinterpret_cast<float4*>(dHp + (int64_t)row * H);
#pragma unroll
      for (int q = 0; q < H / 4; ++q) od[q] = make_float4(dh[4 * q], dh[4 * q + 1], dh[4 * q + 2], dh[4 * q + 3]);
    }
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
  }
  tc::fence_before();
  __syncthreads();
  if ((threadIdx.x >> 5) == 0) tc::tmem_free(tm, NC);
}

// ------------------------------------------------------------------ Σ_rows Aᵀ·B
// A = [A1 (FA1 cols) | A2 (FA2 cols) | ones (if ones)] padded to 128 features;
// B = [B1 (N cols)].  Tiles of RK rows are staged transposed (K = rows).
// Per-CTA partial D [128 × N] written to part[blockIdx.x].
constexpr int kRK = 64;

template <int N>
__global__ void __launch_bounds__(kTcThreads) k_tc_atb(int V, const float* __restrict__ A1, int64_t lda1, int FA1,
                                                       const float* __restrict__ A2, int64_t lda2, int FA2, int ones,
                                                       const float* __restrict__ B, int64_t ldb, int FB,
                                                       float* __restrict__ part) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ uint64_t mbar;
  __shared__ uint32_t tslot;
  unsigned char* ahi = sm;
  unsigned char* alo = ahi + 128 * kRK * 4;
  unsigned char* bhi = alo + 128 * kRK * 4;
  unsigned char* blo = bhi + N * kRK * 4;
  constexpr uint32_t NC = N <= 32 ? 32 : (N <= 64 ? 64 : (N <= 128 ? 128 : 256));
  const int FA = FA1 + FA2;
  // zero the padded feature rows [FA, 128) once (ones row set per tile below)
  for (int e = threadIdx.x; e < 128 * kRK; e += kTcThreads) {
    const int f = e / kRK, k = e % kRK;
    if (f >= FA) {
      const float v = (ones && f == FA) ? 1.0f : 0.0f;
      *reinterpret_cast<float*>(ahi + tc::kmaj_off(f, k, kRK)) = v;
      *reinterpret_cast<float*>(alo + tc::kmaj_off(f, k, kRK)) = 0.0f;
    }
  }
  for (int e = threadIdx.x; e < (N - FB) * kRK; e += kTcThreads) {   // zero B feature padding once
    const int f = FB + e / kRK, k = e % kRK;
    *reinterpret_cast<float*>(bhi + tc::kmaj_off(f, k, kRK)) = 0.0f;
    *reinterpret_cast<float*>(blo + tc::kmaj_off(f, k, kRK)) = 0.0f;
  }
  if ((threadIdx.x >> 5) == 0) tc::tmem_alloc(&tslot, NC);
  if (threadIdx.x == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = tslot;
  uint32_t phase = 0;
  const uint32_t idesc = tc::idesc_tf32(128, N, 0, 0);
  const int ntiles = (V + kRK - 1) / kRK;
  bool first = true;
  for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int r0 = tile * kRK, nv = V - r0;
    tc::stage_rows_T(ahi, alo, A1 + (int64_t)r0 * lda1, lda1, nv, FA1, 0, 0, kRK);
    if (FA2) tc::stage_rows_T(ahi, alo, A2 + (int64_t)r0 * lda2, lda2, nv, FA2, 0, FA1, kRK);
    if (ones && nv < kRK) {   // ones row must be zero on padding rows of the last tile
      for (int k = threadIdx.x; k < kRK; k += kTcThreads)
        *reinterpret_cast<float*>(ahi + tc::kmaj_off(FA, k, kRK)) = k < nv ? 1.0f : 0.0f;
    }
    tc::stage_rows_T(bhi, blo, B + (int64_t)r0 * ldb, ldb, nv, FB, 0, 0, kRK);
    sync_mma_operands();
    if (threadIdx.x == 0) {
      mma_seg(tm, tc::smem_u32(ahi), tc::smem_u32(alo), kRK, 0, tc::smem_u32(bhi), tc::smem_u32(blo), kRK, 0, kRK,
              idesc, first);
      tc::commit(&mbar);
    }
    wait_mma(&mbar, phase);
    first = false;
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
  }
  // epilogue: thread t = feature row t of D
  float* out = part + (int64_t)blockIdx.x * 128 * N + (int64_t)threadIdx.x * N;
  if (first) {
    for (int c = 0; c < N; ++c) out[c] = 0.f;
  } else {
    float v[N];
    tmem_row_load<N>(tm, 0, v);
    for (int c = 0; c < N; ++c) out[c] = v[c];
  }
  tc::fence_before();
  __syncthreads();
  if ((threadIdx.x >> 5) == 0) tc::tmem_free(tm, NC);
}

// out[i] += Σ_b part[b][map(i)] in a fixed order (blocks of 16), for the
// [rows × cols] sub-block starting at (row0, col0) of the [128 × N] partials;
// transpose != 0 writes out[c*rows + r].
__global__ void k_tc_reduce(const float* __restrict__ part, int nb, int N, int row0, int rows, int col0, int cols,
                            int transpose, float* __restrict__ out) {
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < rows * cols; e += gridDim.x * blockDim.x) {
    const int r = e / cols, c = e % cols;
    const int64_t src = (int64_t)(row0 + r) * N + col0 + c;
    float tot = 0.f;
    for (int b0 = 0; b0 < nb; b0 += 16) {
      float blk = 0.f;
      const int b1 = min(b0 + 16, nb);
      for (int b = b0; b < b1; ++b) blk += part[(int64_t)b * 128 * N + src];
      tot += blk;
    }
    out[transpose ? (int64_t)c * rows + r : (int64_t)r * cols + c] += tot;
  }
}

// db = Σ_rows dC = dl_g·L_g¹ᵀ per gate (linear in the per-gate sums of da).
__global__ void k_db_from_dl(int H, const float* __restrict__ dl_new, const float* __restrict__ L,
                             float* __restrict__ db) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= 3 * H) return;
  const int g = c / H, i = c % H;
  const float* Lg = L + (int64_t)g * 2 * H * H;
  float s = 0.f;
  for (int j = 0; j < H; ++j) s = fmaf(dl_new[g * H + j], Lg[i * H + j], s);
  db[c] += s;
}

template <class K>
int occupancy_blocks(K fn, size_t smem) {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kTcThreads, smem) != cudaSuccess || per_sm < 1) {
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
// part for tc_dw / tc_dl: 2 · tc_atb_max_blocks() · 128 · max(3H, roundup16(F)) floats

stg_status tc_xw(int V, int F, int H, const float* X, const float* W, const float* rs, float* P, cudaStream_t s) {
  const int N = 3 * H, Kp = (F + 7) / 8 * 8;
  const size_t smem = (size_t)2 * N * Kp * 4 + (size_t)2 * 128 * Kp * 4;
  const int ntiles = (V + 127) / 128;
  if (H == 32) {
    STG_TRY(prep(k_tc_xw<96>, smem));
    const int nb = std::min(ntiles, occupancy_blocks(k_tc_xw<96>, smem));
    k_tc_xw<96><<<nb, kTcThreads, smem, s>>>(V, F, Kp, X, W, rs, P);
  } else {
    STG_TRY(prep(k_tc_xw<48>, smem));
    const int nb = std::min(ntiles, occupancy_blocks(k_tc_xw<48>, smem));
    k_tc_xw<48><<<nb, kTcThreads, smem, s>>>(V, F, Kp, X, W, rs, P);
  }
  count_launch();
  return check_launch("tc_xw");
}

stg_status tc_gru_fwd(int V, int H, const float* C, const float* Hp, const float* L, const float* l, float* Hn,
                      cudaStream_t s) {
  const int ntiles = (V + 127) / 128;
  if (H == 32) {
    const size_t smem = 6 * GruSmem<32>::BG + 2 * GruSmem<32>::A1;
    STG_TRY(prep(k_tc_gru_fwd<32>, smem));
    const int nb = std::min(ntiles, occupancy_blocks(k_tc_gru_fwd<32>, smem));
    k_tc_gru_fwd<32><<<nb, kTcThreads, smem, s>>>(V, C, Hp, L, l, Hn);
  } else {
    const size_t smem = 6 * GruSmem<16>::BG + 2 * GruSmem<16>::A1;
    STG_TRY(prep(k_tc_gru_fwd<16>, smem));
    const int nb = std::min(ntiles, occupancy_blocks(k_tc_gru_fwd<16>, smem));
    k_tc_gru_fwd<16><<<nb, kTcThreads, smem, s>>>(V, C, Hp, L, l, Hn);
  }
  count_launch();
  return check_launch("tc_gru_fwd");
}

stg_status tc_gru_bwd(int V, int H, const float* C, const float* Hp, const float* G, const float* L, const float* l,
                      const float* ndst, float* dCs, float* dHp, float* da, float* RH, cudaStream_t s) {
  const int ntiles = (V + 127) / 128;
  if (H == 32) {
    const size_t smem = 12 * GruSmem<32>::BG + 2 * GruSmem<32>::A1;
    STG_TRY(prep(k_tc_gru_bwd<32>, smem));
    const int nb = std::min(ntiles, occupancy_blocks(k_tc_gru_bwd<32>, smem));
    k_tc_gru_bwd<32><<<nb, kTcThreads, smem, s>>>(V, C, Hp, G, L, l, ndst, dCs, dHp, da, RH);
  } else {
    const size_t smem = 12 * GruSmem<16>::BG + 2 * GruSmem<16>::A1;
    STG_TRY(prep(k_tc_gru_bwd<16>, smem));
    const int nb = std::min(ntiles, occupancy_blocks(k_tc_gru_bwd<16>, smem));
    k_tc_gru_bwd<16><<<nb, kTcThreads, smem, s>>>(V, C, Hp, G, L, l, ndst, dCs, dHp, da, RH);
  }
  count_launch();
  return check_launch("tc_gru_bwd");
}

// part must hold grid_max * 128 * N floats; returns the number of partial blocks.
template <int N>
static stg_status atb(int V, const float* A1, int64_t lda1, int FA1, const float* A2, int64_t lda2, int FA2, int ones,
                      const float* B, int64_t ldb, int FB, float* part, int max_blocks, int* nb_out, cudaStream_t s) {
  const size_t smem = (size_t)2 * 128 * kRK * 4 + (size_t)2 * N * kRK * 4;
  STG_TRY(prep(k_tc_atb<N>, smem));
  const int ntiles = (V + kRK - 1) / kRK;
  int nb = std::min(std::min(ntiles, occupancy_blocks(k_tc_atb<N>, smem)), max_blocks);
  if (nb < 1) nb = 1;
  k_tc_atb<N><<<nb, kTcThreads, smem, s>>>(V, A1, lda1, FA1, A2, lda2, FA2, ones, B, ldb, FB, part);
  count_launch();
  *nb_out = nb;
  return check_launch("tc_atb");
}

int tc_atb_max_blocks() { return 2 * num_sms(); }

// dW[f][c] += Σ_v X[v,f]·dP[v,c]  via D = dPᵀ·X  ([3H pad 128] × F)
stg_status tc_dw(int V, int F, int H, const float* X, const float* dP, float* part, float* dW, cudaStream_t s) {
  int nb = 0;
  const int Np = (F + 15) / 16 * 16;
  switch (Np) {
    case 16: STG_TRY(atb<16>(V, dP, 3 * H, 3 * H, nullptr, 0, 0, 0, X, F, F, part, tc_atb_max_blocks(), &nb, s)); break;
    case 32: STG_TRY(atb<32>(V, dP, 3 * H, 3 * H, nullptr, 0, 0, 0, X, F, F, part, tc_atb_max_blocks(), &nb, s)); break;
    case 48: STG_TRY(atb<48>(V, dP, 3 * H, 3 * H, nullptr, 0, 0, 0, X, F, F, part, tc_atb_max_blocks(), &nb, s)); break;
    case 64: STG_TRY(atb<64>(V, dP, 3 * H, 3 * H, nullptr, 0, 0, 0, X, F, F, part, tc_atb_max_blocks(), &nb, s)); break;
    case 96: STG_TRY(atb<96>(V, dP, 3 * H, 3 * H, nullptr, 0, 0, 0, X, F, F, part, tc_atb_max_blocks(), &nb, s)); break;
    case 128: STG_TRY(atb<128>(V, dP, 3 * H, 3 * H, nullptr, 0, 0, 0, X, F, F, part, tc_atb_max_blocks(), &nb, s)); break;
    default: return fail(STG_ERR_INVALID_ARG, "tc_dw: F=%d", F);
  }
  // D row c (dP feature) × column f (X feature) -> dW[f][c] (transpose)
  k_tc_reduce<<<(3 * H * F + 255) / 256, 256, 0, s>>>(part, nb, Np, 0, 3 * H, 0, F, 1, dW);
  count_launch();
  return check_launch("tc_dw");
}

// dL, dl, db from C, H, RH, da (see k_tc_gru_bwd).  scratch: part (2 × max_blocks × 128 × 3H), dl_tmp [3H].
stg_status tc_dl(int V, int H, const float* C, const float* Hp, const float* RH, const float* da, float* part,
                 float* dl_tmp, float* dL, float* dl, float* db, const float* L, cudaStream_t s) {
  const int H3 = 3 * H, LG = 2 * H * H;
  int nb1 = 0, nb2 = 0;
  float* part2 = part + (size_t)tc_atb_max_blocks() * 128 * H3;
  // D1 = [C_z|C_r|C_h|H]ᵀ · [da_z|da_r|da_h]   (4H = 128 feature rows for H = 32)
  // D2 = [RH | 1]ᵀ · [da_z|da_r|da_h]
  if (H == 32) {
    STG_TRY(atb<96>(V, C, H3, H3, Hp, H, H, 0, da, H3, H3, part, tc_atb_max_blocks(), &nb1, s));
    STG_TRY(atb<96>(V, RH, H, H, nullptr, 0, 0, 1, da, H3, H3, part2, tc_atb_max_blocks(), &nb2, s));
  } else {
    STG_TRY(atb<48>(V, C, H3, H3, Hp, H, H, 0, da, H3, H3, part, tc_atb_max_blocks(), &nb1, s));
    STG_TRY(atb<48>(V, RH, H, H, nullptr, 0, 0, 1, da, H3, H3, part2, tc_atb_max_blocks(), &nb2, s));
  }
  for (int g = 0; g < 3; ++g) {
    // dL_g¹ [H × H] = D1 block (rows gH.., cols gH..); dL_g² (z, r) = D1 rows 3H.., cols gH..
    k_tc_reduce<<<(H * H + 255) / 256, 256, 0, s>>>(part, nb1, H3, g * H, H, g * H, H, 0, dL + g * LG);
    if (g < 2)
      k_tc_reduce<<<(H * H + 255) / 256, 256, 0, s>>>(part, nb1, H3, 3 * H, H, g * H, H, 0, dL + g * LG + H * H);
    else
      k_tc_reduce<<<(H * H + 255) / 256, 256, 0, s>>>(part2, nb2, H3, 0, H, 2 * H, H, 0, dL + g * LG + H * H);
  }
  cudaMemsetAsync(dl_tmp, 0, sizeof(float) * H3, s);
  k_tc_reduce<<<1, 256, 0, s>>>(part2, nb2, H3, H, 1, 0, H3, 0, dl_tmp);
  k_db_from_dl<<<1, 128, 0, s>>>(H, dl_tmp, L, db);
  count_launch(7);
  // dl += dl_tmp
  k_tc_reduce<<<1, 256, 0, s>>>(part2, nb2, H3, H, 1, 0, H3, 0, dl);
  count_launch();
  return check_launch("tc_dl");
}

}  // namespace stg
