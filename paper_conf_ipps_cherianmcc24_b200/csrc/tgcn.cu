// tgcn.cu — TGCN step (GCN + GRU, readings C13-C15), State Stack,
// surrogate MSE head, SGD, and Algorithm 1's per-sequence driver.
//
// Per timestamp (a7):  P' = diag(n_src)·X·W   (k_xw, row-scale epilogue)
//                      C  = diag(n_dst)·A·P' + b  (aggregation kernel, bias epilogue)
//                      Z, R, Ĥ, H'               (k_gru_fwd, fused)
// Backward (a8):       k_gru_bwd (recompute gates, chain rule, dC' = n_dst⊙dC,
//                      per-block parameter-gradient partials) → aggregation over
//                      the out-CSR (dP) → k_dw (Xᵀ·dP partials) → fixed-order
//                      reduction.  No float atomics: deterministic run to run.
#include <algorithm>
#include <atomic>
#include <map>
#include <mutex>
#include <vector>

#include "graph.cuh"

namespace stg {
bool dtdg_materialised(const stg_dtdg* g);
bool tc_supported(int F, int H);
int tc_atb_max_blocks();
stg_status tc_xw(int V, int F, int H, const float* X, const float* W, const float* rs, float* P, cudaStream_t s,
                 int rs_div = 1, const float* bias = nullptr);
stg_status tc_gru_seq_fwd(int V, int S, int H, const float* C_all, const float* H0, const float* L, const float* l,
                          float* H_seq, float* Hp_all, const float* Y_all, const float* w_o, const float* b_o,
                          double* lpart, int* nb_out, cudaStream_t s);
stg_status tc_gru_seq_bwd(int V, int S, int H, const float* C_all, const float* Hp_all, const float* H_seq,
                          const float* L, const float* l, const float* ndst, const float* Y_all, const float* w_o,
                          const float* b_o, float inv_vn, float* dC_all, float* da_all, float* RH_all, float* gpart,
                          int* nb_out, cudaStream_t s);
stg_status tc_seq_head_reduce(int nb, int H, const double* lpart, const float* gpart, double inv_vn, float* loss,
                              float* dw_o, float* db_o, cudaStream_t s);
stg_status tc_gru_fwd(int V, int H, const float* C, const float* Hp, const float* L, const float* l, float* Hn,
                      cudaStream_t s, const HeadArgs* head = nullptr);
stg_status tc_gru_bwd(int V, int H, const float* C, const float* Hp, const float* G, const float* L, const float* l,
                      const float* ndst, float* dCs, float* dHp, float* da, float* RH, cudaStream_t s,
                      const float2* hg = nullptr, const float* w_o = nullptr);
int tc_gru_blocks(int V);
bool tc_cat_supported(int K1, int K2, int N);
stg_status tc_catmm(int V, const float* A1, int K1, int64_t ld1, const float* A2, int K2, int64_t ld2, const float* W,
                    int64_t sk, int64_t sn, int N, const float* rs, float* out, int64_t ldo, bool accumulate,
                    cudaStream_t s);
stg_status tc_atb_cat(int V, const float* A1, int K1, const float* A2, int K2, const float* B, int N, float* part,
                      float* tot, float* grad, cudaStream_t s);
stg_status tc_dw(int V, int F, int H, const float* X, const float* dP, float* part, float* tot, float* dW,
                 cudaStream_t s);
stg_status tc_dl(int V, int H, const float* C, const float* Hp, const float* RH, const float* da, float* part,
                 float* tot, float* dL, float* dl, float* db, const float* L, cudaStream_t s);
}

namespace stg {
namespace {

constexpr int kT = 256;  // threads per block for the TGCN kernels

__device__ __forceinline__ float sigm(float a) { return 1.0f / (1.0f + expf(-a)); }

// ---------------------------------------------------------------- P' = n ⊙ XW
// Row tile of 32 rows; W [F, N] and the X tile live in shared memory.
__global__ void __launch_bounds__(kT) k_xw(int32_t V, int32_t F, int32_t N, const float* __restrict__ X,
                                           const float* __restrict__ W, const float* __restrict__ rs,
                                           float* __restrict__ P) {
  extern __shared__ float sm[];
  float* sW = sm;                 // [F][N]
  float* sX = sm + F * N;         // [32][F]
  constexpr int BR = 32;
  for (int i = threadIdx.x; i < F * N; i += kT) sW[i] = W[i];
  const int64_t ntiles = (V + BR - 1) / BR;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t r0 = tile * BR;
    __syncthreads();
    for (int i = threadIdx.x; i < BR * F; i += kT) {
      int64_t r = r0 + i / F;
      sX[i] = r < V ? X[r * F + i % F] : 0.0f;
    }
    __syncthreads();
    for (int o = threadIdx.x; o < BR * N; o += kT) {
      const int r = o / N, c = o % N;
      if (r0 + r >= V) continue;
      const float* xr = sX + r * F;
      float acc = 0.0f;
      for (int f = 0; f < F; ++f) acc = fmaf(xr[f], sW[f * N + c], acc);
      P[(r0 + r) * N + c] = rs ? rs[r0 + r] * acc : acc;
    }
  }
}

// ---------------------------------------------------------------- GRU forward
// Row tile of BR rows.  smem: L [3][2H][H], l [3][H], C [BR][3H], H [BR][H],
// Z, R, RH [BR][H].
template <int BR>
__global__ void __launch_bounds__(kT) k_gru_fwd(int32_t V, int32_t H, const float* __restrict__ C,
                                                const float* __restrict__ Hp, const float* __restrict__ L,
                                                const float* __restrict__ l, float* __restrict__ Hn) {
  extern __shared__ float sm[];
  const int H3 = 3 * H, LG = 2 * H * H;
  float* sL = sm;
  float* sl = sL + 3 * LG;
  float* sC = sl + H3;
  float* sH = sC + BR * H3;
  float* sZ = sH + BR * H;
  float* sR = sZ + BR * H;
  float* sRH = sR + BR * H;
  for (int i = threadIdx.x; i < 3 * LG; i += kT) sL[i] = L[i];
  for (int i = threadIdx.x; i < H3; i += kT) sl[i] = l[i];
  const float* Lz = sL; const float* Lr = sL + LG; const float* Lh = sL + 2 * LG;
  const int64_t ntiles = (V + BR - 1) / BR;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t r0 = tile * BR;
    __syncthreads();
    for (int i = threadIdx.x; i < BR * H3; i += kT) {
      int64_t r = r0 + i / H3;
      sC[i] = r < V ? C[r * H3 + i % H3] : 0.0f;
    }
    for (int i = threadIdx.x; i < BR * H; i += kT) {
      int64_t r = r0 + i / H;
      sH[i] = r < V ? Hp[r * H + i % H] : 0.0f;
    }
    __syncthreads();
    for (int o = threadIdx.x; o < BR * H; o += kT) {
      const int r = o / H, j = o % H;
      const float* cz = sC + r * H3; const float* cr = cz + H; const float* hv = sH + r * H;
      float az = sl[j], ar = sl[H + j];
      for (int i = 0; i < H; ++i) {
        az = fmaf(cz[i], Lz[i * H + j], az);
        az = fmaf(hv[i], Lz[(H + i) * H + j], az);
        ar = fmaf(cr[i], Lr[i * H + j], ar);
        ar = fmaf(hv[i], Lr[(H + i) * H + j], ar);
      }
      const float z = sigm(az), rr = sigm(ar);
      sZ[o] = z; sR[o] = rr; sRH[o] = rr * hv[j];
    }
    __syncthreads();
    for (int o = threadIdx.x; o < BR * H; o += kT) {
      const int r = o / H, j = o % H;
      if (r0 + r >= V) continue;
      const float* ch = sC + r * H3 + 2 * H; const float* rh = sRH + r * H;
      float ah = sl[2 * H + j];
      for (int i = 0; i < H; ++i) {
        ah = fmaf(ch[i], Lh[i * H + j], ah);
        ah = fmaf(rh[i], Lh[(H + i) * H + j], ah);
      }
      const float hh = tanhf(ah), z = sZ[o];
      Hn[(r0 + r) * H + j] = z * sH[o] + (1.0f - z) * hh;
    }
  }
}

// ---------------------------------------------------------------- GRU backward
// Recomputes Z, R, Ĥ from {C, H} (A8), applies the chain rule,
// writes dC' = n_dst ⊙ dC and dH_prev, and accumulates per-block partials of
// [dL (6H²) | dl (3H) | db (3H)] in a fixed row order.
template <int BR>
__global__ void __launch_bounds__(kT) k_gru_bwd(int32_t V, int32_t H, const float* __restrict__ C,
                                                const float* __restrict__ Hp, const float* __restrict__ G,
                                                const float* __restrict__ L, const float* __restrict__ l,
                                                const float* __restrict__ ndst, float* __restrict__ dCs,
                                                float* __restrict__ dHp, float* __restrict__ part) {
  extern __shared__ float sm[];
  const int H3 = 3 * H, LG = 2 * H * H, HH = H * H;
  const int NP = 6 * HH + 6 * H;     // partial layout: dL[3][2H][H], dl[3][H], db[3H]
  float* sL = sm;
  float* sl = sL + 3 * LG;
  float* sC = sl + H3;
  float* sH = sC + BR * H3;
  float* sG = sH + BR * H;
  float* sZ = sG + BR * H;
  float* sR = sZ + BR * H;
  float* sHh = sR + BR * H;
  float* sdaz = sHh + BR * H;
  float* sdar = sdaz + BR * H;
  float* sdah = sdar + BR * H;
  float* sdC = sdah + BR * H;        // [BR][3H] unscaled dC
  float* sAcc = sdC + BR * H3;       // [NP]
  for (int i = threadIdx.x; i < 3 * LG; i += kT) sL[i] = L[i];
  for (int i = threadIdx.x; i < H3; i += kT) sl[i] = l[i];
  for (int i = threadIdx.x; i < NP; i += kT) sAcc[i] = 0.0f;
  const float* Lz = sL; const float* Lr = sL + LG; const float* Lh = sL + 2 * LG;
  const int64_t ntiles = (V + BR - 1) / BR;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t r0 = tile * BR;
    __syncthreads();
    for (int i = threadIdx.x; i < BR * H3; i += kT) {
      int64_t r = r0 + i / H3;
      sC[i] = r < V ? C[r * H3 + i % H3] : 0.0f;
    }
    for (int i = threadIdx.x; i < BR * H; i += kT) {
      int64_t r = r0 + i / H;
      sH[i] = r < V ? Hp[r * H + i % H] : 0.0f;
      sG[i] = r < V ? G[r * H + i % H] : 0.0f;
    }
    __syncthreads();
    // gates (identical arithmetic to k_gru_fwd)
    for (int o = threadIdx.x; o < BR * H; o += kT) {
      const int r = o / H, j = o % H;
      const float* cz = sC + r * H3; const float* cr = cz + H; const float* hv = sH + r * H;
      float az = sl[j], ar = sl[H + j];
      for (int i = 0; i < H; ++i) {
        az = fmaf(cz[i], Lz[i * H + j], az);
        az = fmaf(hv[i], Lz[(H + i) * H + j], az);
        ar = fmaf(cr[i], Lr[i * H + j], ar);
        ar = fmaf(hv[i], Lr[(H + i) * H + j], ar);
      }
      sZ[o] = sigm(az); sR[o] = sigm(ar);
    }
    __syncthreads();
    for (int o = threadIdx.x; o < BR * H; o += kT) {
      const int r = o / H, j = o % H;
      const float* ch = sC + r * H3 + 2 * H; const float* hv = sH + r * H; const float* rr = sR + r * H;
      float ah = sl[2 * H + j];
      for (int i = 0; i < H; ++i) {
        ah = fmaf(ch[i], Lh[i * H + j], ah);
        ah = fmaf(rr[i] * hv[i], Lh[(H + i) * H + j], ah);
      }
      const float hh = tanhf(ah);
      sHh[o] = hh;
      const float g = sG[o], z = sZ[o];
      const float dZ = g * (hv[j] - hh), dHh = g * (1.0f - z);
      sdah[o] = dHh * (1.0f - hh * hh);
      sdaz[o] = dZ * z * (1.0f - z);
    }
    __syncthreads();
    // dC_h, dRH -> dR -> da_r ; dH accumulates in sG (reused as dH after G is consumed)
    for (int o = threadIdx.x; o < BR * H; o += kT) {
      const int r = o / H, i = o % H;
      const float* dah = sdah + r * H;
      float s1 = 0.0f, s2 = 0.0f;
      for (int j = 0; j < H; ++j) {
        s1 = fmaf(dah[j], Lh[i * H + j], s1);
        s2 = fmaf(dah[j], Lh[(H + i) * H + j], s2);
      }
      sdC[r * H3 + 2 * H + i] = s1;
      const float rr = sR[o], hv = sH[o];
      sdar[o] = s2 * hv * rr * (1.0f - rr);
      sHh[o] = s2 * rr;             // dH contribution through R⊙H (Ĥ no longer needed)
    }
    __syncthreads();
    for (int o = threadIdx.x; o < BR * H; o += kT) {
      const int r = o / H, i = o % H;
      const float* dar = sdar + r * H; const float* daz = sdaz + r * H;
      float sr1 = 0.0f, sr2 = 0.0f, sz1 = 0.0f, sz2 = 0.0f;
      for (int j = 0; j < H; ++j) {
        sr1 = fmaf(dar[j], Lr[i * H + j], sr1);
        sr2 = fmaf(dar[j], Lr[(H + i) * H + j], sr2);
        sz1 = fmaf(daz[j], Lz[i * H + j], sz1);
        sz2 = fmaf(daz[j], Lz[(H + i) * H + j], sz2);
      }
      sdC[r * H3 + H + i] = sr1;
      sdC[r * H3 + i] = sz1;
      const int64_t row = r0 + r;
      if (row < V) dHp[row * H + i] = sG[o] * sZ[o] + sHh[o] + (sr2 + sz2);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < BR * H3; i += kT) {
      int64_t r = r0 + i / H3;
      if (r < V) dCs[r * H3 + i % H3] = ndst[r] * sdC[i];
    }
    // parameter-gradient partials (each entry owned by one thread; rows in order)
    const int nrows = (int)(V - r0 < BR ? V - r0 : BR);
    for (int e = threadIdx.x; e < NP; e += kT) {
      float acc = sAcc[e];
      if (e < 6 * HH) {
        const int g = e / LG, rem = e % LG, i = rem / H, j = rem % H;
        const float* da = g == 0 ? sdaz : (g == 1 ? sdar : sdah);
        for (int r = 0; r < nrows; ++r) {
          float a;
          if (i < H) a = sC[r * H3 + g * H + i];
          else a = (g == 2) ? sR[r * H + (i - H)] * sH[r * H + (i - H)] : sH[r * H + (i - H)];
          acc = fmaf(a, da[r * H + j], acc);
        }
      } else if (e < 6 * HH + 3 * H) {
        const int g = (e - 6 * HH) / H, j = (e - 6 * HH) % H;
        const float* da = g == 0 ? sdaz : (g == 1 ? sdar : sdah);
        for (int r = 0; r < nrows; ++r) acc += da[r * H + j];
      } else {
        const int c = e - 6 * HH - 3 * H;
        for (int r = 0; r < nrows; ++r) acc += sdC[r * H3 + c];
      }
      sAcc[e] = acc;
    }
  }
  __syncthreads();
  for (int e = threadIdx.x; e < NP; e += kT) part[(int64_t)blockIdx.x * NP + e] = sAcc[e];
}

// ---------------------------------------------------------------- dW partials
// dW[f,c] += Σ_v X[v,f]·dP[v,c]; block-private accumulators, rows in order.
__global__ void __launch_bounds__(kT) k_dw(int32_t V, int32_t F, int32_t N, const float* __restrict__ X,
                                           const float* __restrict__ dP, float* __restrict__ part) {
  extern __shared__ float sm[];
  constexpr int BR = 32;
  float* sX = sm;              // [BR][F]
  float* sD = sX + BR * F;     // [BR][N]
  float* sAcc = sD + BR * N;   // [F][N]
  for (int i = threadIdx.x; i < F * N; i += kT) sAcc[i] = 0.0f;
  const int64_t ntiles = (V + BR - 1) / BR;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t r0 = tile * BR;
    __syncthreads();
    for (int i = threadIdx.x; i < BR * F; i += kT) {
      int64_t r = r0 + i / F;
      sX[i] = r < V ? X[r * F + i % F] : 0.0f;
    }
    for (int i = threadIdx.x; i < BR * N; i += kT) {
      int64_t r = r0 + i / N;
      sD[i] = r < V ? dP[r * N + i % N] : 0.0f;
    }
    __syncthreads();
    const int nrows = (int)(V - r0 < BR ? V - r0 : BR);
    for (int e = threadIdx.x; e < F * N; e += kT) {
      const int f = e / N, c = e % N;
      float acc = sAcc[e];
      for (int r = 0; r < nrows; ++r) acc = fmaf(sX[r * F + f], sD[r * N + c], acc);
      sAcc[e] = acc;
    }
  }
  __syncthreads();
  for (int e = threadIdx.x; e < F * N; e += kT) part[(int64_t)blockIdx.x * F * N + e] = sAcc[e];
}

// out[e] += Σ_b part[b][e], blocks of 16 summed first (fixed order).
__global__ void k_reduce_part(const float* __restrict__ part, int32_t nb, int32_t n, float* __restrict__ out0,
                              int32_t n0, float* __restrict__ out1, int32_t n1, float* __restrict__ out2) {
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < n; e += gridDim.x * blockDim.x) {
    float tot = 0.0f;
    for (int b0 = 0; b0 < nb; b0 += 16) {
      float blk = 0.0f;
      const int b1 = min(b0 + 16, nb);
      for (int b = b0; b < b1; ++b) blk += part[(int64_t)b * n + e];
      tot += blk;
    }
    if (e < n0) out0[e] += tot;
    else if (e < n0 + n1) out1[e - n0] += tot;
    else out2[e - n0 - n1] += tot;
  }
}

// ---------------------------------------------------------------- MSE head
// LPR = H/4 lanes per row (float4 each), 32/LPR rows per warp step, several
// rows in flight per warp.  Per-block partials [loss | dw_o (H) | db_o]
// (fp32 gradients, fp64 loss), reduced in a fixed order by k_mse_reduce.
template <int LPR>
__global__ void __launch_bounds__(kT) k_mse_head(int32_t V, int32_t Vn, int32_t H, const float* __restrict__ Hn,
                                                 const float* __restrict__ y, const float* __restrict__ w_o,
                                                 const float* __restrict__ b_o, float* __restrict__ dH, int accumulate,
                                                 int want_grad, double* __restrict__ lpart,
                                                 float* __restrict__ gpart) {
  constexpr int RPW = 32 / LPR;                 // rows per warp step
  __shared__ double sl[kT / 32];
  __shared__ float sg[kT / 32][129];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int rl = lane / LPR, ql = lane % LPR;   // row slot, float4 index within the row
  double lacc = 0.0;
  float4 gw = make_float4(0.f, 0.f, 0.f, 0.f);
  float gb = 0.f;
  const float b = b_o[0];
  const float invV = 1.0f / (float)Vn;               // mean over the whole graph's Vn rows
  const float4 wo = reinterpret_cast<const float4*>(w_o)[ql];
  const int64_t step = (int64_t)gridDim.x * (kT / 32) * RPW;
  // U row steps per iteration with all their loads issued first (memory-level
  // parallelism); the steps are then processed in order, so every accumulation
  // keeps the one-step-at-a-time order
  constexpr int U = 4;
  const float4 z4 = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int64_t vb = ((int64_t)blockIdx.x * (kT / 32) + w) * RPW; vb < V; vb += U * step) {
    float4 hu[U], du[U];
    float yu[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = vb + u * step + rl;
      const bool ok = v < V;
      hu[u] = ok ? reinterpret_cast<const float4*>(Hn + v * H)[ql] : z4;
      yu[u] = (ok && ql == 0) ? y[v] : 0.f;
      du[u] = (ok && want_grad && dH && accumulate) ? reinterpret_cast<const float4*>(dH + v * H)[ql] : z4;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
    const int64_t v0 = vb + u * step;
    if (v0 >= V) break;                            // warp-uniform
    const int64_t v = v0 + rl;
    const bool ok = v < V;
    const float4 h = hu[u];
    const float yv = yu[u];
    float4 r = make_float4(fmaxf(h.x, 0.f), fmaxf(h.y, 0.f), fmaxf(h.z, 0.f), fmaxf(h.w, 0.f));
    float s = r.x * wo.x + r.y * wo.y + r.z * wo.z + r.w * wo.w;
#pragma unroll
    for (int o = LPR / 2; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const float yy = __shfl_sync(0xffffffffu, yv, rl * LPR);
    const float e = (s + b) - yy;
    if (ok && ql == 0) lacc += (double)e * (double)e;
    if (want_grad && ok) {
      const float g = 2.0f * e * invV;
      if (dH) {
        float4 d = make_float4(h.x > 0.f ? g * wo.x : 0.f, h.y > 0.f ? g * wo.y : 0.f, h.z > 0.f ? g * wo.z : 0.f,
                               h.w > 0.f ? g * wo.w : 0.f);
        float4* dp = reinterpret_cast<float4*>(dH + v * H) + ql;
        if (accumulate) {
          const float4 o = du[u];
          d.x += o.x; d.y += o.y; d.z += o.z; d.w += o.w;
        }
        *dp = d;
      }
      gw.x = fmaf(g, r.x, gw.x); gw.y = fmaf(g, r.y, gw.y); gw.z = fmaf(g, r.z, gw.z); gw.w = fmaf(g, r.w, gw.w);
      if (ql == 0) gb += g;
    }
    }
  }
  // fixed-order reduction: over the RPW row slots of the warp, then over warps
#pragma unroll
  for (int o = LPR; o < 32; o <<= 1) {
    gw.x += __shfl_xor_sync(0xffffffffu, gw.x, o); gw.y += __shfl_xor_sync(0xffffffffu, gw.y, o);
    gw.z += __shfl_xor_sync(0xffffffffu, gw.z, o); gw.w += __shfl_xor_sync(0xffffffffu, gw.w, o);
    gb += __shfl_xor_sync(0xffffffffu, gb, o);
    lacc += __shfl_xor_sync(0xffffffffu, lacc, o);
  }
  if (lane == 0) { sl[w] = lacc; sg[w][128] = gb; }
  if (lane < LPR) { sg[w][4 * lane] = gw.x; sg[w][4 * lane + 1] = gw.y; sg[w][4 * lane + 2] = gw.z; sg[w][4 * lane + 3] = gw.w; }
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int i = 0; i < kT / 32; ++i) t += sl[i];
    lpart[blockIdx.x] = t;
  }
  for (int k = threadIdx.x; k < H + 1; k += kT) {
    float t = 0.0f;
    const int src = k < H ? k : 128;
    for (int i = 0; i < kT / 32; ++i) t += sg[i][src];
    gpart[(int64_t)blockIdx.x * (H + 1) + k] = t;
  }
}

// Fixed-order reduction of the per-block partials: block k < H sums column k
// of gpart (dw_o), block H the db_o column, block H+1 the loss partials; each
// thread sums a fixed strided subset, then a fixed shared-memory tree.
__global__ void __launch_bounds__(256) k_mse_reduce(int32_t nb, int32_t H, int32_t Vn, const double* __restrict__ lpart,
                                                    const float* __restrict__ gpart, float* __restrict__ loss,
                                                    float* __restrict__ dw_o, float* __restrict__ db_o) {
  __shared__ double sd[256];
  const int k = blockIdx.x;
  double t = 0.0;
  if (k <= H) {
    for (int b = threadIdx.x; b < nb; b += 256) t += (double)gpart[(int64_t)b * (H + 1) + k];
  } else {
    for (int b = threadIdx.x; b < nb; b += 256) t += lpart[b];
  }
  sd[threadIdx.x] = t;
  __syncthreads();
  for (int o = 128; o; o >>= 1) {
    if (threadIdx.x < o) sd[threadIdx.x] += sd[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    if (k < H) { if (dw_o) dw_o[k] += (float)sd[0]; }
    else if (k == H) { if (db_o) db_o[0] += (float)sd[0]; }
    else if (loss) *loss += (float)(sd[0] / (double)Vn);
  }
}

__global__ void k_sgd(float* __restrict__ p, float* __restrict__ g, int64_t n, float lr) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    p[i] -= lr * g[i];
    g[i] = 0.0f;
  }
}

// Sequence-batched layouts: X_all[v][t][:] = X_t[v][:], Y_all[v][t] = y_t[v], b_all[t][:] = b
constexpr int kSeqMax = 64;
struct SeqPtrs {
  const float* x[kSeqMax];
  const float* y[kSeqMax];
};
__global__ void k_seq_gather(const SeqPtrs ptrs, int S, int V, int F, const float* __restrict__ b, int H3,
                             float* __restrict__ X_all, float* __restrict__ Y_all, float* __restrict__ b_all) {
  const int64_t nx = (int64_t)V * S * F;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nx; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = e / ((int64_t)S * F);
    const int t = (int)((e / F) % S), f = (int)(e % F);
    X_all[e] = __ldg(ptrs.x[t] + v * F + f);
  }
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < (int64_t)V * S;
       e += (int64_t)gridDim.x * blockDim.x)
    Y_all[e] = __ldg(ptrs.y[e % S] + e / S);
  for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < S * H3; e += gridDim.x * blockDim.x) b_all[e] = b[e % H3];
}

// ---------------------------------------------------------------- original T-GCN (NEXT-2)
// The cell convolves [X, H] (orc_tgcn2_fwd): per timestep two
// linear-first graph convolutions Â([X,H]Wg) + bg (width 2H) and Â([X, r⊙H]Wc) + bc
// (width H) around the gates.  SIMT kernels: the dense parts are small (K = F+H,
// N <= 2H) and the aggregations run in the library's aggregation kernels.

// out[r, c] (+)= rs[r] · Σ_k A[r, k] · W(k, c) with A = [A1 (K1 cols) | A2 (K2 cols)]
// and W(k, c) = W[k·sk + c·sn] (a transposed slice is just other strides).  32-row
// tiles in shared memory; a thread computes 4 consecutive columns of one row.
__global__ void __launch_bounds__(kT) k_cat_mm(int32_t V, const float* __restrict__ A1, int32_t K1, int64_t ld1,
                                               const float* __restrict__ A2, int32_t K2, int64_t ld2,
                                               const float* __restrict__ W, int64_t sk, int64_t sn, int32_t N,
                                               const float* __restrict__ rs, float* __restrict__ out, int64_t ldo,
                                               int accumulate) {
  extern __shared__ float sm[];
  constexpr int BR = 32;
  const int K = K1 + K2, KP = K + 1;
  float* sW = sm;                 // [K][N]
  float* sA = sm + K * N;         // [BR][K+1]
  for (int i = threadIdx.x; i < K * N; i += kT) sW[i] = W[(int64_t)(i / N) * sk + (int64_t)(i % N) * sn];
  const int NG = N / 4;
  const int64_t ntiles = (V + BR - 1) / BR;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t r0 = tile * BR;
    __syncthreads();
    for (int i = threadIdx.x; i < BR * K; i += kT) {
      const int r = i / K, k = i % K;
      const int64_t row = r0 + r;
      float v = 0.0f;
      if (row < V) v = k < K1 ? A1[row * ld1 + k] : A2[row * ld2 + (k - K1)];
      sA[r * KP + k] = v;
    }
    __syncthreads();
    for (int o = threadIdx.x; o < BR * NG; o += kT) {
      const int r = o / NG, c = 4 * (o % NG);
      const int64_t row = r0 + r;
      if (row >= V) continue;
      float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
      const float* ar = sA + r * KP;
      for (int k = 0; k < K; ++k) {
        const float a = ar[k];
        const float4 w = *reinterpret_cast<const float4*>(sW + k * N + c);
        acc.x = fmaf(a, w.x, acc.x); acc.y = fmaf(a, w.y, acc.y);
        acc.z = fmaf(a, w.z, acc.z); acc.w = fmaf(a, w.w, acc.w);
      }
      const float sc = rs ? rs[row] : 1.0f;
      float* o4 = out + row * ldo + c;
      if (accumulate) {
        o4[0] += sc * acc.x; o4[1] += sc * acc.y; o4[2] += sc * acc.z; o4[3] += sc * acc.w;
      } else {
        o4[0] = sc * acc.x; o4[1] = sc * acc.y; o4[2] = sc * acc.z; o4[3] = sc * acc.w;
      }
    }
  }
}

// part[b][k][c] = Σ_{rows of block b} A[r, k] · B[r, c], A = [A1 | A2]; B [V, N] (ld N).
// Fixed row order per block; k_reduce_part adds the block partials in a fixed order.
__global__ void __launch_bounds__(kT) k_cat_atb(int32_t V, const float* __restrict__ A1, int32_t K1,
                                                const float* __restrict__ A2, int32_t K2,
                                                const float* __restrict__ B, int32_t N, float* __restrict__ part) {
  extern __shared__ float sm[];
  constexpr int BR = 32;
  const int K = K1 + K2;
  float* sA = sm;                 // [BR][K]
  float* sB = sA + BR * K;        // [BR][N]
  float* sAcc = sB + BR * N;      // [K][N]
  for (int i = threadIdx.x; i < K * N; i += kT) sAcc[i] = 0.0f;
  const int NG = N / 4;
  const int64_t ntiles = (V + BR - 1) / BR;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t r0 = tile * BR;
    __syncthreads();
    for (int i = threadIdx.x; i < BR * K; i += kT) {
      const int r = i / K, k = i % K;
      const int64_t row = r0 + r;
      sA[i] = row < V ? (k < K1 ? A1[row * K1 + k] : A2[row * K2 + (k - K1)]) : 0.0f;
    }
    for (int i = threadIdx.x; i < BR * N; i += kT) {
      const int64_t row = r0 + i / N;
      sB[i] = row < V ? B[row * N + i % N] : 0.0f;
    }
    __syncthreads();
    const int nrows = (int)(V - r0 < BR ? V - r0 : BR);
    for (int e = threadIdx.x; e < K * NG; e += kT) {
      const int k = e / NG, c = 4 * (e % NG);
      float4 acc = *reinterpret_cast<float4*>(sAcc + k * N + c);
      for (int r = 0; r < nrows; ++r) {
        const float a = sA[r * K + k];
        const float4 b = *reinterpret_cast<const float4*>(sB + r * N + c);
        acc.x = fmaf(a, b.x, acc.x); acc.y = fmaf(a, b.y, acc.y);
        acc.z = fmaf(a, b.z, acc.z); acc.w = fmaf(a, b.w, acc.w);
      }
      *reinterpret_cast<float4*>(sAcc + k * N + c) = acc;
    }
  }
  __syncthreads();
  for (int e = threadIdx.x; e < K * N; e += kT) part[(int64_t)blockIdx.x * K * N + e] = sAcc[e];
}

__device__ __forceinline__ float t2_sig(float a) { return 1.0f / (1.0f + expf(-a)); }

// The cell's element-wise parts, one float4 of a row per thread (Q = H/4 float4 per
// row; a thread's column group jq = index % Q is fixed under the grid stride, as
// 256 % Q == 0).  The backward kernels also form the bias-gradient column sums of
// what they produce (fixed order: the thread's rows in stride order, then the
// block's threads of a column group in index order; k_reduce_part adds the blocks).
__device__ __forceinline__ float4 ld4(const float* p) { return *reinterpret_cast<const float4*>(p); }
__device__ __forceinline__ void st4(float* p, float4 v) { *reinterpret_cast<float4*>(p) = v; }
__device__ __forceinline__ float4 sig4(float4 a) { return make_float4(t2_sig(a.x), t2_sig(a.y), t2_sig(a.z), t2_sig(a.w)); }
__device__ __forceinline__ float4 add4(float4 a, float4 b) { return make_float4(a.x + b.x, a.y + b.y, a.z + b.z, a.w + b.w); }

// r = σ(A[:, :H]), u = σ(A[:, H:]) -> RUC[:, 0:H), [H:2H); rH = r ⊙ Hp
template <int Q>
__global__ void __launch_bounds__(256) k_t2_gates(int32_t V, const float* __restrict__ A, const float* __restrict__ Hp,
                                                  float* __restrict__ RUC, float* __restrict__ rH) {
  constexpr int H = 4 * Q;
  const int64_t n = (int64_t)V * Q;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = i / Q;
    const int c = 4 * (int)(i % Q);
    const float4 r = sig4(ld4(A + v * 2 * H + c)), u = sig4(ld4(A + v * 2 * H + H + c)), h = ld4(Hp + v * H + c);
    st4(RUC + v * 3 * H + c, r);
    st4(RUC + v * 3 * H + H + c, u);
    st4(rH + v * H + c, make_float4(r.x * h.x, r.y * h.y, r.z * h.z, r.w * h.w));
  }
}

// c = tanh(A) -> RUC[:, 2H:3H);  H' = u ⊙ Hp + (1 − u) ⊙ c
template <int Q>
__global__ void __launch_bounds__(256) k_t2_cand(int32_t V, const float* __restrict__ A, const float* __restrict__ Hp,
                                                 float* __restrict__ RUC, float* __restrict__ Hn) {
  constexpr int H = 4 * Q;
  const int64_t n = (int64_t)V * Q;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = i / Q;
    const int c = 4 * (int)(i % Q);
    const float4 a = ld4(A + v * H + c), u = ld4(RUC + v * 3 * H + H + c), h = ld4(Hp + v * H + c);
    const float4 cc = make_float4(tanhf(a.x), tanhf(a.y), tanhf(a.z), tanhf(a.w));
    st4(RUC + v * 3 * H + 2 * H + c, cc);
    st4(Hn + v * H + c, make_float4(u.x * h.x + (1.0f - u.x) * cc.x, u.y * h.y + (1.0f - u.y) * cc.y,
                                    u.z * h.z + (1.0f - u.z) * cc.z, u.w * h.w + (1.0f - u.w) * cc.w));
  }
}

// block partial of NG float4 column groups per thread-column jq: part[b][g·H + 4jq ..]
template <int Q, int NG>
__device__ __forceinline__ void t2_block_colsum(const float4 (&acc)[NG], float* __restrict__ part) {
  constexpr int H = 4 * Q;
  __shared__ float4 red[NG][256];
#pragma unroll
  for (int g = 0; g < NG; ++g) red[g][threadIdx.x] = acc[g];
  __syncthreads();
  if (threadIdx.x < NG * Q) {
    const int g = threadIdx.x / Q, jq = threadIdx.x % Q;
    float4 t = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int sl = 0; sl < 256 / Q; ++sl) t = add4(t, red[g][sl * Q + jq]);
    st4(part + (int64_t)blockIdx.x * NG * H + g * H + 4 * jq, t);
  }
}

// du = G ⊙ (Hp − c); dAc = G ⊙ (1 − u) ⊙ (1 − c²); dHp = G ⊙ u; rH = r ⊙ Hp; part: colsum dAc
template <int Q>
__global__ void __launch_bounds__(256) k_t2_cand_bwd(int32_t V, const float* __restrict__ G,
                                                     const float* __restrict__ Hp, const float* __restrict__ RUC,
                                                     float* __restrict__ dAc, float* __restrict__ du,
                                                     float* __restrict__ dHp, float* __restrict__ rH,
                                                     float* __restrict__ part) {
  constexpr int H = 4 * Q;
  const int64_t n = (int64_t)V * Q;
  float4 acc[1] = {make_float4(0.f, 0.f, 0.f, 0.f)};
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = i / Q;
    const int c = 4 * (int)(i % Q);
    const float* ruc = RUC + v * 3 * H + c;
    const float4 r = ld4(ruc), u = ld4(ruc + H), cc = ld4(ruc + 2 * H);
    const float4 g = ld4(G + v * H + c), h = ld4(Hp + v * H + c);
    st4(du + v * H + c, make_float4(g.x * (h.x - cc.x), g.y * (h.y - cc.y), g.z * (h.z - cc.z), g.w * (h.w - cc.w)));
    const float4 da = make_float4(g.x * (1.0f - u.x) * (1.0f - cc.x * cc.x), g.y * (1.0f - u.y) * (1.0f - cc.y * cc.y),
                                  g.z * (1.0f - u.z) * (1.0f - cc.z * cc.z), g.w * (1.0f - u.w) * (1.0f - cc.w * cc.w));
    st4(dAc + v * H + c, da);
    acc[0] = add4(acc[0], da);
    st4(dHp + v * H + c, make_float4(g.x * u.x, g.y * u.y, g.z * u.z, g.w * u.w));
    st4(rH + v * H + c, make_float4(r.x * h.x, r.y * h.y, r.z * h.z, r.w * h.w));
  }
  t2_block_colsum<Q, 1>(acc, part);
}

// dr = d(rH) ⊙ Hp;  dHp += d(rH) ⊙ r;  dAg = [dr ⊙ r(1−r) | du ⊙ u(1−u)]; part: colsum dAg
template <int Q>
__global__ void __launch_bounds__(256) k_t2_gate_bwd(int32_t V, const float* __restrict__ drH,
                                                     const float* __restrict__ Hp, const float* __restrict__ RUC,
                                                     const float* __restrict__ du, float* __restrict__ dHp,
                                                     float* __restrict__ dAg, float* __restrict__ part) {
  constexpr int H = 4 * Q;
  const int64_t n = (int64_t)V * Q;
  float4 acc[2] = {make_float4(0.f, 0.f, 0.f, 0.f), make_float4(0.f, 0.f, 0.f, 0.f)};
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = i / Q;
    const int c = 4 * (int)(i % Q);
    const float4 r = ld4(RUC + v * 3 * H + c), u = ld4(RUC + v * 3 * H + H + c);
    const float4 d = ld4(drH + v * H + c), h = ld4(Hp + v * H + c), w = ld4(du + v * H + c);
    float4 o = ld4(dHp + v * H + c);
    o = make_float4(o.x + d.x * r.x, o.y + d.y * r.y, o.z + d.z * r.z, o.w + d.w * r.w);
    st4(dHp + v * H + c, o);
    const float4 gr = make_float4(d.x * h.x * r.x * (1.0f - r.x), d.y * h.y * r.y * (1.0f - r.y),
                                  d.z * h.z * r.z * (1.0f - r.z), d.w * h.w * r.w * (1.0f - r.w));
    const float4 gu = make_float4(w.x * u.x * (1.0f - u.x), w.y * u.y * (1.0f - u.y), w.z * u.z * (1.0f - u.z),
                                  w.w * u.w * (1.0f - u.w));
    st4(dAg + v * 2 * H + c, gr);
    st4(dAg + v * 2 * H + H + c, gu);
    acc[0] = add4(acc[0], gr);
    acc[1] = add4(acc[1], gu);
  }
  t2_block_colsum<Q, 2>(acc, part);
}

int grid_blocks(const void* fn, size_t smem, int64_t tiles) {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kT, smem) != cudaSuccess || per_sm < 1) {
    cudaGetLastError();
    per_sm = 1;
  }
  int64_t b = (int64_t)per_sm * num_sms();
  if (tiles < b) b = tiles;
  return (int)(b < 1 ? 1 : b);
}

template <class K>
stg_status set_smem(K fn, size_t smem) {
  if (smem > 48 * 1024) STG_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  return STG_OK;
}

}  // namespace

// Scratch used by the TGCN kernels (grow-only).
struct TgcnWs {
  DArray<float> P, dC, dP, part_gru, part_dw, gpart, da, RH, part_tc, dl_tmp, part_dl, dl_tmp2;
  DArray<double> lpart;
  // sequence-batched path: X_all, Y_all, b_all, then [V][S][·] activations and the head partials
  DArray<float> sX, sY, sb, sP, sC, sHp, sdC, sdP, sda, sRH, sgpart;
  DArray<double> slpart;
  // original T-GCN (NEXT-2) scratch
  DArray<float> t2z, t2a, t2b, t2c, t2d, t2part;
  // per-step driver with the surrogate head fused into the GRU kernels: per-row
  // {g, ReLU mask} of every timestamp of the sequence, per-CTA head partials
  DArray<float2> hg;
  DArray<float> hd_gpart;
  DArray<double> hd_lpart;
};

}  // namespace stg

using namespace stg;

struct StackEntry {
  const float* Hp;
  float* C;
  int32_t V, H;
  size_t bytes;
  float* A = nullptr;     // aggregate-first: ÂX of the step (NULL: linear-first)
};

struct stg_state_stack {
  DArray<unsigned char> arena;
  size_t cap = 0, top = 0;
  std::vector<StackEntry> entries;
  TgcnWs ws;
};

static TgcnWs& global_ws() {
  static TgcnWs ws;
  return ws;
}

static stg_status check_params(const stg_tgcn_params* p) {
  if (!p || !p->W || !p->b || !p->L || !p->l) return fail(STG_ERR_INVALID_ARG, "tgcn: NULL parameter pointer");
  if (p->F < 1 || p->H < 1) return fail(STG_ERR_INVALID_ARG, "tgcn: F=%d H=%d must be >= 1", p->F, p->H);
  if (p->H > 64) return fail(STG_ERR_INVALID_ARG, "tgcn: H=%d > 64 is not supported", p->H);
  if ((size_t)p->F * 3 * p->H * 4 + 32 * p->F * 4 > 200 * 1024)
    return fail(STG_ERR_INVALID_ARG, "tgcn: F=%d too large for the resident-weight kernel", p->F);
  return STG_OK;
}

static size_t gru_fwd_smem(int H, int BR) { return sizeof(float) * (6 * H * H + 3 * H + BR * 3 * H + 4 * BR * H); }
static size_t gru_bwd_smem(int H, int BR) {
  return sizeof(float) * (6 * H * H + 3 * H + BR * 3 * H + 8 * BR * H + BR * 3 * H + 6 * H * H + 6 * H);
}

// Convolution order (reading C14 / SURVEY §8(f) NEXT-1): 0 = linear-first
// C = Â(XW) + b (the default: P' = n_src ⊙ XW is aggregated forward, dP = Âᵀ dC'
// backward over the out-CSR); 1 = aggregate-first C = (ÂX)W + b (X is aggregated
// at width F, dW = (ÂX)ᵀ dC, no backward aggregation).  Same model and gradients.
std::atomic<int> g_conv_order{0};
bool agg_first() { return g_conv_order.load(std::memory_order_relaxed) != 0; }

static size_t stack_bytes(int32_t V, int32_t H, int32_t F = 0) {
  const size_t c = (sizeof(float) * (size_t)V * 3 * H + 255) & ~size_t(255);
  return c + (F > 0 ? (sizeof(float) * (size_t)V * F + 255) & ~size_t(255) : 0);
}
// the aggregate-first state: A = ÂX after C in the same stack slot
static float* stack_A(float* C, int32_t V, int32_t H) {
  return reinterpret_cast<float*>(reinterpret_cast<unsigned char*>(C) +
                                  ((sizeof(float) * (size_t)V * 3 * H + 255) & ~size_t(255)));
}
static stg_status check_agg_first(const stg_tgcn_params* p) {
  if (!tc_supported(p->F, p->H) || p->F > 64)
    return fail(STG_ERR_INVALID_ARG, "aggregate-first order needs the tensor-core path (H in {16,32}, F <= 64, "
                "F %% 4 == 0); F=%d H=%d", p->F, p->H);
  return STG_OK;
}

// ---- the TGCN step in stream-explicit pieces (stg_tgcn_step runs them on one
// stream; stg_tgcn_train_sequence pipelines them over several, see there).
// Sharded views (resident mode): P' for all Vall source rows
// (X is resident on every rank), C / GRU / H for the V = R local rows.

// P'[i] = n[i]·X[i]·W over n_rows rows (n = NULL: unscaled)
static stg_status project_rows(int32_t n_rows, const stg_tgcn_params* p, const float* X, const float* n, float* P,
                               cudaStream_t s) {
  const int32_t F = p->F, H = p->H, H3 = 3 * H;
  ProfScope prof(PH_XW, s);
  if (n_rows == 0) return STG_OK;
  if (tc_supported(F, H)) return tc_xw(n_rows, F, H, X, p->W, n, P, s);
  const size_t smem = sizeof(float) * (size_t)(F * H3 + 32 * F);
  STG_TRY(set_smem(k_xw, smem));
  const int nb = grid_blocks((const void*)k_xw, smem, (n_rows + 31) / 32);
  k_xw<<<nb, kT, smem, s>>>(n_rows, F, H3, X, p->W, n, P);
  count_launch();
  return check_launch("tgcn project");
}

// P' = diag(n_src)·X·W (all Vall rows) and C = diag(n_dst)·A·P' + b (local rows);
// aggregate-first (A != NULL): A = ÂX (local rows, width F), C = A·W + b
static stg_status fwd_conv(const stg_csr_view* g, const stg_tgcn_params* p, const float* X, float* P, float* C,
                           cudaStream_t s, float* A = nullptr) {
  const int32_t Vall = g->num_nodes, H3 = 3 * p->H;
  if (A) {
    const int32_t V = g->row_end - g->row_begin, F = p->F;
    const float* ndst_loc = g->norm_dst ? g->norm_dst + g->row_begin : nullptr;
    STG_TRY(aggregate_launch(g, 0, F, X, F, A, F, ndst_loc, g->norm_src, nullptr, s));
    ProfScope prof(PH_XW, s);
    if (V == 0) return STG_OK;
    return tc_xw(V, F, p->H, A, p->W, nullptr, C, s, 1, p->b);
  }
  STG_TRY(project_rows(Vall, p, X, g->norm_src, P, s));
  const float* ndst_loc = g->norm_dst ? g->norm_dst + g->row_begin : nullptr;
  return aggregate_launch(g, 0, H3, P, H3, C, H3, ndst_loc, nullptr, p->b, s);
}

// GRU over V local rows: H_next from C and H_prev (tensor-core path: with the
// surrogate head fused if `head` is given)
static stg_status fwd_gru(int32_t V, const stg_tgcn_params* p, const float* C, const float* H_prev, float* H_next,
                          cudaStream_t s, const HeadArgs* head = nullptr) {
  const int32_t H = p->H;
  ProfScope prof_gru(PH_GRU_FWD, s);
  if (V == 0) return STG_OK;
  if (tc_supported(p->F, H)) {
    STG_TRY(tc_gru_fwd(V, H, C, H_prev, p->L, p->l, H_next, s, head));
  } else if (H <= 32) {
    const size_t smem = gru_fwd_smem(H, 32);
    STG_TRY(set_smem(k_gru_fwd<32>, smem));
    const int nb = grid_blocks((const void*)k_gru_fwd<32>, smem, (V + 31) / 32);
    k_gru_fwd<32><<<nb, kT, smem, s>>>(V, H, C, H_prev, p->L, p->l, H_next);
    count_launch();
  } else {
    const size_t smem = gru_fwd_smem(H, 16);
    STG_TRY(set_smem(k_gru_fwd<16>, smem));
    const int nb = grid_blocks((const void*)k_gru_fwd<16>, smem, (V + 15) / 16);
    k_gru_fwd<16><<<nb, kT, smem, s>>>(V, H, C, H_prev, p->L, p->l, H_next);
    count_launch();
  }
  return check_launch("tgcn fwd_gru");
}

// Backward buffers of one step (buffer set k of ws): dC' [V,3H], dP [Vall,3H],
// and on the tensor-core path da [V,3H], RH [V,H]
struct BwdBufs {
  float *dC[2], *dP[2], *da[2], *RH[2];
};

static stg_status bwd_alloc(TgcnWs& ws, const stg_csr_view* g, const stg_tgcn_params* p, int nsets, BwdBufs* b) {
  const int32_t Vall = g->num_nodes, V = g->row_end - g->row_begin, H = p->H, H3 = 3 * H;
  const size_t nC = ((size_t)V * H3 + 64) & ~size_t(63), nP = ((size_t)Vall * H3 + 64) & ~size_t(63);
  const size_t nR = ((size_t)V * H + 64) & ~size_t(63);
  STG_TRY(ws.dC.alloc(nC * nsets));
  STG_TRY(ws.dP.alloc(nP * nsets));
  const bool tc = tc_supported(p->F, H);
  if (tc) {
    STG_TRY(ws.da.alloc(nC * nsets));
    STG_TRY(ws.RH.alloc(nR * nsets));
    STG_TRY(ws.part_tc.alloc((size_t)tc_atb_max_blocks() * 2 * 128 * 128));
    STG_TRY(ws.dl_tmp.alloc(2 * 128 * 128));
    STG_TRY(ws.part_dl.alloc((size_t)tc_atb_max_blocks() * 2 * 128 * 128));   // dL scratch (own stream order)
    STG_TRY(ws.dl_tmp2.alloc(2 * 128 * 128));
  }
  for (int k = 0; k < 2; ++k) {
    const int kk = k < nsets ? k : 0;
    b->dC[k] = ws.dC.p + kk * nC;
    b->dP[k] = ws.dP.p + kk * nP;
    b->da[k] = tc ? ws.da.p + kk * nC : nullptr;
    b->RH[k] = tc ? ws.RH.p + kk * nR : nullptr;
  }
  return STG_OK;
}

// GRU backward over the V local rows into buffer set 0 of `bb` (dC', da, RH)
// and dH_prev.  SIMT path: also the dL, dl, db partials (fused in its kernel).
static stg_status bwd_gru(const stg_csr_view* g, const stg_tgcn_params* p, const float* C, const float* Hp,
                          const float* dH_next, float* dH_prev, stg_tgcn_grads* grads, TgcnWs& ws,
                          const BwdBufs& bb, cudaStream_t s, const float2* hg = nullptr, const float* w_o = nullptr) {
  const int32_t V = g->row_end - g->row_begin, H = p->H;
  const float* ndst_loc = g->norm_dst ? g->norm_dst + g->row_begin : nullptr;
  ProfScope prof(PH_GRU_BWD, s);
  if (V == 0) return STG_OK;
  if (tc_supported(p->F, H))
    return tc_gru_bwd(V, H, C, Hp, dH_next, p->L, p->l, ndst_loc, bb.dC[0], dH_prev, bb.da[0], bb.RH[0], s, hg,
                      w_o);
  const int BR = H <= 32 ? 16 : 4;
  const size_t smem = gru_bwd_smem(H, BR);
  const int NP = 6 * H * H + 6 * H;
  int nbg;
  if (BR == 16) {
    STG_TRY(set_smem(k_gru_bwd<16>, smem));
    nbg = grid_blocks((const void*)k_gru_bwd<16>, smem, (V + 15) / 16);
  } else {
    STG_TRY(set_smem(k_gru_bwd<4>, smem));
    nbg = grid_blocks((const void*)k_gru_bwd<4>, smem, (V + 3) / 4);
  }
  STG_TRY(ws.part_gru.alloc((size_t)nbg * NP));
  if (BR == 16)
    k_gru_bwd<16><<<nbg, kT, smem, s>>>(V, H, C, Hp, dH_next, p->L, p->l, ndst_loc, bb.dC[0], dH_prev,
                                        ws.part_gru.p);
  else
    k_gru_bwd<4><<<nbg, kT, smem, s>>>(V, H, C, Hp, dH_next, p->L, p->l, ndst_loc, bb.dC[0], dH_prev,
                                       ws.part_gru.p);
  count_launch();
  k_reduce_part<<<(NP + 255) / 256, 256, 0, s>>>(ws.part_gru.p, nbg, NP, grads->L, 6 * H * H, grads->l, 3 * H,
                                                 grads->b);
  count_launch();
  return check_launch("tgcn bwd_gru");
}

// The parameter-gradient reductions of one step from buffer set 0 of `bb`:
// dL, dl, db = Σ_rows [C|H]ᵀda, [RH|1]ᵀda (tensor-core path), dP = diag(n_src)·Aᵀ·dC'
// over the out-CSR, dW += Xᵀ·dP.
// dL, dl, db = Σ_rows [C|H]ᵀda, [RH|1]ᵀda (tensor-core path; the SIMT GRU kernel fuses them)
static stg_status bwd_dl(const stg_csr_view* g, const stg_tgcn_params* p, const float* C, const float* Hp,
                         stg_tgcn_grads* grads, TgcnWs& ws, const BwdBufs& bb, cudaStream_t s) {
  const int32_t V = g->row_end - g->row_begin, H = p->H;
  if (!tc_supported(p->F, H) || V == 0) return STG_OK;
  ProfScope prof(PH_DL, s);
  return tc_dl(V, H, C, Hp, bb.RH[0], bb.da[0], ws.part_dl.p, ws.dl_tmp2.p, grads->L, grads->l, grads->b, p->L, s);
}

static stg_status bwd_grads(const stg_csr_view* g, const stg_tgcn_params* p, const float* X, const float* C,
                            const float* Hp, stg_tgcn_grads* grads, TgcnWs& ws, const BwdBufs& bb, cudaStream_t s,
                            bool with_dl = true, const float* A = nullptr) {
  const int32_t Vall = g->num_nodes, V = g->row_end - g->row_begin, F = p->F, H = p->H, H3 = 3 * H;
  const bool tc = tc_supported(F, H);
  if (with_dl) STG_TRY(bwd_dl(g, p, C, Hp, grads, ws, bb, s));
  if (A) {                                   // aggregate-first: dW += (ÂX)ᵀ dC over the local rows
    ProfScope prof(PH_DW, s);
    if (V == 0) return STG_OK;
    return tc_dw(V, F, H, A, bb.dC[0], ws.part_tc.p, ws.dl_tmp.p, grads->W, s);
  }
  STG_TRY(aggregate_launch(g, 1, H3, bb.dC[0], H3, bb.dP[0], H3, g->norm_src, nullptr, nullptr, s));
  ProfScope prof(PH_DW, s);
  if (tc) return tc_dw(Vall, F, H, X, bb.dP[0], ws.part_tc.p, ws.dl_tmp.p, grads->W, s);
  const size_t sm2 = sizeof(float) * (size_t)(32 * F + 32 * H3 + F * H3);
  STG_TRY(set_smem(k_dw, sm2));
  const int nb = grid_blocks((const void*)k_dw, sm2, (Vall + 31) / 32);
  STG_TRY(ws.part_dw.alloc((size_t)nb * F * H3));
  k_dw<<<nb, kT, sm2, s>>>(Vall, F, H3, X, bb.dP[0], ws.part_dw.p);
  k_reduce_part<<<(F * H3 + 255) / 256, 256, 0, s>>>(ws.part_dw.p, nb, F * H3, grads->W, F * H3, nullptr, 0,
                                                     nullptr);
  count_launch(2);
  return check_launch("tgcn bwd_grads");
}

extern "C" {

stg_status stg_state_stack_create(int64_t capacity_bytes, stg_state_stack** out) {
  if (!out || capacity_bytes < 0) return fail(STG_ERR_INVALID_ARG, "stg_state_stack_create: bad arguments");
  auto* s = new stg_state_stack();
  s->cap = (size_t)capacity_bytes;
  if (s->cap) {
    stg_status st = s->arena.alloc(s->cap);
    if (st != STG_OK) { delete s; return st; }
  }
  *out = s;
  return STG_OK;
}

int32_t stg_state_stack_depth(const stg_state_stack* s) { return s ? (int32_t)s->entries.size() : -1; }

void stg_state_stack_destroy(stg_state_stack* s) {
  if (s) cudaDeviceSynchronize();
  delete s;
}

stg_status stg_tgcn_step(const stg_csr_view* g, const stg_tgcn_params* p, const float* X, const float* H_prev,
                         float* H_next, stg_state_stack* stack, stg_stream_t stream) {
  STG_TRY(check_params(p));
  if (!g || !X || !H_prev || !H_next) return fail(STG_ERR_INVALID_ARG, "stg_tgcn_step: NULL argument");
  cudaStream_t s = (cudaStream_t)stream;
  const int32_t Vall = g->num_nodes, V = g->row_end - g->row_begin, H = p->H, H3 = 3 * H;
  TgcnWs& ws = stack ? stack->ws : global_ws();
  const bool af = agg_first();
  if (af) STG_TRY(check_agg_first(p));
  if (!af) STG_TRY(ws.P.alloc((size_t)Vall * H3));
  float* C = nullptr;
  const size_t need = stack_bytes(V, H, af ? p->F : 0);
  if (stack) {
    if (stack->top + need > stack->cap)
      return fail(STG_ERR_NO_MEMORY, "stg_tgcn_step: state stack full (%zu + %zu > %zu bytes)", stack->top, need,
                  stack->cap);
    C = reinterpret_cast<float*>(stack->arena.p + stack->top);
  } else {
    STG_TRY(ws.dC.alloc(need / sizeof(float) + 4));
    C = ws.dC.p;
  }
  float* A = af ? stack_A(C, V, H) : nullptr;
  STG_TRY(fwd_conv(g, p, X, ws.P.p, C, s, A));
  STG_TRY(fwd_gru(V, p, C, H_prev, H_next, s));
  if (stack) {
    stack->entries.push_back(StackEntry{H_prev, C, V, H, need, A});
    stack->top += need;
  }
  return STG_OK;
}

stg_status stg_tgcn_step_backward(const stg_csr_view* g, const stg_tgcn_params* p, const float* X,
                                  const float* dH_next, float* dH_prev, stg_tgcn_grads* grads,
                                  stg_state_stack* stack, stg_stream_t stream) {
  STG_TRY(check_params(p));
  if (!g || !X || !dH_next || !dH_prev || !grads || !stack)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_step_backward: NULL argument");
  if (!grads->W || !grads->b || !grads->L || !grads->l)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_step_backward: NULL gradient pointer");
  if (stack->entries.empty()) return fail(STG_ERR_STATE, "stg_tgcn_step_backward: state stack is empty");
  const StackEntry e = stack->entries.back();
  const int32_t V = g->row_end - g->row_begin, H = p->H;
  if (e.V != V || e.H != H) return fail(STG_ERR_STATE, "stg_tgcn_step_backward: stack top does not match (V,H)");
  cudaStream_t s = (cudaStream_t)stream;
  BwdBufs bb;
  STG_TRY(bwd_alloc(stack->ws, g, p, 1, &bb));
  if (e.A) {                              // aggregate-first: dC unscaled, no backward aggregation
    stg_csr_view gv = *g;
    gv.norm_dst = nullptr;
    STG_TRY(bwd_gru(&gv, p, e.C, e.Hp, dH_next, dH_prev, grads, stack->ws, bb, s));
    STG_TRY(bwd_grads(g, p, X, e.C, e.Hp, grads, stack->ws, bb, s, true, e.A));
  } else {
    STG_TRY(bwd_gru(g, p, e.C, e.Hp, dH_next, dH_prev, grads, stack->ws, bb, s));
    STG_TRY(bwd_grads(g, p, X, e.C, e.Hp, grads, stack->ws, bb, s));
  }
  stack->entries.pop_back();
  stack->top -= e.bytes;
  return STG_OK;
}

// ---- sharded mode over peer memory (include/stg.h): P' of the local rows only,
// the aggregation gathers P' rows from their owners, the backward leaves
// partial dP rows for every source that stg_reduce_scatter_rows sums per owner.
stg_status stg_tgcn_project(const stg_csr_view* g, const stg_tgcn_params* p, const float* X_loc, float* P_loc,
                            stg_stream_t stream) {
  STG_TRY(check_params(p));
  if (!g || !X_loc || !P_loc) return fail(STG_ERR_INVALID_ARG, "stg_tgcn_project: NULL argument");
  const int32_t R = g->row_end - g->row_begin;
  return project_rows(R, p, X_loc, g->norm_src ? g->norm_src + g->row_begin : nullptr, P_loc, (cudaStream_t)stream);
}

stg_status stg_tgcn_step_peer(const stg_csr_view* g, const stg_tgcn_params* p, const stg_peer_rows* P,
                              const float* H_prev, float* H_next, stg_state_stack* stack, stg_stream_t stream) {
  STG_TRY(check_params(p));
  if (!g || !P || !H_prev || !H_next) return fail(STG_ERR_INVALID_ARG, "stg_tgcn_step_peer: NULL argument");
  cudaStream_t s = (cudaStream_t)stream;
  const int32_t V = g->row_end - g->row_begin, H = p->H, H3 = 3 * H;
  TgcnWs& ws = stack ? stack->ws : global_ws();
  float* C = nullptr;
  const size_t need = stack_bytes(V, H);
  if (stack) {
    if (stack->top + need > stack->cap)
      return fail(STG_ERR_NO_MEMORY, "stg_tgcn_step_peer: state stack full (%zu + %zu > %zu bytes)", stack->top,
                  need, stack->cap);
    C = reinterpret_cast<float*>(stack->arena.p + stack->top);
  } else {
    STG_TRY(ws.dC.alloc((size_t)V * H3 + 4));
    C = ws.dC.p;
  }
  const float* ndst_loc = g->norm_dst ? g->norm_dst + g->row_begin : nullptr;
  STG_TRY(aggregate_launch(g, 0, H3, nullptr, 0, C, H3, ndst_loc, nullptr, p->b, s, P));
  STG_TRY(fwd_gru(V, p, C, H_prev, H_next, s));
  if (stack) {
    stack->entries.push_back(StackEntry{H_prev, C, V, H, need});
    stack->top += need;
  }
  return STG_OK;
}

stg_status stg_tgcn_step_backward_peer(const stg_csr_view* g, const stg_tgcn_params* p, const float* dH_next,
                                       float* dH_prev, stg_tgcn_grads* grads, float* dP_part, stg_state_stack* stack,
                                       stg_stream_t stream) {
  STG_TRY(check_params(p));
  if (!g || !dH_next || !dH_prev || !grads || !stack || !dP_part)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_step_backward_peer: NULL argument");
  if (!grads->W || !grads->b || !grads->L || !grads->l)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_step_backward_peer: NULL gradient pointer");
  if (stack->entries.empty()) return fail(STG_ERR_STATE, "stg_tgcn_step_backward_peer: state stack is empty");
  const StackEntry e = stack->entries.back();
  const int32_t V = g->row_end - g->row_begin, H = p->H, H3 = 3 * H;
  if (e.V != V || e.H != H) return fail(STG_ERR_STATE, "stg_tgcn_step_backward_peer: stack top does not match (V,H)");
  cudaStream_t s = (cudaStream_t)stream;
  BwdBufs bb;
  STG_TRY(bwd_alloc(stack->ws, g, p, 1, &bb));
  STG_TRY(bwd_gru(g, p, e.C, e.Hp, dH_next, dH_prev, grads, stack->ws, bb, s));
  STG_TRY(bwd_dl(g, p, e.C, e.Hp, grads, stack->ws, bb, s));
  STG_TRY(aggregate_launch(g, 1, H3, bb.dC[0], H3, dP_part, H3, g->norm_src, nullptr, nullptr, s));
  stack->entries.pop_back();
  stack->top -= e.bytes;
  return STG_OK;
}

stg_status stg_tgcn_dw(const stg_tgcn_params* p, int32_t R, const float* X_loc, const float* dP_loc,
                       stg_tgcn_grads* grads, stg_state_stack* stack, stg_stream_t stream) {
  STG_TRY(check_params(p));
  if (R < 0 || (R > 0 && (!X_loc || !dP_loc)) || !grads || !grads->W || !stack)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_dw: bad arguments");
  if (R == 0) return STG_OK;
  cudaStream_t s = (cudaStream_t)stream;
  const int32_t F = p->F, H = p->H, H3 = 3 * H;
  TgcnWs& ws = stack->ws;
  ProfScope prof(PH_DW, s);
  if (tc_supported(F, H)) {
    STG_TRY(ws.part_tc.alloc((size_t)tc_atb_max_blocks() * 2 * 128 * 128));
    STG_TRY(ws.dl_tmp.alloc(2 * 128 * 128));
    return tc_dw(R, F, H, X_loc, dP_loc, ws.part_tc.p, ws.dl_tmp.p, grads->W, s);
  }
  const size_t sm2 = sizeof(float) * (size_t)(32 * F + 32 * H3 + F * H3);
  STG_TRY(set_smem(k_dw, sm2));
  const int nb = grid_blocks((const void*)k_dw, sm2, (R + 31) / 32);
  STG_TRY(ws.part_dw.alloc((size_t)nb * F * H3));
  k_dw<<<nb, kT, sm2, s>>>(R, F, H3, X_loc, dP_loc, ws.part_dw.p);
  k_reduce_part<<<(F * H3 + 255) / 256, 256, 0, s>>>(ws.part_dw.p, nb, F * H3, grads->W, F * H3, nullptr, 0,
                                                     nullptr);
  count_launch(2);
  return check_launch("stg_tgcn_dw");
}

// ---- original T-GCN (NEXT-2) host side
static stg_status t2_mm(int32_t V, const float* A1, int32_t K1, int64_t ld1, const float* A2, int32_t K2, int64_t ld2,
                        const float* W, int64_t sk, int64_t sn, int32_t N, const float* rs, float* out, int64_t ldo,
                        bool accumulate, cudaStream_t s) {
  if (V == 0) return STG_OK;
  const int K = K1 + K2;
  if (tc_cat_supported(K1, K2, N) && ld1 % 4 == 0 && (K2 == 0 || ld2 % 4 == 0) && ldo % 4 == 0)   // tensor cores
    return tc_catmm(V, A1, K1, ld1, A2, K2, ld2, W, sk, sn, N, rs, out, ldo, accumulate, s);
  const size_t smem = sizeof(float) * ((size_t)K * N + 32 * (size_t)(K + 1));
  STG_TRY(set_smem(k_cat_mm, smem));
  const int nb = grid_blocks((const void*)k_cat_mm, smem, (V + 31) / 32);
  k_cat_mm<<<nb, kT, smem, s>>>(V, A1, K1, ld1, A2, K2, ld2, W, sk, sn, N, rs, out, ldo, accumulate ? 1 : 0);
  count_launch();
  return check_launch("tgcn2 mm");
}

// grad[K][N] += [A1 | A2]ᵀ B   (fixed-order partials)
static stg_status t2_atb(int32_t V, const float* A1, int32_t K1, const float* A2, int32_t K2, const float* B,
                         int32_t N, float* grad, TgcnWs& ws, cudaStream_t s) {
  if (V == 0) return STG_OK;
  const int K = K1 + K2;
  if (tc_cat_supported(K1, K2, N)) {                  // tensor cores (Σ AᵀB with TMA MN-major operands)
    STG_TRY(ws.part_tc.alloc((size_t)tc_atb_max_blocks() * 2 * 128 * 128));
    STG_TRY(ws.dl_tmp.alloc(2 * 128 * 128));
    return tc_atb_cat(V, A1, K1, A2, K2, B, N, ws.part_tc.p, ws.dl_tmp.p, grad, s);
  }
  const size_t smem = sizeof(float) * (32 * (size_t)K + 32 * (size_t)N + (size_t)K * N);
  STG_TRY(set_smem(k_cat_atb, smem));
  const int nb = grid_blocks((const void*)k_cat_atb, smem, (V + 31) / 32);
  STG_TRY(ws.t2part.alloc((size_t)nb * K * N));
  k_cat_atb<<<nb, kT, smem, s>>>(V, A1, K1, A2, K2, B, N, ws.t2part.p);
  k_reduce_part<<<(K * N + 255) / 256, 256, 0, s>>>(ws.t2part.p, nb, K * N, grad, K * N, nullptr, 0, nullptr);
  count_launch(2);
  return check_launch("tgcn2 atb");
}

// out[e] += Σ_b part[b][e] for many blocks b and few columns e: a block owns 32 columns,
// warp w sums the blocks b ≡ w (mod 8) in ascending order (loads unrolled 8 deep),
// then one lane adds the 8 warp sums in order (fixed order, run to run).
__global__ void __launch_bounds__(256) k_reduce_part_wide(const float* __restrict__ part, int32_t nb, int32_t n,
                                                          float* __restrict__ out) {
  __shared__ float ws[8][33];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int e = blockIdx.x * 32 + lane;
  float t = 0.0f;
  if (e < n) {
    int b = w;
    for (; b + 56 < nb; b += 64) {
      float x[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) x[k] = __ldg(part + (int64_t)(b + 8 * k) * n + e);
#pragma unroll
      for (int k = 0; k < 8; ++k) t += x[k];
    }
    for (; b < nb; b += 8) t += __ldg(part + (int64_t)b * n + e);
  }
  ws[w][lane] = t;
  __syncthreads();
  if (w == 0 && e < n) {
    float tot = 0.0f;
#pragma unroll
    for (int k = 0; k < 8; ++k) tot += ws[k][lane];
    out[e] += tot;
  }
}

// element-wise parts of the cell (H = 4Q, Q in {1, 2, 4, 8, 16})
static unsigned t2_blocks(int64_t n4) {
  return (unsigned)std::min<int64_t>(std::max<int64_t>((n4 + 255) / 256, 1), (int64_t)num_sms() * 8);
}
#define STG_T2_LAUNCH(H, KERNEL, NB, ...)                                 \
  switch (H) {                                                            \
    case 4: KERNEL<1><<<NB, 256, 0, s>>>(__VA_ARGS__); break;             \
    case 8: KERNEL<2><<<NB, 256, 0, s>>>(__VA_ARGS__); break;             \
    case 16: KERNEL<4><<<NB, 256, 0, s>>>(__VA_ARGS__); break;            \
    case 32: KERNEL<8><<<NB, 256, 0, s>>>(__VA_ARGS__); break;            \
    default: KERNEL<16><<<NB, 256, 0, s>>>(__VA_ARGS__); break;           \
  }

static stg_status t2_gates(int32_t V, int32_t H, const float* A, const float* Hp, float* RUC, float* rH,
                           cudaStream_t s) {
  if (V == 0) return STG_OK;
  STG_T2_LAUNCH(H, k_t2_gates, t2_blocks((int64_t)V * H / 4), V, A, Hp, RUC, rH);
  count_launch();
  return check_launch("tgcn2 gates");
}

static stg_status t2_cand(int32_t V, int32_t H, const float* A, const float* Hp, float* RUC, float* Hn,
                          cudaStream_t s) {
  if (V == 0) return STG_OK;
  STG_T2_LAUNCH(H, k_t2_cand, t2_blocks((int64_t)V * H / 4), V, A, Hp, RUC, Hn);
  count_launch();
  return check_launch("tgcn2 candidate");
}

// ... and their gradients, with db_c += Σ_rows dA_c and db_g += Σ_rows dA_g
static stg_status t2_cand_bwd(int32_t V, int32_t H, const float* G, const float* Hp, const float* RUC, float* dAc,
                              float* du, float* dHp, float* rH, float* gbc, TgcnWs& ws, cudaStream_t s) {
  if (V == 0) return STG_OK;
  const unsigned nb = t2_blocks((int64_t)V * H / 4);
  STG_TRY(ws.t2part.alloc((size_t)nb * H));
  STG_T2_LAUNCH(H, k_t2_cand_bwd, nb, V, G, Hp, RUC, dAc, du, dHp, rH, ws.t2part.p);
  k_reduce_part_wide<<<(H + 31) / 32, 256, 0, s>>>(ws.t2part.p, (int32_t)nb, H, gbc);
  count_launch(2);
  return check_launch("tgcn2 candidate backward");
}

static stg_status t2_gate_bwd(int32_t V, int32_t H, const float* drH, const float* Hp, const float* RUC,
                              const float* du, float* dHp, float* dAg, float* gbg, TgcnWs& ws, cudaStream_t s) {
  if (V == 0) return STG_OK;
  const unsigned nb = t2_blocks((int64_t)V * H / 4);
  STG_TRY(ws.t2part.alloc((size_t)nb * 2 * H));
  STG_T2_LAUNCH(H, k_t2_gate_bwd, nb, V, drH, Hp, RUC, du, dHp, dAg, ws.t2part.p);
  k_reduce_part_wide<<<(2 * H + 31) / 32, 256, 0, s>>>(ws.t2part.p, (int32_t)nb, 2 * H, gbg);
  count_launch(2);
  return check_launch("tgcn2 gate backward");
}
#undef STG_T2_LAUNCH

static stg_status check_tgcn2(const stg_csr_view* g, const stg_tgcn2_params* p) {
  if (!g || !p || !p->Wg || !p->bg || !p->Wc || !p->bc) return fail(STG_ERR_INVALID_ARG, "tgcn2: NULL argument");
  if (p->F < 1 || p->H < 4 || p->H > 64 || p->H % 4 || (p->H & (p->H - 1)))
    return fail(STG_ERR_INVALID_ARG, "tgcn2: need F >= 1 and H in {4, 8, 16, 32, 64} (H=%d)", p->H);
  if ((size_t)(p->F + p->H) * 2 * p->H * 4 + 32 * (size_t)(p->F + p->H + 1) * 4 > 200 * 1024)
    return fail(STG_ERR_INVALID_ARG, "tgcn2: F+H=%d too large for the shared-memory weights", p->F + p->H);
  if (g->row_begin != 0 || g->row_end != g->num_nodes)
    return fail(STG_ERR_INVALID_ARG, "tgcn2: sharded views are not supported");
  return STG_OK;
}

static stg_status t2_ws(TgcnWs& ws, int32_t V, int32_t H) {
  const size_t n2 = (size_t)V * 2 * H + 4, n1 = (size_t)V * H + 4;
  STG_TRY(ws.t2z.alloc(n2)); STG_TRY(ws.t2a.alloc(n2)); STG_TRY(ws.t2b.alloc(n1));
  STG_TRY(ws.t2c.alloc(n1)); STG_TRY(ws.t2d.alloc(n1));
  return STG_OK;
}

stg_status stg_tgcn2_step(const stg_csr_view* g, const stg_tgcn2_params* p, const float* X, const float* H_prev,
                          float* H_next, stg_state_stack* stack, stg_stream_t stream) {
  STG_TRY(check_tgcn2(g, p));
  if (!X || !H_prev || !H_next) return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_step: NULL argument");
  cudaStream_t s = (cudaStream_t)stream;
  const int32_t V = g->num_nodes, F = p->F, H = p->H, H2 = 2 * H;
  TgcnWs& ws = stack ? stack->ws : global_ws();
  STG_TRY(t2_ws(ws, V, H));
  float* RUC = nullptr;                                   // [V,3H]: r | u | c, the saved state
  const size_t need = stack_bytes(V, H);
  if (stack) {
    if (stack->top + need > stack->cap)
      return fail(STG_ERR_NO_MEMORY, "stg_tgcn2_step: state stack full (%zu + %zu > %zu bytes)", stack->top, need,
                  stack->cap);
    RUC = reinterpret_cast<float*>(stack->arena.p + stack->top);
  } else {
    STG_TRY(ws.dC.alloc((size_t)V * 3 * H + 4));
    RUC = ws.dC.p;
  }
  float *Z = ws.t2z.p, *A = ws.t2a.p, *rH = ws.t2b.p;
  // gates: A = Â([X, H]·Wg) + bg  (P'-style: rows pre-scaled by n_src, n_dst per output row)
  STG_TRY(t2_mm(V, X, F, F, H_prev, H, H, p->Wg, H2, 1, H2, g->norm_src, Z, H2, false, s));
  STG_TRY(aggregate_launch(g, 0, H2, Z, H2, A, H2, g->norm_dst, nullptr, p->bg, s));
  STG_TRY(t2_gates(V, H, A, H_prev, RUC, rH, s));
  // candidate: A = Â([X, r⊙H]·Wc) + bc
  STG_TRY(t2_mm(V, X, F, F, rH, H, H, p->Wc, H, 1, H, g->norm_src, Z, H, false, s));
  STG_TRY(aggregate_launch(g, 0, H, Z, H, A, H, g->norm_dst, nullptr, p->bc, s));
  STG_TRY(t2_cand(V, H, A, H_prev, RUC, H_next, s));
  if (stack) {
    stack->entries.push_back(StackEntry{H_prev, RUC, V, H, need});
    stack->top += need;
  }
  return check_launch("stg_tgcn2_step");
}

stg_status stg_tgcn2_step_backward(const stg_csr_view* g, const stg_tgcn2_params* p, const float* X,
                                   const float* dH_next, float* dH_prev, stg_tgcn2_grads* grads,
                                   stg_state_stack* stack, stg_stream_t stream) {
  STG_TRY(check_tgcn2(g, p));
  if (!X || !dH_next || !dH_prev || !grads || !stack || !grads->Wg || !grads->bg || !grads->Wc || !grads->bc)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_step_backward: NULL argument");
  if (stack->entries.empty()) return fail(STG_ERR_STATE, "stg_tgcn2_step_backward: state stack is empty");
  const StackEntry e = stack->entries.back();
  const int32_t V = g->num_nodes, F = p->F, H = p->H, H2 = 2 * H;
  if (e.V != V || e.H != H) return fail(STG_ERR_STATE, "stg_tgcn2_step_backward: stack top does not match (V,H)");
  if (!g->out_rowptr) return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_step_backward: view lacks the backward CSR");
  cudaStream_t s = (cudaStream_t)stream;
  TgcnWs& ws = stack->ws;
  STG_TRY(t2_ws(ws, V, H));
  const float* RUC = e.C;
  const float* Hp = e.Hp;
  float *dAg = ws.t2z.p, *Y = ws.t2a.p, *rH = ws.t2b.p, *D1 = ws.t2c.p, *du = ws.t2d.p;
  STG_TRY(t2_cand_bwd(V, H, dH_next, Hp, RUC, D1, du, dH_prev, rH, grads->bc, ws, s));
  // candidate convolution: dbc, dY = Âᵀ dAc, dWc += [X, r⊙H]ᵀ dY, d(r⊙H) = dY · Wc[F:, :]ᵀ
  STG_TRY(aggregate_launch(g, 1, H, D1, H, Y, H, g->norm_src, g->norm_dst, nullptr, s));
  STG_TRY(t2_atb(V, X, F, rH, H, Y, H, grads->Wc, ws, s));
  STG_TRY(t2_mm(V, Y, H, H, nullptr, 0, 0, p->Wc + (size_t)F * H, 1, H, H, nullptr, D1, H, false, s));
  STG_TRY(t2_gate_bwd(V, H, D1, Hp, RUC, du, dH_prev, dAg, grads->bg, ws, s));
  // gate convolution: dbg, dY = Âᵀ dAg, dWg += [X, H]ᵀ dY, dH += dY · Wg[F:, :]ᵀ
  STG_TRY(aggregate_launch(g, 1, H2, dAg, H2, Y, H2, g->norm_src, g->norm_dst, nullptr, s));
  STG_TRY(t2_atb(V, X, F, Hp, H, Y, H2, grads->Wg, ws, s));
  STG_TRY(t2_mm(V, Y, H2, H2, nullptr, 0, 0, p->Wg + (size_t)F * H2, 1, H2, H, nullptr, dH_prev, H, true, s));
  stack->entries.pop_back();
  stack->top -= e.bytes;
  return check_launch("stg_tgcn2_step_backward");
}

// ---- original T-GCN in sharded mode over peer memory (NEXT-2 x §8(e)): both
// convolutions gather their source rows — which carry H — from the owners' blocks,
// so hidden-state rows cross ranks every timestep.  Phases are separated by the
// caller's cross-rank barrier (parallel.PeerTGCN2).
static stg_status check_tgcn2_peer(const stg_csr_view* g, const stg_tgcn2_params* p) {
  if (!g || !p || !p->Wg || !p->bg || !p->Wc || !p->bc) return fail(STG_ERR_INVALID_ARG, "tgcn2_peer: NULL argument");
  if (p->F < 1 || p->H < 4 || p->H > 64 || p->H % 4 || (p->H & (p->H - 1)))
    return fail(STG_ERR_INVALID_ARG, "tgcn2_peer: need F >= 1 and H in {4, 8, 16, 32, 64} (H=%d)", p->H);
  if ((size_t)(p->F + p->H) * 2 * p->H * 4 + 32 * (size_t)(p->F + p->H + 1) * 4 > 200 * 1024)
    return fail(STG_ERR_INVALID_ARG, "tgcn2_peer: F+H=%d too large for the shared-memory weights", p->F + p->H);
  return STG_OK;
}

stg_status stg_tgcn2_peer_fwd(int32_t phase, const stg_csr_view* g, const stg_tgcn2_params* p, const float* X_loc,
                              const float* H_loc, const stg_peer_rows* Z, float* Z_loc, float* H_next,
                              stg_state_stack* stack, stg_stream_t stream) {
  STG_TRY(check_tgcn2_peer(g, p));
  if (!X_loc || !H_loc || !stack || phase < 0 || phase > 2)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_peer_fwd: bad arguments (phase %d)", phase);
  cudaStream_t s = (cudaStream_t)stream;
  const int32_t R = g->row_end - g->row_begin, F = p->F, H = p->H, H2 = 2 * H;
  const float* ns_loc = g->norm_src ? g->norm_src + g->row_begin : nullptr;
  const float* nd_loc = g->norm_dst ? g->norm_dst + g->row_begin : nullptr;
  TgcnWs& ws = stack->ws;
  STG_TRY(t2_ws(ws, R > 0 ? R : 1, H));
  const size_t need = stack_bytes(R, H);
  if (stack->top + need > stack->cap) return fail(STG_ERR_NO_MEMORY, "stg_tgcn2_peer_fwd: state stack full");
  float* RUC = reinterpret_cast<float*>(stack->arena.p + stack->top);   // pushed at phase 2
  if (phase == 0) {                          // Zg rows of this block -> the peer buffer
    if (!Z_loc && R > 0) return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_peer_fwd: Z_loc is NULL");
    return t2_mm(R, X_loc, F, F, H_loc, H, H, p->Wg, H2, 1, H2, ns_loc, Z_loc, H2, false, s);
  }
  if (!Z) return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_peer_fwd: row table is NULL");
  float* A = ws.t2a.p;
  if (phase == 1) {                          // gates from the gathered Zg, then this block's Zc
    if (R == 0) return STG_OK;
    if (!Z_loc) return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_peer_fwd: Z_loc is NULL");
    STG_TRY(aggregate_launch(g, 0, H2, nullptr, 0, A, H2, nd_loc, nullptr, p->bg, s, Z));
    STG_TRY(t2_gates(R, H, A, H_loc, RUC, ws.t2b.p, s));
    return t2_mm(R, X_loc, F, F, ws.t2b.p, H, H, p->Wc, H, 1, H, ns_loc, Z_loc, H, false, s);
  }
  if (!H_next && R > 0) return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_peer_fwd: H_next is NULL");
  if (R > 0) {                               // candidate from the gathered Zc, H_next; push
    STG_TRY(aggregate_launch(g, 0, H, nullptr, 0, A, H, nd_loc, nullptr, p->bc, s, Z));
    STG_TRY(t2_cand(R, H, A, H_loc, RUC, H_next, s));
  }
  stack->entries.push_back(StackEntry{H_loc, RUC, R, H, need});
  stack->top += need;
  return check_launch("stg_tgcn2_peer_fwd");
}

stg_status stg_tgcn2_peer_bwd(int32_t phase, const stg_csr_view* g, const stg_tgcn2_params* p, const float* X_loc,
                              const float* dH_next, float* dH_prev, stg_tgcn2_grads* grads, int32_t rank,
                              int32_t world, const int32_t* bounds, const float* const* parts, float* part_out,
                              stg_state_stack* stack, stg_stream_t stream) {
  STG_TRY(check_tgcn2_peer(g, p));
  if (!X_loc || !dH_prev || !grads || !grads->Wg || !grads->bg || !grads->Wc || !grads->bc || !stack || phase < 0 ||
      phase > 2)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_peer_bwd: bad arguments (phase %d)", phase);
  if (stack->entries.empty()) return fail(STG_ERR_STATE, "stg_tgcn2_peer_bwd: state stack is empty");
  const StackEntry e = stack->entries.back();
  const int32_t V = g->num_nodes, R = g->row_end - g->row_begin, F = p->F, H = p->H, H2 = 2 * H;
  if (e.V != R || e.H != H) return fail(STG_ERR_STATE, "stg_tgcn2_peer_bwd: stack top does not match (R,H)");
  cudaStream_t s = (cudaStream_t)stream;
  TgcnWs& ws = stack->ws;
  STG_TRY(t2_ws(ws, R > 0 ? R : 1, H));
  const float* nd_loc = g->norm_dst ? g->norm_dst + g->row_begin : nullptr;
  const float* RUC = e.C;
  const float* Hp = e.Hp;
  float *dAg = ws.t2z.p, *Yl = ws.t2a.p, *rH = ws.t2b.p, *D1 = ws.t2c.p, *du = ws.t2d.p;
  if (phase == 0) {                          // candidate backward; partial dY_c of the local edges for all V
    if (!dH_next || !part_out) return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_peer_bwd: NULL dH_next / part_out");
    if (R > 0) {
      STG_TRY(t2_cand_bwd(R, H, dH_next, Hp, RUC, D1, du, dH_prev, rH, grads->bc, ws, s));
    }
    return aggregate_launch(g, 1, H, D1, H, part_out, H, g->norm_src, nd_loc, nullptr, s);
  }
  if (!parts || !bounds || world < 1 || rank < 0 || rank >= world)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_peer_bwd: bad peer arguments");
  if (phase == 1) {                          // reduce-scatter dY_c; dWc, d(r⊙H), gate backward; partial dY_g
    if (!part_out) return fail(STG_ERR_INVALID_ARG, "stg_tgcn2_peer_bwd: part_out is NULL");
    if (R > 0) {
      STG_TRY(stg_reduce_scatter_rows(world, bounds, parts, H, rank, H, Yl, H, stream));
      STG_TRY(t2_atb(R, X_loc, F, rH, H, Yl, H, grads->Wc, ws, s));
      STG_TRY(t2_mm(R, Yl, H, H, nullptr, 0, 0, p->Wc + (size_t)F * H, 1, H, H, nullptr, D1, H, false, s));
      STG_TRY(t2_gate_bwd(R, H, D1, Hp, RUC, du, dH_prev, dAg, grads->bg, ws, s));
    }
    (void)V;
    return aggregate_launch(g, 1, H2, dAg, H2, part_out, H2, g->norm_src, nd_loc, nullptr, s);
  }
  if (R > 0) {                               // reduce-scatter dY_g; dWg, dH; pop
    STG_TRY(stg_reduce_scatter_rows(world, bounds, parts, H2, rank, H2, Yl, H2, stream));
    STG_TRY(t2_atb(R, X_loc, F, Hp, H, Yl, H2, grads->Wg, ws, s));
    STG_TRY(t2_mm(R, Yl, H2, H2, nullptr, 0, 0, p->Wg + (size_t)F * H2, 1, H2, H, nullptr, dH_prev, H, true, s));
  }
  stack->entries.pop_back();
  stack->top -= e.bytes;
  return check_launch("stg_tgcn2_peer_bwd");
}

stg_status stg_mse_head(int32_t V, int32_t H, const float* Hn, const float* y, const float* w_o, const float* b_o,
                        float* loss_accum, float* dH, int32_t accumulate, float* dw_o, float* db_o,
                        stg_stream_t stream) {
  return stg_mse_head_ex(V, V, H, Hn, y, w_o, b_o, loss_accum, dH, accumulate, dw_o, db_o, stream);
}

stg_status stg_mse_head_ex(int32_t V, int32_t V_total, int32_t H, const float* Hn, const float* y, const float* w_o,
                           const float* b_o, float* loss_accum, float* dH, int32_t accumulate, float* dw_o,
                           float* db_o, stg_stream_t stream) {
  if (V_total < 1 || V_total < V)
    return fail(STG_ERR_INVALID_ARG, "stg_mse_head: V_total=%d must be >= max(1, V=%d)", V_total, V);
  if (V < 0) return fail(STG_ERR_INVALID_ARG, "stg_mse_head: V=%d < 0", V);
  if (V == 0) return STG_OK;
  if (H < 1 || H > 128 || H % 4 || !Hn || !y || !w_o || !b_o)
    return fail(STG_ERR_INVALID_ARG, "stg_mse_head: bad arguments (V=%d H=%d; H %% 4 == 0, H <= 128)", V, H);
  if (((uintptr_t)Hn | (uintptr_t)w_o | (uintptr_t)(dH ? dH : Hn)) % 16)
    return fail(STG_ERR_INVALID_ARG, "stg_mse_head: Hn, w_o, dH must be 16-byte aligned");
  cudaStream_t s = (cudaStream_t)stream;
  TgcnWs& ws = global_ws();
  const int LPR = H / 4 <= 1 ? 1 : (H / 4 <= 2 ? 2 : (H / 4 <= 4 ? 4 : (H / 4 <= 8 ? 8 : (H / 4 <= 16 ? 16 : 32))));
  if (LPR * 4 != H) return fail(STG_ERR_INVALID_ARG, "stg_mse_head: H=%d must be 4·2^k", H);
  const int rows_per_block = (kT / 32) * (32 / LPR);
  int nb = (int)std::min<int64_t>((V + rows_per_block - 1) / rows_per_block, (int64_t)num_sms() * 8);
  STG_TRY(ws.lpart.alloc(nb));
  STG_TRY(ws.gpart.alloc((size_t)nb * (H + 1)));
  const int want = (dH || dw_o || db_o) ? 1 : 0;
  ProfScope prof(PH_HEAD, s);
  switch (LPR) {
    case 1: k_mse_head<1><<<nb, kT, 0, s>>>(V, V_total, H, Hn, y, w_o, b_o, dH, accumulate, want, ws.lpart.p, ws.gpart.p); break;
    case 2: k_mse_head<2><<<nb, kT, 0, s>>>(V, V_total, H, Hn, y, w_o, b_o, dH, accumulate, want, ws.lpart.p, ws.gpart.p); break;
    case 4: k_mse_head<4><<<nb, kT, 0, s>>>(V, V_total, H, Hn, y, w_o, b_o, dH, accumulate, want, ws.lpart.p, ws.gpart.p); break;
    case 8: k_mse_head<8><<<nb, kT, 0, s>>>(V, V_total, H, Hn, y, w_o, b_o, dH, accumulate, want, ws.lpart.p, ws.gpart.p); break;
    case 16: k_mse_head<16><<<nb, kT, 0, s>>>(V, V_total, H, Hn, y, w_o, b_o, dH, accumulate, want, ws.lpart.p, ws.gpart.p); break;
    default: k_mse_head<32><<<nb, kT, 0, s>>>(V, V_total, H, Hn, y, w_o, b_o, dH, accumulate, want, ws.lpart.p, ws.gpart.p); break;
  }
  k_mse_reduce<<<H + 2, 256, 0, s>>>(nb, H, V_total, ws.lpart.p, ws.gpart.p, loss_accum, want ? dw_o : nullptr,
                                     want ? db_o : nullptr);
  count_launch(2);
  return check_launch("stg_mse_head");
}

stg_status stg_sgd_update(float* p, float* g, int64_t n, float lr, stg_stream_t stream) {
  if (n < 0 || (n > 0 && (!p || !g))) return fail(STG_ERR_INVALID_ARG, "stg_sgd_update: bad arguments");
  if (!n) return STG_OK;
  cudaStream_t s = (cudaStream_t)stream;
  k_sgd<<<(unsigned)std::min<int64_t>(ceil_div(n, 256), 4096), 256, 0, s>>>(p, g, n, lr);
  count_launch();
  return check_launch("stg_sgd_update");
}

namespace {
// per-device side streams (0: snapshot builds, 1: the pipelined compute) and
// sequence events of stg_tgcn_train_sequence
cudaStream_t side_stream(int which) {
  static std::mutex mu;
  static std::map<std::pair<int, int>, cudaStream_t> streams;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(mu);
  auto key = std::make_pair(dev, which);
  auto it = streams.find(key);
  if (it != streams.end()) return it->second;
  cudaStream_t s = nullptr;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  return streams[key] = s;
}
cudaEvent_t seq_event(int k) {
  static std::mutex mu;
  static std::map<std::pair<int, int>, cudaEvent_t> evs;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(mu);
  auto key = std::make_pair(dev, k);
  auto it = evs.find(key);
  if (it != evs.end()) return it->second;
  cudaEvent_t e = nullptr;
  cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
  return evs[key] = e;
}
// where the dL/dl/db reductions run in the pipelined backward: 0 = with the other
// reductions on the aux stream (default; measured 129.2 vs 131.6 ms/epoch for 1 =
// after the GRU backward on the H-chain stream, profiles/r01_sched_sweep.jsonl)
int dl_on_chain() {
  static const int v = [] {
    const char* e = getenv("STG_DL_STREAM");
    return e ? atoi(e) : 0;
  }();
  return v;
}
// forward: the snapshot build of t+1 starts after conv(t) (default) or after conv(t-1)
int snap_after_conv() {
  static const int v = [] {
    const char* e = getenv("STG_SNAP_AFTER_CONV");
    return e ? atoi(e) : 1;
  }();
  return v;
}
std::atomic<int> g_pipeline{1};                   // stg_set_pipeline
bool pipeline_enabled() { return g_pipeline.load(std::memory_order_relaxed) != 0; }
// compute on an aux stream beside the H chain (1, default) or on the caller's
// stream with only the snapshot builds overlapped (0)
bool aux_stream_enabled() {
  static const bool on = [] {
    const char* v = getenv("STG_AUX_STREAM");
    return !(v && v[0] == '0');
  }();
  return on;
}
}  // namespace

// Algorithm 1 for one sequence, scheduled over three streams (streams instead of
// a tracing compiler).  Per timestamp the work splits into a GRU chain that
// carries H (forward GRU + head; backward head + GRU) and H-independent work:
//   forward : Get-Graph(t+1) [snapshot stream SS] -> P' = XW, C = ÂP'+b [aux A]
//             -> GRU(t), head(t) [caller stream M]
//   backward: Get-Backward-Graph(t-1) [SS]; head(t), GRU bwd(t) [M]
//             -> dL/dl/db, dP = Âᵀ dC', dW [A]
// so the X·W and aggregations of t+1 (forward) and the reductions, backward
// aggregation and dW of t (backward) overlap the GRU chain.  Events order
// every reuse: snapshot slot pairs (a build waits for the last reader of its
// slot), the two backward buffer sets (GRU bwd(t) waits for the reductions of
// t+2), and the stack arena (a new sequence starts after the old one joined).
// Same arithmetic in the same order as the single-stream stg_tgcn_step path.
stg_status stg_set_conv_order(int32_t order) {
  if (order != 0 && order != 1) return fail(STG_ERR_INVALID_ARG, "stg_set_conv_order: %d (0 or 1)", order);
  g_conv_order.store(order, std::memory_order_relaxed);
  return STG_OK;
}

stg_status stg_set_pipeline(int32_t on) {
  g_pipeline.store(on ? 1 : 0, std::memory_order_relaxed);
  return STG_OK;
}

stg_status stg_tgcn_train_sequence(const stg_graph* graph, stg_dtdg* dtdg, int32_t t0, int32_t S,
                                   const stg_tgcn_params* p, const float* w_o, const float* b_o,
                                   const float* const* X, const float* const* Y, const float* H0, float* H_seq,
                                   float* G_work, stg_tgcn_grads* grads, float* dw_o, float* db_o,
                                   float* loss_accum, stg_state_stack* stack, stg_stream_t stream) {
  return stg_tgcn_train_sequence_ev(graph, dtdg, t0, S, p, w_o, b_o, X, Y, H0, H_seq, G_work, grads, dw_o, db_o,
                                    loss_accum, stack, nullptr, stream);
}

stg_status stg_tgcn_train_sequence_ev(const stg_graph* graph, stg_dtdg* dtdg, int32_t t0, int32_t S,
                                      const stg_tgcn_params* p, const float* w_o, const float* b_o,
                                      const float* const* X, const float* const* Y, const float* H0, float* H_seq,
                                      float* G_work, stg_tgcn_grads* grads, float* dw_o, float* db_o,
                                      float* loss_accum, stg_state_stack* stack, const stg_event_t* xy_ready,
                                      stg_stream_t stream) {
  if ((graph == nullptr) == (dtdg == nullptr))
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence: exactly one of graph / dtdg must be given");
  if (S < 1 || !X || !Y || !H0 || !H_seq || !G_work || !stack)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence: bad arguments");
  if (!grads || !grads->W || !grads->b || !grads->L || !grads->l)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence: NULL gradient pointer");
  STG_TRY(check_params(p));
  stg_csr_view view;
  if (graph) {
    STG_TRY(stg_graph_view(graph, &view));
  } else {
    if (t0 < 0 || t0 + S > stg_dtdg_num_timestamps(dtdg))
      return fail(STG_ERR_OUT_OF_RANGE, "stg_tgcn_train_sequence: [%d,%d) outside the DTDG", t0, t0 + S);
    STG_TRY(stg_dtdg_get_snapshot_parts(dtdg, t0, 0, STG_PART_IN, stream, &view));
  }
  const int32_t V = view.row_end - view.row_begin;  // local rows (all V unless sharded)
  const int32_t Vall = view.num_nodes, H = p->H;
  const size_t VH = (size_t)V * H;
  cudaStream_t ms = (cudaStream_t)stream;
  const bool pipe = pipeline_enabled();
  const bool af = agg_first();                      // aggregate-first order: no backward graph needed
  if (af) STG_TRY(check_agg_first(p));
  stg_csr_view view_af = view;                      // (its dims only; dC stays unscaled)
  view_af.norm_dst = nullptr;
  // With every snapshot materialised (STG_NAIVE) there are no builds to hide: HBM-bound
  // steps (P' larger than L2) then run faster one at a time (C5: 112.6 vs 140.6 ms per
  // epoch), L2-resident ones still gain from the overlap (C4: 10.9 vs 11.9 ms;
  // profiles/r01_table3_naive_vs_ondemand.jsonl)
  static const int l2_bytes = [] {
    int dev = 0, b = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&b, cudaDevAttrL2CacheSize, dev);
    return b;
  }();
  const bool hbm_bound = (double)Vall * 3 * H * sizeof(float) > (double)l2_bytes;
  cudaStream_t as = (pipe && aux_stream_enabled() && !(dtdg_materialised(dtdg) && hbm_bound)) ? side_stream(1) : ms;
  cudaStream_t ss = (dtdg && pipe) ? side_stream(0) : ms;
  // every buffer is sized before any asynchronous use (grow-only reallocations
  // would free memory another stream may still read)
  TgcnWs& ws = stack->ws;
  STG_TRY(ws.P.alloc((size_t)Vall * 3 * H));
  BwdBufs bb;
  STG_TRY(bwd_alloc(ws, &view, p, 2, &bb));
  // the surrogate head runs inside the tensor-core GRU kernels (forward: loss, dw_o,
  // db_o and each row's {g, ReLU mask}; backward: adds g·w_o ⊙ mask to G)
  const bool fuse_head = tc_supported(p->F, H) && V > 0;
  const int nbh = fuse_head ? tc_gru_blocks(V) : 0;
  if (fuse_head) {
    STG_TRY(ws.hg.alloc((size_t)S * V));
    STG_TRY(ws.hd_lpart.alloc((size_t)nbh));
    STG_TRY(ws.hd_gpart.alloc((size_t)nbh * (H + 1)));
  }
  const size_t need = stack_bytes(V, H, af ? p->F : 0);
  if (stack->top + (size_t)S * need > stack->cap)
    return fail(STG_ERR_NO_MEMORY, "stg_tgcn_train_sequence: state stack too small (%zu + %d x %zu > %zu bytes)",
                stack->top, S, need, stack->cap);
  cudaEvent_t ev_start = seq_event(0), ev_conv[2] = {seq_event(1), seq_event(2)};
  cudaEvent_t ev_built[2] = {seq_event(3), seq_event(4)}, ev_gru[2] = {seq_event(5), seq_event(6)};
  cudaEvent_t ev_bdone[2] = {seq_event(7), seq_event(8)};
  auto wait = [](cudaStream_t st, cudaEvent_t e, cudaStream_t rec) -> stg_status {
    if (st != rec) STG_CUDA(cudaStreamWaitEvent(st, e, 0));
    return STG_OK;
  };
  auto record = [](cudaEvent_t e, cudaStream_t st) -> stg_status {
    STG_CUDA(cudaEventRecord(e, st));
    return STG_OK;
  };
  if (pipe) {
    STG_TRY(record(ev_start, ms));                       // Get-Graph(t0) and everything before
    STG_TRY(wait(as, ev_start, ms));
    if (ss != ms) STG_TRY(wait(ss, ev_start, ms));
  }
  std::vector<int32_t> graph_stack;
  stg_csr_view views[2] = {view, view};
  // ---- forward, Algorithm 1 lines 7-16
  for (int32_t i = 0; i < S; ++i) {
    const int32_t t = t0 + i;
    const int k = dtdg ? (i & 1) : 0;
    float* C = reinterpret_cast<float*>(stack->arena.p + stack->top);   // state-stack.push target
    if (dtdg && i > 0) STG_TRY(wait(as, ev_built[i & 1], ss));
    if (xy_ready && xy_ready[i]) STG_CUDA(cudaStreamWaitEvent(as, (cudaEvent_t)xy_ready[i], 0));   // X_t landed
    float* A = af ? stack_A(C, V, H) : nullptr;
    STG_TRY(fwd_conv(&views[k], p, X[i], ws.P.p, C, as, A));            // P', C (H-independent)
    STG_TRY(record(ev_conv[i & 1], as));
    if (dtdg && i + 1 < S) {                                            // prefetch Get-Graph(t+1)
      // after conv(t) (which implies conv(t-1) is done with that slot): the build of t+1
      // then runs beside the GRU of t rather than beside the aggregation (two
      // memory-bound gathers side by side slow each other; STG_SNAP_AFTER_CONV=0: old order)
      if (snap_after_conv()) STG_TRY(wait(ss, ev_conv[i & 1], as));
      else if (i >= 1) STG_TRY(wait(ss, ev_conv[(i + 1) & 1], as));     // conv(t-1) done with that slot
      STG_TRY(stg_dtdg_get_snapshot_parts(dtdg, t + 1, 0, STG_PART_IN, ss, &views[(i + 1) & 1]));
      STG_TRY(record(ev_built[(i + 1) & 1], ss));
    }
    if (dtdg) graph_stack.push_back(t);                                 // graph-stack.push(t)
    STG_TRY(wait(ms, ev_conv[i & 1], as));
    const float* Hp = i == 0 ? H0 : H_seq + (size_t)(i - 1) * VH;
    if (xy_ready && xy_ready[i] && ms != as) STG_CUDA(cudaStreamWaitEvent(ms, (cudaEvent_t)xy_ready[i], 0));
    if (fuse_head) {                                                    // fwdprop + loss += loss-fn(out)
      const HeadArgs ha{Y[i], w_o, b_o, 1.0f / (float)Vall, ws.hd_lpart.p, ws.hd_gpart.p, ws.hg.p + (size_t)i * V};
      STG_TRY(fwd_gru(V, p, C, Hp, H_seq + (size_t)i * VH, ms, &ha));
      ProfScope prof_h(PH_HEAD, ms);
      STG_TRY(tc_seq_head_reduce(nbh, H, ws.hd_lpart.p, ws.hd_gpart.p, 1.0 / (double)Vall, loss_accum, dw_o, db_o,
                                 ms));
    } else {
      STG_TRY(fwd_gru(V, p, C, Hp, H_seq + (size_t)i * VH, ms));         // fwdprop
      STG_TRY(stg_mse_head_ex(V, Vall, H, H_seq + (size_t)i * VH, Y[i], w_o, b_o, loss_accum, nullptr, 0, nullptr,
                              nullptr, stream));                        // loss += loss-fn(out)
    }
    stack->entries.push_back(StackEntry{Hp, C, V, H, need, A});
    stack->top += need;
  }
  // ---- backward in LIFO order, lines 18-25
  float* G = G_work;
  float* Gn = G_work + VH;
  STG_CUDA(cudaMemsetAsync(G, 0, sizeof(float) * VH, ms));
  stg_csr_view bviews[2] = {views[0], views[1]};
  const bool bgraph = dtdg && !af;   // aggregate-first: the backward needs no graph (dW = (ÂX)ᵀ dC)
  if (bgraph) {    // the forward head; its out-CSR by a transpose (Alg. 3), needed by the reductions only
    STG_TRY(stg_dtdg_get_snapshot_parts(dtdg, graph_stack.back(), 1, STG_PART_OUT, ss, &bviews[(S - 1) & 1]));
    STG_TRY(record(ev_built[(S - 1) & 1], ss));
  }
  for (int32_t i = S - 1; i >= 0; --i) {
    const int b = i & 1;
    if (dtdg) graph_stack.pop_back();                                   // graph-stack.pop()
    if (bgraph) {
      if (i > 0) {                                                      // prefetch Get-Backward-Graph(t-1)
        if (i + 1 <= S - 1) STG_TRY(wait(ss, ev_bdone[(i + 1) & 1], as));   // step t+1 done with that slot
        STG_TRY(stg_dtdg_get_snapshot_parts(dtdg, graph_stack.back(), 1, STG_PART_OUT, ss, &bviews[(i - 1) & 1]));
        STG_TRY(record(ev_built[(i - 1) & 1], ss));
      }
      if (i < S - 1) STG_TRY(wait(ms, ev_built[i & 1], ss));
    }
    if (i + 2 <= S - 1) STG_TRY(wait(ms, ev_bdone[b], as));             // buffer set b free (step t+2)
    const stg_csr_view& v = af ? view_af : bviews[dtdg ? (i & 1) : 0];
    // G = dℓ_t/dH_t + dH from step t+1 (fused head: the GRU backward adds dℓ_t/dH_t)
    if (!fuse_head)
      STG_TRY(stg_mse_head_ex(V, Vall, H, H_seq + (size_t)i * VH, Y[i], w_o, b_o, nullptr, G, 1, dw_o, db_o,
                              stream));
    if (stack->entries.empty()) return fail(STG_ERR_STATE, "stg_tgcn_train_sequence: state stack underflow");
    const StackEntry e = stack->entries.back();                         // state-stack.pop()
    BwdBufs sb = bb;
    sb.dC[0] = bb.dC[b]; sb.dP[0] = bb.dP[b]; sb.da[0] = bb.da[b]; sb.RH[0] = bb.RH[b];
    STG_TRY(bwd_gru(&v, p, e.C, e.Hp, G, Gn, grads, ws, sb, ms, fuse_head ? ws.hg.p + (size_t)i * V : nullptr,
                    w_o));                                              // bwdprop: the H chain
    STG_TRY(record(ev_gru[b], ms));
    const bool dl_chain = pipe && dl_on_chain();
    if (dl_chain) STG_TRY(bwd_dl(&v, p, e.C, e.Hp, grads, ws, sb, ms));   // dL after the GRU, off the A stream
    STG_TRY(wait(as, ev_gru[b], ms));
    if (bgraph) STG_TRY(wait(as, ev_built[i & 1], ss));               // the out-CSR of t
    STG_TRY(bwd_grads(&v, p, X[i], e.C, e.Hp, grads, ws, sb, as, !dl_chain, e.A));   // parameter gradients
    STG_TRY(record(ev_bdone[b], as));
    stack->entries.pop_back();
    stack->top -= e.bytes;
    std::swap(G, Gn);
  }
  for (int b = 0; b < 2 && b < S; ++b) STG_TRY(wait(ms, ev_bdone[b], as));   // join
  return STG_OK;
}

// Sequence-batched Algorithm 1 over a STATIC graph: the
// same model and gradients as stg_tgcn_train_sequence, scheduled per sequence
// instead of per timestamp (see k_tc_gru_seq_fwd).  10 kernel launches per
// sequence instead of ~17 per timestamp.
stg_status stg_tgcn_train_sequence_batched(const stg_graph* graph, int32_t S, const stg_tgcn_params* p,
                                           const float* w_o, const float* b_o, const float* const* X,
                                           const float* const* Y, const float* H0, float* H_seq,
                                           stg_tgcn_grads* grads, float* dw_o, float* db_o, float* loss_accum,
                                           stg_state_stack* stack, stg_stream_t stream) {
  if (!graph || S < 1 || !X || !Y || !H0 || !H_seq || !stack || !w_o || !b_o)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_batched: bad arguments");
  if (S > kSeqMax) return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_batched: S=%d > %d", S, kSeqMax);
  if (!grads || !grads->W || !grads->b || !grads->L || !grads->l)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_batched: NULL gradient pointer");
  STG_TRY(check_params(p));
  const int32_t F = p->F, H = p->H, H3 = 3 * H;
  if (!tc_supported(F, H) || F > 64)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_batched: needs the tensor-core path (H 16|32, F%%4, F<=64)");
  stg_csr_view view;
  STG_TRY(stg_graph_view(graph, &view));
  if (view.row_begin != 0 || view.row_end != view.num_nodes)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_batched: sharded graphs use the per-step driver");
  const int32_t V = view.num_nodes;
  const size_t VS = (size_t)V * S;
  cudaStream_t s = (cudaStream_t)stream;
  TgcnWs& ws = stack->ws;
  const int nbmax = std::max(num_sms(), V);          // head partials: one per CTA (<= V for the small-graph kernels)
  STG_TRY(ws.sX.alloc(VS * F)); STG_TRY(ws.sY.alloc(VS)); STG_TRY(ws.sb.alloc((size_t)S * H3));
  STG_TRY(ws.sP.alloc(VS * H3)); STG_TRY(ws.sC.alloc(VS * H3)); STG_TRY(ws.sHp.alloc(VS * H));
  STG_TRY(ws.sdC.alloc(VS * H3)); STG_TRY(ws.sdP.alloc(VS * H3)); STG_TRY(ws.sda.alloc(VS * H3));
  STG_TRY(ws.sRH.alloc(VS * H)); STG_TRY(ws.slpart.alloc(nbmax)); STG_TRY(ws.sgpart.alloc((size_t)nbmax * (H + 1)));
  STG_TRY(ws.part_tc.alloc((size_t)tc_atb_max_blocks() * 2 * 128 * 128));
  STG_TRY(ws.dl_tmp.alloc(2 * 128 * 128));
  SeqPtrs ptrs{};
  for (int t = 0; t < S; ++t) {
    if (!X[t] || !Y[t]) return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_batched: NULL X/Y at %d", t);
    ptrs.x[t] = X[t];
    ptrs.y[t] = Y[t];
  }
  k_seq_gather<<<(unsigned)std::min<int64_t>(ceil_div((int64_t)VS * F, 256), 4096), 256, 0, s>>>(
      ptrs, S, V, F, p->b, H3, ws.sX.p, ws.sY.p, ws.sb.p);
  count_launch();
  {
    ProfScope prof(PH_XW, s);                        // P'_all = diag(n_src)·X_all·W over V·S rows
    STG_TRY(tc_xw(V * S, F, H, ws.sX.p, p->W, view.norm_src, ws.sP.p, s, S));
  }
  // C_all = Â·P'_all + b: one aggregation of width S·3H for the whole sequence
  STG_TRY(aggregate_launch(&view, 0, S * H3, ws.sP.p, S * H3, ws.sC.p, S * H3, view.norm_dst, nullptr, ws.sb.p, s));
  int nb1 = 0, nb2 = 0;
  {
    ProfScope prof(PH_GRU_FWD, s);                   // GRU over t = 0..S-1 + loss
    STG_TRY(tc_gru_seq_fwd(V, S, H, ws.sC.p, H0, p->L, p->l, H_seq, ws.sHp.p, ws.sY.p, w_o, b_o, ws.slpart.p, &nb1,
                           s));
    STG_TRY(tc_seq_head_reduce(nb1, H, ws.slpart.p, nullptr, 1.0 / V, loss_accum, nullptr, nullptr, s));
  }
  {
    ProfScope prof(PH_GRU_BWD, s);                   // GRU backward over t = S-1..0 + head gradient
    STG_TRY(tc_gru_seq_bwd(V, S, H, ws.sC.p, ws.sHp.p, H_seq, p->L, p->l, view.norm_dst, ws.sY.p, w_o, b_o,
                           1.0f / (float)V, ws.sdC.p, ws.sda.p, ws.sRH.p, ws.sgpart.p, &nb2, s));
    STG_TRY(tc_seq_head_reduce(nb2, H, nullptr, ws.sgpart.p, 0.0, nullptr, dw_o, db_o, s));
  }
  {
    ProfScope prof(PH_DL, s);                        // dL, dl, db over all V·S (row, t) pairs
    STG_TRY(tc_dl(V * S, H, ws.sC.p, ws.sHp.p, ws.sRH.p, ws.sda.p, ws.part_tc.p, ws.dl_tmp.p, grads->L, grads->l,
                  grads->b, p->L, s));
  }
  // dP_all = diag(n_src)·Âᵀ·dC'_all (width S·3H), dW += X_allᵀ·dP_all
  STG_TRY(aggregate_launch(&view, 1, S * H3, ws.sdC.p, S * H3, ws.sdP.p, S * H3, view.norm_src, nullptr, nullptr, s));
  ProfScope prof(PH_DW, s);
  return tc_dw(V * S, F, H, ws.sX.p, ws.sdP.p, ws.part_tc.p, ws.dl_tmp.p, grads->W, s);
}

}  // extern "C"

// ---------------------------------------------------------------- sharded mode in the library
// Stream memory operations (driver API, via the runtime's entry-point query): a
// stream waits for a peer's counter / publishes its own after the preceding work.
namespace {
typedef CUresult (*PFN_waitValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
typedef CUresult (*PFN_writeValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
struct StreamMemOps {
  PFN_waitValue32 wait = nullptr;
  PFN_writeValue32 write = nullptr;
};
stg_status stream_mem_ops(StreamMemOps* ops) {
  static StreamMemOps o;
  static std::once_flag once;
  std::call_once(once, [] {
    cudaDriverEntryPointQueryResult q;
    void* f = nullptr;
    if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      o.wait = reinterpret_cast<PFN_waitValue32>(f);
    f = nullptr;
    if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      o.write = reinterpret_cast<PFN_writeValue32>(f);
    cudaGetLastError();
  });
  if (!o.wait || !o.write) return fail(STG_ERR_CUDA, "stream memory operations unavailable");
  *ops = o;
  return STG_OK;
}
// wait until every rank's counter `slot` reached `value`
stg_status wait_all(const StreamMemOps& ops, const stg_peer_exchange* px, int slot, uint32_t value, cudaStream_t s) {
  if (value == 0) return STG_OK;
  for (int q = 0; q < px->world; ++q) {
    const CUresult r = ops.wait((CUstream)s, (CUdeviceptr)(px->flags[q] + slot), value, CU_STREAM_WAIT_VALUE_GEQ);
    if (r != CUDA_SUCCESS) return fail(STG_ERR_CUDA, "cuStreamWaitValue32 (rank %d slot %d): error %d", q, slot, (int)r);
  }
  return STG_OK;
}
stg_status publish(const StreamMemOps& ops, const stg_peer_exchange* px, int slot, uint32_t value, cudaStream_t s) {
  const CUresult r = ops.write((CUstream)s, (CUdeviceptr)(px->flags[px->rank] + slot), value, 0);
  if (r != CUDA_SUCCESS) return fail(STG_ERR_CUDA, "cuStreamWriteValue32 (slot %d): error %d", slot, (int)r);
  return STG_OK;
}
}  // namespace

stg_status stg_tgcn_train_sequence_peer(stg_dtdg* dtdg, int32_t t0, int32_t S, const stg_tgcn_params* p,
                                        const float* w_o, const float* b_o, const float* const* X_loc,
                                        const float* const* Y_loc, const float* H0, float* H_seq, float* G_work,
                                        float* dP_loc, stg_tgcn_grads* grads, float* dw_o, float* db_o,
                                        float* loss_accum, stg_state_stack* stack, stg_peer_exchange* px,
                                        stg_stream_t stream) {
  STG_TRY(check_params(p));
  if (!dtdg || !px || S < 1 || !X_loc || !Y_loc || !H0 || !H_seq || !G_work || !dP_loc || !grads || !stack ||
      !w_o || !b_o)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_peer: bad arguments");
  if (px->world < 1 || px->world > STG_MAX_PEERS || px->rank < 0 || px->rank >= px->world || !px->bounds)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_peer: bad world / rank / bounds");
  for (int q = 0; q < px->world; ++q)
    if (!px->flags[q] || !px->P[0][q] || !px->P[1][q] || !px->dP[0][q] || !px->dP[1][q])
      return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_peer: NULL exchange buffer of rank %d", q);
  if (!tc_supported(p->F, p->H)) return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_peer: needs H in {16,32}");
  if (t0 < 0 || t0 + S > stg_dtdg_num_timestamps(dtdg))
    return fail(STG_ERR_OUT_OF_RANGE, "stg_tgcn_train_sequence_peer: [%d,%d) outside the DTDG", t0, t0 + S);
  StreamMemOps ops;
  STG_TRY(stream_mem_ops(&ops));
  cudaStream_t s = (cudaStream_t)stream;
  const int32_t rb = px->bounds[px->rank], R = px->bounds[px->rank + 1] - rb, H = p->H, H3 = 3 * H;
  stg_csr_view v;
  STG_TRY(stg_dtdg_get_snapshot_parts(dtdg, t0, 0, STG_PART_IN, stream, &v));
  const int32_t Vall = v.num_nodes;
  if (v.row_begin != rb || v.row_end - v.row_begin != R)
    return fail(STG_ERR_INVALID_ARG, "stg_tgcn_train_sequence_peer: the DTDG's row block is not bounds[rank]");
  const size_t VH = (size_t)R * H;
  TgcnWs& ws = stack->ws;
  const int nbh = tc_gru_blocks(std::max(R, 1));
  STG_TRY(ws.hg.alloc((size_t)S * std::max(R, 1)));
  STG_TRY(ws.hd_lpart.alloc((size_t)nbh));
  STG_TRY(ws.hd_gpart.alloc((size_t)nbh * (H + 1)));
  const size_t need = stack_bytes(R, H);
  if (stack->top + (size_t)S * need > stack->cap)
    return fail(STG_ERR_NO_MEMORY, "stg_tgcn_train_sequence_peer: state stack too small");
  const float* blocks[2][STG_MAX_PEERS];
  const float* dblocks[2][STG_MAX_PEERS];
  for (int b = 0; b < 2; ++b)
    for (int q = 0; q < px->world; ++q) { blocks[b][q] = px->P[b][q]; dblocks[b][q] = px->dP[b][q]; }
  // ---- forward
  for (int32_t i = 0; i < S; ++i) {
    if (i > 0) STG_TRY(stg_dtdg_get_snapshot_parts(dtdg, t0 + i, 0, STG_PART_IN, stream, &v));
    const uint32_t n = ++px->fwd_count;
    const int b = (int)(n & 1u);
    STG_TRY(wait_all(ops, px, 1, n >= 2 ? n - 2 : 0, s));             // every reader of buffer b is done
    STG_TRY(stg_tgcn_project(&v, p, X_loc[i], px->P[b][px->rank], stream));
    STG_TRY(publish(ops, px, 0, n, s));
    STG_TRY(wait_all(ops, px, 0, n, s));                                // every owner's P' rows are there
    float* C = reinterpret_cast<float*>(stack->arena.p + stack->top);
    const float* Hp = i == 0 ? H0 : H_seq + (size_t)(i - 1) * VH;
    const stg_peer_rows rows{px->world, px->bounds, blocks[b], (int64_t)H3};
    const float* ndst_loc = v.norm_dst ? v.norm_dst + v.row_begin : nullptr;
    if (px->world == 1)                                                 // one owner: a plain local gather
      STG_TRY(aggregate_launch(&v, 0, H3, px->P[b][0], H3, C, H3, ndst_loc, nullptr, p->b, s));
    else
      STG_TRY(aggregate_launch(&v, 0, H3, nullptr, 0, C, H3, ndst_loc, nullptr, p->b, s, &rows));
    STG_TRY(publish(ops, px, 1, n, s));
    const HeadArgs ha{Y_loc[i], w_o, b_o, 1.0f / (float)Vall, ws.hd_lpart.p, ws.hd_gpart.p,
                      ws.hg.p + (size_t)i * std::max(R, 1)};
    STG_TRY(fwd_gru(R, p, C, Hp, H_seq + (size_t)i * VH, s, R > 0 ? &ha : nullptr));
    if (R > 0) {
      ProfScope prof_h(PH_HEAD, s);
      STG_TRY(tc_seq_head_reduce(nbh, H, ws.hd_lpart.p, ws.hd_gpart.p, 1.0 / (double)Vall, loss_accum, dw_o, db_o,
                                 s));
    }
    stack->entries.push_back(StackEntry{Hp, C, R, H, need});
    stack->top += need;
  }
  // ---- backward (LIFO)
  float* G = G_work;
  float* Gn = G_work + VH;
  if (VH) STG_CUDA(cudaMemsetAsync(G, 0, sizeof(float) * VH, s));
  for (int32_t i = S - 1; i >= 0; --i) {
    STG_TRY(stg_dtdg_get_snapshot_parts(dtdg, t0 + i, 1, STG_PART_OUT, stream, &v));
    const uint32_t m = ++px->bwd_count;
    const int b = (int)(m & 1u);
    STG_TRY(wait_all(ops, px, 3, m >= 2 ? m - 2 : 0, s));
    if (stack->entries.empty()) return fail(STG_ERR_STATE, "stg_tgcn_train_sequence_peer: state stack underflow");
    const StackEntry e = stack->entries.back();
    BwdBufs bb;
    STG_TRY(bwd_alloc(ws, &v, p, 1, &bb));
    STG_TRY(bwd_gru(&v, p, e.C, e.Hp, G, Gn, grads, ws, bb, s, R > 0 ? ws.hg.p + (size_t)i * std::max(R, 1) : nullptr,
                    w_o));
    STG_TRY(bwd_dl(&v, p, e.C, e.Hp, grads, ws, bb, s));
    // one rank: its partial dP is the whole dP (no reduce-scatter copy)
    STG_TRY(aggregate_launch(&v, 1, H3, bb.dC[0], H3, px->world == 1 ? dP_loc : px->dP[b][px->rank], H3, v.norm_src,
                             nullptr, nullptr, s));
    STG_TRY(publish(ops, px, 2, m, s));
    STG_TRY(wait_all(ops, px, 2, m, s));                                // every rank's partial dP is there
    if (px->world > 1)
      STG_TRY(stg_reduce_scatter_rows(px->world, px->bounds, dblocks[b], H3, px->rank, H3, dP_loc, H3, stream));
    STG_TRY(publish(ops, px, 3, m, s));
    STG_TRY(stg_tgcn_dw(p, R, X_loc[i], dP_loc, grads, stack, stream));
    stack->entries.pop_back();
    stack->top -= e.bytes;
    std::swap(G, Gn);
  }
  return check_launch("stg_tgcn_train_sequence_peer");
}
