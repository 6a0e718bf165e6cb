// tc.cuh — tcgen05 / TMEM / mbarrier building blocks for sm_100a (inline PTX).
//
// Operands live in shared memory in the canonical UMMA K-major SWIZZLE_NONE
// ("interleave") layout: a core matrix is 8 rows × 16 bytes (8 × 4 fp32);
// element (r, k) of an [R × K] fp32 tile sits at
//     (r % 8)·16 + (r / 8)·SBO + (k % 4)·4 + (k / 4)·LBO      bytes
// with LBO = 128 (K-adjacent core matrices contiguous) and SBO = (K/4)·128.
// Row reductions (Xᵀ·dP, [C|H]ᵀ·da) stage their operands TRANSPOSED in this
// same K-major layout (K = rows): tf32 MN-major operands would need the
// SW128_32B layout, so we transpose while staging instead (stage_rows_T).
//
// fp32-class accuracy from TF32 tensor cores by the 3xTF32 split
// a = hi + lo (hi = a with the low 13 mantissa bits cleared, lo = a − hi exact):
//   A·B ≈ A_lo·B_hi + A_hi·B_lo + A_hi·B_hi, accumulated in fp32 in TMEM.
#pragma once

#include <cstdint>

namespace stg {
namespace tc {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// SM100 shared-memory matrix descriptor, SWIZZLE_NONE, version 1.
__device__ __forceinline__ uint64_t desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;
  return d;
}

// Instruction descriptor: kind::tf32, D fp32, A/B tf32, dense.
__host__ __device__ constexpr uint32_t idesc_tf32(int M, int N, int a_mn, int b_mn) {
  return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)a_mn << 15) | ((uint32_t)b_mn << 16) |
         ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ void mma_tf32(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n" ::"r"(tmem_d),
      "l"(a), "l"(b), "r"(idesc), "r"(accum));
}

__device__ __forceinline__ void commit(uint64_t* mbar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(mbar))
               : "memory");
}

__device__ __forceinline__ void mbar_init(uint64_t* mbar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(mbar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* mbar, uint32_t phase) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra DONE_%=;\n\t"
      "bra WAIT_%=;\n"
      "DONE_%=:\n\t}\n" ::"r"(smem_u32(mbar)),
      "r"(phase)
      : "memory");
}

__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
// make generic-proxy st.shared visible to the tensor core (async proxy)
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }

// Executed by one whole warp.
__device__ __forceinline__ void tmem_alloc(uint32_t* slot, uint32_t ncols) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(slot)), "r"(ncols)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_free(uint32_t taddr, uint32_t ncols) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}

// Warp w reads TMEM lanes [32w, 32w+32): thread l gets lane 32w+l, 8 columns.
__device__ __forceinline__ void tmem_ld8(uint32_t taddr, float (&v)[8]) {
  uint32_t r[8];
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
               : "r"(taddr));
#pragma unroll
  for (int i = 0; i < 8; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float (&v)[16]) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ float tf32_hi(float a) { return __uint_as_float(__float_as_uint(a) & 0xFFFFE000u); }

// byte offset of element (r, k) in a K-major SWIZZLE_NONE tile with K columns
__host__ __device__ __forceinline__ uint32_t kmaj_off(int r, int k, int K) {
  return (uint32_t)((r & 7) * 16 + (r >> 3) * (K / 4) * 128 + (k & 3) * 4 + (k >> 2) * 128);
}

// Store a float4 of row r, columns [4j, 4j+4) of a K-major tile as hi and lo parts.
__device__ __forceinline__ void st_split4(unsigned char* hi_base, unsigned char* lo_base, int r, int j, int K,
                                          float4 v) {
  const uint32_t off = (uint32_t)((r & 7) * 16 + (r >> 3) * (K / 4) * 128 + j * 128);
  float4 h = make_float4(tf32_hi(v.x), tf32_hi(v.y), tf32_hi(v.z), tf32_hi(v.w));
  float4 l = make_float4(v.x - h.x, v.y - h.y, v.z - h.z, v.w - h.w);
  *reinterpret_cast<float4*>(hi_base + off) = h;
  *reinterpret_cast<float4*>(lo_base + off) = l;
}

// Stage rows [0,rows) × columns [f0, f0+F) of a row-major fp32 array (leading
// dimension ld, 16-byte aligned rows) into columns [k0, k0+F) of a K-major tile
// of width Ktile, split hi/lo.  Rows >= nvalid are written as zeros.  Lane map:
// 8 rows × 4 float4 chunks per warp step -> 64-byte global segments, and one
// 128-byte smem wavefront per 8 lanes (conflict-free).  F % 4 == 0.
__device__ __forceinline__ void stage_rows(unsigned char* hi, unsigned char* lo, const float* __restrict__ src,
                                           int64_t ld, int nvalid, int rows, int F, int f0, int k0, int Ktile) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const int nj = F / 4, njb = (nj + 3) / 4, nrb = rows / 8, total = nrb * njb;
  constexpr int B = 8;   // loads in flight per thread before the first store
  for (int base = warp; base < total; base += B * nw) {
    float4 v[B];
#pragma unroll
    for (int i = 0; i < B; ++i) {
      const int it = base + i * nw;
      const int r = (it % nrb) * 8 + (lane & 7);
      const int j = (it / nrb) * 4 + (lane >> 3);
      v[i] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (it < total && j < nj && r < nvalid)
        v[i] = __ldg(reinterpret_cast<const float4*>(src + (int64_t)r * ld + f0 + 4 * j));
    }
#pragma unroll
    for (int i = 0; i < B; ++i) {
      const int it = base + i * nw;
      const int r = (it % nrb) * 8 + (lane & 7);
      const int j = (it / nrb) * 4 + (lane >> 3);
      if (it < total && j < nj) st_split4(hi, lo, r, (k0 >> 2) + j, Ktile, v[i]);
    }
  }
}

// Stage rows [0,RK) × columns [f0, f0+F) of a row-major array as the TRANSPOSED
// K-major operand: element (feature f, row r) of an [F' × RK] tile (K = rows)
// at feature row fd0 + f.  Conflict-free: lane = (r%4, chunk parity, rotation s)
// and the 4 scalars of each float4 are stored in a lane-rotated order so one
// warp store touches 32 distinct banks.  F % 4 == 0, RK % 16 == 0.
__device__ __forceinline__ void stage_rows_T(unsigned char* hi, unsigned char* lo, const float* __restrict__ src,
                                             int64_t ld, int nvalid, int F, int f0, int fd0, int RK) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const int rr = (lane & 3) + 4 * (lane >> 3);
  const int jj = (lane >> 2) & 1;
  const int s = lane >> 3;
  const int nrb = RK / 16, njb = (F + 7) / 8, total = nrb * njb;
  const uint32_t sbo = (uint32_t)(RK / 4) * 128;
  constexpr int B = 8;
  for (int base = warp; base < total; base += B * nw) {
    float4 v[B];
#pragma unroll
    for (int i = 0; i < B; ++i) {
      const int it = base + i * nw;
      const int r = (it % nrb) * 16 + rr;
      const int j = (it / nrb) * 2 + jj;
      v[i] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (it < total && 4 * j < F && r < nvalid)
        v[i] = __ldg(reinterpret_cast<const float4*>(src + (int64_t)r * ld + f0 + 4 * j));
    }
#pragma unroll
    for (int i = 0; i < B; ++i) {
      const int it = base + i * nw;
      const int r = (it % nrb) * 16 + rr;
      const int j = (it / nrb) * 2 + jj;
      if (it >= total || 4 * j >= F) continue;
#pragma unroll
      for (int t = 0; t < 4; ++t) {
        const int ci = (t + s) & 3;
        const float x = ci == 0 ? v[i].x : (ci == 1 ? v[i].y : (ci == 2 ? v[i].z : v[i].w));
        const int f = fd0 + 4 * j + ci;
        const uint32_t off = (uint32_t)((f & 7) * 16) + (uint32_t)(f >> 3) * sbo + (uint32_t)((r & 3) * 4) +
                             (uint32_t)(r >> 2) * 128;
        const float h = tf32_hi(x);
        *reinterpret_cast<float*>(hi + off) = h;
        *reinterpret_cast<float*>(lo + off) = x - h;
      }
    }
  }
}

// Stage a small row-major matrix W [K × N] (weights, read once per CTA) as the
// K-major B operand [N × Kp] (transpose), zero for k >= K.
__device__ __forceinline__ void stage_weight_T(unsigned char* hi, unsigned char* lo, const float* __restrict__ W,
                                               int K, int N, int Kp, int ldw) {
  for (int e = threadIdx.x; e < N * Kp; e += blockDim.x) {
    const int n = e / Kp, k = e % Kp;
    const float v = k < K ? W[(int64_t)k * ldw + n] : 0.0f;
    const float h = tf32_hi(v);
    *reinterpret_cast<float*>(hi + kmaj_off(n, k, Kp)) = h;
    *reinterpret_cast<float*>(lo + kmaj_off(n, k, Kp)) = v - h;
  }
}

// Issue the 3xTF32 MMA chain D (+)= A·B over K (multiple of 8) for one tile:
// A tiles [M × K] and B tiles [N × K] K-major with the layout above.
__device__ __forceinline__ void mma_3xtf32_kmajor(uint32_t tmem_d, uint32_t a_hi, uint32_t a_lo, uint32_t b_hi,
                                                  uint32_t b_lo, int K, uint32_t idesc, bool accumulate) {
  const uint32_t sbo_a = (uint32_t)(K / 4) * 128, sbo_b = sbo_a;
  for (int k = 0; k < K; k += 8) {
    const uint32_t off = (uint32_t)(k / 4) * 128;   // two core matrices per K=8 step
    const uint32_t acc = (accumulate || k > 0) ? 1u : 0u;
    mma_tf32(tmem_d, desc(a_lo + off, 128, sbo_a), desc(b_hi + off, 128, sbo_b), idesc, acc);
    mma_tf32(tmem_d, desc(a_hi + off, 128, sbo_a), desc(b_lo + off, 128, sbo_b), idesc, 1u);
    mma_tf32(tmem_d, desc(a_hi + off, 128, sbo_a), desc(b_hi + off, 128, sbo_b), idesc, 1u);
  }
}

}  // namespace tc
}  // namespace stg
