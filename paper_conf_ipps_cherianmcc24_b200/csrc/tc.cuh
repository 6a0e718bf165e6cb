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

#include <cuda.h>

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

// SM100 descriptor of an MN-major operand in the SWIZZLE_128B_BASE32B layout
// (layout type 1): 128-byte rows of 32 tf32 along M/N, K = rows; atoms of 4
// K-rows (SBO = 512 B apart along K), 32-element M/N chunks LBO bytes apart.
__device__ __forceinline__ uint64_t desc_mn_sw128_32b(uint32_t saddr, uint32_t lbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((512u >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)1 << 61;
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

// 1-D bulk copy global -> shared (TMA engine), completion counted in bytes on mbar
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* mbar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(mbar))
               : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* mbar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(mbar)), "r"(bytes) : "memory");
}

// 2-D TMA tensor load of box (c0, r0) of a tensor map into shared memory
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, int c0, int r0, uint64_t* mbar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(r0), "r"(smem_u32(mbar))
      : "memory");
}
// byte offset of 16-byte chunk c (0..7) of row r in a 128-byte-swizzled box (rows of 128 B)
__device__ __forceinline__ uint32_t swz128(int r, int c) { return (uint32_t)(r * 128 + ((c ^ (r & 7)) << 4)); }

// plain arrive (count 1) on an mbarrier from a thread
__device__ __forceinline__ void mbar_arrive(uint64_t* mbar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(mbar)) : "memory");
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

// Warp w writes TMEM lanes [32(w%4), +32): thread l -> lane 32(w%4)+l, 8 columns.
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const float (&v)[8]) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"r"(taddr),
               "r"(__float_as_uint(v[0])), "r"(__float_as_uint(v[1])), "r"(__float_as_uint(v[2])),
               "r"(__float_as_uint(v[3])), "r"(__float_as_uint(v[4])), "r"(__float_as_uint(v[5])),
               "r"(__float_as_uint(v[6])), "r"(__float_as_uint(v[7]))
               : "memory");
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const float (&v)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15, %16};" ::"r"(taddr),
      "r"(__float_as_uint(v[0])), "r"(__float_as_uint(v[1])), "r"(__float_as_uint(v[2])), "r"(__float_as_uint(v[3])),
      "r"(__float_as_uint(v[4])), "r"(__float_as_uint(v[5])), "r"(__float_as_uint(v[6])), "r"(__float_as_uint(v[7])),
      "r"(__float_as_uint(v[8])), "r"(__float_as_uint(v[9])), "r"(__float_as_uint(v[10])), "r"(__float_as_uint(v[11])),
      "r"(__float_as_uint(v[12])), "r"(__float_as_uint(v[13])), "r"(__float_as_uint(v[14])), "r"(__float_as_uint(v[15]))
      : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// D (+)= A·B with A in TENSOR MEMORY (K-major: lane = row, column = k) and B in
// shared memory; kind::tf32 (CUTLASS SM100_MMA_TF32_TS).
__device__ __forceinline__ void mma_tf32_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t b, uint32_t idesc,
                                            uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(b), "r"(idesc), "r"(accum));
}

// explicit shared-space 16-byte accesses (a pointer realigned through uintptr_t is generic:
// LD.E/ST.E with long-scoreboard latency instead of LDS/STS)
__device__ __forceinline__ float4 lds128(uint32_t saddr) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(saddr));
  return v;
}
__device__ __forceinline__ void sts128(uint32_t saddr, float4 v) {
  asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(saddr), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w)
               : "memory");
}
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

// As stage_rows, executed by a group of nthr threads (tid = index in the
// group, a multiple of 32 threads) instead of the whole block: producer warps
// of a warp-specialised kernel.  All loads of the thread are issued before the
// first store (up to 16 float4 in flight per thread).
template <int MAXB = 16>
__device__ __forceinline__ void stage_rows_grp(unsigned char* hi, unsigned char* lo, const float* __restrict__ src,
                                               int64_t ld, int nvalid, int rows, int F, int f0, int k0, int Ktile,
                                               int tid, int nthr) {
  const int lane = tid & 31, warp = tid >> 5, nw = nthr >> 5;
  const int nj = F / 4, njb = (nj + 3) / 4, nrb = rows / 8, total = nrb * njb;
  for (int base = warp; base < total; base += MAXB * nw) {
    float4 v[MAXB];
#pragma unroll
    for (int i = 0; i < MAXB; ++i) {
      const int it = base + i * nw;
      const int r = (it % nrb) * 8 + (lane & 7);
      const int j = (it / nrb) * 4 + (lane >> 3);
      v[i] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (it < total && j < nj && r < nvalid)
        v[i] = __ldg(reinterpret_cast<const float4*>(src + (int64_t)r * ld + f0 + 4 * j));
    }
#pragma unroll
    for (int i = 0; i < MAXB; ++i) {
      const int it = base + i * nw;
      const int r = (it % nrb) * 8 + (lane & 7);
      const int j = (it / nrb) * 4 + (lane >> 3);
      if (it < total && j < nj) st_split4(hi, lo, r, (k0 >> 2) + j, Ktile, v[i]);
    }
  }
}

// Two-phase form of stage_rows_grp for register prefetch: grp_load issues the
// thread's (at most MAXB) float4 loads of a tile, grp_store splits and stores
// them; a producer loads tile i+1 while it waits for a free ring slot.
template <int MAXB>
__device__ __forceinline__ void grp_load(float4 (&v)[MAXB], const float* __restrict__ src, int64_t ld, int nvalid,
                                         int rows, int F, int f0, int tid, int nthr) {
  const int lane = tid & 31, warp = tid >> 5, nw = nthr >> 5;
  const int nj = F / 4, njb = (nj + 3) / 4, nrb = rows / 8, total = nrb * njb;
#pragma unroll
  for (int i = 0; i < MAXB; ++i) {
    const int it = warp + i * nw;
    const int r = (it % nrb) * 8 + (lane & 7);
    const int j = (it / nrb) * 4 + (lane >> 3);
    v[i] = make_float4(0.f, 0.f, 0.f, 0.f);
    if (it < total && j < nj && r < nvalid) v[i] = __ldg(reinterpret_cast<const float4*>(src + (int64_t)r * ld + f0 + 4 * j));
  }
}
template <int MAXB>
__device__ __forceinline__ void grp_store(const float4 (&v)[MAXB], unsigned char* hi, unsigned char* lo, int rows,
                                          int F, int k0, int Ktile, int tid, int nthr) {
  const int lane = tid & 31, warp = tid >> 5, nw = nthr >> 5;
  const int nj = F / 4, njb = (nj + 3) / 4, nrb = rows / 8, total = nrb * njb;
#pragma unroll
  for (int i = 0; i < MAXB; ++i) {
    const int it = warp + i * nw;
    const int r = (it % nrb) * 8 + (lane & 7);
    const int j = (it / nrb) * 4 + (lane >> 3);
    if (it < total && j < nj) st_split4(hi, lo, r, (k0 >> 2) + j, Ktile, v[i]);
  }
}

// Coalesced row-tile store for a thread-per-row epilogue: the 32 lanes of a
// warp each hold one row (NC float4 columns) in registers.  The rows go to a
// per-warp shared-memory stage with an odd row pitch of kStagePitch<NC> float4
// (so the row-per-lane writes and the chunk-parallel reads are free of bank
// conflicts), then the warp writes them out chunk-parallel: lane l stores chunk
// q = it·32 + l of the 32-row block (row q / NC, column q % NC), i.e. lanes
// write consecutive 16-byte chunks of a row instead of 32 scattered rows per
// instruction.  dst row r = dst + (row0 + r)·ld (16-byte aligned); rows >=
// nvalid are not written.  stage: 32 · kStagePitch<NC> float4 of this warp.
template <int NC>
constexpr int kStagePitch = NC + 1 + (NC & 1);

// Write the warp's 32 staged rows out chunk-parallel (after the lanes filled
// their rows of the stage; includes the __syncwarp on both sides).
template <int NC>
__device__ __forceinline__ void flush_stage_rows(const float4* stage, float* dst, int64_t ld, int row0, int nvalid) {
  constexpr int P = kStagePitch<NC>;
  const int lane = threadIdx.x & 31;
  __syncwarp();
#pragma unroll 4
  for (int it = 0; it < NC; ++it) {
    const int q = it * 32 + lane;
    const int r = q / NC, c = q % NC;
    if (r < nvalid) reinterpret_cast<float4*>(dst + (int64_t)(row0 + r) * ld)[c] = stage[r * P + c];
  }
  __syncwarp();
}

template <int NC>
__device__ __forceinline__ void store_rows_coalesced(float4* stage, const float4 (&v)[NC], float* dst, int64_t ld,
                                                     int row0, int nvalid) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int c = 0; c < NC; ++c) stage[lane * kStagePitch<NC> + c] = v[c];
  flush_stage_rows<NC>(stage, dst, ld, row0, nvalid);
}

// TRANSPOSED operand tiles (K = rows) use a padded K-major layout: element
// (feature f, row r) of an [F' × RK] tile at
//     (f % 8)·16 + (f / 8)·SBO_T + (r % 4)·4 + (r / 4)·LBO_T,
// LBO_T = 144 (128 + 16: consecutive K core matrices shifted by one 16-byte bank
// quad), SBO_T = (RK / 4)·144.  The descriptor carries LBO_T / SBO_T.
constexpr uint32_t kLboT = 144;
__host__ __device__ __forceinline__ uint32_t sbo_t(int RK) { return (uint32_t)(RK / 4) * kLboT; }
__host__ __device__ __forceinline__ uint32_t tmaj_off(int f, int r, int RK) {
  return (uint32_t)((f & 7) * 16 + (r & 3) * 4) + (uint32_t)(f >> 3) * sbo_t(RK) + (uint32_t)(r >> 2) * kLboT;
}

// Stage rows [0,RK) × columns [f0, f0+F) of a row-major array as the TRANSPOSED
// operand (feature rows fd0.., K = rows).  Each thread owns a 4×4 block:
// 4 float4 loads (4 rows × 4 features), an in-register transpose, and four
// 16-byte stores (one per feature, 4 consecutive rows).  With LBO_T the 32
// lanes of a store (8 row quads × 4 feature quads) cover every bank quad 4
// times: conflict-free.  F % 4 == 0, RK % 4 == 0.
__device__ __forceinline__ void stage_rows_T(unsigned char* hi, unsigned char* lo, const float* __restrict__ src,
                                             int64_t ld, int nvalid, int F, int f0, int fd0, int RK) {
  const int nrq = RK / 4, nfq = F / 4, total = nrq * nfq;
  const uint32_t sbo = sbo_t(RK);
  for (int b = threadIdx.x; b < total; b += blockDim.x) {
    const int rq = b % nrq, fq = b / nrq;
    float4 v[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int r = 4 * rq + i;
      v[i] = r < nvalid ? __ldg(reinterpret_cast<const float4*>(src + (int64_t)r * ld + f0 + 4 * fq))
                        : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    const int fb = fd0 + 4 * fq;
    const uint32_t base = (uint32_t)(fb >> 3) * sbo + (uint32_t)rq * kLboT + (uint32_t)((fb & 7) * 16);
    const float t[4][4] = {{v[0].x, v[1].x, v[2].x, v[3].x}, {v[0].y, v[1].y, v[2].y, v[3].y},
                           {v[0].z, v[1].z, v[2].z, v[3].z}, {v[0].w, v[1].w, v[2].w, v[3].w}};
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      const float4 h = make_float4(tf32_hi(t[c][0]), tf32_hi(t[c][1]), tf32_hi(t[c][2]), tf32_hi(t[c][3]));
      const float4 l = make_float4(t[c][0] - h.x, t[c][1] - h.y, t[c][2] - h.z, t[c][3] - h.w);
      *reinterpret_cast<float4*>(hi + base + 16 * c) = h;
      *reinterpret_cast<float4*>(lo + base + 16 * c) = l;
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

// ---- per-warp TMA box stores (outputs leave asynchronously: no register
// dependency, no LSU store queue).  A warp owns 32 consecutive rows; its box is
// 32 rows x NCOL fp32 (NCOL*4 = 64 or 32 bytes), stored in shared memory in the
// TMA SWIZZLE_64B / SWIZZLE_32B layout (16-byte chunk c of row r at
// r*NCOL*4 + ((c ^ s(r)) << 4)), so the row-per-lane writes are conflict-free.
template <int NCOL>
__device__ __forceinline__ uint32_t box_off(int r, int c) {
  static_assert(NCOL == 16 || NCOL == 8, "box of 64 or 32 bytes");
  if constexpr (NCOL == 16) return (uint32_t)(r * 64 + ((c ^ ((r >> 1) & 3)) << 4));
  else return (uint32_t)(r * 32 + ((c ^ ((r >> 2) & 1)) << 4));
}
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, int c0, int r0, const void* src) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(c0), "r"(r0), "r"(smem_u32(src))
               : "memory");
}
__device__ __forceinline__ void tma_store_3d(const CUtensorMap* map, int c0, int r0, int z, const void* src) {
  asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%1, %2, %3}], [%4];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(c0), "r"(r0), "r"(z), "r"(smem_u32(src))
               : "memory");
}
// out[box] += smem box (fp32 add in the memory system; one add per element, so the
// result is out + v rounded once, as a load-add-store would give)
__device__ __forceinline__ void tma_reduce_add_2d(const CUtensorMap* map, int c0, int r0, const void* src) {
  asm volatile("cp.reduce.async.bulk.tensor.2d.global.shared::cta.add.tile.bulk_group [%0, {%1, %2}], [%3];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(c0), "r"(r0), "r"(smem_u32(src))
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// Double-buffered per-warp box store: buffers buf[0], buf[1] (each 32*NCOL*4
// bytes, 1024-aligned); `slot` alternates 0/1 across calls of this warp.
// Writes v*s (this lane's row) into the free buffer, then lane 0 issues the
// TMA store of box (c0, r0).  Rows past the tensor end are clipped by TMA.
template <int NCOL, bool ADD = false>
__device__ __forceinline__ void warp_box_store(unsigned char* buf0, int& slot, const float (&v)[NCOL], float s,
                                               const CUtensorMap* map, int c0, int r0) {
  constexpr int BYTES = 32 * NCOL * 4;
  const int lane = threadIdx.x & 31;
  unsigned char* buf = buf0 + slot * BYTES;
  if (lane == 0) bulk_wait_read<1>();           // the store that last used this buffer has read it
  __syncwarp();
#pragma unroll
  for (int c = 0; c < NCOL / 4; ++c) {
    const float4 x = make_float4(s * v[4 * c], s * v[4 * c + 1], s * v[4 * c + 2], s * v[4 * c + 3]);
    asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(smem_u32(buf + box_off<NCOL>(lane, c))),
                 "f"(x.x), "f"(x.y), "f"(x.z), "f"(x.w)
                 : "memory");
  }
  fence_proxy_async();
  __syncwarp();
  if (lane == 0) {
    if constexpr (ADD) tma_reduce_add_2d(map, c0, r0, buf);
    else tma_store_2d(map, c0, r0, buf);
    bulk_commit();
  }
  slot ^= 1;
}

// the same into plane z of a 3-D tensor [Z][rows][cols] (rows past the plane end are clipped)
template <int NCOL>
__device__ __forceinline__ void warp_box_store3(unsigned char* buf0, int& slot, const float (&v)[NCOL],
                                                const CUtensorMap* map, int c0, int r0, int z) {
  constexpr int BYTES = 32 * NCOL * 4;
  const int lane = threadIdx.x & 31;
  unsigned char* buf = buf0 + slot * BYTES;
  if (lane == 0) bulk_wait_read<1>();
  __syncwarp();
#pragma unroll
  for (int c = 0; c < NCOL / 4; ++c)
    asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(smem_u32(buf + box_off<NCOL>(lane, c))),
                 "f"(v[4 * c]), "f"(v[4 * c + 1]), "f"(v[4 * c + 2]), "f"(v[4 * c + 3])
                 : "memory");
  fence_proxy_async();
  __syncwarp();
  if (lane == 0) {
    tma_store_3d(map, c0, r0, z, buf);
    bulk_commit();
  }
  slot ^= 1;
}

}  // namespace tc
}  // namespace stg
