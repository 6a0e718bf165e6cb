// snapshot.cu — the per-timestamp snapshot update of a DTDG (Algorithm 2's
// Get-Graph / Get-Backward-Graph step) and the node_ids /
// schedule builder (the degree presort), in few launches:
//
//   one delta step of one CSR direction (apply_dir2):
//     k_touch2       mark the sorted add / delete ranges of every touched row
//     k_rowscan      single-pass scan (decoupled look-back) of the new degrees
//                    deg' = deg + |adds| - |dels| -> rowptr', deg', the GCN
//                    norms, and the per-tile histogram of the node_ids key
//     k_merge2       old edges move to rowptr'[v] + i - #dels<c + #adds<c (deleted
//                    ones dropped), added edges are inserted; the row of an old
//                    edge comes from the old rowptr (no COO row array is kept)
//   node_ids + schedule (ids_sched_build):
//     k_ids_offsets  one CTA: digit-major exclusive scan of the tile histograms
//     k_ids_scatter  stable counting-sort scatter (warp match_any ranks)
//     k_ids_finish   one CTA: exact order of the saturated prefix (degree >=
//                    kIdsSat), hub-chunk pointers, schedule header and tiers
//     k_items2       work items in node_ids order; clears the touch marks
//
// node_ids = rows by (degree desc, id asc) (reading C4): a stable
// counting sort on the key min(deg, kIdsSat) (kIdsSat + 1 buckets, plus one
// for rows outside a sharded block, which sort last) is exact except among
// rows of degree >= kIdsSat; those form a short prefix that one CTA sorts by
// (degree desc, id asc).  Everything is integer work: bit-exact against the
// oracle (tests/test_gpu_dtdg.py, test_gpu_fullsize.py).
#include <atomic>

#include "graph.cuh"
#include "prims.cuh"

namespace stg {

namespace {

constexpr int kRowTile = 4096;                   // rows per scan / scatter tile (1024: no faster on C5, offsets 2x slower)
constexpr int kRowThreads = 256;
constexpr int kRowIPT = kRowTile / kRowThreads;  // rows per thread
constexpr int kScatRounds = kRowTile / kRowThreads;   // 32-row rounds per warp in k_ids_scatter
constexpr int kIdsSat = 1023;                    // degrees >= this share bucket 0
constexpr int kIdsBuckets = kIdsSat + 2;         // 0..kIdsSat: degree buckets, kIdsSat+1: outside the block
constexpr int kIdsOut = kIdsSat + 1;
constexpr int kSatSortMax = 8192;                // saturated prefix sorted in shared memory
constexpr int kSatRankMax = 2048;                // ... ranked by counting up to this size (O(m²/1024) per thread)
constexpr int kMergeTile = 2048;                 // old edges per merge CTA

__device__ __forceinline__ int ids_digit(int32_t v, int32_t d, int32_t rb, int32_t re) {
  if (v < rb || v >= re) return kIdsOut;
  return kIdsSat - min(d, kIdsSat);               // descending degree
}

// ------------------------------------------------------------ delta marks
// touch[row] = {add_lo, add_hi, del_lo, del_hi} (ranges in the sorted delta lists)
__global__ void k_touch2(const uint64_t* __restrict__ add, int64_t nadd, const uint64_t* __restrict__ del,
                         int64_t ndel, int nb, int4* __restrict__ touch) {
  const int64_t n = nadd + ndel;
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
    const bool is_add = k < nadd;
    const uint64_t* d = is_add ? add : del;
    const int64_t m = is_add ? nadd : ndel;
    const int64_t i = is_add ? k : k - nadd;
    const int32_t r = (int32_t)(d[i] >> nb);
    const bool first = i == 0 || (int32_t)(d[i - 1] >> nb) != r;
    const bool last = i == m - 1 || (int32_t)(d[i + 1] >> nb) != r;
    int* t = reinterpret_cast<int*>(touch + r);
    if (first) t[is_add ? 0 : 2] = (int)i;
    if (last) t[is_add ? 1 : 3] = (int)(i + 1);
  }
}

// whole-graph degree histogram of the add (+sign) and delete (-sign) batches
__global__ void k_degree_hist2(const uint64_t* __restrict__ add, int64_t nadd, const uint64_t* __restrict__ del,
                               int64_t ndel, int nb, int sign, int32_t* __restrict__ gin, int32_t* __restrict__ gout) {
  const uint64_t mask = (uint64_t(1) << nb) - 1;
  const int64_t n = nadd + ndel;
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t key = k < nadd ? add[k] : del[k - nadd];
    const int sg = k < nadd ? sign : -sign;
    atomicAdd(gin + (int32_t)(key & mask), sg);
    if (gout) atomicAdd(gout + (int32_t)(key >> nb), sg);
  }
}

// ------------------------------------------------------------ row scan
// Decoupled look-back status word of a tile: epoch (bits 34..63), flag (32..33:
// 1 = tile aggregate, 2 = inclusive prefix), value (0..31).
__device__ __forceinline__ uint64_t lb_pack(uint32_t epoch, uint32_t flag, uint32_t v) {
  return ((uint64_t)epoch << 34) | ((uint64_t)flag << 32) | v;
}
__device__ __forceinline__ void lb_store(uint64_t* p, uint64_t w) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(w) : "memory");
}
__device__ __forceinline__ uint64_t lb_load(const uint64_t* p) {
  uint64_t w;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(w) : "l"(p) : "memory");
  return w;
}

struct RowScanArgs {
  int32_t V, rb, re;
  const int32_t* deg_old;       // this direction's degrees (TOUCH) or the degrees themselves (!TOUCH)
  const int4* touch;            // TOUCH only
  int32_t* deg_new;             // TOUCH only
  int32_t* rowptr_new;          // TOUCH only ([V+1])
  int32_t* hist;                // [kIdsBuckets][ntiles]
  int32_t ntiles;
  uint64_t* status;             // [ntiles] look-back words (TOUCH only)
  uint32_t* ticket;             // tile counter, zero at launch (TOUCH only)
  uint32_t epoch;
  // GCN norms from the whole-graph degrees (may be NULL: not computed)
  const int32_t* gin;
  const int32_t* gout;
  int dgl_both;
  float* norm_src;
  float* norm_dst;
  // (TOUCH) the old CSR's row pointer: tile_row[t] = row of old edge t·kMergeTile
  const int32_t* orowptr;
  int32_t* tile_row;
};

template <bool TOUCH>
__global__ void __launch_bounds__(kRowThreads) k_rowscan(const RowScanArgs a) {
  __shared__ int32_t h[kIdsBuckets];
  __shared__ int64_t sh[32];
  __shared__ uint32_t s_tile;
  __shared__ int64_t s_prefix;
  for (int d = threadIdx.x; d < kIdsBuckets; d += kRowThreads) h[d] = 0;
  if (TOUCH) {
    if (threadIdx.x == 0) s_tile = atomicAdd(a.ticket, 1u);   // tiles in start order: look-back never waits on an unstarted tile
  }
  __syncthreads();
  const int32_t tile = TOUCH ? (int32_t)s_tile : (int32_t)blockIdx.x;
  // striped rows (coalesced): row k of this thread = tile·kRowTile + k·kRowThreads + t
  const int64_t r0 = (int64_t)tile * kRowTile + threadIdx.x;
  int32_t d[kRowIPT];
#pragma unroll
  for (int k = 0; k < kRowIPT; ++k) {
    const int64_t v = r0 + (int64_t)k * kRowThreads;
    int32_t x = 0;
    if (v < a.V) {
      x = __ldg(a.deg_old + v);
      if (TOUCH) {
        const int4 t = __ldg(a.touch + v);
        x += (t.y - t.x) - (t.w - t.z);
      }
    }
    d[k] = x;
  }
  if (a.norm_dst) {                                    // (independent of the scan: issued first)
    int32_t gi[kRowIPT], go[kRowIPT];
#pragma unroll
    for (int k = 0; k < kRowIPT; ++k) {
      const int64_t v = r0 + (int64_t)k * kRowThreads;
      gi[k] = v < a.V ? __ldg(a.gin + v) : 0;
      go[k] = (v < a.V && a.dgl_both) ? __ldg(a.gout + v) : 0;
    }
#pragma unroll
    for (int k = 0; k < kRowIPT; ++k) {
      const int64_t v = r0 + (int64_t)k * kRowThreads;
      if (v >= a.V) continue;
      const float nd = gi[k] > 0 ? 1.0f / sqrtf((float)gi[k]) : 0.0f;
      a.norm_dst[v] = nd;
      a.norm_src[v] = a.dgl_both ? (go[k] > 0 ? 1.0f / sqrtf((float)go[k]) : 0.0f) : nd;
    }
  }
  if (TOUCH) {                                          // merge tile starts inside these (old) rows
    const int ln = threadIdx.x & 31;
    int32_t ob[kRowIPT], oe31[kRowIPT];
#pragma unroll
    for (int k = 0; k < kRowIPT; ++k) {                 // row v + 1 is the next lane's row (lane 31 loads it)
      const int64_t v = r0 + (int64_t)k * kRowThreads;
      ob[k] = v <= a.V ? __ldg(a.orowptr + v) : 0;     // (row V: the end of the last row)
      oe31[k] = (ln == 31 && v < a.V) ? __ldg(a.orowptr + v + 1) : 0;
    }
#pragma unroll
    for (int k = 0; k < kRowIPT; ++k) {
      const int64_t v = r0 + (int64_t)k * kRowThreads;
      const int32_t nx = __shfl_down_sync(0xffffffffu, ob[k], 1);
      const int32_t oe = ln == 31 ? oe31[k] : nx;
      if (v < a.V)
        for (int32_t t = (ob[k] + kMergeTile - 1) / kMergeTile; (int64_t)t * kMergeTile < oe; ++t)
          a.tile_row[t] = (int32_t)v;
    }
  }
  // node_ids key histogram (shared atomics, warp-aggregated by match_any)
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int k = 0; k < kRowIPT; ++k) {
    const int64_t v = r0 + (int64_t)k * kRowThreads;
    const int dg = v < a.V ? ids_digit((int32_t)v, d[k], a.rb, a.re) : kIdsBuckets + lane;
    const unsigned peers = __match_any_sync(0xffffffffu, dg);
    if (dg < kIdsBuckets && (peers & ((1u << lane) - 1u)) == 0) atomicAdd(&h[dg], __popc(peers));
  }
  if (TOUCH) {
    // exclusive prefix of every row within the tile: the striped degrees go through
    // shared memory so that each thread scans 16 consecutive rows (one block scan)
    __shared__ int32_t sd[kRowTile + kRowTile / 32];  // padded (index i at i + i/32)
    auto pad = [](int i) { return i + (i >> 5); };
#pragma unroll
    for (int k = 0; k < kRowIPT; ++k) sd[pad(k * kRowThreads + (int)threadIdx.x)] = d[k];
    __syncthreads();
    int32_t run = 0;
#pragma unroll
    for (int k = 0; k < kRowIPT; ++k) run += sd[pad((int)threadIdx.x * kRowIPT + k)];
    int64_t tot;
    int64_t base = block_excl_scan(run, sh, &tot);
#pragma unroll
    for (int k = 0; k < kRowIPT; ++k) {
      const int i = pad((int)threadIdx.x * kRowIPT + k);
      const int32_t x = sd[i];
      sd[i] = (int32_t)base;                            // exclusive prefix within the tile
      base += x;
    }
    if (threadIdx.x < 32) {                             // warp 0: publish, then look back 32 tiles at a time
      uint64_t* st = a.status + tile;
      if (threadIdx.x == 0) lb_store(st, lb_pack(a.epoch, tile == 0 ? 2u : 1u, (uint32_t)tot));
      int64_t prefix = 0;
      for (int32_t j0 = tile - 1; j0 >= 0; j0 -= 32) {
        const int32_t j = j0 - lane;
        uint64_t w = 0;
        uint32_t fl = 2u;                               // lanes past tile 0 act as an inclusive zero
        if (j >= 0) {
          do { w = lb_load(a.status + j); } while ((uint32_t)(w >> 34) != a.epoch || ((w >> 32) & 3u) == 0);
          fl = (uint32_t)(w >> 32) & 3u;
        }
        const unsigned incl = __ballot_sync(0xffffffffu, fl == 2u);
        const int first = __ffs(incl) - 1;              // the nearest tile with an inclusive prefix (-1: none)
        int64_t v = (j >= 0 && (first < 0 || lane <= first)) ? (int64_t)(uint32_t)w : 0;
#pragma unroll
        for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        prefix += v;
        if (first >= 0) break;
      }
      if (threadIdx.x == 0) {
        if (tile > 0) lb_store(st, lb_pack(a.epoch, 2u, (uint32_t)(prefix + tot)));
        s_prefix = prefix;
        if ((int64_t)(tile + 1) * kRowTile >= a.V) a.rowptr_new[a.V] = (int32_t)(prefix + tot);
      }
    }
    __syncthreads();
    const int64_t pre = s_prefix;
#pragma unroll
    for (int k = 0; k < kRowIPT; ++k) {
      const int64_t v = r0 + (int64_t)k * kRowThreads;
      if (v < a.V) {
        a.rowptr_new[v] = (int32_t)(pre + sd[pad(k * kRowThreads + (int)threadIdx.x)]);
        a.deg_new[v] = d[k];
      }
    }
  }
  __syncthreads();
  for (int dg = threadIdx.x; dg < kIdsBuckets; dg += kRowThreads) a.hist[(int64_t)dg * a.ntiles + tile] = h[dg];
}

// ------------------------------------------------------------ node_ids
// Warp per bucket d: offs[d][t] = rows of bucket d in tiles < t (relative to the
// bucket's base), totals[d] = rows of bucket d.  The bucket bases (exclusive scan
// of the totals) are formed by each consumer from the totals.
__global__ void __launch_bounds__(1024) k_ids_offsets(const int32_t* __restrict__ hist, int32_t ntiles,
                                                      int32_t* __restrict__ offs, int32_t* __restrict__ totals) {
  const int lane = threadIdx.x & 31;
  const int d = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (d >= kIdsBuckets) return;
  const int32_t* hr = hist + (int64_t)d * ntiles;
  int32_t* orow = offs + (int64_t)d * ntiles;
  int32_t carry = 0;
  for (int t0 = 0; t0 < ntiles; t0 += 32) {
    const int t = t0 + lane;
    const int32_t x = t < ntiles ? hr[t] : 0;
    int32_t inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t y = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += y;
    }
    if (t < ntiles) orow[t] = carry + inc - x;
    carry += __shfl_sync(0xffffffffu, inc, 31);
  }
  if (lane == 0) totals[d] = carry;
}

// bucket bases: s_base[d] = Σ_{d' < d} totals[d'] (block of kRowThreads threads)
__device__ __forceinline__ void bucket_bases(const int32_t* __restrict__ totals, int32_t* s_base, int64_t* sh) {
  constexpr int PER = (kIdsBuckets + kRowThreads - 1) / kRowThreads;
  int32_t loc[PER];
  int64_t sum = 0;
#pragma unroll
  for (int k = 0; k < PER; ++k) {
    const int d = threadIdx.x * PER + k;
    loc[k] = d < kIdsBuckets ? __ldg(totals + d) : 0;
    sum += loc[k];
  }
  int64_t run = block_excl_scan(sum, sh, nullptr);
#pragma unroll
  for (int k = 0; k < PER; ++k) {
    const int d = threadIdx.x * PER + k;
    if (d < kIdsBuckets) s_base[d] = (int32_t)run;
    run += loc[k];
  }
}

// Stable scatter of one kRowTile-row tile: warp w owns rows [w·kRowTile/8, (w+1)·kRowTile/8)
// of the tile in kScatRounds rounds of 32; ranks from match_any, per-warp bucket counters.
__global__ void __launch_bounds__(kRowThreads) k_ids_scatter(const int32_t* __restrict__ deg, int32_t V, int32_t rb,
                                                             int32_t re, const int32_t* __restrict__ offs,
                                                             const int32_t* __restrict__ totals, int32_t ntiles,
                                                             int32_t* __restrict__ ids) {
  __shared__ int32_t wcnt[kRowThreads / 32][kIdsBuckets];
  __shared__ int32_t s_base[kIdsBuckets];
  __shared__ int64_t sh[32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int d = lane; d < kIdsBuckets; d += 32) wcnt[w][d] = 0;
  bucket_bases(totals, s_base, sh);
  __syncwarp();
  const int64_t base = (int64_t)blockIdx.x * kRowTile + (int64_t)w * (kRowTile / 8);
  const unsigned lt = (1u << lane) - 1u;
  int dig[kScatRounds], rank[kScatRounds];
#pragma unroll
  for (int r = 0; r < kScatRounds; ++r) {
    const int64_t v = base + r * 32 + lane;
    const bool ok = v < V;
    const int dg = ok ? ids_digit((int32_t)v, __ldg(deg + v), rb, re) : kIdsBuckets + lane;
    const unsigned peers = __match_any_sync(0xffffffffu, dg);
    const int before = ok ? wcnt[w][dg] : 0;
    rank[r] = before + __popc(peers & lt);
    dig[r] = dg;
    __syncwarp();
    if (ok && (peers & lt) == 0) wcnt[w][dg] = before + __popc(peers);
    __syncwarp();
  }
  __syncthreads();
  for (int d = threadIdx.x; d < kIdsBuckets; d += kRowThreads) {   // exclusive prefix over warps + tile offset
    int32_t run = s_base[d] + offs[(int64_t)d * ntiles + blockIdx.x];
#pragma unroll
    for (int ww = 0; ww < kRowThreads / 32; ++ww) {
      const int32_t c = wcnt[ww][d];
      wcnt[ww][d] = run;
      run += c;
    }
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < kScatRounds; ++r) {
    const int64_t v = base + r * 32 + lane;
    if (v < V) ids[wcnt[w][dig[r]] + rank[r]] = (int32_t)v;
  }
}

// One CTA: (1) the saturated prefix ids[0, m) (degree >= kIdsSat, ascending id)
// re-ordered by (degree desc, id asc); (2) n_hub = rows with degree > kHubChunk,
// their chunk pointers cptr[0..n_hub] and n_chunks; (3) the schedule header and
// the light-row tier boundaries (degree order makes them bucket-count prefixes).
__global__ void __launch_bounds__(1024) k_ids_finish(int32_t* __restrict__ ids, const int32_t* __restrict__ deg,
                                                     const int32_t* __restrict__ totals, int32_t R, int64_t coff,
                                                     int32_t* __restrict__ sched, int32_t* __restrict__ tmp) {
  extern __shared__ uint64_t sk[];                      // [kSatSortMax] sort keys
  __shared__ int32_t s_wsum[32];
  __shared__ int32_t s_btot;
  __shared__ int32_t s_cnt[3];
  const int m = totals[0];
  const int nt = blockDim.x;
  if (threadIdx.x < 3) s_cnt[threadIdx.x] = 0;
  __syncthreads();
  {    // rows with degree > kHubChunk / > kTierB / > kTierC: bucket-count prefixes
    int32_t c0 = 0, c1 = 0, c2 = 0;
    for (int d = threadIdx.x; d < kIdsSat + 1; d += nt) {
      const int32_t dd = kIdsSat - d;                   // the degree of bucket d (>= for bucket 0)
      const int32_t c = __ldg(totals + d);
      if (dd > kHubChunk) c0 += c;
      if (dd > kTierB) c1 += c;
      if (dd > kTierC) c2 += c;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      c0 += __shfl_xor_sync(0xffffffffu, c0, o);
      c1 += __shfl_xor_sync(0xffffffffu, c1, o);
      c2 += __shfl_xor_sync(0xffffffffu, c2, o);
    }
    if ((threadIdx.x & 31) == 0) { atomicAdd(&s_cnt[0], c0); atomicAdd(&s_cnt[1], c1); atomicAdd(&s_cnt[2], c2); }
  }
  if (m > 1) {
    if (m <= kSatRankMax) {                             // rank by counting over the keys in shared memory
      for (int i = threadIdx.x; i < m; i += nt) {
        const int32_t v = ids[i];
        sk[i] = ((uint64_t)(uint32_t)(0x7fffffff - deg[v]) << 32) | (uint32_t)v;
      }
      __syncthreads();
      for (int i = threadIdx.x; i < m; i += nt) {
        const uint64_t ki = sk[i];
        int r = 0;
        for (int j = 0; j < m; ++j) r += sk[j] < ki;   // same j in every lane: broadcast reads
        ids[r] = (int32_t)(uint32_t)ki;
      }
    } else if (m <= kSatSortMax) {                      // bitonic sort of (~deg, id) in shared memory
      int P = 1;
      while (P < m) P <<= 1;
      for (int i = threadIdx.x; i < P; i += nt) {
        if (i < m) {
          const int32_t v = ids[i];
          sk[i] = ((uint64_t)(uint32_t)(0x7fffffff - deg[v]) << 32) | (uint32_t)v;
        } else {
          sk[i] = ~uint64_t(0);
        }
      }
      __syncthreads();
      for (int k = 2; k <= P; k <<= 1) {
        for (int j = k >> 1; j > 0; j >>= 1) {
          for (int i = threadIdx.x; i < P; i += nt) {
            const int ixj = i ^ j;
            if (ixj > i) {
              const uint64_t a = sk[i], b = sk[ixj];
              const bool up = (i & k) == 0;
              if ((a > b) == up) { sk[i] = b; sk[ixj] = a; }
            }
          }
          __syncthreads();
        }
      }
      for (int i = threadIdx.x; i < m; i += nt) ids[i] = (int32_t)(uint32_t)sk[i];
    } else {                                            // (very large hubs only) rank by counting, O(m²)
      for (int i = threadIdx.x; i < m; i += nt) {
        const int32_t vi = ids[i], di = deg[vi];
        int r = 0;
        for (int j = 0; j < m; ++j) {
          const int32_t vj = ids[j], dj = deg[vj];
          r += dj > di || (dj == di && vj < vi);
        }
        tmp[r] = vi;
      }
      __syncthreads();
      for (int i = threadIdx.x; i < m; i += nt) ids[i] = tmp[i];
    }
    __syncthreads();
  }
  __syncthreads();
  const int32_t n_hub = s_cnt[0], n_b = s_cnt[1], n_c = s_cnt[2];
  // chunk pointers over the hub rows: exclusive scan of ceil(deg / kHubChunk); each
  // round's kFinishPT loads per thread are issued together (independent chains)
  constexpr int kFinishPT = 16;
  int32_t* cptr = sched + coff;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int32_t carry = 0;
  for (int h0 = 0; h0 < n_hub; h0 += nt * kFinishPT) {
    int32_t x[kFinishPT];
#pragma unroll
    for (int k = 0; k < kFinishPT; ++k) {
      const int h = h0 + k * nt + threadIdx.x;
      x[k] = h < n_hub ? (__ldg(deg + __ldg(ids + h)) + kHubChunk - 1) / kHubChunk : 0;
    }
    for (int k = 0; k < kFinishPT && h0 + k * nt < n_hub; ++k) {
      const int h = h0 + k * nt + threadIdx.x;
      int32_t inc = x[k];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
      }
      if (lane == 31) s_wsum[w] = inc;
      __syncthreads();
      if (w == 0) {
        const int32_t sv = lane < (nt >> 5) ? s_wsum[lane] : 0;
        int32_t si = sv;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int32_t y = __shfl_up_sync(0xffffffffu, si, o);
          if (lane >= o) si += y;
        }
        s_wsum[lane] = si - sv;                         // exclusive warp offsets
        if (lane == 31) s_btot = si;                    // block total
      }
      __syncthreads();
      if (h < n_hub) cptr[h] = carry + s_wsum[w] + inc - x[k];
      carry += s_btot;
      __syncthreads();
    }
  }
  if (threadIdx.x == 0) {
    cptr[n_hub] = carry;
    const int32_t n_chunks = carry;
    const int32_t total = n_chunks + R - n_hub;
    sched[0] = n_hub;
    sched[1] = n_chunks;
    sched[2] = (int32_t)coff;
    sched[3] = total;
    sched[4] = n_chunks + n_b - n_hub;
    sched[5] = n_chunks + n_c - n_hub;
  }
}

// Work items in node_ids order (layout in graph.cuh); then clear the touch marks
// of this step's deltas (the next step starts from zero marks).
__global__ void k_items2(const int32_t* __restrict__ ids, const int32_t* __restrict__ rowptr, int64_t cap_items,
                         int32_t* __restrict__ sched, const uint64_t* __restrict__ add, int64_t nadd,
                         const uint64_t* __restrict__ del, int64_t ndel, int nb, int4* __restrict__ touch) {
  const int32_t n_hub = sched[0], n_chunks = sched[1];
  const int32_t* cptr = sched + sched[2];
  const int64_t total = sched[3];
  int4* items = reinterpret_cast<int4*>(sched + kSchedHdr);
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total && i < cap_items; i += stride) {
    if (i < n_chunks) {
      int32_t lo = 0, hi = n_hub;      // largest h with cptr[h] <= i
      while (lo < hi) {
        const int32_t mid = (lo + hi + 1) >> 1;
        if (cptr[mid] <= i) lo = mid; else hi = mid - 1;
      }
      const int32_t v = ids[lo], rb = rowptr[v], re = rowptr[v + 1];
      const int32_t beg = rb + (int32_t)(i - cptr[lo]) * kHubChunk;
      items[i] = make_int4(v, beg, min(kHubChunk, re - beg), lo);
    } else {
      const int32_t v = ids[n_hub + (i - n_chunks)];
      const int32_t rb = rowptr[v];
      items[i] = make_int4(v, rb, rowptr[v + 1] - rb, -1);
    }
  }
  if (touch) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nadd + ndel; k += stride) {
      const uint64_t key = k < nadd ? add[k] : del[k - nadd];
      touch[(int32_t)(key >> nb)] = make_int4(0, 0, 0, 0);
    }
  }
}

// ------------------------------------------------------------ merge
__device__ __forceinline__ int64_t lb_u64(const uint64_t* a, int64_t lo, int64_t hi, uint64_t k) {
  while (lo < hi) {
    const int64_t mid = (lo + hi) >> 1;
    if (a[mid] < k) lo = mid + 1; else hi = mid;
  }
  return lo;
}
// the row of CSR position j: largest r in [lo, hi] with rowptr[r] <= j
__device__ __forceinline__ int32_t row_of(const int32_t* rp, int32_t lo, int32_t hi, int64_t j) {
  while (lo < hi) {
    const int32_t mid = (lo + hi + 1) >> 1;
    if (rp[mid] <= j) lo = mid; else hi = mid - 1;
  }
  return lo;
}

struct MergeArgs {
  int32_t V, nb;
  const int32_t* orowptr;
  const int32_t* ocol;
  int64_t E_old;
  const int32_t* nrowptr;
  const int4* touch;
  const uint64_t* add;
  int64_t nadd;
  const uint64_t* del;
  int32_t* ncol;
  int64_t old_tiles;
  // edge labels: in-direction pass records emap[old pos] = new pos
  // (-1 deleted); out-direction pass sets eid_new[new pos] = emap_in[eid_old[old pos]]
  // and searches the label of an added out-edge in the new in-CSR
  int32_t* emap_out;
  const int32_t* emap_in;
  const int32_t* eid_old;
  int32_t* eid_new;
  const int32_t* in_rowptr_new;
  const int32_t* in_col_new;
  const int32_t* tile_row;      // row of the first old edge of every tile (k_rowscan)
};

// Old edges: a CTA takes kMergeTile consecutive positions.  The tile's rows
// (rows [tile_row[t], tile_row[t+1]], from k_rowscan) have their old / new row
// pointers and touch marks cached in shared memory, and the row of every position
// comes from a max-scan of the row-start marks.  Merge path: old edges, adds and
// deletes are all sorted by key = (row << nb) | col, so each add / delete key of the
// tile's rows finds its rank among the tile's old keys ONCE (binary search in shared
// memory) and leaves a mark there; an inclusive scan of the marks gives, for every
// position k, #adds < key_k and #dels < key_k over the tile's rows; subtracting the
// earlier rows' counts (contiguous in the sorted lists, from the touch marks) leaves
// the row-local counts of the shift
//     new position = rowptr'[v] + (j − rowptr[v]) + #adds_v < key_j − #dels_v < key_j.
// Consecutive threads take consecutive positions, so the stores coalesce.  Tiles
// spanning more than kMergeRows rows (mean degree < 4) take a per-edge search path.
constexpr int kMergeRows = 512;                  // rows whose rowptr / touch / new rowptr are cached
constexpr int kMergeIPT = kMergeTile / 256;      // positions per thread

__global__ void __launch_bounds__(256) k_merge2(const MergeArgs a) {
  __shared__ int32_t scol[kMergeTile], srow[kMergeTile], smark[kMergeTile];   // marks: adds | dels << 16
  __shared__ uint8_t sdl[kMergeTile];                                          // old edge deleted
  __shared__ int32_t srp[kMergeRows + 1], snrp[kMergeRows];
  __shared__ int4 stc[kMergeRows];
  __shared__ int32_t s_lo, s_hi, s_rng[4], s_wsum[8];
  const int64_t add_blocks = (int64_t)gridDim.x - a.old_tiles;      // added edges first: their searches
  const int64_t tile = (int64_t)blockIdx.x - add_blocks;             // overlap the tiles instead of trailing
  if (tile >= 0) {
    const int64_t e0 = tile * kMergeTile;
    const int64_t e1 = min(e0 + (int64_t)kMergeTile, a.E_old);
    const int n = (int)(e1 - e0);
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    if (threadIdx.x == 0) {                            // rows [s_lo, s_hi] hold the tile's edges
      s_lo = __ldg(a.tile_row + tile);
      s_hi = tile + 1 < a.old_tiles ? __ldg(a.tile_row + tile + 1) : a.V - 1;
      s_rng[0] = INT32_MAX; s_rng[1] = INT32_MIN; s_rng[2] = INT32_MAX; s_rng[3] = INT32_MIN;
    }
#pragma unroll
    for (int i = 0; i < kMergeIPT; ++i) {
      const int k = threadIdx.x + i * 256;
      if (k < n) scol[k] = __ldcs(a.ocol + e0 + k);
      srow[k] = -1;
      smark[k] = 0;
      sdl[k] = 0;
    }
    __syncthreads();
    const int32_t rlo = s_lo, rhi = s_hi, nr = rhi - rlo + 1;
    bool cached = nr <= kMergeRows;                    // (the tile's rows: ~kMergeTile / mean degree)
    if (cached) {
      int32_t a0 = INT32_MAX, a1 = INT32_MIN, d0 = INT32_MAX, d1 = INT32_MIN;
      for (int k = threadIdx.x; k <= nr; k += blockDim.x) {
        srp[k] = __ldg(a.orowptr + rlo + k);
        if (k < nr) {
          const int4 t = __ldg(a.touch + rlo + k);
          stc[k] = t;
          snrp[k] = __ldg(a.nrowptr + rlo + k);
          if (t.y > t.x) { a0 = min(a0, t.x); a1 = max(a1, t.y); }
          if (t.w > t.z) { d0 = min(d0, t.z); d1 = max(d1, t.w); }
        }
      }
      if (a1 > a0) { atomicMin(&s_rng[0], a0); atomicMax(&s_rng[1], a1); }
      if (d1 > d0) { atomicMin(&s_rng[2], d0); atomicMax(&s_rng[3], d1); }
      __syncthreads();
      for (int k = threadIdx.x; k < nr; k += blockDim.x) {   // row-start marks (non-empty rows)
        const int32_t b = srp[k], e = srp[k + 1];
        if (e > b && b < e1) srow[max((int64_t)b - e0, (int64_t)0)] = k;
      }
    }
    __syncthreads();
    // the tile rows' add / delete keys are the contiguous ranges [A0, A1), [D0, D1)
    const int32_t A0 = s_rng[0], D0 = s_rng[2];
    const int32_t na = s_rng[1] > A0 ? s_rng[1] - A0 : 0, nd = s_rng[3] > D0 ? s_rng[3] - D0 : 0;
    cached = cached && na < 65536 && nd < 32768;       // 16-bit mark fields
    if (cached) {                                      // inclusive max-scan of the row-start marks
      int32_t m[kMergeIPT];
      int32_t run = -1;
#pragma unroll
      for (int i = 0; i < kMergeIPT; ++i) { run = max(run, srow[threadIdx.x * kMergeIPT + i]); m[i] = run; }
      int32_t inc = run;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc = max(inc, y);
      }
      if (lane == 31) s_wsum[w] = inc;
      int32_t ex = __shfl_up_sync(0xffffffffu, inc, 1);
      if (lane == 0) ex = -1;
      __syncthreads();
      for (int ww = 0; ww < w; ++ww) ex = max(ex, s_wsum[ww]);
#pragma unroll
      for (int i = 0; i < kMergeIPT; ++i) srow[threadIdx.x * kMergeIPT + i] = max(ex, m[i]);
    }
    __syncthreads();
    if (cached) {                                      // ranks of the delta keys among the tile's old keys
      const int nb = a.nb;
      auto key_at = [&](int i) { return ((uint64_t)(rlo + srow[i]) << nb) | (uint64_t)(uint32_t)scol[i]; };
      auto rank = [&](uint64_t key) {                  // # old tile keys < key
        int lo = 0, hi = n;
        while (lo < hi) { const int mid = (lo + hi) >> 1; if (key_at(mid) < key) lo = mid + 1; else hi = mid; }
        return lo;
      };
      for (int i = threadIdx.x; i < na; i += blockDim.x) {   // add a counts for positions with key > a
        const int r = rank(__ldg(a.add + A0 + i));
        if (r < n) atomicAdd(&smark[r], 1);
      }
      for (int i = threadIdx.x; i < nd; i += blockDim.x) {   // delete d: removes its old edge, counts after it
        const uint64_t key = __ldg(a.del + D0 + i);
        const int r = rank(key);
        if (r < n && key_at(r) == key) {
          sdl[r] = 1;
          if (r + 1 < n) atomicAdd(&smark[r + 1], 1 << 16);
        } else if (r == 0) {
          atomicAdd(&smark[0], 1 << 16);              // an old edge of the first row before the tile
        }
      }
    }
    __syncthreads();
    if (cached) {                                      // inclusive scan of the packed marks
      int32_t m[kMergeIPT];
      int32_t run = 0;
#pragma unroll
      for (int i = 0; i < kMergeIPT; ++i) { run += smark[threadIdx.x * kMergeIPT + i]; m[i] = run; }
      int32_t inc = run;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
      }
      if (lane == 31) s_wsum[w] = inc;
      int32_t ex = inc - run;
      __syncthreads();
      for (int ww = 0; ww < w; ++ww) ex += s_wsum[ww];
#pragma unroll
      for (int i = 0; i < kMergeIPT; ++i) smark[threadIdx.x * kMergeIPT + i] = ex + m[i];
    }
    __syncthreads();
#pragma unroll 2
    for (int i = 0; i < kMergeIPT; ++i) {
      const int k = threadIdx.x + i * 256;
      if (k >= n) break;
      const int64_t j = e0 + k;
      int64_t pos;
      if (cached) {
        const int32_t r = srow[k];
        const int4 t = stc[r];
        const int32_t mk = smark[k];
        const int32_t adds = t.y > t.x ? (mk & 0xffff) - (t.x - A0) : 0;
        const int32_t dels = t.w > t.z ? (mk >> 16) - (t.z - D0) : 0;
        pos = sdl[k] ? -1 : (int64_t)snrp[r] + (j - srp[r]) + adds - dels;
      } else {                                         // per-edge searches in the global lists
        const int32_t v = row_of(a.orowptr, rlo, rhi, j);
        const int4 t = __ldg(a.touch + v);
        pos = (int64_t)__ldg(a.nrowptr + v) + (j - __ldg(a.orowptr + v));
        if (t.y != t.x || t.w != t.z) {
          const uint64_t key = ((uint64_t)v << a.nb) | (uint64_t)(uint32_t)scol[k];
          const int64_t al = lb_u64(a.add, t.x, t.y, key), dl = lb_u64(a.del, t.z, t.w, key);
          if (dl < t.w && __ldg(a.del + dl) == key) pos = -1;
          else pos += (al - t.x) - (dl - t.z);
        }
      }
      if (a.emap_out) a.emap_out[j] = (int32_t)pos;
      if (pos < 0) continue;
      a.ncol[pos] = scol[k];
      if (a.eid_new) a.eid_new[pos] = __ldg(a.emap_in + __ldcs(a.eid_old + j));
    }
  } else {                                            // added edges
    const uint64_t mask = (uint64_t(1) << a.nb) - 1;
    const int64_t nthr = add_blocks * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.nadd; i += nthr) {
      const uint64_t key = a.add[i];
      const int32_t v = (int32_t)(key >> a.nb), c = (int32_t)(key & mask);
      const int4 t = __ldg(a.touch + v);
      int32_t lo = __ldg(a.orowptr + v), b = lo, e = __ldg(a.orowptr + v + 1);
      while (b < e) {
        const int32_t mid = (b + e) >> 1;
        if (a.ocol[mid] < c) b = mid + 1; else e = mid;
      }
      const int64_t dl = lb_u64(a.del, t.z, t.w, key);
      const int64_t pos = (int64_t)__ldg(a.nrowptr + v) + (i - t.x) + (b - lo) - (dl - t.z);
      a.ncol[pos] = c;
      if (a.eid_new) {                                // label = position of (v -> c) in the new in-CSR
        int32_t l2 = a.in_rowptr_new[c], h2 = a.in_rowptr_new[c + 1];
        while (l2 < h2) {
          const int32_t mid = (l2 + h2) >> 1;
          if (a.in_col_new[mid] < v) l2 = mid + 1; else h2 = mid;
        }
        a.eid_new[pos] = l2;
      }
    }
  }
}

inline unsigned grid_n(int64_t n, int threads = 256, int64_t max_blocks = 148 * 16) {
  const int64_t b = ceil_div(n > 0 ? n : 1, threads);
  return (unsigned)(b < max_blocks ? b : max_blocks);
}

}  // namespace

// ---------------------------------------------------------------- host side
stg_status ids_ws_reserve(BuildWs& ws, int32_t V, int64_t cap, cudaStream_t s) {
  const int64_t ntiles = ceil_div(V > 0 ? V : 1, kRowTile);
  STG_TRY(ws.ids_hist.alloc((size_t)kIdsBuckets * ntiles, s));
  STG_TRY(ws.ids_offs.alloc((size_t)kIdsBuckets * ntiles, s));
  STG_TRY(ws.ids_tot.alloc(kIdsBuckets, s));
  STG_TRY(ws.sat_tmp.alloc((size_t)std::min<int64_t>(V, cap / kIdsSat + 1), s));
  if (ws.lb_status.n < (size_t)ntiles || !ws.lb_status.p) {     // fresh status words: never a valid epoch
    STG_TRY(ws.lb_status.alloc((size_t)ntiles, s));
    STG_CUDA(cudaMemsetAsync(ws.lb_status.p, 0, sizeof(uint64_t) * ws.lb_status.n, s));
  }
  STG_TRY(ws.lb_ticket.alloc(1, s));
  STG_TRY(ws.merge_rows.alloc((size_t)ceil_div(cap > 0 ? cap : 1, kMergeTile) + 1, s));
  return STG_OK;
}

// node_ids + schedule of one direction whose key histogram is already in ws.ids_hist
static stg_status ids_sched_from_hist(const int32_t* deg, const int32_t* rowptr, int32_t V, int32_t R, int32_t* ids,
                                      int32_t* sched, int64_t cap, BuildWs& ws, cudaStream_t s, int32_t rb,
                                      int32_t re, const DirDelta* clear, int nb, int4* touch) {
  const int32_t ntiles = (int32_t)ceil_div(V, kRowTile);
  k_ids_offsets<<<(kIdsBuckets + 31) / 32, 1024, 0, s>>>(ws.ids_hist.p, ntiles, ws.ids_offs.p, ws.ids_tot.p);
  k_ids_scatter<<<ntiles, kRowThreads, 0, s>>>(deg, V, rb, re, ws.ids_offs.p, ws.ids_tot.p, ntiles, ids);
  {                                                      // dynamic shared memory opt-in, once per device
    static std::atomic<uint64_t> done{0};
    int dev = 0;
    STG_CUDA(cudaGetDevice(&dev));
    const uint64_t bit = uint64_t(1) << (dev & 63);
    if (!(done.load() & bit)) {
      STG_CUDA(cudaFuncSetAttribute(k_ids_finish, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)(kSatSortMax * sizeof(uint64_t))));
      done.fetch_or(bit);
    }
  }
  const int64_t coff = sched_cptr_off(V, cap);
  k_ids_finish<<<1, 1024, kSatSortMax * sizeof(uint64_t), s>>>(ids, deg, ws.ids_tot.p, R, coff, sched,
                                                                ws.sat_tmp.p);
  const int64_t icap = sched_items_cap(V, cap);
  const int64_t nclr = clear ? clear->nadd + clear->ndel : 0;
  k_items2<<<grid_n(std::max<int64_t>(std::min<int64_t>(icap, (int64_t)R + cap / kHubChunk + 2), nclr)), 256, 0, s>>>(
      ids, rowptr, icap, sched, clear ? clear->add : nullptr, clear ? clear->nadd : 0, clear ? clear->del : nullptr,
      clear ? clear->ndel : 0, nb, touch);
  count_launch(4);
  return check_launch("ids_sched");
}

stg_status ids_sched_build(const int32_t* deg, const int32_t* rowptr, int32_t V, int32_t R, int32_t rb, int32_t re,
                           int32_t* ids, int32_t* sched, int64_t cap, BuildWs& ws, cudaStream_t s) {
  STG_TRY(ids_ws_reserve(ws, V, cap, s));
  const int32_t ntiles = (int32_t)ceil_div(V, kRowTile);
  RowScanArgs a{};
  a.V = V; a.rb = rb; a.re = re;
  a.deg_old = deg;
  a.hist = ws.ids_hist.p;
  a.ntiles = ntiles;
  k_rowscan<false><<<ntiles, kRowThreads, 0, s>>>(a);
  count_launch();
  return ids_sched_from_hist(deg, rowptr, V, R, ids, sched, cap, ws, s, rb, re, nullptr, 0, nullptr);
}

stg_status degree_hist2(const DirDelta& d, int nb, int sign, int32_t* gin, int32_t* gout, cudaStream_t s) {
  if (d.nadd + d.ndel <= 0) return STG_OK;
  k_degree_hist2<<<grid_n(d.nadd + d.ndel), 256, 0, s>>>(d.add, d.nadd, d.del, d.ndel, nb, sign, gin, gout);
  count_launch();
  return STG_OK;
}

// One delta step of one CSR direction (see the file comment).  `norms`: also
// write the GCN norms of dst from its whole-graph degrees (gin / gout).
stg_status apply_dir2(const Snapshot& src, Snapshot& dst, bool in_dir, const DirDelta& d, int4* touch, BuildWs& ws,
                      cudaStream_t s, bool norms, int32_t* emap_out, const int32_t* emap_in, const int32_t* eid_old,
                      int32_t* eid_new, const int32_t* in_rowptr_new, const int32_t* in_col_new) {
  const int32_t V = src.V;
  STG_TRY(ids_ws_reserve(ws, V, dst.cap, s));
  const int32_t ntiles = (int32_t)ceil_div(V, kRowTile);
  if (d.nadd + d.ndel > 0) {
    k_touch2<<<grid_n(d.nadd + d.ndel), 256, 0, s>>>(d.add, d.nadd, d.del, d.ndel, src.nb, touch);
    count_launch();
  }
  const bool blk = in_dir && dst.sharded;
  RowScanArgs a{};
  a.V = V;
  a.rb = blk ? dst.rb : 0;
  a.re = blk ? dst.re : V;
  a.deg_old = in_dir ? src.in_deg.p : src.out_deg.p;
  a.touch = touch;
  a.deg_new = in_dir ? dst.in_deg.p : dst.out_deg.p;
  a.rowptr_new = in_dir ? dst.in_rowptr.p : dst.out_rowptr.p;
  a.hist = ws.ids_hist.p;
  a.ntiles = ntiles;
  a.status = ws.lb_status.p;
  a.ticket = ws.lb_ticket.p;
  a.epoch = (++ws.lb_epoch) & 0x3fffffffu;
  if (norms) {
    a.gin = dst.gin_deg.p; a.gout = dst.gout_deg.p; a.dgl_both = dst.dgl_both;
    a.norm_src = dst.norm_src.p; a.norm_dst = dst.norm_dst.p;
  }
  a.orowptr = in_dir ? src.in_rowptr.p : src.out_rowptr.p;
  a.tile_row = ws.merge_rows.p;
  STG_CUDA(cudaMemsetAsync(ws.lb_ticket.p, 0, sizeof(uint32_t), s));
  k_rowscan<true><<<ntiles, kRowThreads, 0, s>>>(a);
  count_launch();
  MergeArgs m{};
  m.V = V; m.nb = src.nb;
  m.orowptr = in_dir ? src.in_rowptr.p : src.out_rowptr.p;
  m.ocol = in_dir ? src.in_col.p : src.out_col.p;
  m.E_old = src.E;
  m.nrowptr = a.rowptr_new;
  m.touch = touch;
  m.add = d.add; m.nadd = d.nadd; m.del = d.del;
  m.ncol = in_dir ? dst.in_col.p : dst.out_col.p;
  m.old_tiles = ceil_div(src.E, kMergeTile);
  m.emap_out = emap_out; m.emap_in = emap_in; m.eid_old = eid_old; m.eid_new = eid_new;
  m.in_rowptr_new = in_rowptr_new; m.in_col_new = in_col_new;
  m.tile_row = ws.merge_rows.p;
  const int64_t add_blocks = d.nadd > 0 ? std::min<int64_t>(ceil_div(d.nadd, 256), 4 * 148) : 0;
  if (m.old_tiles + add_blocks > 0) {
    k_merge2<<<(unsigned)(m.old_tiles + add_blocks), 256, 0, s>>>(m);
    count_launch();
  }
  const int32_t R = blk ? dst.rows() : V;
  return ids_sched_from_hist(a.deg_new, a.rowptr_new, V, R, in_dir ? dst.in_ids.p : dst.out_ids.p,
                             in_dir ? dst.in_sched.p : dst.out_sched.p, dst.cap, ws, s, a.rb, a.re, &d, src.nb,
                             touch);
}

}  // namespace stg
