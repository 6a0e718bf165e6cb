// snapshot.cu — the per-timestamp snapshot update of a DTDG (Algorithm 2's
// Get-Graph / Get-Backward-Graph step) and the node_ids /
// schedule builder (the degree presort), in few launches:
//
//   one delta step of one CSR direction (apply_dir2):
//     k_touch3       mark the sorted add / delete ranges of every touched row;
//                    place every delta key in the OLD CSR (its merge-path
//                    position); the whole-graph degree deltas of the step
//     k_rowscan      single-pass scan (decoupled look-back) of the new degrees
//                    deg' = deg + |adds| - |dels| -> rowptr', deg', the
//                    whole-graph degrees and GCN norms, the per-tile
//                    histogram of the node_ids key, and the merge tiles'
//                    first add / delete
//     k_merge4       global merge path over the sorted (row, col) keys: old
//                    edge j -> j - #dels before j + #adds placed <= j, add i at
//                    old position p -> p - #dels before p + i (a warp per 256
//                    old positions; no row lookups, no shared memory)
//   node_ids + schedule (ids_sched_build):
//     k_ids_offsets  one CTA: digit-major exclusive scan of the tile histograms
//     k_ids_scatter  stable counting-sort scatter (warp match_any ranks)
//     k_ids_finish   one CTA: exact order of the saturated prefix (degree >=
//                    kIdsSat), its hub-chunk pointers, the per-bucket chunk
//                    bases, schedule header and tiers
//     k_items2       work items in node_ids order (the other hub-chunk
//                    pointers in closed form); clears the step's marks
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

__device__ __forceinline__ int ids_digit(int32_t v, int32_t d, int32_t rb, int32_t re) {
  if (v < rb || v >= re) return kIdsOut;
  return kIdsSat - min(d, kIdsSat);               // descending degree
}

// ------------------------------------------------------------ delta marks
// One launch over the step's delta keys (sorted, effective: adds absent from the
// old CSR, deletes present):
//   touch[row] = {add_lo, add_hi, del_lo, del_hi} (ranges in the sorted lists);
//   padd[i] / pdel[i] = the key's position in the OLD CSR (insertion point of an
//     add = number of old keys below it; a delete's own position) — old CSR
//     positions are the global (row, col) key order, so these are the merge
//     path of k_merge4;
//   (gdeg) the whole-graph degree deltas into the zeroed scratch din / dout.
struct TouchArgs {
  const uint64_t* add;
  int64_t nadd;
  const uint64_t* del;
  int64_t ndel;
  int nb;
  int4* touch;
  const int32_t* orowptr;
  const int32_t* ocol;
  int32_t* padd;
  int32_t* pdel;
  const uint64_t* gadd;         // whole-graph keys (may be NULL)
  int64_t ngadd;
  const uint64_t* gdel;
  int64_t ngdel;
  int sign;
  int32_t* din;
  int32_t* dout;
};

constexpr int kMergeShift = 8;
constexpr int kMergeTile = 1 << kMergeShift;     // old positions per merge warp task

__device__ __forceinline__ int32_t old_pos(const int32_t* __restrict__ orowptr, const int32_t* __restrict__ ocol,
                                           uint64_t key, int nb) {
  const int32_t r = (int32_t)(key >> nb), c = (int32_t)(key & ((uint64_t(1) << nb) - 1));
  int32_t b = __ldg(orowptr + r), e = __ldg(orowptr + r + 1);
  // lower bound of c in ocol[b, e): 8-ary steps (7 independent probes per level, so a
  // hub row of 10^5 edges takes 6 dependent rounds instead of 17), binary below 8
  while (e - b > 8) {
    const int32_t len = e - b;
    int32_t lt = 0;                                   // probes below c (they are monotone)
#pragma unroll
    for (int k = 1; k < 8; ++k) lt += __ldg(ocol + b + (int32_t)(((int64_t)len * k) >> 3)) < c;
    const int32_t nb_ = lt ? b + (int32_t)(((int64_t)len * lt) >> 3) + 1 : b;
    e = lt < 7 ? b + (int32_t)(((int64_t)len * (lt + 1)) >> 3) : e;
    b = nb_;
  }
  while (b < e) {
    const int32_t mid = (b + e) >> 1;
    if (__ldg(ocol + mid) < c) b = mid + 1; else e = mid;
  }
  return b;
}

__global__ void __launch_bounds__(256) k_touch3(const TouchArgs a) {
  const int64_t n = a.nadd + a.ndel, ng = a.ngadd + a.ngdel;
  const uint64_t gmask = (uint64_t(1) << a.nb) - 1;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t kend = max(n, ng);
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < kend; k += stride) {
    if (k < ng) {
      const uint64_t key = k < a.ngadd ? a.gadd[k] : a.gdel[k - a.ngadd];
      const int sg = k < a.ngadd ? a.sign : -a.sign;
      if (a.din) atomicAdd(a.din + (int32_t)(key & gmask), sg);
      if (a.dout) atomicAdd(a.dout + (int32_t)(key >> a.nb), sg);
    }
    const bool on = k < n;
    const bool is_add = k < a.nadd;
    const uint64_t* d = is_add ? a.add : a.del;
    const int64_t m = is_add ? a.nadd : a.ndel;
    const int64_t i = is_add ? k : k - a.nadd;
    if (on) {
      const uint64_t key = d[i];
      const int32_t r = (int32_t)(key >> a.nb);
      const bool first = i == 0 || (int32_t)(d[i - 1] >> a.nb) != r;
      const bool last = i == m - 1 || (int32_t)(d[i + 1] >> a.nb) != r;
      int* t = reinterpret_cast<int*>(a.touch + r);
      if (first) t[is_add ? 0 : 2] = (int)i;
      if (last) t[is_add ? 1 : 3] = (int)(i + 1);
      (is_add ? a.padd : a.pdel)[i] = old_pos(a.orowptr, a.ocol, key, a.nb);
    }
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
  uint32_t* ticket;             // (TOUCH) [tile claims, finished tiles, generation], zero-initialised;
                                // each launch's last tile resets the counts and bumps the generation
  // GCN norms from the whole-graph degrees (may be NULL: not computed)
  const int32_t* gin;
  const int32_t* gout;
  int dgl_both;
  float* norm_src;
  float* norm_dst;
  // fused whole-graph degree step (may be NULL): gin / gout are the source slot's,
  // the degrees are gin + din, gout + dout, written to gin_w / gout_w
  const int32_t* din;           // (NULL with self_dir 1: the in-degrees are this scan's own)
  const int32_t* dout;          // (NULL with self_dir 2: the out-degrees are this scan's own)
  int self_dir;                 // unsharded: 1 = this is the in-CSR, 2 = the out-CSR (its deg' is whole-graph)
  int32_t* gin_w;
  int32_t* gout_w;
  // (TOUCH) merge-tile boundaries from the old-CSR positions of k_touch3:
  // abnd[t] / dbnd[t] = adds / deletes placed in merge tiles < t, t in [0, ntm]
  const int32_t* padd;
  int64_t nadd;
  const int32_t* pdel;
  int64_t ndel;
  int32_t* abnd;
  int32_t* dbnd;
  int32_t ntm;
};

// B[t] = entries of the sorted position list P[0, n) in tiles < t (t in [0, ntm]):
// positions are monotone, so entry i writes the tiles between its predecessor's and
// its own (entry n: up to ntm)
__device__ __forceinline__ void tile_bounds(const int32_t* __restrict__ P, int64_t n, int32_t ntm,
                                            int32_t* __restrict__ B, int64_t gid, int64_t gstride) {
  for (int64_t i = gid; i <= n; i += gstride) {
    const int32_t tp = i > 0 ? (__ldg(P + i - 1) >> kMergeShift) : -1;
    const int32_t ti = i < n ? (__ldg(P + i) >> kMergeShift) : ntm;
    for (int32_t t = tp + 1; t <= ti; ++t) B[t] = (int32_t)i;
  }
}

template <bool TOUCH>
__global__ void __launch_bounds__(kRowThreads) k_rowscan(const RowScanArgs a) {
  __shared__ int32_t h[kIdsBuckets];
  __shared__ int64_t sh[32];
  __shared__ uint32_t s_tile, s_epoch;
  __shared__ int64_t s_prefix;
  for (int d = threadIdx.x; d < kIdsBuckets; d += kRowThreads) h[d] = 0;
  if (TOUCH) {
    if (threadIdx.x == 0) {
      s_tile = atomicAdd(a.ticket, 1u);                // tiles in start order: look-back never waits on an unstarted tile
      // this launch's status-word tag: the generation the previous launch left, plus one
      // (device-side, so a CUDA-graph replay of the launch gets a fresh tag too)
      s_epoch = *reinterpret_cast<volatile uint32_t*>(a.ticket + 2) % 0x3fffffffu + 1u;
    }
  }
  __syncthreads();
  const int32_t tile = TOUCH ? (int32_t)s_tile : (int32_t)blockIdx.x;
  const uint32_t epoch = TOUCH ? s_epoch : 0u;
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
    if (a.gin_w) {                                     // whole-graph degrees of this step (both kept current)
      int32_t di[kRowIPT], dd[kRowIPT];
#pragma unroll
      for (int k = 0; k < kRowIPT; ++k) {
        const int64_t v = r0 + (int64_t)k * kRowThreads;
        const bool ok = v < a.V;
        gi[k] = (ok && a.self_dir != 1) ? __ldg(a.gin + v) : 0;
        go[k] = (ok && a.self_dir != 2) ? __ldg(a.gout + v) : 0;
        di[k] = (ok && a.self_dir != 1) ? __ldcg(a.din + v) : 0;
        dd[k] = (ok && a.self_dir != 2) ? __ldcg(a.dout + v) : 0;
      }
#pragma unroll
      for (int k = 0; k < kRowIPT; ++k) {
        const int64_t v = r0 + (int64_t)k * kRowThreads;
        gi[k] = a.self_dir == 1 ? d[k] : gi[k] + di[k];
        go[k] = a.self_dir == 2 ? d[k] : go[k] + dd[k];
        if (v < a.V) { a.gin_w[v] = gi[k]; a.gout_w[v] = go[k]; }
      }
    } else {
#pragma unroll
      for (int k = 0; k < kRowIPT; ++k) {
        const int64_t v = r0 + (int64_t)k * kRowThreads;
        gi[k] = v < a.V ? __ldg(a.gin + v) : 0;
        go[k] = (v < a.V && a.dgl_both) ? __ldg(a.gout + v) : 0;
      }
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
      if (threadIdx.x == 0) lb_store(st, lb_pack(epoch, tile == 0 ? 2u : 1u, (uint32_t)tot));
      int64_t prefix = 0;
      for (int32_t j0 = tile - 1; j0 >= 0; j0 -= 32) {
        const int32_t j = j0 - lane;
        uint64_t w = 0;
        uint32_t fl = 2u;                               // lanes past tile 0 act as an inclusive zero
        if (j >= 0) {
          do { w = lb_load(a.status + j); } while ((uint32_t)(w >> 34) != epoch || ((w >> 32) & 3u) == 0);
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
        if (tile > 0) lb_store(st, lb_pack(epoch, 2u, (uint32_t)(prefix + tot)));
        s_prefix = prefix;
        if ((int64_t)(tile + 1) * kRowTile >= a.V) a.rowptr_new[a.V] = (int32_t)(prefix + tot);
      }
    } else if (a.abnd) {                                // warps 1..7 meanwhile: the merge-tile boundaries
      constexpr int kB = kRowThreads - 32;
      const int64_t gid = (int64_t)tile * kB + (threadIdx.x - 32), gs = (int64_t)a.ntiles * kB;
      tile_bounds(a.padd, a.nadd, a.ntm, a.abnd, gid, gs);
      tile_bounds(a.pdel, a.ndel, a.ntm, a.dbnd, gid, gs);
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
  if (TOUCH && threadIdx.x == 0) {                      // last tile out: reset the claims, publish the generation
    __threadfence();
    if (atomicAdd(a.ticket + 1, 1u) == gridDim.x - 1) {
      a.ticket[0] = 0;
      a.ticket[1] = 0;
      a.ticket[2] = epoch;
    }
  }
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
  constexpr int kOffPT = (kIdsBuckets + kRowThreads - 1) / kRowThreads;
  int32_t toff[kOffPT];                                   // this tile's bucket offsets, issued first
#pragma unroll
  for (int k = 0; k < kOffPT; ++k) {
    const int d = threadIdx.x + k * kRowThreads;
    toff[k] = d < kIdsBuckets ? __ldg(offs + (int64_t)d * ntiles + blockIdx.x) : 0;
  }
  for (int d = lane; d < kIdsBuckets; d += 32) wcnt[w][d] = 0;
  bucket_bases(totals, s_base, sh);
  __syncwarp();
  const int64_t base = (int64_t)blockIdx.x * kRowTile + (int64_t)w * (kRowTile / 8);
  const unsigned lt = (1u << lane) - 1u;
  int dig[kScatRounds], rank[kScatRounds];
#pragma unroll
  for (int r = 0; r < kScatRounds; ++r) {             // every degree of the warp's rows in flight first
    const int64_t v = base + r * 32 + lane;
    dig[r] = v < V ? __ldg(deg + v) : 0;
  }
#pragma unroll
  for (int r = 0; r < kScatRounds; ++r) {
    const int64_t v = base + r * 32 + lane;
    const bool ok = v < V;
    const int dg = ok ? ids_digit((int32_t)v, dig[r], rb, re) : kIdsBuckets + lane;
    const unsigned peers = __match_any_sync(0xffffffffu, dg);
    const int before = ok ? wcnt[w][dg] : 0;
    rank[r] = before + __popc(peers & lt);
    dig[r] = dg;
    __syncwarp();
    if (ok && (peers & lt) == 0) wcnt[w][dg] = before + __popc(peers);
    __syncwarp();
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kOffPT; ++k) {                      // exclusive prefix over warps + tile offset
    const int d = threadIdx.x + k * kRowThreads;
    if (d >= kIdsBuckets) break;
    int32_t run = s_base[d] + toff[k];
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
// re-ordered by (degree desc, id asc); (2) n_hub = rows with degree > kHubChunk
// and the schedule header / light-row tiers (degree order makes them bucket-count
// prefixes); (3) the hub-chunk pointers of the saturated prefix (a scan over its m
// rows) and, for every other hub bucket b (all of its rows have degree exactly
// kIdsSat - b, so ceil(deg / kHubChunk) chunks each), the bucket's first chunk
// bk[b] and first row bk[kIdsBuckets + b]: k_items2 derives the rest of cptr in
// closed form, so no per-hub pass runs in this single CTA.
__global__ void __launch_bounds__(1024) k_ids_finish(int32_t* __restrict__ ids, const int32_t* __restrict__ deg,
                                                     const int32_t* __restrict__ totals, int32_t R, int64_t coff,
                                                     int32_t* __restrict__ sched, int32_t* __restrict__ tmp,
                                                     int32_t* __restrict__ bk) {
  extern __shared__ uint64_t sk[];                      // [kSatSortMax] sort keys
  __shared__ int32_t s_wsum[32];
  __shared__ int32_t s_btot;
  __shared__ int32_t s_cnt[3];
  const int m = totals[0];
  const int nt = blockDim.x;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  // block-wide exclusive scan (nt threads); *tot = the block total
  auto bscan = [&](int32_t x, int32_t* tot) -> int32_t {
    int32_t inc = x;
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
      s_wsum[lane] = si - sv;                           // exclusive warp offsets
      if (lane == 31) s_btot = si;                      // block total
    }
    __syncthreads();
    const int32_t ex = s_wsum[w] + inc - x;
    *tot = s_btot;
    __syncthreads();                                    // s_wsum / s_btot reused by the next scan
    return ex;
  };
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
  }
  __syncthreads();
  const int32_t n_hub = s_cnt[0], n_b = s_cnt[1], n_c = s_cnt[2];
  // (3a) chunk pointers over the saturated prefix (every row of it is a hub)
  int32_t* cptr = sched + coff;
  int32_t carry = 0;
  for (int h0 = 0; h0 < m; h0 += nt) {
    const int h = h0 + threadIdx.x;
    const int32_t x = h < m ? (__ldg(deg + __ldg(ids + h)) + kHubChunk - 1) / kHubChunk : 0;
    int32_t tot;
    const int32_t ex = bscan(x, &tot);
    if (h < m) cptr[h] = carry + ex;
    carry += tot;
  }
  const int32_t csat = carry;
  // (3b) the other hub buckets b in [1, kIdsSat - kHubChunk): first chunk and first row
  {
    const int b = threadIdx.x;                          // nt >= kIdsSat + 1 threads
    const bool hubb = b >= 1 && b < kIdsSat - kHubChunk;
    const int32_t cnt = hubb ? __ldg(totals + b) : 0;
    const int32_t nc = hubb ? (kIdsSat - b + kHubChunk - 1) / kHubChunk : 0;
    int32_t tchunks, trows;
    const int32_t exc = bscan(cnt * nc, &tchunks);
    const int32_t exr = bscan(cnt, &trows);
    if (b < kIdsBuckets) {
      bk[b] = carry + exc;
      bk[kIdsBuckets + b] = m + exr;
    }
    carry += tchunks;
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
    sched[6] = m;                                       // saturated rows (cptr[0..m) written here)
    sched[7] = csat;                                    // their chunks
  }
}

// Work items in node_ids order (layout in graph.cuh); then clear the touch marks
// of this step's deltas (the next step starts from zero marks).  A hub chunk item
// finds its row in the saturated prefix by a search over cptr[0..m], else through
// the bucket tables of k_ids_finish (closed form: every row of bucket b has the
// same chunk count); the first chunk of each such row writes its cptr entry.
__global__ void k_items2(const int32_t* __restrict__ ids, const int32_t* __restrict__ rowptr, int64_t cap_items,
                         int32_t* __restrict__ sched, const int32_t* __restrict__ bk, const uint64_t* __restrict__ add,
                         int64_t nadd, const uint64_t* __restrict__ del, int64_t ndel, int nb,
                         int4* __restrict__ touch, const uint64_t* __restrict__ gadd, int64_t ngadd,
                         const uint64_t* __restrict__ gdel, int64_t ngdel, int32_t* __restrict__ din,
                         int32_t* __restrict__ dout) {
  const int32_t n_hub = sched[0], n_chunks = sched[1], m = sched[6], csat = sched[7];
  int32_t* cptr = sched + sched[2];
  const int64_t total = sched[3];
  int4* items = reinterpret_cast<int4*>(sched + kSchedHdr);
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total && i < cap_items; i += stride) {
    if (i < n_chunks) {
      int32_t h, j;
      if (i < csat) {
        int32_t lo = 0, hi = m - 1;                     // largest h with cptr[h] <= i
        while (lo < hi) {
          const int32_t mid = (lo + hi + 1) >> 1;
          if (cptr[mid] <= i) lo = mid; else hi = mid - 1;
        }
        h = lo;
        j = (int32_t)i - cptr[lo];
      } else {
        int32_t lo = 1, hi = kIdsSat - kHubChunk - 1;   // largest hub bucket b with bk[b] <= i
        while (lo < hi) {
          const int32_t mid = (lo + hi + 1) >> 1;
          if (__ldg(bk + mid) <= i) lo = mid; else hi = mid - 1;
        }
        const int32_t nc = (kIdsSat - lo + kHubChunk - 1) / kHubChunk;
        const int32_t off = (int32_t)i - __ldg(bk + lo);
        h = __ldg(bk + kIdsBuckets + lo) + off / nc;
        j = off % nc;
        if (j == 0) cptr[h] = (int32_t)i;
      }
      const int32_t v = ids[h], rb = rowptr[v], re = rowptr[v + 1];
      const int32_t beg = rb + j * kHubChunk;
      items[i] = make_int4(v, beg, min(kHubChunk, re - beg), h);
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
  if (din || dout) {
    const uint64_t mask = (uint64_t(1) << nb) - 1;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < ngadd + ngdel; k += stride) {
      const uint64_t key = k < ngadd ? gadd[k] : gdel[k - ngadd];
      if (din) din[(int32_t)(key & mask)] = 0;
      if (dout) dout[(int32_t)(key >> nb)] = 0;
    }
  }
}

// ------------------------------------------------------------ merge
// The CSR of one direction, read in position order, is the sorted key sequence
// (row << nb | col); the new CSR is the merge of the surviving old keys and the
// added keys (both sorted), so with D(j) = deletes at old positions < j and
// A(j) = adds whose insertion point p <= j (k_touch3):
//   surviving old edge j  ->  j − D(j) + A(j)
//   added key i (point p) ->  p − D(p) + i
// (rows need not be known: rowptr' comes from the degree scan).
struct MergeArgs {
  int nb;
  const int32_t* ocol;
  int64_t E_old;
  const uint64_t* add;
  const int32_t* padd;
  const int32_t* pdel;
  const int32_t* abnd;
  const int32_t* dbnd;
  int32_t* ncol;
  // edge labels: in-direction pass records emap[old pos] = new pos
  // (-1 deleted); out-direction pass sets eid_new[new pos] = emap_in[eid_old[old pos]]
  // and searches the label of an added out-edge in the new in-CSR
  int32_t* emap_out;
  const int32_t* emap_in;
  const int32_t* eid_old;
  int32_t* eid_new;
  const int32_t* in_rowptr_new;
  const int32_t* in_col_new;
};

// One warp per merge tile of kMergeTile old positions, in rounds of 32 (lane =
// position, so loads and stores coalesce).  The tile's adds / deletes are the
// contiguous ranges [a0, a1) / [d0, d1) of the sorted lists (k_rowscan); the warp
// loads all its old columns and the first 32 entries of each range (with the
// add keys) in one go, then per round every lane counts the entries before its
// own position with a warp-uniform loop over the round's entries (typically 0-2;
// a range longer than 32 reloads its next 32).  The list index where a round
// starts is the count of entries before it, so
//   D(j) = deletes before j,  A(j) = adds placed at or before j
// are global without any scan.  No shared memory, no block synchronisation.
constexpr int kMergeRounds = kMergeTile / 32;

struct MergeChunk {              // 32 consecutive entries of a sorted position list, one per lane
  int32_t base;                  // list index of lane 0's entry
  int32_t off;                   // entries of the chunk consumed
  int32_t p;                     // this lane's position (INT32_MAX past the range)
  int32_t idx;                   // this lane's list index
};

__device__ __forceinline__ void chunk_load(MergeChunk& ch, const int32_t* __restrict__ P, int32_t base, int32_t end,
                                           int lane) {
  ch.base = base;
  ch.off = 0;
  ch.idx = base + lane;
  ch.p = ch.idx < end ? __ldg(P + ch.idx) : INT32_MAX;
}

template <bool LABELS>
__global__ void __launch_bounds__(256, LABELS ? 5 : 8) k_merge4(const MergeArgs a, int32_t ntm) {
  const unsigned FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const int32_t t = (int32_t)(blockIdx.x * 8 + (threadIdx.x >> 5));
  if (t >= ntm) return;                               // (warp-uniform)
  const int64_t e0 = (int64_t)t << kMergeShift;
  const int32_t a1 = __ldg(a.abnd + t + 1), d1 = __ldg(a.dbnd + t + 1);
  const int32_t a0 = __ldg(a.abnd + t), d0 = __ldg(a.dbnd + t);
  const uint64_t mask = (uint64_t(1) << a.nb) - 1;
  int32_t c[kMergeRounds], eo[LABELS ? kMergeRounds : 1];
#pragma unroll
  for (int r = 0; r < kMergeRounds; ++r) {            // every old column of the tile in flight
    const int64_t j = e0 + r * 32 + lane;
    c[r] = j < a.E_old ? __ldcs(a.ocol + j) : 0;
    if (LABELS) eo[r] = j < a.E_old ? __ldcs(a.eid_old + j) : 0;
  }
  MergeChunk cd, ca;
  chunk_load(cd, a.pdel, d0, d1, lane);
  chunk_load(ca, a.padd, a0, a1, lane);
  uint64_t key = ca.idx < a1 ? __ldg(a.add + ca.idx) : 0;
  // Fast path (the common tile: at most 32 adds and 32 deletes, no two adds at one
  // point): per round a 32-bit mask of deleted positions and one of add points
  // (warp OR-reductions), lane r < 8 holding round r's masks and the counts before
  // it; every position then needs a popcount, every add a shuffle.
  const int32_t p_prev = __shfl_up_sync(FULL, ca.p, 1);
  const bool dup = (ca.idx < a1) && lane > 0 && p_prev == ca.p;
  if (d1 - d0 <= 32 && a1 - a0 <= 32 && !__any_sync(FULL, dup)) {
    const int32_t e0i = (int32_t)e0;
    const bool vd = cd.idx < d1, va = ca.idx < a1;
    const int rd = vd ? (cd.p - e0i) >> 5 : -1, ra = va ? (ca.p - e0i) >> 5 : -1;
    uint32_t md = 0, ma = 0;                          // lane r < 8: round r's masks
#pragma unroll
    for (int r = 0; r < kMergeRounds; ++r) {
      const uint32_t xd = __reduce_or_sync(FULL, rd == r ? 1u << (cd.p & 31) : 0u);
      const uint32_t xa = __reduce_or_sync(FULL, ra == r ? 1u << (ca.p & 31) : 0u);
      if (lane == r) { md = xd; ma = xa; }
    }
    // counts before round `lane` (exclusive scan over the 8 rounds), as global list indices
    int32_t sd = __popc(md), sa = __popc(ma);
#pragma unroll
    for (int o = 1; o < 8; o <<= 1) {
      const int32_t yd = __shfl_up_sync(FULL, sd, o), ya = __shfl_up_sync(FULL, sa, o);
      if (lane >= o) { sd += yd; sa += ya; }
    }
    const int32_t Dr = d0 + sd - __popc(md), Ar = a0 + sa - __popc(ma);
    const uint32_t lt = (1u << lane) - 1u, le = lt | (1u << lane);
#pragma unroll
    for (int r = 0; r < kMergeRounds; ++r) {          // the surviving old edges
      const int32_t j = e0i + r * 32 + lane;
      const uint32_t mdr = __shfl_sync(FULL, md, r), mar = __shfl_sync(FULL, ma, r);
      const int32_t D = __shfl_sync(FULL, Dr, r) + __popc(mdr & lt);
      const int32_t A = __shfl_sync(FULL, Ar, r) + __popc(mar & le);
      if ((int64_t)j < a.E_old) {
        const bool deleted = (mdr >> lane) & 1u;
        const int32_t pos = deleted ? -1 : j - D + A;
        if (a.emap_out) a.emap_out[j] = pos;
        if (!deleted) {
          a.ncol[pos] = c[r];
          if (LABELS) a.eid_new[pos] = __ldg(a.emap_in + eo[LABELS ? r : 0]);
        }
      }
    }
    // the adds: deletes before point p = round (p >> 5)'s count + the mask bits below p
    const int rr = ra < 0 ? 0 : ra;
    const uint32_t mdp = __shfl_sync(FULL, md, rr);
    const int32_t Dp = __shfl_sync(FULL, Dr, rr) + __popc(mdp & ((1u << (ca.p & 31)) - 1u));
    if (va) {
      const int64_t q = (int64_t)ca.p - Dp + ca.idx;
      const int32_t v = (int32_t)(key >> a.nb), cc = (int32_t)(key & mask);
      a.ncol[q] = cc;
      if (LABELS) {                                   // label = position of (v -> cc) in the new in-CSR
        int32_t l2 = a.in_rowptr_new[cc], h2 = a.in_rowptr_new[cc + 1];
        while (l2 < h2) {
          const int32_t mid = (l2 + h2) >> 1;
          if (a.in_col_new[mid] < v) l2 = mid + 1; else h2 = mid;
        }
        a.eid_new[q] = l2;
      }
    }
    return;
  }
#pragma unroll
  for (int r = 0; r < kMergeRounds; ++r) {
    const int64_t base = e0 + r * 32;
    const int64_t j = base + lane;
    // deletes of this round
    int32_t D = cd.base + cd.off;                     // deletes before the round
    bool deleted = false;
    while (true) {
      const int nin = __popc(__ballot_sync(FULL, lane >= cd.off && cd.p < base + 32));
      for (int l = cd.off; l < cd.off + nin; ++l) {
        const int32_t ql = __shfl_sync(FULL, cd.p, l);
        D += ql < j;
        deleted |= ql == j;
      }
      cd.off += nin;
      if (cd.off < 32 || cd.base + 32 >= d1) break;
      chunk_load(cd, a.pdel, cd.base + 32, d1, lane);  // (a range longer than 32)
    }
    // adds of this round: count, and place them (the deletes before an add's point
    // p are lane (p - base)'s D)
    int32_t A = ca.base + ca.off;
    while (true) {
      const bool in = lane >= ca.off && ca.p < base + 32;
      const int nin = __popc(__ballot_sync(FULL, in));
      for (int l = ca.off; l < ca.off + nin; ++l) A += __shfl_sync(FULL, ca.p, l) <= j;
      const int32_t Dp = __shfl_sync(FULL, D, in ? (int)(ca.p - base) : 0);
      if (in) {
        const int64_t q = (int64_t)ca.p - Dp + ca.idx;
        const int32_t v = (int32_t)(key >> a.nb), cc = (int32_t)(key & mask);
        a.ncol[q] = cc;
        if (LABELS) {                                 // label = position of (v -> cc) in the new in-CSR
          int32_t l2 = a.in_rowptr_new[cc], h2 = a.in_rowptr_new[cc + 1];
          while (l2 < h2) {
            const int32_t mid = (l2 + h2) >> 1;
            if (a.in_col_new[mid] < v) l2 = mid + 1; else h2 = mid;
          }
          a.eid_new[q] = l2;
        }
      }
      ca.off += nin;
      if (ca.off < 32 || ca.base + 32 >= a1) break;
      chunk_load(ca, a.padd, ca.base + 32, a1, lane);
      key = ca.idx < a1 ? __ldg(a.add + ca.idx) : 0;
    }
    if (j < a.E_old) {                                // the surviving old edges
      const int64_t pos = deleted ? -1 : j - D + A;
      if (a.emap_out) a.emap_out[j] = (int32_t)pos;
      if (!deleted) {
        a.ncol[pos] = c[r];
        if (LABELS) a.eid_new[pos] = __ldg(a.emap_in + eo[LABELS ? r : 0]);
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
  STG_TRY(ws.ids_tot.alloc(3 * kIdsBuckets, s));   // totals | bucket chunk bases | bucket row bases
  STG_TRY(ws.sat_tmp.alloc((size_t)std::min<int64_t>(V, cap / kIdsSat + 1), s));
  if (ws.lb_status.n < (size_t)ntiles || !ws.lb_status.p) {     // fresh status words: never a valid epoch
    STG_TRY(ws.lb_status.alloc((size_t)ntiles, s));
    STG_CUDA(cudaMemsetAsync(ws.lb_status.p, 0, sizeof(uint64_t) * ws.lb_status.n, s));
  }
  if (!ws.lb_ticket.p) {                                // self-resetting claim counters + generation
    STG_TRY(ws.lb_ticket.alloc(3, s));
    STG_CUDA(cudaMemsetAsync(ws.lb_ticket.p, 0, 3 * sizeof(uint32_t), s));
  }
  if (ws.gdeg.n < 2 * (size_t)V || !ws.gdeg.p) {        // whole-graph degree deltas: zero between steps
    STG_TRY(ws.gdeg.alloc(2 * (size_t)(V > 0 ? V : 1), s));
    STG_CUDA(cudaMemsetAsync(ws.gdeg.p, 0, sizeof(int32_t) * ws.gdeg.n, s));
  }
  return STG_OK;
}

// node_ids + schedule of one direction whose key histogram is already in ws.ids_hist
static stg_status ids_sched_from_hist(const int32_t* deg, const int32_t* rowptr, int32_t V, int32_t R, int32_t* ids,
                                      int32_t* sched, int64_t cap, BuildWs& ws, cudaStream_t s, int32_t rb,
                                      int32_t re, const DirDelta* clear, int nb, int4* touch,
                                      const DirDelta* gclear = nullptr, int self_dir = 0) {
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
                                                                ws.sat_tmp.p, ws.ids_tot.p + kIdsBuckets);
  const int64_t icap = sched_items_cap(V, cap);
  const int64_t nclr = std::max<int64_t>(clear ? clear->nadd + clear->ndel : 0, gclear ? gclear->nadd + gclear->ndel : 0);
  k_items2<<<grid_n(std::max<int64_t>(std::min<int64_t>(icap, (int64_t)R + cap / kHubChunk + 2), nclr)), 256, 0, s>>>(
      ids, rowptr, icap, sched, ws.ids_tot.p + kIdsBuckets, clear ? clear->add : nullptr, clear ? clear->nadd : 0,
      clear ? clear->del : nullptr, clear ? clear->ndel : 0, nb, touch, gclear ? gclear->add : nullptr,
      gclear ? gclear->nadd : 0, gclear ? gclear->del : nullptr, gclear ? gclear->ndel : 0,
      gclear && self_dir != 1 ? ws.gdeg.p : nullptr, gclear && self_dir != 2 ? ws.gdeg.p + V : nullptr);
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
                      int32_t* eid_new, const int32_t* in_rowptr_new, const int32_t* in_col_new,
                      const GDegStep* gdeg) {
  const int32_t V = src.V;
  STG_TRY(ids_ws_reserve(ws, V, dst.cap, s));
  const int32_t ntiles = (int32_t)ceil_div(V, kRowTile);
  if (gdeg && !norms) return fail(STG_ERR_STATE, "apply_dir2: the degree step rides on the norms pass");
  const int64_t ng = gdeg ? gdeg->keys.nadd + gdeg->keys.ndel : 0;
  const int64_t nk = d.nadd + d.ndel;
  // unsharded: this direction's new degrees are the whole graph's (in- or out-degrees)
  const int self_dir = dst.sharded ? 0 : (in_dir ? 1 : 2);
  const int32_t ntm = (int32_t)(src.E >> kMergeShift) + 1;    // merge tiles: positions [0, E_old]
  STG_TRY(ws.mpos.alloc((size_t)std::max<int64_t>(nk, 1), s));
  STG_TRY(ws.mbnd.alloc(2 * ((size_t)ntm + 1), s));
  const int32_t* orowptr = in_dir ? src.in_rowptr.p : src.out_rowptr.p;
  const int32_t* ocol = in_dir ? src.in_col.p : src.out_col.p;
  {                                                      // touch marks, merge positions, (whole-graph degrees)
    TouchArgs t{};
    t.add = d.add; t.nadd = d.nadd; t.del = d.del; t.ndel = d.ndel; t.nb = src.nb;
    t.touch = touch; t.orowptr = orowptr; t.ocol = ocol;
    t.padd = ws.mpos.p; t.pdel = ws.mpos.p + d.nadd;
    if (ng > 0) {
      t.gadd = gdeg->keys.add; t.ngadd = gdeg->keys.nadd; t.gdel = gdeg->keys.del; t.ngdel = gdeg->keys.ndel;
      t.sign = gdeg->sign;
      t.din = self_dir == 1 ? nullptr : ws.gdeg.p;
      t.dout = self_dir == 2 ? nullptr : ws.gdeg.p + V;
    }
    k_touch3<<<grid_n(std::max<int64_t>(std::max<int64_t>(nk, ng), 1)), 256, 0, s>>>(t);
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
  if (norms) {
    a.gin = dst.gin_deg.p; a.gout = dst.gout_deg.p; a.dgl_both = dst.dgl_both;
    a.norm_src = dst.norm_src.p; a.norm_dst = dst.norm_dst.p;
    if (gdeg) {                                          // dst's degrees = src's + this step's deltas
      a.gin = gdeg->gin_src; a.gout = gdeg->gout_src;
      a.din = self_dir == 1 ? nullptr : ws.gdeg.p;
      a.dout = self_dir == 2 ? nullptr : ws.gdeg.p + V;
      a.self_dir = self_dir;
      a.gin_w = gdeg->gin_dst; a.gout_w = gdeg->gout_dst;
    }
  }
  a.padd = ws.mpos.p; a.nadd = d.nadd; a.pdel = ws.mpos.p + d.nadd; a.ndel = d.ndel;
  a.abnd = ws.mbnd.p; a.dbnd = ws.mbnd.p + ntm + 1; a.ntm = ntm;
  k_rowscan<true><<<ntiles, kRowThreads, 0, s>>>(a);
  count_launch();
  MergeArgs m{};
  m.nb = src.nb;
  m.ocol = ocol;
  m.E_old = src.E;
  m.add = d.add;
  m.padd = ws.mpos.p; m.pdel = ws.mpos.p + d.nadd;
  m.abnd = ws.mbnd.p; m.dbnd = ws.mbnd.p + ntm + 1;
  m.ncol = in_dir ? dst.in_col.p : dst.out_col.p;
  m.emap_out = emap_out; m.emap_in = emap_in; m.eid_old = eid_old; m.eid_new = eid_new;
  m.in_rowptr_new = in_rowptr_new; m.in_col_new = in_col_new;
  if (m.eid_new) k_merge4<true><<<(unsigned)ceil_div(ntm, 8), 256, 0, s>>>(m, ntm);
  else k_merge4<false><<<(unsigned)ceil_div(ntm, 8), 256, 0, s>>>(m, ntm);
  count_launch();
  const int32_t R = blk ? dst.rows() : V;
  return ids_sched_from_hist(a.deg_new, a.rowptr_new, V, R, in_dir ? dst.in_ids.p : dst.out_ids.p,
                             in_dir ? dst.in_sched.p : dst.out_sched.p, dst.cap, ws, s, a.rb, a.re, &d, src.nb,
                             touch, gdeg ? &gdeg->keys : nullptr, self_dir);
}

}  // namespace stg
