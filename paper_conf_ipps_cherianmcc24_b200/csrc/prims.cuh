// prims.cuh — device primitives for the snapshot builders (hand-written, no CUB):
//   * exclusive scan with fused input/output functors (reduce-then-scan),
//   * stable LSD radix sort of (key[,value]) with warp match_any ranking,
//   * predicate compaction via the scan.
// All are deterministic; all run on the caller's stream with no host sync.
#pragma once

#include "common.cuh"

namespace stg {

struct ScanWs {
  DArray<int64_t> tiles;
};
struct RadixWs {
  DArray<int32_t> counts;
  DArray<int64_t> offsets;
  ScanWs scan;
};
struct BuildWs {
  RadixWs radix;
  ScanWs scan;
  DArray<uint64_t> kalt;
  DArray<uint32_t> dkey, dkey_alt;
  DArray<int32_t> dval, dval_alt;
  DArray<int64_t> count;
  DArray<int32_t> emap;        // delta apply: old in-CSR position -> new position (-1 = deleted)
  // node_ids counting sort and the single-pass row scan (snapshot.cu)
  DArray<int32_t> ids_hist, ids_offs, ids_tot, sat_tmp;
  DArray<int32_t> mpos;        // old-CSR positions of one step's adds | deletes (merge path)
  DArray<int32_t> mbnd;        // per merge tile: first add | first delete placed in it
  DArray<int32_t> rows;        // COO row ids of one direction (transposes / labels only)
  DArray<uint64_t> lb_status;  // decoupled look-back words, one per row tile
  DArray<uint32_t> lb_ticket;  // [tile claims, finished tiles, generation] of the row scan (self-resetting)
  DArray<int32_t> gdeg;        // [2V] whole-graph degree deltas of one step (zero between steps)
};

namespace {

constexpr int kScanThreads = 256;
constexpr int kScanIPT = 8;
constexpr int kScanTile = kScanThreads * kScanIPT;  // 2048 items per tile

__device__ __forceinline__ int64_t warp_incl_scan(int64_t v) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int64_t t = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += t;
  }
  return v;
}

// Block-wide exclusive scan of one value per thread (blockDim.x == kScanThreads).
__device__ __forceinline__ int64_t block_excl_scan(int64_t v, int64_t* sh /*[32]*/, int64_t* total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int64_t inc = warp_incl_scan(v);
  if (lane == 31) sh[w] = inc;
  __syncthreads();
  if (w == 0) {
    int64_t s = lane < (kScanThreads / 32) ? sh[lane] : 0;
    s = warp_incl_scan(s);
    sh[lane] = s;
  }
  __syncthreads();
  int64_t wpre = w ? sh[w - 1] : 0;
  if (total) *total = sh[kScanThreads / 32 - 1];
  return wpre + inc - v;
}

template <class In>
__global__ void __launch_bounds__(kScanThreads) k_scan_tile_sums(In in, int64_t n, int64_t* tile_sums) {
  __shared__ int64_t sh[32];
  const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanIPT;
  int64_t s = 0;
#pragma unroll
  for (int k = 0; k < kScanIPT; ++k)
    if (base + k < n) s += (int64_t)in(base + k);
  int64_t tot;
  block_excl_scan(s, sh, &tot);
  if (threadIdx.x == 0) tile_sums[blockIdx.x] = tot;
}

// One block: exclusive scan of the tile sums in place; grand total to *total64 / *total32.
__global__ void __launch_bounds__(kScanThreads) k_scan_tiles(int64_t* tile_sums, int64_t ntiles,
                                                             int64_t* total64, int32_t* total32) {
  __shared__ int64_t sh[32];
  int64_t carry = 0;
  for (int64_t b = 0; b < ntiles; b += kScanThreads) {
    int64_t i = b + threadIdx.x;
    int64_t v = i < ntiles ? tile_sums[i] : 0;
    int64_t tot;
    int64_t ex = block_excl_scan(v, sh, &tot);
    if (i < ntiles) tile_sums[i] = carry + ex;
    carry += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    if (total64) *total64 = carry;
    if (total32) *total32 = (int32_t)carry;
  }
}

template <class In, class Out>
__global__ void __launch_bounds__(kScanThreads) k_scan_apply(In in, int64_t n, const int64_t* tile_off, Out out) {
  __shared__ int64_t sh[32];
  const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanIPT;
  int64_t v[kScanIPT];
  int64_t s = 0;
#pragma unroll
  for (int k = 0; k < kScanIPT; ++k) {
    v[k] = base + k < n ? (int64_t)in(base + k) : 0;
    s += v[k];
  }
  int64_t ex = block_excl_scan(s, sh, nullptr) + tile_off[blockIdx.x];
#pragma unroll
  for (int k = 0; k < kScanIPT; ++k) {
    if (base + k < n) out(base + k, ex, v[k]);
    ex += v[k];
  }
}


// Exclusive scan: out(i, prefix_before_i, value_i) for every i in [0,n);
// grand total written to *total64 / *total32 (device, optional).
template <class In, class Out>
stg_status scan(In in, Out out, int64_t n, ScanWs& ws, cudaStream_t s, int64_t* total64 = nullptr,
                int32_t* total32 = nullptr) {
  int64_t ntiles = n > 0 ? ceil_div(n, kScanTile) : 0;
  STG_TRY(ws.tiles.alloc(ntiles + 1, s));
  if (ntiles) {
    k_scan_tile_sums<<<(unsigned)ntiles, kScanThreads, 0, s>>>(in, n, ws.tiles.p);
    count_launch();
  }
  k_scan_tiles<<<1, kScanThreads, 0, s>>>(ws.tiles.p, ntiles, total64, total32);
  count_launch();
  if (ntiles) {
    k_scan_apply<<<(unsigned)ntiles, kScanThreads, 0, s>>>(in, n, ws.tiles.p, out);
    count_launch();
  }
  return check_launch("scan");
}

// ------------------------------------------------------------- radix sort
constexpr int kRadixThreads = 256;
constexpr int kRadixWarps = kRadixThreads / 32;
constexpr int kRadixIPT = 8;                                 // items per lane
constexpr int kRadixWarpItems = 32 * kRadixIPT;              // 512
constexpr int kRadixTile = kRadixWarpItems * kRadixWarps;    // 4096
constexpr int kRadixBits = 8;
constexpr int kRadixDigits = 1 << kRadixBits;

template <class K>
__global__ void __launch_bounds__(kRadixThreads) k_radix_hist(const K* __restrict__ keys, int64_t n, int shift,
                                                              int32_t* __restrict__ counts, int64_t ntiles) {
  __shared__ int32_t h[kRadixDigits];
  for (int d = threadIdx.x; d < kRadixDigits; d += kRadixThreads) h[d] = 0;
  __syncthreads();
  const int64_t base = (int64_t)blockIdx.x * kRadixTile;
  const int lane = threadIdx.x & 31;
  // warp-aggregated: one shared atomic per distinct digit per warp (skewed keys such
  // as vertex degrees would otherwise serialise on a few counters)
  for (int k = threadIdx.x; k < kRadixTile; k += kRadixThreads) {
    const int64_t i = base + k;
    const int d = i < n ? (int)((keys[i] >> shift) & (kRadixDigits - 1)) : kRadixDigits + lane;
    const unsigned peers = __match_any_sync(0xffffffffu, d);
    if (d < kRadixDigits && (peers & ((1u << lane) - 1u)) == 0) atomicAdd(&h[d], __popc(peers));
  }
  __syncthreads();
  for (int d = threadIdx.x; d < kRadixDigits; d += kRadixThreads) counts[(int64_t)d * ntiles + blockIdx.x] = h[d];
}

// Stable scatter: items of tile b, warp w, round r, lane l are in input order
// (b, w, r, l); ranks within a warp come from match_any over the digit.
template <class K, class V, bool HAS_V>
__global__ void __launch_bounds__(kRadixThreads) k_radix_scatter(const K* __restrict__ kin, K* __restrict__ kout,
                                                                 const V* __restrict__ vin, V* __restrict__ vout,
                                                                 int64_t n, int shift,
                                                                 const int64_t* __restrict__ offsets, int64_t ntiles) {
  __shared__ int32_t wcnt[kRadixWarps][kRadixDigits];
  __shared__ int64_t toff[kRadixDigits];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int d = lane; d < kRadixDigits; d += 32) wcnt[w][d] = 0;
  for (int d = threadIdx.x; d < kRadixDigits; d += kRadixThreads)
    toff[d] = offsets[(int64_t)d * ntiles + blockIdx.x];
  __syncwarp();
  const int64_t base = (int64_t)blockIdx.x * kRadixTile + (int64_t)w * kRadixWarpItems;
  K key[kRadixIPT];
  int rank[kRadixIPT];
  const unsigned lt = (1u << lane) - 1u;
#pragma unroll
  for (int r = 0; r < kRadixIPT; ++r) {
    int64_t i = base + r * 32 + lane;
    bool ok = i < n;
    key[r] = ok ? kin[i] : K(0);
    int d = ok ? (int)((key[r] >> shift) & (kRadixDigits - 1)) : (kRadixDigits + lane);
    unsigned peers = __match_any_sync(0xffffffffu, d);
    int before = ok ? wcnt[w][d] : 0;
    rank[r] = before + __popc(peers & lt);
    __syncwarp();
    if (ok && (peers & lt) == 0) wcnt[w][d] = before + __popc(peers);
    __syncwarp();
  }
  __syncthreads();
  // exclusive prefix over warps, per digit
  for (int d = threadIdx.x; d < kRadixDigits; d += kRadixThreads) {
    int32_t run = 0;
#pragma unroll
    for (int ww = 0; ww < kRadixWarps; ++ww) {
      int32_t c = wcnt[ww][d];
      wcnt[ww][d] = run;
      run += c;
    }
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < kRadixIPT; ++r) {
    int64_t i = base + r * 32 + lane;
    if (i < n) {
      int d = (int)((key[r] >> shift) & (kRadixDigits - 1));
      int64_t pos = toff[d] + wcnt[w][d] + rank[r];
      kout[pos] = key[r];
      if (HAS_V) vout[pos] = vin[i];
    }
  }
}

struct CountsIn {
  const int32_t* c;
  __device__ int64_t operator()(int64_t i) const { return c[i]; }
};
struct StoreExcl64 {
  int64_t* o;
  __device__ void operator()(int64_t i, int64_t ex, int64_t) const { o[i] = ex; }
};


// Stable LSD radix sort of keys[0..n) on bits [begin_bit, end_bit), carrying
// values if vals != nullptr.  Ping-pongs between (keys, keys_alt) and
// (vals, vals_alt); on return the sorted data is in *keys / *vals (pointers
// swapped as needed).
template <class K, class V>
stg_status radix_sort(K** keys, K** keys_alt, V** vals, V** vals_alt, int64_t n, int begin_bit, int end_bit,
                      RadixWs& ws, cudaStream_t s) {
  if (n <= 1 || end_bit <= begin_bit) return STG_OK;
  const int64_t ntiles = ceil_div(n, kRadixTile);
  STG_TRY(ws.counts.alloc((size_t)ntiles * kRadixDigits, s));
  STG_TRY(ws.offsets.alloc((size_t)ntiles * kRadixDigits, s));
  const bool has_v = vals != nullptr && *vals != nullptr;
  for (int shift = begin_bit; shift < end_bit; shift += kRadixBits) {
    k_radix_hist<K><<<(unsigned)ntiles, kRadixThreads, 0, s>>>(*keys, n, shift, ws.counts.p, ntiles);
    count_launch();
    STG_TRY(scan(CountsIn{ws.counts.p}, StoreExcl64{ws.offsets.p}, ntiles * kRadixDigits, ws.scan, s));
    if (has_v) {
      k_radix_scatter<K, V, true><<<(unsigned)ntiles, kRadixThreads, 0, s>>>(*keys, *keys_alt, *vals, *vals_alt, n,
                                                                              shift, ws.offsets.p, ntiles);
      std::swap(*vals, *vals_alt);
    } else {
      k_radix_scatter<K, V, false><<<(unsigned)ntiles, kRadixThreads, 0, s>>>(*keys, *keys_alt, nullptr, nullptr,
                                                                               n, shift, ws.offsets.p, ntiles);
    }
    count_launch();
    std::swap(*keys, *keys_alt);
  }
  return check_launch("radix_sort");
}

inline int bits_for(int64_t maxval) {  // bits to represent values in [0, maxval]
  int b = 1;
  while (b < 62 && (int64_t(1) << b) <= maxval) ++b;
  return b;
}

}  // namespace
}  // namespace stg
