// graph.cuh — device-resident snapshot (the STGraphBase arrays)
// and the builders shared by static graphs and DTDG snapshots.
#pragma once

#include <algorithm>
#include <memory>
#include <mutex>
#include <vector>

#include "common.cuh"

namespace stg {

// Rows with more than kHubChunk in-edges are split into chunks of kHubChunk
// edges (degree-bucketed schedule); each light row / hub chunk is
// one work item of the aggregation kernel.  64 keeps every fp32 accumulator
// chain <= 64 terms with a single accumulator.
constexpr int32_t kHubChunk = 64;

// upper bound on the number of hub rows (deg > kHubChunk) of an E-edge graph
inline int64_t sched_cap(int64_t E) { return E / (kHubChunk + 1) + 2; }

// Degree-bucketed schedule of one CSR direction (int32 array `sched`):
//   sched[0] = n_hub    rows with deg > kHubChunk (the prefix ids[0, n_hub))
//   sched[1] = n_chunks total hub chunks
//   sched[2] = cptr_off offset (in int32) of cptr[0..n_hub] (exclusive chunk prefix)
//   sched[3] = n_items  = n_chunks + V - n_hub
//   sched[4] = first item of the light rows with n <= kTierB (items are in degree order)
//   sched[5] = first item of the light rows with n <= kTierC
//   sched[6] = m        rows of the saturated node_ids prefix (degree >= 1023, snapshot.cu)
//   sched[7] = their hub chunks (cptr[m]); build-time only (items stay 16-byte aligned)
//   sched[8 ..]         = items, int4 {v, beg, n, hub} in node_ids order: hub
//                         chunks first (hub = index into ids / cptr), then the
//                         light rows (hub = -1).  n <= kHubChunk.
constexpr int64_t kSchedHdr = 8;
// light-row tiers of the edge-stream work groups (aggregate.cu): rows with more edges go
// in smaller groups so that no warp walks a long group of the heaviest light rows
constexpr int32_t kTierB = 16, kTierC = 4;
inline int64_t sched_items_cap(int64_t V, int64_t E) { return V + E / kHubChunk + 2; }
inline int64_t sched_cptr_off(int64_t V, int64_t E) { return kSchedHdr + 4 * sched_items_cap(V, E); }
inline int64_t sched_size(int64_t V, int64_t E) {
  return sched_cptr_off(V, E) + std::min<int64_t>(V, sched_cap(E)) + 2;
}

// Aggregation scratch owned by a graph / dtdg object: hub-chunk partial sums
// and per-hub-row completion counters (self-resetting, zero between calls).
// The aggregation kernels' host launcher (aggregate.cu); `peers` != NULL is the
// sharded-mode gather from the owners' row blocks (stg_gcn_aggregate_peer).
stg_status aggregate_launch(const stg_csr_view* gv, int backward, int32_t W, const float* in, int64_t ldin,
                            float* out, int64_t ldout, const float* srow, const float* scol, const float* bias,
                            cudaStream_t s, const stg_peer_rows* peers = nullptr, const float* ew = nullptr);

struct AggScratch {
  DArray<float> partials;
  DArray<int32_t> counters;
  int64_t counters_n = 0;
  DArray<uint32_t> queue;        // edge-stream work-queue heads, one per column chunk (reset per launch)
};
// One scratch area per stream that has aggregated over the object: calls on
// different streams never share a work queue, partials or counters (each call
// is ordered only on its own stream, include/stg.h).
struct AggWs {
  std::mutex mu;
  std::vector<std::pair<cudaStream_t, std::unique_ptr<AggScratch>>> per;
  AggScratch* get(cudaStream_t s) {
    std::lock_guard<std::mutex> lk(mu);
    for (auto& e : per)
      if (e.first == s) return e.second.get();
    per.emplace_back(s, std::make_unique<AggScratch>());
    return per.back().second.get();
  }
};

// Row-block sharding: a sharded snapshot holds only the edges
// whose destination lies in [rb, re).  Its CSRs keep global vertex numbering
// (in-CSR rows outside the block are empty; the out-CSR has all V rows), its
// in_ids list the local rows first, and the GCN norms come from the degrees
// of the WHOLE graph (gin_deg / gout_deg), maintained from the global deltas.
// Parts of a snapshot (a DTDG builds only the direction a pass needs: the
// forward in-CSR for Get-Graph, the reverse out-CSR for Get-Backward-Graph,
// the other one by a transpose when asked for, Algorithm 3).
enum : uint32_t { PART_IN = 1u, PART_OUT = 2u, PART_EID = 4u, PART_ALL = 7u };

struct Snapshot {
  int32_t V = 0, nb = 1;   // nb: bits per id in packed keys
  int32_t t = -1;
  int32_t rb = 0, re = 0;  // local destination rows [rb, re) (whole graph: [0, V))
  int64_t E = 0, cap = 0;  // current (local) edges, edge capacity
  bool edge_ids = false, dgl_both = false, sharded = false;
  uint32_t parts = 0;      // valid parts (PART_*); degrees and norms are always valid
  DArray<int32_t> in_rowptr, in_col, in_deg, in_ids;
  DArray<int32_t> out_rowptr, out_col, out_deg, out_ids, out_eid;
  DArray<int32_t> in_sched, out_sched;  // [sched_size(V, cap)], layout above
  DArray<int32_t> gin_deg, gout_deg;    // whole-graph degrees (the norms' source; maintained per step)
  DArray<float> norm_src, norm_dst;

  stg_status alloc(int32_t V_, int64_t cap_, bool eids, bool dgl, int32_t rb_ = 0, int32_t re_ = -1);
  int32_t rows() const { return re - rb; }
  size_t bytes() const;   // device bytes held
  void view(stg_csr_view* v, AggWs* ws) const;
};

// Shared builder scratch (radix sort / scan buffers), grow-only.
struct BuildWs;
BuildWs* buildws_create();
void buildws_destroy(BuildWs*);

// whole-graph degree histograms of packed (src << nb | dst) keys (sign = +1 / -1),
// added into gin (by dst) and gout (by src; may be NULL)
void degree_hist(const uint64_t* keys, int64_t n, int nb, int sign, int32_t* gin, int32_t* gout, cudaStream_t s);
// compact the packed keys whose destination (low nb bits if dst_low, else high) lies in [rb, re);
// the count is written to *d_count (device)
stg_status filter_block(const uint64_t* keys, int64_t n, int nb, bool dst_low, int32_t rb, int32_t re,
                        uint64_t* out, int64_t* d_count, BuildWs& ws, cudaStream_t s);


// Build every array of `out` from the sorted unique packed out-keys
// (src << nb | dst) of the snapshot edge set.  No host synchronisation.
stg_status build_from_out_keys(const uint64_t* keys, int64_t E, Snapshot& out, BuildWs& ws, cudaStream_t s);

// Sort + unique packed keys in place.  keys/alt hold n entries; on return
// *keys points to the sorted unique keys; the unique count is written to
// *d_count (device).  Does not synchronise.
stg_status sort_unique_keys(uint64_t** keys, uint64_t** alt, int64_t n, int nbits, int64_t* d_count,
                            BuildWs& ws, cudaStream_t s);

// Recompute degrees' dependents: node_ids and the hub schedules of the
// directions in `parts`.  Needs the deg arrays and rowptrs of those parts.
stg_status build_ids_and_sched(Snapshot& g, BuildWs& ws, cudaStream_t s, uint32_t parts = PART_IN | PART_OUT);
stg_status build_out_eid(Snapshot& g, BuildWs& ws, cudaStream_t s);
// GCN norms from the whole-graph degrees gin_deg / gout_deg (reading C1)
void build_norms(Snapshot& g, cudaStream_t s);
// Complete the missing CSR direction(s) of `g` from the one it has by a stable
// transpose (Algorithm 3, with the canonical order of reading C7),
// plus node_ids, schedule and (edge_ids) the shared labels.  want: PART_* mask.
stg_status complete_parts(Snapshot& g, uint32_t want, BuildWs& ws, cudaStream_t s);

// Delta application (DTDG Get-Graph / Get-Backward-Graph step).  For one
// direction: the sorted packed deltas (row << nb | col) of that direction.
struct DirDelta {
  const uint64_t* add;
  int64_t nadd;
  const uint64_t* del;
  int64_t ndel;
};
// snapshot.cu: node_ids (degree desc, id asc) and the schedule of one CSR
// direction by a counting sort (rows outside [rb, re) sort last; R = rows in it)
stg_status ids_sched_build(const int32_t* deg, const int32_t* rowptr, int32_t V, int32_t R, int32_t rb, int32_t re,
                           int32_t* ids, int32_t* sched, int64_t cap, BuildWs& ws, cudaStream_t s);
// whole-graph degree histogram of one delta batch (adds +sign, deletes -sign)
stg_status degree_hist2(const DirDelta& d, int nb, int sign, int32_t* gin, int32_t* gout, cudaStream_t s);
// whole-graph degree update of one delta step, fused into the first direction's pass:
// dst's gin / gout = src's + the ±1 histogram of the whole-graph (src << nb | dst) keys
struct GDegStep {
  DirDelta keys;                 // whole-graph effective deltas (add = +sign, del = -sign)
  int sign;
  const int32_t* gin_src;
  const int32_t* gout_src;
  int32_t* gin_dst;
  int32_t* gout_dst;
};
// one delta step of one CSR direction of src into dst (rowptr, col, degrees,
// node_ids, schedule; the GCN norms too if `norms`); labels as in apply_delta
stg_status apply_dir2(const Snapshot& src, Snapshot& dst, bool in_dir, const DirDelta& d, int4* touch, BuildWs& ws,
                      cudaStream_t s, bool norms, int32_t* emap_out, const int32_t* emap_in, const int32_t* eid_old,
                      int32_t* eid_new, const int32_t* in_rowptr_new, const int32_t* in_col_new,
                      const GDegStep* gdeg = nullptr);

// Applies the delta to the directions in `parts` (src must hold them; labels
// are carried when both directions and src's labels are present).  The caller
// has already updated dst's whole-graph degrees (gin_deg / gout_deg).
stg_status apply_delta(const Snapshot& src, Snapshot& dst, const DirDelta& in_dir, const DirDelta& out_dir,
                       int64_t E_new, int32_t t_new, int4* touch_in, int4* touch_out, BuildWs& ws,
                       cudaStream_t s, uint32_t parts = PART_ALL, const GDegStep* gdeg = nullptr);

}  // namespace stg

// Opaque objects of the C ABI.
struct stg_graph {
  stg::Snapshot snap;
  stg::AggWs ws;
};
