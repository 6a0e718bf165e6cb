// graph.cu — snapshot builders (static graph create, CSR pair, node_ids, edge
// labels, hub schedule) and the DTDG delta-apply step.  Hand-written sm_100a
// kernels; the paper's Thrust/CUB routines and Algorithm 3's atomic
// transpose are replaced by sort/merge constructions that give
// the canonical (ascending-neighbour) order deterministically (reading C3/C7).
#include "graph.cuh"
#include "prims.cuh"

namespace stg {

BuildWs* buildws_create() { return new BuildWs(); }
void buildws_destroy(BuildWs* w) { delete w; }

static inline unsigned grid_for(int64_t n, int threads, int64_t max_blocks = 148 * 16) {
  int64_t b = ceil_div(n > 0 ? n : 1, threads);
  return (unsigned)(b < max_blocks ? b : max_blocks);
}

stg_status Snapshot::alloc(int32_t V_, int64_t cap_, bool eids, bool dgl, int32_t rb_, int32_t re_) {
  V = V_;
  rb = rb_;
  re = re_ < 0 ? V_ : re_;
  sharded = rb != 0 || re != V;
  cap = cap_ > 0 ? cap_ : 1;
  nb = 1;
  while ((int64_t(1) << nb) < (int64_t)V) ++nb;
  edge_ids = eids;
  dgl_both = dgl;
  const int64_t sc = sched_size(V, cap);
  STG_TRY(in_rowptr.alloc(V + 1)); STG_TRY(out_rowptr.alloc(V + 1));
  STG_TRY(in_col.alloc(cap));
  STG_TRY(out_col.alloc(cap));
  if (eids) STG_TRY(out_eid.alloc(cap));
  STG_TRY(in_deg.alloc(V)); STG_TRY(out_deg.alloc(V));
  STG_TRY(in_ids.alloc(V)); STG_TRY(out_ids.alloc(V));
  STG_TRY(in_sched.alloc(sc)); STG_TRY(out_sched.alloc(sc));
  STG_TRY(norm_src.alloc(V)); STG_TRY(norm_dst.alloc(V));
  STG_TRY(gin_deg.alloc(V)); STG_TRY(gout_deg.alloc(V));
  parts = 0;
  return STG_OK;
}

size_t Snapshot::bytes() const {
  const DArray<int32_t>* ia[] = {&in_rowptr, &in_col, &in_deg, &in_ids, &out_rowptr, &out_col,
                                 &out_deg, &out_ids, &out_eid, &in_sched, &out_sched, &gin_deg, &gout_deg};
  size_t b = 0;
  for (const auto* a : ia) b += a->n * sizeof(int32_t);
  return b + (norm_src.n + norm_dst.n) * sizeof(float);
}

void Snapshot::view(stg_csr_view* v, AggWs* ws) const {
  v->num_nodes = V;
  v->row_begin = rb;
  v->row_end = re;
  v->timestamp = t;
  v->num_edges = E;
  // rows below rb are empty, so in_rowptr[rb] = 0: the local row pointer is a suffix.
  // Parts this snapshot does not hold are NULL.
  const bool hi = (parts & PART_IN) != 0, ho = (parts & PART_OUT) != 0;
  v->in_rowptr = hi ? in_rowptr.p + rb : nullptr; v->in_col = hi ? in_col.p : nullptr;
  v->out_rowptr = ho ? out_rowptr.p : nullptr; v->out_col = ho ? out_col.p : nullptr;
  v->out_eid = (edge_ids && (parts & PART_EID)) ? out_eid.p : nullptr;
  // degrees: whole-graph (always current) unless sharded, where they describe the held edges
  v->in_deg = sharded ? (hi ? in_deg.p : nullptr) : gin_deg.p;
  v->out_deg = sharded ? (ho ? out_deg.p : nullptr) : gout_deg.p;
  v->in_ids = hi ? in_ids.p : nullptr; v->out_ids = ho ? out_ids.p : nullptr;
  v->norm_src = norm_src.p; v->norm_dst = norm_dst.p;
  v->in_sched = hi ? in_sched.p : nullptr; v->out_sched = ho ? out_sched.p : nullptr;
  v->workspace = ws;
}

// ------------------------------------------------------------------ kernels
__global__ void k_unpack(const uint64_t* __restrict__ keys, int64_t E, int nb, int32_t* __restrict__ row,
                         int32_t* __restrict__ col) {
  const uint64_t mask = (uint64_t(1) << nb) - 1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < E; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t k = keys[i];
    row[i] = (int32_t)(k >> nb);
    col[i] = (int32_t)(k & mask);
  }
}

__global__ void k_swap_keys(const uint64_t* __restrict__ in, int64_t E, int nb, uint64_t* __restrict__ out) {
  const uint64_t mask = (uint64_t(1) << nb) - 1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < E; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t k = in[i];
    out[i] = ((k & mask) << nb) | (k >> nb);
  }
}

// rowptr of a row-sorted COO: rowptr[v] = first index with row >= v.
__global__ void k_rowptr(const int32_t* __restrict__ rows, int64_t E, int32_t V, int32_t* __restrict__ rowptr) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= E; i += (int64_t)gridDim.x * blockDim.x) {
    int32_t prev = i == 0 ? -1 : rows[i - 1];
    int32_t cur = i == E ? V : rows[i];
    for (int32_t v = prev + 1; v <= cur; ++v) rowptr[v] = (int32_t)i;
  }
}

__global__ void k_deg(const int32_t* __restrict__ rowptr, int32_t V, int32_t* __restrict__ deg) {
  for (int32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x)
    deg[v] = rowptr[v + 1] - rowptr[v];
}

// COO row ids of a CSR: rows[j] = r for rowptr[r] <= j < rowptr[r+1]: a thread per
// row, rows of more than 32 edges written by the whole warp
__global__ void k_expand_rows(const int32_t* __restrict__ rowptr, int32_t V, int32_t* __restrict__ rows) {
  const int lane = threadIdx.x & 31;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x + threadIdx.x - lane; base < V; base += stride) {
    const int64_t r = base + lane;
    int32_t b = 0, e = 0;
    if (r < V) { b = rowptr[r]; e = rowptr[r + 1]; }
    const bool big = e - b > 32;
    if (!big)
      for (int32_t j = b; j < e; ++j) rows[j] = (int32_t)r;
    for (unsigned m = __ballot_sync(0xffffffffu, big); m; m &= m - 1) {
      const int src = __ffs(m) - 1;
      const int32_t bb = __shfl_sync(0xffffffffu, b, src), ee = __shfl_sync(0xffffffffu, e, src);
      for (int32_t j = bb + lane; j < ee; j += 32) rows[j] = (int32_t)(base + src);
    }
  }
}

// GCN normalisation vectors (reading C1): IEEE 1/sqrtf, 0 for degree 0.
// A sharded snapshot passes the whole-graph degrees (gin_deg / gout_deg).
__global__ void k_norm(const int32_t* __restrict__ in_deg, const int32_t* __restrict__ out_deg, int32_t V,
                       int dgl_both, float* __restrict__ n_src, float* __restrict__ n_dst) {
  for (int32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x) {
    int32_t di = in_deg[v];
    float nd = di > 0 ? 1.0f / sqrtf((float)di) : 0.0f;
    n_dst[v] = nd;
    if (dgl_both) {
      int32_t d = out_deg[v];
      n_src[v] = d > 0 ? 1.0f / sqrtf((float)d) : 0.0f;
    } else {
      n_src[v] = nd;
    }
  }
}

// shared edge labels: out_eid[j] = in-CSR position of out-edge j = (u -> v)
__global__ void k_out_eid(const int32_t* __restrict__ out_row, const int32_t* __restrict__ out_col, int64_t E,
                          const int32_t* __restrict__ in_rowptr, const int32_t* __restrict__ in_col,
                          int32_t* __restrict__ out_eid) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < E; j += (int64_t)gridDim.x * blockDim.x) {
    int32_t u = out_row[j], v = out_col[j];
    int32_t lo = in_rowptr[v], hi = in_rowptr[v + 1];
    while (lo < hi) {
      int32_t mid = (lo + hi) >> 1;
      if (in_col[mid] < u) lo = mid + 1; else hi = mid;
    }
    out_eid[j] = lo;
  }
}

struct UniqIn {
  const uint64_t* k;
  __device__ int64_t operator()(int64_t i) const { return i == 0 || k[i] != k[i - 1]; }
};
struct UniqOut {
  const uint64_t* k;
  uint64_t* o;
  __device__ void operator()(int64_t i, int64_t ex, int64_t f) const {
    if (f) o[ex] = k[i];
  }
};

// ---------------------------------------------------- row-block sharding
__global__ void k_degree_hist(const uint64_t* __restrict__ keys, int64_t n, int nb, int sign, int32_t* __restrict__ gin,
                              int32_t* __restrict__ gout) {
  const uint64_t mask = (uint64_t(1) << nb) - 1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t k = keys[i];
    atomicAdd(gin + (int32_t)(k & mask), sign);
    if (gout) atomicAdd(gout + (int32_t)(k >> nb), sign);
  }
}

void degree_hist(const uint64_t* keys, int64_t n, int nb, int sign, int32_t* gin, int32_t* gout, cudaStream_t s) {
  if (n <= 0) return;
  k_degree_hist<<<grid_for(n, 256), 256, 0, s>>>(keys, n, nb, sign, gin, gout);
  count_launch();
}

struct InBlock {
  const uint64_t* k;
  int nb;
  bool dst_low;
  int32_t rb, re;
  __device__ int64_t operator()(int64_t i) const {
    const uint64_t key = k[i];
    const int32_t d = dst_low ? (int32_t)(key & ((uint64_t(1) << nb) - 1)) : (int32_t)(key >> nb);
    return d >= rb && d < re;
  }
};

stg_status filter_block(const uint64_t* keys, int64_t n, int nb, bool dst_low, int32_t rb, int32_t re, uint64_t* out,
                        int64_t* d_count, BuildWs& ws, cudaStream_t s) {
  if (n <= 0) {
    STG_CUDA(cudaMemsetAsync(d_count, 0, sizeof(int64_t), s));
    return STG_OK;
  }
  return scan(InBlock{keys, nb, dst_low, rb, re}, UniqOut{keys, out}, n, ws.scan, s, d_count);
}

stg_status sort_unique_keys(uint64_t** keys, uint64_t** alt, int64_t n, int nbits, int64_t* d_count, BuildWs& ws,
                            cudaStream_t s) {
  uint32_t* nov = nullptr;
  STG_TRY((radix_sort<uint64_t, uint32_t>(keys, alt, nullptr, &nov, n, 0, nbits, ws.radix, s)));
  STG_TRY(scan(UniqIn{*keys}, UniqOut{*keys, *alt}, n, ws.scan, s, d_count));
  std::swap(*keys, *alt);
  return STG_OK;
}

stg_status build_ids_and_sched(Snapshot& g, BuildWs& ws, cudaStream_t s, uint32_t parts) {
  for (int dir = 0; dir < 2; ++dir) {
    if (!(parts & (dir == 0 ? PART_IN : PART_OUT))) continue;
    // rows of this direction's schedule: the local block (in-CSR) or all V sources
    const bool blk = dir == 0 && g.sharded;
    STG_TRY(ids_sched_build(dir == 0 ? g.in_deg.p : g.out_deg.p, dir == 0 ? g.in_rowptr.p : g.out_rowptr.p, g.V,
                            blk ? g.rows() : g.V, blk ? g.rb : 0, blk ? g.re : g.V, dir == 0 ? g.in_ids.p : g.out_ids.p,
                            dir == 0 ? g.in_sched.p : g.out_sched.p, g.cap, ws, s));
  }
  return check_launch("build_ids_and_sched");
}

stg_status build_out_eid(Snapshot& g, BuildWs& ws, cudaStream_t s) {
  if (!g.edge_ids || g.E <= 0) return STG_OK;
  STG_TRY(ws.rows.alloc((size_t)g.E, s));
  k_expand_rows<<<grid_for(g.V, 256), 256, 0, s>>>(g.out_rowptr.p, g.V, ws.rows.p);
  k_out_eid<<<grid_for(g.E, 256), 256, 0, s>>>(ws.rows.p, g.out_col.p, g.E, g.in_rowptr.p, g.in_col.p, g.out_eid.p);
  count_launch(2);
  return check_launch("out_eid");
}

stg_status build_from_out_keys(const uint64_t* keys, int64_t E, Snapshot& g, BuildWs& ws, cudaStream_t s) {
  const int32_t V = g.V;
  g.E = E;
  // backward CSR (rows = src): keys are already (src, dst)-sorted
  STG_TRY(ws.rows.alloc((size_t)(E > 0 ? E : 1), s));
  k_unpack<<<grid_for(E, 256), 256, 0, s>>>(keys, E, g.nb, ws.rows.p, g.out_col.p);
  k_rowptr<<<grid_for(E + 1, 256), 256, 0, s>>>(ws.rows.p, E, V, g.out_rowptr.p);
  count_launch(2);
  // forward CSR (rows = dst): re-key as (dst, src) and sort (the transpose)
  STG_TRY(ws.kalt.alloc(2 * (size_t)(E > 0 ? E : 1)));
  uint64_t* a = ws.kalt.p;
  uint64_t* b = ws.kalt.p + (E > 0 ? E : 1);
  k_swap_keys<<<grid_for(E, 256), 256, 0, s>>>(keys, E, g.nb, a);
  count_launch();
  uint32_t* nov = nullptr;
  STG_TRY((radix_sort<uint64_t, uint32_t>(&a, &b, nullptr, &nov, E, 0, 2 * g.nb, ws.radix, s)));
  k_unpack<<<grid_for(E, 256), 256, 0, s>>>(a, E, g.nb, ws.rows.p, g.in_col.p);
  k_rowptr<<<grid_for(E + 1, 256), 256, 0, s>>>(ws.rows.p, E, V, g.in_rowptr.p);
  k_deg<<<grid_for(V, 256), 256, 0, s>>>(g.in_rowptr.p, V, g.in_deg.p);
  k_deg<<<grid_for(V, 256), 256, 0, s>>>(g.out_rowptr.p, V, g.out_deg.p);
  count_launch(4);
  if (!g.sharded) {                   // whole graph: the whole-graph degrees are the row lengths
    STG_CUDA(cudaMemcpyAsync(g.gin_deg.p, g.in_deg.p, sizeof(int32_t) * V, cudaMemcpyDeviceToDevice, s));
    STG_CUDA(cudaMemcpyAsync(g.gout_deg.p, g.out_deg.p, sizeof(int32_t) * V, cudaMemcpyDeviceToDevice, s));
  }
  build_norms(g, s);
  STG_TRY(check_launch("build_from_out_keys"));
  STG_TRY(build_ids_and_sched(g, ws, s));
  g.parts = PART_IN | PART_OUT | (g.edge_ids ? PART_EID : 0u);
  return build_out_eid(g, ws, s);
}

void build_norms(Snapshot& g, cudaStream_t s) {
  k_norm<<<grid_for(g.V, 256), 256, 0, s>>>(g.gin_deg.p, g.gout_deg.p, g.V, g.dgl_both, g.norm_src.p, g.norm_dst.p);
  count_launch();
}

// ------------------------------------------------------- transpose (Alg. 3)
__global__ void k_iota(int32_t* __restrict__ a, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    a[i] = (int32_t)i;
}
// dst[i] = src[idx[i]]
__global__ void k_gather_i32(const int32_t* __restrict__ src, const int32_t* __restrict__ idx, int64_t n,
                             int32_t* __restrict__ dst) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dst[i] = __ldg(src + __ldg(idx + i));
}
// dst[idx[i]] = i
__global__ void k_scatter_pos(const int32_t* __restrict__ idx, int64_t n, int32_t* __restrict__ dst) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dst[idx[i]] = (int32_t)i;
}

// One direction from the other: a stable LSD radix sort of the edge positions
// by the other endpoint.  The source CSR is sorted by (row, col), so sorting
// its edges stably by col gives (col, row) order: the transpose in canonical
// order (reading C3/C7); the sorted positions are the shared edge labels.
stg_status complete_parts(Snapshot& g, uint32_t want, BuildWs& ws, cudaStream_t s) {
  const bool need_in = (want & PART_IN) && !(g.parts & PART_IN);
  const bool need_out = (want & PART_OUT) && !(g.parts & PART_OUT);
  const bool need_eid = g.edge_ids && (want & PART_EID) && !(g.parts & PART_EID);
  if (!need_in && !need_out && !need_eid) return STG_OK;
  if (!(g.parts & (PART_IN | PART_OUT))) return fail(STG_ERR_STATE, "snapshot holds no CSR to transpose");
  ProfScope prof(PH_SNAP_XPOSE, s);
  const int64_t E = g.E, En = E > 0 ? E : 1;
  const int32_t V = g.V;
  STG_TRY(ws.kalt.alloc(2 * (size_t)En));
  uint32_t* k1 = reinterpret_cast<uint32_t*>(ws.kalt.p);
  uint32_t* k2 = k1 + En;
  int32_t* v1 = reinterpret_cast<int32_t*>(k2 + En);
  int32_t* v2 = v1 + En;
  const bool from_in = (g.parts & PART_IN) != 0;   // transpose in -> out (else out -> in)
  const int32_t* key_src = from_in ? g.in_col.p : g.out_col.p;
  // the source direction's COO rows (the other endpoint of every edge)
  STG_TRY(ws.rows.alloc((size_t)En, s));
  int32_t* rows = ws.rows.p;
  k_expand_rows<<<grid_for(V, 256), 256, 0, s>>>(from_in ? g.in_rowptr.p : g.out_rowptr.p, V, rows);
  count_launch();
  if (E > 0) {
    STG_CUDA(cudaMemcpyAsync(k1, key_src, sizeof(int32_t) * E, cudaMemcpyDeviceToDevice, s));
    k_iota<<<grid_for(E, 256), 256, 0, s>>>(v1, E);
    count_launch();
    uint32_t* kk = k1; uint32_t* ka = k2; int32_t* vv = v1; int32_t* va = v2;
    STG_TRY((radix_sort<uint32_t, int32_t>(&kk, &ka, &vv, &va, E, 0, g.nb, ws.radix, s)));
    k1 = kk; v1 = vv;
  }
  if (from_in) {
    // out rows = sorted src (k1), out_col = in row of pos, out_eid = pos
    if (E > 0) {
      k_gather_i32<<<grid_for(E, 256), 256, 0, s>>>(rows, v1, E, g.out_col.p);
      count_launch();
      if (g.edge_ids) STG_CUDA(cudaMemcpyAsync(g.out_eid.p, v1, sizeof(int32_t) * E, cudaMemcpyDeviceToDevice, s));
    }
    k_rowptr<<<grid_for(E + 1, 256), 256, 0, s>>>(reinterpret_cast<const int32_t*>(k1), E, V, g.out_rowptr.p);
    k_deg<<<grid_for(V, 256), 256, 0, s>>>(g.out_rowptr.p, V, g.out_deg.p);
    count_launch(2);
    STG_TRY(build_ids_and_sched(g, ws, s, PART_OUT));
    g.parts |= PART_OUT | (g.edge_ids ? PART_EID : 0u);
  } else {
    // in rows = sorted dst (k1), in_col = out row of pos; out_eid[pos] = in position
    if (E > 0) {
      k_gather_i32<<<grid_for(E, 256), 256, 0, s>>>(rows, v1, E, g.in_col.p);
      count_launch();
      if (g.edge_ids) { k_scatter_pos<<<grid_for(E, 256), 256, 0, s>>>(v1, E, g.out_eid.p); count_launch(); }
    }
    k_rowptr<<<grid_for(E + 1, 256), 256, 0, s>>>(reinterpret_cast<const int32_t*>(k1), E, V, g.in_rowptr.p);
    k_deg<<<grid_for(V, 256), 256, 0, s>>>(g.in_rowptr.p, V, g.in_deg.p);
    count_launch(2);
    STG_TRY(build_ids_and_sched(g, ws, s, PART_IN));
    g.parts |= PART_IN | (g.edge_ids ? PART_EID : 0u);
  }
  return check_launch("complete_parts");
}

// -------------------------------------------------------------- delta apply
// (the per-direction kernels are in snapshot.cu)
stg_status apply_delta(const Snapshot& src, Snapshot& dst, const DirDelta& in_dir, const DirDelta& out_dir,
                       int64_t E_new, int32_t t_new, int4* touch_in, int4* touch_out, BuildWs& ws, cudaStream_t s,
                       uint32_t parts, const GDegStep* gdeg) {
  const bool do_in = (parts & PART_IN) != 0, do_out = (parts & PART_OUT) != 0;
  if ((do_in && !(src.parts & PART_IN)) || (do_out && !(src.parts & PART_OUT)))
    return fail(STG_ERR_STATE, "apply_delta: source snapshot lacks a requested direction");
  // labels are carried incrementally when both directions and the source labels are there:
  // the in-direction pass records old -> new in-CSR positions (emap), the out-direction
  // pass looks every surviving out-edge's label up through it
  const bool carry = dst.edge_ids && src.edge_ids && (src.parts & PART_EID) && do_in && do_out && src.E > 0;
  int32_t* emap = nullptr;
  if (carry) {
    STG_TRY(ws.emap.alloc((size_t)src.E, s));
    emap = ws.emap.p;
  }
  if (gdeg && !do_in && !do_out) {                  // no direction pass to carry the degree update
    const size_t vb = sizeof(int32_t) * (size_t)src.V;
    STG_CUDA(cudaMemcpyAsync(gdeg->gin_dst, gdeg->gin_src, vb, cudaMemcpyDeviceToDevice, s));
    STG_CUDA(cudaMemcpyAsync(gdeg->gout_dst, gdeg->gout_src, vb, cudaMemcpyDeviceToDevice, s));
    STG_TRY(degree_hist2(gdeg->keys, src.nb, gdeg->sign, gdeg->gin_dst, gdeg->gout_dst, s));
  }
  if (do_in)
    STG_TRY(apply_dir2(src, dst, true, in_dir, touch_in, ws, s, true, emap, nullptr, nullptr, nullptr, nullptr,
                       nullptr, gdeg));
  if (do_out)
    STG_TRY(apply_dir2(src, dst, false, out_dir, touch_out, ws, s, !do_in, nullptr, carry ? emap : nullptr,
                       carry ? src.out_eid.p : nullptr, carry ? dst.out_eid.p : nullptr,
                       carry ? dst.in_rowptr.p : nullptr, carry ? dst.in_col.p : nullptr, do_in ? nullptr : gdeg));
  dst.E = E_new;
  dst.t = t_new;
  dst.parts = (do_in ? PART_IN : 0u) | (do_out ? PART_OUT : 0u);
  if (dst.edge_ids && do_in && do_out) {
    if (!carry) STG_TRY(build_out_eid(dst, ws, s));
    dst.parts |= PART_EID;
  }
  return check_launch("apply_delta");
}

// ------------------------------------------------------------ static graph
__global__ void k_validate_pack(const int32_t* __restrict__ src, const int32_t* __restrict__ dst, int64_t E,
                                int32_t V, int nb, int loops, uint64_t* __restrict__ keys, int32_t* __restrict__ bad) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < E + (loops ? V : 0);
       i += (int64_t)gridDim.x * blockDim.x) {
    int32_t a, b;
    if (i < E) { a = src[i]; b = dst[i]; }
    else { a = b = (int32_t)(i - E); }
    if ((unsigned)a >= (unsigned)V || (unsigned)b >= (unsigned)V) { atomicExch(bad, 1); a = b = 0; }
    keys[i] = ((uint64_t)a << nb) | (uint64_t)b;
  }
}

}  // namespace stg

using namespace stg;

extern "C" {

stg_status stg_static_graph_create(int32_t V, int64_t E, const int32_t* src, const int32_t* dst, uint32_t flags,
                                   const stg_dist* dist, stg_stream_t stream, stg_graph** out) {
  if (!out) return fail(STG_ERR_INVALID_ARG, "stg_static_graph_create: out is NULL");
  *out = nullptr;
  if (V < 1 || V >= (1 << 30)) return fail(STG_ERR_OUT_OF_RANGE, "stg_static_graph_create: V=%d outside [1,2^30)", V);
  if (E < 0) return fail(STG_ERR_INVALID_ARG, "stg_static_graph_create: E < 0");
  if (E + ((flags & STG_SELF_LOOPS) ? V : 0) >= (int64_t(1) << 31))
    return fail(STG_ERR_OUT_OF_RANGE, "stg_static_graph_create: E=%lld >= 2^31", (long long)E);
  if (E > 0 && (!src || !dst)) return fail(STG_ERR_INVALID_ARG, "stg_static_graph_create: src/dst NULL");
  if (dist && (dist->row_begin < 0 || dist->row_end > V || dist->row_begin > dist->row_end))
    return fail(STG_ERR_INVALID_ARG, "stg_static_graph_create: row block [%d,%d) outside [0,%d]", dist->row_begin,
                dist->row_end, V);
  cudaStream_t s = (cudaStream_t)stream;
  auto* g = new stg_graph();
  BuildWs ws;
  const int loops = (flags & STG_SELF_LOOPS) ? 1 : 0;
  const int64_t n = E + (loops ? V : 0);
  Snapshot& sn = g->snap;
  stg_status st = sn.alloc(V, n, (flags & STG_EDGE_IDS) != 0, (flags & STG_NORM_DGL_BOTH) != 0,
                           dist ? dist->row_begin : 0, dist ? dist->row_end : -1);
  DArray<uint64_t> k1, k2;
  DArray<int32_t> bad;
  DArray<int64_t> cnt;
  if (st == STG_OK) st = k1.alloc(n);
  if (st == STG_OK) st = k2.alloc(n);
  if (st == STG_OK) st = bad.alloc(1);
  if (st == STG_OK) st = cnt.alloc(1);
  int32_t hbad = 0;
  int64_t E2 = 0;
  if (st == STG_OK) {
    sn.t = -1;
    cudaMemsetAsync(bad.p, 0, sizeof(int32_t), s);
    k_validate_pack<<<grid_for(n, 256), 256, 0, s>>>(src, dst, E, V, sn.nb, loops, k1.p, bad.p);
    count_launch();
    uint64_t* a = k1.p; uint64_t* b = k2.p;
    st = sort_unique_keys(&a, &b, n, 2 * sn.nb, cnt.p, ws, s);
    if (st == STG_OK) {
      if (cudaMemcpyAsync(&hbad, bad.p, sizeof(int32_t), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
          cudaMemcpyAsync(&E2, cnt.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
          cudaStreamSynchronize(s) != cudaSuccess)
        st = fail(STG_ERR_CUDA, "stg_static_graph_create: %s", cudaGetErrorString(cudaGetLastError()));
    }
    if (st == STG_OK && hbad) st = fail(STG_ERR_OUT_OF_RANGE, "stg_static_graph_create: vertex id outside [0,%d)", V);
    if (st == STG_OK && sn.sharded) {
      // whole-graph degrees for the norms, then keep the edges into the local block
      cudaMemsetAsync(sn.gin_deg.p, 0, sizeof(int32_t) * V, s);
      cudaMemsetAsync(sn.gout_deg.p, 0, sizeof(int32_t) * V, s);
      degree_hist(a, E2, sn.nb, 1, sn.gin_deg.p, sn.gout_deg.p, s);
      st = filter_block(a, E2, sn.nb, true, sn.rb, sn.re, b, cnt.p, ws, s);
      if (st == STG_OK && (cudaMemcpyAsync(&E2, cnt.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
                           cudaStreamSynchronize(s) != cudaSuccess))
        st = fail(STG_ERR_CUDA, "stg_static_graph_create: %s", cudaGetErrorString(cudaGetLastError()));
      std::swap(a, b);
    }
    if (st == STG_OK) st = build_from_out_keys(a, E2, sn, ws, s);
    if (st == STG_OK && cudaStreamSynchronize(s) != cudaSuccess)
      st = fail(STG_ERR_CUDA, "stg_static_graph_create: %s", cudaGetErrorString(cudaGetLastError()));
  }
  if (st != STG_OK) { delete g; return st; }
  *out = g;
  return STG_OK;
}

stg_status stg_graph_view(const stg_graph* g, stg_csr_view* out) {
  if (!g || !out) return fail(STG_ERR_INVALID_ARG, "stg_graph_view: NULL argument");
  g->snap.view(out, const_cast<AggWs*>(&g->ws));
  return STG_OK;
}

void stg_graph_destroy(stg_graph* g) {
  if (g) cudaDeviceSynchronize();
  delete g;
}

}  // extern "C"

namespace stg {
// bounds[k] = first row r with rowptr[r] >= k·E/world (nnz-balanced blocks).
__global__ void k_partition(const int32_t* __restrict__ rowptr, int32_t V, int32_t world, int32_t* __restrict__ b) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k > world) return;
  if (k == 0) { b[0] = 0; return; }
  if (k == world) { b[world] = V; return; }
  const int64_t E = rowptr[V];
  const int64_t target = (E * k + world - 1) / world;
  int32_t lo = 0, hi = V;
  while (lo < hi) {
    int32_t mid = (lo + hi) >> 1;
    if (rowptr[mid] < target) lo = mid + 1; else hi = mid;
  }
  b[k] = lo;
}
}  // namespace stg

extern "C" stg_status stg_partition_rows(int32_t V, const int32_t* in_rowptr, int32_t world, int32_t* bounds,
                                         stg_stream_t stream) {
  using namespace stg;
  if (V < 1 || world < 1 || !in_rowptr || !bounds) return fail(STG_ERR_INVALID_ARG, "stg_partition_rows: bad arguments");
  cudaStream_t s = (cudaStream_t)stream;
  DArray<int32_t> d;
  STG_TRY(d.alloc(world + 1));
  k_partition<<<(world + 128) / 128, 128, 0, s>>>(in_rowptr, V, world, d.p);
  count_launch();
  STG_CUDA(cudaMemcpyAsync(bounds, d.p, sizeof(int32_t) * (world + 1), cudaMemcpyDeviceToHost, s));
  STG_CUDA(cudaStreamSynchronize(s));
  // blocks must be non-decreasing; enforce (equal bounds = empty block)
  for (int k = 1; k <= world; ++k)
    if (bounds[k] < bounds[k - 1]) bounds[k] = bounds[k - 1];
  return STG_OK;
}
