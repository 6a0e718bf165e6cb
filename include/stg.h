/*
 * stg.h — C ABI of libstg, the B200 (sm_100a) hot path of STGraph
 * (Cherian et al., "STGraph: A Framework for Temporal Graph Neural Networks").
 *
 * Citations: "P:Lnnn" = /root/reference/PAPER.md line nnn (section in brackets);
 * "C<k>" = reading k in DESIGN.md §Readings.
 *
 * Conventions (all entry points):
 *  - Every array argument is a DEVICE pointer (cudaMalloc'd or torch-owned)
 *    unless marked (host).  Floating point is fp32 row-major; ids are int32.
 *  - Ownership: the caller owns every buffer it passes; inputs are only read
 *    during the call (plus the documented by-reference retention of the state
 *    stack).  The library owns graph / snapshot / stack storage, freed by the
 *    matching *_destroy.  Views (stg_csr_view) are BORROWED.
 *  - Streams: every call is ordered on the given stream (NULL = legacy default
 *    stream).  Only *_create calls synchronise the host.  stg_dtdg_get_* never
 *    synchronise: every snapshot size E_t is fixed at create time.
 *  - Errors: calls return a status and never throw or abort across the ABI.
 *    Argument checks are synchronous; asynchronous CUDA faults surface as
 *    STG_ERR_CUDA on a later call.  stg_last_error() gives a thread-local text.
 *  - Limits: V < 2^30, every edge count < 2^31 (else STG_ERR_OUT_OF_RANGE).
 */
#ifndef STG_H_
#define STG_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* stg_stream_t;   /* == cudaStream_t */

typedef enum {
  STG_OK = 0,
  STG_ERR_INVALID_ARG = 1,   /* NULL / negative / misaligned argument */
  STG_ERR_OUT_OF_RANGE = 2,  /* id outside [0,V), t outside [0,T), size overflow */
  STG_ERR_NO_MEMORY = 3,     /* device or host allocation failed */
  STG_ERR_CUDA = 4,          /* a CUDA runtime error (possibly from earlier async work) */
  STG_ERR_NCCL = 5,          /* reserved for collective failures */
  STG_ERR_STATE = 6          /* object in the wrong state, e.g. pop of an empty state stack */
} stg_status;

/* Thread-local description of the last non-OK status returned on this thread. */
const char* stg_last_error(void);
/* Library version as an integer MAJOR*10000 + MINOR*100 + PATCH. */
int32_t stg_version(void);
/* Number of device kernels this library launched since load (all threads). */
int64_t stg_kernel_launch_count(void);

/* Optional allocator hook (the Python binding installs PyTorch's caching
 * allocator at import; env STG_TORCH_ALLOCATOR=0 keeps cudaMalloc).  Every
 * library-owned device buffer (graph / DTDG snapshot slots and deltas, state
 * stack arena, scratch) then comes from alloc: bytes >= requested, 256-byte
 * aligned, or NULL (the call fails with STG_ERR_NO_MEMORY).  A block is
 * returned to the free function it was allocated with (after a device
 * synchronisation, cudaFree's ordering), so the hook may be changed at any
 * time.  Called from the host thread that calls into the library.  Passing
 * NULL, NULL restores cudaMalloc/cudaFree. */
typedef void* (*stg_alloc_fn)(size_t bytes, stg_stream_t stream, void* ctx);
typedef void (*stg_free_fn)(void* ptr, stg_stream_t stream, void* ctx);
stg_status stg_set_allocator(stg_alloc_fn alloc, stg_free_fn free_fn, void* ctx);
/* Process teardown: forget every block obtained through the hook (their later
 * frees, e.g. by static library state destroyed at exit, are skipped) and
 * restore cudaMalloc / cudaFree.  For a hook whose owner (an interpreter) is
 * shutting down; the memory goes back with the process. */
stg_status stg_allocator_detach(void);

/* Graph creation flags. */
enum {
  STG_SELF_LOOPS = 1u << 0,     /* add (v,v) for every v (idempotent; reading C1/C11).
                                   In a DTDG the loops are pinned: never deleted. */
  STG_EDGE_IDS = 1u << 1,       /* compute out_eid, the shared edge labels (C6) */
  STG_VALIDATE = 1u << 2,       /* DTDG: reject ill-formed batches (duplicate adds, adds of
                                   present edges, deletes of absent edges) instead of
                                   normalising them (reading C9) */
  STG_NORM_DGL_BOTH = 1u << 3,  /* n_src = out_deg^-1/2, n_dst = in_deg^-1/2 (default:
                                   both = in_deg^-1/2, PyG gcn_norm, reading C1) */
  STG_NAIVE = 1u << 4           /* DTDG NaiveGraph mode:
                                   materialise every snapshot S_0..S_{T-1} at create
                                   (memory ∝ Σ_t |E_t|); Get-Graph / Get-Backward-Graph
                                   are lookups.  Unsharded only. */
};

/* Row-block sharding (north_star "partitioned ... by
 * destination-vertex row blocks"): an object created with a non-NULL stg_dist
 * holds only the edges whose destination lies in [row_begin,row_end): the
 * forward in-CSR has the R = row_end-row_begin local rows, the backward
 * out-CSR has all V source rows but only the local edges.  Vertex ids stay
 * global.  Degrees and node_ids describe the held edges (in_ids lists the R
 * local rows first); norm_src / norm_dst are those of the WHOLE graph (the
 * library keeps the whole-graph degrees current from the whole-graph deltas),
 * so the local results are exactly the rows / partial sums of the whole-graph
 * computation.  Snapshot builds need no communication.  rank / world are
 * informational.  row_begin <= row_end must lie in [0,V]
 * (STG_ERR_INVALID_ARG otherwise).  NULL = whole graph.
 *
 * Deviation from SURVEY §8(b) (`stg_dist {nccl_comm, rank, world}`,
 * `stg_allgather_rows(stg_dist*, view, ...)`): the library holds no NCCL
 * communicator.  The per-timestep row exchange of sharded mode is done over
 * peer memory instead — every rank maps the others' row blocks once
 * (stg_peer_alloc / stg_peer_open, CUDA IPC, NVLink on a multi-GPU box) and the
 * forward gather reads a source row straight from its owner's block
 * (stg_gcn_aggregate_peer), so the all-gather is fused into the aggregation
 * tile by tile instead of being a separate NCCL call (north_star's "NCCL
 * all-gather over NVLink" would be the unfused baseline); stg_allgather_rows
 * takes that peer-row table.  The one collective left, the per-sequence
 * gradient all-reduce (~51 KB), is issued by the caller (torch.distributed /
 * NCCL), which owns the communicator and the process group. */
typedef struct {
  int32_t rank, world;
  int32_t row_begin, row_end;
} stg_dist;

/* A BORROWED view of one snapshot.  Valid until the owning object is destroyed
 * or, for a DTDG, until the next stg_dtdg_get_* call on it.  Layout (Fig. 3,
 * P:L183-185):
 *   forward CSR  : in_rowptr[R+1] (R = row_end-row_begin, local rows),
 *                  in_col[E] = source ids ascending within a row
 *   backward CSR : out_rowptr[V+1], out_col[E] = destination ids ascending
 *   (no COO row arrays are kept: a row's edges are [rowptr[r], rowptr[r+1]))
 *   out_eid[E]   : in-CSR position of out-edge j (shared edge label), or NULL
 *   in_deg/out_deg[V], in_ids/out_ids[V] = vertices by degree desc, id asc
 *   norm_src/norm_dst[V] fp32 GCN normalisation vectors (reading C1)
 *   in_sched/out_sched: library-internal degree-bucket schedules for the
 *   aggregation kernels (may be NULL in caller-built views).
 *   workspace: library-internal scratch handle (may be NULL). */
typedef struct {
  int32_t num_nodes;
  int32_t row_begin, row_end;
  int32_t timestamp;            /* -1 for a static graph */
  int64_t num_edges;            /* edges held by this view (local edges if sharded) */
  const int32_t *in_rowptr, *in_col;
  const int32_t *out_rowptr, *out_col;
  const int32_t *out_eid;
  const int32_t *in_deg, *out_deg, *in_ids, *out_ids;
  const float *norm_src, *norm_dst;
  const int32_t *in_sched, *out_sched;
  void* workspace;
} stg_csr_view;

typedef struct stg_graph stg_graph;
typedef struct stg_dtdg stg_dtdg;
typedef struct stg_state_stack stg_state_stack;

/* ---- static graph (Definition II.1; STGraphBase) ----
 * Builds the edge SET {(src[i],dst[i])} (duplicates removed, loops added with
 * STG_SELF_LOOPS), both CSRs, degrees, node_ids, norms and (STG_EDGE_IDS) the
 * shared edge labels, all on the device.  src/dst: E device ids in [0,V).
 * Synchronises `stream`.  *out is owned by the caller; free with _destroy. */
stg_status stg_static_graph_create(int32_t V, int64_t E, const int32_t* src, const int32_t* dst,
                                   uint32_t flags, const stg_dist* dist, stg_stream_t stream,
                                   stg_graph** out);
stg_status stg_graph_view(const stg_graph* g, stg_csr_view* out);
void stg_graph_destroy(stg_graph* g);

/* ---- DTDG (Definition II.2; GPMAGraph behaviour) ----
 * Base snapshot S_0 = {(src0,dst0)} plus per-timestamp batches: batch t is
 * add_src/add_dst[add_off[t] .. add_off[t+1]) and likewise for deletes, with
 * S_t = (S_{t-1} \ D_t) ∪ A_t.  add_off/del_off are HOST arrays of
 * T+1 int64; batch 0 must be empty.  The batches are normalised here to the
 * effective deltas A'_t = A_t \ S_{t-1}, D'_t = (D_t \ A_t) ∩ S_{t-1} (reading C9),
 * stored on the device in both (dst,src) and (src,dst) order; every E_t is then
 * known.  Synchronises `stream`. */
stg_status stg_dtdg_create(int32_t V, int32_t T, int64_t E0, const int32_t* src0, const int32_t* dst0,
                           const int64_t* add_off, const int32_t* add_src, const int32_t* add_dst,
                           const int64_t* del_off, const int32_t* del_src, const int32_t* del_dst,
                           uint32_t flags, const stg_dist* dist, stg_stream_t stream, stg_dtdg** out);
/* Get-Graph(G, t) (Algorithm 2; reading C8): returns the
 * snapshot for t built on demand from the nearest cached snapshot (base, the
 * forward head, the backward cursor) by applying |Δt| delta steps on `stream`. */
stg_status stg_dtdg_get_snapshot(stg_dtdg* g, int32_t t, stg_stream_t stream, stg_csr_view* out);
/* Get-Backward-Graph(G, t): the same snapshot t for the backward pass,
 * reached from the backward cursor by reverse updates, without disturbing the
 * cached forward head (which the next sequence starts from). */
stg_status stg_dtdg_get_backward_snapshot(stg_dtdg* g, int32_t t, stg_stream_t stream, stg_csr_view* out);
/* Snapshot parts (stg_dtdg_get_snapshot_parts): a pass that needs one CSR
 * direction asks for that one only — the forward in-CSR for Get-Graph, the
 * reverse out-CSR for Get-Backward-Graph — and the library delta-merges only
 * that direction per step.  A cached snapshot that lacks a requested
 * direction gets it by a stable transpose of the one it has (Algorithm 3,
 * P:L218-251, in the canonical order of reading C7).  Degrees and norms are
 * always current (whole-graph degree histograms of the deltas). */
enum { STG_PART_IN = 1u << 0, STG_PART_OUT = 1u << 1, STG_PART_EID = 1u << 2 /* implies both */ };
/* Get-Graph (backward = 0) / Get-Backward-Graph (backward = 1) of the parts in
 * `parts` (STG_PART_*; at least one direction).  The view's pointers of the
 * parts not requested may be NULL (in_rowptr/in_col/in_ids/in_sched
 * for the in-CSR, likewise out_*; out_eid unless STG_PART_EID).  Same
 * validity and stream rules as stg_dtdg_get_snapshot, which equals
 * parts = IN|OUT|EID (EID only with STG_EDGE_IDS). */
stg_status stg_dtdg_get_snapshot_parts(stg_dtdg* g, int32_t t, int32_t backward, uint32_t parts,
                                       stg_stream_t stream, stg_csr_view* out);
int64_t stg_dtdg_num_edges(const stg_dtdg* g, int32_t t);    /* edges held at t (the local block's if sharded); -1 if t out of range */
int32_t stg_dtdg_num_timestamps(const stg_dtdg* g);
/* Number of effective added / deleted edges of step t (0 for t = 0). */
int64_t stg_dtdg_num_deltas(const stg_dtdg* g, int32_t t, int32_t deletes);
/* Device bytes held by a DTDG (the Table III / Fig. 8 memory comparison):
 * the normalised delta arrays, the snapshot cache (Alg. 2 slots, scratch), and the
 * snapshots materialised by STG_NAIVE (0 otherwise). */
stg_status stg_dtdg_memory(const stg_dtdg* g, int64_t* deltas, int64_t* cache, int64_t* materialised);
void stg_dtdg_destroy(stg_dtdg* g);

/* ---- GCN aggregation (north_star) ----
 * forward : y[v,:] = n_dst[v] · Σ_{u∈N_in(v)} n_src[u] · x[u,:]   over the in-CSR,
 *           for the local rows v of the view (y row i ↔ vertex row_begin+i).
 * backward: gx[u,:] = n_src[u] · Σ_{v∈N_out(u)} n_dst[v] · gy[v,:] over the out-CSR
 *           (the exact transpose), for all V sources (partial sums if sharded;
 *           gy then holds the R local rows: gy row i ↔ vertex row_begin+i).
 * x/gy: [V,W] (forward: all sources) with leading dimension ldx >= W;
 * y/gx: leading dimension ldy >= W.  fp32 accumulation in a fixed order per
 * row: results are deterministic run to run (no float atomics; reading C20).
 * Float4 path when W, ldx, ldy are multiples of 4 and x, y are 16-byte aligned. */
stg_status stg_gcn_aggregate_fwd(const stg_csr_view* g, int32_t W, const float* x, int64_t ldx,
                                 float* y, int64_t ldy, stg_stream_t stream);
stg_status stg_gcn_aggregate_bwd(const stg_csr_view* g, int32_t W, const float* gy, int64_t ldgy,
                                 float* gx, int64_t ldgx, stg_stream_t stream);
/* General form used by both: backward=0 → in-CSR, 1 → out-CSR;
 *   out[r,:] = scale_row[r] · Σ_{c∈row r} scale_col[c] · in[c,:] + bias[:]
 * with scale_row / scale_col / bias each optional (NULL = 1 / 1 / 0).
 * In a sharded view the arrays indexed by a DESTINATION vertex hold the local
 * rows only (forward: out, scale_row; backward: in, scale_col). */
stg_status stg_gcn_aggregate_ex(const stg_csr_view* g, int32_t backward, int32_t W,
                                const float* in, int64_t ldin, float* out, int64_t ldout,
                                const float* scale_row, const float* scale_col, const float* bias,
                                stg_stream_t stream);

/* Edge-weighted aggregation (features "of nodes and edges",
 * P:L50; shared edge labels):
 *   out[r,:] = scale_row[r] · Σ_{j ∈ row r} w_j · scale_col[c_j] · in[c_j,:] + bias[:]
 * where w_j is the weight of the EDGE at position j: ew is indexed by the edge
 * label = in-CSR position (reading C6), so the forward reads ew[j] and the
 * backward (out-CSR) reads ew[out_eid[j]] — the transpose uses the same weights
 * without a permuted copy.  ew [E] fp32 device array in in-CSR order.  The backward
 * needs a view with out_eid (STG_EDGE_IDS).  Float4 path only: W % 4 == 0,
 * W <= 512, 16-byte aligned rows, a library view (STG_ERR_INVALID_ARG otherwise).
 * Other conventions as stg_gcn_aggregate_ex. */
stg_status stg_gcn_aggregate_weighted(const stg_csr_view* g, int32_t backward, int32_t W, const float* ew,
                                      const float* in, int64_t ldin, float* out, int64_t ldout,
                                      const float* scale_row, const float* scale_col, const float* bias,
                                      stg_stream_t stream);
/* Weighted GCN normalisation (PyG gcn_norm with edge weights; reading C21):
 * norm[i] = (Σ_{j ∈ in-row i} ew[j])^-1/2, 0 if the sum is <= 0, for the R local rows
 * of the view (R = V unsharded; the symmetric norm uses it for both n_src and n_dst).
 * Per-row sums in fp64 (fixed order), result rounded to fp32. */
stg_status stg_gcn_weighted_norm(const stg_csr_view* g, const float* ew, float* norm, stg_stream_t stream);

/* Work decomposition of the aggregation (process-wide; every strategy is
 * deterministic, uses no float atomics, and keeps each fp32 chain <= 64 terms).
 * The snapshot schedule lists rows in node_ids order (degree presort,
 * P:L175/L322) as items of <= 64 edges (hub rows cut into chunks).
 * 2 (default) = edge stream: a warp walks the concatenated edge lists of 32
 *     items, gathering several neighbour rows at once across row boundaries
 *     (float4 path, 32 < W <= 128 per column launch; wider W is split into
 *     launches of <= 128 columns; otherwise strategy 1 is used);
 * 1 = pipelined items: FA-TGA lane groups serve 32/G rows per warp
 *     with the next items' descriptors and columns prefetched (float4 path);
 * 0 = row items with register gathers (any width/alignment; also the path of
 *     caller-built views without a schedule). */
stg_status stg_aggregate_set_strategy(int32_t strategy);
/* Tunables of strategy 2 (STG_ERR_INVALID_ARG for a bad key/value):
 * key 0: neighbour rows in flight per warp, 4 | 8 | 16 (default 4);
 * key 1: minimum resident blocks per SM (register budget), 2..6 (default 6;
 *        supported pairs (rows, blocks): (4,6) (8,4) (16,2) (16,3));
 * key 2: 0 | 8 | 16 | 32 | 64 (default 0): strategy 2 serves launch widths above this. */
stg_status stg_aggregate_set_param(int32_t key, int64_t value);

/* ---- TGCN (GCN + GRU; reading C13-C15) ----
 * W [F,3H] (gates z|r|h), b [3H], L [3][2H][H] (gate g: rows 0..H-1 = L_g¹ act
 * on C_g, rows H..2H-1 = L_g² act on H or R⊙H), l [3][H]. */
typedef struct {
  int32_t F, H;
  const float *W, *b, *L, *l;
} stg_tgcn_params;
typedef struct {
  float *W, *b, *L, *l;        /* gradients, ACCUMULATED (+=), same layouts */
} stg_tgcn_grads;

/* State Stack: LIFO of per-timestamp forward state.  Each push
 * stores C_t [V,3H] in the stack's device arena (capacity_bytes) and retains
 * H_prev BY REFERENCE: the caller keeps that buffer unmodified until the
 * matching backward pops it (reading A8: only {H_{t-1}, C_t} are saved). */
stg_status stg_state_stack_create(int64_t capacity_bytes, stg_state_stack** out);
int32_t stg_state_stack_depth(const stg_state_stack* s);
void stg_state_stack_destroy(stg_state_stack* s);

/* Forward step at one timestamp (a7):
 *   P' = diag(n_src)·X·W;  C = diag(n_dst)·A·P' + b;  GRU gates;  H_next.
 * X [V,F] (all vertices, resident on every rank), H_prev/H_next [R,H] with
 * R = row_end-row_begin (R = V unsharded): a sharded view computes P' for all V
 * sources and C, the GRU and H_next for its R local rows only.
 * stack == NULL: inference, nothing retained. */
stg_status stg_tgcn_step(const stg_csr_view* g_fwd, const stg_tgcn_params* p, const float* X,
                         const float* H_prev, float* H_next, stg_state_stack* stack,
                         stg_stream_t stream);
/* Backward step (a8): pops {H_prev, C} pushed by the matching forward step and,
 * given dH_next = dℓ/dH_t (total), writes dH_prev = dℓ/dH_{t-1} and accumulates
 * parameter gradients.  g_bwd must be the snapshot of the same t (its out-CSR
 * carries dP = Âᵀ·dC).  dH_prev may alias nothing else.  Sharded: dH_next /
 * dH_prev are [R,H]; dP holds the partial sums of the local edges for all V
 * sources, so the accumulated gradients are this rank's share: their sum over
 * ranks (one all-reduce per sequence, before the optimiser step) is the
 * whole-graph gradient. */
stg_status stg_tgcn_step_backward(const stg_csr_view* g_bwd, const stg_tgcn_params* p, const float* X,
                                  const float* dH_next, float* dH_prev, stg_tgcn_grads* grads,
                                  stg_state_stack* stack, stg_stream_t stream);

/* ---- original T-GCN cell (the model cited at P:L58, whose
 * graph convolution acts on [X, H]; oracle orc_tgcn2_fwd/bwd):
 *   [r | u] = σ(Â([X, H]·Wg) + bg),  c = tanh(Â([X, r⊙H]·Wc) + bc),  H' = u⊙H + (1−u)⊙c
 * Wg [F+H, 2H] (columns r | u), bg [2H], Wc [F+H, H], bc [H]; X [V,F], H [V,H].
 * Two aggregations per step (widths 2H and H) sit on the recurrent path; the
 * backward runs two over the out-CSR.  Unsharded views; H in {4,8,16,32,64}.
 * The state stack saves [r | u | c] per step (H_prev by reference, as stg_tgcn_step);
 * gradients accumulate (+=), dH_prev is overwritten. */
typedef struct {
  int32_t F, H;
  const float *Wg, *bg, *Wc, *bc;
} stg_tgcn2_params;
typedef struct {
  float *Wg, *bg, *Wc, *bc;
} stg_tgcn2_grads;
stg_status stg_tgcn2_step(const stg_csr_view* g, const stg_tgcn2_params* p, const float* X, const float* H_prev,
                          float* H_next, stg_state_stack* stack, stg_stream_t stream);
stg_status stg_tgcn2_step_backward(const stg_csr_view* g, const stg_tgcn2_params* p, const float* X,
                                   const float* dH_next, float* dH_prev, stg_tgcn2_grads* grads,
                                   stg_state_stack* stack, stg_stream_t stream);

/* Surrogate MSE head (timing only; A15): ŷ_v = Σ_k ReLU(H_vk)·w_o[k] + b_o[0],
 *   ℓ = mean_v (ŷ_v − y_v)².
 * loss_accum (device scalar, may be NULL) += ℓ.  If dH != NULL: dH (+)= dℓ/dH
 * (accumulate=1 adds into dH, 0 overwrites) and dw_o/db_o (if non-NULL) += grads. */
stg_status stg_mse_head(int32_t V, int32_t H, const float* Hn, const float* y, const float* w_o,
                        const float* b_o, float* loss_accum, float* dH, int32_t accumulate,
                        float* dw_o, float* db_o, stg_stream_t stream);
/* The same over V local rows of a V_total-row graph (sharded): the mean is
 * taken over V_total, so the per-rank losses and gradients add up. */
stg_status stg_mse_head_ex(int32_t V, int32_t V_total, int32_t H, const float* Hn, const float* y,
                           const float* w_o, const float* b_o, float* loss_accum, float* dH,
                           int32_t accumulate, float* dw_o, float* db_o, stg_stream_t stream);

/* p -= lr·g over n elements, then g = 0 for the next accumulation (the
 * per-sequence optimiser step, reading C17). */
stg_status stg_sgd_update(float* p, float* g, int64_t n, float lr, stg_stream_t stream);

/* Algorithm 1 for ONE sequence s = [t0, t0+S): forward for t ∈ s
 * (DTDG: Get-Graph, graph-stack push; state-stack push; step; loss), then
 * backward in LIFO order (graph-stack pop, Get-Backward-Graph, head gradient,
 * step_backward).  Exactly one of `graph` / `dtdg` is non-NULL.
 * X (host)[S] device pointers to X_t [V,F]; Y (host)[S] device pointers to y_t [R];
 * H0 [R,H] initial state (detached); H_seq [S][R,H] receives H_t (H_seq[S-1] is
 * the state the next sequence starts from, reading C15); G_work [2][R,H] scratch
 * (R = the local rows of a sharded graph / dtdg, else V).
 * Gradients (grads, dw_o, db_o) and loss_accum are accumulated. */
stg_status stg_tgcn_train_sequence(const stg_graph* graph, stg_dtdg* dtdg, int32_t t0, int32_t S,
                                   const stg_tgcn_params* p, const float* w_o, const float* b_o,
                                   const float* const* X, const float* const* Y, const float* H0,
                                   float* H_seq, float* G_work, stg_tgcn_grads* grads, float* dw_o,
                                   float* db_o, float* loss_accum, stg_state_stack* stack,
                                   stg_stream_t stream);

/* The same with per-timestamp input readiness: xy_ready (host)[S] holds a cudaEvent_t
 * (as stg_event_t) per timestamp, recorded after X[i] and Y[i] were written (e.g. by
 * a host->device copy on another stream), or NULL entries / a NULL array.  The step
 * of timestamp i waits for its event only, so a sequence starts computing as soon as
 * its first inputs have landed while later ones are still being copied (e2e). */
typedef void* stg_event_t;
stg_status stg_tgcn_train_sequence_ev(const stg_graph* graph, stg_dtdg* dtdg, int32_t t0, int32_t S,
                                      const stg_tgcn_params* p, const float* w_o, const float* b_o,
                                      const float* const* X, const float* const* Y, const float* H0,
                                      float* H_seq, float* G_work, stg_tgcn_grads* grads, float* dw_o,
                                      float* db_o, float* loss_accum, stg_state_stack* stack,
                                      const stg_event_t* xy_ready, stg_stream_t stream);

/* Sequence-batched Algorithm 1 for a STATIC graph: the
 * same forward, loss and gradients as stg_tgcn_train_sequence over t = 0..S-1
 * (P:L120-171), scheduled per sequence.  Because C_t = Â(X_t W) + b does not
 * depend on H (reading C13/C14), X_t W and the aggregation run once for all S
 * timestamps (one SpMM of width S·3H over [V][S][3H] rows), the GRU recurrence
 * and the MSE head run for all t inside one persistent row-tile kernel per
 * direction, and dL/dl/db, dP = Âᵀ dC', dW reduce over all V·S (vertex, t)
 * rows at once.  Requirements: unsharded graph, tensor-core shapes (H 16|32,
 * F % 4 == 0, F <= 64), 1 <= S <= 64.  Arguments as stg_tgcn_train_sequence
 * (X/Y (host)[S] device pointers, H0 [V,H], H_seq [S][V,H] receives H_t,
 * gradients and loss accumulated); the stack only provides scratch. */
stg_status stg_tgcn_train_sequence_batched(const stg_graph* graph, int32_t S, const stg_tgcn_params* p,
                                           const float* w_o, const float* b_o, const float* const* X,
                                           const float* const* Y, const float* H0, float* H_seq,
                                           stg_tgcn_grads* grads, float* dw_o, float* db_o,
                                           float* loss_accum, stg_state_stack* stack, stg_stream_t stream);

/* ---- multi-GPU helpers ----
 * nnz-balanced destination row blocks: bounds (host)[world+1] with bounds[0]=0,
 * bounds[world]=V, block k ≈ E/world in-edges.  in_rowptr is a DEVICE [V+1]
 * array of a whole-graph view.  Synchronises `stream`. */
stg_status stg_partition_rows(int32_t V, const int32_t* in_rowptr, int32_t world, int32_t* bounds,
                              stg_stream_t stream);

/* ---- sharded mode over peer memory (SURVEY §8(e) "sharded mode"; north_star
 * "partitioned ... by destination-vertex row blocks, with ... all-gather over
 * NVLink of the source feature/hidden rows each timestep") ----
 * Every rank owns the rows of its block of a [V,W] row matrix (P' = diag(n_src)XW,
 * or any feature/hidden rows).  Instead of copying the whole matrix to every rank
 * and then aggregating, the aggregation kernel loads each neighbour row directly
 * from its OWNER's buffer (NVLink peer loads of CUDA-IPC-mapped memory), so the
 * exchange is fused into the gather, tile by tile, with no staging copy.
 * Ordering across ranks is the caller's: the owners' writes must be complete
 * (e.g. a stream-ordered NCCL all-reduce of one element, or a host barrier after a
 * synchronize) before a rank gathers, and a buffer is rewritten only after every
 * reader finished (double-buffer per timestep).
 *
 * A row table: block k (0 <= k < world <= STG_MAX_PEERS) holds the rows
 * [bounds[k], bounds[k+1]) of the matrix, block-local row 0 = vertex bounds[k],
 * leading dimension ld (floats, % 4 == 0), base 16-byte aligned.  bounds (host)
 * [world+1], non-decreasing, bounds[0] = 0, bounds[world] = V; blocks (host)
 * [world] DEVICE pointers valid on the calling device (local, or opened with
 * stg_peer_open).  A NULL block is allowed only when the block is empty. */
#define STG_MAX_PEERS 8
typedef struct {
  int32_t world;
  const int32_t* bounds;
  const float* const* blocks;
  int64_t ld;
} stg_peer_rows;

/* CUDA IPC handle of a peer-visible allocation (opaque, 64 bytes). */
typedef struct { unsigned char reserved[64]; } stg_ipc_handle;
/* Allocates `bytes` of zero-initialised device memory that other processes may
 * map (cudaMalloc'd, not pooled) and returns its IPC handle.  Free with stg_peer_free. */
stg_status stg_peer_alloc(int64_t bytes, void** dptr, stg_ipc_handle* handle);
stg_status stg_peer_free(void* dptr);
/* Maps another process's allocation (same or peer device, peer access enabled
 * lazily over NVLink).  STG_ERR_CUDA if the handle was created in this process. */
stg_status stg_peer_open(const stg_ipc_handle* handle, void** dptr);
stg_status stg_peer_close(void* dptr);

/* ---- sharded-mode Algorithm 1 in the library (the per-timestep exchange ordered
 * by device-side flags instead of host barriers) ----
 * Every rank holds, in peer-mapped memory (stg_peer_alloc / stg_peer_open):
 *   P[b][k]  : rank k's P' rows [R_k, 3H] (b = exchange parity: two buffers),
 *   dP[b][k] : rank k's partial dP over all V source rows [V, 3H],
 *   flags[k] : 4 uint32 counters of rank k, zero at allocation — 0: forward
 *              exchanges published, 1: forward exchanges consumed, 2: backward
 *              exchanges published, 3: backward exchanges consumed.
 * Forward exchange n (b = n % 2): wait until every rank consumed exchange n-2
 * (its buffer), project this rank's P' rows, publish n, wait until every rank
 * published n, gather + GRU (+ the fused head), mark n consumed.  Backward
 * exchange m: wait until every rank consumed m-2, GRU backward + partial
 * Âᵀ dC' into dP[b][rank], publish m, wait for all, reduce-scatter this rank's
 * rows in rank order, mark m consumed, dW += X_locᵀ dP_loc.  Waits and
 * publications are stream memory operations (cuStreamWaitValue32 /
 * cuStreamWriteValue32 on the peers' counters), so no host synchronisation and
 * no NCCL call sits on the data path; the per-sequence gradient all-reduce
 * stays with the caller.  fwd_count / bwd_count: exchanges done so far by
 * every rank (in/out; all ranks call with the same values). */
typedef struct {
  int32_t world, rank;
  const int32_t* bounds;              /* (host) [world+1] */
  float* P[2][STG_MAX_PEERS];
  float* dP[2][STG_MAX_PEERS];
  uint32_t* flags[STG_MAX_PEERS];
  uint32_t fwd_count, bwd_count;
} stg_peer_exchange;

/* Algorithm 1 for one sequence of S timestamps on this rank's row block
 * (sharded mode, X row-sharded): dtdg is this rank's sharded DTDG (stg_dist
 * = its block), X_loc / Y_loc (host)[S] device pointers to its rows, H0 /
 * H_seq [S][R,H] / G_work [2][R,H] its rows; gradients are this rank's share
 * (sum over ranks = the whole-graph gradients).  dP_loc [R,3H] scratch.
 * Needs the tensor-core path (tc_supported).  Errors as stg_tgcn_train_sequence. */
stg_status stg_tgcn_train_sequence_peer(stg_dtdg* dtdg, int32_t t0, int32_t S, const stg_tgcn_params* p,
                                        const float* w_o, const float* b_o, const float* const* X_loc,
                                        const float* const* Y_loc, const float* H0, float* H_seq, float* G_work,
                                        float* dP_loc, stg_tgcn_grads* grads, float* dw_o, float* db_o,
                                        float* loss_accum, stg_state_stack* stack, stg_peer_exchange* px,
                                        stg_stream_t stream);

/* All-gather of row blocks over peer loads: full[u,:] = row u of its owner's block,
 * for all u in [0,V), W columns; full has leading dimension ldf >= W.  (The
 * explicit form of the exchange, for consumers other than the fused gather.) */
stg_status stg_allgather_rows(const stg_peer_rows* src, int32_t W, float* full, int64_t ldf,
                              stg_stream_t stream);

/* Fused forward aggregation over peer memory: as stg_gcn_aggregate_ex with
 * backward = 0, but each source row in[c,:] is read from its owner's block of `x`
 * (x->bounds must cover the view's num_nodes).  Width 4 <= W <= 512, W % 4 == 0,
 * and the view must carry the library schedule (views of library objects do). */
stg_status stg_gcn_aggregate_peer(const stg_csr_view* g, int32_t W, const stg_peer_rows* x,
                                  float* out, int64_t ldout, const float* scale_row,
                                  const float* scale_col, const float* bias, stg_stream_t stream);

/* Reduce-scatter over peer loads: for the rows u of `rank`'s block
 * [bounds[rank], bounds[rank+1]), out[u - bounds[rank], :] = Σ_{q=0..world-1}
 * partials[q][u, :] summed in rank order q = 0, 1, ... (deterministic).
 * partials (host)[world] device pointers to every rank's FULL [V, ld] buffer. */
stg_status stg_reduce_scatter_rows(int32_t world, const int32_t* bounds, const float* const* partials,
                                   int64_t ld, int32_t rank, int32_t W, float* out, int64_t ldout,
                                   stg_stream_t stream);

/* The TGCN step in sharded mode (X row-sharded, nothing replicated):
 *   stg_tgcn_project      P'_loc = diag(n_src[rows]) · X_loc · W for the R local rows
 *                         (X_loc [R,F], P_loc [R,3H]);
 *   stg_tgcn_step_peer    C = diag(n_dst)·A·P' + b with P' gathered from the owners
 *                         (stg_gcn_aggregate_peer), GRU, H_next; pushes {H_prev, C};
 *   stg_tgcn_step_backward_peer  pops, GRU backward, dL/dl/db, and the partial
 *                         dP_part = diag(n_src)·Aᵀ_loc·dC' [V,3H] of the local edges
 *                         for all V sources (no dW);
 *   stg_reduce_scatter_rows  dP_loc = Σ_ranks dP_part over the owner's rows;
 *   stg_tgcn_dw           dW += X_locᵀ · dP_loc.
 * The per-rank gradients add up to the whole-graph gradient (all-reduce per
 * sequence, as in resident mode). */
stg_status stg_tgcn_project(const stg_csr_view* g, const stg_tgcn_params* p, const float* X_loc,
                            float* P_loc, stg_stream_t stream);
stg_status stg_tgcn_step_peer(const stg_csr_view* g_fwd, const stg_tgcn_params* p, const stg_peer_rows* P,
                              const float* H_prev, float* H_next, stg_state_stack* stack,
                              stg_stream_t stream);
stg_status stg_tgcn_step_backward_peer(const stg_csr_view* g_bwd, const stg_tgcn_params* p,
                                       const float* dH_next, float* dH_prev, stg_tgcn_grads* grads,
                                       float* dP_part, stg_state_stack* stack, stg_stream_t stream);
stg_status stg_tgcn_dw(const stg_tgcn_params* p, int32_t R, const float* X_loc, const float* dP_loc,
                       stg_tgcn_grads* grads, stg_state_stack* stack, stg_stream_t stream);

/* The original T-GCN cell in sharded mode over peer memory: both convolutions gather
 * rows that carry H from their owners (north_star "all-gather ... of the source
 * feature/hidden rows each timestep"), so the hidden state crosses ranks every
 * step.  Each call runs one phase; the caller puts a cross-rank barrier between
 * phases (parallel.PeerTGCN2).  R = local rows of the sharded view.
 *   fwd phase 0: Z_loc [R,2H] = n_src ⊙ [X_loc, H_loc]·Wg   (this rank's block of Zg)
 *       phase 1: gates from Â·Zg (rows gathered through Z) + bg; Z_loc [R,H] = n_src ⊙ [X_loc, r⊙H]·Wc
 *       phase 2: c from Â·Zc (rows gathered through Z) + bc; H_next [R,H]; state pushed
 *   bwd phase 0: candidate backward, dbc; part_out [V,H] = partial Âᵀ dA_c of the local edges
 *       phase 1: dY_c = Σ_ranks parts (stg_reduce_scatter_rows), dWc, gate backward, dbg;
 *                part_out [V,2H] = partial Âᵀ dA_g
 *       phase 2: dY_g = Σ_ranks parts, dWg, dH_prev += dY_g·Wg[F:]ᵀ; state popped
 * parts (host)[world] = every rank's part_out of the previous phase.  Gradients are this
 * rank's share (sum over ranks = whole-graph gradient). */
stg_status stg_tgcn2_peer_fwd(int32_t phase, const stg_csr_view* g, const stg_tgcn2_params* p, const float* X_loc,
                              const float* H_loc, const stg_peer_rows* Z, float* Z_loc, float* H_next,
                              stg_state_stack* stack, stg_stream_t stream);
stg_status stg_tgcn2_peer_bwd(int32_t phase, const stg_csr_view* g, const stg_tgcn2_params* p, const float* X_loc,
                              const float* dH_next, float* dH_prev, stg_tgcn2_grads* grads, int32_t rank,
                              int32_t world, const int32_t* bounds, const float* const* parts, float* part_out,
                              stg_state_stack* stack, stg_stream_t stream);


/* Per-phase device timing with CUDA events recorded on the launching stream
 * around each phase (bench.py; the GNN vs graph-update split of Fig. 9,
 * P:L316/L345).  phase: 0 aggregation fwd, 1 aggregation bwd, 2 snapshot
 * build (Get-Graph / Get-Backward-Graph), 3 P' = X·W, 4 GRU fwd, 5 GRU bwd,
 * 6 dW, 7 head, 8 dL/dl/db reductions; sub-phases of 2: 9 one delta step of
 * one CSR direction (Algorithm 2's update), 10 one transpose (Algorithm 3).
 * Phases launched on different streams may overlap (stg_set_pipeline(0)
 * serialises a training sequence for an exact split).  stg_profile_read
 * synchronises on the recorded events and returns the accumulated
 * milliseconds and count (reset != 0 clears them). */
stg_status stg_profile_enable(int32_t on);
stg_status stg_profile_read(int32_t phase, double* total_ms, int64_t* count, int32_t reset);

/* Schedule of stg_tgcn_train_sequence(_ev): 1 (default) = the three-stream pipeline (snapshot builds and the
 * H-independent work overlap the GRU chain); 0 = everything on the caller's
 * stream, one kernel after another (same arithmetic, same results; used to
 * measure the per-phase split). */
stg_status stg_set_pipeline(int32_t on);

/* Environment schedule tunables, read once when the library first needs them.
 * None changes the arithmetic or skips work; each selects between measured
 * schedules (defaults are the measured best on C5):
 *   STG_ATB_SMEM_KB (220)  ring budget of the Σ AᵀB reduction kernel, KB
 *   STG_ATB_CTAS (1)       allow 2 CTAs per SM for it when 3 stages fit twice
 *   STG_ATB_L1 (0)         its 2-hi-stage / 1-lo-slot variant at 2 CTAs per SM
 *   STG_SMALL_RB (auto)    rows per CTA of the small-graph sequence kernels
 *   STG_DL_STREAM (0)      dL/dl reductions on the H-chain stream (1) or aux stream
 *   STG_AUX_STREAM (1)     H-independent work on an aux stream (0: caller's stream)
 *   STG_SNAP_AFTER_CONV (1) the forward build of Get-Graph(t+1) starts after the
 *                          convolution of t (0: after that of t-1, beside the gather)
 *   STG_DL3 (1)            H = 32 dL/dl as three gate-blocked products (0: the two
 *                          full [C|H]ᵀda, [RH|1]ᵀda products; same gradients to fp32)
 *   STG_TORCH_ALLOCATOR    (binding) 0 keeps cudaMalloc instead of torch's pool */

/* Order of the graph convolution in the TGCN step (reading C14; SURVEY §8(f)
 * NEXT-1): 0 (default) = linear-first C = Â(XW) + b — the forward aggregates
 * P' = n_src ⊙ XW (width 3H) over the in-CSR and the backward aggregates dC'
 * over the out-CSR (dP = Âᵀ dC, dW = Xᵀ dP); 1 = aggregate-first C = (ÂX)W + b —
 * the forward aggregates X (width F) and keeps ÂX on the state stack, the
 * backward needs no graph (dW = (ÂX)ᵀ dC), so a DTDG sequence builds no
 * backward snapshots.  Same model, same gradients up to rounding.  Order 1
 * needs the tensor-core path (H in {16, 32}, F <= 64, F % 4 == 0) and is used
 * by stg_tgcn_step / _backward and stg_tgcn_train_sequence(_ev); the state
 * stack then needs V·(3H + F)·4 bytes per step.  STG_ERR_INVALID_ARG for
 * another value. */
stg_status stg_set_conv_order(int32_t order);

/* Diagnostic tcgen05 3xTF32 GEMM (tests pin the UMMA conventions with it):
 * mode 0: C[M,N] = A[M,K]·B[K,N] (M % 128 == 0, K % 8 == 0, K <= 256);
 * mode 1: C[128,N] = Aᵀ·B with A [R,128], B [R,N] (R % 128 == 0).
 * N % 16 == 0, 16 <= N <= 256.  Row-major fp32 device arrays. */
stg_status stg_debug_tc_gemm(int32_t mode, int32_t M, int32_t N, int32_t K, int32_t R, const float* A,
                             const float* B, float* C, stg_stream_t stream);

/* Diagnostic: the fixed-order sum tot[e] = Σ_b part[b·n + e] of the Σ AᵀB
 * reductions (per-CTA partials part[nb][n], added in blocks of 16 in block
 * order, then over the blocks in order).  variant 0: one thread per element;
 * variant 1: parallel over the 16-partial blocks (nb <= 1024).  Both give the
 * same bits (tests/test_gpu_tc.py).  Device arrays; STG_ERR_INVALID_ARG for
 * nb < 1, n < 1 or an unknown variant. */
stg_status stg_debug_sum_parts(const float* part, int32_t nb, int32_t n, float* tot, int32_t variant,
                               stg_stream_t stream);

/* Stream-ordered byte copy (kind: 0 device->device, 1 host->device,
 * 2 device->host); lets bindings read borrowed view arrays. */
stg_status stg_memcpy(void* dst, const void* src, size_t bytes, int32_t kind, stg_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* STG_H_ */
