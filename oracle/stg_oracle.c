/*
 * stg_oracle.c — plain, slow, obviously-correct CPU reference (fp64) for the
 * STGraph hot path.  TEST INFRASTRUCTURE ONLY: nothing in the product path
 * (paper_conf_ipps_cherianmcc24_b200/, include/) may include, link or call it;
 * only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference
 * arm use it.  It shares no code, header or constant with the CUDA library.
 *
 * Citations: "P:Lnnn" = /root/reference/PAPER.md line nnn; "C<k>" = a reading
 * listed in DESIGN.md §Readings.
 *
 * Every function below is the plain definition: sets are sorted arrays of
 * uint64 keys (src<<32 | dst), built with qsort; sums run in ascending
 * neighbour order in double precision; no blocking, fusion or reordering.
 *
 * Parity status: edge sets / CSRs / degrees / node_ids pinned
 * (P:L185 worked example, invariants, brute force); aggregation pinned (4-node
 * closed forms, dense brute force, adjoint, complete-graph mean); snapshots
 * pinned (fold == event-window rebuild); TGCN pinned (finite
 * differences, zero-parameter closed form, Â=I GRU reduction).  The edge-label
 * scheme (out_eid, reading C6) is our canonical choice: "parity unpinned"
 * against the paper, pinned only by its definition.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static uint64_t mk(int32_t s, int32_t d) { return ((uint64_t)(uint32_t)s << 32) | (uint32_t)d; }
static int32_t ksrc(uint64_t k) { return (int32_t)(k >> 32); }
static int32_t kdst(uint64_t k) { return (int32_t)(k & 0xffffffffu); }

static int cmp_u64(const void* a, const void* b) {
  uint64_t x = *(const uint64_t*)a, y = *(const uint64_t*)b;
  return (x > y) - (x < y);
}

/* sort + unique in place; returns the new length */
static int64_t sort_unique(uint64_t* a, int64_t n) {
  if (n <= 0) return 0;
  qsort(a, (size_t)n, sizeof(uint64_t), cmp_u64);
  int64_t m = 1;
  for (int64_t i = 1; i < n; ++i)
    if (a[i] != a[m - 1]) a[m++] = a[i];
  return m;
}

static int contains(const uint64_t* a, int64_t n, uint64_t k) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    int64_t mid = lo + (hi - lo) / 2;
    if (a[mid] < k) lo = mid + 1; else hi = mid;
  }
  return lo < n && a[lo] == k;
}

/* ---------------------------------------------------------------------------
 * Edge set of a graph (G is a set of edges; reading C1/C11: with
 * self_loops, (v,v) is added for every v, idempotent with existing loops).
 * out: capacity E + V keys, sorted by (src, dst).  Returns |S|.
 * ------------------------------------------------------------------------- */
int64_t orc_edge_set(int32_t V, int64_t E, const int32_t* src, const int32_t* dst,
                     int32_t self_loops, uint64_t* out) {
  int64_t n = 0;
  for (int64_t i = 0; i < E; ++i) out[n++] = mk(src[i], dst[i]);
  if (self_loops)
    for (int32_t v = 0; v < V; ++v) out[n++] = mk(v, v);
  return sort_unique(out, n);
}

typedef struct { int32_t deg, id; } degid;
static int cmp_degid(const void* a, const void* b) {   /* degree desc, id asc (C4) */
  const degid* x = (const degid*)a; const degid* y = (const degid*)b;
  if (x->deg != y->deg) return (x->deg < y->deg) - (x->deg > y->deg);
  return (x->id > y->id) - (x->id < y->id);
}

static void node_ids(int32_t V, const int32_t* deg, int32_t* ids) {
  degid* t = (degid*)malloc(sizeof(degid) * (size_t)(V > 0 ? V : 1));
  for (int32_t v = 0; v < V; ++v) { t[v].deg = deg[v]; t[v].id = v; }
  qsort(t, (size_t)V, sizeof(degid), cmp_degid);
  for (int32_t v = 0; v < V; ++v) ids[v] = t[v].id;
  free(t);
}

/* ---------------------------------------------------------------------------
 * STGraphBase arrays of one snapshot (Fig. 3):
 *  - forward CSR = in-neighbours (rows = dst, cols = src ascending, C2/C3)
 *  - backward CSR = out-neighbours (rows = src, cols = dst ascending)
 *  - shared edge labels: eid = in-CSR position; out_eid[j] = in-CSR index of
 *    out-edge j (reading C6)
 *  - node_ids: vertices by degree desc, ties by id asc (C4/C5)
 *  - GCN normalisation (C1): default n_src = n_dst = in_deg^{-1/2}, 0^{-1/2}:=0;
 *    dgl_both: n_src = out_deg^{-1/2}, n_dst = in_deg^{-1/2}.
 * S: sorted unique keys (src,dst), n = |S|.
 * ------------------------------------------------------------------------- */
void orc_csr_build(int32_t V, int64_t n, const uint64_t* S, int32_t dgl_both,
                   int32_t* in_rowptr, int32_t* in_col,
                   int32_t* out_rowptr, int32_t* out_col, int32_t* out_eid,
                   int32_t* in_deg, int32_t* out_deg, int32_t* in_ids, int32_t* out_ids,
                   double* norm_src, double* norm_dst) {
  memset(in_deg, 0, sizeof(int32_t) * (size_t)V);
  memset(out_deg, 0, sizeof(int32_t) * (size_t)V);
  for (int64_t i = 0; i < n; ++i) { in_deg[kdst(S[i])]++; out_deg[ksrc(S[i])]++; }
  in_rowptr[0] = 0; out_rowptr[0] = 0;
  for (int32_t v = 0; v < V; ++v) {
    in_rowptr[v + 1] = in_rowptr[v] + in_deg[v];
    out_rowptr[v + 1] = out_rowptr[v] + out_deg[v];
  }
  /* out-CSR: S is already ordered by (src, dst) */
  for (int64_t i = 0; i < n; ++i) out_col[i] = kdst(S[i]);
  /* in-CSR: counting sort by dst, stable in src order => cols ascending */
  int32_t* fill = (int32_t*)calloc((size_t)(V > 0 ? V : 1), sizeof(int32_t));
  for (int64_t i = 0; i < n; ++i) {
    int32_t v = kdst(S[i]);
    in_col[in_rowptr[v] + fill[v]++] = ksrc(S[i]);
  }
  free(fill);
  /* shared edge labels: the in-CSR position of every out-edge (the row of v
   * is sorted ascending, so the position of u is found by bisection) */
  for (int32_t u = 0; u < V; ++u)
    for (int32_t j = out_rowptr[u]; j < out_rowptr[u + 1]; ++j) {
      int32_t v = out_col[j], lo = in_rowptr[v], hi = in_rowptr[v + 1];
      while (lo < hi) {
        int32_t mid = lo + (hi - lo) / 2;
        if (in_col[mid] < u) lo = mid + 1; else hi = mid;
      }
      out_eid[j] = (lo < in_rowptr[v + 1] && in_col[lo] == u) ? lo : -1;
    }
  node_ids(V, in_deg, in_ids);    /* forward pass order: in-degree */
  node_ids(V, out_deg, out_ids);  /* backward pass order: out-degree */
  for (int32_t v = 0; v < V; ++v) {
    double di = in_deg[v] > 0 ? 1.0 / sqrt((double)in_deg[v]) : 0.0;
    double dout = out_deg[v] > 0 ? 1.0 / sqrt((double)out_deg[v]) : 0.0;
    norm_dst[v] = di;
    norm_src[v] = dgl_both ? dout : di;
  }
}

/* ---------------------------------------------------------------------------
 * Vertex-centric GCN aggregation (north_star):
 *   y[v,:] = sum_{j in row v, u = col[j]} nrow[v] * ncol[u] * x[u,:]
 * forward : in-CSR,  nrow = n_dst, ncol = n_src  (y_v = sum_{u in N_in(v)} c_uv x_u)
 * backward: out-CSR, nrow = n_src, ncol = n_dst  (the exact transpose, a6)
 * ncol may be NULL (treated as 1).  Rows in ascending order, neighbours
 * ascending, fp64.
 * ------------------------------------------------------------------------- */
void orc_aggregate(int32_t R, const int32_t* rowptr, const int32_t* col,
                   const double* nrow, const double* ncol, int32_t W,
                   const double* x, double* y) {
#ifdef _OPENMP
#pragma omp parallel for schedule(dynamic, 1024)
#endif
  for (int32_t v = 0; v < R; ++v) {
    double* yv = y + (int64_t)v * W;
    for (int32_t k = 0; k < W; ++k) yv[k] = 0.0;
    for (int32_t j = rowptr[v]; j < rowptr[v + 1]; ++j) {
      int32_t u = col[j];
      double c = nrow[v] * (ncol ? ncol[u] : 1.0);
      const double* xu = x + (int64_t)u * W;
      for (int32_t k = 0; k < W; ++k) yv[k] += c * xu[k];
    }
  }
}

/* ---------------------------------------------------------------------------
 * Edge-weighted aggregation (edge features; the
 * weights PyG-T's TGCN passes to its GCN, reading C21), written over the edge
 * SET itself (no CSR, no labels): S sorted unique keys (src,dst), w[k] = the
 * weight of edge S[k].
 *   forward : y[v,:]  += n[v] * w(u,v) * n[u] * x[u,:]   for every (u,v) in S
 *   backward: gx[u,:] += n[u] * w(u,v) * n[v] * gy[v,:]  for every (u,v) in S
 * (nrow = the scale of the output vertex, ncol = the scale of the input vertex;
 * ncol may be NULL = 1).  y has V rows and is overwritten.  fp64.
 * ------------------------------------------------------------------------- */
void orc_aggregate_edges(int32_t V, int64_t n, const uint64_t* S, const double* w, const double* nrow,
                         const double* ncol, int32_t backward, int32_t W, const double* x, double* y) {
  for (int64_t i = 0; i < (int64_t)V * W; ++i) y[i] = 0.0;
  for (int64_t k = 0; k < n; ++k) {
    int32_t u = ksrc(S[k]), v = kdst(S[k]);
    int32_t o = backward ? u : v, in = backward ? v : u;      /* output row, input row */
    double c = nrow[o] * w[k] * (ncol ? ncol[in] : 1.0);
    for (int32_t j = 0; j < W; ++j) y[(int64_t)o * W + j] += c * x[(int64_t)in * W + j];
  }
}

/* Weighted GCN normalisation (PyG gcn_norm with edge weights):
 * deg[v] = sum_{(u,v) in S} w(u,v);  norm[v] = deg^-1/2, 0 if deg <= 0. */
void orc_weighted_norm(int32_t V, int64_t n, const uint64_t* S, const double* w, double* norm) {
  for (int32_t v = 0; v < V; ++v) norm[v] = 0.0;
  for (int64_t k = 0; k < n; ++k) norm[kdst(S[k])] += w[k];
  for (int32_t v = 0; v < V; ++v) norm[v] = norm[v] > 0.0 ? 1.0 / sqrt(norm[v]) : 0.0;
}

/* ---------------------------------------------------------------------------
 * DTDG snapshots (base graph + list of edge additions/deletions).
 * S_t = (S_{t-1} \ D_t) ∪ A_t.  S sorted unique; A, D arbitrary multisets.
 * out capacity: n + na.  Returns |S_t|.
 * ------------------------------------------------------------------------- */
int64_t orc_set_apply(const uint64_t* S, int64_t n, const uint64_t* D, int64_t nd,
                      const uint64_t* A, int64_t na, uint64_t* out) {
  uint64_t* d = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(nd > 0 ? nd : 1));
  memcpy(d, D, sizeof(uint64_t) * (size_t)nd);
  int64_t m = sort_unique(d, nd);
  int64_t k = 0;
  for (int64_t i = 0; i < n; ++i)
    if (!contains(d, m, S[i])) out[k++] = S[i];
  for (int64_t i = 0; i < na; ++i) out[k++] = A[i];
  free(d);
  return sort_unique(out, k);
}

/* Snapshot from the event-window definition: the distinct (src,dst)
 * pairs of events [lo, hi).  out capacity hi-lo.  Returns the count. */
int64_t orc_window_set(const int32_t* ev_src, const int32_t* ev_dst, int64_t lo, int64_t hi,
                       uint64_t* out) {
  int64_t k = 0;
  for (int64_t e = lo; e < hi; ++e) out[k++] = mk(ev_src[e], ev_dst[e]);
  return sort_unique(out, k);
}

/* Effective deltas (reading C9, set semantics, add wins):
 *   A'_t = A_t \ S_{t-1};   D'_t = (D_t \ A_t) ∩ S_{t-1} \ I_loops
 * so that S_t = (S_{t-1} \ D'_t) ∪ A'_t and the reverse S_{t-1} = (S_t \ A'_t) ∪ D'_t
 * is exact.  pinned_loops: self-loops are never deleted (STG_SELF_LOOPS).
 * outA capacity na, outD capacity nd; counts returned through na_out/nd_out. */
void orc_effective_deltas(const uint64_t* Sprev, int64_t n, const uint64_t* A, int64_t na,
                          const uint64_t* D, int64_t nd, int32_t pinned_loops,
                          uint64_t* outA, int64_t* na_out, uint64_t* outD, int64_t* nd_out) {
  uint64_t* a = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(na > 0 ? na : 1));
  memcpy(a, A, sizeof(uint64_t) * (size_t)na);
  int64_t ma = sort_unique(a, na);
  int64_t ka = 0;
  for (int64_t i = 0; i < ma; ++i)
    if (!contains(Sprev, n, a[i])) outA[ka++] = a[i];
  uint64_t* d = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(nd > 0 ? nd : 1));
  memcpy(d, D, sizeof(uint64_t) * (size_t)nd);
  int64_t md = sort_unique(d, nd);
  int64_t kd = 0;
  for (int64_t i = 0; i < md; ++i) {
    if (pinned_loops && ksrc(d[i]) == kdst(d[i])) continue;
    if (contains(a, ma, d[i])) continue;
    if (contains(Sprev, n, d[i])) outD[kd++] = d[i];
  }
  free(a); free(d);
  *na_out = ka; *nd_out = kd;
}

/* ---------------------------------------------------------------------------
 * TGCN step (reading C13-C15; SURVEY §8(c) equations).  Row-major fp64.
 *   P  = X·W                      X [V,F], W [F,3H]  (P = [P_z|P_r|P_h])
 *   C  = Â·P + 1·bᵀ               Â_vu = n_dst[v]·n_src[u] over the in-CSR
 *   a_z = C_z·L_z¹ + H·L_z² + l_z ;  Z = σ(a_z)
 *   a_r = C_r·L_r¹ + H·L_r² + l_r ;  R = σ(a_r)
 *   a_h = C_h·L_h¹ + (R⊙H)·L_h² + l_h ;  Ĥ = tanh(a_h)
 *   H' = Z⊙H + (1−Z)⊙Ĥ
 * L [3][2H][H] (gate g rows 0..H-1 = L_g¹, rows H..2H-1 = L_g²), l [3][H].
 * Outputs C [V,3H], Z,R,Hh [V,H], Hn [V,H].
 * ------------------------------------------------------------------------- */
static double sigm(double a) { return 1.0 / (1.0 + exp(-a)); }

void orc_tgcn_fwd(int32_t V, int32_t F, int32_t H,
                  const int32_t* in_rowptr, const int32_t* in_col,
                  const double* n_src, const double* n_dst,
                  const double* X, const double* Hp,
                  const double* W, const double* b, const double* L, const double* l,
                  double* C, double* Z, double* R, double* Hh, double* Hn) {
  const int32_t H3 = 3 * H;
  double* P = (double*)calloc((size_t)V * H3 + 1, sizeof(double));
#ifdef _OPENMP
#pragma omp parallel for schedule(static)
#endif
  for (int32_t v = 0; v < V; ++v)
    for (int32_t c = 0; c < H3; ++c) {
      double s = 0.0;
      for (int32_t f = 0; f < F; ++f) s += X[(int64_t)v * F + f] * W[(int64_t)f * H3 + c];
      P[(int64_t)v * H3 + c] = s;
    }
  orc_aggregate(V, in_rowptr, in_col, n_dst, n_src, H3, P, C);
  for (int64_t i = 0; i < (int64_t)V * H3; ++i) C[i] += b[i % H3];
  free(P);
  const double* Lz = L;  const double* Lr = L + 2 * H * H;  const double* Lh = L + 4 * H * H;
#ifdef _OPENMP
#pragma omp parallel for schedule(static)
#endif
  for (int32_t v = 0; v < V; ++v) {
    const double* cz = C + (int64_t)v * H3;  const double* cr = cz + H;  const double* ch = cz + 2 * H;
    const double* hv = Hp + (int64_t)v * H;
    for (int32_t j = 0; j < H; ++j) {
      double az = l[j], ar = l[H + j];
      for (int32_t i = 0; i < H; ++i) {
        az += cz[i] * Lz[i * H + j] + hv[i] * Lz[(H + i) * H + j];
        ar += cr[i] * Lr[i * H + j] + hv[i] * Lr[(H + i) * H + j];
      }
      Z[(int64_t)v * H + j] = sigm(az);
      R[(int64_t)v * H + j] = sigm(ar);
    }
    for (int32_t j = 0; j < H; ++j) {
      double ah = l[2 * H + j];
      for (int32_t i = 0; i < H; ++i)
        ah += ch[i] * Lh[i * H + j] + R[(int64_t)v * H + i] * hv[i] * Lh[(H + i) * H + j];
      Hh[(int64_t)v * H + j] = tanh(ah);
    }
    for (int32_t j = 0; j < H; ++j) {
      double z = Z[(int64_t)v * H + j];
      Hn[(int64_t)v * H + j] = z * hv[j] + (1.0 - z) * Hh[(int64_t)v * H + j];
    }
  }
}

/* ---------------------------------------------------------------------------
 * TGCN step backward (chain rule of orc_tgcn_fwd), given
 * G = dℓ/dH' (total).  Recomputes Z, R, Ĥ from the saved {H, C} (A8).
 *   dZ = G⊙(H−Ĥ);  dĤ = G⊙(1−Z);  dH = G⊙Z
 *   da_h = dĤ⊙(1−Ĥ²); dL_h¹ += C_hᵀda_h; dL_h² += (R⊙H)ᵀda_h; dl_h += 1ᵀda_h
 *   dC_h = da_h·L_h¹ᵀ; dRH = da_h·L_h²ᵀ; dR = dRH⊙H; dH += dRH⊙R
 *   da_r = dR⊙R⊙(1−R); dL_r¹ += C_rᵀda_r; dL_r² += Hᵀda_r; dl_r += 1ᵀda_r
 *   dC_r = da_r·L_r¹ᵀ; dH += da_r·L_r²ᵀ
 *   da_z = dZ⊙Z⊙(1−Z); dL_z¹ += C_zᵀda_z; dL_z² += Hᵀda_z; dl_z += 1ᵀda_z
 *   dC_z = da_z·L_z¹ᵀ; dH += da_z·L_z²ᵀ
 *   db += 1ᵀdC;  dP = Âᵀ·dC (out-CSR of snapshot t);  dW += Xᵀ·dP;  dH_{t−1} = dH
 * Gradients are ACCUMULATED (+=) into dW, db, dL, dl.
 * ------------------------------------------------------------------------- */
void orc_tgcn_bwd(int32_t V, int32_t F, int32_t H,
                  const int32_t* out_rowptr, const int32_t* out_col,
                  const double* n_src, const double* n_dst,
                  const double* X, const double* Hp, const double* C, const double* G,
                  const double* L,
                  const double* Z, const double* R, const double* Hh,
                  double* dHp, double* dW, double* db, double* dL, double* dl) {
  const int32_t H3 = 3 * H;
  const double* Lz = L;  const double* Lr = L + 2 * H * H;  const double* Lh = L + 4 * H * H;
  double* dC = (double*)calloc((size_t)V * H3 + 1, sizeof(double));
  /* (the OpenMP timing build, bench.py's all-core baseline, gives every thread its
   * own row scratch and reduces dL / dl over threads; the plain build runs the
   * loop below as written, rows in ascending order) */
#ifdef _OPENMP
#pragma omp parallel
#endif
  {
  double* dah = (double*)malloc(sizeof(double) * (size_t)(H + 1));
  double* dar = (double*)malloc(sizeof(double) * (size_t)(H + 1));
  double* daz = (double*)malloc(sizeof(double) * (size_t)(H + 1));
  double* dR = (double*)malloc(sizeof(double) * (size_t)(H + 1));
  double* dRH = (double*)malloc(sizeof(double) * (size_t)(H + 1));
#ifdef _OPENMP
#pragma omp for schedule(static) reduction(+ : dL[:6 * H * H], dl[:3 * H])
#endif
  for (int32_t v = 0; v < V; ++v) {
    double* dLz = dL;  double* dLr = dL + 2 * H * H;  double* dLh = dL + 4 * H * H;
    const double* g = G + (int64_t)v * H;  const double* hv = Hp + (int64_t)v * H;
    const double* z = Z + (int64_t)v * H;  const double* r = R + (int64_t)v * H;
    const double* hh = Hh + (int64_t)v * H;
    const double* cz = C + (int64_t)v * H3;  const double* cr = cz + H;  const double* ch = cz + 2 * H;
    double* dh = dHp + (int64_t)v * H;
    double* dcz = dC + (int64_t)v * H3;  double* dcr = dcz + H;  double* dch = dcz + 2 * H;
    for (int32_t j = 0; j < H; ++j) {
      dh[j] = g[j] * z[j];
      double dZ = g[j] * (hv[j] - hh[j]);
      double dHh = g[j] * (1.0 - z[j]);
      dah[j] = dHh * (1.0 - hh[j] * hh[j]);
      daz[j] = dZ * z[j] * (1.0 - z[j]);
    }
    for (int32_t i = 0; i < H; ++i) {          /* dC_h, dRH = da_h·L_hᵀ */
      double s1 = 0.0, s2 = 0.0;
      for (int32_t j = 0; j < H; ++j) { s1 += dah[j] * Lh[i * H + j]; s2 += dah[j] * Lh[(H + i) * H + j]; }
      dch[i] = s1; dRH[i] = s2;
    }
    for (int32_t i = 0; i < H; ++i) {
      dR[i] = dRH[i] * hv[i];
      dh[i] += dRH[i] * r[i];
      dar[i] = dR[i] * r[i] * (1.0 - r[i]);
    }
    for (int32_t i = 0; i < H; ++i) {          /* dC_r, dC_z and the H-paths */
      double sr1 = 0.0, sr2 = 0.0, sz1 = 0.0, sz2 = 0.0;
      for (int32_t j = 0; j < H; ++j) {
        sr1 += dar[j] * Lr[i * H + j];  sr2 += dar[j] * Lr[(H + i) * H + j];
        sz1 += daz[j] * Lz[i * H + j];  sz2 += daz[j] * Lz[(H + i) * H + j];
      }
      dcr[i] = sr1; dcz[i] = sz1;
      dh[i] += sr2 + sz2;
    }
    for (int32_t i = 0; i < H; ++i)            /* parameter gradients */
      for (int32_t j = 0; j < H; ++j) {
        dLh[i * H + j] += ch[i] * dah[j];
        dLh[(H + i) * H + j] += r[i] * hv[i] * dah[j];
        dLr[i * H + j] += cr[i] * dar[j];
        dLr[(H + i) * H + j] += hv[i] * dar[j];
        dLz[i * H + j] += cz[i] * daz[j];
        dLz[(H + i) * H + j] += hv[i] * daz[j];
      }
    for (int32_t j = 0; j < H; ++j) { dl[j] += daz[j]; dl[H + j] += dar[j]; dl[2 * H + j] += dah[j]; }
  }
  free(dah); free(dar); free(daz); free(dR); free(dRH);
  }
  for (int64_t i = 0; i < (int64_t)V * H3; ++i) db[i % H3] += dC[i];
  double* dP = (double*)calloc((size_t)V * H3 + 1, sizeof(double));
  orc_aggregate(V, out_rowptr, out_col, n_src, n_dst, H3, dC, dP);   /* Âᵀ·dC */
#ifdef _OPENMP
#pragma omp parallel for schedule(static) reduction(+ : dW[:F * H3])
#endif
  for (int32_t v = 0; v < V; ++v)
    for (int32_t f = 0; f < F; ++f) {
      double xv = X[(int64_t)v * F + f];
      for (int32_t c = 0; c < H3; ++c) dW[(int64_t)f * H3 + c] += xv * dP[(int64_t)v * H3 + c];
    }
  free(dP); free(dC);
}

/* ---------------------------------------------------------------------------
 * Timing surrogate head (not on the hot path, A15):
 *   ŷ_v = Σ_k ReLU(H_vk)·w_o[k] + b_o;  ℓ = mean_v (ŷ_v − y_v)²
 * Returns ℓ; writes dH = dℓ/dH and ACCUMULATES dw_o, db_o.
 * ------------------------------------------------------------------------- */
double orc_mse_head(int32_t V, int32_t H, const double* Hn, const double* y,
                    const double* w_o, double b_o, double* dH, double* dw_o, double* db_o) {
  double loss = 0.0;
  for (int32_t v = 0; v < V; ++v) {
    const double* h = Hn + (int64_t)v * H;
    double yh = b_o;
    for (int32_t k = 0; k < H; ++k) yh += (h[k] > 0.0 ? h[k] : 0.0) * w_o[k];
    double e = yh - y[v];
    loss += e * e;
    double g = 2.0 * e / (double)V;
    for (int32_t k = 0; k < H; ++k) {
      dH[(int64_t)v * H + k] = h[k] > 0.0 ? g * w_o[k] : 0.0;
      dw_o[k] += g * (h[k] > 0.0 ? h[k] : 0.0);
    }
    *db_o += g;
  }
  return loss / (double)V;
}

/* ---------------------------------------------------------------------------
 * Original T-GCN cell (the model the paper cites for TGCN,
 * P:L58, whose graph convolution acts on the concatenation [X, H] — reading C13
 * alternative).  Written in the order of that formulation (aggregate first):
 *   XH  = [X | H]                      [V, F+H]
 *   G   = (Â·XH)·Wg + bg               Wg [F+H, 2H] (columns r | u)
 *   r   = σ(G[:, :H]),  u = σ(G[:, H:])
 *   XR  = [X | r⊙H]
 *   Cc  = tanh((Â·XR)·Wc + bc)         Wc [F+H, H]
 *   H'  = u⊙H + (1−u)⊙Cc
 * Â_vu = n_dst[v]·n_src[u] over the in-CSR (the same GCN normalisation, C1).
 * Outputs R, U, Cc, Hn [V,H].  fp64, row-major.
 * ------------------------------------------------------------------------- */
static void cat_rows(int32_t V, int32_t F, int32_t H, const double* X, const double* Hm, const double* mul,
                     double* out) {
  for (int32_t v = 0; v < V; ++v) {
    for (int32_t f = 0; f < F; ++f) out[(int64_t)v * (F + H) + f] = X[(int64_t)v * F + f];
    for (int32_t j = 0; j < H; ++j)
      out[(int64_t)v * (F + H) + F + j] = Hm[(int64_t)v * H + j] * (mul ? mul[(int64_t)v * H + j] : 1.0);
  }
}

static void matmul(int32_t V, int32_t K, int32_t N, const double* A, const double* W, const double* bias,
                   double* out) {
  for (int32_t v = 0; v < V; ++v)
    for (int32_t c = 0; c < N; ++c) {
      double s = bias ? bias[c] : 0.0;
      for (int32_t k = 0; k < K; ++k) s += A[(int64_t)v * K + k] * W[(int64_t)k * N + c];
      out[(int64_t)v * N + c] = s;
    }
}

void orc_tgcn2_fwd(int32_t V, int32_t F, int32_t H, const int32_t* in_rowptr, const int32_t* in_col,
                   const double* n_src, const double* n_dst, const double* X, const double* Hp,
                   const double* Wg, const double* bg, const double* Wc, const double* bc,
                   double* R, double* U, double* Cc, double* Hn) {
  const int32_t K = F + H;
  double* cat = (double*)malloc(sizeof(double) * ((size_t)V * K + 1));
  double* agg = (double*)malloc(sizeof(double) * ((size_t)V * K + 1));
  double* G = (double*)malloc(sizeof(double) * ((size_t)V * 2 * H + 1));
  cat_rows(V, F, H, X, Hp, NULL, cat);
  orc_aggregate(V, in_rowptr, in_col, n_dst, n_src, K, cat, agg);
  matmul(V, K, 2 * H, agg, Wg, bg, G);
  for (int32_t v = 0; v < V; ++v)
    for (int32_t j = 0; j < H; ++j) {
      R[(int64_t)v * H + j] = sigm(G[(int64_t)v * 2 * H + j]);
      U[(int64_t)v * H + j] = sigm(G[(int64_t)v * 2 * H + H + j]);
    }
  cat_rows(V, F, H, X, Hp, R, cat);
  orc_aggregate(V, in_rowptr, in_col, n_dst, n_src, K, cat, agg);
  matmul(V, K, H, agg, Wc, bc, Cc);
  for (int64_t i = 0; i < (int64_t)V * H; ++i) {
    Cc[i] = tanh(Cc[i]);
    Hn[i] = U[i] * Hp[i] + (1.0 - U[i]) * Cc[i];
  }
  free(cat); free(agg); free(G);
}

/* Backward of orc_tgcn2_fwd by the chain rule, given G = dℓ/dH' (total):
 *   du = G⊙(H−Cc); dCc = G⊙(1−u); dH = G⊙u
 *   dzc = dCc⊙(1−Cc²);  dWc += (Â·XR)ᵀ dzc;  dbc += 1ᵀdzc
 *   dXR = Âᵀ·(dzc·Wcᵀ);  d(r⊙H) = dXR[:, F:];  dr = d(r⊙H)⊙H;  dH += d(r⊙H)⊙r
 *   dzg = [dr⊙r(1−r) | du⊙u(1−u)];  dWg += (Â·XH)ᵀ dzg;  dbg += 1ᵀdzg
 *   dXH = Âᵀ·(dzg·Wgᵀ);  dH += dXH[:, F:]
 * Âᵀ runs over the out-CSR (rows = sources; ncol = n_dst of the destinations).
 * Gradients accumulate (+=); dHp is overwritten. */
void orc_tgcn2_bwd(int32_t V, int32_t F, int32_t H, const int32_t* in_rowptr, const int32_t* in_col,
                   const int32_t* out_rowptr, const int32_t* out_col, const double* n_src, const double* n_dst,
                   const double* X, const double* Hp, const double* Wg, const double* Wc, const double* R,
                   const double* U, const double* Cc, const double* Gd, double* dHp, double* dWg, double* dbg,
                   double* dWc, double* dbc) {
  const int32_t K = F + H, H2 = 2 * H;
  double* cat = (double*)malloc(sizeof(double) * ((size_t)V * K + 1));
  double* agg = (double*)malloc(sizeof(double) * ((size_t)V * K + 1));
  double* dz = (double*)calloc((size_t)V * H2 + 1, sizeof(double));
  double* dcat = (double*)malloc(sizeof(double) * ((size_t)V * K + 1));
  double* dxr = (double*)malloc(sizeof(double) * ((size_t)V * K + 1));
  double* du = (double*)malloc(sizeof(double) * ((size_t)V * H + 1));
  for (int64_t i = 0; i < (int64_t)V * H; ++i) {
    du[i] = Gd[i] * (Hp[i] - Cc[i]);
    dz[i] = Gd[i] * (1.0 - U[i]) * (1.0 - Cc[i] * Cc[i]);      /* dzc, [V,H] */
    dHp[i] = Gd[i] * U[i];
  }
  /* candidate: dWc, dbc, dXR */
  cat_rows(V, F, H, X, Hp, R, cat);
  orc_aggregate(V, in_rowptr, in_col, n_dst, n_src, K, cat, agg);
  for (int32_t v = 0; v < V; ++v)
    for (int32_t c = 0; c < H; ++c) {
      const double d = dz[(int64_t)v * H + c];
      dbc[c] += d;
      for (int32_t k = 0; k < K; ++k) dWc[(int64_t)k * H + c] += agg[(int64_t)v * K + k] * d;
    }
  for (int32_t v = 0; v < V; ++v)
    for (int32_t k = 0; k < K; ++k) {
      double s = 0.0;
      for (int32_t c = 0; c < H; ++c) s += dz[(int64_t)v * H + c] * Wc[(int64_t)k * H + c];
      dcat[(int64_t)v * K + k] = s;
    }
  orc_aggregate(V, out_rowptr, out_col, n_src, n_dst, K, dcat, dxr);
  double* dzg = (double*)calloc((size_t)V * H2 + 1, sizeof(double));
  for (int32_t v = 0; v < V; ++v)
    for (int32_t j = 0; j < H; ++j) {
      const int64_t i = (int64_t)v * H + j;
      const double drh = dxr[(int64_t)v * K + F + j];
      const double dr = drh * Hp[i];
      dHp[i] += drh * R[i];
      dzg[(int64_t)v * H2 + j] = dr * R[i] * (1.0 - R[i]);
      dzg[(int64_t)v * H2 + H + j] = du[i] * U[i] * (1.0 - U[i]);
    }
  /* gates: dWg, dbg, dXH */
  cat_rows(V, F, H, X, Hp, NULL, cat);
  orc_aggregate(V, in_rowptr, in_col, n_dst, n_src, K, cat, agg);
  for (int32_t v = 0; v < V; ++v)
    for (int32_t c = 0; c < H2; ++c) {
      const double d = dzg[(int64_t)v * H2 + c];
      dbg[c] += d;
      for (int32_t k = 0; k < K; ++k) dWg[(int64_t)k * H2 + c] += agg[(int64_t)v * K + k] * d;
    }
  for (int32_t v = 0; v < V; ++v)
    for (int32_t k = 0; k < K; ++k) {
      double s = 0.0;
      for (int32_t c = 0; c < H2; ++c) s += dzg[(int64_t)v * H2 + c] * Wg[(int64_t)k * H2 + c];
      dcat[(int64_t)v * K + k] = s;
    }
  orc_aggregate(V, out_rowptr, out_col, n_src, n_dst, K, dcat, dxr);
  for (int32_t v = 0; v < V; ++v)
    for (int32_t j = 0; j < H; ++j) dHp[(int64_t)v * H + j] += dxr[(int64_t)v * K + F + j];
  free(cat); free(agg); free(dz); free(dcat); free(dxr); free(du); free(dzg);
}
