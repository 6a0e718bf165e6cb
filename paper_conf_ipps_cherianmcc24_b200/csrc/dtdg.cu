// dtdg.cu — discrete-time dynamic graph with on-demand snapshots
// (GPMAGraph behaviour; Algorithm 2 Get-Graph, P:L210-216, L253;
// Get-Backward-Graph).  The GPMA gapped arrays are replaced by
// dense sorted CSRs rebuilt per step with a scan + merge delta-apply
// (graph.cu).  Deltas are normalised once, here, to the effective sets
// A'_t = A_t \ S_{t-1}, D'_t = (D_t \ A_t) ∩ S_{t-1} (reading C9) so that every
// step is exactly reversible and every E_t is known without a host sync.
#include <vector>

#include <memory>

#include "graph.cuh"
#include "prims.cuh"

namespace stg {

__global__ void k_pack_batch(const int32_t* __restrict__ src, const int32_t* __restrict__ dst, int64_t n, int32_t V,
                             int nb, uint64_t* __restrict__ keys, int32_t* __restrict__ bad) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    int32_t a = src[i], b = dst[i];
    if ((unsigned)a >= (unsigned)V || (unsigned)b >= (unsigned)V) { atomicExch(bad, 1); a = b = 0; }
    keys[i] = ((uint64_t)a << nb) | (uint64_t)b;
  }
}

__device__ __forceinline__ int64_t lb64(const uint64_t* a, int64_t n, uint64_t k) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (a[mid] < k) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// A' = A \ S
struct NotInS {
  const uint64_t* a;
  const uint64_t* S;
  int64_t ns;
  __device__ int64_t operator()(int64_t i) const {
    uint64_t k = a[i];
    int64_t p = lb64(S, ns, k);
    return !(p < ns && S[p] == k);
  }
};
// D' = (D \ A) ∩ S, minus self-loops when they are pinned
struct DelEff {
  const uint64_t* d;
  const uint64_t* A;
  int64_t na;
  const uint64_t* S;
  int64_t ns;
  int nb;
  int pinned;
  __device__ int64_t operator()(int64_t i) const {
    uint64_t k = d[i];
    if (pinned && (k >> nb) == (k & ((uint64_t(1) << nb) - 1))) return 0;
    int64_t p = lb64(A, na, k);
    if (p < na && A[p] == k) return 0;
    p = lb64(S, ns, k);
    return p < ns && S[p] == k;
  }
};
struct CompactOut {
  const uint64_t* in;
  uint64_t* out;
  __device__ void operator()(int64_t i, int64_t ex, int64_t f) const {
    if (f) out[ex] = in[i];
  }
};

__global__ void k_mark_deleted(const uint64_t* __restrict__ D, int64_t nd, const uint64_t* __restrict__ S, int64_t ns,
                               int32_t* __restrict__ delflag) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nd; i += (int64_t)gridDim.x * blockDim.x)
    delflag[lb64(S, ns, D[i])] = 1;
}
struct KeepIn {
  const int32_t* delflag;
  __device__ int64_t operator()(int64_t i) const { return 1 - delflag[i]; }
};
struct KeepOut {
  const uint64_t* S;
  const uint64_t* A;
  int64_t na;
  int64_t* keep_ex;
  uint64_t* out;
  __device__ void operator()(int64_t i, int64_t ex, int64_t keep) const {
    keep_ex[i] = ex;
    if (keep) out[ex + lb64(A, na, S[i])] = S[i];
  }
};
__global__ void k_place_adds(const uint64_t* __restrict__ A, int64_t na, const uint64_t* __restrict__ S, int64_t ns,
                             const int64_t* __restrict__ keep_ex, uint64_t* __restrict__ out) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < na; j += (int64_t)gridDim.x * blockDim.x)
    out[j + keep_ex[lb64(S, ns, A[j])]] = A[j];
}
__global__ void k_swap_pack(const uint64_t* __restrict__ in, int64_t n, int nb, uint64_t* __restrict__ out) {
  const uint64_t mask = (uint64_t(1) << nb) - 1;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t k = in[i];
    out[i] = ((k & mask) << nb) | (k >> nb);
  }
}

static inline unsigned grid_n(int64_t n) {
  int64_t b = ceil_div(n > 0 ? n : 1, 256);
  return (unsigned)(b < 148 * 16 ? b : 148 * 16);
}

}  // namespace stg

using namespace stg;

struct stg_dtdg {
  int32_t V = 0, T = 0, nb = 1;
  uint32_t flags = 0;
  std::vector<int64_t> E;                          // E_t (edges held: the local block's if sharded)
  std::vector<int64_t> a_off, d_off;               // offsets into the delta arrays, [T+1]
  DArray<uint64_t> add_out, add_in, del_out, del_in;  // effective deltas, packed, sorted per direction
  // row-block sharding: the deltas above are those of the local
  // block; the whole-graph effective deltas (src-major) keep the whole-graph
  // degrees of every slot current for the GCN norms
  bool sharded = false;
  int32_t rb = 0, re = 0;
  int64_t E0_global = 0;
  std::vector<int64_t> ga_off, gd_off;
  DArray<uint64_t> gadd, gdel;
  Snapshot slot[5];                                // 0 = base, 1-2 = forward pair, 3-4 = backward pair
  // NaiveGraph mode (STG_NAIVE): every snapshot
  // materialised at create, Get-Graph is a lookup
  std::vector<std::unique_ptr<Snapshot>> naive;
  int head_f = -1, head_b = -1;
  DArray<int4> touch_in, touch_out;
  BuildWs* ws = nullptr;
  AggWs agg;
  ~stg_dtdg() { buildws_destroy(ws); }

  DirDelta dir(int32_t t, bool in_order, bool reverse) const {
    const uint64_t* A = (in_order ? add_in.p : add_out.p) + a_off[t];
    const uint64_t* D = (in_order ? del_in.p : del_out.p) + d_off[t];
    int64_t na = a_off[t + 1] - a_off[t], nd = d_off[t + 1] - d_off[t];
    if (!reverse) return DirDelta{A, na, D, nd};
    return DirDelta{D, nd, A, na};
  }

  // one delta step from slot `from` (time t0) to slot `to` (time t0 ± 1) of the
  // CSR directions in `parts`; the whole-graph degrees (norms) always follow
  stg_status step(int from, int to, int dirn, uint32_t parts, cudaStream_t s) {
    return step_snap(slot[from], slot[to], dirn, parts, s);
  }
  stg_status step_snap(const Snapshot& sf, Snapshot& st, int dirn, uint32_t parts, cudaStream_t s) {
    ProfScope prof(PH_SNAP_STEP, s);
    const int32_t t0 = sf.t;
    const int32_t t1 = t0 + dirn;
    const int32_t td = dirn > 0 ? t1 : t0;       // batch applied (forward) or undone (reverse)
    const bool rev = dirn < 0;
    const uint64_t* ga = sharded ? gadd.p : add_out.p;
    const uint64_t* gd = sharded ? gdel.p : del_out.p;
    const std::vector<int64_t>& gao = sharded ? ga_off : a_off;
    const std::vector<int64_t>& gdo = sharded ? gd_off : d_off;
    // the whole-graph degrees (norms) follow inside the first direction's pass
    const GDegStep gdeg{DirDelta{ga + gao[td], gao[td + 1] - gao[td], gd + gdo[td], gdo[td + 1] - gdo[td]},
                        rev ? -1 : 1, sf.gin_deg.p, sf.gout_deg.p, st.gin_deg.p, st.gout_deg.p};
    return apply_delta(sf, st, dir(td, true, rev), dir(td, false, rev), E[t1], t1, touch_in.p,
                       touch_out.p, *ws, s, parts & (PART_IN | PART_OUT), &gdeg);
  }

  // Walk from the best cached slot to t, writing into the pair {p0, p0+1}, for
  // the CSR directions in `parts` (the starting slot is completed first by a
  // transpose if it lacks one of them); labels (PART_EID) are added at the end.
  stg_status walk(int32_t t, int p0, uint32_t parts, int& out, cudaStream_t s) {
    ProfScope prof(PH_SNAPSHOT, s);
    int cands[3] = {p0 == 1 ? head_f : head_b, p0 == 1 ? head_b : head_f, 0};
    int best = -1;
    int64_t bd = INT64_MAX;
    for (int c : cands) {
      if (c < 0) continue;
      int64_t d = slot[c].t > t ? slot[c].t - t : t - slot[c].t;
      if (d < bd) { bd = d; best = c; }
    }
    int cur = best;
    const uint32_t dirs = parts & (PART_IN | PART_OUT);
    if (slot[cur].t != t || (slot[cur].parts & dirs) != dirs)
      STG_TRY(complete_parts(slot[cur], dirs, *ws, s));
    while (slot[cur].t != t) {
      int to = (cur == p0) ? p0 + 1 : p0;
      STG_TRY(step(cur, to, slot[cur].t < t ? 1 : -1, dirs, s));
      cur = to;
    }
    STG_TRY(complete_parts(slot[cur], parts, *ws, s));
    out = cur;
    return STG_OK;
  }

  stg_status get(int32_t t, bool backward, uint32_t parts, cudaStream_t s, stg_csr_view* v) {
    if (!naive.empty()) {                          // NaiveGraph: every part of every t is stored
      naive[t]->view(v, &agg);
      return STG_OK;
    }
    int idx = -1;
    if (!backward) {
      if (t == 0 && head_f < 0) {
        idx = 0;
        ProfScope prof(PH_SNAPSHOT, s);
        STG_TRY(complete_parts(slot[0], parts, *ws, s));
      } else {
        STG_TRY(walk(t, 1, parts, idx, s));
        if (idx == 1 || idx == 2) head_f = idx;  // a 0-step hit on base/backward slots leaves the head
      }
    } else {
      if (head_f >= 0 && slot[head_f].t == t) idx = head_f;       // forward head is t itself
      else if (head_b >= 0 && slot[head_b].t == t) idx = head_b;
      else if (t == 0) idx = 0;
      if (idx >= 0) {
        ProfScope prof(PH_SNAPSHOT, s);
        STG_TRY(complete_parts(slot[idx], parts, *ws, s));
      } else {
        STG_TRY(walk(t, 3, parts, idx, s));
        if (idx >= 3) head_b = idx;
      }
    }
    slot[idx].view(v, &agg);
    return STG_OK;
  }
};

extern "C" {

stg_status stg_dtdg_create(int32_t V, int32_t T, int64_t E0, const int32_t* src0, const int32_t* dst0,
                           const int64_t* add_off, const int32_t* add_src, const int32_t* add_dst,
                           const int64_t* del_off, const int32_t* del_src, const int32_t* del_dst, uint32_t flags,
                           const stg_dist* dist, stg_stream_t stream, stg_dtdg** out) {
  if (!out) return fail(STG_ERR_INVALID_ARG, "stg_dtdg_create: out is NULL");
  *out = nullptr;
  if (V < 1 || V >= (1 << 30)) return fail(STG_ERR_OUT_OF_RANGE, "stg_dtdg_create: V=%d outside [1,2^30)", V);
  if (T < 1) return fail(STG_ERR_INVALID_ARG, "stg_dtdg_create: T=%d < 1", T);
  if (E0 < 0 || (E0 > 0 && (!src0 || !dst0))) return fail(STG_ERR_INVALID_ARG, "stg_dtdg_create: bad base edges");
  if (!add_off || !del_off) return fail(STG_ERR_INVALID_ARG, "stg_dtdg_create: add_off/del_off (host) are NULL");
  if (dist && (dist->row_begin < 0 || dist->row_end > V || dist->row_begin > dist->row_end))
    return fail(STG_ERR_INVALID_ARG, "stg_dtdg_create: row block [%d,%d) outside [0,%d]", dist->row_begin,
                dist->row_end, V);
  for (int32_t t = 0; t < T; ++t) {
    if (add_off[t + 1] < add_off[t] || del_off[t + 1] < del_off[t])
      return fail(STG_ERR_INVALID_ARG, "stg_dtdg_create: offsets decrease at t=%d", t);
  }
  if (add_off[1] != add_off[0] || del_off[1] != del_off[0])
    return fail(STG_ERR_INVALID_ARG, "stg_dtdg_create: batch 0 must be empty (S_0 is the base)");
  if ((add_off[T] > add_off[0] && (!add_src || !add_dst)) || (del_off[T] > del_off[0] && (!del_src || !del_dst)))
    return fail(STG_ERR_INVALID_ARG, "stg_dtdg_create: NULL delta arrays");
  if ((flags & STG_NAIVE) && dist && (dist->row_begin != 0 || dist->row_end != V))
    return fail(STG_ERR_INVALID_ARG, "stg_dtdg_create: STG_NAIVE is for unsharded graphs");
  const int loops = (flags & STG_SELF_LOOPS) ? 1 : 0;
  if (E0 + (loops ? V : 0) >= (int64_t(1) << 31)) return fail(STG_ERR_OUT_OF_RANGE, "stg_dtdg_create: E0 >= 2^31");
  cudaStream_t s = (cudaStream_t)stream;

  auto* g = new stg_dtdg();
  g->V = V; g->T = T; g->flags = flags;
  g->rb = dist ? dist->row_begin : 0;
  g->re = dist ? dist->row_end : V;
  g->sharded = g->rb != 0 || g->re != V;
  const bool shard = g->sharded;
  g->ws = buildws_create();
  BuildWs& ws = *g->ws;
  int nb = 1;
  while ((int64_t(1) << nb) < (int64_t)V) ++nb;
  g->nb = nb;
  const int nbits = 2 * nb;
  const int pinned = loops;
  stg_status st = STG_OK;
#define CK(x) do { if (st == STG_OK) st = (x); } while (0)
  DArray<int32_t> bad;
  DArray<int64_t> cnt;
  CK(bad.alloc(1)); CK(cnt.alloc(4));
  int64_t max_batch = 0;
  for (int32_t t = 1; t < T; ++t) {
    max_batch = std::max(max_batch, add_off[t + 1] - add_off[t]);
    max_batch = std::max(max_batch, del_off[t + 1] - del_off[t]);
  }
  // current edge set S (two buffers), batch buffers, scratch
  int64_t scap = E0 + (loops ? V : 0) + add_off[T] - add_off[0] + 1;
  DArray<uint64_t> S1, S2, A1, A2, D1, D2, Ae, De, Ain;
  DArray<int32_t> delflag;
  DArray<int64_t> keep_ex;
  CK(S1.alloc(scap)); CK(S2.alloc(scap));
  CK(A1.alloc(max_batch + 1)); CK(A2.alloc(max_batch + 1)); CK(D1.alloc(max_batch + 1)); CK(D2.alloc(max_batch + 1));
  CK(Ae.alloc(max_batch + 1)); CK(De.alloc(max_batch + 1)); CK(Ain.alloc(2 * max_batch + 2));
  CK(delflag.alloc(scap)); CK(keep_ex.alloc(scap + 1));
  if (st != STG_OK) { delete g; return st; }

  // ---- base S_0
  const int64_t n0 = E0 + (loops ? V : 0);
  cudaMemsetAsync(bad.p, 0, sizeof(int32_t), s);
  if (E0) { k_pack_batch<<<grid_n(E0), 256, 0, s>>>(src0, dst0, E0, V, nb, S1.p, bad.p); count_launch(); }
  if (loops) {
    // append (v,v) for every v via a packed iota
    std::vector<int32_t> h(V);
    for (int32_t v = 0; v < V; ++v) h[v] = v;
    DArray<int32_t> iv;
    CK(iv.alloc(V));
    if (st == STG_OK) {
      cudaMemcpyAsync(iv.p, h.data(), sizeof(int32_t) * V, cudaMemcpyHostToDevice, s);
      k_pack_batch<<<grid_n(V), 256, 0, s>>>(iv.p, iv.p, V, V, nb, S1.p + E0, bad.p);
      count_launch();
      cudaStreamSynchronize(s);
    }
  }
  uint64_t* S = S1.p;
  uint64_t* Salt = S2.p;
  CK(sort_unique_keys(&S, &Salt, n0, nbits, cnt.p, ws, s));
  int64_t hcnt[2] = {0, 0};
  int32_t hbad = 0;
  if (st == STG_OK) {
    cudaMemcpyAsync(&hcnt[0], cnt.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
    cudaMemcpyAsync(&hbad, bad.p, sizeof(int32_t), cudaMemcpyDeviceToHost, s);
    if (cudaStreamSynchronize(s) != cudaSuccess) st = fail(STG_ERR_CUDA, "stg_dtdg_create: %s", cudaGetErrorString(cudaGetLastError()));
  }
  if (st == STG_OK && hbad) st = fail(STG_ERR_OUT_OF_RANGE, "stg_dtdg_create: base vertex id outside [0,%d)", V);
  int64_t ns = hcnt[0];
  g->E.assign(T, 0);
  g->E[0] = ns;
  g->a_off.assign(T + 1, 0);
  g->d_off.assign(T + 1, 0);
  int64_t max_e = ns;

  // The effective deltas are accumulated on the host side list of device
  // buffers first (sizes unknown until normalised), then packed.
  std::vector<std::vector<uint64_t>> hA(T), hD(T);
  std::vector<DArray<uint64_t>> dA(T), dD(T);

  // keep a copy of S_0 keys for the base snapshot build
  DArray<uint64_t> base_keys;
  CK(base_keys.alloc(ns + 1));
  if (st == STG_OK) cudaMemcpyAsync(base_keys.p, S, sizeof(uint64_t) * ns, cudaMemcpyDeviceToDevice, s);
  // sharded: the local block's edge count per t (E_loc) and the whole-graph deltas
  std::vector<DArray<uint64_t>> gA(T), gD(T);
  g->ga_off.assign(T + 1, 0);
  g->gd_off.assign(T + 1, 0);
  int64_t e_loc = ns;
  g->E0_global = ns;
  if (shard && st == STG_OK) {
    CK(filter_block(S, ns, nb, true, g->rb, g->re, Salt, cnt.p, ws, s));
    if (st == STG_OK) {
      cudaMemcpyAsync(&e_loc, cnt.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
      cudaStreamSynchronize(s);
    }
    g->E[0] = e_loc;
    max_e = e_loc;
  }

  for (int32_t t = 1; t < T && st == STG_OK; ++t) {
    const int64_t na = add_off[t + 1] - add_off[t], nd = del_off[t + 1] - del_off[t];
    uint64_t* a = A1.p; uint64_t* aa = A2.p;
    uint64_t* d = D1.p; uint64_t* da = D2.p;
    int64_t nau = 0, ndu = 0, nae = 0, nde = 0;
    cudaMemsetAsync(cnt.p, 0, 4 * sizeof(int64_t), s);
    if (na) {
      k_pack_batch<<<grid_n(na), 256, 0, s>>>(add_src + add_off[t], add_dst + add_off[t], na, V, nb, a, bad.p);
      count_launch();
      CK(sort_unique_keys(&a, &aa, na, nbits, cnt.p + 0, ws, s));
    }
    if (nd) {
      k_pack_batch<<<grid_n(nd), 256, 0, s>>>(del_src + del_off[t], del_dst + del_off[t], nd, V, nb, d, bad.p);
      count_launch();
      CK(sort_unique_keys(&d, &da, nd, nbits, cnt.p + 1, ws, s));
    }
    int64_t c2[2] = {0, 0};
    if (st == STG_OK) {
      cudaMemcpyAsync(c2, cnt.p, 2 * sizeof(int64_t), cudaMemcpyDeviceToHost, s);
      cudaStreamSynchronize(s);
    }
    nau = c2[0]; ndu = c2[1];
    // effective deltas
    if (nau) CK(scan(NotInS{a, S, ns}, CompactOut{a, Ae.p}, nau, ws.scan, s, cnt.p + 2));
    if (ndu) CK(scan(DelEff{d, a, nau, S, ns, nb, pinned}, CompactOut{d, De.p}, ndu, ws.scan, s, cnt.p + 3));
    if (st == STG_OK) {
      cudaMemcpyAsync(c2, cnt.p + 2, 2 * sizeof(int64_t), cudaMemcpyDeviceToHost, s);
      cudaMemcpyAsync(&hbad, bad.p, sizeof(int32_t), cudaMemcpyDeviceToHost, s);
      if (cudaStreamSynchronize(s) != cudaSuccess) st = fail(STG_ERR_CUDA, "stg_dtdg_create: %s", cudaGetErrorString(cudaGetLastError()));
    }
    if (st == STG_OK && hbad) st = fail(STG_ERR_OUT_OF_RANGE, "stg_dtdg_create: vertex id outside [0,%d) in batch %d", V, t);
    nae = nau ? c2[0] : 0; nde = ndu ? c2[1] : 0;
    if (st == STG_OK && (flags & STG_VALIDATE) && (nae != na || nde != nd))
      st = fail(STG_ERR_INVALID_ARG, "stg_dtdg_create: batch %d is not effective (%lld/%lld adds, %lld/%lld deletes)",
                t, (long long)nae, (long long)na, (long long)nde, (long long)nd);
    if (st != STG_OK) break;
    // S_t = (S_{t-1} \ D') ∪ A'
    cudaMemsetAsync(delflag.p, 0, sizeof(int32_t) * (ns + 1), s);
    if (nde) { k_mark_deleted<<<grid_n(nde), 256, 0, s>>>(De.p, nde, S, ns, delflag.p); count_launch(); }
    CK(scan(KeepIn{delflag.p}, KeepOut{S, Ae.p, nae, keep_ex.p, Salt}, ns, ws.scan, s, keep_ex.p + ns));
    if (nae) { k_place_adds<<<grid_n(nae), 256, 0, s>>>(Ae.p, nae, S, ns, keep_ex.p, Salt); count_launch(); }
    std::swap(S, Salt);
    ns = ns - nde + nae;
    g->E[t] = ns;
    if (shard) {
      // whole-graph deltas for the degrees; the local block's deltas for the CSRs
      CK(gA[t].alloc(nae + 1)); CK(gD[t].alloc(nde + 1));
      if (st == STG_OK) {
        if (nae) cudaMemcpyAsync(gA[t].p, Ae.p, sizeof(uint64_t) * nae, cudaMemcpyDeviceToDevice, s);
        if (nde) cudaMemcpyAsync(gD[t].p, De.p, sizeof(uint64_t) * nde, cudaMemcpyDeviceToDevice, s);
      }
      g->ga_off[t + 1] = g->ga_off[t] + nae;
      g->gd_off[t + 1] = g->gd_off[t] + nde;
      int64_t c3[2] = {0, 0};
      CK(filter_block(gA[t].p, nae, nb, true, g->rb, g->re, A1.p, cnt.p + 2, ws, s));
      CK(filter_block(gD[t].p, nde, nb, true, g->rb, g->re, D1.p, cnt.p + 3, ws, s));
      if (st == STG_OK) {
        cudaMemcpyAsync(c3, cnt.p + 2, 2 * sizeof(int64_t), cudaMemcpyDeviceToHost, s);
        cudaStreamSynchronize(s);
      }
      if (nae) cudaMemcpyAsync(Ae.p, A1.p, sizeof(uint64_t) * c3[0], cudaMemcpyDeviceToDevice, s);
      if (nde) cudaMemcpyAsync(De.p, D1.p, sizeof(uint64_t) * c3[1], cudaMemcpyDeviceToDevice, s);
      nae = c3[0];
      nde = c3[1];
      e_loc += nae - nde;
      g->E[t] = e_loc;
    }
    max_e = std::max(max_e, g->E[t]);
    // keep A'_t, D'_t (src-major order now)
    CK(dA[t].alloc(nae + 1)); CK(dD[t].alloc(nde + 1));
    if (st == STG_OK) {
      if (nae) cudaMemcpyAsync(dA[t].p, Ae.p, sizeof(uint64_t) * nae, cudaMemcpyDeviceToDevice, s);
      if (nde) cudaMemcpyAsync(dD[t].p, De.p, sizeof(uint64_t) * nde, cudaMemcpyDeviceToDevice, s);
    }
    g->a_off[t + 1] = g->a_off[t] + nae;
    g->d_off[t + 1] = g->d_off[t] + nde;
  }
  if (st == STG_OK && T >= 1) { g->a_off[1] = g->a_off[0]; }
  // pack deltas into contiguous arrays, both orders
  const int64_t TA = g->a_off[T], TD = g->d_off[T];
  CK(g->add_out.alloc(TA + 1)); CK(g->add_in.alloc(TA + 1)); CK(g->del_out.alloc(TD + 1)); CK(g->del_in.alloc(TD + 1));
  for (int32_t t = 1; t < T && st == STG_OK; ++t) {
    for (int kind = 0; kind < 2 && st == STG_OK; ++kind) {
      const int64_t off = kind == 0 ? g->a_off[t] : g->d_off[t];
      const int64_t n = (kind == 0 ? g->a_off[t + 1] : g->d_off[t + 1]) - off;
      if (!n) continue;
      uint64_t* o_out = (kind == 0 ? g->add_out.p : g->del_out.p) + off;
      uint64_t* o_in = (kind == 0 ? g->add_in.p : g->del_in.p) + off;
      const uint64_t* srcd = kind == 0 ? dA[t].p : dD[t].p;
      cudaMemcpyAsync(o_out, srcd, sizeof(uint64_t) * n, cudaMemcpyDeviceToDevice, s);
      uint64_t* k1 = Ain.p; uint64_t* k2 = Ain.p + n;
      k_swap_pack<<<grid_n(n), 256, 0, s>>>(srcd, n, nb, k1);
      count_launch();
      uint32_t* nov = nullptr;
      CK((radix_sort<uint64_t, uint32_t>(&k1, &k2, nullptr, &nov, n, 0, nbits, ws.radix, s)));
      if (st == STG_OK) cudaMemcpyAsync(o_in, k1, sizeof(uint64_t) * n, cudaMemcpyDeviceToDevice, s);
    }
    dA[t].reset(); dD[t].reset();
  }
  if (shard) {                                     // whole-graph deltas, contiguous
    CK(g->gadd.alloc(g->ga_off[T] + 1)); CK(g->gdel.alloc(g->gd_off[T] + 1));
    for (int32_t t = 1; t < T && st == STG_OK; ++t) {
      const int64_t na = g->ga_off[t + 1] - g->ga_off[t], nd = g->gd_off[t + 1] - g->gd_off[t];
      if (na) cudaMemcpyAsync(g->gadd.p + g->ga_off[t], gA[t].p, sizeof(uint64_t) * na, cudaMemcpyDeviceToDevice, s);
      if (nd) cudaMemcpyAsync(g->gdel.p + g->gd_off[t], gD[t].p, sizeof(uint64_t) * nd, cudaMemcpyDeviceToDevice, s);
    }
    if (st == STG_OK) cudaStreamSynchronize(s);
    for (int32_t t = 0; t < T; ++t) { gA[t].reset(); gD[t].reset(); }
  }
  // snapshot slots
  const bool eids = (flags & STG_EDGE_IDS) != 0, dgl = (flags & STG_NORM_DGL_BOTH) != 0;
  for (int i = 0; i < 5 && st == STG_OK; ++i) CK(g->slot[i].alloc(V, max_e, eids, dgl, g->rb, g->re));
  CK(g->touch_in.alloc(V)); CK(g->touch_out.alloc(V));
  if (st == STG_OK) {
    cudaMemsetAsync(g->touch_in.p, 0, sizeof(int4) * V, s);
    cudaMemsetAsync(g->touch_out.p, 0, sizeof(int4) * V, s);
    g->slot[0].t = 0;
    const uint64_t* bk = base_keys.p;
    if (shard) {                                   // whole-graph degrees of S_0, local edges of S_0
      Snapshot& b0 = g->slot[0];
      cudaMemsetAsync(b0.gin_deg.p, 0, sizeof(int32_t) * V, s);
      cudaMemsetAsync(b0.gout_deg.p, 0, sizeof(int32_t) * V, s);
      degree_hist(base_keys.p, g->E0_global, nb, 1, b0.gin_deg.p, b0.gout_deg.p, s);
      CK(filter_block(base_keys.p, g->E0_global, nb, true, g->rb, g->re, S2.p, cnt.p, ws, s));
      bk = S2.p;
    }
    CK(build_from_out_keys(bk, g->E[0], g->slot[0], ws, s));
  }
  // NaiveGraph mode: materialise S_0 .. S_{T-1} (both CSRs, labels, schedules) by
  // walking the deltas forward once
  if (st == STG_OK && (flags & STG_NAIVE)) {
    g->naive.resize(T);
    for (int32_t t = 0; t < T && st == STG_OK; ++t) {
      g->naive[t].reset(new Snapshot());
      Snapshot& sn = *g->naive[t];
      CK(sn.alloc(V, std::max<int64_t>(g->E[t], 1), eids, dgl, g->rb, g->re));
      if (st != STG_OK) break;
      if (t == 0) {
        sn.t = 0;
        CK(build_from_out_keys(base_keys.p, g->E[0], sn, ws, s));
      } else {
        CK(g->step_snap(*g->naive[t - 1], sn, 1, PART_IN | PART_OUT, s));
        CK(complete_parts(sn, PART_ALL, ws, s));
      }
    }
  }
  if (st == STG_OK && cudaStreamSynchronize(s) != cudaSuccess)
    st = fail(STG_ERR_CUDA, "stg_dtdg_create: %s", cudaGetErrorString(cudaGetLastError()));
#undef CK
  if (st != STG_OK) { delete g; return st; }
  *out = g;
  return STG_OK;
}

stg_status stg_dtdg_get_snapshot(stg_dtdg* g, int32_t t, stg_stream_t stream, stg_csr_view* out) {
  if (!g || !out) return fail(STG_ERR_INVALID_ARG, "stg_dtdg_get_snapshot: NULL argument");
  if (t < 0 || t >= g->T) return fail(STG_ERR_OUT_OF_RANGE, "stg_dtdg_get_snapshot: t=%d outside [0,%d)", t, g->T);
  return g->get(t, false, PART_ALL, (cudaStream_t)stream, out);
}

stg_status stg_dtdg_get_backward_snapshot(stg_dtdg* g, int32_t t, stg_stream_t stream, stg_csr_view* out) {
  if (!g || !out) return fail(STG_ERR_INVALID_ARG, "stg_dtdg_get_backward_snapshot: NULL argument");
  if (t < 0 || t >= g->T)
    return fail(STG_ERR_OUT_OF_RANGE, "stg_dtdg_get_backward_snapshot: t=%d outside [0,%d)", t, g->T);
  return g->get(t, true, PART_ALL, (cudaStream_t)stream, out);
}

stg_status stg_dtdg_get_snapshot_parts(stg_dtdg* g, int32_t t, int32_t backward, uint32_t parts,
                                       stg_stream_t stream, stg_csr_view* out) {
  if (!g || !out) return fail(STG_ERR_INVALID_ARG, "stg_dtdg_get_snapshot_parts: NULL argument");
  if (t < 0 || t >= g->T) return fail(STG_ERR_OUT_OF_RANGE, "stg_dtdg_get_snapshot_parts: t=%d outside [0,%d)", t, g->T);
  if (!(parts & (STG_PART_IN | STG_PART_OUT)) || (parts & ~(uint32_t)(STG_PART_IN | STG_PART_OUT | STG_PART_EID)))
    return fail(STG_ERR_INVALID_ARG, "stg_dtdg_get_snapshot_parts: parts=0x%x", parts);
  uint32_t p = ((parts & STG_PART_IN) ? PART_IN : 0u) | ((parts & STG_PART_OUT) ? PART_OUT : 0u);
  if (parts & STG_PART_EID) p = PART_ALL;          // labels tie both directions
  return g->get(t, backward != 0, p, (cudaStream_t)stream, out);
}

int64_t stg_dtdg_num_edges(const stg_dtdg* g, int32_t t) {
  if (!g || t < 0 || t >= g->T) return -1;
  return g->E[t];
}

int32_t stg_dtdg_num_timestamps(const stg_dtdg* g) { return g ? g->T : -1; }

int64_t stg_dtdg_num_deltas(const stg_dtdg* g, int32_t t, int32_t deletes) {
  if (!g || t < 0 || t >= g->T) return -1;
  return deletes ? g->d_off[t + 1] - g->d_off[t] : g->a_off[t + 1] - g->a_off[t];
}

}  // extern "C"

namespace stg {
bool dtdg_materialised(const stg_dtdg* g) { return g && !g->naive.empty(); }
}  // namespace stg

extern "C" {

stg_status stg_dtdg_memory(const stg_dtdg* g, int64_t* deltas, int64_t* cache, int64_t* materialised) {
  if (!g || !deltas || !cache || !materialised) return fail(STG_ERR_INVALID_ARG, "stg_dtdg_memory: NULL argument");
  const DArray<uint64_t>* d[] = {&g->add_out, &g->add_in, &g->del_out, &g->del_in, &g->gadd, &g->gdel};
  int64_t b = 0;
  for (const auto* a : d) b += (int64_t)(a->n * sizeof(uint64_t));
  *deltas = b;
  b = (int64_t)((g->touch_in.n + g->touch_out.n) * sizeof(int4));
  for (const auto& sl : g->slot) b += (int64_t)sl.bytes();
  *cache = b;
  b = 0;
  for (const auto& sn : g->naive) b += (int64_t)sn->bytes();
  *materialised = b;
  return STG_OK;
}

void stg_dtdg_destroy(stg_dtdg* g) {
  if (g) cudaDeviceSynchronize();
  delete g;
}

}  // extern "C"
