"""ORACLE — plain fp64 CPU reference for the STGraph hot path.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` arm may import this package.  It shares no
code with the CUDA library (paper_conf_ipps_cherianmcc24_b200/) and neither
imports the other; the only shared module is gen/ (seeded inputs, no method
arithmetic).

The arithmetic lives in stg_oracle.c (plain C, fp64, plain definitions, see the
citations there).  This file only marshals numpy arrays through ctypes and
strings the per-timestamp definitions together in Algorithm 1's order
 for the sequence-level reference.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "stg_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")


_LIB_OMP = os.path.join(_HERE, "liboracle_omp.so")


def build(force: bool = False, omp: bool = False) -> str:
    """Compile stg_oracle.c with plain gcc -O2 (no fast-math).  omp=True builds the
    SAME source with -fopenmp (liboracle_omp.so): its `#pragma omp` lines split the
    row loops over threads — used only to time the all-core CPU baseline
    (bench.py); every parity test runs the plain single-thread build."""
    out = _LIB_OMP if omp else _LIB
    if force or not os.path.exists(out) or os.path.getmtime(out) < os.path.getmtime(_SRC):
        tmp = out + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-fno-fast-math"] +
                              (["-fopenmp"] if omp else []) + ["-o", tmp, _SRC, "-lm"])
        os.replace(tmp, out)
    if not omp:
        build(force, omp=True)
    return out


_libs = {}
_mode = {"omp": False}


def use_openmp(on: bool) -> int:
    """Route the oracle calls to the OpenMP timing build (True) or the plain build
    (False).  Returns the thread count the OpenMP runtime will use."""
    _mode["omp"] = bool(on)
    if not on:
        return 1
    lib()
    try:
        gomp = ctypes.CDLL("libgomp.so.1")
        return int(gomp.omp_get_max_threads())
    except OSError:
        return os.cpu_count() or 1


def lib():
    omp = _mode["omp"]
    if omp not in _libs:
        _lib = ctypes.CDLL(build(omp=omp) if omp else build())
        _libs[omp] = _lib
        P = ctypes.c_void_p
        i32, i64 = ctypes.c_int32, ctypes.c_int64
        _lib.orc_edge_set.restype = i64
        _lib.orc_edge_set.argtypes = [i32, i64, P, P, i32, P]
        _lib.orc_csr_build.restype = None
        _lib.orc_csr_build.argtypes = [i32, i64, P, i32] + [P] * 11
        _lib.orc_aggregate.restype = None
        _lib.orc_aggregate.argtypes = [i32, P, P, P, P, i32, P, P]
        _lib.orc_aggregate_edges.restype = None
        _lib.orc_aggregate_edges.argtypes = [i32, i64, P, P, P, P, i32, i32, P, P]
        _lib.orc_weighted_norm.restype = None
        _lib.orc_weighted_norm.argtypes = [i32, i64, P, P, P]
        _lib.orc_set_apply.restype = i64
        _lib.orc_set_apply.argtypes = [P, i64, P, i64, P, i64, P]
        _lib.orc_window_set.restype = i64
        _lib.orc_window_set.argtypes = [P, P, i64, i64, P]
        _lib.orc_effective_deltas.restype = None
        _lib.orc_effective_deltas.argtypes = [P, i64, P, i64, P, i64, i32, P, P, P, P]
        _lib.orc_tgcn_fwd.restype = None
        _lib.orc_tgcn_fwd.argtypes = [i32, i32, i32] + [P] * 15
        _lib.orc_tgcn_bwd.restype = None
        _lib.orc_tgcn_bwd.argtypes = [i32, i32, i32] + [P] * 17
        _lib.orc_tgcn2_fwd.restype = None
        _lib.orc_tgcn2_fwd.argtypes = [i32, i32, i32] + [P] * 14
        _lib.orc_tgcn2_bwd.restype = None
        _lib.orc_tgcn2_bwd.argtypes = [i32, i32, i32] + [P] * 19
        _lib.orc_mse_head.restype = ctypes.c_double
        _lib.orc_mse_head.argtypes = [i32, i32, P, P, P, ctypes.c_double, P, P, P]
    return _libs[omp]


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


# ----------------------------------------------------------------- edge sets
def keys(src, dst) -> np.ndarray:
    return (np.asarray(src, np.int64).astype(np.uint64) << np.uint64(32)) | np.asarray(dst, np.int64).astype(np.uint64)


def unkey(k: np.ndarray):
    k = np.asarray(k, np.uint64)
    return (k >> np.uint64(32)).astype(np.int32), (k & np.uint64(0xFFFFFFFF)).astype(np.int32)


def edge_set(V: int, src, dst, self_loops: bool = False) -> np.ndarray:
    src, dst = _c(src, np.int32), _c(dst, np.int32)
    out = np.empty(src.size + (V if self_loops else 0) + 1, np.uint64)
    n = lib().orc_edge_set(V, src.size, _p(src), _p(dst), int(self_loops), _p(out))
    return out[:n].copy()


def csr(V: int, S: np.ndarray, dgl_both: bool = False) -> dict:
    """All STGraphBase arrays of the snapshot whose sorted edge-key set is S."""
    S = _c(S, np.uint64)
    n = S.size
    r = {k: np.zeros(V + 1, np.int32) for k in ("in_rowptr", "out_rowptr")}
    for k in ("in_col", "out_col", "out_eid"):
        r[k] = np.zeros(max(n, 1), np.int32)
    for k in ("in_deg", "out_deg", "in_ids", "out_ids"):
        r[k] = np.zeros(max(V, 1), np.int32)
    r["norm_src"] = np.zeros(max(V, 1), np.float64)
    r["norm_dst"] = np.zeros(max(V, 1), np.float64)
    lib().orc_csr_build(V, n, _p(S), int(dgl_both), _p(r["in_rowptr"]), _p(r["in_col"]),
                        _p(r["out_rowptr"]), _p(r["out_col"]), _p(r["out_eid"]),
                        _p(r["in_deg"]), _p(r["out_deg"]), _p(r["in_ids"]), _p(r["out_ids"]),
                        _p(r["norm_src"]), _p(r["norm_dst"]))
    for k in ("in_col", "out_col", "out_eid"):
        r[k] = r[k][:n]
    for k in ("in_deg", "out_deg", "in_ids", "out_ids", "norm_src", "norm_dst"):
        r[k] = r[k][:V]
    r["V"], r["E"] = V, n
    return r


def static_graph(V: int, src, dst, self_loops: bool = False, dgl_both: bool = False) -> dict:
    return csr(V, edge_set(V, src, dst, self_loops), dgl_both)


# --------------------------------------------------------------- aggregation
def aggregate(rowptr, col, nrow, ncol, x) -> np.ndarray:
    rowptr, col = _c(rowptr, np.int32), _c(col, np.int32)
    x = _c(x, np.float64)
    R = rowptr.size - 1
    W = x.shape[1]
    nrow = _c(nrow, np.float64)
    ncol_p = None if ncol is None else _c(ncol, np.float64)
    y = np.zeros((R, W), np.float64)
    lib().orc_aggregate(R, _p(rowptr), _p(col if col.size else np.zeros(1, np.int32)), _p(nrow),
                        None if ncol_p is None else _p(ncol_p), W, _p(x), _p(y))
    return y


def aggregate_fwd(g: dict, x) -> np.ndarray:
    """y_v = Σ_{u∈N_in(v)} n_dst[v]·n_src[u]·x_u over the in-CSR (a5)."""
    return aggregate(g["in_rowptr"], g["in_col"], g["norm_dst"], g["norm_src"], x)


def aggregate_bwd(g: dict, gy) -> np.ndarray:
    """gx_u = n_src[u]·Σ_{v∈N_out(u)} n_dst[v]·gy_v over the out-CSR (a6)."""
    return aggregate(g["out_rowptr"], g["out_col"], g["norm_src"], g["norm_dst"], gy)


def aggregate_scale(g: dict, x, bwd: bool = False) -> np.ndarray:
    """Same aggregation over |x| — the per-element condition scale s_i of reading C19."""
    return (aggregate_bwd if bwd else aggregate_fwd)(g, np.abs(np.asarray(x, np.float64)))


def aggregate_edges(V: int, S, w, nrow, ncol, x, backward: bool = False) -> np.ndarray:
    """Edge-weighted aggregation over the edge set S with per-edge weights w
    (aligned with the sorted keys S): forward y_v = Σ_{(u,v)∈S} n[v]·w·n[u]·x_u,
    backward the transpose (NEXT-4)."""
    S, w = _c(S, np.uint64), _c(w, np.float64)
    x = _c(x, np.float64)
    W = x.shape[1]
    nrow = _c(nrow, np.float64)
    ncol_p = None if ncol is None else _c(ncol, np.float64)
    y = np.zeros((V, W), np.float64)
    lib().orc_aggregate_edges(V, S.size, _p(S if S.size else np.zeros(1, np.uint64)),
                              _p(w if w.size else np.zeros(1)), _p(nrow), None if ncol_p is None else _p(ncol_p),
                              int(backward), W, _p(x), _p(y))
    return y


def weighted_norm(V: int, S, w) -> np.ndarray:
    S, w = _c(S, np.uint64), _c(w, np.float64)
    out = np.zeros(max(V, 1), np.float64)
    lib().orc_weighted_norm(V, S.size, _p(S if S.size else np.zeros(1, np.uint64)), _p(w if w.size else np.zeros(1)),
                            _p(out))
    return out[:V]


# ------------------------------------------------------------------ snapshots
def set_apply(S, D, A) -> np.ndarray:
    S, D, A = _c(S, np.uint64), _c(D, np.uint64), _c(A, np.uint64)
    out = np.empty(S.size + A.size + 1, np.uint64)
    n = lib().orc_set_apply(_p(S), S.size, _p(D if D.size else np.zeros(1, np.uint64)), D.size,
                            _p(A if A.size else np.zeros(1, np.uint64)), A.size, _p(out))
    return out[:n].copy()


def window_set(ev_src, ev_dst, lo: int, hi: int) -> np.ndarray:
    ev_src, ev_dst = _c(ev_src, np.int32), _c(ev_dst, np.int32)
    out = np.empty(max(hi - lo, 1), np.uint64)
    n = lib().orc_window_set(_p(ev_src), _p(ev_dst), lo, hi, _p(out))
    return out[:n].copy()


def effective_deltas(Sprev, A, D, pinned_loops: bool = False):
    Sprev, A, D = _c(Sprev, np.uint64), _c(A, np.uint64), _c(D, np.uint64)
    oa = np.empty(A.size + 1, np.uint64); od = np.empty(D.size + 1, np.uint64)
    na = ctypes.c_int64(0); nd = ctypes.c_int64(0)
    z = np.zeros(1, np.uint64)
    lib().orc_effective_deltas(_p(Sprev if Sprev.size else z), Sprev.size, _p(A if A.size else z), A.size,
                               _p(D if D.size else z), D.size, int(pinned_loops),
                               _p(oa), ctypes.byref(na), _p(od), ctypes.byref(nd))
    return oa[:na.value].copy(), od[:nd.value].copy()


def batch(d, t: int):
    """(A_t, D_t) raw key batches of a gen.DTDG."""
    a0, a1 = int(d.add_off[t]), int(d.add_off[t + 1])
    d0, d1 = int(d.del_off[t]), int(d.del_off[t + 1])
    return keys(d.add_src[a0:a1], d.add_dst[a0:a1]), keys(d.del_src[d0:d1], d.del_dst[d0:d1])


def snapshot_sets_fold(d, self_loops: bool = False):
    """Generator of S_t for t = 0..T-1 by folding S_t = (S_{t-1} \\ D_t) ∪ A_t."""
    S = edge_set(d.V, d.src0, d.dst0, self_loops)
    yield S
    loops = keys(np.arange(d.V), np.arange(d.V)) if self_loops else np.zeros(0, np.uint64)
    for t in range(1, d.T):
        A, D = batch(d, t)
        if self_loops:    # loops are pinned: never deleted (reading C11/C9)
            s_, d_ = unkey(D)
            D = D[s_ != d_]
            A = np.concatenate([A, loops])
        S = set_apply(S, D, A)
        yield S


def snapshot_set_window(d, t: int, self_loops: bool = False) -> np.ndarray:
    """S_t from the event-window definition, independent of the deltas."""
    lo, hi = d.window(t)
    S = window_set(d.ev_src, d.ev_dst, lo, hi)
    if self_loops:
        S = np.union1d(S, keys(np.arange(d.V), np.arange(d.V)))
    return S


# ---------------------------------------------------------------------- TGCN
def tgcn_fwd(g: dict, p: dict, X, Hp) -> dict:
    V, F = X.shape
    H = Hp.shape[1]
    X, Hp = _c(X, np.float64), _c(Hp, np.float64)
    W, b, L, l = (_c(p[k], np.float64) for k in ("W", "b", "L", "l"))
    out = {k: np.zeros((V, H), np.float64) for k in ("Z", "R", "Hh", "Hn")}
    out["C"] = np.zeros((V, 3 * H), np.float64)
    ns, nd = _c(g["norm_src"], np.float64), _c(g["norm_dst"], np.float64)
    col = g["in_col"] if g["in_col"].size else np.zeros(1, np.int32)
    lib().orc_tgcn_fwd(V, F, H, _p(_c(g["in_rowptr"], np.int32)), _p(_c(col, np.int32)), _p(ns), _p(nd),
                       _p(X), _p(Hp), _p(W), _p(b), _p(L), _p(l),
                       _p(out["C"]), _p(out["Z"]), _p(out["R"]), _p(out["Hh"]), _p(out["Hn"]))
    return out


def zero_grads(F: int, H: int) -> dict:
    return {"W": np.zeros((F, 3 * H)), "b": np.zeros(3 * H), "L": np.zeros((3, 2 * H, H)),
            "l": np.zeros((3, H)), "w_o": np.zeros(H), "b_o": np.zeros(1)}


def tgcn_bwd(g: dict, p: dict, X, Hp, fwd: dict, G, grads: dict) -> np.ndarray:
    """Accumulates into grads (float64 arrays); returns dH_{t-1}."""
    V, F = X.shape
    H = Hp.shape[1]
    X, Hp, G = _c(X, np.float64), _c(Hp, np.float64), _c(G, np.float64)
    L = _c(p["L"], np.float64)
    dHp = np.zeros((V, H), np.float64)
    ns, nd = _c(g["norm_src"], np.float64), _c(g["norm_dst"], np.float64)
    col = g["out_col"] if g["out_col"].size else np.zeros(1, np.int32)
    for k in ("W", "b", "L", "l"):
        assert grads[k].dtype == np.float64 and grads[k].flags.c_contiguous
    lib().orc_tgcn_bwd(V, F, H, _p(_c(g["out_rowptr"], np.int32)), _p(_c(col, np.int32)), _p(ns), _p(nd),
                       _p(X), _p(Hp), _p(_c(fwd["C"], np.float64)), _p(G), _p(L),
                       _p(_c(fwd["Z"], np.float64)), _p(_c(fwd["R"], np.float64)), _p(_c(fwd["Hh"], np.float64)),
                       _p(dHp), _p(grads["W"]), _p(grads["b"]), _p(grads["L"]), _p(grads["l"]))
    return dHp


def mse_head(Hn, y, w_o, b_o, grads: dict):
    V, H = Hn.shape
    Hn, y, w_o = _c(Hn, np.float64), _c(y, np.float64), _c(w_o, np.float64)
    dH = np.zeros((V, H), np.float64)
    loss = lib().orc_mse_head(V, H, _p(Hn), _p(y), _p(w_o), float(np.asarray(b_o).reshape(-1)[0]),
                              _p(dH), _p(grads["w_o"]), _p(grads["b_o"]))
    return loss, dH


def train_sequence(graphs_fwd, graphs_bwd, p: dict, Xs, Ys, H0):
    """Algorithm 1 lines 6-25 for ONE sequence s, in fp64.

    graphs_fwd[i] / graphs_bwd[i]: oracle CSR dicts of snapshot t_i (for a static
    graph the same dict).  Forward for t in s with the state pushed; then the
    backward pops in LIFO order; gradients accumulate over the sequence (C17).
    Returns (sum of losses, grads, H_last).
    """
    S = len(Xs)
    F = Xs[0].shape[1]
    H = H0.shape[1]
    grads = zero_grads(F, H)
    stack = []
    Hc = np.asarray(H0, np.float64)
    loss = 0.0
    for i in range(S):                               # forward, lines 7-16
        f = tgcn_fwd(graphs_fwd[i], p, Xs[i], Hc)
        stack.append((Hc, f))                        # state-stack.push
        l_i, dH_head = mse_head(f["Hn"], Ys[i], p["w_o"], p["b_o"], grads)
        f["dH_head"] = dH_head
        loss += l_i
        Hc = f["Hn"]
    Gnext = np.zeros_like(Hc)
    for i in reversed(range(S)):                     # backward, lines 18-25 (LIFO)
        Hp, f = stack.pop()
        G = f["dH_head"] + Gnext
        Gnext = tgcn_bwd(graphs_bwd[i], p, Xs[i], Hp, f, G, grads)
    return loss, grads, Hc


# ------------------------------------------------------ original T-GCN (NEXT-2)
def tgcn2_fwd(g: dict, p: dict, X, Hp) -> dict:
    """Original T-GCN cell (GCN over [X, H], aggregate-first as written; NEXT-2)."""
    V, F = X.shape
    H = Hp.shape[1]
    X, Hp = _c(X, np.float64), _c(Hp, np.float64)
    Wg, bg, Wc, bc = (_c(p[k], np.float64) for k in ("Wg", "bg", "Wc", "bc"))
    out = {k: np.zeros((V, H), np.float64) for k in ("R", "U", "Cc", "Hn")}
    ns, nd = _c(g["norm_src"], np.float64), _c(g["norm_dst"], np.float64)
    col = g["in_col"] if g["in_col"].size else np.zeros(1, np.int32)
    lib().orc_tgcn2_fwd(V, F, H, _p(_c(g["in_rowptr"], np.int32)), _p(_c(col, np.int32)), _p(ns), _p(nd),
                        _p(X), _p(Hp), _p(Wg), _p(bg), _p(Wc), _p(bc),
                        _p(out["R"]), _p(out["U"]), _p(out["Cc"]), _p(out["Hn"]))
    return out


def zero_grads2(F: int, H: int) -> dict:
    return {"Wg": np.zeros((F + H, 2 * H)), "bg": np.zeros(2 * H), "Wc": np.zeros((F + H, H)),
            "bc": np.zeros(H), "w_o": np.zeros(H), "b_o": np.zeros(1)}


def tgcn2_bwd(g: dict, p: dict, X, Hp, fwd: dict, G, grads: dict) -> np.ndarray:
    """Accumulates into grads (float64 arrays); returns dH_{t-1}."""
    V, F = X.shape
    H = Hp.shape[1]
    X, Hp, G = _c(X, np.float64), _c(Hp, np.float64), _c(G, np.float64)
    dHp = np.zeros((V, H), np.float64)
    ns, nd = _c(g["norm_src"], np.float64), _c(g["norm_dst"], np.float64)
    icol = g["in_col"] if g["in_col"].size else np.zeros(1, np.int32)
    ocol = g["out_col"] if g["out_col"].size else np.zeros(1, np.int32)
    for k in ("Wg", "bg", "Wc", "bc"):
        assert grads[k].dtype == np.float64 and grads[k].flags.c_contiguous
    lib().orc_tgcn2_bwd(V, F, H, _p(_c(g["in_rowptr"], np.int32)), _p(_c(icol, np.int32)),
                        _p(_c(g["out_rowptr"], np.int32)), _p(_c(ocol, np.int32)), _p(ns), _p(nd),
                        _p(X), _p(Hp), _p(_c(p["Wg"], np.float64)), _p(_c(p["Wc"], np.float64)),
                        _p(_c(fwd["R"], np.float64)), _p(_c(fwd["U"], np.float64)), _p(_c(fwd["Cc"], np.float64)),
                        _p(G), _p(dHp), _p(grads["Wg"]), _p(grads["bg"]), _p(grads["Wc"]), _p(grads["bc"]))
    return dHp


def train_sequence2(graphs, p: dict, Xs, Ys, H0):
    """Algorithm 1 for one sequence with the original T-GCN cell (NEXT-2), fp64.
    Returns (sum of losses, grads, H_last)."""
    S = len(Xs)
    F = Xs[0].shape[1]
    H = H0.shape[1]
    grads = zero_grads2(F, H)
    stack = []
    Hc = np.asarray(H0, np.float64)
    loss = 0.0
    for i in range(S):
        f = tgcn2_fwd(graphs[i], p, Xs[i], Hc)
        stack.append((Hc, f))
        l_i, _ = mse_head(f["Hn"], Ys[i], p["w_o"], p["b_o"], {"w_o": np.zeros(H), "b_o": np.zeros(1)})
        loss += l_i
        Hc = f["Hn"]
    dH = np.zeros_like(Hc)
    for i in range(S - 1, -1, -1):
        Hp, f = stack.pop()
        _, dh_head = mse_head(f["Hn"], Ys[i], p["w_o"], p["b_o"], grads)
        dH = tgcn2_bwd(graphs[i], p, Xs[i], Hp, f, dH + dh_head, grads)
    return loss, grads, Hc
