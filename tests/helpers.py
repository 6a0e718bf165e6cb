"""Shared helpers for the GPU parity tests: comparisons against the oracle."""
import numpy as np
import torch

import oracle

GRAPH_KEYS = ("in_rowptr", "in_col", "out_rowptr", "out_col", "in_deg", "out_deg", "in_ids", "out_ids")


def assert_graph_equal(gpu: dict, ref: dict, edge_ids: bool = True, tag=""):
    """Bit-exact for every integer array; norms within one fp32 rounding of fp64."""
    for k in GRAPH_KEYS:
        a = gpu[k].cpu().numpy()
        b = np.asarray(ref[k])
        assert a.shape == b.shape, (tag, k, a.shape, b.shape)
        if not np.array_equal(a, b):
            bad = np.nonzero(a != b)[0][:10]
            raise AssertionError("%s %s differs at %s: gpu %s ref %s" % (tag, k, bad, a[bad], b[bad]))
    if edge_ids:
        assert np.array_equal(gpu["out_eid"].cpu().numpy(), ref["out_eid"]), (tag, "out_eid")
    for k in ("norm_src", "norm_dst"):
        a = gpu[k].cpu().numpy().astype(np.float64)
        np.testing.assert_allclose(a, ref[k], rtol=2.5e-7, atol=0, err_msg=k)


def cond_err(y_gpu, y_ref, scale) -> float:
    """Reading C19: max_i |y_gpu - y_ref| / s_i with s_i the oracle over |x|;
    rows/entries with s_i = 0 must be exactly 0 on the GPU."""
    y = np.asarray(y_gpu, np.float64)
    r = np.asarray(y_ref, np.float64)
    s = np.asarray(scale, np.float64)
    zero = s == 0
    assert np.all(y[zero] == 0.0), "nonzero output where the condition scale is 0"
    d = np.abs(y - r)[~zero] / s[~zero]
    return float(d.max()) if d.size else 0.0


def to_gpu(a, dtype=torch.float32):
    return torch.from_numpy(np.ascontiguousarray(a)).to(device="cuda", dtype=dtype)


def oracle_graph_from_set(V, S, dgl_both=False):
    return oracle.csr(V, S, dgl_both)


# ---------------------------------------------------------------- TGCN condition scales
# Element-wise tolerances for the TGCN step / sequence: every GPU
# result r_i is compared as |r_gpu − r_ref| <= tau · s_i, where s_i is "the same
# computation over |·|" — every input, parameter and intermediate replaced by its
# absolute value (first-order propagation of relative rounding errors), computed
# from the oracle's own fp64 intermediates.  It generalises reading C19 (the
# aggregation's Σ|terms|) to the GRU chain and the Σ-over-rows reductions.  These
# are test-side error bounds only; the oracle's arithmetic is untouched.
TAU_TGCN = 1e-5


def _abs_gates(p, H):
    L = np.abs(np.asarray(p["L"], np.float64))
    return L[0, :H], L[0, H:], L[1, :H], L[1, H:], L[2, :H], L[2, H:]


def tgcn_fwd_scale(g: dict, p: dict, X, Hp, sHp, f: dict) -> dict:
    """Forward scales of one step.  Rules (s(x) >= |x|, first order): s(a±b) =
    s(a)+s(b); s(ab) = s(a)|b| + |a|s(b); s(f(a)) = |f(a)| + |f'(a)|s(a); exact
    inputs s(x) = |x|.  Hp / sHp: the value and scale of H_{t-1}; f: the oracle's
    intermediates.  Returns the scales of C, Z, R, R⊙H, Ĥ and H'."""
    H = Hp.shape[1]
    aH = np.abs(np.asarray(Hp, np.float64))
    sP = np.abs(np.asarray(X, np.float64)) @ np.abs(np.asarray(p["W"], np.float64))
    sC = oracle.aggregate_fwd(g, sP) + np.abs(np.asarray(p["b"], np.float64))
    Lz1, Lz2, Lr1, Lr2, Lh1, Lh2 = _abs_gates(p, H)
    al = np.abs(np.asarray(p["l"], np.float64))
    Z, R, Hh = f["Z"], f["R"], f["Hh"]
    sZ = Z + Z * (1 - Z) * (sC[:, :H] @ Lz1 + sHp @ Lz2 + al[0])
    sR = R + R * (1 - R) * (sC[:, H:2 * H] @ Lr1 + sHp @ Lr2 + al[1])
    sRH = sR * aH + R * sHp
    sHh = np.abs(Hh) + (1 - Hh ** 2) * (sC[:, 2 * H:] @ Lh1 + sRH @ Lh2 + al[2])
    sHn = sZ * (aH + np.abs(Hh)) + Z * sHp + (1 - Z) * sHh
    return {"C": sC, "Z": sZ, "R": sR, "RH": sRH, "Hh": sHh, "Hn": sHn}


def tgcn_bwd_scales(g: dict, p: dict, X, Hp, sHp, f: dict, fs: dict, G, sG, acc: dict):
    """Backward scales of one step (same rules; G / sG: the value and scale of the
    upstream gradient): adds the per-parameter gradient scales into acc and
    returns s(dH_{t-1})."""
    H = Hp.shape[1]
    aH = np.abs(np.asarray(Hp, np.float64))
    aG = np.abs(np.asarray(G, np.float64))
    Lz1, Lz2, Lr1, Lr2, Lh1, Lh2 = _abs_gates(p, H)
    L = np.asarray(p["L"], np.float64)
    Z, R, Hh, C = f["Z"], f["R"], f["Hh"], np.abs(f["C"])
    G = np.asarray(G, np.float64)
    dZ, dHh = G * (Hp - Hh), G * (1 - Z)
    s_dZ = sG * np.abs(Hp - Hh) + aG * (sHp + fs["Hh"])
    s_dHh = sG * (1 - Z) + aG * fs["Z"]
    dah = dHh * (1 - Hh ** 2)
    s_dah = s_dHh * (1 - Hh ** 2) + np.abs(dHh) * 2 * np.abs(Hh) * fs["Hh"]
    daz = dZ * Z * (1 - Z)
    s_daz = s_dZ * Z * (1 - Z) + np.abs(dZ) * np.abs(1 - 2 * Z) * fs["Z"]
    dRH = dah @ L[2, H:].T
    s_dRH = s_dah @ Lh2.T
    dR = dRH * Hp
    s_dR = s_dRH * aH + np.abs(dRH) * sHp
    dar = dR * R * (1 - R)
    s_dar = s_dR * R * (1 - R) + np.abs(dR) * np.abs(1 - 2 * R) * fs["R"]
    s_dC = np.concatenate([s_daz @ Lz1.T, s_dar @ Lr1.T, s_dah @ Lh1.T], axis=1)
    s_dP = oracle.aggregate_bwd(g, s_dC)
    sCg = [fs["C"][:, :H], fs["C"][:, H:2 * H], fs["C"][:, 2 * H:]]
    Cg = [C[:, :H], C[:, H:2 * H], C[:, 2 * H:]]
    das, s_das = [daz, dar, dah], [s_daz, s_dar, s_dah]
    rows2 = [(aH, sHp), (aH, sHp), (np.abs(R * Hp), fs["RH"])]
    sc = {"W": np.abs(np.asarray(X, np.float64)).T @ s_dP, "b": s_dC.sum(0),
          "L": np.stack([np.concatenate([sCg[k].T @ np.abs(das[k]) + Cg[k].T @ s_das[k],
                                         rows2[k][1].T @ np.abs(das[k]) + rows2[k][0].T @ s_das[k]])
                         for k in range(3)]),
          "l": np.stack([s_daz.sum(0), s_dar.sum(0), s_dah.sum(0)])}
    for k, v in sc.items():
        acc[k] = acc.get(k, 0) + v
    return sG * Z + aG * fs["Z"] + s_dRH * R + np.abs(dRH) * fs["R"] + s_dar @ Lr2.T + s_daz @ Lz2.T


def head_scales(Hn, sHn, y, w_o, b_o, acc: dict):
    """Scales of the MSE surrogate head (ŷ = ReLU(H)·w_o + b_o, ℓ = mean (ŷ−y)²):
    adds s(dw_o), s(db_o) into acc; returns (s(dH), s(ℓ))."""
    V = Hn.shape[0]
    b = float(np.asarray(b_o).reshape(-1)[0])
    w = np.asarray(w_o, np.float64)
    pos = Hn > 0
    rh = np.where(pos, Hn, 0.0)
    s_rh = np.where(pos, sHn, 0.0)
    e = rh @ w + b - y
    s_e = s_rh @ np.abs(w) + abs(b) + np.abs(y)
    s_g = 2 * s_e / V
    acc["w_o"] = acc.get("w_o", 0) + rh.T @ s_g + s_rh.T @ (2 * np.abs(e) / V)
    acc["b_o"] = acc.get("b_o", 0) + np.array([s_g.sum()])
    return np.outer(s_g, np.abs(w)) * pos, float(np.sum(2 * np.abs(e) * s_e) / V)


def sequence_scales(graphs_fwd, graphs_bwd, p: dict, Xs, Ys, H0, chain: bool = False) -> dict:
    """Condition scales of oracle.train_sequence's outputs (Algorithm 1 over one
    sequence): per-parameter gradient scales ("W", "b", "L", "l", "w_o", "b_o"),
    the loss scale ("loss"), s(H_t) for every step ("H") and s(dH_0) ("dH0")."""
    S = len(Xs)
    H = H0.shape[1]
    acc, steps, sH, sl = {}, [], [], 0.0
    Hc = np.asarray(H0, np.float64)
    sHc = np.abs(Hc)
    for i in range(S):
        f = oracle.tgcn_fwd(graphs_fwd[i], p, Xs[i], Hc)
        fs = tgcn_fwd_scale(graphs_fwd[i], p, Xs[i], Hc, sHc, f)
        steps.append((Hc, sHc, f, fs))
        sH.append(fs["Hn"])
        Hc, sHc = f["Hn"], fs["Hn"]
    Gnext, s_next = np.zeros_like(Hc), np.zeros_like(Hc)
    for i in reversed(range(S)):
        Hp, sHp, f, fs = steps[i]
        _, dHh = oracle.mse_head(f["Hn"], Ys[i], p["w_o"], p["b_o"], oracle.zero_grads(Xs[i].shape[1], H))
        s_head, s_li = head_scales(f["Hn"], fs["Hn"], np.asarray(Ys[i], np.float64), p["w_o"], p["b_o"], acc)
        sl += s_li
        # the upstream gradient enters each step's scale by its value (|G|, plus the
        # head's own rounding scale): abs-propagating scales through the whole BPTT
        # chain bounds the error by the product of |Jacobian| norms, which grows
        # ~1.3x per step and stops being informative after a few steps
        G = dHh + Gnext
        sG = s_head + (np.abs(Gnext) if chain is False else s_next)
        s_next = tgcn_bwd_scales(graphs_bwd[i], p, Xs[i], Hp, sHp, f, fs, G, sG, acc)
        Gnext = oracle.tgcn_bwd(graphs_bwd[i], p, Xs[i], Hp, f, G, oracle.zero_grads(Xs[i].shape[1], H))
    acc["loss"] = sl
    acc["H"] = sH
    acc["dH0"] = s_next
    return acc


def elementwise_err(gpu, ref, scale) -> float:
    """max_i |gpu_i − ref_i| / s_i (s_i = 0 requires an exact match)."""
    a = np.asarray(gpu, np.float64).reshape(-1)
    r = np.asarray(ref, np.float64).reshape(-1)
    s = np.broadcast_to(np.asarray(scale, np.float64), np.asarray(ref).shape).reshape(-1)
    zero = s == 0
    assert np.all(a[zero] == r[zero]), "mismatch where the condition scale is 0"
    d = np.abs(a - r)[~zero] / s[~zero]
    return float(d.max()) if d.size else 0.0


def parity_log(tag, **vals):
    """Append measured error ratios to $STG_PARITY_LOG (JSON lines) when set: the
    evidence behind the tolerances in DESIGN.md §7."""
    import json
    import os
    path = os.environ.get("STG_PARITY_LOG")
    if path:
        with open(path, "a") as fh:
            fh.write(json.dumps({"tag": str(tag), **{k: float(v) for k, v in vals.items()}}) + "\n")


def check_sequence(tag, gpu: dict, ref_grads: dict, scales: dict, tau: float = TAU_TGCN, normwise: float | None = None):
    """Element-wise parity of sequence gradients: |g_gpu − g_ref| <= tau · s (the
    condition scales of sequence_scales); optionally also the normwise bound
    max|Δ| <= normwise · max|ref| per tensor.  gpu: name -> numpy array."""
    errs = {}
    for k, a in gpu.items():
        e = elementwise_err(a, ref_grads[k], scales[k])
        errs[k] = e
        if normwise is not None:
            r = np.asarray(ref_grads[k], np.float64)
            den = np.max(np.abs(r)) or 1.0
            nw = float(np.max(np.abs(np.asarray(a, np.float64) - r)) / den)
            errs[k + "_normwise"] = nw
    parity_log(tag, **errs)
    for k in gpu:
        assert errs[k] <= tau, (tag, k, errs[k], tau)
        if normwise is not None:
            assert errs[k + "_normwise"] <= normwise, (tag, k, errs[k + "_normwise"], normwise)
    return errs
