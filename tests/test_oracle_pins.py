"""Pins of the fp64 oracle against things other than itself (-m "not gpu").

Each test names what fixes the expected value: the paper's worked example
(tests/golden/fig3_four_node.json), closed forms derived by hand,
mathematical invariants (adjoint, transpose), brute force with dense numpy
matrices, the paper's own Algorithm 3 as an independent transpose,
the event-window definition of a snapshot, torch.nn.GRUCell as the
textbook GRU in the special cases where the TGCN reading reduces to it, and
central finite differences for every gradient.
"""
import json
import os
import random

import numpy as np
import pytest
import torch

import gen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden", "fig3_four_node.json")


@pytest.fixture(scope="module")
def fig3():
    with open(GOLD) as f:
        return json.load(f)


# ------------------------------------------------------------------ CSR pins
def test_fig3_csr_and_node_ids(fig3):
    g = oracle.static_graph(fig3["V"], fig3["src"], fig3["dst"])
    exp = fig3["no_loops"]
    for k in ("in_rowptr", "in_col", "out_rowptr", "out_col", "out_eid", "in_deg", "out_deg",
              "out_ids", "in_ids"):
        assert g[k].tolist() == exp[k], k
    # "V2 followed by V0, V1 and then finally V3"
    assert g["out_ids"].tolist() == [2, 0, 1, 3]


def test_fig3_self_loop_degrees(fig3):
    g = oracle.static_graph(4, fig3["src"], fig3["dst"], self_loops=True)
    assert g["in_deg"].tolist() == fig3["self_loops"]["in_deg"]
    assert g["out_deg"].tolist() == fig3["self_loops"]["out_deg"]


def test_fig3_aggregation_closed_forms(fig3):
    x = np.array(fig3["self_loops"]["x"], np.float64)[:, None]
    g = oracle.static_graph(4, fig3["src"], fig3["dst"], self_loops=True)
    np.testing.assert_allclose(oracle.aggregate_fwd(g, x).ravel(), fig3["self_loops"]["y_fwd"], rtol=1e-14)
    gy = np.array(fig3["self_loops"]["gy"], np.float64)[:, None]
    gx = oracle.aggregate_bwd(g, gy).ravel()
    np.testing.assert_allclose(gx, fig3["self_loops"]["gx_bwd"], rtol=1e-14)
    # adjoint: <1, Â x> = <Âᵀ 1, x>
    assert abs(float(gx @ x.ravel()) - fig3["self_loops"]["adjoint_sum"]) < 1e-12
    g0 = oracle.static_graph(4, fig3["src"], fig3["dst"])
    np.testing.assert_allclose(oracle.aggregate_fwd(g0, x).ravel(), fig3["no_loops"]["y_fwd"], rtol=1e-14)
    gd = oracle.static_graph(4, fig3["src"], fig3["dst"], self_loops=True, dgl_both=True)
    np.testing.assert_allclose(oracle.aggregate_fwd(gd, x).ravel(), fig3["self_loops"]["dgl_both_y_fwd"], rtol=1e-14)


def _dense_reference(V, src, dst, loops, dgl_both, x):
    """Brute force: dense adjacency A[v,u] = 1 iff u->v, Â = N_d A N_s, y = Â x."""
    A = np.zeros((V, V))
    A[np.asarray(dst), np.asarray(src)] = 1.0
    if loops:
        A[np.arange(V), np.arange(V)] = 1.0
    din, dout = A.sum(1), A.sum(0)
    inv = lambda d: np.where(d > 0, 1.0 / np.sqrt(np.maximum(d, 1)), 0.0)
    nd = inv(din)
    ns = inv(dout) if dgl_both else inv(din)
    Ahat = nd[:, None] * A * ns[None, :]
    return Ahat, A


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("loops", [False, True])
@pytest.mark.parametrize("dgl_both", [False, True])
def test_aggregation_dense_brute_force(seed, loops, dgl_both):
    rng = np.random.default_rng(seed)
    V = int(rng.integers(1, 65))
    E = int(rng.integers(0, 4 * V))
    src, dst = gen.random_edges(seed, V, E)
    W = int(rng.integers(1, 7))
    x = gen.uniform_pm1(seed, 77, V * W).reshape(V, W).astype(np.float64)
    g = oracle.static_graph(V, src, dst, self_loops=loops, dgl_both=dgl_both)
    Ahat, A = _dense_reference(V, src, dst, loops, dgl_both, x)
    assert g["E"] == int(A.sum())
    np.testing.assert_allclose(oracle.aggregate_fwd(g, x), Ahat @ x, rtol=1e-12, atol=1e-13)
    gy = gen.uniform_pm1(seed, 78, V * W).reshape(V, W).astype(np.float64)
    np.testing.assert_allclose(oracle.aggregate_bwd(g, gy), Ahat.T @ gy, rtol=1e-12, atol=1e-13)
    # degrees and rowptr against the dense matrix
    assert g["in_deg"].tolist() == A.sum(1).astype(int).tolist()
    assert g["out_deg"].tolist() == A.sum(0).astype(int).tolist()


def test_transpose_invariant_bit_exact():
    """bwd(G; n_s, n_d) == fwd(Gᵀ; n_d, n_s) exactly in the oracle."""
    V = 300
    src, dst = gen.random_edges(11, V, 2500)
    g = oracle.static_graph(V, src, dst, self_loops=True)
    gt = oracle.static_graph(V, dst, src, self_loops=True)
    x = gen.uniform_pm1(11, 5, V * 3).reshape(V, 3)
    bwd = oracle.aggregate(g["out_rowptr"], g["out_col"], g["norm_src"], g["norm_dst"], x)
    fwdT = oracle.aggregate(gt["in_rowptr"], gt["in_col"], g["norm_src"], g["norm_dst"], x)
    assert np.array_equal(bwd, fwdT)


def test_complete_graph_is_mean():
    """C3 shape: complete graph with loops => y_v = mean_u x_u for every v."""
    cfg = gen.CONFIGS["C3"]
    s, d = gen.static_edges(cfg)
    g = oracle.static_graph(cfg.V, s, d, self_loops=True)
    assert g["E"] == cfg.V * cfg.V
    x = gen.features(cfg, 0).astype(np.float64)
    y = oracle.aggregate_fwd(g, x)
    np.testing.assert_allclose(y, np.broadcast_to(x.mean(0), y.shape), rtol=1e-12, atol=1e-14)


def test_empty_graph_with_loops_is_identity():
    V = 37
    g = oracle.static_graph(V, np.zeros(0, np.int32), np.zeros(0, np.int32), self_loops=True)
    x = gen.uniform_pm1(3, 3, V * 5).reshape(V, 5).astype(np.float64)
    assert np.array_equal(oracle.aggregate_fwd(g, x), x)
    g0 = oracle.static_graph(V, np.zeros(0, np.int32), np.zeros(0, np.int32))
    assert np.array_equal(oracle.aggregate_fwd(g0, x), np.zeros_like(x))


def _reverse_gpma(V, row_offset, col, eids, in_degrees, order_seed):
    """Algorithm 3, reading C7 (0-based, end-exclusive, loc = old-1),
    with the parallel loop over i executed in a random order (atomic interleaving)."""
    r_row_offset = np.cumsum(in_degrees).astype(np.int64)       # inclusive prefix sum
    E = int(row_offset[-1])
    r_col = np.full(E, -1, np.int64)
    r_eids = np.full(E, -1, np.int64)
    rows = list(range(V))
    random.Random(order_seed).shuffle(rows)
    for i in rows:
        for j in range(row_offset[i], row_offset[i + 1]):
            dst, eid = col[j], eids[j]
            r_row_offset[dst] -= 1                                 # atomic_sub -> old-1
            loc = r_row_offset[dst]
            r_col[loc] = i
            r_eids[loc] = eid
    return np.append(r_row_offset, E), r_col, r_eids


@pytest.mark.parametrize("name", ["C1", "C2", "C6"])
def test_algorithm3_transpose_matches_csr(name):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    g = oracle.static_graph(cfg.V, s, d, self_loops=True)
    for seed in range(3):
        rro, rcol, reid = _reverse_gpma(cfg.V, g["out_rowptr"], g["out_col"], g["out_eid"], g["in_deg"], seed)
        assert rro.tolist() == g["in_rowptr"].tolist()
        for v in range(cfg.V):
            a, b = rro[v], rro[v + 1]
            o = np.argsort(rcol[a:b], kind="stable")            # reading C3: ascending ids
            assert rcol[a:b][o].tolist() == g["in_col"][a:b].tolist()
            # shared edge labels: the label carried by Alg. 3 is the in-CSR slot
            assert reid[a:b][o].tolist() == list(range(a, b))


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C6"])
def test_csr_invariants(name):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    for loops in (False, True):
        g = oracle.static_graph(cfg.V, s, d, self_loops=loops)
        E = g["E"]
        assert g["in_rowptr"][-1] == E == g["out_rowptr"][-1]
        assert g["in_deg"].sum() == E == g["out_deg"].sum()
        for k, dk in (("in_ids", "in_deg"), ("out_ids", "out_deg")):
            ids = g[k]
            assert sorted(ids.tolist()) == list(range(cfg.V))
            dd = g[dk][ids]
            assert np.all(dd[:-1] >= dd[1:])
            tie = dd[:-1] == dd[1:]
            assert np.all(ids[:-1][tie] < ids[1:][tie])
        u = np.repeat(np.arange(cfg.V), np.diff(g["out_rowptr"]))
        assert np.array_equal(g["in_col"][g["out_eid"]], u)
        v_of_in = np.repeat(np.arange(cfg.V), np.diff(g["in_rowptr"]))
        assert np.array_equal(v_of_in[g["out_eid"]], g["out_col"])
    if name == "C1":
        assert oracle.static_graph(cfg.V, s, d)["E"] == 102       # Table II: 102 edges
    if name == "C3":
        assert oracle.static_graph(cfg.V, s, d)["E"] == 101761    # 319^2 ("102K")


# -------------------------------------------------------------- snapshot pins
def test_effective_deltas_brute_force():
    rng = random.Random(5)
    for trial in range(200):
        V = rng.randint(1, 6)
        pairs = [(a, b) for a in range(V) for b in range(V)]
        S = set(rng.sample(pairs, rng.randint(0, len(pairs))))
        A = [rng.choice(pairs) for _ in range(rng.randint(0, 8))]
        D = [rng.choice(pairs) for _ in range(rng.randint(0, 8))]
        loops = trial % 2 == 1
        if loops:
            S |= {(v, v) for v in range(V)}
        k = lambda L: oracle.keys([p[0] for p in L], [p[1] for p in L]) if L else np.zeros(0, np.uint64)
        Sk = np.sort(k(sorted(S)))
        a, d = oracle.effective_deltas(Sk, k(A), k(D), pinned_loops=loops)
        expA = set(A) - S
        expD = {p for p in (set(D) - set(A)) & S if not (loops and p[0] == p[1])}
        got = lambda arr: set(zip(*[x.tolist() for x in oracle.unkey(arr)])) if arr.size else set()
        assert got(a) == expA and got(d) == expD
        # the effective deltas reproduce S_t = (S \ D) ∪ A and are exactly reversible
        St = (S - (set(D) - (set((v, v) for v in range(V)) if loops else set()))) | set(A)
        St2 = oracle.set_apply(Sk, d, a)
        assert got(St2) == St
        back = oracle.set_apply(St2, a, d)
        assert np.array_equal(back, Sk)


@pytest.mark.parametrize("name", ["C4", "C5s"])
def test_snapshot_fold_equals_event_window(name):
    """S_t by folding the stored batches == S_t straight from the window."""
    cfg = gen.CONFIGS[name]
    d = gen.dtdg(cfg)
    assert d.add_off[1] == 0 and d.del_off[1] == 0            # batch 0 is empty (base)
    for t, S in enumerate(oracle.snapshot_sets_fold(d)):
        assert np.array_equal(S, oracle.snapshot_set_window(d, t)), t
    # the generator's batches are already effective: normalisation is the identity
    S_prev = None
    for t, S in enumerate(oracle.snapshot_sets_fold(d)):
        if S_prev is not None:
            A, D = oracle.batch(d, t)
            a, dd = oracle.effective_deltas(S_prev, A, D)
            assert np.array_equal(np.sort(A), a) and np.array_equal(np.sort(D), dd)
        S_prev = S
        if t > 6:
            break


def test_snapshot_change_rate_is_about_5_percent():
    """Reading C12: slide chosen so the mean change per step is ≈5%."""
    for name in ("C4", "C5s"):
        d = gen.dtdg(gen.CONFIGS[name])
        sizes, changes = [], []
        for t, S in enumerate(oracle.snapshot_sets_fold(d)):
            if t:
                n = (d.add_off[t + 1] - d.add_off[t]) + (d.del_off[t + 1] - d.del_off[t])
                changes.append(n / sizes[-1])
            sizes.append(S.size)
        assert 0.04 < np.mean(changes) < 0.06, (name, np.mean(changes))
        assert max(changes) < 0.10                                # "always less than 10%"


# ------------------------------------------------------------------ TGCN pins
def _tiny(seed=0, V=7, F=3, H=2, loops=True):
    s, d = gen.random_edges(seed, V, 3 * V)
    g = oracle.static_graph(V, s, d, self_loops=loops)
    p = {k: v.astype(np.float64) for k, v in gen.tgcn_params(F, H, seed, scale=2.0).items()}
    X = gen.uniform_pm1(seed, 1, V * F).reshape(V, F).astype(np.float64)
    Hp = gen.uniform_pm1(seed, 2, V * H).reshape(V, H).astype(np.float64)
    return g, p, X, Hp


def test_tgcn_zero_parameters_closed_form():
    g, p, X, Hp = _tiny()
    p0 = {k: np.zeros_like(v) for k, v in p.items()}
    f = oracle.tgcn_fwd(g, p0, X, Hp)
    assert np.all(f["Z"] == 0.5) and np.all(f["R"] == 0.5) and np.all(f["Hh"] == 0.0)
    assert np.array_equal(f["Hn"], 0.5 * Hp)


@pytest.mark.parametrize("seed", range(3))
def test_tgcn_identity_graph_reduces_to_torch_grucell(seed):
    """Â = I (no edges + self-loops) and a diagonal L_h²: the TGCN cell equals
    torch.nn.GRUCell on input P = X·W + b (the two reset-gate placements agree
    when the hidden-to-candidate map is diagonal)."""
    V, F, H = 9, 4, 3
    g = oracle.static_graph(V, np.zeros(0, np.int32), np.zeros(0, np.int32), self_loops=True)
    _, p, X, Hp = _tiny(seed, V, F, H)
    p["L"][2, H:, :] = np.diag(np.diag(p["L"][2, H:, :]))
    f = oracle.tgcn_fwd(g, p, X, Hp)
    P = X @ p["W"] + p["b"]
    cell = torch.nn.GRUCell(3 * H, H, bias=True).double()
    Lz, Lr, Lh = p["L"]
    with torch.no_grad():
        # torch row order of weight_ih / weight_hh: r, z, n
        Wih = np.zeros((3 * H, 3 * H)); Whh = np.zeros((3 * H, H))
        Wih[0:H, H:2 * H] = Lr[:H].T; Wih[H:2 * H, 0:H] = Lz[:H].T; Wih[2 * H:, 2 * H:] = Lh[:H].T
        Whh[0:H] = Lr[H:].T; Whh[H:2 * H] = Lz[H:].T; Whh[2 * H:] = Lh[H:].T
        cell.weight_ih.copy_(torch.from_numpy(Wih)); cell.weight_hh.copy_(torch.from_numpy(Whh))
        bih = np.concatenate([p["l"][1], p["l"][0], p["l"][2]])
        cell.bias_ih.copy_(torch.from_numpy(bih)); cell.bias_hh.zero_()
        ref = cell(torch.from_numpy(P), torch.from_numpy(Hp)).numpy()
    np.testing.assert_allclose(f["C"], P, rtol=1e-14, atol=1e-15)
    np.testing.assert_allclose(f["Hn"], ref, rtol=1e-12, atol=1e-13)


def _fd_check(fun, arr, analytic, h=1e-6, rtol=1e-6, n=12, seed=0):
    rng = np.random.default_rng(seed)
    flat = arr.reshape(-1)
    idx = rng.choice(flat.size, size=min(n, flat.size), replace=False)
    for i in idx:
        old = flat[i]
        flat[i] = old + h; fp = fun()
        flat[i] = old - h; fm = fun()
        flat[i] = old
        num = (fp - fm) / (2 * h)
        an = analytic.reshape(-1)[i]
        assert abs(num - an) <= rtol * max(1.0, abs(num), abs(an)) + 1e-9, (i, num, an)


@pytest.mark.parametrize("seed", range(3))
def test_tgcn_backward_finite_differences(seed):
    g, p, X, Hp = _tiny(seed)
    V, H = Hp.shape
    G = gen.uniform_pm1(seed, 9, V * H).reshape(V, H).astype(np.float64)
    loss = lambda: float(np.sum(G * oracle.tgcn_fwd(g, p, X, Hp)["Hn"]))
    f = oracle.tgcn_fwd(g, p, X, Hp)
    grads = oracle.zero_grads(X.shape[1], H)
    dHp = oracle.tgcn_bwd(g, p, X, Hp, f, G, grads)
    for k in ("W", "b", "L", "l"):
        _fd_check(loss, p[k], grads[k], seed=seed)
    _fd_check(loss, Hp, dHp, seed=seed)


def test_sequence_bptt_and_head_finite_differences():
    """Algorithm 1 over one sequence: accumulated grads == d(Σ_t ℓ_t)/dθ."""
    V, F, H, S = 6, 3, 2, 4
    g, p, _, H0 = _tiny(4, V, F, H)
    Xs = [gen.uniform_pm1(4, 100 + t, V * F).reshape(V, F).astype(np.float64) for t in range(S)]
    Ys = [gen.uniform_pm1(4, 200 + t, V).astype(np.float64) for t in range(S)]
    gs = [g] * S
    loss0, grads, _ = oracle.train_sequence(gs, gs, p, Xs, Ys, H0)
    fun = lambda: oracle.train_sequence(gs, gs, p, Xs, Ys, H0)[0]
    for k in ("W", "b", "L", "l", "w_o", "b_o"):
        _fd_check(fun, p[k], grads[k], n=8)


def test_mse_head_hand_derived_golden():
    """orc_mse_head's LOSS VALUE and gradients against hand-derived closed forms
    (tests/golden/mse_head_hand.json): pins the surrogate's definition itself
    (mean, not sum; ReLU before w_o; b_o outside the ReLU), which the finite
    difference tests cannot (they only check the gradient against the loss)."""
    import json
    import os
    spec = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "mse_head_hand.json")))
    for c in spec["cases"]:
        Hn = np.array(c["H"], np.float64)
        grads = {"w_o": np.zeros(Hn.shape[1]), "b_o": np.zeros(1)}
        loss, dH = oracle.mse_head(Hn, np.array(c["y"]), np.array(c["w_o"]), c["b_o"], grads)
        assert loss == pytest.approx(c["loss"], rel=1e-15, abs=1e-15), c["name"]
        np.testing.assert_allclose(dH, np.array(c["dH"]), rtol=1e-15, atol=1e-15, err_msg=c["name"])
        np.testing.assert_allclose(grads["w_o"], np.array(c["dw_o"]), rtol=1e-15, atol=1e-15, err_msg=c["name"])
        assert grads["b_o"][0] == pytest.approx(c["db_o"], rel=1e-15, abs=1e-15), c["name"]


def test_openmp_timing_build_matches_plain():
    """The OpenMP build of the same source (bench.py's all-core CPU baseline only)
    computes the same step: row-parallel results bit-identical, thread-reduced
    parameter gradients equal up to fp64 reassociation."""
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    g = oracle.static_graph(cfg.V, s, d, self_loops=True)
    p = gen.tgcn_params(cfg.F, cfg.H, 5)
    X = gen.features(cfg, 3)
    Hp = gen.uniform_pm1(2, 2, cfg.V * cfg.H).reshape(cfg.V, cfg.H)
    G = gen.uniform_pm1(3, 3, cfg.V * cfg.H).reshape(cfg.V, cfg.H)
    out = []
    try:
        for omp in (False, True):
            oracle.use_openmp(omp)
            f = oracle.tgcn_fwd(g, p, X, Hp)
            gr = oracle.zero_grads(cfg.F, cfg.H)
            dH = oracle.tgcn_bwd(g, p, X, Hp, f, G, gr)
            out.append((f, gr, dH))
    finally:
        oracle.use_openmp(False)
    (f0, g0, d0), (f1, g1, d1) = out
    for k in ("C", "Z", "R", "Hh", "Hn"):
        assert np.array_equal(f0[k], f1[k]), k
    assert np.array_equal(d0, d1)
    for k in ("W", "b", "L", "l"):
        np.testing.assert_allclose(g1[k], g0[k], rtol=1e-12, atol=1e-12 * np.abs(g0[k]).max(), err_msg=k)
