"""Pins of the original T-GCN oracle (GCN over [X, H], the
model the paper cites for TGCN):
* a one-vertex closed form derived by hand (tests/golden/tgcn2_scalar.json);
* zero parameters: r = u = 1/2, c = tanh(0) = 0, so H' = H/2 exactly;
* central finite differences of every gradient of the step and of a whole
  Algorithm-1 sequence with the surrogate head (BPTT through the state stack);
* the graph part: with Â = I (no edges, self-loops) the cell does not mix
  vertices, so permuting the vertices permutes H' (a property, not a retyping).
"""
import json
import os

import numpy as np
import pytest

import gen
import oracle

GOLD = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "tgcn2_scalar.json")


def _graph(V, seed, loops=True):
    s, d = gen.random_edges(seed, V, 3 * V, loops=loops)
    return oracle.static_graph(V, s, d, self_loops=True)


def test_scalar_closed_form():
    g0 = json.load(open(GOLD))
    gr = oracle.static_graph(1, [0], [0], self_loops=True)
    p = {"Wg": np.array(g0["Wg"]), "bg": np.array(g0["bg"]), "Wc": np.array(g0["Wc"]), "bc": np.array(g0["bc"])}
    f = oracle.tgcn2_fwd(gr, p, np.array([[g0["x"]]]), np.array([[g0["h"]]]))
    for k, key in (("R", "r"), ("U", "u"), ("Cc", "c"), ("Hn", "h_next")):
        assert abs(f[k][0, 0] - g0[key]) <= 1e-15, k


def test_zero_parameters_halve_the_state():
    V, F, H = 30, 5, 6
    g = _graph(V, 1)
    p = {"Wg": np.zeros((F + H, 2 * H)), "bg": np.zeros(2 * H), "Wc": np.zeros((F + H, H)), "bc": np.zeros(H)}
    X = np.random.default_rng(0).standard_normal((V, F))
    Hp = np.random.default_rng(1).standard_normal((V, H))
    f = oracle.tgcn2_fwd(g, p, X, Hp)
    np.testing.assert_array_equal(f["Hn"], 0.5 * Hp)


def test_identity_graph_permutation_equivariance():
    V, F, H = 16, 3, 4
    g = oracle.static_graph(V, [], [], self_loops=True)
    p = gen.tgcn2_params(F, H, 3)
    rng = np.random.default_rng(2)
    X, Hp = rng.standard_normal((V, F)), rng.standard_normal((V, H))
    perm = rng.permutation(V)
    a = oracle.tgcn2_fwd(g, p, X, Hp)["Hn"]
    b = oracle.tgcn2_fwd(g, p, X[perm], Hp[perm])["Hn"]
    np.testing.assert_allclose(b, a[perm], rtol=0, atol=1e-15)


def _fd_check(fun, x, g_analytic, idx, h=1e-6, tol=1e-6):
    for i in idx:
        xp, xm = x.copy(), x.copy()
        xp.flat[i] += h
        xm.flat[i] -= h
        num = (fun(xp) - fun(xm)) / (2 * h)
        assert abs(num - g_analytic.flat[i]) <= tol * max(1.0, abs(num)), (i, num, g_analytic.flat[i])


@pytest.mark.parametrize("seed", [0, 1])
def test_step_finite_differences(seed):
    V, F, H = 14, 3, 4
    g = _graph(V, 10 + seed)
    p = {k: np.asarray(v, np.float64) for k, v in gen.tgcn2_params(F, H, seed).items()}
    rng = np.random.default_rng(seed)
    X, Hp, Q = rng.standard_normal((V, F)), rng.standard_normal((V, H)), rng.standard_normal((V, H))

    def loss(pp, Hc):
        return float(np.sum(oracle.tgcn2_fwd(g, pp, X, Hc)["Hn"] * Q))
    f = oracle.tgcn2_fwd(g, p, X, Hp)
    grads = oracle.zero_grads2(F, H)
    dHp = oracle.tgcn2_bwd(g, p, X, Hp, f, Q, grads)
    sel = rng.choice
    for k in ("Wg", "bg", "Wc", "bc"):
        def fk(v, k=k):
            pp = dict(p)
            pp[k] = v
            return loss(pp, Hp)
        _fd_check(fk, p[k], grads[k], sel(p[k].size, min(12, p[k].size), replace=False))
    _fd_check(lambda v: loss(p, v), Hp, dHp, sel(Hp.size, 12, replace=False))


def test_sequence_bptt_finite_differences():
    V, F, H, S = 12, 3, 4, 3
    g = _graph(V, 21)
    p = {k: np.asarray(v, np.float64) for k, v in gen.tgcn2_params(F, H, 5).items()}
    rng = np.random.default_rng(7)
    Xs = [rng.standard_normal((V, F)) for _ in range(S)]
    Ys = [rng.standard_normal(V) for _ in range(S)]
    H0 = np.zeros((V, H))
    _, grads, _ = oracle.train_sequence2([g] * S, p, Xs, Ys, H0)
    for k in ("Wg", "bg", "Wc", "bc", "w_o", "b_o"):
        def fk(v, k=k):
            pp = dict(p)
            pp[k] = v
            return oracle.train_sequence2([g] * S, pp, Xs, Ys, H0)[0]
        _fd_check(fk, p[k], grads[k], rng.choice(p[k].size, min(8, p[k].size), replace=False))
