"""Pins of the edge-weighted oracle (reading C21: PyG gcn_norm
with edge weights).  Each test pins oracle.aggregate_edges / oracle.weighted_norm to
something other than themselves:
* hand-derived closed forms on the weighted Fig. 3 graph (tests/golden/fig3_weighted.json);
* unit weights reduce exactly to the unweighted oracle (plain in-degree norms);
* dense brute force N·A_w·N·x with the weighted adjacency built by numpy;
* the adjoint identity <gy, Â_w x> = <Â_wᵀ gy, x>;
* a zero-weight edge is the same as a missing edge.
"""
import json
import os

import numpy as np
import pytest

import gen
import oracle

GOLD = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "fig3_weighted.json")


def _set_and_weights(V, src, dst, w):
    S = oracle.keys(src, dst)
    order = np.argsort(S)
    return S[order], np.asarray(w, np.float64)[order]


def test_fig3_weighted_closed_forms():
    g = json.load(open(GOLD))
    S, w = _set_and_weights(g["V"], g["src"], g["dst"], g["w"])
    n = oracle.weighted_norm(g["V"], S, w)
    np.testing.assert_allclose(n, g["norm"], rtol=1e-14)
    np.testing.assert_allclose(n ** -2, g["deg_w"], rtol=1e-14)
    x = np.asarray(g["x"], np.float64)[:, None]
    y = oracle.aggregate_edges(g["V"], S, w, n, n, x)
    np.testing.assert_allclose(y[:, 0], g["y"], rtol=1e-13)
    gx = oracle.aggregate_edges(g["V"], S, w, n, n, np.ones((4, 1)), backward=True)
    np.testing.assert_allclose(gx[:, 0], g["gx"], rtol=1e-13)


@pytest.mark.parametrize("name", ["C1", "C2", "C6"])
def test_unit_weights_reduce_to_unweighted(name):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    S = oracle.edge_set(cfg.V, s, d, self_loops=True)
    g = oracle.csr(cfg.V, S)
    w = np.ones(S.size)
    n = oracle.weighted_norm(cfg.V, S, w)
    np.testing.assert_allclose(n, g["norm_dst"], rtol=1e-15)
    x = gen.features(cfg, 0, width=8).astype(np.float64)
    np.testing.assert_allclose(oracle.aggregate_edges(cfg.V, S, w, n, n, x), oracle.aggregate_fwd(g, x),
                               rtol=1e-12, atol=1e-13)
    np.testing.assert_allclose(oracle.aggregate_edges(cfg.V, S, w, n, n, x, backward=True),
                               oracle.aggregate_bwd(g, x), rtol=1e-12, atol=1e-13)


@pytest.mark.parametrize("seed", range(12))
def test_weighted_dense_brute_force(seed):
    V = 5 + seed * 4
    s, d = gen.random_edges(seed, V, 3 * V, loops=True)
    S = oracle.edge_set(V, s, d, self_loops=True)
    w = gen.edge_weights(seed, S.size).astype(np.float64)
    if seed % 3 == 0:
        w[::5] = 0.0                                        # zero weights allowed
    u, v = oracle.unkey(S)
    A = np.zeros((V, V))
    A[v, u] = w                                             # A[v, u] = w(u -> v)
    deg = A.sum(axis=1)
    n = np.where(deg > 0, 1.0 / np.sqrt(np.where(deg > 0, deg, 1.0)), 0.0)
    np.testing.assert_allclose(oracle.weighted_norm(V, S, w), n, rtol=1e-14)
    x = gen.features(gen.CONFIGS["C1"], seed, width=3).astype(np.float64)[:V] if V <= 20 else \
        np.sin(np.arange(V * 3, dtype=np.float64)).reshape(V, 3)
    Ahat = n[:, None] * A * n[None, :]
    np.testing.assert_allclose(oracle.aggregate_edges(V, S, w, n, n, x), Ahat @ x, rtol=1e-12, atol=1e-14)
    np.testing.assert_allclose(oracle.aggregate_edges(V, S, w, n, n, x, backward=True), Ahat.T @ x, rtol=1e-12,
                               atol=1e-14)


def test_weighted_adjoint_and_zero_weight_edge():
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    S = oracle.edge_set(cfg.V, s, d, self_loops=True)
    w = gen.edge_weights(3, S.size).astype(np.float64)
    n = oracle.weighted_norm(cfg.V, S, w)
    x = gen.features(cfg, 0, width=4).astype(np.float64)
    gy = gen.features(cfg, 1, width=4).astype(np.float64)
    lhs = np.sum(gy * oracle.aggregate_edges(cfg.V, S, w, n, n, x))
    rhs = np.sum(oracle.aggregate_edges(cfg.V, S, w, n, n, gy, backward=True) * x)
    assert abs(lhs - rhs) <= 1e-10 * max(1.0, abs(lhs))
    # an edge with weight 0 contributes nothing (same as removing it, norms included)
    w0 = w.copy()
    w0[7] = 0.0
    keep = np.ones(S.size, bool)
    keep[7] = False
    n0 = oracle.weighted_norm(cfg.V, S, w0)
    np.testing.assert_array_equal(n0, oracle.weighted_norm(cfg.V, S[keep], w[keep]))
    np.testing.assert_allclose(oracle.aggregate_edges(cfg.V, S, w0, n0, n0, x),
                               oracle.aggregate_edges(cfg.V, S[keep], w[keep], n0, n0, x), rtol=0, atol=0)
