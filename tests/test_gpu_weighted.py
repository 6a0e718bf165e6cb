"""GPU parity of the edge-weighted aggregation against the
edge-set oracle (oracle.aggregate_edges / weighted_norm, pinned in
tests/test_oracle_weighted.py).  The weights live in in-CSR order (the edge label,
P:L197, reading C6): the forward reads ew[j], the backward reaches the same weight
through out_eid.  Tolerances: C19 condition-scaled 1e-5 for the aggregation,
fp32 rounding of an fp64 sum for the norms."""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import cond_err, to_gpu

pytestmark = pytest.mark.gpu


def _in_csr_weights(S, w, in_rowptr, in_col):
    """The weight of every in-CSR position (edge (in_col[j] -> row)), looked up by edge key."""
    V = len(in_rowptr) - 1
    rows = np.repeat(np.arange(V), np.diff(in_rowptr))
    k = oracle.keys(np.asarray(in_col), rows)
    idx = np.searchsorted(S, k)
    assert np.array_equal(S[idx], k)
    return np.asarray(w)[idx]


def _weighted_case(stg, V, S, w, view, W, seed):
    a = stg.view_arrays(view)
    ew_np = _in_csr_weights(S, w, a["in_rowptr"].cpu().numpy(), a["in_col"].cpu().numpy())
    ew = to_gpu(ew_np)
    n_ref = oracle.weighted_norm(V, S, w.astype(np.float64))
    n = stg.stg_gcn_weighted_norm(view, ew)
    np.testing.assert_allclose(n.cpu().numpy().astype(np.float64), n_ref, rtol=2.5e-7, atol=0)
    cfg = gen.CONFIGS["C1"]
    x = gen.uniform_pm1(seed, 50, V * W).reshape(V, W).astype(np.float64)
    y = stg.stg_gcn_aggregate_weighted(view, False, ew, to_gpu(x), scale_row=n, scale_col=n).cpu().numpy()
    ref = oracle.aggregate_edges(V, S, w, n_ref, n_ref, x)
    sc = oracle.aggregate_edges(V, S, w, n_ref, n_ref, np.abs(x))
    assert cond_err(y, ref, sc) <= 1e-5
    gx = stg.stg_gcn_aggregate_weighted(view, True, ew, to_gpu(x), scale_row=n, scale_col=n).cpu().numpy()
    ref = oracle.aggregate_edges(V, S, w, n_ref, n_ref, x, backward=True)
    sc = oracle.aggregate_edges(V, S, w, n_ref, n_ref, np.abs(x), backward=True)
    assert cond_err(gx, ref, sc) <= 1e-5
    return ew, n


@pytest.mark.parametrize("name,W", [("C1", 48), ("C2", 96), ("C6", 8), ("C3", 64), ("C2", 256)])
def test_weighted_static(stg, name, W):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    S = oracle.edge_set(cfg.V, s, d, self_loops=True)
    w = gen.edge_weights(cfg.seed, S.size).astype(np.float64)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    _weighted_case(stg, cfg.V, S, w, g.view(), W, cfg.seed)


def test_weighted_dtdg_snapshots(stg):
    """Weights of a DTDG snapshot (hub rows with chunk partials): Get-Graph and Get-Backward-Graph views."""
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    g = stg.stg_dtdg_create(dd.V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off,
                            dd.del_src, dd.del_dst, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    sets = list(oracle.snapshot_sets_fold(dd, self_loops=True))
    for t in (0, 3):
        S = sets[t]
        w = gen.edge_weights(t + 7, S.size).astype(np.float64)
        _weighted_case(stg, dd.V, S, w, stg.stg_dtdg_get_snapshot(g, t), 96, t)


def test_unit_weights_bit_identical_to_unweighted(stg):
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    v = g.view()
    a = stg.view_arrays(v)
    ones = torch.ones(v.num_edges, device="cuda")
    n = stg.stg_gcn_weighted_norm(v, ones)
    # the library's unweighted norms are 1.0f/sqrtf(deg) (two fp32 roundings, reading C1); the
    # weighted norm is the correctly rounded deg^-1/2: equal to within one ulp
    torch.testing.assert_close(n, a["norm_dst"], rtol=2.5e-7, atol=0)
    x = to_gpu(gen.features(cfg, 0, width=96))
    for bwd in (False, True):
        y0 = stg.stg_gcn_aggregate_ex(v, bwd, x, scale_row=a["norm_dst"], scale_col=a["norm_src"])
        y1 = stg.stg_gcn_aggregate_weighted(v, bwd, ones, x, scale_row=a["norm_dst"], scale_col=a["norm_src"])
        assert torch.equal(y0, y1), bwd


def test_weighted_rejects_bad_args(stg):
    cfg = gen.CONFIGS["C6"]
    s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)      # no edge labels
    v = g.view()
    ew = torch.ones(v.num_edges, device="cuda")
    x = torch.zeros(cfg.V, 8, device="cuda")
    with pytest.raises(stg.StgError):                       # backward needs out_eid
        stg.stg_gcn_aggregate_weighted(v, True, ew, x)
    with pytest.raises(stg.StgError):                       # W % 4
        stg.stg_gcn_aggregate_weighted(v, False, ew, torch.zeros(cfg.V, 6, device="cuda"))


def test_weighted_sharded_blocks(stg):
    """Row-block sharded views: each rank's weights in ITS in-CSR order; the
    forward rows equal the whole-graph rows, the backward partials sum to the oracle."""
    from paper_conf_ipps_cherianmcc24_b200 import parallel
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    V, W, world = cfg.V, 64, 3
    S = oracle.edge_set(V, s, d, self_loops=True)
    w = gen.edge_weights(11, S.size).astype(np.float64)
    flags = stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS
    gfull = stg.stg_static_graph_create(V, s, d, flags)
    af = stg.view_arrays(gfull.view())
    ew_full = to_gpu(_in_csr_weights(S, w, af["in_rowptr"].cpu().numpy(), af["in_col"].cpu().numpy()))
    n = stg.stg_gcn_weighted_norm(gfull.view(), ew_full)
    n_ref = oracle.weighted_norm(V, S, w)
    x = gen.uniform_pm1(5, 90, V * W).reshape(V, W).astype(np.float64)
    y_full = stg.stg_gcn_aggregate_weighted(gfull.view(), False, ew_full, to_gpu(x), scale_row=n, scale_col=n)
    b = parallel.base_row_blocks(V, s, d, world)
    gx_sum = np.zeros((V, W))
    for k in range(world):
        lo, hi = b[k], b[k + 1]
        g = stg.stg_static_graph_create(V, s, d, flags, dist=(k, world, lo, hi))
        v = g.view()
        a = stg.view_arrays(v)
        rows = np.repeat(np.arange(lo, hi), np.diff(a["in_rowptr"].cpu().numpy()))
        keys = oracle.keys(a["in_col"].cpu().numpy(), rows)
        ew = to_gpu(np.asarray(w)[np.searchsorted(S, keys)])
        y = stg.stg_gcn_aggregate_weighted(v, False, ew, to_gpu(x), scale_row=n[lo:hi].contiguous(), scale_col=n)
        assert torch.equal(y, y_full[lo:hi]), k
        gx = stg.stg_gcn_aggregate_weighted(v, True, ew, to_gpu(x[lo:hi]), scale_row=n,
                                            scale_col=n[lo:hi].contiguous())
        gx_sum += gx.cpu().numpy()
    ref = oracle.aggregate_edges(V, S, w, n_ref, n_ref, x, backward=True)
    sc = oracle.aggregate_edges(V, S, w, n_ref, n_ref, np.abs(x), backward=True)
    assert cond_err(gx_sum, ref, sc) <= 1e-5
