"""GPU parity: static graph build and the GCN aggregation vs the fp64 oracle."""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import assert_graph_equal, cond_err, to_gpu

pytestmark = pytest.mark.gpu

TOL = 1e-5   # north_star: max relative error 1e-5 (condition-scaled, reading C19)


def _build(stg, V, s, d, loops=False, dgl=False, eids=True):
    flags = (stg.STG_SELF_LOOPS if loops else 0) | (stg.STG_NORM_DGL_BOTH if dgl else 0) | \
            (stg.STG_EDGE_IDS if eids else 0)
    g = stg.stg_static_graph_create(V, s, d, flags)
    ref = oracle.static_graph(V, s, d, self_loops=loops, dgl_both=dgl)
    return g, ref


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C6"])
@pytest.mark.parametrize("loops", [False, True])
def test_static_graph_bit_exact(stg, name, loops):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    g, ref = _build(stg, cfg.V, s, d, loops=loops)
    v = g.view()
    assert v.num_edges == ref["E"] and v.num_nodes == cfg.V
    assert_graph_equal(stg.view_arrays(v), ref, tag=name)


@pytest.mark.parametrize("seed", range(8))
def test_random_graph_bit_exact(stg, seed):
    rng = np.random.default_rng(seed)
    V = int(rng.integers(1, 5000))
    E = int(rng.integers(0, 20 * V))
    s, d = gen.random_edges(seed, V, E)         # duplicates and loops included
    for loops in (False, True):
        for dgl in (False, True):
            g, ref = _build(stg, V, s, d, loops=loops, dgl=dgl)
            assert_graph_equal(stg.view_arrays(g.view()), ref, tag=(seed, loops, dgl))


def test_fig3_worked_example(stg, ):
    import json, os
    fx = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "fig3_four_node.json")))
    g = stg.stg_static_graph_create(4, fx["src"], fx["dst"], stg.STG_EDGE_IDS)
    a = stg.view_arrays(g.view())
    for k in ("in_rowptr", "in_col", "out_rowptr", "out_col", "out_eid", "in_deg", "out_ids", "in_ids"):
        assert a[k].cpu().tolist() == fx["no_loops"][k], k
    gl = stg.stg_static_graph_create(4, fx["src"], fx["dst"], stg.STG_SELF_LOOPS)
    x = torch.tensor(fx["self_loops"]["x"], dtype=torch.float32, device="cuda")[:, None].contiguous()
    y = stg.stg_gcn_aggregate_fwd(gl.view(), x)
    np.testing.assert_allclose(y.cpu().numpy().ravel(), fx["self_loops"]["y_fwd"], rtol=1e-6)
    gx = stg.stg_gcn_aggregate_bwd(gl.view(), torch.ones(4, 1, device="cuda"))
    np.testing.assert_allclose(gx.cpu().numpy().ravel(), fx["self_loops"]["gx_bwd"], rtol=1e-6)


def test_invalid_ids_rejected(stg):
    with pytest.raises(stg.StgError) as e:
        stg.stg_static_graph_create(10, [0, 1, 10], [1, 2, 3])
    assert e.value.status == 2


def _agg_check(stg, g, ref, x, bwd=False):
    xg = to_gpu(x)
    if bwd:
        y = stg.stg_gcn_aggregate_bwd(g.view(), xg)
        r = oracle.aggregate_bwd(ref, x)
    else:
        y = stg.stg_gcn_aggregate_fwd(g.view(), xg)
        r = oracle.aggregate_fwd(ref, x)
    s = oracle.aggregate_scale(ref, x, bwd=bwd)
    return cond_err(y.cpu().numpy(), r, s), y


WIDTHS = [1, 3, 4, 8, 16, 48, 64, 96, 128, 132, 200, 516]


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C6"])
@pytest.mark.parametrize("W", WIDTHS)
def test_aggregation_parity_configs(stg, name, W):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    g, ref = _build(stg, cfg.V, s, d, loops=True)
    x = gen.features(cfg, 3, width=W).astype(np.float64)
    for bwd in (False, True):
        e, _ = _agg_check(stg, g, ref, x, bwd)
        assert e <= TOL, (name, W, bwd, e)
    # nonnegative inputs: plain relative error
    xp = gen.features(cfg, 4, width=W, nonneg=True).astype(np.float64)
    y = stg.stg_gcn_aggregate_fwd(g.view(), to_gpu(xp)).cpu().numpy()
    r = oracle.aggregate_fwd(ref, xp)
    nz = r > 0
    assert np.all(y[~nz] == 0)
    assert np.max(np.abs(y[nz] - r[nz]) / r[nz]) <= TOL


def test_aggregation_hubs_and_ragged(stg):
    """Power-law star hubs (multiple hub chunks, >16 chunks per row), empty rows, ragged tail."""
    V = 70001
    rng = np.random.default_rng(1)
    hub_src = rng.integers(0, V, 60000)
    s = np.concatenate([hub_src, np.full(3000, 5), rng.integers(0, V, 40000)])
    d = np.concatenate([np.full(60000, 17), rng.integers(0, V, 3000), rng.integers(0, 1000, 40000)])
    for loops, dgl in ((True, False), (False, True)):
        g, ref = _build(stg, V, s, d, loops=loops, dgl=dgl)
        assert stg.view_arrays(g.view())["in_sched"][0].item() > 0        # hub rows exist
        for W in (4, 64, 96, 7):
            x = gen.uniform_pm1(9, W, V * W).reshape(V, W).astype(np.float64)
            for bwd in (False, True):
                e, _ = _agg_check(stg, g, ref, x, bwd)
                assert e <= TOL, (loops, dgl, W, bwd, e)


def test_aggregation_empty_and_single(stg):
    g = stg.stg_static_graph_create(5, np.zeros(0, np.int32), np.zeros(0, np.int32))
    x = torch.randn(5, 8, device="cuda")
    assert torch.count_nonzero(stg.stg_gcn_aggregate_fwd(g.view(), x)) == 0
    g1 = stg.stg_static_graph_create(1, [0], [0])
    y = stg.stg_gcn_aggregate_fwd(g1.view(), torch.full((1, 3), 2.0, device="cuda"))
    assert torch.equal(y, torch.full((1, 3), 2.0, device="cuda"))


def test_aggregation_strided_and_unaligned(stg):
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    g, ref = _build(stg, cfg.V, s, d, loops=True)
    W = 32
    big = to_gpu(gen.uniform_pm1(5, 5, cfg.V * 41).reshape(cfg.V, 41))
    x = big[:, 1:1 + W]                 # ld = 41, misaligned start -> scalar path
    out = torch.zeros(cfg.V, 37, device="cuda")
    stg._check(stg._lib.stg_gcn_aggregate_fwd(stg.ctypes.byref(g.view()), W, stg.ctypes.c_void_p(x.data_ptr()),
                                              41, stg.ctypes.c_void_p(out.data_ptr()), 37, stg._stream()))
    xr = big.cpu().numpy()[:, 1:1 + W].astype(np.float64)
    r = oracle.aggregate_fwd(ref, xr)
    e = cond_err(out[:, :W].cpu().numpy(), r, oracle.aggregate_scale(ref, xr))
    assert e <= TOL
    assert torch.count_nonzero(out[:, W:]) == 0


def test_aggregation_deterministic(stg):
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    g, _ = _build(stg, cfg.V, s, d, loops=True)
    x = to_gpu(gen.features(cfg, 1, width=96))
    y1 = stg.stg_gcn_aggregate_fwd(g.view(), x)
    y2 = stg.stg_gcn_aggregate_fwd(g.view(), x)
    assert torch.equal(y1, y2)
    b1 = stg.stg_gcn_aggregate_bwd(g.view(), x)
    b2 = stg.stg_gcn_aggregate_bwd(g.view(), x)
    assert torch.equal(b1, b2)


def test_aggregation_ex_scales_and_bias(stg):
    cfg = gen.CONFIGS["C6"]
    s, d = gen.static_edges(cfg)
    g, ref = _build(stg, cfg.V, s, d, loops=True)
    W = 12
    x = gen.features(cfg, 2, width=W).astype(np.float64)
    srow = gen.uniform_01(7, 1, cfg.V).astype(np.float64)
    scol = gen.uniform_01(7, 2, cfg.V).astype(np.float64)
    bias = gen.uniform_pm1(7, 3, W).astype(np.float64)
    y = stg.stg_gcn_aggregate_ex(g.view(), False, to_gpu(x), scale_row=to_gpu(srow), scale_col=to_gpu(scol),
                                 bias=to_gpu(bias)).cpu().numpy()
    r = oracle.aggregate(ref["in_rowptr"], ref["in_col"], srow, scol, x) + bias
    sc = oracle.aggregate(ref["in_rowptr"], ref["in_col"], srow, scol, np.abs(x)) + np.abs(bias)
    assert cond_err(y, r, sc) <= TOL


@pytest.mark.parametrize("strategy", [0, 1, 2])
@pytest.mark.parametrize("W", [4, 7, 16, 64, 68, 96, 128, 192, 256, 300])
def test_every_strategy_matches_oracle(stg, strategy, W):
    """Each work decomposition (row items, pipelined items, edge stream) meets the 1e-5 bound
    and is deterministic, incl. hub rows spanning many 64-edge chunks, odd widths (scalar
    path) and widths split into several column launches."""
    V = 30000
    rng = np.random.default_rng(7)
    s = np.concatenate([rng.integers(0, V, 20000), rng.integers(0, V, 90000), np.arange(V)])
    d = np.concatenate([np.full(20000, 29999), rng.integers(0, V, 90000), (np.arange(V) * 7) % V])
    g, ref = _build(stg, V, s, d, loops=True)
    x = gen.uniform_pm1(5, W, V * W).reshape(V, W).astype(np.float64)
    try:
        stg.stg_aggregate_set_strategy(strategy)
        for bwd in (False, True):
            e, y1 = _agg_check(stg, g, ref, x, bwd)
            assert e <= TOL, (strategy, W, bwd, e)
            _, y2 = _agg_check(stg, g, ref, x, bwd)
            assert torch.equal(y1, y2)               # deterministic
    finally:
        stg.stg_aggregate_set_strategy(2)


def test_device_partition_matches_host(stg):
    from paper_conf_ipps_cherianmcc24_b200 import parallel
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)
    rp = stg.view_arrays(g.view())["in_rowptr"]
    for world in (1, 2, 4, 8):
        assert stg.stg_partition_rows(cfg.V, rp, world) == parallel.row_blocks(rp.cpu().numpy(), world)
