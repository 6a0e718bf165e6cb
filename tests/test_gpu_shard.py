"""GPU parity of row-block sharding (north_star "partitioned ... by
destination-vertex row blocks").  Only one GPU is available, so the ranks of a
world are simulated one after another in this process: each rank's library
objects hold only the edges into its block, and

* its CSRs equal the oracle CSRs of that edge subset, its norms the whole-graph
  norms (bit-exact integers, fp32-rounded norms);
* its forward aggregation equals the whole-graph aggregation's rows of the block
  (bit-identical to the unsharded GPU run: same items, same order);
* the sum over ranks of its backward partial sums matches the oracle (1e-5,
  reading C19);
* a TGCN training sequence per rank gives the block's rows of H_t, and the sum
  over ranks of the losses / gradients (what the per-sequence all-reduce forms)
  matches the whole-graph oracle sequence.
The block bounds come from the host partitioner (paper_conf_ipps_cherianmcc24_b200.parallel).
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import cond_err, to_gpu

pytestmark = pytest.mark.gpu

TOL = 1e-5


def _blocks(ref, world):
    from paper_conf_ipps_cherianmcc24_b200 import parallel
    return parallel.row_blocks(ref["in_rowptr"], world)


def _local_ref(V, S, lo, hi, dgl=False):
    """Oracle of rank [lo, hi): the CSRs of the edges into the block, whole-graph norms."""
    keys = np.asarray(S)
    _, dst = oracle.unkey(keys)
    loc = oracle.csr(V, keys[(dst >= lo) & (dst < hi)], dgl)
    full = oracle.csr(V, keys, dgl)
    loc["norm_src"], loc["norm_dst"] = full["norm_src"], full["norm_dst"]
    return loc, full


def _check_local(stg, v, ref, lo, hi, tag):
    a = stg.view_arrays(v)
    R = hi - lo
    assert (v.row_begin, v.row_end, v.num_edges) == (lo, hi, ref["E"]), tag
    rp = np.asarray(ref["in_rowptr"])
    assert np.array_equal(a["in_rowptr"].cpu().numpy(), rp[lo:hi + 1] - rp[lo]), tag
    for k in ("in_col", "out_rowptr", "out_col", "out_deg", "out_ids"):
        assert np.array_equal(a[k].cpu().numpy(), np.asarray(ref[k])), (tag, k)
    ids = np.asarray(ref["in_ids"])
    want = ids[(ids >= lo) & (ids < hi)]
    assert np.array_equal(a["in_ids"].cpu().numpy()[:R], want), (tag, "in_ids")
    if "out_eid" in a:
        assert np.array_equal(a["out_eid"].cpu().numpy(), np.asarray(ref["out_eid"])), (tag, "out_eid")
    for k in ("norm_src", "norm_dst"):
        np.testing.assert_allclose(a[k].cpu().numpy().astype(np.float64), ref[k], rtol=2.5e-7, atol=0,
                                   err_msg=str((tag, k)))


@pytest.mark.parametrize("name,world", [("C2", 3), ("C6", 2), ("C1", 4)])
@pytest.mark.parametrize("dgl", [False, True])
def test_static_sharded_csr_and_aggregation(stg, name, world, dgl):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    V = cfg.V
    flags = stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS | (stg.STG_NORM_DGL_BOTH if dgl else 0)
    S = oracle.edge_set(V, s, d, self_loops=True)
    full_ref = oracle.csr(V, S, dgl)
    gfull = stg.stg_static_graph_create(V, s, d, flags)
    b = _blocks(full_ref, world)
    x = gen.features(cfg, 0, width=96).astype(np.float64)
    gy = gen.features(cfg, 1, width=96).astype(np.float64)
    yfull = stg.stg_gcn_aggregate_fwd(gfull.view(), to_gpu(x)).cpu().numpy()
    gx_sum = np.zeros((V, 96))
    for k in range(world):
        lo, hi = b[k], b[k + 1]
        g = stg.stg_static_graph_create(V, s, d, flags, dist=(k, world, lo, hi))
        loc, _ = _local_ref(V, S, lo, hi, dgl)
        _check_local(stg, g.view(), loc, lo, hi, (name, k))
        y = stg.stg_gcn_aggregate_fwd(g.view(), to_gpu(x)).cpu().numpy()
        assert y.shape == (hi - lo, 96)
        assert np.array_equal(y, yfull[lo:hi]), (name, k, "fwd rows differ from the unsharded run")
        gx = stg.stg_gcn_aggregate_bwd(g.view(), to_gpu(gy[lo:hi])).cpu().numpy()
        gx_sum += gx
    r = oracle.aggregate_bwd(full_ref, gy)
    sc = oracle.aggregate_scale(full_ref, gy, bwd=True)
    assert cond_err(gx_sum, r, sc) <= TOL


def test_sharded_rejects_bad_block(stg):
    with pytest.raises(stg.StgError) as e:
        stg.stg_static_graph_create(10, [0, 1], [1, 2], 0, dist=(0, 2, 6, 4))
    assert e.value.status == 1


@pytest.mark.parametrize("world", [2, 3])
def test_dtdg_sharded_snapshots(stg, world):
    """Get-Graph forward over all t, then Get-Backward-Graph back down, per rank."""
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    V = dd.V
    sets = list(oracle.snapshot_sets_fold(dd, self_loops=True))
    b = _blocks(oracle.csr(V, sets[0]), world)
    flags = stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS
    for k in range(world):
        lo, hi = b[k], b[k + 1]
        g = stg.stg_dtdg_create(V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off,
                                dd.del_src, dd.del_dst, flags, dist=(k, world, lo, hi))
        order = list(range(dd.T)) + list(range(dd.T - 2, -1, -1))
        for i, t in enumerate(order):
            v = stg.stg_dtdg_get_snapshot(g, t) if i < dd.T else stg.stg_dtdg_get_backward_snapshot(g, t)
            loc, _ = _local_ref(V, sets[t], lo, hi)
            assert g.num_edges(t) == loc["E"]
            _check_local(stg, v, loc, lo, hi, (k, t, i >= dd.T))


def test_tgcn_sequence_sharded_sums_to_whole_graph(stg):
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    V, F, H, S, world = cfg.V, cfg.F, cfg.H, 4, 3
    flags = stg.STG_SELF_LOOPS
    p = gen.tgcn_params(F, H, 1)
    pg = {k: torch.from_numpy(v).cuda() for k, v in p.items()}
    Xs = [gen.features(cfg, t) for t in range(S)]
    Ys = [gen.labels(cfg, t) for t in range(S)]
    Xg = [torch.from_numpy(x).cuda() for x in Xs]

    def run(dist, lo, hi):
        R = hi - lo
        g = stg.stg_dtdg_create(V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off,
                                dd.del_src, dd.del_dst, flags, dist=dist)
        grads = {"W": torch.zeros(F, 3 * H, device="cuda"), "b": torch.zeros(3 * H, device="cuda"),
                 "L": torch.zeros(3, 2 * H, H, device="cuda"), "l": torch.zeros(3, H, device="cuda")}
        dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
        Hs = torch.empty(S, R, H, device="cuda")
        Gw = torch.empty(2, R, H, device="cuda")
        st = stg.stg_state_stack_create(S * max(R, 1) * 3 * H * 4 + (1 << 20))
        stg.stg_tgcn_train_sequence(g, 0, S, pg, pg["w_o"], pg["b_o"], Xg,
                                    [torch.from_numpy(y[lo:hi].copy()).cuda() for y in Ys],
                                    torch.zeros(R, H, device="cuda"), Hs, Gw, grads, dw, db, loss, st)
        torch.cuda.synchronize()
        out = {k: v.cpu().numpy().astype(np.float64) for k, v in grads.items()}
        out.update(w_o=dw.cpu().numpy().astype(np.float64), b_o=db.cpu().numpy().astype(np.float64))
        return loss.item(), out, Hs.cpu().numpy()

    l_full, g_full, H_full = run(None, 0, V)
    sets = list(oracle.snapshot_sets_fold(dd, self_loops=True))
    b = _blocks(oracle.csr(V, sets[0]), world)
    l_sum, g_sum = 0.0, None
    for k in range(world):
        lo, hi = b[k], b[k + 1]
        lk, gk, Hk = run((k, world, lo, hi), lo, hi)
        np.testing.assert_allclose(Hk, H_full[:, lo:hi], rtol=0, atol=1e-6, err_msg="rank %d H_t rows" % k)
        l_sum += lk
        g_sum = gk if g_sum is None else {n: g_sum[n] + gk[n] for n in g_sum}
    snaps = [oracle.csr(V, sets[t]) for t in range(S)]
    rl, rg, _ = oracle.train_sequence(snaps, snaps, p, Xs, Ys, np.zeros((V, H)))
    assert abs(l_sum - rl) <= 1e-5 * abs(rl), (l_sum, rl)
    assert abs(l_full - rl) <= 1e-5 * abs(rl), (l_full, rl)
    tol = max(1e-4, 1e-6 * np.sqrt(V * S))          # tests/test_gpu_tgcn.py g_tol
    for n in ("W", "b", "L", "l", "w_o", "b_o"):
        ref = np.asarray(rg[n], np.float64)
        err = np.max(np.abs(g_sum[n] - ref)) / max(np.max(np.abs(ref)), 1e-300)
        assert err <= tol, (n, err)
