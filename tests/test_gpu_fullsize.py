"""Parity at BASELINE.json's full size (configs[4], C5: 2^20 vertices, ~9 M edges per
snapshot, F = 64, H = 32) in the configuration bench.py times (STG_SELF_LOOPS |
STG_EDGE_IDS, default aggregation strategy, W = 3H = 96, the pipelined Algorithm-1
driver):

* snapshots: the Get-Graph / Get-Backward-Graph views equal, array for array and bit
  for bit, the oracle CSRs of the event-window definition of S_t — the whole
  snapshot, not a sample;
* aggregation: sampled rows (the 64 largest hubs of each direction plus random rows)
  against the oracle one row at a time, reading C19 tolerance 1e-5;
* training: one two-timestep Algorithm-1 sequence against the fp64 oracle sequence
  (loss, every H_t entry, every gradient; DESIGN.md §7 tolerances).
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import assert_graph_equal, cond_err, to_gpu

pytestmark = pytest.mark.gpu

FLAGS_NAME = "C5"


@pytest.fixture(scope="module")
def c5(stg):
    cfg = gen.CONFIGS[FLAGS_NAME]
    d = gen.dtdg(cfg)
    g = stg.stg_dtdg_create(d.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src,
                            d.del_dst, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    cache = {}

    def ref(t):
        if t not in cache:
            cache[t] = oracle.csr(d.V, oracle.snapshot_set_window(d, t, self_loops=True))
        return cache[t]
    return cfg, d, g, ref


def test_c5_snapshots_bit_exact(stg, c5):
    cfg, d, g, ref = c5
    for t in range(0, 4):                                   # forward head walks 0 -> 3
        v = stg.stg_dtdg_get_snapshot(g, t)
    assert v.num_edges == ref(3)["E"]
    assert_graph_equal(stg.view_arrays(v), ref(3), tag=("C5", 3, "fwd"))
    v = stg.stg_dtdg_get_backward_snapshot(g, 2)            # backward cursor one step down
    assert_graph_equal(stg.view_arrays(v), ref(2), tag=("C5", 2, "bwd"))


def _sample_rows(rowptr, n_rand, seed):
    deg = np.diff(rowptr)
    hubs = np.argsort(-deg, kind="stable")[:64]
    rnd = gen.permutation(seed, 60, rowptr.size - 1)[:n_rand]
    return np.unique(np.concatenate([hubs, rnd])).astype(np.int64)


def _sub_csr(rowptr, col, rows):
    starts, ends = rowptr[rows], rowptr[rows + 1]
    sub_ptr = np.concatenate([[0], np.cumsum(ends - starts)]).astype(np.int32)
    sub_col = np.concatenate([col[s:e] for s, e in zip(starts, ends)]).astype(np.int32)
    return sub_ptr, sub_col


@pytest.mark.parametrize("bwd", [False, True])
def test_c5_aggregation_sampled_rows(stg, c5, bwd):
    cfg, d, g, ref = c5
    r = ref(2)
    v = stg.stg_dtdg_get_snapshot(g, 2)
    W = 3 * cfg.H
    x = gen.uniform_pm1(11, 61, cfg.V * W).reshape(cfg.V, W)
    xg = to_gpu(x)
    y = (stg.stg_gcn_aggregate_bwd(v, xg) if bwd else stg.stg_gcn_aggregate_fwd(v, xg)).cpu().numpy()
    rp, col = (r["out_rowptr"], r["out_col"]) if bwd else (r["in_rowptr"], r["in_col"])
    nrow, ncol = (r["norm_src"], r["norm_dst"]) if bwd else (r["norm_dst"], r["norm_src"])
    rows = _sample_rows(np.asarray(rp, np.int64), 3000, 3 if bwd else 4)
    sp, sc = _sub_csr(np.asarray(rp, np.int64), np.asarray(col), rows)
    x64 = x.astype(np.float64)
    want = oracle.aggregate(sp, sc, np.asarray(nrow)[rows], ncol, x64)
    scale = oracle.aggregate(sp, sc, np.asarray(nrow)[rows], ncol, np.abs(x64))
    assert int(np.diff(sp).max()) > 10_000            # the hub rows are in the sample
    assert cond_err(y[rows], want, scale) <= 1e-5


def test_c5_training_sequence(stg, c5):
    cfg, d, g, ref = c5
    V, F, H, S = cfg.V, cfg.F, cfg.H, 2
    p = gen.tgcn_params(F, H, cfg.seed)
    pg = {k: torch.from_numpy(v).cuda() for k, v in p.items()}
    Xs = [gen.features(cfg, t) for t in range(S)]
    Ys = [gen.labels(cfg, t) for t in range(S)]
    grads = {"W": torch.zeros(F, 3 * H, device="cuda"), "b": torch.zeros(3 * H, device="cuda"),
             "L": torch.zeros(3, 2 * H, H, device="cuda"), "l": torch.zeros(3, H, device="cuda")}
    dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
    Hs = torch.empty(S, V, H, device="cuda")
    st = stg.stg_state_stack_create(S * V * 3 * H * 4 + (64 << 20))
    stg.stg_tgcn_train_sequence(g, 0, S, pg, pg["w_o"], pg["b_o"], [torch.from_numpy(x).cuda() for x in Xs],
                                [torch.from_numpy(y).cuda() for y in Ys], torch.zeros(V, H, device="cuda"), Hs,
                                torch.empty(2, V, H, device="cuda"), grads, dw, db, loss, st)
    torch.cuda.synchronize()
    snaps = [ref(t) for t in range(S)]
    rl, rg, rH = oracle.train_sequence(snaps, snaps, p, Xs, Ys, np.zeros((V, H)))
    assert abs(loss.item() - rl) <= 1e-5 * abs(rl), (loss.item(), rl)
    assert np.max(np.abs(Hs[-1].cpu().numpy() - rH)) <= 2e-5
    gd = {k: t.cpu().numpy().astype(np.float64) for k, t in grads.items()}
    gd.update(w_o=dw.cpu().numpy().astype(np.float64), b_o=db.cpu().numpy().astype(np.float64))
    tol = max(1e-4, 1e-6 * np.sqrt(V * S))
    for n in ("W", "b", "L", "l", "w_o", "b_o"):
        refn = np.asarray(rg[n], np.float64)
        err = np.max(np.abs(gd[n] - refn)) / max(np.max(np.abs(refn)), 1e-300)
        assert err <= tol, (n, err)
