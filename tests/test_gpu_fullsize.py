r"""Parity at BASELINE.json's full size (configs[4], C5: 2^20 vertices, ~9 M edges per
snapshot, F = 64, H = 32) in the configuration bench.py times (STG_SELF_LOOPS |
STG_EDGE_IDS, default aggregation strategy, W = 3H = 96, the pipelined Algorithm-1
driver):

* snapshots: ALL T = 41 Get-Graph views of the forward walk 0 -> 40 equal, array for
  array and bit for bit, the oracle CSRs of the folded deltas S_t = (S_{t-1} \ D_t) ∪ A_t
  (P:L208), and all 41 Get-Backward-Graph views of the walk 40 -> 0 equal the oracle
  CSRs of the event-window definition — whole snapshots, not samples;
* aggregation: EVERY row of both directions against the fp64 oracle over the whole
  snapshot, reading C19 tolerance 1e-5 (plus the plain relative error for x >= 0);
* training: one two-timestep Algorithm-1 sequence against the fp64 oracle sequence
  (loss, every H_t entry, every gradient; element-wise condition-scaled).
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import assert_graph_equal, check_sequence, cond_err, elementwise_err, parity_log, sequence_scales, \
    TAU_TGCN, to_gpu

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


@pytest.mark.slow
def test_c5_all_snapshots_both_walks(stg, c5):
    """Every snapshot of the bench's DTDG: the forward head walks t = 0..T-1 (one
    delta step each, as Algorithm 1 does), then the backward cursor walks T-1..0."""
    cfg, d, g, _ = c5
    for t, S in enumerate(oracle.snapshot_sets_fold(d, self_loops=True)):
        v = stg.stg_dtdg_get_snapshot(g, t)
        r = oracle.csr(d.V, S)
        assert v.num_edges == r["E"] == g.num_edges(t)
        assert_graph_equal(stg.view_arrays(v), r, tag=("C5", t, "fwd"))
    for t in range(d.T - 1, -1, -1):
        v = stg.stg_dtdg_get_backward_snapshot(g, t)
        r = oracle.csr(d.V, oracle.snapshot_set_window(d, t, self_loops=True))
        assert_graph_equal(stg.view_arrays(v), r, tag=("C5", t, "bwd"))


@pytest.mark.slow
@pytest.mark.parametrize("bwd", [False, True])
@pytest.mark.parametrize("nonneg,W", [(False, 96), (True, 96), (False, 64), (False, 32), (False, 16)])
def test_c5_aggregation_every_row(stg, c5, bwd, nonneg, W):
    """All 2^20 output rows of the aggregation at t = 2 (the hubs carry up to 72 K
    in-edges) against the fp64 oracle: C19 condition-scaled error <= 1e-5, and for
    x >= 0 also the plain relative error <= 1e-5.  W = 3H is the TGCN's width; 2H, H
    are the original T-GCN's (NEXT-2) gate and candidate widths, 16 the narrowest
    edge-stream launch."""
    cfg, d, g, ref = c5
    r = ref(2)
    v = stg.stg_dtdg_get_snapshot(g, 2)
    x = (gen.uniform_01 if nonneg else gen.uniform_pm1)(11, 61, cfg.V * W).reshape(cfg.V, W)
    xg = to_gpu(x)
    y = (stg.stg_gcn_aggregate_bwd(v, xg) if bwd else stg.stg_gcn_aggregate_fwd(v, xg)).cpu().numpy()
    x64 = x.astype(np.float64)
    want = (oracle.aggregate_bwd if bwd else oracle.aggregate_fwd)(r, x64)
    scale = oracle.aggregate_scale(r, x64, bwd=bwd)
    rp = r["out_rowptr"] if bwd else r["in_rowptr"]
    assert int(np.diff(np.asarray(rp, np.int64)).max()) > 10_000            # hub rows present
    e = cond_err(y, want, scale)
    parity_log(("c5_agg_every_row", "bwd" if bwd else "fwd", "nonneg" if nonneg else "pm1", W), cond=e)
    assert e <= 1e-5
    if nonneg:
        nz = want > 0
        assert np.all(y[~nz] == 0)
        assert np.max(np.abs(y[nz] - want[nz]) / want[nz]) <= 1e-5


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
    sc = sequence_scales(snaps, snaps, p, Xs, Ys, np.zeros((V, H)))
    eH = elementwise_err(Hs[-1].cpu().numpy(), rH, sc["H"][-1])
    el = abs(loss.item() - rl) / sc["loss"]
    parity_log("c5_train_seq", H=eH, loss=el)
    assert eH <= TAU_TGCN and el <= TAU_TGCN, (eH, el)
    gd = {k: t.cpu().numpy().astype(np.float64) for k, t in grads.items()}
    gd.update(w_o=dw.cpu().numpy().astype(np.float64), b_o=db.cpu().numpy().astype(np.float64))
    check_sequence("c5_train_seq", gd, rg, sc, normwise=max(1e-4, 1e-6 * np.sqrt(V * S)))
