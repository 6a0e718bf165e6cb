"""GPU parity: TGCN step forward/backward and Algorithm 1 sequences vs the oracle.

Tolerances: every output is compared ELEMENT-WISE against a
condition scale s_i — the same computation over |·| (helpers.tgcn_fwd_scale /
tgcn_bwd_scales / sequence_scales, the generalisation of reading C19 to the GRU
chain and the Σ-over-rows reductions): |r_gpu − r_ref| <= TAU_TGCN · s_i for H',
dH_{t-1}, the loss and every parameter gradient.  The earlier normwise bounds
(H' absolute 2e-5; gradients max|Δ| <= g_tol(n)·max|ref|, n = rows reduced) are
kept as a second check.
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import TAU_TGCN, check_sequence, elementwise_err, parity_log, sequence_scales, \
    tgcn_bwd_scales, tgcn_fwd_scale, to_gpu

pytestmark = pytest.mark.gpu

H_TOL = 2e-5
G_TOL = 1e-4


def g_tol(n_rows: int) -> float:
    return max(1e-4, 1e-6 * float(np.sqrt(n_rows)))


def _params(F, H, seed):
    p = gen.tgcn_params(F, H, seed)
    return p, {k: to_gpu(v) for k, v in p.items()}


def _zero_grads(F, H):
    return {"W": torch.zeros(F, 3 * H, device="cuda"), "b": torch.zeros(3 * H, device="cuda"),
            "L": torch.zeros(3, 2 * H, H, device="cuda"), "l": torch.zeros(3, H, device="cuda")}


def _normwise(a, ref):
    a = np.asarray(a, np.float64)
    ref = np.asarray(ref, np.float64)
    den = np.max(np.abs(ref))
    return float(np.max(np.abs(a - ref)) / (den if den > 0 else 1.0))


def _graph(stg, name):
    cfg = gen.CONFIGS[name]
    if cfg.kind == "static":
        s, d = gen.static_edges(cfg)
        return cfg, stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS), \
            oracle.static_graph(cfg.V, s, d, self_loops=True)
    dd = gen.dtdg(cfg)
    S0 = next(oracle.snapshot_sets_fold(dd, self_loops=True))
    return cfg, stg.stg_static_graph_create(cfg.V, oracle.unkey(S0)[0], oracle.unkey(S0)[1], 0), oracle.csr(cfg.V, S0)


@pytest.mark.parametrize("name,H,F", [("C1", 16, None), ("C2", 32, None), ("C6", 16, None), ("C5s", 32, None),
                                      ("C2", 64, None), ("C1", 5, None), ("C2", 32, 12), ("C2", 32, 96),
                                      ("C2", 16, 128), ("C5s", 32, 40)])
def test_tgcn_step_parity(stg, name, H, F):
    """F overrides cover every X·W path: pipelined (F <= 64, incl. K padding) and
    one-tile-at-a-time (64 < F <= 128)."""
    cfg, g, ref = _graph(stg, name)
    V = cfg.V
    if F is None:
        F = cfg.F
        X = gen.features(cfg, 5)
    else:
        X = gen.uniform_pm1(9, F, V * F).reshape(V, F)
    p, pg = _params(F, H, 11)
    Hp = gen.uniform_pm1(3, 3, V * H).reshape(V, H)
    Xg, Hg = to_gpu(X), to_gpu(Hp)
    stack = stg.stg_state_stack_create(64 << 20)
    Hn = stg.stg_tgcn_step(g.view(), pg, Xg, Hg, stack=stack)
    f = oracle.tgcn_fwd(ref, p, X, Hp)
    err = np.max(np.abs(Hn.cpu().numpy() - f["Hn"]))
    assert err <= H_TOL, err
    fs = tgcn_fwd_scale(ref, p, X, Hp, np.abs(Hp), f)
    eH = elementwise_err(Hn.cpu().numpy(), f["Hn"], fs["Hn"])
    # backward with a random upstream gradient (an exact input: s(G) = |G|)
    G = gen.uniform_pm1(4, 4, V * H).reshape(V, H)
    grads = _zero_grads(F, H)
    dHp = stg.stg_tgcn_step_backward(g.view(), pg, Xg, to_gpu(G), grads, stack)
    assert stack.depth == 0
    rg = oracle.zero_grads(F, H)
    rdH = oracle.tgcn_bwd(ref, p, X, Hp, f, G, rg)
    sc = {}
    s_dH = tgcn_bwd_scales(ref, p, X, Hp, np.abs(Hp), f, fs, G, np.abs(G), sc)
    edH = elementwise_err(dHp.cpu().numpy(), rdH, s_dH)
    parity_log(("step", name, H, F), H=eH, dH=edH)
    assert eH <= TAU_TGCN and edH <= TAU_TGCN, (eH, edH)
    assert _normwise(dHp.cpu().numpy(), rdH) <= G_TOL
    check_sequence(("step", name, H, F), {k: grads[k].cpu().numpy() for k in ("W", "b", "L", "l")}, rg, sc,
                   normwise=g_tol(V))


def test_tgcn_inference_and_stack_errors(stg):
    cfg, g, ref = _graph(stg, "C1")
    p, pg = _params(cfg.F, cfg.H, 1)
    X = to_gpu(gen.features(cfg, 0))
    H0 = torch.zeros(cfg.V, cfg.H, device="cuda")
    Hn = stg.stg_tgcn_step(g.view(), pg, X, H0)          # no stack: inference
    f = oracle.tgcn_fwd(ref, p, gen.features(cfg, 0), np.zeros((cfg.V, cfg.H)))
    assert np.max(np.abs(Hn.cpu().numpy() - f["Hn"])) <= H_TOL
    stack = stg.stg_state_stack_create(1 << 20)
    with pytest.raises(stg.StgError) as e:
        stg.stg_tgcn_step_backward(g.view(), pg, X, H0, _zero_grads(cfg.F, cfg.H), stack)
    assert e.value.status == 6
    tiny = stg.stg_state_stack_create(16)
    with pytest.raises(stg.StgError) as e:
        stg.stg_tgcn_step(g.view(), pg, X, H0, stack=tiny)
    assert e.value.status == 3


def test_zero_parameters_closed_form(stg):
    cfg, g, _ = _graph(stg, "C2")
    pg = {k: torch.zeros_like(v) for k, v in _params(cfg.F, cfg.H, 0)[1].items()}
    Hp = to_gpu(gen.uniform_pm1(1, 1, cfg.V * cfg.H).reshape(cfg.V, cfg.H))
    Hn = stg.stg_tgcn_step(g.view(), pg, to_gpu(gen.features(cfg, 0)), Hp)
    assert torch.equal(Hn, 0.5 * Hp)


def _check_seq(tag, graphs, p, Xs, Ys, H0, loss, grads, dw, db, Hseq, rl, rg, rH, n_rows):
    """Element-wise parity of one Algorithm-1 sequence (loss, every H_t, every
    gradient) against the oracle, plus the normwise bounds."""
    sc = sequence_scales(graphs, graphs, p, Xs, Ys, H0)
    Hs = Hseq.cpu().numpy()
    eH = max(elementwise_err(Hs[i], h, s) for i, (h, s) in enumerate(zip(_oracle_states(graphs, p, Xs, H0), sc["H"])))
    el = abs(loss - rl) / sc["loss"]
    parity_log(tag, H_steps=eH, loss=el)
    assert eH <= TAU_TGCN, (tag, "H", eH)
    assert el <= TAU_TGCN and abs(loss - rl) <= 1e-5 * abs(rl), (tag, loss, rl)
    assert np.max(np.abs(Hs[-1] - rH)) <= H_TOL
    gpu = {k: grads[k].cpu().numpy() for k in ("W", "b", "L", "l")}
    gpu.update(w_o=dw.cpu().numpy(), b_o=db.cpu().numpy())
    check_sequence(tag, gpu, rg, sc, normwise=g_tol(n_rows))


def _oracle_states(graphs, p, Xs, H0):
    out, Hc = [], np.asarray(H0, np.float64)
    for g, X in zip(graphs, Xs):
        Hc = oracle.tgcn_fwd(g, p, X, Hc)["Hn"]
        out.append(Hc)
    return out


def _run_sequence(stg, source, cfg, pg, Xs, Ys, H0, S, t0):
    V, H, F = cfg.V, pg["L"].shape[2], cfg.F
    grads = _zero_grads(F, H)
    dw = torch.zeros(H, device="cuda")
    db = torch.zeros(1, device="cuda")
    loss = torch.zeros(1, device="cuda")
    Hseq = torch.empty(S, V, H, device="cuda")
    Gw = torch.empty(2, V, H, device="cuda")
    stack = stg.stg_state_stack_create(S * V * 3 * H * 4 + (1 << 20))
    stg.stg_tgcn_train_sequence(source, t0, S, pg, pg["w_o"], pg["b_o"], Xs, Ys, H0, Hseq, Gw, grads, dw, db,
                                loss, stack)
    assert stack.depth == 0
    return loss.item(), grads, dw, db, Hseq


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_train_sequence_static(stg, name):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)
    ref = oracle.static_graph(cfg.V, s, d, self_loops=True)
    S, t0 = 8, 16
    p, pg = _params(cfg.F, cfg.H, 2)
    Xs = [gen.features(cfg, t0 + i) for i in range(S)]
    Ys = [gen.labels(cfg, t0 + i) for i in range(S)]
    H0 = gen.uniform_pm1(8, 8, cfg.V * cfg.H).reshape(cfg.V, cfg.H)
    loss, grads, dw, db, Hseq = _run_sequence(stg, g, cfg, pg, [to_gpu(x) for x in Xs], [to_gpu(y) for y in Ys],
                                              to_gpu(H0), S, t0)
    rl, rg, rH = oracle.train_sequence([ref] * S, [ref] * S, p, Xs, Ys, H0)
    _check_seq(("seq", name), [ref] * S, p, Xs, Ys, H0, loss, grads, dw, db, Hseq, rl, rg, rH, cfg.V * S)


@pytest.mark.parametrize("name", ["C4", "C5s"])
def test_train_sequence_dtdg(stg, name):
    cfg = gen.CONFIGS[name]
    d = gen.dtdg(cfg)
    g = stg.stg_dtdg_create(d.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src,
                            d.del_dst, stg.STG_SELF_LOOPS)
    snaps = [oracle.csr(d.V, S) for S in oracle.snapshot_sets_fold(d, self_loops=True)]
    H = cfg.H
    p, pg = _params(cfg.F, H, 3)
    H0 = np.zeros((cfg.V, H))
    Hc = to_gpu(H0)
    S = 4
    for t0 in (0, S, 2 * S):             # three consecutive sequences (cached head reuse)
        Xs = [gen.features(cfg, t0 + i) for i in range(S)]
        Ys = [gen.labels(cfg, t0 + i) for i in range(S)]
        loss, grads, dw, db, Hseq = _run_sequence(stg, g, cfg, pg, [to_gpu(x) for x in Xs],
                                                  [to_gpu(y) for y in Ys], Hc, S, t0)
        rl, rg, rH = oracle.train_sequence(snaps[t0:t0 + S], snaps[t0:t0 + S], p, Xs, Ys, H0)
        _check_seq(("seq", name, t0), snaps[t0:t0 + S], p, Xs, Ys, H0, loss, grads, dw, db, Hseq, rl, rg, rH,
                   cfg.V * S)
        H0 = rH
        Hc = Hseq[-1].clone()


def test_sgd_update(stg):
    p = torch.arange(10, dtype=torch.float32, device="cuda")
    g = torch.ones(10, device="cuda")
    stg.stg_sgd_update(p, g, 0.5)
    assert torch.equal(p, torch.arange(10, dtype=torch.float32, device="cuda") - 0.5)
    assert torch.count_nonzero(g) == 0


def _run_batched(stg, g, cfg, pg, Xs, Ys, H0, S):
    V, H, F = cfg.V, pg["L"].shape[2], cfg.F
    grads = _zero_grads(F, H)
    dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
    Hseq = torch.empty(S, V, H, device="cuda")
    stack = stg.stg_state_stack_create(1 << 20)
    stg.stg_tgcn_train_sequence_batched(g, S, pg, pg["w_o"], pg["b_o"], Xs, Ys, H0, Hseq, grads, dw, db, loss, stack)
    torch.cuda.synchronize()
    return loss.item(), grads, dw, db, Hseq


@pytest.mark.parametrize("name,S", [("C1", 16), ("C2", 8), ("C3", 5), ("C6", 3), ("C2", 1)])
def test_train_sequence_batched_static(stg, name, S):
    """NEXT-1 (sequence-batched schedule) against the fp64 oracle's Algorithm 1 and
    against the per-timestamp GPU driver: same losses, states and gradients."""
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)
    ref = oracle.static_graph(cfg.V, s, d, self_loops=True)
    p, pg = _params(cfg.F, cfg.H, 3)
    Xs = [gen.features(cfg, 40 + i) for i in range(S)]
    Ys = [gen.labels(cfg, 40 + i) for i in range(S)]
    H0 = gen.uniform_pm1(9, 9, cfg.V * cfg.H).reshape(cfg.V, cfg.H)
    Xg, Yg = [to_gpu(x) for x in Xs], [to_gpu(y) for y in Ys]
    loss, grads, dw, db, Hseq = _run_batched(stg, g, cfg, pg, Xg, Yg, to_gpu(H0), S)
    rl, rg, rH = oracle.train_sequence([ref] * S, [ref] * S, p, Xs, Ys, H0)
    _check_seq(("batched", name, S), [ref] * S, p, Xs, Ys, H0, loss, grads, dw, db, Hseq, rl, rg, rH, cfg.V * S)
    # the per-timestamp driver on the same inputs: identical H_t (same per-row arithmetic)
    l2, g2, dw2, db2, H2 = _run_sequence(stg, g, cfg, pg, Xg, Yg, to_gpu(H0), S, 0)
    assert np.max(np.abs(Hseq.cpu().numpy() - H2.cpu().numpy())) <= 1e-6
    assert abs(loss - l2) <= 1e-6 * abs(l2)


def test_train_sequence_batched_rejects(stg):
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)
    p, pg = _params(cfg.F, cfg.H, 3)
    X = [to_gpu(gen.features(cfg, 0))] * 65
    Y = [to_gpu(gen.labels(cfg, 0))] * 65
    with pytest.raises(stg.StgError) as e:
        _run_batched(stg, g, cfg, pg, X, Y, torch.zeros(cfg.V, cfg.H, device="cuda"), 65)
    assert e.value.status == 1


@pytest.mark.parametrize("V,H,S", [(100, 16, 16), (128, 32, 4), (47, 32, 9)])
def test_train_sequence_batched_small_graph_row_blocks(stg, V, H, S):
    """The one-CTA-per-row-block SIMT recurrence of small graphs (V <= 128; several
    CTAs when V·H exceeds one block) against the fp64 oracle sequence."""
    from types import SimpleNamespace
    F = 8
    s, d = gen.random_edges(V, V, 4 * V, loops=False)
    cfg = SimpleNamespace(V=V, F=F, H=H)
    g = stg.stg_static_graph_create(V, s, d, stg.STG_SELF_LOOPS)
    ref = oracle.static_graph(V, s, d, self_loops=True)
    p, pg = _params(F, H, 5)
    Xs = [gen.uniform_pm1(60 + i, 61, V * F).reshape(V, F) for i in range(S)]
    Ys = [gen.uniform_pm1(70 + i, 71, V) for i in range(S)]
    H0 = gen.uniform_pm1(8, 8, V * H).reshape(V, H)
    loss, grads, dw, db, Hseq = _run_batched(stg, g, cfg, pg, [to_gpu(x) for x in Xs], [to_gpu(y) for y in Ys],
                                             to_gpu(H0), S)
    rl, rg, rH = oracle.train_sequence([ref] * S, [ref] * S, p, Xs, Ys, H0)
    _check_seq(("small", V, H, S), [ref] * S, p, Xs, Ys, H0, loss, grads, dw, db, Hseq, rl, rg, rH, V * S)


def test_mse_head_hand_derived_golden(stg):
    """The GPU surrogate head against the hand-derived values of
    tests/golden/mse_head_hand.json (loss, dH, dw_o, db_o) — all exact in fp32."""
    import json
    import os
    spec = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "mse_head_hand.json")))
    for c in spec["cases"]:
        # the GPU head needs H % 4 == 0: pad with zero hidden units (ReLU(0) = 0 and w_o = 0
        # there, so the loss and every other entry are unchanged; their gradients are 0)
        H0 = len(c["w_o"])
        H = (H0 + 3) // 4 * 4
        pad = lambda a: np.pad(np.array(a, np.float64), [(0, 0)] * (np.ndim(a) - 1) + [(0, H - H0)])
        c = dict(c, H=pad(c["H"]), w_o=pad(c["w_o"]), dH=pad(c["dH"]), dw_o=pad(c["dw_o"]))
        Hn = to_gpu(c["H"])
        V = Hn.shape[0]
        loss = torch.zeros(1, device="cuda")
        dH = torch.full((V, H), 7.0, device="cuda")
        dw = torch.zeros(H, device="cuda")
        db = torch.zeros(1, device="cuda")
        stg.stg_mse_head(Hn, to_gpu(np.array(c["y"])), to_gpu(np.array(c["w_o"])), to_gpu(np.array([c["b_o"]])),
                         loss_accum=loss, dH=dH, accumulate=False, dw_o=dw, db_o=db)
        assert loss.item() == pytest.approx(c["loss"], rel=1e-6), c["name"]
        np.testing.assert_allclose(dH.cpu().numpy(), np.array(c["dH"]), rtol=1e-6, atol=0, err_msg=c["name"])
        np.testing.assert_allclose(dw.cpu().numpy(), np.array(c["dw_o"]), rtol=1e-6, atol=0, err_msg=c["name"])
        assert db.item() == pytest.approx(c["db_o"], rel=1e-6), c["name"]


@pytest.fixture
def agg_first(stg):
    """Run a test under the aggregate-first convolution order (NEXT-1), restoring the default."""
    stg.stg_set_conv_order(1)
    yield
    stg.stg_set_conv_order(0)


@pytest.mark.parametrize("name,H", [("C2", 32), ("C5s", 32), ("C1", 16)])
def test_tgcn_step_parity_aggregate_first(stg, agg_first, name, H):
    """(ÂX)W + b (NEXT-1) is the same model as the oracle's Â(XW) + b: the step and its
    gradients match the fp64 oracle element-wise (condition scales of DESIGN.md §7)."""
    cfg, g, ref = _graph(stg, name)
    V, F = cfg.V, cfg.F
    X = gen.features(cfg, 5)
    p, pg = _params(F, H, 11)
    Hp = gen.uniform_pm1(3, 3, V * H).reshape(V, H)
    Xg, Hg = to_gpu(X), to_gpu(Hp)       # (the state stack keeps H_{t-1} by reference)
    stack = stg.stg_state_stack_create(64 << 20)
    Hn = stg.stg_tgcn_step(g.view(), pg, Xg, Hg, stack=stack)
    f = oracle.tgcn_fwd(ref, p, X, Hp)
    fs = tgcn_fwd_scale(ref, p, X, Hp, np.abs(Hp), f)
    eH = elementwise_err(Hn.cpu().numpy(), f["Hn"], fs["Hn"])
    G = gen.uniform_pm1(4, 4, V * H).reshape(V, H)
    grads = _zero_grads(F, H)
    dHp = stg.stg_tgcn_step_backward(g.view(), pg, Xg, to_gpu(G), grads, stack)
    rg = oracle.zero_grads(F, H)
    rdH = oracle.tgcn_bwd(ref, p, X, Hp, f, G, rg)
    sc = {}
    s_dH = tgcn_bwd_scales(ref, p, X, Hp, np.abs(Hp), f, fs, G, np.abs(G), sc)
    edH = elementwise_err(dHp.cpu().numpy(), rdH, s_dH)
    parity_log(("step_aggfirst", name, H), H=eH, dH=edH)
    assert eH <= TAU_TGCN and edH <= TAU_TGCN, (eH, edH)
    check_sequence(("step_aggfirst", name, H), {k: grads[k].cpu().numpy() for k in ("W", "b", "L", "l")}, rg, sc,
                   normwise=g_tol(V))


def test_train_sequence_dtdg_aggregate_first(stg, agg_first):
    """Algorithm 1 over DTDG sequences in aggregate-first order: no backward snapshots
    are built, and loss, H_t and every gradient match the oracle sequence."""
    cfg = gen.CONFIGS["C5s"]
    d = gen.dtdg(cfg)
    g = stg.stg_dtdg_create(d.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src,
                            d.del_dst, stg.STG_SELF_LOOPS)
    snaps = [oracle.csr(d.V, S) for S in oracle.snapshot_sets_fold(d, self_loops=True)]
    p, pg = _params(cfg.F, cfg.H, 3)
    H0 = np.zeros((cfg.V, cfg.H))
    Hc = to_gpu(H0)
    S = 4
    for t0 in (0, S):
        Xs = [gen.features(cfg, t0 + i) for i in range(S)]
        Ys = [gen.labels(cfg, t0 + i) for i in range(S)]
        grads = _zero_grads(cfg.F, cfg.H)
        dw, db, loss = torch.zeros(cfg.H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
        Hseq = torch.empty(S, cfg.V, cfg.H, device="cuda")
        stack = stg.stg_state_stack_create(S * cfg.V * (3 * cfg.H + cfg.F) * 4 + (1 << 20))
        stg.stg_tgcn_train_sequence(g, t0, S, pg, pg["w_o"], pg["b_o"], [to_gpu(x) for x in Xs],
                                    [to_gpu(y) for y in Ys], Hc, Hseq, torch.empty(2, cfg.V, cfg.H, device="cuda"),
                                    grads, dw, db, loss, stack)
        assert stack.depth == 0
        rl, rg, rH = oracle.train_sequence(snaps[t0:t0 + S], snaps[t0:t0 + S], p, Xs, Ys, H0)
        _check_seq(("seq_aggfirst", t0), snaps[t0:t0 + S], p, Xs, Ys, H0, loss.item(), grads, dw, db, Hseq, rl, rg,
                   rH, cfg.V * S)
        H0 = rH
        Hc = Hseq[-1].clone()


def test_aggregate_first_rejects_unsupported(stg, agg_first):
    cfg, g, ref = _graph(stg, "C2")
    p, pg = _params(cfg.F, 64, 1)                 # H = 64: no tensor-core path
    with pytest.raises(stg.StgError) as e:
        stg.stg_tgcn_step(g.view(), pg, to_gpu(gen.features(cfg, 0)), torch.zeros(cfg.V, 64, device="cuda"))
    assert e.value.status == 1
    with pytest.raises(stg.StgError):
        stg.stg_set_conv_order(2)


@pytest.mark.parametrize("name,S", [("C2", 8), ("C5s", 4)])
def test_static_sequence_cuda_graph_replay(stg, name, S):
    """A sequence-batched training sequence captured as one CUDA graph (on a stream that
    already ran it, as bench.py does) replays to the eager run's losses, gradients and
    states bit for bit (every kernel is deterministic; nothing allocates while capturing)."""
    cfg = gen.CONFIGS[name]
    if name == "C5s":                                   # a static graph of the DTDG's base edges
        dd = gen.dtdg(cfg)
        s, d = dd.src0, dd.dst0
    else:
        s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)
    _, pg = _params(cfg.F, cfg.H, 3)
    H = cfg.H
    Xg = [to_gpu(gen.features(cfg, 40 + i)) for i in range(S)]
    Yg = [to_gpu(gen.labels(cfg, 40 + i)) for i in range(S)]
    H0 = to_gpu(gen.uniform_pm1(9, 9, cfg.V * H).reshape(cfg.V, H))
    grads = _zero_grads(cfg.F, H)
    dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
    Hseq = torch.empty(S, cfg.V, H, device="cuda")
    stack = stg.stg_state_stack_create(1 << 20)

    def run():
        for t in (*grads.values(), dw, db, loss):
            t.zero_()
        stg.stg_tgcn_train_sequence_batched(g, S, pg, pg["w_o"], pg["b_o"], Xg, Yg, H0, Hseq, grads, dw, db, loss,
                                            stack)

    cs = torch.cuda.Stream()
    cs.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(cs):
        run()
    torch.cuda.synchronize()
    ref = {k: v.clone() for k, v in {**grads, "dw": dw, "db": db, "loss": loss, "H": Hseq}.items()}
    for t in (*grads.values(), dw, db, loss, Hseq):
        t.fill_(float("nan"))
    cg = torch.cuda.CUDAGraph()
    with torch.cuda.graph(cg, stream=cs, capture_error_mode="relaxed"):
        run()
    got = {**grads, "dw": dw, "db": db, "loss": loss, "H": Hseq}
    for rep in range(3):
        cg.replay()
        torch.cuda.synchronize()
        for k in ref:
            assert torch.equal(got[k], ref[k]), (rep, k)


@pytest.mark.parametrize("order", [0, 1])
def test_dtdg_sequences_cuda_graph_replay(stg, order):
    """Two Algorithm-1 sequences over a DTDG (on-demand snapshots on the library's side
    stream, the three-stream pipeline) captured as one CUDA graph on a stream that already
    ran them: the replay reproduces an eager run with the same snapshot-cache walk pattern
    bit for bit.  (A graph replays GPU work only: it is valid while the host-side cache
    state at replay equals the state at capture, which a fixed per-epoch walk keeps.)"""
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    g = stg.stg_dtdg_create(dd.V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off,
                            dd.del_src, dd.del_dst, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    _, pg = _params(cfg.F, cfg.H, 3)
    V, H, F, S = cfg.V, cfg.H, cfg.F, 4
    seqs = [(0, S), (S, S)]
    Xg = [to_gpu(gen.features(cfg, 40 + i)) for i in range(2 * S)]
    Yg = [to_gpu(gen.labels(cfg, 40 + i)) for i in range(2 * S)]
    H0 = torch.zeros(V, H, device="cuda")
    grads = _zero_grads(F, H)
    dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
    Hbuf = [torch.empty(S, V, H, device="cuda") for _ in range(2)]
    Gw = torch.empty(2, V, H, device="cuda")
    stack = stg.stg_state_stack_create(S * V * (3 * H + F) * 4 + (1 << 20))
    stg.stg_set_conv_order(order)
    try:
        def run():
            for t in (*grads.values(), dw, db, loss):
                t.zero_()
            Hp = H0
            for k, (t0, n) in enumerate(seqs):
                stg.stg_tgcn_train_sequence(g, t0, n, pg, pg["w_o"], pg["b_o"], Xg[t0:t0 + n], Yg[t0:t0 + n], Hp,
                                            Hbuf[k], Gw, grads, dw, db, loss, stack)
                Hp = Hbuf[k][n - 1]

        cs = torch.cuda.Stream()
        cs.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(cs):
            run()                                       # warm-up: scratch, slots and cache heads settle
            run()                                       # the reference, in the steady walk pattern
        torch.cuda.synchronize()
        ref = {k: v.clone() for k, v in {**grads, "dw": dw, "db": db, "loss": loss, "H0": Hbuf[0],
                                          "H1": Hbuf[1]}.items()}
        for t in (*grads.values(), dw, db, loss, *Hbuf):
            t.fill_(float("nan"))
        cg = torch.cuda.CUDAGraph()
        with torch.cuda.graph(cg, stream=cs, capture_error_mode="relaxed"):
            run()
        got = {**grads, "dw": dw, "db": db, "loss": loss, "H0": Hbuf[0], "H1": Hbuf[1]}
        for rep in range(3):                            # repeated replays: no host-side state baked in
            cg.replay()
            torch.cuda.synchronize()
            for k in ref:
                assert torch.equal(got[k], ref[k]), (rep, k)
        assert stack.depth == 0
        with torch.cuda.stream(cs):                     # and eager calls after the replays still agree
            run()
        torch.cuda.synchronize()
        for k in ref:
            assert torch.equal(got[k], ref[k]), ("eager after replays", k)
    finally:
        stg.stg_set_conv_order(0)
