"""GPU parity of the original T-GCN cell (GCN over [X, H])
against the fp64 oracle (orc_tgcn2_fwd/bwd, pinned in tests/test_oracle_tgcn2.py).
The GPU runs the convolutions linear-first, Â([X,H]W) (same maths, reading C14);
tolerances as for the PyG-T cell: H' absolute 2e-5, gradients
normwise max(1e-4, 1e-6·sqrt(n)).  A whole Algorithm-1 sequence (forward with the
state stack, surrogate head, BPTT in LIFO order) runs over DTDG snapshots."""
import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu


def _zero2(F, H):
    return {"Wg": torch.zeros(F + H, 2 * H, device="cuda"), "bg": torch.zeros(2 * H, device="cuda"),
            "Wc": torch.zeros(F + H, H, device="cuda"), "bc": torch.zeros(H, device="cuda")}


def _gtol(n):
    return max(1e-4, 1e-6 * np.sqrt(n))


def _check(gpu: dict, ref: dict, n, keys=("Wg", "bg", "Wc", "bc")):
    for k in keys:
        a = gpu[k].cpu().numpy().astype(np.float64) if isinstance(gpu[k], torch.Tensor) else gpu[k]
        r = np.asarray(ref[k], np.float64)
        err = np.max(np.abs(a - r)) / max(np.max(np.abs(r)), 1e-300)
        assert err <= _gtol(n), (k, err)


@pytest.mark.parametrize("name,H", [("C2", 32), ("C1", 16), ("C6", 8)])
def test_tgcn2_step_fwd_bwd(stg, name, H):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    V, F = cfg.V, cfg.F
    g = stg.stg_static_graph_create(V, s, d, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    ref_g = oracle.static_graph(V, s, d, self_loops=True)
    p = gen.tgcn2_params(F, H, cfg.seed)
    pg = {k: torch.from_numpy(v).cuda() for k, v in p.items()}
    X = gen.features(cfg, 0)
    Hp = gen.uniform_pm1(cfg.seed, 70, V * H).reshape(V, H)
    Gd = gen.uniform_pm1(cfg.seed, 71, V * H).reshape(V, H)
    st = stg.stg_state_stack_create(V * 3 * H * 4 + (1 << 20))
    Hpg = torch.from_numpy(Hp).cuda()
    Hn = stg.stg_tgcn2_step(g.view(), pg, torch.from_numpy(X).cuda(), Hpg, stack=st)
    f = oracle.tgcn2_fwd(ref_g, p, X, Hp)
    assert np.max(np.abs(Hn.cpu().numpy() - f["Hn"])) <= 2e-5
    grads = _zero2(F, H)
    dHp = stg.stg_tgcn2_step_backward(g.view(), pg, torch.from_numpy(X).cuda(), torch.from_numpy(Gd).cuda(), grads,
                                      st)
    torch.cuda.synchronize()
    rg = oracle.zero_grads2(F, H)
    rdH = oracle.tgcn2_bwd(ref_g, p, X, Hp, f, Gd, rg)
    _check(grads, rg, V)
    err = np.max(np.abs(dHp.cpu().numpy() - rdH)) / max(np.max(np.abs(rdH)), 1e-300)
    assert err <= 1e-4, err
    assert st.depth == 0


def test_tgcn2_zero_parameters_halve_state(stg):
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)
    F, H = cfg.F, 32
    pg = _zero2(F, H)
    Hp = torch.from_numpy(gen.uniform_pm1(1, 72, cfg.V * H).reshape(cfg.V, H)).cuda()
    Hn = stg.stg_tgcn2_step(g.view(), pg, torch.from_numpy(gen.features(cfg, 0)).cuda(), Hp)
    assert torch.equal(Hn, 0.5 * Hp)


def test_tgcn2_sequence_over_dtdg(stg):
    """Algorithm 1 with the original T-GCN cell over DTDG snapshots (Get-Graph forward,
    Get-Backward-Graph in LIFO order), surrogate head, BPTT."""
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    V, F, H, S = cfg.V, cfg.F, cfg.H, 3
    dg = stg.stg_dtdg_create(dd.V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off,
                             dd.del_src, dd.del_dst, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    p = gen.tgcn2_params(F, H, 4)
    pg = {k: torch.from_numpy(v).cuda() for k, v in p.items()}
    Xs = [gen.features(cfg, t) for t in range(S)]
    Ys = [gen.labels(cfg, t) for t in range(S)]
    Xg = [torch.from_numpy(x).cuda() for x in Xs]
    Yg = [torch.from_numpy(y).cuda() for y in Ys]
    st = stg.stg_state_stack_create(S * V * 3 * H * 4 + (1 << 20))
    grads = _zero2(F, H)
    dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
    Hs = [torch.zeros(V, H, device="cuda")]
    for t in range(S):
        v = stg.stg_dtdg_get_snapshot(dg, t)
        Hs.append(stg.stg_tgcn2_step(v, pg, Xg[t], Hs[-1], stack=st))
        stg.stg_mse_head(Hs[-1], Yg[t], pg["w_o"], pg["b_o"], loss_accum=loss)
    G = torch.zeros(V, H, device="cuda")
    for t in range(S - 1, -1, -1):
        v = stg.stg_dtdg_get_backward_snapshot(dg, t)
        stg.stg_mse_head(Hs[t + 1], Yg[t], pg["w_o"], pg["b_o"], dH=G, accumulate=True, dw_o=dw, db_o=db)
        G = stg.stg_tgcn2_step_backward(v, pg, Xg[t], G, grads, st)
    torch.cuda.synchronize()
    sets = list(oracle.snapshot_sets_fold(dd, self_loops=True))
    rl, rg, rH = oracle.train_sequence2([oracle.csr(V, sets[t]) for t in range(S)], p, Xs, Ys, np.zeros((V, H)))
    assert abs(loss.item() - rl) <= 1e-5 * abs(rl), (loss.item(), rl)
    assert np.max(np.abs(Hs[-1].cpu().numpy() - rH)) <= 2e-5
    gd = dict(grads)
    gd["w_o"], gd["b_o"] = dw, db
    _check(gd, rg, V * S, keys=("Wg", "bg", "Wc", "bc", "w_o", "b_o"))
