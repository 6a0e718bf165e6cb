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


@pytest.mark.parametrize("name", ["C5s", "C4"])
def test_tgcn2_sequence_over_dtdg(stg, name):
    """Algorithm 1 with the original T-GCN cell over DTDG snapshots (Get-Graph forward,
    Get-Backward-Graph in LIFO order), BPTT.  The loss goes through the surrogate head;
    the upstream gradient of step t is a fixed random G_t plus the gradient carried back
    from step t+1.  (The head's ReLU is a decision: an H entry within the fp32 error of 0
    flips its mask between fp32 and fp64 and moves a whole row's contribution to dW by
    O(1/√rows) normwise -- measured 5e-4 on C5s -- so the gradient chain is driven by G_t,
    not by the head; the head's gradient has its own element-wise tests.)  C4 (F = 8)
    runs the Σ AᵀB reductions with padded operand slots at 2 CTAs per SM."""
    cfg = gen.CONFIGS[name]
    dd = gen.dtdg(cfg)
    V, F, H, S = cfg.V, cfg.F, cfg.H, 3
    dg = stg.stg_dtdg_create(dd.V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off,
                             dd.del_src, dd.del_dst, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    p = gen.tgcn2_params(F, H, 4)
    pg = {k: torch.from_numpy(v).cuda() for k, v in p.items()}
    Xs = [gen.features(cfg, t) for t in range(S)]
    Ys = [gen.labels(cfg, t) for t in range(S)]
    Gs = [gen.uniform_pm1(cfg.seed, 80 + t, V * H).reshape(V, H) for t in range(S)]
    Xg = [torch.from_numpy(x).cuda() for x in Xs]
    Yg = [torch.from_numpy(y).cuda() for y in Ys]
    st = stg.stg_state_stack_create(S * V * 3 * H * 4 + (1 << 20))
    grads = _zero2(F, H)
    loss = torch.zeros(1, device="cuda")
    Hs = [torch.zeros(V, H, device="cuda")]
    for t in range(S):
        v = stg.stg_dtdg_get_snapshot(dg, t)
        Hs.append(stg.stg_tgcn2_step(v, pg, Xg[t], Hs[-1], stack=st))
        stg.stg_mse_head(Hs[-1], Yg[t], pg["w_o"], pg["b_o"], loss_accum=loss)
    G = torch.zeros(V, H, device="cuda")
    for t in range(S - 1, -1, -1):
        v = stg.stg_dtdg_get_backward_snapshot(dg, t)
        G = stg.stg_tgcn2_step_backward(v, pg, Xg[t], G + torch.from_numpy(Gs[t]).cuda(), grads, st)
    torch.cuda.synchronize()
    sets = list(oracle.snapshot_sets_fold(dd, self_loops=True))
    graphs = [oracle.csr(V, sets[t]) for t in range(S)]
    rg = oracle.zero_grads2(F, H)
    Hc, fs, rl = np.zeros((V, H)), [], 0.0
    for t in range(S):
        f = oracle.tgcn2_fwd(graphs[t], p, Xs[t], Hc)
        fs.append((Hc, f))
        rl += oracle.mse_head(f["Hn"], Ys[t], p["w_o"], p["b_o"], {"w_o": np.zeros(H), "b_o": np.zeros(1)})[0]
        Hc = f["Hn"]
    rdH = np.zeros((V, H))
    for t in range(S - 1, -1, -1):
        Hp, f = fs[t]
        rdH = oracle.tgcn2_bwd(graphs[t], p, Xs[t], Hp, f, rdH + Gs[t], rg)
    assert abs(loss.item() - rl) <= 1e-5 * abs(rl), (loss.item(), rl)
    assert np.max(np.abs(Hs[-1].cpu().numpy() - Hc)) <= 2e-5
    _check(dict(grads), rg, V * S, keys=("Wg", "bg", "Wc", "bc"))
    err = np.max(np.abs(G.cpu().numpy() - rdH)) / np.max(np.abs(rdH))
    assert err <= 1e-4, err


def test_tgcn2_sharded_peer_simulated_ranks(stg):
    """Sharded original T-GCN (hidden-state rows cross ranks every step): three ranks of a
    DTDG interleaved phase by phase in one process (every block its own allocation);
    the rows of H_t match the oracle and the summed loss / gradients match the
    whole-graph oracle sequence."""
    from paper_conf_ipps_cherianmcc24_b200 import parallel
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    V, F, H, S, world = cfg.V, cfg.F, cfg.H, 3, 3
    p = gen.tgcn2_params(F, H, 6)
    pg = {k: torch.from_numpy(v).cuda() for k, v in p.items()}
    Xs = [gen.features(cfg, t) for t in range(S)]
    Ys = [gen.labels(cfg, t) for t in range(S)]
    b = parallel.base_row_blocks(V, dd.src0, dd.dst0, world)
    ranks = []
    for k in range(world):
        lo, hi = b[k], b[k + 1]
        R = hi - lo
        r = {"lo": lo, "hi": hi, "R": R, "grads": _zero2(F, H)}
        r["g"] = stg.stg_dtdg_create(V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off,
                                     dd.del_src, dd.del_dst, stg.STG_SELF_LOOPS, dist=(k, world, lo, hi))
        r["dw"], r["db"], r["loss"] = (torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"),
                                       torch.zeros(1, device="cuda"))
        r["Hs"] = [torch.zeros(R, H, device="cuda")] + [torch.empty(R, H, device="cuda") for _ in range(S)]
        r["X"] = [torch.from_numpy(x[lo:hi].copy()).cuda() for x in Xs]
        r["Y"] = [torch.from_numpy(y[lo:hi].copy()).cuda() for y in Ys]
        r["Zg"] = torch.empty(max(R, 1), 2 * H, device="cuda")
        r["Zc"] = torch.empty(max(R, 1), H, device="cuda")
        r["Dc"] = torch.empty(V, H, device="cuda")
        r["Dg"] = torch.empty(V, 2 * H, device="cuda")
        r["G"] = [torch.zeros(R, H, device="cuda"), torch.empty(R, H, device="cuda")]
        r["st"] = stg.stg_state_stack_create(S * max(R, 1) * 3 * H * 4 + (1 << 20))
        ranks.append(r)
    for i in range(S):
        vs = [stg.stg_dtdg_get_snapshot_parts(r["g"], i, stg.STG_PART_IN) for r in ranks]
        for r, v in zip(ranks, vs):
            stg.stg_tgcn2_peer_fwd(0, v, pg, r["X"][i], r["Hs"][i], Z_loc=r["Zg"], stack=r["st"])
        tg = stg.PeerRows(b, [r["Zg"].data_ptr() for r in ranks], 2 * H)
        for r, v in zip(ranks, vs):
            stg.stg_tgcn2_peer_fwd(1, v, pg, r["X"][i], r["Hs"][i], rows=tg, Z_loc=r["Zc"], stack=r["st"])
        tc = stg.PeerRows(b, [r["Zc"].data_ptr() for r in ranks], H)
        for r, v in zip(ranks, vs):
            stg.stg_tgcn2_peer_fwd(2, v, pg, r["X"][i], r["Hs"][i], rows=tc, H_next=r["Hs"][i + 1], stack=r["st"])
            stg.stg_mse_head(r["Hs"][i + 1], r["Y"][i], pg["w_o"], pg["b_o"], loss_accum=r["loss"], V_total=V)
    for i in range(S - 1, -1, -1):
        vs = [stg.stg_dtdg_get_snapshot_parts(r["g"], i, stg.STG_PART_OUT, backward=True) for r in ranks]
        for r, v in zip(ranks, vs):
            G, Gn = r["G"]
            stg.stg_mse_head(r["Hs"][i + 1], r["Y"][i], pg["w_o"], pg["b_o"], dH=G, accumulate=True, dw_o=r["dw"],
                             db_o=r["db"], V_total=V)
            stg.stg_tgcn2_peer_bwd(0, v, pg, r["X"][i], G, Gn, r["grads"], 0, b, None, r["Dc"], r["st"])
        for k, (r, v) in enumerate(zip(ranks, vs)):
            stg.stg_tgcn2_peer_bwd(1, v, pg, r["X"][i], None, r["G"][1], r["grads"], k, b,
                                   [q["Dc"] for q in ranks], r["Dg"], r["st"])
        for k, (r, v) in enumerate(zip(ranks, vs)):
            stg.stg_tgcn2_peer_bwd(2, v, pg, r["X"][i], None, r["G"][1], r["grads"], k, b,
                                   [q["Dg"] for q in ranks], None, r["st"])
            r["G"] = [r["G"][1], r["G"][0]]
    torch.cuda.synchronize()
    sets = list(oracle.snapshot_sets_fold(dd, self_loops=True))
    rl, rg, rH = oracle.train_sequence2([oracle.csr(V, sets[t]) for t in range(S)], p, Xs, Ys, np.zeros((V, H)))
    l_sum, g_sum = 0.0, None
    for r in ranks:
        np.testing.assert_allclose(r["Hs"][-1].cpu().numpy(), rH[r["lo"]:r["hi"]], rtol=0, atol=2e-5)
        l_sum += r["loss"].item()
        gk = {n: t.cpu().numpy().astype(np.float64) for n, t in r["grads"].items()}
        gk.update(w_o=r["dw"].cpu().numpy().astype(np.float64), b_o=r["db"].cpu().numpy().astype(np.float64))
        g_sum = gk if g_sum is None else {n: g_sum[n] + gk[n] for n in g_sum}
    assert abs(l_sum - rl) <= 1e-5 * abs(rl), (l_sum, rl)
    _check(g_sum, rg, V * S, keys=("Wg", "bg", "Wc", "bc", "w_o", "b_o"))


def _ipc_worker2(rank, world, port, outdir):
    import faulthandler
    faulthandler.enable()
    import os
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist
    import paper_conf_ipps_cherianmcc24_b200 as stg
    from paper_conf_ipps_cherianmcc24_b200 import parallel
    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world)
    torch.cuda.set_device(0)
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    V, F, H, S = cfg.V, cfg.F, cfg.H, 2
    b = parallel.base_row_blocks(V, dd.src0, dd.dst0, world)
    lo, hi = b[rank], b[rank + 1]
    R = hi - lo
    g = stg.stg_dtdg_create(V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off, dd.del_src,
                            dd.del_dst, stg.STG_SELF_LOOPS, dist=(rank, world, lo, hi))
    p = {k: torch.from_numpy(v).cuda() for k, v in gen.tgcn2_params(F, H, 6).items()}
    grads = _zero2(F, H)
    dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
    drv = parallel.PeerTGCN2(stg, b, V, F, H, S)
    X = [torch.from_numpy(gen.features(cfg, t)[lo:hi].copy()).cuda() for t in range(S)]
    Y = [torch.from_numpy(gen.labels(cfg, t)[lo:hi].copy()).cuda() for t in range(S)]
    Hs = torch.empty(S, R, H, device="cuda")
    H0 = torch.zeros(R, H, device="cuda")          # alive until the sequence's kernels ran
    drv.train_sequence(g, 0, p, p["w_o"], p["b_o"], X, Y, H0, Hs, grads, dw, db, loss)
    torch.cuda.synchronize()
    out = {n: t.cpu().numpy() for n, t in grads.items()}
    out.update(w_o=dw.cpu().numpy(), b_o=db.cpu().numpy(), loss=loss.cpu().numpy(), H=Hs[-1].cpu().numpy(),
               lo=np.array(lo), hi=np.array(hi))
    np.savez(os.path.join(outdir, "rank%d.npz" % rank), **out)
    parallel.stream_barrier()
    drv.close()
    dist.destroy_process_group()


def test_tgcn2_sharded_peer_two_processes(stg, tmp_path):
    import os
    import socket
    import torch.multiprocessing as mp
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    world = 2
    mp.start_processes(_ipc_worker2, args=(world, port, str(tmp_path)), nprocs=world, join=True,
                       start_method="spawn")
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    V, H, S = cfg.V, cfg.H, 2
    p = gen.tgcn2_params(cfg.F, H, 6)
    sets = list(oracle.snapshot_sets_fold(dd, self_loops=True))
    rl, rg, rH = oracle.train_sequence2([oracle.csr(V, sets[t]) for t in range(S)], p,
                                        [gen.features(cfg, t) for t in range(S)],
                                        [gen.labels(cfg, t) for t in range(S)], np.zeros((V, H)))
    l_sum, g_sum = 0.0, None
    for r in range(world):
        z = np.load(os.path.join(str(tmp_path), "rank%d.npz" % r))
        lo, hi = int(z["lo"]), int(z["hi"])
        np.testing.assert_allclose(z["H"], rH[lo:hi], rtol=0, atol=2e-5)
        l_sum += float(z["loss"][0])
        gk = {n: z[n].astype(np.float64) for n in ("Wg", "bg", "Wc", "bc", "w_o", "b_o")}
        g_sum = gk if g_sum is None else {n: g_sum[n] + gk[n] for n in g_sum}
    assert abs(l_sum - rl) <= 1e-5 * abs(rl), (l_sum, rl)
    _check(g_sum, rg, V * S, keys=("Wg", "bg", "Wc", "bc", "w_o", "b_o"))
