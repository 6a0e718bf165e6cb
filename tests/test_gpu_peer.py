"""GPU parity of the sharded mode over peer memory (SURVEY §8(e) "sharded mode";
north_star: destination-row blocks, source rows exchanged over NVLink each
timestep).  The exchange is fused into the aggregation: a rank reads each
neighbour row from its owner's block (stg_gcn_aggregate_peer).

One GPU is available, so

* the ranks of a world are simulated in this process (every block a separate
  allocation, the aggregation reading through the row table exactly as it reads
  IPC-mapped peer memory): rows must be bit-identical to the resident-mode
  aggregation (same schedule, same order), the all-gather bit-identical to the
  concatenation, the reduce-scatter bit-identical to the rank-ordered fp32 sum,
  and a whole TGCN sequence must sum to the whole-graph oracle sequence;
* two real processes share the GPU through CUDA IPC handles (stg_peer_alloc /
  stg_peer_open) and run parallel.PeerTGCN with a gloo barrier: their summed
  loss and gradients must match the oracle.
"""
import os

import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import to_gpu

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _blocks(V, s, d, world):
    from paper_conf_ipps_cherianmcc24_b200 import parallel
    return parallel.base_row_blocks(V, s, d, world)


def _table(stg, x, bounds):
    """Each block of x in its own allocation (as on separate GPUs)."""
    blocks = [x[bounds[k]:bounds[k + 1]].clone() for k in range(len(bounds) - 1)]
    ptrs = [b.data_ptr() if b.shape[0] else 0 for b in blocks]
    return stg.PeerRows(bounds, ptrs, x.shape[1]), blocks


@pytest.mark.parametrize("name,world,W", [("C2", 3, 96), ("C1", 4, 48), ("C6", 2, 8), ("C2", 1, 96),
                                          ("C2", 2, 256)])
def test_aggregate_peer_bit_identical_to_resident(stg, name, world, W):
    cfg = gen.CONFIGS[name]
    s, d = gen.static_edges(cfg)
    V = cfg.V
    flags = stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS
    b = _blocks(V, s, d, world)
    x = to_gpu(gen.features(cfg, 0, width=W))
    rows, keep = _table(stg, x, b)
    bias = to_gpu(gen.features(cfg, 5, width=W)[0])
    for k in range(world):
        lo, hi = b[k], b[k + 1]
        g = stg.stg_static_graph_create(V, s, d, flags, dist=(k, world, lo, hi))
        v = g.view()
        y_res = stg.stg_gcn_aggregate_fwd(v, x)
        y_peer = stg.stg_gcn_aggregate_peer(v, rows, W, scale_row=_loc(stg, v, "norm_dst"),
                                            scale_col=_loc(stg, v, "norm_src", full=True))
        if W > 32:
            assert torch.equal(y_peer, y_res), (name, k)
        else:       # resident W <= 32 runs the row-item kernel: same sums, other fp32 order
            torch.testing.assert_close(y_peer, y_res, rtol=1e-6, atol=1e-6)
        # bias + no column scale (the TGCN form: P' pre-scaled)
        y2 = stg.stg_gcn_aggregate_ex(v, False, x, scale_row=_loc(stg, v, "norm_dst"), bias=bias)
        y2p = stg.stg_gcn_aggregate_peer(v, rows, W, scale_row=_loc(stg, v, "norm_dst"), bias=bias)
        if W > 32:
            assert torch.equal(y2p, y2), (name, k, "bias")
        else:
            torch.testing.assert_close(y2p, y2, rtol=1e-6, atol=1e-6)


def _loc(stg, v, key, full=False):
    a = stg.view_arrays(v)[key]
    return a if full else a[v.row_begin:v.row_end].contiguous()


def test_aggregate_peer_empty_blocks(stg):
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    V = cfg.V
    b = [0, 0, 400, 400, V]                        # two empty blocks
    x = to_gpu(gen.features(cfg, 2, width=64))
    rows, keep = _table(stg, x, b)
    for k in range(4):
        g = stg.stg_static_graph_create(V, s, d, stg.STG_SELF_LOOPS, dist=(k, 4, b[k], b[k + 1]))
        v = g.view()
        y = stg.stg_gcn_aggregate_peer(v, rows, 64, scale_row=_loc(stg, v, "norm_dst"),
                                       scale_col=_loc(stg, v, "norm_src", full=True))
        assert torch.equal(y, stg.stg_gcn_aggregate_fwd(v, x)), k


def test_aggregate_peer_rejects_bad_tables(stg):
    cfg = gen.CONFIGS["C6"]
    s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)
    x = torch.zeros(cfg.V, 8, device="cuda")
    for bounds, ptrs, W in (([0, 10], [x.data_ptr()], 8),                  # does not span V
                            ([0, cfg.V], [x.data_ptr() + 4], 8),            # misaligned block
                            ([0, cfg.V], [x.data_ptr()], 6),                # W % 4
                            ([0, 5, cfg.V], [x.data_ptr(), 0], 8)):         # NULL non-empty block
        with pytest.raises(stg.StgError) as e:
            stg.stg_gcn_aggregate_peer(g.view(), stg.PeerRows(bounds, ptrs, 8), W)
        assert e.value.status == 1


@pytest.mark.parametrize("W", [96, 30])
def test_allgather_and_reduce_scatter_rows(stg, W):
    V, world = 1000, 3
    b = [0, 123, 123, V] if W == 30 else [0, 300, 650, V]
    world = len(b) - 1
    x = torch.randn(V, W, device="cuda")
    rows, keep = _table(stg, x, b)
    full = torch.empty(V, W, device="cuda")
    stg.stg_allgather_rows(rows, W, full)
    assert torch.equal(full, x)
    parts = [torch.randn(V, W, device="cuda") for _ in range(world)]
    for r in range(world):
        out = torch.empty(b[r + 1] - b[r], W, device="cuda")
        stg.stg_reduce_scatter_rows(b, parts, W, r, W, out)
        ref = parts[0][b[r]:b[r + 1]].clone()
        for q in range(1, world):
            ref = ref + parts[q][b[r]:b[r + 1]]
        assert torch.equal(out, ref), r


def _sequence_reference(cfg, dd, S, p, Xs, Ys):
    V, H = cfg.V, cfg.H
    sets = list(oracle.snapshot_sets_fold(dd, self_loops=True))
    snaps = [oracle.csr(V, sets[t]) for t in range(S)]
    return oracle.train_sequence(snaps, snaps, p, Xs, Ys, np.zeros((V, H))), sets


def _check_grads(l_sum, g_sum, rl, rg, V, S):
    assert abs(l_sum - rl) <= 1e-5 * abs(rl), (l_sum, rl)
    tol = max(1e-4, 1e-6 * np.sqrt(V * S))          # tests/test_gpu_tgcn.py g_tol
    for n in ("W", "b", "L", "l", "w_o", "b_o"):
        ref = np.asarray(rg[n], np.float64)
        err = np.max(np.abs(g_sum[n] - ref)) / max(np.max(np.abs(ref)), 1e-300)
        assert err <= tol, (n, err)


def test_tgcn_peer_sequence_simulated_ranks(stg):
    """Sharded-mode Algorithm 1 on a DTDG, three ranks interleaved phase by phase
    (project -> [barrier] -> gather+GRU; backward -> [barrier] -> reduce-scatter, dW)."""
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    V, F, H, S, world = cfg.V, cfg.F, cfg.H, 4, 3
    p = gen.tgcn_params(F, H, 1)
    pg = {k: torch.from_numpy(v).cuda() for k, v in p.items()}
    Xs = [gen.features(cfg, t) for t in range(S)]
    Ys = [gen.labels(cfg, t) for t in range(S)]
    (rl, rg, rH), sets = _sequence_reference(cfg, dd, S, p, Xs, Ys)
    b = _blocks(V, dd.src0, dd.dst0, world)
    ranks = []
    for k in range(world):
        lo, hi = b[k], b[k + 1]
        R = hi - lo
        r = {"lo": lo, "hi": hi, "R": R}
        r["g"] = stg.stg_dtdg_create(V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off,
                                     dd.del_src, dd.del_dst, stg.STG_SELF_LOOPS, dist=(k, world, lo, hi))
        r["grads"] = {"W": torch.zeros(F, 3 * H, device="cuda"), "b": torch.zeros(3 * H, device="cuda"),
                      "L": torch.zeros(3, 2 * H, H, device="cuda"), "l": torch.zeros(3, H, device="cuda")}
        r["dw"], r["db"], r["loss"] = (torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"),
                                       torch.zeros(1, device="cuda"))
        r["Hs"] = torch.empty(S, R, H, device="cuda")
        r["G"] = [torch.zeros(R, H, device="cuda"), torch.empty(R, H, device="cuda")]
        r["X"] = [torch.from_numpy(x[lo:hi].copy()).cuda() for x in Xs]
        r["Y"] = [torch.from_numpy(y[lo:hi].copy()).cuda() for y in Ys]
        r["P"] = [torch.empty(max(R, 1), 3 * H, device="cuda") for _ in range(2)]
        r["dP"] = [torch.empty(V, 3 * H, device="cuda") for _ in range(2)]
        r["dPl"] = torch.empty(max(R, 1), 3 * H, device="cuda")
        r["st"] = stg.stg_state_stack_create(S * max(R, 1) * 3 * H * 4 + (1 << 20))
        ranks.append(r)
    for i in range(S):
        views = [stg.stg_dtdg_get_snapshot_parts(r["g"], i, stg.STG_PART_IN) for r in ranks]
        for r, v in zip(ranks, views):
            stg.stg_tgcn_project(v, pg, r["X"][i], r["P"][i & 1])
        table = stg.PeerRows(b, [r["P"][i & 1].data_ptr() for r in ranks], 3 * H)
        for r, v in zip(ranks, views):
            if i == 0:
                r["H0"] = torch.zeros(r["R"], H, device="cuda")   # kept: the stack holds H_{t-1} by reference
            Hp = r["H0"] if i == 0 else r["Hs"][i - 1]
            stg.stg_tgcn_step_peer(v, pg, table, Hp, r["Hs"][i], r["st"])
            stg.stg_mse_head(r["Hs"][i], r["Y"][i], pg["w_o"], pg["b_o"], loss_accum=r["loss"], V_total=V)
    for i in range(S - 1, -1, -1):
        views = [stg.stg_dtdg_get_snapshot_parts(r["g"], i, stg.STG_PART_OUT, backward=True) for r in ranks]
        for r, v in zip(ranks, views):
            G, Gn = r["G"][0], r["G"][1]
            stg.stg_mse_head(r["Hs"][i], r["Y"][i], pg["w_o"], pg["b_o"], dH=G, accumulate=True, dw_o=r["dw"],
                             db_o=r["db"], V_total=V)
            stg.stg_tgcn_step_backward_peer(v, pg, G, Gn, r["grads"], r["dP"][i & 1], r["st"])
            r["G"] = [Gn, G]
        for k, r in enumerate(ranks):
            stg.stg_reduce_scatter_rows(b, [q["dP"][i & 1] for q in ranks], 3 * H, k, 3 * H, r["dPl"][:r["R"]])
            stg.stg_tgcn_dw(pg, r["X"][i], r["dPl"][:r["R"]], r["grads"], r["st"])
    torch.cuda.synchronize()
    l_sum, g_sum = 0.0, None
    for r in ranks:
        np.testing.assert_allclose(r["Hs"][-1].cpu().numpy(), rH[r["lo"]:r["hi"]], rtol=0, atol=2e-5)
        l_sum += r["loss"].item()
        gk = {n: t.cpu().numpy().astype(np.float64) for n, t in r["grads"].items()}
        gk.update(w_o=r["dw"].cpu().numpy().astype(np.float64), b_o=r["db"].cpu().numpy().astype(np.float64))
        g_sum = gk if g_sum is None else {n: g_sum[n] + gk[n] for n in g_sum}
    _check_grads(l_sum, g_sum, rl, rg, V, S)


def _ipc_worker(rank, world, port, outdir):
    import faulthandler
    import sys
    faulthandler.enable()
    sys.path.insert(0, ROOT)
    import torch.distributed as dist
    import paper_conf_ipps_cherianmcc24_b200 as stg
    from paper_conf_ipps_cherianmcc24_b200 import parallel
    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world)
    torch.cuda.set_device(0)
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    V, F, H, S = cfg.V, cfg.F, cfg.H, 3
    b = parallel.base_row_blocks(V, dd.src0, dd.dst0, world)
    lo, hi = b[rank], b[rank + 1]
    R = hi - lo
    g = stg.stg_dtdg_create(V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off, dd.del_src,
                            dd.del_dst, stg.STG_SELF_LOOPS, dist=(rank, world, lo, hi))
    p = {k: torch.from_numpy(v).cuda() for k, v in gen.tgcn_params(F, H, 1).items()}
    grads = {"W": torch.zeros(F, 3 * H, device="cuda"), "b": torch.zeros(3 * H, device="cuda"),
             "L": torch.zeros(3, 2 * H, H, device="cuda"), "l": torch.zeros(3, H, device="cuda")}
    dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
    drv = parallel.PeerTGCN(stg, b, V, F, H, S)
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


def test_peer_ipc_two_processes(stg, tmp_path):
    import socket
    import torch.multiprocessing as mp
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    world = 2
    mp.start_processes(_ipc_worker, args=(world, port, str(tmp_path)), nprocs=world, join=True,
                       start_method="spawn")
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    S = 3
    p = gen.tgcn_params(cfg.F, cfg.H, 1)
    Xs = [gen.features(cfg, t) for t in range(S)]
    Ys = [gen.labels(cfg, t) for t in range(S)]
    (rl, rg, rH), _ = _sequence_reference(cfg, dd, S, p, Xs, Ys)
    l_sum, g_sum = 0.0, None
    for r in range(world):
        z = np.load(os.path.join(str(tmp_path), "rank%d.npz" % r))
        lo, hi = int(z["lo"]), int(z["hi"])
        np.testing.assert_allclose(z["H"], rH[lo:hi], rtol=0, atol=2e-5)
        l_sum += float(z["loss"][0])
        gk = {n: z[n].astype(np.float64) for n in ("W", "b", "L", "l", "w_o", "b_o")}
        g_sum = gk if g_sum is None else {n: g_sum[n] + gk[n] for n in g_sum}
    _check_grads(l_sum, g_sum, rl, rg, cfg.V, S)
