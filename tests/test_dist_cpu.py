"""World-size-2 gloo tests of the row-block sharding plumbing, on CPU.

Each rank holds the destination rows of its nnz-balanced block; the forward
aggregation of the local rows, all-gathered, must equal the whole-graph
aggregation, and the backward partial sums over local edges, all-reduced, must
equal the whole-graph backward.  The local compute here is the fp64 oracle (no
GPU on this host); the collectives and the partition are the product helpers.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle
from paper_conf_ipps_cherianmcc24_b200 import parallel


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, name, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        cfg = gen.CONFIGS[name]
        if cfg.kind == "static":
            s, d = gen.static_edges(cfg)
            g = oracle.static_graph(cfg.V, s, d, self_loops=True)
        else:
            dd = gen.dtdg(cfg)
            g = oracle.csr(cfg.V, next(oracle.snapshot_sets_fold(dd, self_loops=True)))
        V = cfg.V
        W = 24
        x = gen.uniform_pm1(3, 3, V * W).reshape(V, W).astype(np.float64)
        bounds = parallel.row_blocks(g["in_rowptr"], world)
        lo, hi = bounds[rank], bounds[rank + 1]
        # forward: local destination rows, all sources
        rp, col = parallel.local_in_csr(g["in_rowptr"], g["in_col"], lo, hi)
        y_loc = oracle.aggregate(rp, col, g["norm_dst"][lo:hi], g["norm_src"], x)
        y = parallel.allgather_rows(torch.from_numpy(y_loc), bounds).numpy()
        ok_f = np.allclose(y, oracle.aggregate_fwd(g, x), rtol=1e-13, atol=1e-14)
        # backward: out-CSR of the local edges, partial sums for every source
        orp, ocol = parallel.local_out_csr(g["in_rowptr"], g["in_col"], V, lo, hi)
        gx_loc = oracle.aggregate(orp, ocol, g["norm_src"], g["norm_dst"], x)
        gx = parallel.allreduce_sum_(torch.from_numpy(gx_loc)).numpy()
        ok_b = np.allclose(gx, oracle.aggregate_bwd(g, x), rtol=1e-12, atol=1e-13)
        # balance: each block holds about E/world in-edges
        E = int(g["in_rowptr"][-1])
        nnz = int(g["in_rowptr"][hi] - g["in_rowptr"][lo])
        maxdeg = int(np.max(np.diff(g["in_rowptr"])))
        ok_bal = abs(nnz - E / world) <= maxdeg + 1
        q.put((rank, bool(ok_f), bool(ok_b), bool(ok_bal), bounds))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - surfaced through the queue
        q.put((rank, False, False, False, repr(e)))


@pytest.mark.parametrize("name", ["C2", "C5s"])
def test_row_block_sharding_world2(name):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, ok_f, ok_b, ok_bal, info in res:
        assert ok_f and ok_b and ok_bal, (rank, ok_f, ok_b, ok_bal, info)
    assert res[0][4] == res[1][4]           # both ranks agree on the partition


def test_row_blocks_properties():
    rng = np.random.default_rng(0)
    for _ in range(50):
        V = int(rng.integers(1, 500))
        deg = rng.integers(0, 20, V)
        deg[rng.integers(0, V)] += int(rng.integers(0, 500))     # a hub
        rp = np.concatenate([[0], np.cumsum(deg)])
        for world in (1, 2, 3, 8):
            b = parallel.row_blocks(rp, world)
            assert b[0] == 0 and b[-1] == V and all(b[i] <= b[i + 1] for i in range(world))
            E = rp[-1]
            for k in range(world):
                nnz = rp[b[k + 1]] - rp[b[k]]
                assert nnz <= E / world + deg.max() + 1


def test_base_row_blocks_match_the_oracle_rowptr():
    """bench.py's partition of the DTDG base (edge list -> edge set + loops -> blocks)
    equals row_blocks over the oracle's in-CSR row pointer of S_0."""
    for name in ("C4", "C5s"):
        cfg = gen.CONFIGS[name]
        dd = gen.dtdg(cfg)
        g = oracle.csr(cfg.V, next(oracle.snapshot_sets_fold(dd, self_loops=True)))
        for world in (2, 3, 8):
            assert parallel.base_row_blocks(cfg.V, dd.src0, dd.dst0, world) == \
                parallel.row_blocks(g["in_rowptr"], world), (name, world)


def _grad_worker(rank, world, port, q):
    """Sharded TGCN gradients: rank k's share of every parameter gradient
    is the sum over its local rows / edges; bench.py all-reduces one flat buffer per
    sequence.  Here the shares are the fp64 oracle's per-block row sums of a separable
    gradient (Σ_rows Aᵀ B over the block) and the all-reduce must give the whole sum."""
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        V, F, N = 1000, 8, 12
        A = gen.uniform_pm1(5, 1, V * F).reshape(V, F).astype(np.float64)
        B = gen.uniform_pm1(5, 2, V * N).reshape(V, N).astype(np.float64)
        rp = np.arange(V + 1)
        bounds = parallel.row_blocks(rp, world)
        lo, hi = bounds[rank], bounds[rank + 1]
        flat = torch.zeros(F * N + N, dtype=torch.float64)
        flat[: F * N] = torch.from_numpy((A[lo:hi].T @ B[lo:hi]).ravel())
        flat[F * N:] = torch.from_numpy(B[lo:hi].sum(0))
        parallel.allreduce_sum_(flat)
        ok = np.allclose(flat[: F * N].numpy().reshape(F, N), A.T @ B, rtol=1e-12, atol=1e-12) and \
            np.allclose(flat[F * N:].numpy(), B.sum(0), rtol=1e-12, atol=1e-12)
        q.put((rank, bool(ok), None))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put((rank, False, repr(e)))


def test_sharded_gradient_allreduce_world2():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_grad_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, ok, info in res:
        assert ok, (rank, info)
