"""Degenerate and boundary cases of the hot path (③: empty / ragged inputs, maximum
sizes, the method's degenerate cases), each against the oracle or a closed form:
* a DTDG with T = 1 (the base only) and one whose snapshot becomes EMPTY (every
  edge deleted, no self-loops) and is rebuilt afterwards;
* aggregation and a TGCN step on the empty snapshot (Â = 0, so C = b);
* a one-vertex graph (V = 1) through graph build, aggregation and a TGCN step;
* size limits: E >= 2^31 and V >= 2^30 rejected with STG_ERR_OUT_OF_RANGE before
  any device work."""
import ctypes
import os

import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import assert_graph_equal, to_gpu

pytestmark = pytest.mark.gpu


def _dtdg(stg, V, T, s0, d0, adds, dels, flags):
    """adds/dels: list over t of (src, dst) lists; batch 0 empty."""
    def pack(b):
        off = [0]
        ss, dd = [], []
        for (s, d) in b:
            ss += list(s)
            dd += list(d)
            off.append(len(ss))
        return np.array(off, np.int64), np.array(ss, np.int32), np.array(dd, np.int32)
    ao, a_s, a_d = pack(adds)
    do, d_s, d_d = pack(dels)
    return stg.stg_dtdg_create(V, T, s0, d0, ao, a_s, a_d, do, d_s, d_d, flags)


def _oracle_sets(V, s0, d0, adds, dels):
    S = oracle.edge_set(V, s0, d0)
    out = [S]
    for t in range(1, len(adds)):
        A = oracle.keys(*adds[t]) if len(adds[t][0]) else np.zeros(0, np.uint64)
        D = oracle.keys(*dels[t]) if len(dels[t][0]) else np.zeros(0, np.uint64)
        S = oracle.set_apply(S, D, A)
        out.append(S)
    return out


def test_dtdg_single_timestamp(stg):
    V = 50
    s, d = gen.random_edges(3, V, 120, loops=False)
    g = _dtdg(stg, V, 1, s, d, [([], [])], [([], [])], stg.STG_EDGE_IDS)
    ref = oracle.csr(V, oracle.edge_set(V, s, d))
    assert_graph_equal(stg.view_arrays(stg.stg_dtdg_get_snapshot(g, 0)), ref, tag="T=1 fwd")
    assert_graph_equal(stg.view_arrays(stg.stg_dtdg_get_backward_snapshot(g, 0)), ref, tag="T=1 bwd")


def test_dtdg_snapshot_becomes_empty(stg):
    V = 40
    s, d = gen.random_edges(5, V, 90, loops=False)
    S0 = oracle.edge_set(V, s, d)
    us, ud = oracle.unkey(S0)
    adds = [([], []), ([], []), (list(us[:30]), list(ud[:30]))]
    dels = [([], []), (list(us), list(ud)), ([], [])]
    g = _dtdg(stg, V, 3, s, d, adds, dels, stg.STG_EDGE_IDS)
    sets = _oracle_sets(V, s, d, adds, dels)
    assert sets[1].size == 0 and g.num_edges(1) == 0
    for t in (0, 1, 2, 1, 0):
        v = stg.stg_dtdg_get_snapshot(g, t)
        assert_graph_equal(stg.view_arrays(v), oracle.csr(V, sets[t]), tag=("empty walk", t))
    v = stg.stg_dtdg_get_backward_snapshot(g, 1)
    assert_graph_equal(stg.view_arrays(v), oracle.csr(V, sets[1]), tag="empty bwd")
    # aggregation over the empty snapshot: every row has degree 0 -> norm 0 -> y = 0
    x = to_gpu(gen.uniform_pm1(1, 80, V * 64).reshape(V, 64))
    assert torch.count_nonzero(stg.stg_gcn_aggregate_fwd(v, x)) == 0
    assert torch.count_nonzero(stg.stg_gcn_aggregate_bwd(v, x)) == 0
    # a TGCN step on it: Â = 0, so C = b and the GRU sees only the bias (oracle)
    F, H = 8, 32
    p = gen.tgcn_params(F, H, 2)
    pg = {k: torch.from_numpy(val).cuda() for k, val in p.items()}
    X = gen.uniform_pm1(2, 81, V * F).reshape(V, F)
    Hp = gen.uniform_pm1(2, 82, V * H).reshape(V, H)
    Hn = stg.stg_tgcn_step(stg.stg_dtdg_get_snapshot(g, 1), pg, torch.from_numpy(X).cuda(),
                           torch.from_numpy(Hp).cuda())
    ref = oracle.tgcn_fwd(oracle.csr(V, sets[1]), p, X, Hp)
    assert np.max(np.abs(Hn.cpu().numpy() - ref["Hn"])) <= 2e-5


def test_single_vertex_graph(stg):
    g = stg.stg_static_graph_create(1, [0], [0], stg.STG_EDGE_IDS)
    ref = oracle.static_graph(1, [0], [0])
    assert_graph_equal(stg.view_arrays(g.view()), ref, tag="V=1")
    x = to_gpu(np.array([[1.0, -2.0, 3.0, 0.5]], np.float32))
    y = stg.stg_gcn_aggregate_fwd(g.view(), x)
    assert torch.equal(y, x)                                  # Â = [1]: y = x exactly
    F, H = 4, 16
    p = gen.tgcn_params(F, H, 9)
    pg = {k: torch.from_numpy(val).cuda() for k, val in p.items()}
    X = gen.uniform_pm1(9, 83, F).reshape(1, F)
    Hp = gen.uniform_pm1(9, 84, H).reshape(1, H)
    Hn = stg.stg_tgcn_step(g.view(), pg, torch.from_numpy(X).cuda(), torch.from_numpy(Hp).cuda())
    assert np.max(np.abs(Hn.cpu().numpy() - oracle.tgcn_fwd(ref, p, X, Hp)["Hn"])) <= 2e-5


def test_size_limits_rejected(stg):
    lib = stg._lib
    out = ctypes.c_void_p()
    dummy = ctypes.c_void_p(16)
    st = lib.stg_static_graph_create(1000, 1 << 31, dummy, dummy, 0, None, None, ctypes.byref(out))
    assert st == 2 and not out.value                          # STG_ERR_OUT_OF_RANGE
    st = lib.stg_static_graph_create(1 << 30, 10, dummy, dummy, 0, None, None, ctypes.byref(out))
    assert st == 2
    st = lib.stg_static_graph_create((1 << 31) - 2, (1 << 31) - 1 - 10, dummy, dummy, stg.STG_SELF_LOOPS, None,
                                     None, ctypes.byref(out))
    assert st == 2


def test_two_streams_on_one_graph(stg):
    """Aggregations of one graph on two streams at once (per-stream
    scratch): every result equals the single-stream result bit for bit."""
    cfg = gen.CONFIGS["C4"]
    d = gen.dtdg(cfg)
    g = stg.stg_dtdg_create(d.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src,
                            d.del_dst, stg.STG_SELF_LOOPS)
    v = stg.stg_dtdg_get_snapshot(g, 1)
    torch.cuda.synchronize()
    xs = [to_gpu(gen.uniform_pm1(5 + i, 7, cfg.V * 96).reshape(cfg.V, 96)) for i in range(2)]
    want = [stg.stg_gcn_aggregate_fwd(v, x).clone() for x in xs]
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    outs = [[torch.empty(cfg.V, 96, device="cuda") for _ in range(8)] for _ in range(2)]
    for k in range(8):
        for i in range(2):
            with torch.cuda.stream(streams[i]):
                stg.stg_gcn_aggregate_fwd(v, xs[i], outs[i][k], stream=streams[i])
    torch.cuda.synchronize()
    for i in range(2):
        for k in range(8):
            assert torch.equal(outs[i][k], want[i]), (i, k)


def test_wrong_dtype_rejected(stg):
    """float64 / int64 tensors are refused at the binding (they would reach the
    fp32 / int32 kernels as raw bytes)."""
    cfg = gen.CONFIGS["C2"]
    s, d = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s, d, stg.STG_SELF_LOOPS)
    x = torch.zeros(cfg.V, 8, dtype=torch.float64, device="cuda")
    with pytest.raises(stg.StgError) as e:
        stg.stg_gcn_aggregate_fwd(g.view(), x)
    assert e.value.status == 1


def test_torch_allocator_hook(stg):
    """Library-owned buffers come from torch's caching allocator (stg_set_allocator,
    installed by the binding): creating objects calls the hook and shows up in
    torch's memory statistics; destroying them returns every block."""
    import gc
    if os.environ.get("STG_TORCH_ALLOCATOR", "1") == "0":
        pytest.skip("allocator hook disabled by the environment")
    torch.cuda.synchronize()
    s0 = stg.allocator_stats()
    m0 = torch.cuda.memory_allocated()
    cfg = gen.CONFIGS["C4"]
    d = gen.dtdg(cfg)
    g = stg.stg_dtdg_create(d.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src,
                            d.del_dst, stg.STG_SELF_LOOPS)
    stack = stg.stg_state_stack_create(64 << 20)
    v = stg.stg_dtdg_get_snapshot(g, 2)
    x = to_gpu(gen.uniform_pm1(1, 2, cfg.V * 96).reshape(cfg.V, 96))
    y = stg.stg_gcn_aggregate_fwd(v, x)
    torch.cuda.synchronize()
    s1 = stg.allocator_stats()
    assert s1["alloc"] > s0["alloc"]
    assert torch.cuda.memory_allocated() - m0 >= (64 << 20)       # at least the state stack arena
    ref = oracle.csr(d.V, oracle.snapshot_set_window(d, 2, self_loops=True))
    want = oracle.aggregate_fwd(ref, x.cpu().numpy().astype(np.float64))
    assert np.max(np.abs(y.cpu().numpy() - want) / np.maximum(oracle.aggregate_scale(ref, x.cpu().numpy()), 1e-300)) <= 1e-5
    live = (s1["alloc"] - s0["alloc"]) - (s1["free"] - s0["free"])     # blocks held (grown buffers were freed)
    del v, stack, g
    gc.collect()
    torch.cuda.synchronize()
    s2 = stg.allocator_stats()
    assert s2["free"] - s1["free"] >= live
