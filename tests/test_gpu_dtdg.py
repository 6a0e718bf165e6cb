"""GPU parity: on-demand DTDG snapshots (Get-Graph / Get-Backward-Graph) are
bit-exact against the oracle's cumulative rebuild, in every access order."""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import assert_graph_equal, cond_err, to_gpu

pytestmark = pytest.mark.gpu


def _create(stg, d, flags):
    return stg.stg_dtdg_create(d.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src,
                               d.del_dst, flags)


def _oracle_snaps(d, loops):
    return [oracle.csr(d.V, S) for S in oracle.snapshot_sets_fold(d, self_loops=loops)]


@pytest.fixture(scope="module", params=["C4", "C5s"])
def dtdg_case(request, stg):
    d = gen.dtdg(gen.CONFIGS[request.param])
    refs = {loops: _oracle_snaps(d, loops) for loops in (False, True)}
    return request.param, d, refs


@pytest.mark.parametrize("loops", [False, True])
def test_forward_walk_bit_exact(stg, dtdg_case, loops):
    name, d, refs = dtdg_case
    flags = stg.STG_EDGE_IDS | (stg.STG_SELF_LOOPS if loops else 0)
    g = _create(stg, d, flags)
    assert g.T == d.T
    for t in range(d.T):
        assert g.num_edges(t) == refs[loops][t]["E"], t
    for t in range(d.T):
        v = stg.stg_dtdg_get_snapshot(g, t)
        assert v.timestamp == t
        assert_graph_equal(stg.view_arrays(v), refs[loops][t], tag=(name, "fwd", t))


@pytest.mark.parametrize("loops", [False, True])
def test_backward_walk_and_random_access(stg, dtdg_case, loops):
    name, d, refs = dtdg_case
    flags = stg.STG_EDGE_IDS | (stg.STG_SELF_LOOPS if loops else 0)
    g = _create(stg, d, flags)
    T = d.T
    # Algorithm 1 pattern: sequences of S forward, then backward in LIFO order
    S = 4
    for t0 in range(0, T, S):
        ts = list(range(t0, min(T, t0 + S)))
        for t in ts:
            assert_graph_equal(stg.view_arrays(stg.stg_dtdg_get_snapshot(g, t)), refs[loops][t], tag=(name, "f", t))
        for t in reversed(ts):
            v = stg.stg_dtdg_get_backward_snapshot(g, t)
            assert_graph_equal(stg.view_arrays(v), refs[loops][t], tag=(name, "b", t))
    # random access, both kinds
    rng = np.random.default_rng(0)
    for _ in range(12):
        t = int(rng.integers(0, T))
        f = stg.stg_dtdg_get_backward_snapshot if rng.integers(0, 2) else stg.stg_dtdg_get_snapshot
        assert_graph_equal(stg.view_arrays(f(g, t)), refs[loops][t], tag=(name, "r", t))
    # full backward walk from the end to 0
    stg.stg_dtdg_get_snapshot(g, T - 1)
    for t in reversed(range(T)):
        assert_graph_equal(stg.view_arrays(stg.stg_dtdg_get_backward_snapshot(g, t)), refs[loops][t],
                           tag=(name, "bw", t))


def test_snapshot_aggregation(stg, dtdg_case):
    name, d, refs = dtdg_case
    g = _create(stg, d, stg.STG_SELF_LOOPS)
    W = 64
    for t in (0, 1, d.T // 2, d.T - 1):
        v = stg.stg_dtdg_get_snapshot(g, t)
        x = gen.uniform_pm1(t, 77, d.V * W).reshape(d.V, W).astype(np.float64)
        y = stg.stg_gcn_aggregate_fwd(v, to_gpu(x)).cpu().numpy()
        ref = refs[True][t]
        assert cond_err(y, oracle.aggregate_fwd(ref, x), oracle.aggregate_scale(ref, x)) <= 1e-5
        vb = stg.stg_dtdg_get_backward_snapshot(g, t)
        gx = stg.stg_gcn_aggregate_bwd(vb, to_gpu(x)).cpu().numpy()
        assert cond_err(gx, oracle.aggregate_bwd(ref, x), oracle.aggregate_scale(ref, x, bwd=True)) <= 1e-5


def _noisy(seed, V=300, T=9):
    """Raw batches with duplicates, deletes of absent edges, add∩delete and loops."""
    rng = np.random.default_rng(seed)
    s0, d0 = rng.integers(0, V, 2000), rng.integers(0, V, 2000)
    A, D = [(np.zeros(0, int), np.zeros(0, int))], [(np.zeros(0, int), np.zeros(0, int))]
    for t in range(1, T):
        na, nd = int(rng.integers(0, 300)), int(rng.integers(0, 300))
        a = (rng.integers(0, V, na), rng.integers(0, V, na))
        dd = (rng.integers(0, V, nd), rng.integers(0, V, nd))
        if na > 10:   # add ∩ delete and duplicates
            dd = (np.concatenate([dd[0], a[0][:5]]), np.concatenate([dd[1], a[1][:5]]))
            a = (np.concatenate([a[0], a[0][:5]]), np.concatenate([a[1], a[1][:5]]))
        A.append(a); D.append(dd)
    off = lambda L: np.concatenate([[0], np.cumsum([x[0].size for x in L])]).astype(np.int64)
    cat = lambda L, i: np.concatenate([x[i] for x in L]).astype(np.int32)
    return gen.DTDG(V=V, T=T, W=0, slide=0, ev_src=None, ev_dst=None, src0=s0.astype(np.int32),
                    dst0=d0.astype(np.int32), add_off=off(A), add_src=cat(A, 0), add_dst=cat(A, 1),
                    del_off=off(D), del_src=cat(D, 0), del_dst=cat(D, 1))


@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("loops", [False, True])
def test_raw_batches_are_normalised(stg, seed, loops):
    d = _noisy(seed)
    refs = _oracle_snaps(d, loops)
    g = _create(stg, d, stg.STG_EDGE_IDS | (stg.STG_SELF_LOOPS if loops else 0))
    for t in range(d.T):
        assert_graph_equal(stg.view_arrays(stg.stg_dtdg_get_snapshot(g, t)), refs[t], tag=(seed, t))
    for t in reversed(range(d.T)):
        assert_graph_equal(stg.view_arrays(stg.stg_dtdg_get_backward_snapshot(g, t)), refs[t], tag=(seed, "b", t))
    # effective delta counts equal the oracle's normalisation
    S_prev = None
    for t, S in enumerate(oracle.snapshot_sets_fold(d, self_loops=loops)):
        if t:
            A, D = oracle.batch(d, t)
            a, dd = oracle.effective_deltas(S_prev, A, D, pinned_loops=loops)
            assert g.num_deltas(t, False) == a.size and g.num_deltas(t, True) == dd.size
        S_prev = S


def test_validate_rejects_ineffective_batches(stg):
    d = _noisy(1)
    with pytest.raises(stg.StgError) as e:
        _create(stg, d, stg.STG_VALIDATE)
    assert e.value.status == 1


def test_bad_arguments(stg):
    d = gen.dtdg(gen.CONFIGS["C5s"])
    g = _create(stg, d, 0)
    with pytest.raises(stg.StgError) as e:
        stg.stg_dtdg_get_snapshot(g, d.T)
    assert e.value.status == 2
    bad_off = d.add_off.copy()
    bad_off[1] = 1
    with pytest.raises(stg.StgError):
        stg.stg_dtdg_create(d.V, d.T, d.src0, d.dst0, bad_off, d.add_src, d.add_dst, d.del_off, d.del_src,
                            d.del_dst, 0)


def _check_parts(a, ref, parts, tag):
    """The directions in `parts` bit-exact; degrees (whole graph) and norms always."""
    V = ref["V"]
    if parts & 1:
        for k in ("in_rowptr", "in_col", "in_ids"):
            assert np.array_equal(a[k].cpu().numpy(), ref[k]), (tag, k)
        assert np.array_equal(a["in_row"].cpu().numpy(), np.repeat(np.arange(V), np.diff(ref["in_rowptr"]))), tag
    if parts & 2:
        for k in ("out_rowptr", "out_col", "out_ids"):
            assert np.array_equal(a[k].cpu().numpy(), ref[k]), (tag, k)
    if parts & 4:
        assert np.array_equal(a["out_eid"].cpu().numpy(), ref["out_eid"]), (tag, "out_eid")
    for k in ("in_deg", "out_deg"):
        assert np.array_equal(a[k].cpu().numpy(), ref[k]), (tag, k)
    for k in ("norm_src", "norm_dst"):
        np.testing.assert_allclose(a[k].cpu().numpy().astype(np.float64), ref[k], rtol=2.5e-7, atol=0,
                                   err_msg=str((tag, k)))


@pytest.mark.parametrize("loops", [False, True])
def test_snapshot_parts_and_transpose(stg, dtdg_case, loops):
    """Direction-only walks (the Algorithm-1 pattern of the TGCN driver: in-CSR forward,
    out-CSR backward from a transposed head), then full views at random t that force
    transposes in -> out and out -> in with labels."""
    name, d, refs = dtdg_case
    flags = stg.STG_EDGE_IDS | (stg.STG_SELF_LOOPS if loops else 0)
    g = _create(stg, d, flags)
    T, S = d.T, 5
    IN, OUT, EID = stg.STG_PART_IN, stg.STG_PART_OUT, stg.STG_PART_EID
    for t0 in range(0, T, S):
        ts = list(range(t0, min(T, t0 + S)))
        for t in ts:
            v = stg.stg_dtdg_get_snapshot_parts(g, t, IN)      # other parts may be present (e.g. the base)
            _check_parts(stg.view_arrays(v), refs[loops][t], IN, (name, "fin", t))
        for t in reversed(ts):
            v = stg.stg_dtdg_get_snapshot_parts(g, t, OUT, backward=True)
            _check_parts(stg.view_arrays(v), refs[loops][t], OUT, (name, "bout", t))
    rng = np.random.default_rng(3)
    for _ in range(12):
        t = int(rng.integers(0, T))
        bwd = bool(rng.integers(0, 2))
        parts = [IN, OUT, IN | OUT, IN | OUT | EID][int(rng.integers(0, 4))]
        v = stg.stg_dtdg_get_snapshot_parts(g, t, parts, backward=bwd)
        want = parts | ((IN | OUT) if parts & EID else 0)
        _check_parts(stg.view_arrays(v), refs[loops][t], want, (name, "rand", t, bwd, parts))
        full = stg.stg_dtdg_get_backward_snapshot(g, t) if bwd else stg.stg_dtdg_get_snapshot(g, t)
        assert_graph_equal(stg.view_arrays(full), refs[loops][t], tag=(name, "full", t, bwd))


def test_snapshot_parts_rejects_bad_mask(stg):
    d = gen.dtdg(gen.CONFIGS["C5s"])
    g = _create(stg, d, stg.STG_SELF_LOOPS)
    for bad in (0, 8, stg.STG_PART_IN | 16):
        with pytest.raises(stg.StgError) as e:
            stg.stg_dtdg_get_snapshot_parts(g, 1, bad)
        assert e.value.status == 1


def _merge_cases(seed=0, V=5000):
    """Batches aimed at the snapshot merge (snapshot.cu k_touch3 / k_merge3): a base of
    exactly 3 merge tiles (3·2048 unique edges), thousands of adds at ONE insertion point
    (a row gaining edges past its last one, the last row of the graph: adds at the very
    end), deletes at merge-tile boundaries and of whole rows, a step that empties the
    graph and one that refills it from nothing."""
    rng = np.random.default_rng(seed)
    flat = rng.choice(V * V, 3 * 2048, replace=False)
    s0, d0 = (flat // V).astype(np.int64), (flat % V).astype(np.int64)
    key0 = np.sort(d0 * V + s0)                 # in-CSR order (dst, src)
    A, D = [(np.zeros(0, int), np.zeros(0, int))], [(np.zeros(0, int), np.zeros(0, int))]
    # t=1: row 17 (in-CSR row = dst) gains 3000 sources > all of its current ones; the last
    # row V-1 gains 2500 (adds at the very end of the old CSR); 200 random adds
    A.append((np.concatenate([np.arange(V - 3000, V), np.arange(V - 2500, V), rng.integers(0, V, 200)]),
              np.concatenate([np.full(3000, 17), np.full(2500, V - 1), rng.integers(0, V, 200)])))
    D.append((np.zeros(0, int), np.zeros(0, int)))
    # t=2: delete the edges at old in-CSR positions 0, 2047, 2048, 4095, 4096 (tile boundaries, t=0
    # order is a superset here: pick them from the base keys) and all of row 17's new sources
    pick = key0[[0, 2047, 2048, 4095, 4096, 6143]]
    D.append((np.concatenate([pick % V, np.arange(V - 3000, V)]), np.concatenate([pick // V, np.full(3000, 17)])))
    A.append((rng.integers(0, V, 100), rng.integers(0, V, 100)))
    # t=3: delete everything that can exist (the oracle normalises absent deletes away)
    allk = np.unique(np.concatenate([key0, (A[1][1] * V + A[1][0]), (A[2][1] * V + A[2][0])]))
    D.append((allk % V, allk // V))
    A.append((np.zeros(0, int), np.zeros(0, int)))
    # t=4: refill from an empty graph; t=5: a mixed step
    A.append((rng.integers(0, V, 4000), rng.integers(0, V, 4000)))
    D.append((np.zeros(0, int), np.zeros(0, int)))
    A.append((rng.integers(0, V, 3000), rng.integers(0, V, 3000)))
    D.append((rng.integers(0, V, 3000), rng.integers(0, V, 3000)))
    off = lambda L: np.concatenate([[0], np.cumsum([x[0].size for x in L])]).astype(np.int64)
    cat = lambda L, i: np.concatenate([x[i] for x in L]).astype(np.int32)
    return gen.DTDG(V=V, T=len(A), W=0, slide=0, ev_src=None, ev_dst=None, src0=s0.astype(np.int32),
                    dst0=d0.astype(np.int32), add_off=off(A), add_src=cat(A, 0), add_dst=cat(A, 1),
                    del_off=off(D), del_src=cat(D, 0), del_dst=cat(D, 1))


@pytest.mark.parametrize("loops", [False, True])
def test_merge_edge_cases(stg, loops):
    d = _merge_cases()
    refs = _oracle_snaps(d, loops)
    assert refs[3]["E"] == (d.V if loops else 0)          # the emptied snapshot
    g = _create(stg, d, stg.STG_EDGE_IDS | (stg.STG_SELF_LOOPS if loops else 0))
    for t in range(d.T):
        assert_graph_equal(stg.view_arrays(stg.stg_dtdg_get_snapshot(g, t)), refs[t], tag=("merge", t))
    for t in reversed(range(d.T)):
        assert_graph_equal(stg.view_arrays(stg.stg_dtdg_get_backward_snapshot(g, t)), refs[t], tag=("merge", "b", t))
    IN, OUT = stg.STG_PART_IN, stg.STG_PART_OUT
    g2 = _create(stg, d, stg.STG_SELF_LOOPS if loops else 0)
    for t in range(d.T):
        _check_parts(stg.view_arrays(stg.stg_dtdg_get_snapshot_parts(g2, t, IN)), refs[t], IN, ("min", t))
    for t in reversed(range(d.T)):
        _check_parts(stg.view_arrays(stg.stg_dtdg_get_snapshot_parts(g2, t, OUT, backward=True)), refs[t], OUT,
                     ("mout", t))
