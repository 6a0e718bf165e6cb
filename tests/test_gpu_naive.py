"""NaiveGraph mode (STG_NAIVE; every snapshot stored,
the baseline the paper's GPMA/on-demand design is measured against in Table III).
Every materialised snapshot must equal the oracle snapshot bit for bit (CSRs,
degrees, node_ids, labels) and the on-demand views; a training sequence must give
bit-identical results either way; the memory accounting must show the trade-off."""
import numpy as np
import pytest
import torch

import gen
import oracle
from helpers import assert_graph_equal

pytestmark = pytest.mark.gpu

FLAGS = None


def _create(stg, dd, naive):
    flags = stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS | (stg.STG_NAIVE if naive else 0)
    return stg.stg_dtdg_create(dd.V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off,
                               dd.del_src, dd.del_dst, flags)


@pytest.mark.parametrize("name", ["C5s", "C4"])
def test_naive_snapshots_equal_oracle_and_on_demand(stg, name):
    dd = gen.dtdg(gen.CONFIGS[name])
    gn, go = _create(stg, dd, True), _create(stg, dd, False)
    sets = list(oracle.snapshot_sets_fold(dd, self_loops=True))
    order = list(range(dd.T)) + list(range(dd.T - 2, -1, -1))
    for i, t in enumerate(order):
        bwd = i >= dd.T
        vn = stg.stg_dtdg_get_backward_snapshot(gn, t) if bwd else stg.stg_dtdg_get_snapshot(gn, t)
        an = stg.view_arrays(vn)
        assert vn.timestamp == t and vn.num_edges == sets[t].size
        assert_graph_equal(an, oracle.csr(dd.V, sets[t]), tag=(name, t, bwd))
        vo = stg.stg_dtdg_get_backward_snapshot(go, t) if bwd else stg.stg_dtdg_get_snapshot(go, t)
        ao = stg.view_arrays(vo)
        for k in an:
            assert torch.equal(an[k], ao[k]), (name, t, k)


def test_naive_memory_accounting(stg):
    dd = gen.dtdg(gen.CONFIGS["C5s"])
    gn, go = _create(stg, dd, True), _create(stg, dd, False)
    mn, mo = gn.memory(), go.memory()
    assert mo["materialised"] == 0 and mn["materialised"] > 0
    assert mn["deltas"] == mo["deltas"] and mo["deltas"] > 0
    # every materialised snapshot holds at least its 4 edge arrays + labels (5 int32 per edge)
    assert mn["materialised"] >= sum(20 * gn.num_edges(t) for t in range(dd.T))
    # the trade-off of Table III: T snapshots cost far more than base + deltas + cache
    assert mn["materialised"] > 2 * (mo["deltas"] + mo["cache"])


def test_naive_training_sequence_identical(stg):
    cfg = gen.CONFIGS["C5s"]
    dd = gen.dtdg(cfg)
    V, F, H, S = cfg.V, cfg.F, cfg.H, 4
    p = {k: torch.from_numpy(v).cuda() for k, v in gen.tgcn_params(F, H, 1).items()}
    Xs = [torch.from_numpy(gen.features(cfg, t)).cuda() for t in range(S)]
    Ys = [torch.from_numpy(gen.labels(cfg, t)).cuda() for t in range(S)]
    out = []
    for naive in (False, True):
        g = _create(stg, dd, naive)
        grads = {"W": torch.zeros(F, 3 * H, device="cuda"), "b": torch.zeros(3 * H, device="cuda"),
                 "L": torch.zeros(3, 2 * H, H, device="cuda"), "l": torch.zeros(3, H, device="cuda")}
        dw, db, loss = torch.zeros(H, device="cuda"), torch.zeros(1, device="cuda"), torch.zeros(1, device="cuda")
        Hs = torch.empty(S, V, H, device="cuda")
        st = stg.stg_state_stack_create(S * V * 3 * H * 4 + (1 << 20))
        stg.stg_tgcn_train_sequence(g, 0, S, p, p["w_o"], p["b_o"], Xs, Ys, torch.zeros(V, H, device="cuda"), Hs,
                                    torch.empty(2, V, H, device="cuda"), grads, dw, db, loss, st)
        torch.cuda.synchronize()
        out.append((loss.clone(), Hs.clone(), {k: v.clone() for k, v in grads.items()}))
    assert torch.equal(out[0][0], out[1][0])
    assert torch.equal(out[0][1], out[1][1])
    for k in out[0][2]:
        assert torch.equal(out[0][2][k], out[1][2][k]), k


def test_naive_rejects_sharding(stg):
    dd = gen.dtdg(gen.CONFIGS["C5s"])
    with pytest.raises(stg.StgError):
        stg.stg_dtdg_create(dd.V, dd.T, dd.src0, dd.dst0, dd.add_off, dd.add_src, dd.add_dst, dd.del_off,
                            dd.del_src, dd.del_dst, stg.STG_SELF_LOOPS | stg.STG_NAIVE, dist=(0, 2, 0, dd.V // 2))
