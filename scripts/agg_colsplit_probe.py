"""Probe: does splitting the W=96 aggregation into sequential column passes (each
pass's source working set is smaller, so more of it stays in L2) beat one pass?
CUDA-event time per full aggregation on a C5 snapshot; one JSON line per variant."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

cfg = gen.CONFIGS["C5"]
d = gen.dtdg(cfg)
g = stg.stg_dtdg_create(cfg.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src, d.del_dst,
                        stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
v = stg.stg_dtdg_get_snapshot(g, 1)
V, E, W = v.num_nodes, v.num_edges, 96
x = torch.rand(V, W, device="cuda") * 2 - 1
y = torch.empty(V, W, device="cuda")
ref = torch.empty(V, W, device="cuda")
flush = torch.empty(64 << 20, device="cuda")


def run(passes, bwd):
    if passes == 1:
        stg.stg_gcn_aggregate_ex(v, bwd, x, out=y)
        return
    wp = W // passes
    for k in range(passes):
        xs, ys = x[:, k * wp:(k + 1) * wp], y[:, k * wp:(k + 1) * wp]
        stg._check(stg._lib.stg_gcn_aggregate_ex(stg.ctypes.byref(v), bwd, wp, stg.ctypes.c_void_p(xs.data_ptr()),
                                                 W, stg.ctypes.c_void_p(ys.data_ptr()), W, None, None, None,
                                                 stg._stream(None)))


for bwd in (0, 1):
    run(1, bwd)
    ref.copy_(y)
    for passes in (1, 2, 3):
        for d_, mb in ((16, 3), (8, 4), (4, 6)):
            stg.stg_aggregate_set_param(0, d_)
            stg.stg_aggregate_set_param(1, mb)
            run(passes, bwd)
            torch.cuda.synchronize()
            ok = torch.equal(y, ref)
            ts = []
            for it in range(8):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                run(passes, bwd)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            ts.sort()
            print(json.dumps({"bwd": bwd, "passes": passes, "D": d_, "minb": mb, "ms_median": ts[len(ts) // 2],
                              "ms_min": ts[0], "bit_identical": ok}), flush=True)
    stg.stg_aggregate_set_param(0, 16)
    stg.stg_aggregate_set_param(1, 3)
