"""Aggregation time per launch width on the C5 snapshot: the edge-stream kernel
(strategy 2) against the pipelined row items (strategy 1) for W <= 64, chosen by
stg_aggregate_set_param(2, wmin) (stream serves W > wmin).  CUDA events, fwd and bwd;
one JSON line per (W, wmin, direction)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

cfg = gen.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C5"]
d = gen.dtdg(cfg)
g = stg.stg_dtdg_create(cfg.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src, d.del_dst,
                        stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
v = stg.stg_dtdg_get_snapshot(g, 2)
V, E = cfg.V, v.num_edges
for W in (16, 32, 48, 64, 96):
    x = torch.rand(V, W, device="cuda")
    y = torch.empty(V, W, device="cuda")
    for wmin in (64, 32, 16, 0):
        if wmin >= W and wmin != 64:
            continue
        stg.stg_aggregate_set_param(2, wmin)
        for bwd in (False, True):
            f = stg.stg_gcn_aggregate_bwd if bwd else stg.stg_gcn_aggregate_fwd
            for _ in range(3):
                f(v, x, y)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(20):
                f(v, x, y)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / 20
            print(json.dumps({"config": cfg.name, "W": W, "wmin": wmin, "kernel": "stream" if W > wmin else "items",
                              "dir": "bwd" if bwd else "fwd", "ms": round(ms, 4),
                              "edges_per_s": round(E / ms / 1e6, 1)}), flush=True)
stg.stg_aggregate_set_param(2, 0)
