"""Aggregation strategy / tunable sweep on one C5 snapshot (W = 96, the TGCN
width): CUDA-event time per launch (fwd over the in-CSR, bwd over the out-CSR),
compulsory-byte GB/s, and the max relative deviation from strategy 0.
Prints one JSON line per configuration."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5")
ap.add_argument("--W", type=int, default=96)
ap.add_argument("--iters", type=int, default=10)
ap.add_argument("--t", type=int, default=1)
ap.add_argument("--quick", action="store_true")
ap.add_argument("--only", default=None, help="run only configs whose name contains this (profiling)")
a = ap.parse_args()

cfg = gen.CONFIGS[a.config]
if cfg.kind == "static":
    s_e, d_e = gen.static_edges(cfg)
    g = stg.stg_static_graph_create(cfg.V, s_e, d_e, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    v = g.view()
else:
    d = gen.dtdg(cfg)
    g = stg.stg_dtdg_create(cfg.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src,
                            d.del_dst, stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
    v = stg.stg_dtdg_get_snapshot(g, a.t)
V, E, W = v.num_nodes, v.num_edges, a.W
torch.manual_seed(0)
x = torch.rand(V, W, device="cuda") * 2 - 1
alg = 4 * E + 4 * (V + 1) + 4 * V + 4 * V + 8 * V * W


def run(bwd):
    return stg.stg_gcn_aggregate_ex(v, bwd, x, out=ys[bwd], scale_row=None, scale_col=None)


ys = [torch.empty(V, W, device="cuda"), torch.empty(V, W, device="cuda")]


def timeit(bwd):
    for _ in range(2):
        run(bwd)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(a.iters):
        run(bwd)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / a.iters


stg.stg_aggregate_set_strategy(0)
ref = []
for bwd in (0, 1):
    run(bwd)
    ref.append(ys[bwd].clone())
scale = [r.abs().amax(dim=1, keepdim=True).clamp_min(1e-30) for r in ref]

configs = [("s0", 0, {}), ("s1", 1, {})]
for d, mb in ((4, 6), (8, 4), (16, 2), (16, 3)):
    configs.append(("s2 d%d minb%d" % (d, mb), 2, {0: d, 1: mb}))
configs.append(("s2 d16 minb3 wmin64", 2, {0: 16, 1: 3, 2: 64}))
defaults = {0: 4, 1: 6, 2: 32}
if a.only:
    configs = [c for c in configs if a.only in c[0]]
for name, strat, params in configs:
    stg.stg_aggregate_set_strategy(strat)
    for k, dv in defaults.items():
        stg.stg_aggregate_set_param(k, params.get(k, dv))
    res = {"name": name, "V": V, "E": E, "W": W}
    for bwd in (0, 1):
        ms = timeit(bwd)
        run(bwd)
        torch.cuda.synchronize()
        err = ((ys[bwd] - ref[bwd]).abs() / scale[bwd]).max().item()
        res["bwd" if bwd else "fwd"] = {"ms": round(ms, 4), "GBps_compulsory": round(alg / ms / 1e6, 1),
                                        "max_dev_vs_s0": err}
    print(json.dumps(res), flush=True)
stg.stg_aggregate_set_strategy(2)
for k, dv in defaults.items():
    stg.stg_aggregate_set_param(k, dv)
