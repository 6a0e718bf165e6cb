"""Edge-weighted aggregation (NEXT-4) vs unweighted on a C5 snapshot: CUDA-event time
per launch, fwd (in-CSR, ew[j]) and bwd (out-CSR, ew[out_eid[j]]), W = 64 and 96.
Compulsory bytes add 4E for the weights (+4E for out_eid in the bwd)."""
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
V, E = v.num_nodes, v.num_edges
a = stg.view_arrays(v)
ew = torch.from_numpy(gen.edge_weights(1, E)).cuda()
norm = stg.stg_gcn_weighted_norm(v, ew)


def timeit(fn, iters=10):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(iters):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / iters


print(json.dumps({"weighted_norm_ms": timeit(lambda: stg.stg_gcn_weighted_norm(v, ew, norm)), "E": E}), flush=True)
for W in (64, 96):
    x = torch.rand(V, W, device="cuda") * 2 - 1
    y = torch.empty(V, W, device="cuda")
    for bwd in (0, 1):
        tu = timeit(lambda: stg.stg_gcn_aggregate_ex(v, bwd, x, out=y, scale_row=a["norm_dst"], scale_col=a["norm_src"]))
        tw = timeit(lambda: stg.stg_gcn_aggregate_weighted(v, bwd, ew, x, out=y, scale_row=norm, scale_col=norm))
        comp = 4 * E + 4 * (V + 1) + 4 * V + 4 * V + 8 * V * W + 4 * V     # + the column scale vector
        compw = comp + 4 * E + (4 * E if bwd else 0)
        print(json.dumps({"W": W, "bwd": bwd, "unweighted_ms": tu, "weighted_ms": tw,
                          "unweighted_GBps_compulsory": comp / tu / 1e6, "weighted_GBps_compulsory": compw / tw / 1e6}),
              flush=True)
