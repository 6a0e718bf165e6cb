"""CUDA-event time of on-demand snapshot builds on C5: Get-Graph(t) of the in-CSR for
t = 1..T-1 (forward head walking up) and Get-Backward-Graph(t) of the out-CSR walking
back down (the two builds of every Algorithm-1 timestep).  One JSON line."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

cfg = gen.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C5"]
d = gen.dtdg(cfg)
g = stg.stg_dtdg_create(cfg.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src, d.del_dst,
                        stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
res = {}
for rep in range(2):
    e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    stg.stg_dtdg_get_snapshot_parts(g, 0, stg.STG_PART_IN)
    torch.cuda.synchronize()
    e0.record()
    for t in range(1, d.T):
        stg.stg_dtdg_get_snapshot_parts(g, t, stg.STG_PART_IN)
    e1.record()
    for t in range(d.T - 2, -1, -1):
        stg.stg_dtdg_get_snapshot_parts(g, t, stg.STG_PART_OUT, backward=True)
    e2.record()
    torch.cuda.synchronize()
    res = {"config": cfg.name, "T": d.T, "fwd_in_build_ms": e0.elapsed_time(e1) / (d.T - 1),
           "bwd_out_build_ms": e1.elapsed_time(e2) / (d.T - 1)}
print(json.dumps(res), flush=True)
