"""Per-step cost of the DTDG snapshot update on C5 (Get-Graph forward walk of the
in-CSR, Get-Backward-Graph reverse walk of the out-CSR), CUDA events around each
step on one stream; PROBE_NCU=1 runs 2 + 2 steps only (for an ncu launch list)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

NCU = os.environ.get("PROBE_NCU") == "1"
cfg = gen.CONFIGS["C5"]
d = gen.dtdg(cfg)
g = stg.stg_dtdg_create(cfg.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src, d.del_dst,
                        stg.STG_SELF_LOOPS | stg.STG_EDGE_IDS)
for name, s in (("default", torch.cuda.current_stream()), ("side", torch.cuda.Stream())):
    with torch.cuda.stream(s):
        stg.stg_dtdg_get_snapshot_parts(g, 0, stg.STG_PART_IN, stream=s)
        torch.cuda.synchronize()
        n = 2 if NCU else 12
        rec = {"stream": name, "fwd_ms": [], "bwd_ms": []}
        for t in range(1, 1 + n):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            stg.stg_dtdg_get_snapshot_parts(g, t, stg.STG_PART_IN, stream=s)
            e1.record(s)
            torch.cuda.synchronize()
            rec["fwd_ms"].append(round(e0.elapsed_time(e1), 4))
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        stg.stg_dtdg_get_snapshot_parts(g, n, stg.STG_PART_OUT, backward=True, stream=s)    # transpose
        e1.record(s)
        torch.cuda.synchronize()
        rec["transpose_ms"] = round(e0.elapsed_time(e1), 4)
        for t in range(n - 1, 0, -1):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            stg.stg_dtdg_get_snapshot_parts(g, t, stg.STG_PART_OUT, backward=True, stream=s)
            e1.record(s)
            torch.cuda.synchronize()
            rec["bwd_ms"].append(round(e0.elapsed_time(e1), 4))
        print(json.dumps(rec), flush=True)
