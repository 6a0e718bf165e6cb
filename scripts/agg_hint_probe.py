"""(Needs libstg at commit 63db492, where k_agg_stream had the HINT variants; the hints
were measured slower and removed.)  Source-row cache hints in the edge-stream aggregation (k_agg_stream,
stg_aggregate_set_param keys 3/4) on the C5 snapshot at W = 96: the view's column
ids are replaced by hot-first labels (the rank of the source in out-degree order
for the forward, in in-degree order for the backward), so rows u < hotk are the
hottest sources.  Times fwd and bwd per (hint, hotk) with CUDA events; with
PROBE_NCU=1 launches each variant once for an ncu --metrics pass.  One JSON line
per variant.  (The values are not checked: only the memory pattern matters.)"""
import ctypes
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
v = stg.stg_dtdg_get_snapshot(g, 2)
arr = stg.view_arrays(v)
V, W = cfg.V, 96


def relabel(col, ids):
    rank = torch.empty(V, dtype=torch.int64, device="cuda")
    rank[ids.long()] = torch.arange(V, device="cuda")
    return rank[col.long()].to(torch.int32).contiguous()


colf = relabel(arr["in_col"], arr["out_ids"])
colb = relabel(arr["out_col"], arr["in_ids"])
vr = stg.stg_csr_view()
ctypes.memmove(ctypes.addressof(vr), ctypes.addressof(v), ctypes.sizeof(v))
vr.in_col = colf.data_ptr()
vr.out_col = colb.data_ptr()
x = torch.rand(V, W, device="cuda")
y = torch.empty(V, W, device="cuda")
E = v.num_edges
alg = 4 * E + 4 * (V + 1) + 8 * V + 8 * V * W


def timed(view, bwd):
    f = stg.stg_gcn_aggregate_bwd if bwd else stg.stg_gcn_aggregate_fwd
    if NCU:
        f(view, x, y)
        torch.cuda.synchronize()
        return None
    for _ in range(3):
        f(view, x, y)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        f(view, x, y)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / 20


variants = [("orig", 0, 0), ("relabel", 0, 0)]
for hotk in (65536, 131072, 262144, 393216):
    for hint in (1, 2, 3, 4):
        variants.append(("relabel", hint, hotk))
for name, hint, hotk in variants:
    stg.stg_aggregate_set_param(3, hint)
    stg.stg_aggregate_set_param(4, hotk)
    view = v if name == "orig" else vr
    for bwd in (False, True):
        ms = timed(view, bwd)
        rec = {"view": name, "hint": hint, "hotk": hotk, "dir": "bwd" if bwd else "fwd"}
        if ms is not None:
            rec.update(ms=round(ms, 4), frac_compulsory=round(alg / ms / 1e6 / 6535.4, 3))
        print(json.dumps(rec), flush=True)
stg.stg_aggregate_set_param(3, 0)
stg.stg_aggregate_set_param(4, 0)
