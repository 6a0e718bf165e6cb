"""Locality probe for the C5 aggregation (scripts/agg_locality_probe.cu): time
each (layout, hint, K) variant of the aggregation memory pattern with CUDA
events; with PROBE_NCU=1 launch each variant once (for an ncu --metrics pass).

Prints one JSON line per variant."""
import ctypes
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

so = os.path.join(ROOT, "scripts", "libagg_locality_probe.so")
subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-shared", "-Xcompiler", "-fPIC",
                       "-o", so, os.path.join(ROOT, "scripts", "agg_locality_probe.cu")])
lib = ctypes.CDLL(so)
lib.probe_run.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                          ctypes.c_int64, ctypes.c_int32, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int,
                          ctypes.c_void_p]
lib.set_persist.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_float, ctypes.c_size_t]
NCU = os.environ.get("PROBE_NCU") == "1"

cfg = gen.CONFIGS["C5"]
d = gen.dtdg(cfg)
g = stg.stg_dtdg_create(cfg.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src, d.del_dst,
                        stg.STG_SELF_LOOPS)
arr = stg.view_arrays(stg.stg_dtdg_get_snapshot(g, 1))
V, W = cfg.V, 96
col = arr["in_col"].contiguous()
row = arr["in_row"].contiguous()
out_ids = arr["out_ids"].long()
rank = torch.empty(V, dtype=torch.int64, device="cuda")
rank[out_ids] = torch.arange(V, device="cuda")
colr = rank[col.long()].to(torch.int32).contiguous()
E = col.numel()
x = torch.rand(V, W, device="cuda")
y = torch.empty(V, W, device="cuda")
s = torch.cuda.Stream()
blocks = 148 * 8
CH = 512


def run(idx, hint, D, K):
    assert lib.probe_run(hint, D, x.data_ptr(), idx.data_ptr(), row.data_ptr(), E, K, CH, y.data_ptr(), blocks,
                         ctypes.c_void_p(s.cuda_stream)) == 0


variants = [("plain", col, 0, 0, 0), ("relabel", colr, 0, 0, 0)]
for K in (65536, 131072, 196608, 262144, 327680):
    for hint in (1, 2, 3, 4):
        variants.append(("relabel", colr, hint, K, 0))
for win in (48, 64, 80):
    variants.append(("relabel", colr, 0, 0, win))
alg = 4 * E + 8 * V * W
for name, idx, hint, K, win in variants:
    rc = lib.set_persist(ctypes.c_void_p(s.cuda_stream), ctypes.c_void_p(x.data_ptr()), win << 20, 1.0,
                         min(win << 20, 80 << 20))
    for D in ((4,) if NCU else (4, 8)):
        with torch.cuda.stream(s):
            if NCU:
                run(idx, hint, D, K)
                torch.cuda.synchronize()
                print(json.dumps({"idx": name, "hint": hint, "K": K, "win_MB": win, "D": D}), flush=True)
                continue
            run(idx, hint, D, K)
            run(idx, hint, D, K)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(10):
                run(idx, hint, D, K)
            e1.record(s)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 10
        print(json.dumps({"idx": name, "hint": hint, "K": K, "win_MB": win, "persist_rc": rc, "D": D,
                          "ms": round(ms, 4), "compulsory_GBps": round(alg / ms / 1e6, 1),
                          "gather_GBps": round(E * 384 / ms / 1e6, 1)}), flush=True)
lib.set_persist(ctypes.c_void_p(s.cuda_stream), ctypes.c_void_p(x.data_ptr()), 0, 1.0, 0)
