"""L2 persistence probe (scripts/gather_bench.cu gather_run_stream/set_persist):
the C5 in-CSR gather (W = 96 fp32 rows) with source rows relabelled in
out-degree-descending order (hot rows contiguous at the front of x) and a
persisting access-policy window over the first `win` MB."""
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_cherianmcc24_b200 as stg  # noqa: E402

lib = ctypes.CDLL(os.path.join(ROOT, "scripts", "libgather_bench.so"))
lib.gather_run_stream.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
                                  ctypes.c_int, ctypes.c_void_p]
lib.set_persist.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_float, ctypes.c_size_t]
lib.max_persist.restype = ctypes.c_size_t
mp = lib.max_persist()
print(json.dumps({"max_persisting_l2": mp >> 32, "max_window": mp & 0xffffffff}), flush=True)
V, W = 1 << 20, 96
x = torch.rand(V, W, device="cuda")
cfg = gen.CONFIGS["C5"]
d = gen.dtdg(cfg)
g = stg.stg_dtdg_create(cfg.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src, d.del_dst,
                        stg.STG_SELF_LOOPS)
arr = stg.view_arrays(stg.stg_dtdg_get_snapshot(g, 1))
col = arr["in_col"].contiguous()
out_ids = arr["out_ids"].long()
rank = torch.empty(V, dtype=torch.int64, device="cuda")
rank[out_ids] = torch.arange(V, device="cuda")
colr = rank[col.long()].to(torch.int32).contiguous()
E = col.numel()
out = torch.empty(148 * 16 * 256 * 4, device="cuda")
s = torch.cuda.Stream()
for name, idx in (("plain", col), ("relabel", colr)):
    for win_mb in (0, 16, 32, 48, 64, 80, 96):
        if name == "plain" and win_mb not in (0, 64):
            continue
        for hr in ((1.0,) if win_mb == 0 else (1.0, 0.75)):
            win = win_mb << 20
            rc = lib.set_persist(ctypes.c_void_p(s.cuda_stream), ctypes.c_void_p(x.data_ptr()), win, hr,
                                 min(win, mp >> 32))
            for D in (4, 8):
                def run():
                    assert lib.gather_run_stream(D, x.data_ptr(), idx.data_ptr(), E, out.data_ptr(), 148 * 8,
                                                 ctypes.c_void_p(s.cuda_stream)) == 0
                with torch.cuda.stream(s):
                    run()
                    run()
                    torch.cuda.synchronize()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(s)
                    for _ in range(10):
                        run()
                    e1.record(s)
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1) / 10
                print(json.dumps({"idx": name, "win_MB": win_mb, "hit_ratio": hr, "set_rc": rc, "D": D,
                                  "ms": round(ms, 4), "gather_GBps": round(E * 384 / ms / 1e6, 1)}), flush=True)
lib.set_persist(ctypes.c_void_p(s.cuda_stream), ctypes.c_void_p(x.data_ptr()), 0, 1.0, 0)
