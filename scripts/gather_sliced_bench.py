"""Feature-sliced gather probe (scripts/gather_bench.cu k_gather_sliced): the C5
in-CSR column stream gathered in S passes of SW fp32 columns, slice-major
[S][V][SW] vs row-major [V][96].  GB/s = all gathered bytes (E x 384 B) / time."""
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
lib.gather_sliced_run.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64,
                                  ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int]
V, W = 1 << 20, 96
x = torch.rand(V * W, device="cuda")
cfg = gen.CONFIGS["C5"]
d = gen.dtdg(cfg)
g = stg.stg_dtdg_create(cfg.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src, d.del_dst,
                        stg.STG_SELF_LOOPS)
arr = stg.view_arrays(stg.stg_dtdg_get_snapshot(g, 1))
col = arr["in_col"].contiguous()
E = col.numel()
out = torch.empty(148 * 16 * 256 * 4, device="cuda")
for SW in (8, 16, 32):
    S = W // SW
    for sm in (1, 0):
        for D in (1, 2, 4, 8):
            if SW == 32 and D == 8:
                continue
            for bps in (4, 8):
                blocks = 148 * bps

                def run():
                    assert lib.gather_sliced_run(SW, D, x.data_ptr(), col.data_ptr(), E, V, S, sm, out.data_ptr(),
                                                 blocks) == 0
                run()
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                for _ in range(5):
                    run()
                e1.record()
                torch.cuda.synchronize()
                ms = e0.elapsed_time(e1) / 5
                print(json.dumps({"SW": SW, "passes": S, "slice_major": sm, "D": D, "blocks_per_sm": bps,
                                  "ms": round(ms, 4), "gather_GBps": round(E * 384 / ms / 1e6, 1)}), flush=True)
