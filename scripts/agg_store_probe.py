"""Does the output stream evict the hot source rows?  The C5 in-CSR gather of
scripts/agg_locality_probe.cu (W = 96) with four output-store variants
(0 none, 1 st.global.cs, 2 st.global + L2 evict_first policy, 3 plain st.global),
timed with CUDA events; PROBE_NCU=1 launches each once for ncu (DRAM bytes, L2
hit rate).  One JSON line per variant."""
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
lib.probe_store_run.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64,
                                ctypes.c_int64, ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
NCU = os.environ.get("PROBE_NCU") == "1"
cfg = gen.CONFIGS["C5"]
d = gen.dtdg(cfg)
g = stg.stg_dtdg_create(cfg.V, d.T, d.src0, d.dst0, d.add_off, d.add_src, d.add_dst, d.del_off, d.del_src, d.del_dst,
                        stg.STG_SELF_LOOPS)
arr = stg.view_arrays(stg.stg_dtdg_get_snapshot(g, 1))
V, W = cfg.V, 96
col = arr["in_col"].contiguous()
row = arr["in_row"].contiguous()
E = col.numel()
uni = torch.randint(0, V, (E,), device="cuda", dtype=torch.int32)
srt = torch.sort(col)[0].to(torch.int32).contiguous()
x = torch.rand(V, W, device="cuda")
y = torch.empty(V, W, device="cuda")
s = torch.cuda.Stream()
for name, idx in (("c5_col", col), ("uniform", uni), ("sorted", srt)):
    for store in (0, 1, 2, 3):
        def run():
            assert lib.probe_store_run(store, x.data_ptr(), idx.data_ptr(), row.data_ptr(), E, 512, y.data_ptr(),
                                       148 * 8, ctypes.c_void_p(s.cuda_stream)) == 0
        with torch.cuda.stream(s):
            run()
            if NCU:
                torch.cuda.synchronize()
                print(json.dumps({"idx": name, "store": store}), flush=True)
                continue
            run()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(10):
                run()
            e1.record(s)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 10
        print(json.dumps({"idx": name, "store": store, "ms": round(ms, 4)}), flush=True)
