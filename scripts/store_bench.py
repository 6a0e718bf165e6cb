"""Store-pattern ceiling for a thread-per-row epilogue (scripts/gather_bench.cu k_store)."""
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
import torch  # noqa: E402

lib = ctypes.CDLL(os.path.join(ROOT, "scripts", "libgather_bench.so"))
lib.store_run.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_int]
V = 1 << 20
y = torch.empty(V, 96, device="cuda")
for mode in (0, 1, 2):
    for blocks, threads in ((148, 128), (296, 128), (592, 128), (1184, 128), (2368, 128)):
        def run():
            assert lib.store_run(mode, y.data_ptr(), V, blocks, threads) == 0
        run()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(10):
            run()
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 10
        print(json.dumps({"mode": mode, "blocks": blocks, "threads": threads, "ms": round(ms, 4),
                          "GBps": round(V * 384 / ms / 1e6, 1)}), flush=True)
