"""Write profiles/agg_traffic.json and profiles/tensor_pipe.json (read by bench.py) from an
ncu_extract.py summary of the round's `ncu --set full` captures (scripts/ncu_capture.sh).
usage: python scripts/ncu_summaries.py profiles/r02_ncu_full_vNN_kernels.json"""
import json
import re
import sys


def num(v):
    """'2.318112 Gbyte' -> bytes / '415.8 us' -> value in the unit's base (us kept as us)."""
    x, u = (v.split() + [""])[:2]
    x = float(x.replace(",", ""))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "us": 1, "ms": 1e3, "ns": 1e-3, "%": 1}
    return x * scale.get(u, 1)


def short(name):
    n = re.sub(r"^.*::(k_[A-Za-z0-9_]+)", r"\1", name.split("(")[0])
    n = re.sub(r"unnamed>::", "", n)
    return n.replace("(int)", "").replace("(bool)", "")


src = sys.argv[1]
d = json.load(open(src))
tp = {"source": "%s (ncu --set full --clock-control none, one launch per kernel: scripts/ncu_capture.sh + "
                "scripts/ncu_extract.py; C5, TGCN H = 32, F = 64)" % src,
      "metric": "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
      "note": "3xTF32 on tcgen05 (three kind::tf32 MMAs per product); the kernels are HBM/latency-bound, so the "
              "tensor pipe is idle most of the time by design: the contraction widths are K <= 128, N <= 128",
      "kernels": {}}
agg = None
for rep, v in d.items():
    k = short(v["Kernel Name"])
    if k.startswith("k_tc_"):
        key = k
        while key in tp["kernels"]:
            key += "'"
        tp["kernels"][key] = {
            "tensor_pipe_pct": num(v["sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"]),
            "duration_us": num(v["gpu__time_duration.sum"]),
            "dram_bytes": num(v["dram__bytes_read.sum"]) + num(v["dram__bytes_write.sum"]),
            "dram_pct_of_peak": num(v["gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]),
            "warps_active_pct": num(v["sm__warps_active.avg.pct_of_peak_sustained_active"])}
    if k.startswith("k_agg_stream") and agg is None:
        r, w = num(v["dram__bytes_read.sum"]), num(v["dram__bytes_write.sum"])
        agg = {"kernel": v["Kernel Name"], "bytes_per_launch": r + w, "dram_read_bytes": r, "dram_write_bytes": w,
               "l2_read_hit_pct": num(v["lts__t_sector_op_read_hit_rate.pct"]),
               "duration_us": num(v["gpu__time_duration.sum"]),
               "source": "%s (k_agg_stream, ncu --set full, C5 W=96 forward)" % src,
               "config": "C5 forward aggregation W=96 (TGCN C = A P'), edge stream, 4 rows in flight, light-row tiers"}
json.dump(tp, open("profiles/tensor_pipe.json", "w"), indent=1)
if agg:
    json.dump(agg, open("profiles/agg_traffic.json", "w"), indent=1)
print("kernels:", list(tp["kernels"]), "agg:", bool(agg))
