"""Key metrics of ncu --set full reports -> JSON (one object per report) for profiles/."""
import csv
import glob
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "lts__t_sector_op_read_hit_rate.pct", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum",
        "l1tex__throughput.avg.pct_of_peak_sustained_active", "lts__throughput.avg.pct_of_peak_sustained_elapsed"]
out = {}
for rep in sorted(glob.glob(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/ncu_*.ncu-rep")):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    if len(rows) < 3:
        continue
    h, u = rows[0], rows[1]
    for n, v in enumerate(rows[2:]):
        d = {"Kernel Name": v[h.index("Kernel Name")]}
        for k in KEYS:
            if k in h:
                d[k] = (v[h.index(k)] + " " + u[h.index(k)]).strip()
        stalls = sorted(((h[i], float(v[i].replace(",", "") or 0)) for i in range(len(h))
                         if "pcsamp_warps_issue_stalled" in h[i] and not h[i].endswith("not_issued")),
                        key=lambda x: -x[1])
        d["top_stalls"] = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): x for k, x in stalls[:5]}
        out[rep.split("/")[-1] + ("" if n == 0 else "#%d" % n)] = d
print(json.dumps(out, indent=1))
