"""Summarise the steady-state part of scripts/seq_launches.sh (launches after the warm-up sequence)."""
import collections
import csv
import re
import sys

csv_path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/launches_seq.csv"
log_path = sys.argv[2] if len(sys.argv) > 2 else "gpurun_out/ncu10.log"
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
rows = list(csv.reader(open(csv_path)))
hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
hdr = rows[hi]
ki, vi, ui, idi = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit"), hdr.index("ID")
warm = int(re.search(r"warm-up launches: (\d+)", open(log_path, errors="ignore").read()).group(1))
agg = collections.defaultdict(lambda: [0.0, 0])
for r in rows[hi + 1:]:
    if len(r) <= vi or int(r[idi]) < warm:
        continue
    name = re.sub(r"^.*::", "", re.sub(r"\(.*", "", r[ki]))[:60]
    sc = {"ns": 1e-3, "nsecond": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(r[ui].strip().lower(), 1e-3)
    agg[name][0] += float(r[vi].replace(",", "")) * sc
    agg[name][1] += 1
T = sum(t for t, _ in agg.values())
print("total %.1f us over %d launches (one steady-state 4-step sequence; ncu serialised, cold cache)"
      % (T, sum(c for _, c in agg.values())))
for k, (t, c) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    print("%-60s %9.1f us %5d  avg %8.2f us %5.1f%%" % (k, t, c, t / c, 100 * t / T))
