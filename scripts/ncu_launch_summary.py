"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): time per kernel."""
import collections
import csv
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
agg = collections.defaultdict(lambda: [0, 0.0])
scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}
for r in rows[hdr + 1:]:
    if len(r) <= vi:
        continue
    v = float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
    name = re.sub(r"^void ", "", r[ki])
    name = re.sub(r"\(.*$", "", name)
    name = re.sub(r"stg::(\(anonymous namespace\)::)?", "", name)
    agg[name][0] += 1
    agg[name][1] += v
tot = sum(v[1] for v in agg.values())
print(f"{'kernel':60s} {'launches':>8s} {'ms':>9s} {'share':>6s}")
for k, v in sorted(agg.items(), key=lambda x: -x[1][1])[: int(sys.argv[2]) if len(sys.argv) > 2 else 30]:
    print(f"{k[:60]:60s} {v[0]:8d} {v[1] / 1e3:9.3f} {100 * v[1] / tot:5.1f}%")
print(f"total {tot / 1e3:.3f} ms over {sum(v[0] for v in agg.values())} launches")
