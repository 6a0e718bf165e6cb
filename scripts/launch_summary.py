"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV) per kernel."""
import collections
import csv
import re
import sys


def main(path, top=40):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[hi]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = collections.defaultdict(lambda: [0.0, 0])
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        name = re.sub(r"\(.*", "", r[ki])
        name = re.sub(r"^.*::", "", name)[:70]
        v = float(r[vi].replace(",", ""))
        u = r[ui].strip().lower()
        scale = {"ns": 1e-3, "nsecond": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(u, 1e-3)
        agg[name][0] += v * scale
        agg[name][1] += 1
    tot = sum(t for t, _ in agg.values())
    print("total %.1f us over %d launches" % (tot, sum(c for _, c in agg.values())))
    for k, (t, c) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
        print("%-70s %11.1f us %6d  avg %9.2f us  %5.1f%%" % (k, t, c, t / c, 100 * t / tot))


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40)
