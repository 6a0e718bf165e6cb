"""Per-kernel summary of the steady-state sequence in a scripts/seq_launches.sh launch
list: launches after the warm-up sequence (from 40 launches before the 5th X·W)."""
import collections
import csv
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hi]
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
ks = [(re.sub(r"\(.*", "", r[ki]), float(r[vi].replace(",", ""))) for r in rows[hi + 1:] if len(r) > vi]
idx = [i for i, (b, c) in enumerate(ks) if "xw_pipe" in b]
start = idx[len(idx) // 2] - 40
agg = collections.defaultdict(lambda: [0.0, 0])
for b, c in ks[start:]:
    b = re.sub(r"^.*::", "", b)[:60]
    agg[b][0] += c / 1e3
    agg[b][1] += 1
tot = sum(v[0] for v in agg.values())
print("total %.1f us over %d launches" % (tot, sum(v[1] for v in agg.values())))
for k, v in sorted(agg.items(), key=lambda x: -x[1][0]):
    print("%-60s %9.1f us %4d  %5.1f%%" % (k, v[0], v[1], 100 * v[0] / tot))
