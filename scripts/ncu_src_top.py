"""Top CUDA source lines / SASS lines by warp-stall samples from an ncu report captured with --import-source."""
import csv, subprocess, sys
rep, view = sys.argv[1], (sys.argv[2] if len(sys.argv) > 2 else "cuda")
n = int(sys.argv[3]) if len(sys.argv) > 3 else 20
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", view],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(txt.splitlines()))
data, h, fname = [], None, ""
for r in rows:
    if r and r[0] in ("File Name", "Kernel Name"):
        fname = r[1].split("/")[-1][:40]; h = None; continue
    if r and r[0] in ("Line No", "Address"):
        h = r if "Warp Stall Sampling (All Samples)" in r else None; continue
    if h and len(r) == len(h):
        i_s = h.index("Warp Stall Sampling (All Samples)")
        try:
            data.append((float(r[i_s] or 0), fname, r[0], r[1]))
        except ValueError:
            pass
tot = sum(d[0] for d in data) or 1
for d in sorted(data, reverse=True)[:n]:
    print(f"{d[0] / tot * 100:5.1f}% {d[1]}:{d[2]} {d[3].strip()[:100]}")
