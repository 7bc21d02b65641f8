"""Summarise an ncu source page (cuda,sass csv) into per-source-line stall samples."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
topn = int(sys.argv[2]) if len(sys.argv) > 2 else 40
fname = "?"
h = None
out = []
for r in rows:
    if len(r) >= 2 and r[0] == "File Name":
        fname = r[1].split("/")[-1]
        continue
    if "Warp Stall Sampling (All Samples)" in r:
        h = r
        si = h.index("Warp Stall Sampling (All Samples)")
        cols = [(c, h.index(c)) for c in h if c.startswith("stall_") and "Not Issued" not in c]
        continue
    if h is None or len(r) <= si or not r[0].strip().isdigit():
        continue
    try:
        v = int(r[si] or 0)
    except ValueError:
        continue
    if v == 0:
        continue
    top = sorted(((int(r[j] or 0), c) for c, j in cols), reverse=True)[:2]
    out.append((v, f"{fname}:{r[0]}", r[1].strip()[:90], top))
tot = sum(o[0] for o in out)
out.sort(reverse=True)
print("total samples", tot)
for v, loc, src, top in out[:topn]:
    print(f"{100*v/tot:5.1f}% {loc:28s} {src:90s} {top}")
