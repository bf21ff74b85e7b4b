"""Top SASS lines by warp-stall samples from `ncu -i X --page source --csv`."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hi]
si = h.index("Warp Stall Sampling (All Samples)")
tot = 0
items = []
for r in rows[hi + 1:]:
    if len(r) <= si or not r[si].strip():
        continue
    try:
        v = float(r[si])
    except ValueError:
        continue
    tot += v
    items.append((v, r[0], r[1]))
items.sort(reverse=True)
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
for v, a, s in items[:n]:
    print(f"{v/tot*100:5.1f}%  {a}  {s[:110]}")
