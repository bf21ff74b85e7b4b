"""Stall-reason totals and the top SASS lines per reason from
`ncu -i X --page source --csv` (one kernel launch).

    python tools/ncu_stalls.py SRC.csv [top]
"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hi]
cols = [i for i, x in enumerate(h) if x.startswith("stall_")]
seen = set()
tot = {h[i]: 0.0 for i in cols}
per = []
for r in rows[hi + 1:]:
    if len(r) <= max(cols) or r[0] in seen:
        continue
    seen.add(r[0])
    for i in cols:
        try:
            v = float(r[i] or 0)
        except ValueError:
            v = 0.0
        tot[h[i]] += v
        if v:
            per.append((v, h[i], r[0], r[1]))
s = sum(tot.values()) or 1.0
for k, v in sorted(tot.items(), key=lambda kv: -kv[1])[:10]:
    print(f"{k:28s} {100 * v / s:5.1f}%")
per.sort(reverse=True)
for v, k, a, src in per[:int(sys.argv[2]) if len(sys.argv) > 2 else 15]:
    print(f"{100 * v / s:5.1f}% {k:22s} {a[-5:]} {src}")
