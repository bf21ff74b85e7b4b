"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) per kernel.

    python tools/ncu_summary.py gpurun_out/launches.csv [--skip N] > profiles/r01_launches.md
"""
import collections
import csv
import re
import sys


def kname(s: str) -> str:
    s = s.replace("void ", "")
    s = re.sub(r"^.*?(unnamed>|anonymous namespace\))::", "", s).replace("asgd::", "")
    s = s.split("(")[0]
    m = re.match(r"([A-Za-z0-9_:]+)(<.*>)?", s)
    base = m.group(1) if m else s
    tmpl = m.group(2) if m and m.group(2) else ""
    return base + (tmpl if base.startswith("k_") and len(tmpl) < 40 else "")


def main(path, skip=0):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[hi]
    ki, vi, ui, gi = (hdr.index(x) for x in ("Kernel Name", "Metric Value", "Metric Unit", "Grid Size"))
    agg = collections.OrderedDict()
    for r in rows[hi + 1 + skip:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", ""))
        u = r[ui]
        v = v / 1e3 if u in ("ns", "nsecond") else (v * 1e3 if u in ("ms", "msecond") else v)
        agg.setdefault((kname(r[ki]), r[gi]), []).append(v)
    tot = sum(sum(v) for v in agg.values())
    print(f"| kernel | grid | launches | mean us | total us | share |")
    print(f"|---|---|---|---|---|---|")
    for (k, g), v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        print(f"| {k} | {g} | {len(v)} | {sum(v)/len(v):.2f} | {sum(v):.1f} | {sum(v)/tot:.3f} |")
    print(f"\ntotal {tot:.1f} us over {sum(len(v) for v in agg.values())} launches")


if __name__ == "__main__":
    skip = int(sys.argv[sys.argv.index("--skip") + 1]) if "--skip" in sys.argv else 0
    main(sys.argv[1], skip)
