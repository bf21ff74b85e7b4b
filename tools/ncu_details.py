"""Key `ncu --set full` metrics per captured launch, as a markdown table.

    python tools/ncu_details.py REP.ncu-rep > profiles/rNN_ncu_full_X.md
"""
import csv
import io
import subprocess
import sys

WANT = ["Duration", "Compute (SM) Throughput", "Memory Throughput", "DRAM Throughput", "L2 Cache Throughput",
        "L2 Hit Rate", "Achieved Occupancy", "Registers Per Thread", "Dynamic Shared Memory Per Block",
        "Issued Warp Per Scheduler", "No Eligible"]


def main(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True,
                         check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[0]
    ki, mi, vi, ui = (h.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    gi = h.index("Grid Size")
    recs = {}
    for r in rows[1:]:
        if len(r) <= vi:
            continue
        name = r[ki].split("(")[0].split("::")[-1].replace("void ", "")
        d = recs.setdefault(r[0], {"kernel": name, "grid": r[gi]})
        if r[mi] in WANT and r[mi] not in d:
            d[r[mi]] = f"{r[vi]} {r[ui]}".strip()
    print("| id | kernel | grid | " + " | ".join(WANT) + " |")
    print("|---|---|---|" + "---|" * len(WANT))
    for i, d in recs.items():
        print(f"| {i} | {d['kernel']} | {d['grid']} | " + " | ".join(d.get(w, "") for w in WANT) + " |")


if __name__ == "__main__":
    main(sys.argv[1])
