"""dram traffic and duration per kernel class from one `ncu --set full` capture.

    python tools/ncu_traffic.py WORKLOAD/PREC OUT.json REP.ncu-rep [REP2.ncu-rep ...]

Kernel -> class follows the profile classes of include/asgd.h (ASGD_K_*), i.e.
the sections bench.py times; a class with several sections per step (dh_b1:
dH reduce + b1 update; merge: sqnorm, prescale, finish) divides its per-step
bytes by its sections so the figure is per timed launch like roofline.achieved.
"""
import csv
import io
import json
import re
import subprocess
import sys

SECTIONS = {"dh_b1": 2, "merge": 3}


def kclass(name: str):
    if name.startswith("k_gemm_tc"):
        # k_gemm_tc<BN, A_MN, B_MN, EPI, X3>: the 4th template argument is the epilogue
        args = re.findall(r"\w+", name.split("<")[1])
        epi = int(args[3])
        return {0: "g1", 1: "g2", 2: "g3", 3: "softmax", 4: "g1", 5: "g1"}[epi]   # 4: sigmoid G1, 5: stats G1
    if name.startswith("k_bwd_dh"):
        return "g2"   # K-3's dH1 half (G1b + G2 + dH reduce): profiled as G2
    for pre, cls in (("k_touched", "touched"), ("k_spmm_fwd", "spmm"), ("k_softmax_ce", "softmax"),
                     ("k_lse", "softmax"), ("k_dh_reduce", "dh_b1"), ("k_b1_update", "dh_b1"),
                     ("k_scatter_sgd", "scatter"), ("k_sqnorm", "merge"), ("k_scale", "merge"),
                     ("k_finish", "merge"), ("k_merge_fused", "merge"), ("k_merge_wait", "merge"),
                     ("k_tile_loss", "softmax"), ("k_sig_center", "softmax"), ("k_sigmoid_ce", "softmax"),
                     ("k_gemm_f32", None), ("k_b2_", "b2")):
        if name.startswith(pre):
            return cls
    return None


def read(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics",
                          "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum"],
                         capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h, units = rows[hi], rows[hi + 1]
    ki = h.index("Kernel Name")
    cols = {m: h.index(m) for m in ("dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum")}
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "us": 1, "usecond": 1,
             "nsecond": 1e-3, "ms": 1e3, "msecond": 1e3}
    per = {}
    for r in rows[hi + 2:]:
        if len(r) <= ki:
            continue
        name = re.sub(r"^.*?(unnamed>|anonymous namespace\))::", "", r[ki]).replace("void ", "").replace("asgd::", "")
        name = name.split("(")[0]
        v = {m: float(r[i].replace(",", "")) * scale.get(units[i], 1) for m, i in cols.items()}
        d = per.setdefault(name, {"n": 0, "bytes": 0.0, "us": 0.0})
        d["n"] += 1
        d["bytes"] += v["dram__bytes_read.sum"] + v["dram__bytes_write.sum"]
        d["us"] += v["gpu__time_duration.sum"]
    return per


def main(key, path, *reps):
    per = {}
    for rep in reps:
        per.update(read(rep))
    cls_bytes = {}
    kernels = {}
    for name, d in per.items():
        mb = d["bytes"] / d["n"]
        kernels[name] = {"launches": d["n"], "dram_bytes_per_launch": round(mb), "us_per_launch": round(d["us"] / d["n"], 2)}
        c = kclass(name)
        if c:
            cls_bytes[c] = cls_bytes.get(c, 0.0) + mb
    per_launch = {c: round(b / SECTIONS.get(c, 1)) for c, b in cls_bytes.items()}
    entry = {"source": [r.split("/")[-1] for r in reps], "per_launch_bytes": per_launch, "kernels": kernels}
    print(json.dumps({key: entry}, indent=1))
    if path != "-":
        try:
            with open(path) as f:
                allv = json.load(f)
        except FileNotFoundError:
            allv = {}
        allv[key] = entry
        with open(path, "w") as f:
            json.dump(allv, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main(*sys.argv[1:])
