"""Per captured launch: duration, tensor-pipe utilisation and DRAM traffic from one
`ncu --set full` report (raw page), as a markdown table.

    python tools/ncu_tensor.py REP.ncu-rep > profiles/r02_tensor_X.md

tensor active  = sm__pipe_tensor_cycles_active (% of the launch's elapsed cycles the tcgen05
                 pipe is busy, averaged over SMs: for a dense bf16 GEMM ~ achieved / peak flops)
tc issue       = sm__pipe_tc_cycles_active (% of elapsed cycles the tc issue pipe is busy)
"""
import csv
import io
import subprocess
import sys

M = {"dur": "gpu__time_duration.sum",
     "tensor": "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
     "bf16": "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed",
     "rd": "dram__bytes_read.sum", "wr": "dram__bytes_write.sum"}


def main(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True,
                         check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[0]
    idx = {k: (h.index(v) if v in h else None) for k, v in M.items()}
    ki = h.index("Kernel Name")
    units = rows[1]
    print("| kernel | duration | tensor pipe active | tc issue pipe active | DRAM read + write |")
    print("|---|---|---|---|---|")
    for r in rows[2:]:
        if len(r) <= ki:
            continue
        name = r[ki].split("(")[0].replace("void ", "").split("::")[-1]

        def g(k):
            i = idx[k]
            return r[i] if i is not None and i < len(r) else ""
        try:
            mb = (float(g("rd").replace(",", "") or 0) * (1e-6 if units[idx["rd"]] == "byte" else 1.0) +
                  float(g("wr").replace(",", "") or 0) * (1e-6 if units[idx["wr"]] == "byte" else 1.0))
            traffic = f"{mb:.1f} {'MB' if units[idx['rd']] == 'byte' else units[idx['rd']]}"
        except (ValueError, TypeError):
            traffic = ""
        print(f"| {name} | {g('dur')} {units[idx['dur']] if idx['dur'] is not None else ''} | {g('tensor')} % | "
              f"{g('bf16')} % | {traffic} |")


if __name__ == "__main__":
    main(sys.argv[1])
