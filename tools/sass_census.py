"""Per-kernel SASS census of libasgd.so: counts of the Blackwell tensor-core /
TMEM / TMA / FMA instructions in every kernel (cuobjdump -sass; no GPU needed).

    python tools/sass_census.py [path/to/libasgd.so] > profiles/r02_sass_census.md
"""
import collections
import os
import re
import subprocess
import sys

LIB = sys.argv[1] if len(sys.argv) > 1 else os.path.join(os.path.dirname(__file__), "..",
                                                          "paper_conf_ipps_marws22_b200", "libasgd.so")
OPS = ["UTCHMMA", "UTCQMMA", "UTCIMMA", "UTCMMA", "UTCBAR", "LDTM", "STTM", "UTMALDG", "UTMASTG", "UBLKCP",
       "SYNCS", "FFMA", "HMMA", "MUFU.EX2", "RED", "ATOMG"]

out = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True).stdout
kern = None
cnt = collections.OrderedDict()
for line in out.splitlines():
    m = re.match(r"\s+Function : (\S+)", line)
    if m:
        kern = m.group(1)
        cnt[kern] = collections.Counter()
        continue
    if kern is None:
        continue
    m = re.search(r"/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)", line)
    if not m:
        continue
    op = m.group(1)
    for o in OPS:
        if op == o or op.startswith(o + "."):
            cnt[kern][o] += 1


def demangle(names):
    r = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True).stdout.splitlines()
    out = []
    for x in r:
        x = x.replace("(anonymous namespace)::", "").replace("asgd::", "")
        x = re.sub(r"^void ", "", x)
        out.append(re.sub(r"\(.*", "", x))
    return out


names = list(cnt)
dem = demangle(names)
cols = [o for o in OPS if any(cnt[k][o] for k in names)]
print(f"# SASS census of `{os.path.relpath(LIB)}` (cuobjdump -sass, sm_100a)\n")
print("Counts of static SASS instructions per kernel. UTCHMMA = tcgen05.mma kind::f16 (bf16/fp16), "
      "UTCMMA/UTCQMMA = other tcgen05.mma kinds (tf32/f8f6f4), LDTM = tcgen05.ld (TMEM -> registers), "
      "UTMALDG/UTMASTG = TMA tensor loads/stores, UBLKCP = cp.async.bulk, FFMA = fp32 SIMT FMA.\n")
print("| kernel | " + " | ".join(cols) + " |")
print("|---|" + "---|" * len(cols))
for k, d in sorted(zip(names, dem), key=lambda x: x[1]):
    print(f"| `{d[:90]}` | " + " | ".join(str(cnt[k][o]) for o in cols) + " |")
