"""One-line summary of a bench.py JSON line: python tools/bench_brief.py FILE"""
import json
import sys

try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
except Exception as e:          # the bench failed: show why
    print("no bench line:", e)
    sys.exit(0)
r = d.get("roofline", {})
print(d.get("config", {}).get("workload"), d.get("dtype"), "value", d.get("value"), "ms/step", d.get("ms_per_step"),
      "dom", r.get("kernel"), r.get("bound"), "frac", r.get("frac"), "e2e", (d.get("e2e") or {}).get("value"),
      "clocks", d.get("clocks"))
kw = d.get("kernels_warmup_profile") or {}
print({k: v["us_per_launch"] for k, v in kw.items()})
for k in ("merge", "time_to_p1", "cpu_baseline"):
    if k in d:
        v = d[k]
        print(k, {a: b for a, b in v.items() if a != "curve_every_4"} if isinstance(v, dict) else v)
