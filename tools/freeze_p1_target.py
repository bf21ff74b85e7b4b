"""Freeze the per-config time-to-P@1 target: run the 1-GPU fp32
path for --megabatches mega-batches, take its best test P@1 as p_best and the
majority-label P@1 as the floor, and write target = floor + 0.9 (p_best - floor)
into configs/p1_targets.json, which bench.py's time_to_p1 then uses at every N.

  python tools/freeze_p1_target.py --config eurlex4k --megabatches 40
"""
import argparse
import datetime
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="eurlex4k")
    p.add_argument("--megabatches", type=int, default=40)
    p.add_argument("--out", default=os.path.join(ROOT, "configs", "p1_targets.json"))
    a = p.parse_args()
    import torch
    import bench
    from synth import config
    bench.frozen_p1_target = lambda name: None          # measure, do not read the old target
    cfg = config(a.config)
    r = bench.time_to_p1(cfg, "fp32", a.megabatches, torch.device("cuda", 0))
    rec = {"target_p1": round(r["p1_floor"] + 0.9 * (r["p1_best"] - r["p1_floor"]), 5),
           "p1_best": r["p1_best"], "p1_floor": r["p1_floor"],
           "source": f"1 B200, fp32 path, {a.megabatches} mega-batches, {r['test_rows']} test rows, "
                     f"lr_max {r['lr_max']}, {datetime.date.today().isoformat()} (tools/freeze_p1_target.py)",
           "curve_every_4": r["curve_every_4"]}
    cur = {}
    if os.path.exists(a.out):
        with open(a.out) as f:
            cur = json.load(f)
    cur[cfg.name] = rec
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(cur, f, indent=1)
    print(json.dumps({cfg.name: {k: v for k, v in rec.items() if k != "curve_every_4"}}))


if __name__ == "__main__":
    main()
