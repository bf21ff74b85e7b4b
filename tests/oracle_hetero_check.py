"""Cross-check of one heterogeneity point of profiles/r01_telemetry.md on the CPU
oracle (test infrastructure, kept under tests/ with the other oracle users; run by hand): EURLex-4K-shaped, 4 replicas, cost
factors 1..1+h, n_mb mega-batches, paper defaults (or --norm ub --scale-every 2).
Prints per-mega-batch b_i of the routed replicas and the final P@1 of the fp64
model, to compare with the CUDA path's trajectory (same routing, bf16 vs fp64)."""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

p = argparse.ArgumentParser()
p.add_argument("--hetero", type=float, default=1.0)
p.add_argument("--megabatches", type=int, default=20)
p.add_argument("--norm", default="u")
p.add_argument("--scale-every", type=int, default=1)
a = p.parse_args()

from oracle import adaptive, metrics, model
from synth import config, generate, init_params, sample_stream

cfg = config("eurlex4k")
data = generate(cfg, "train")
test = generate(cfg, "test", 5000)
n = 4
cf = [1.0 + a.hetero * i / (n - 1) for i in range(n)]
M = cfg.mega_batch
recs = adaptive.run(cfg.F, cfg.H, cfg.L, data, init_params(cfg), lambda mb: sample_stream(cfg, mb * M, M),
                    n_rep=n, n_mb=a.megabatches, M=M, b_max=cfg.b_max, b_min=cfg.b_min, beta=cfg.beta,
                    lr_max=cfg.lr_max, cost_factors=cf, norm=a.norm, scale_every=a.scale_every)
w = recs[-1].w
sub = test.row_slice(np.arange(test.n_rows))
Z = model.forward(w, sub, cfg.F, cfg.H, cfg.L)[-1]
top = metrics.topk(Z, 1)
print(json.dumps({"hetero": a.hetero, "norm": a.norm, "scale_every": a.scale_every,
                  "b": [r.b for r in recs], "perturbed": [bool(r.perturbed) for r in recs],
                  "p1": round(float(metrics.precision_at_k(top, sub.lab_ptr, sub.lab, 1)), 5)}))
