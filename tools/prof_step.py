"""A few local steps of one config (for ncu captures of single kernels):
`warm` untimed steps, then `prof` more; filter the captured launches with
ncu -k / --launch-skip.

    python tools/prof_step.py CONFIG PRECISION LOSS WARM PROF [TRAIN_ROWS]
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_marws22_b200 import api
from synth import config, generate, init_params, sample_stream

name, prec, loss, warm, prof = sys.argv[1], sys.argv[2], sys.argv[3], int(sys.argv[4]), int(sys.argv[5])
rows_n = int(sys.argv[6]) if len(sys.argv) > 6 else None
cfg = config(name)
data = generate(cfg, "train", rows_n)
if rows_n:
    cfg = config(name, n_train=data.n_rows)
nz, nl = api.max_step_sizes([data], cfg.b_max)
rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, prec, w0=init_params(cfg), loss=loss)
dd = api.DeviceCsr(data)
rep.register(dd)
for k in range(warm + prof):
    rows = torch.as_tensor(sample_stream(cfg, k * cfg.b_max, cfg.b_max), device="cuda")
    rep.step(rows, cfg.lr_max)
rep.sync()
print("done", name, prec, loss, warm, prof)
