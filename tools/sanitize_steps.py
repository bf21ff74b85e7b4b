"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck):
a few local steps on the tiny and EURLex-4K shapes in both precisions (K-0's
grid barriers, K-1/K-5's last-arriver combines, the tcgen05 GEMMs), the
sqnorm / prescale / finish merge, a 1-rank fused merge (system-scope counters)
and one top-k evaluation.

    compute-sanitizer --tool memcheck python tools/sanitize_steps.py
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
from paper_conf_ipps_marws22_b200 import api  # noqa: E402
from synth import config, generate, init_params, sample_stream  # noqa: E402

for name in ("tiny", "eurlex4k"):
    cfg = config(name)
    data = generate(cfg, "train", 4096)
    test = generate(cfg, "test", 512)
    nz, nl = api.max_step_sizes([data, test], cfg.b_max)
    for prec in ("fp32", "bf16"):
        rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, prec, w0=init_params(cfg))
        dd = api.DeviceCsr(data)
        rep.register(dd)
        loss = torch.zeros(1, device="cuda")
        for k in range(3):
            rows = sample_stream(config(name, n_train=data.n_rows), k * cfg.b_max, cfg.b_max - 5 * k)
            rep.step(torch.as_tensor(rows, device="cuda"), 0.5, loss)
        sq = torch.zeros(1, dtype=torch.float64, device="cuda")
        rep.sqnorm(sq)
        rep.prescale(1.0)
        rep.finish(0.9)
        rep.peer_open(0, [rep.peer_export()])
        rep.merge_fused([1.0], 0.9)
        td = api.DeviceCsr(test)
        top = rep.eval_topk(td, torch.arange(256, dtype=torch.int32, device="cuda"), 5)
        rep.sync()
        print(name, prec, "loss", float(loss.item()), "sq", float(sq.item()), "top0", top[0].tolist(), flush=True)
        rep.peer_close()
        rep.close()
print("sanitize workload done")
