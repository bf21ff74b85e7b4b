"""Device time of the local step under the current environment's switches (no probes):
K steps of one config back to back from Python (host enqueue ~4 us/step, far below the
device time), CUDA events around them, median of R repetitions.  Prints one JSON line.

    ASGD_K0_FOLD=0 python tools/ab_step.py --config eurlex4k --tag nofold
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="eurlex4k")
    p.add_argument("--precision", default="bf16")
    p.add_argument("--steps", type=int, default=100)
    p.add_argument("--reps", type=int, default=5)
    p.add_argument("--tag", default="")
    a = p.parse_args()
    import numpy as np
    import torch
    from paper_conf_ipps_marws22_b200 import api
    from synth import config, generate, init_params, sample_stream

    cfg = config(a.config)
    data = generate(cfg)
    nz, nl = api.max_step_sizes([data], cfg.b_max)
    rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, a.precision, w0=init_params(cfg))
    dd = api.DeviceCsr(data)
    rep.register(dd)
    K = a.steps
    stream = torch.as_tensor(sample_stream(cfg, 0, K * cfg.b_max), dtype=torch.int32, device="cuda")
    rows = [stream[k * cfg.b_max:(k + 1) * cfg.b_max] for k in range(K)]
    for k in range(K):
        rep.step(rows[k], cfg.lr_max)
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t = []
    for _ in range(a.reps):
        s.record()
        for k in range(K):
            rep.step(rows[k], cfg.lr_max)
        e.record()
        torch.cuda.synchronize()
        t.append(1e3 * s.elapsed_time(e) / K)
    env = {k: v for k, v in os.environ.items() if k.startswith("ASGD_")}
    print(json.dumps({"tag": a.tag, "config": a.config, "precision": a.precision, "us_per_step": float(np.median(t)),
                      "min": float(min(t)), "max": float(max(t)), "env": env}))
    rep.close()


if __name__ == "__main__":
    main()
