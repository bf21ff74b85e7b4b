"""Live kernel timeline of one local step (needs libasgd built with -DASGD_TIMELINE:
    ASGD_NVCC_EXTRA=-DASGD_TIMELINE python -m paper_conf_ipps_marws22_b200.build --force).

Runs `warm` steps, then `steps` steps one at a time (device sync between steps, so a
step starts on an idle GPU; within the step the kernels overlap and chain exactly as in
the bench), and prints per kernel class the median over steps of its first CTA arrival,
its first return from griddepcontrol.wait (on the step's chain: its predecessor's end)
and its last CTA end, relative to the step's first arrival, in us.  Then the same steps
back to back without syncs (the bench's regime) for the mean step time.

    python tools/timeline.py --config eurlex4k --precision bf16 --steps 50
"""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="eurlex4k")
    p.add_argument("--precision", default="bf16")
    p.add_argument("--steps", type=int, default=50)
    p.add_argument("--warm", type=int, default=20)
    p.add_argument("--out", default=None)
    a = p.parse_args()
    import torch
    from paper_conf_ipps_marws22_b200 import api
    from synth import config, generate, init_params, sample_stream

    cfg = config(a.config)
    data = generate(cfg)
    nz, nl = api.max_step_sizes([data], cfg.b_max)
    rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, a.precision, w0=init_params(cfg))
    dd = api.DeviceCsr(data)
    rep.register(dd)
    K = len(api.TIMELINE_KERNELS)
    buf = torch.zeros(3 * K, dtype=torch.int64, device="cuda")
    rows = [torch.as_tensor(sample_stream(cfg, k * cfg.b_max, cfg.b_max), device="cuda")
            for k in range(a.warm + a.steps)]
    for k in range(a.warm):
        rep.step(rows[k], cfg.lr_max)
    rep.sync()
    api.timeline_set(buf)
    recs = []
    init = torch.tensor([-1, -1, 0] * K, dtype=torch.int64, device="cuda")   # ~0 for the min slots
    for k in range(a.warm, a.warm + a.steps):
        buf.copy_(init)
        rep.step(rows[k], cfg.lr_max)
        rep.sync()
        recs.append(buf.cpu().numpy().view(np.uint64).reshape(K, 3).copy())
    api.timeline_set(None)
    out = {}
    rel = []
    for r in recs:
        seen = r[:, 0] != np.uint64(2**64 - 1)
        t0 = r[seen, 0].min()
        rr = np.full((K, 3), np.nan)
        for i in np.nonzero(seen)[0]:
            rr[i] = (r[i].astype(np.float64) - float(t0)) / 1e3
        rel.append(rr)
    rel = np.array(rel)
    med = np.nanmedian(rel, axis=0)
    print(f"{'kernel':10s} {'arrive':>8s} {'ready':>8s} {'end':>8s} {'ready->end':>10s}  (us, median of {a.steps})")
    order = np.argsort(np.where(np.isnan(med[:, 1]), med[:, 2], med[:, 1]))
    for i in order:
        if np.isnan(med[i, 0]) and np.isnan(med[i, 2]):
            continue
        name = api.TIMELINE_KERNELS[i]
        out[name] = dict(arrive=med[i, 0], ready=med[i, 1], end=med[i, 2], span=med[i, 2] - med[i, 1])
        print(f"{name:10s} {med[i, 0]:8.2f} {med[i, 1]:8.2f} {med[i, 2]:8.2f} {med[i, 2] - med[i, 1]:10.2f}")
    step_end = np.nanmax(rel[:, :, 2], axis=1)
    print(f"isolated step (first arrival -> last end): median {np.median(step_end):.2f} us")
    # back to back, the bench's regime
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for k in range(a.warm, a.warm + a.steps):
        rep.step(rows[k], cfg.lr_max)
    e.record()
    torch.cuda.synchronize()
    b2b = s.elapsed_time(e) * 1e3 / a.steps
    print(f"back-to-back step: {b2b:.2f} us")
    if a.out:
        with open(a.out, "w") as f:
            json.dump(dict(config=a.config, precision=a.precision, steps=a.steps, kernels=out,
                           isolated_step_us=float(np.median(step_end)), back_to_back_us=b2b), f, indent=1)
    rep.close()


if __name__ == "__main__":
    main()
