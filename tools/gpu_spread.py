"""B200 analogue of Fig. 1 (§I: "given the same training batch, the
gap between the fastest and slowest GPU is as large as 32% when performing an
epoch ... on a server with 4 NVIDIA V100 GPUs").

Every rank runs the SAME sequence of local steps (same rows, same initial
model) through the CUDA path and times it on its own device with CUDA events;
rank 0 prints per-GPU milliseconds and the (slowest - fastest) / fastest gap.
Repeats give the run-to-run spread on each GPU.

  python -m torch.distributed.run --nproc-per-node 8 --master-addr 127.0.0.1 \
      tools/gpu_spread.py --config eurlex4k --steps 400 --repeats 5
  python tools/gpu_spread.py           # one GPU: run-to-run spread only
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
    p.add_argument("--precision", default="bf16", choices=["fp32", "bf16"])
    p.add_argument("--steps", type=int, default=400)
    p.add_argument("--repeats", type=int, default=5)
    a = p.parse_args()

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_marws22_b200 import api
    from synth import config, generate, init_params, sample_stream

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl")
    cfg = config(a.config)
    data = generate(cfg, "train")
    nz, nl = api.max_step_sizes([data], cfg.b_max)
    rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, a.precision, device=local, w0=init_params(cfg))
    rep.register(api.DeviceCsr(data, device=torch.device("cuda", local)))
    ids = torch.as_tensor(sample_stream(cfg, 0, a.steps * cfg.b_max), device="cuda")
    lr = float(cfg.lr_max)
    params0 = rep.params.clone()
    times = []
    for k in range(a.repeats + 1):            # repeat 0 is warm-up
        rep.params.copy_(params0)             # same model, same work on every repeat and GPU
        rep.params_changed()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        for s in range(a.steps):
            rep.step(ids[s * cfg.b_max:(s + 1) * cfg.b_max], lr)
        e1.record()
        torch.cuda.synchronize()
        if k:
            times.append(e0.elapsed_time(e1))
    t = torch.tensor(times, dtype=torch.float64, device="cuda")
    allt = [torch.zeros_like(t) for _ in range(world)]
    if world > 1:
        dist.all_gather(allt, t)
    else:
        allt = [t]
    if rank == 0:
        per_gpu = [x.cpu().numpy() for x in allt]
        med = [float(np.median(x)) for x in per_gpu]
        out = {"config": cfg.name, "precision": a.precision, "steps": a.steps, "rows_per_step": cfg.b_max,
               "n_gpus": world, "ms_median_per_gpu": [round(m, 3) for m in med],
               "gap_slowest_vs_fastest": round((max(med) - min(med)) / min(med), 4),
               "run_to_run_spread_per_gpu": [round(float((x.max() - x.min()) / x.min()), 4) for x in per_gpu],
               "paper": "V100 x4: up to 32% (Fig. 1, P:136-141)"}
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
