"""Per-rank step log (SURVEY §5 tracing): run mega-batches of the product path with the
library's step trace on and write one JSON line per local step:
  {"rank", "mb", "ticket", "start", "rows", "nnz", "t0_us", "t1_us"}
t0/t1 are the CUDA-event times around the step's enqueue on the rank's stream, relative
to the rank's trace origin (asgd_trace_enable); ticket = the step's position in the shared
scheduler's log (the routing order across ranks).  Works at N = 1 or under torchrun.

  python tools/trace_steps.py --config eurlex4k --megabatches 3 --out gpurun_out/trace
  torchrun --nproc-per-node N --master-addr 127.0.0.1 tools/trace_steps.py ...
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
    p.add_argument("--megabatches", type=int, default=3)
    p.add_argument("--out", default="gpurun_out/trace")
    a = p.parse_args()
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_marws22_b200 import api, train
    from synth import config, generate, init_params, sample_stream
    rank, world = int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    cfg = config(a.config)
    data = generate(cfg, "train")
    nz, nl = api.max_step_sizes([data], cfg.b_max)
    rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, a.precision, device=local, w0=init_params(cfg))
    rep.register(api.DeviceCsr(data, device=dev))
    h = train.Hyper.from_config(cfg)
    shm = f"/asgd_trace_{os.environ.get('MASTER_PORT', os.getpid())}"
    if rank == 0:
        sched = api.Scheduler(shm, world, h.M, create=True)
    if world > 1:
        dist.barrier()
    if rank != 0:
        sched = api.Scheduler(shm, world, h.M, create=False)
    drv = train.DistributedAdaptiveSGD(rep, h, rank, world, sched)
    lens = np.diff(data.row_ptr)
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(f"{a.out}.rank{rank}.jsonl", "w") as f:
        for mb in range(a.megabatches):
            ids = sample_stream(cfg, mb * h.M, h.M)
            rep.trace_enable(True)
            st = drv.megabatch(torch.as_tensor(ids, device=dev), keep_log=True)
            steps = rep.trace_read()
            rep.trace_enable(False)
            order = {}
            if world > 1:
                logs = [None] * world
                dist.all_gather_object(logs, st.routes if rank == 0 else None)
                st_routes = logs[0]
            else:
                st_routes = st.routes
            for tk, r, s0, ln in st_routes:
                order[(r, s0)] = tk
            for s0, rows, t0, t1 in steps:
                f.write(json.dumps({"rank": rank, "mb": mb, "ticket": order.get((rank, s0)), "start": s0,
                                    "rows": rows, "nnz": int(lens[ids[s0:s0 + rows]].sum()),
                                    "t0_us": round(t0 / 1e3, 3), "t1_us": round(t1 / 1e3, 3)}) + "\n")
    if world > 1:
        dist.barrier()
    sched.close()
    print(f"rank {rank}: trace -> {a.out}.rank{rank}.jsonl")


if __name__ == "__main__":
    main()
