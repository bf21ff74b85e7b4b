"""Host cost of enqueuing local steps against their device time (EURLex-shaped).

  * `step` loop: K asgd_local_step calls from Python without a sync: host us/step
    (wall clock of the enqueue loop) vs device us/step (CUDA events);
  * asgd_run_tickets over one mega-batch at inflight 1, 2, 8: host wall clock vs device.
If host us/step >= device us/step the GPU waits on the launches.

    python tools/host_overhead.py --config eurlex4k
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="eurlex4k")
    p.add_argument("--precision", default="bf16")
    p.add_argument("--steps", type=int, default=100)
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
    K = a.steps
    stream = torch.as_tensor(sample_stream(cfg, 0, K * cfg.b_max), dtype=torch.int32, device="cuda")
    rows = [stream[k * cfg.b_max:(k + 1) * cfg.b_max] for k in range(K)]
    for k in range(K):
        rep.step(rows[k], cfg.lr_max)
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for rep_i in range(2):
        s.record()
        t0 = time.perf_counter()
        for k in range(K):
            rep.step(rows[k], cfg.lr_max)
        t1 = time.perf_counter()
        e.record()
        torch.cuda.synchronize()
        print(f"step loop: host {1e6 * (t1 - t0) / K:.2f} us/step, device {1e3 * s.elapsed_time(e) / K:.2f} us/step")
    M = K * cfg.b_max
    sched = api.Scheduler(f"/asgd_ho_{os.getpid()}", 1, M, create=True)
    for inflight in (1, 2, 4, 8):
        for r in range(2):
            sched.reset(r + 1 + 10 * inflight)
            torch.cuda.synchronize()
            s.record()
            t0 = time.perf_counter()
            n = rep.run_tickets(sched, 0, cfg.b_max, stream, cfg.lr_max, None, inflight)
            t1 = time.perf_counter()
            e.record()
            torch.cuda.synchronize()
            t2 = time.perf_counter()
            if r:
                print(f"run_tickets inflight {inflight}: {n} steps, host call {1e6 * (t1 - t0) / n:.2f} us/step, "
                      f"device {1e3 * s.elapsed_time(e) / n:.2f} us/step, wall {1e6 * (t2 - t0) / n:.2f} us/step")
    sched.close()
    rep.close()


if __name__ == "__main__":
    main()
