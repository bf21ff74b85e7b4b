"""Method telemetry sweeps on one GPU: heterogeneity injection
(a B200 analogue of Fig. 6a/6b) and the mega-batch size M
(P:639-643), through the product path (CUDA kernels behind libasgd.so).

N replicas share one GPU and are routed by the simulated clock (reading Q10):
replica i's step costs cost_factor_i * (nnz + per_row * rows), so a factor of
1 + h makes it a (1 + h)x slower "GPU".  For every heterogeneity level h and
every M, the script runs n_mb mega-batches of Adaptive SGD (Alg. 1 + Alg. 2)
and records, per mega-batch, the batch sizes b_i in effect (Fig. 6a), the
updates u_i, whether Alg. 2 perturbed the weights (Fig. 6b), alpha and the
mean loss, plus the final P@1 on held-out rows.  Options pass through the
method variants: --norm u|ub (R12), --scale-every k (R13).

  python tools/hetero_sweep.py --config eurlex4k --replicas 4 --hetero 0,0.5,1,2 \
      --mega-batch-steps 100 --megabatches 20 --out gpurun_out/hetero.json
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="eurlex4k")
    p.add_argument("--precision", default="bf16", choices=["fp32", "bf16"])
    p.add_argument("--replicas", type=int, default=4)
    p.add_argument("--hetero", default="0,0.5,1,2", help="slowdown h of the last replica; factors spread linearly 1..1+h")
    p.add_argument("--mega-batch-steps", default="100", help="M / b_max values to sweep (comma list)")
    p.add_argument("--megabatches", type=int, default=20)
    p.add_argument("--norm", default="u", choices=["u", "ub"])
    p.add_argument("--scale-every", type=int, default=1)
    p.add_argument("--eval-rows", type=int, default=5000)
    p.add_argument("--out", default="gpurun_out/hetero_sweep.json")
    a = p.parse_args()

    import torch
    from paper_conf_ipps_marws22_b200 import api, train
    from synth import config, generate, init_params, sample_stream

    cfg = config(a.config)
    data = generate(cfg, "train")
    test = generate(cfg, "test", a.eval_rows)
    nz, nl = api.max_step_sizes([data, test], cfg.b_max)
    lens = np.diff(data.row_ptr)
    dd = api.DeviceCsr(data)
    td = api.DeviceCsr(test)
    w0 = init_params(cfg)
    eval_ids = np.arange(test.n_rows, dtype=np.int32)
    results = []
    for mbs in [int(x) for x in a.mega_batch_steps.split(",")]:
        for hx in [float(x) for x in a.hetero.split(",")]:
            n = a.replicas
            cf = [1.0 + hx * i / max(1, n - 1) for i in range(n)]
            h = train.Hyper.from_config(cfg, M=mbs * cfg.b_max, norm=a.norm, scale_every=a.scale_every)
            r0 = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, a.precision, w0=w0)
            r0.register(dd)
            reps = [r0]
            for _ in range(n - 1):
                r = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, a.precision, w0=w0, share_global=r0)
                r.register(dd)
                reps.append(r)
            sim = train.SimulatedAdaptiveSGD(reps, h, lens, cf)
            traj = []
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            for mb in range(a.megabatches):
                ids = sample_stream(cfg, mb * h.M, h.M)
                st = sim.megabatch(torch.as_tensor(ids, device="cuda"), ids)
                traj.append({"b": list(st.b), "u": list(st.u), "alpha": [round(x, 6) for x in st.alpha],
                             "perturbed": bool(st.perturbed)})
            torch.cuda.synchronize()
            wall = time.perf_counter() - t0
            p1 = train.precision_at_k(r0, td, test, eval_ids, 1)
            rec = {"mega_batch_steps": mbs, "M": h.M, "hetero": hx, "cost_factors": cf,
                   "perturb_freq": sum(t["perturbed"] for t in traj) / len(traj),
                   "final_b": traj[-1]["b"], "p1": round(float(p1), 5), "wall_s": round(wall, 3),
                   "trajectory": traj}
            print(json.dumps({k: v for k, v in rec.items() if k != "trajectory"}), flush=True)
            results.append(rec)
            for r in reps[::-1]:
                r.close()
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump({"config": cfg.name, "precision": a.precision, "replicas": a.replicas, "norm": a.norm,
                   "scale_every": a.scale_every, "megabatches": a.megabatches, "runs": results}, f)


if __name__ == "__main__":
    main()
