"""A/B of the merge variants and of Elastic SGD on one GPU (SURVEY §8(f) NEXT-2,
reading Q34), through the product path.

N replicas share one B200 and are routed by the simulated clock (Q10): replica
i's step costs c_i (nnz + 5 rows) with c_i = 1 + h i / (N - 1), so the last
replica is a (1 + h)x slower "GPU".  Arms:
  literal   Adaptive SGD as printed: Alg. 1 every mega-batch, Alg. 2 with the
            perturbation and no renormalisation (Q18) -- the default;
  renorm    the same with alpha / sum(alpha) after the perturbation (Q34's
            pert_renorm = true);
  ub_se2    alpha_i = u_i b_i / sum u_j b_j (R12) and Alg. 1 every 2nd mega-batch (R13);
  elastic   Elastic SGD: static b_max batches, rank k mod N, alpha = 1/N (R10);
  renorm_r17  renorm with Alg. 1's adaptive frequency (R17; not in the default --arms).
Per merge it logs ||w||_2 of the global model, sum(alpha), the perturbation flag,
b_i, test P@1, and the simulated makespan of the mega-batch (the time the
slowest replica is busy, in cost units; the paper's wall clock on
heterogeneous GPUs).  Time-to-P@1: the cumulative makespan until P@1 reaches
the target floor + 0.9 (best over all arms - floor), the same target for every
arm of an h.

  python tools/ab_sweep.py --config eurlex4k --replicas 4 --hetero 0,0.5,1 --megabatches 40 \\
      --out gpurun_out/ab.json
"""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

ARMS = {
    "literal": dict(method="adaptive", pert_renorm=False, norm="u", scale_every=1),
    "renorm": dict(method="adaptive", pert_renorm=True, norm="u", scale_every=1),
    "ub_se2": dict(method="adaptive", pert_renorm=False, norm="ub", scale_every=2),
    "elastic": dict(method="elastic", pert_renorm=False, norm="u", scale_every=1),
    "renorm_r17": dict(method="adaptive", pert_renorm=True, norm="u", scale_every=0),
}


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="eurlex4k")
    p.add_argument("--precision", default="bf16", choices=["fp32", "bf16"])
    p.add_argument("--replicas", type=int, default=4)
    p.add_argument("--hetero", default="0,0.5,1")
    p.add_argument("--arms", default="literal,renorm,ub_se2,elastic")
    p.add_argument("--megabatches", type=int, default=40)
    p.add_argument("--eval-rows", type=int, default=5000)
    p.add_argument("--out", default="gpurun_out/ab_sweep.json")
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
    counts = np.bincount(test.lab, minlength=cfg.L)
    floor = float(np.mean([counts.argmax() in set(test.lab[test.lab_ptr[i]:test.lab_ptr[i + 1]].tolist())
                           for i in range(test.n_rows)]))
    sq = torch.zeros(1, dtype=torch.float64, device="cuda")
    results = []
    for hx in [float(x) for x in a.hetero.split(",")]:
        n = a.replicas
        cf = [1.0 + hx * i / max(1, n - 1) for i in range(n)]
        runs = {}
        for arm in a.arms.split(","):
            v = ARMS[arm]
            h = train.Hyper.from_config(cfg, pert_renorm=v["pert_renorm"], norm=v["norm"],
                                        scale_every=v["scale_every"])
            r0 = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, a.precision, w0=w0)
            r0.register(dd)
            reps = [r0]
            for _ in range(n - 1):
                r = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, a.precision, w0=w0, share_global=r0)
                r.register(dd)
                reps.append(r)
            sim = train.SimulatedAdaptiveSGD(reps, h, lens, cf, method=v["method"])
            traj, clock = [], 0.0
            for mb in range(a.megabatches):
                ids = sample_stream(cfg, mb * h.M, h.M)
                st = sim.megabatch(torch.as_tensor(ids, device="cuda"), ids)
                busy = [0.0] * n   # simulated clock: replica r busy c_r (nnz + 5 rows) per batch
                for r, s0, ln in st.routes:
                    busy[r] += cf[r] * (float(lens[ids[s0:s0 + ln]].sum()) + 5.0 * ln)
                clock += max(busy)
                r0.sqnorm(sq)
                p1 = train.precision_at_k(r0, td, test, eval_ids, 1)
                traj.append({"t_sim": round(clock, 1), "p1": round(float(p1), 5),
                             "w_norm": round(float(np.sqrt(sq.item())), 4), "sum_alpha": round(float(sum(st.alpha)), 6),
                             "perturbed": bool(st.perturbed), "b": list(st.b), "u": list(st.u)})
            runs[arm] = traj
            print(json.dumps({"h": hx, "arm": arm, "final_p1": traj[-1]["p1"], "final_w": traj[-1]["w_norm"],
                              "best_p1": max(t["p1"] for t in traj)}), flush=True)
            for r in reps[::-1]:
                r.close()
        best = max(t["p1"] for tr in runs.values() for t in tr)
        target = floor + 0.9 * (best - floor)
        summary = {}
        for arm, tr in runs.items():
            k = next((i for i, t in enumerate(tr) if t["p1"] >= target), None)
            summary[arm] = {"time_to_target_sim": tr[k]["t_sim"] if k is not None else None,
                            "megabatches_to_target": k + 1 if k is not None else None,
                            "final_p1": tr[-1]["p1"], "best_p1": max(t["p1"] for t in tr),
                            "w_norm_first_last": [tr[0]["w_norm"], tr[-1]["w_norm"]],
                            "perturbed": sum(t["perturbed"] for t in tr),
                            "sum_alpha_max": max(t["sum_alpha"] for t in tr)}
        results.append({"hetero": hx, "cost_factors": cf, "target_p1": round(target, 5), "p1_floor": round(floor, 5),
                        "summary": summary, "trajectories": runs})
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump({"config": cfg.name, "precision": a.precision, "replicas": a.replicas,
                   "megabatches": a.megabatches, "results": results}, f)


if __name__ == "__main__":
    main()
