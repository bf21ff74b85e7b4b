"""Race hunt: run the same sequence of local steps twice on fresh replicas and
compare the parameters bitwise after every `check` steps (the step is
deterministic by construction, R5).  Run several copies at once to add
contention (two processes time-sliced on one GPU, as in tests/test_gpu_dist)."""
import sys, os
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_marws22_b200 import api
from synth import config, generate, init_params, sample_stream


def run(cfg, data, prec, n_steps, sizes, seed):
    nz, nl = api.max_step_sizes([data], cfg.b_max)
    rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, prec, w0=init_params(cfg))
    dd = api.DeviceCsr(data)
    rep.register(dd)
    rng = np.random.default_rng(seed)
    snaps = []
    pos = 0
    for k in range(n_steps):
        n = int(sizes[rng.integers(len(sizes))])
        rows = torch.as_tensor(sample_stream(cfg, pos, n), device="cuda")
        pos += n
        rep.step(rows, cfg.lr_max)
        if (k + 1) % 25 == 0:
            snaps.append(rep.params.clone())
    rep.sync()
    return [s.cpu().numpy() for s in snaps]


if __name__ == "__main__":
    name, prec, n_steps = sys.argv[1], sys.argv[2], int(sys.argv[3])
    cfg = config(name)
    data = generate(cfg)
    sizes = [cfg.b_max, cfg.b_max, cfg.b_max - 1, cfg.b_max // 2 + 3, 7, 1]
    a = run(cfg, data, prec, n_steps, sizes, 1)
    b = run(cfg, data, prec, n_steps, sizes, 1)
    bad = [i for i, (x, y) in enumerate(zip(a, b)) if not np.array_equal(x, y)]
    print(name, prec, "snapshots", len(a), "first mismatch", (bad[0] + 1) * 25 if bad else None,
          "maxdiff", max(float(np.abs(x - y).max()) for x, y in zip(a, b)), flush=True)
