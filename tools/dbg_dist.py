"""Repeat the 2-rank one-GPU driver run (tests/test_gpu_dist.py) and print the
normwise error against the oracle replay per mega-batch count, to chase flaky
parity."""
import os, sys, tempfile, uuid
import numpy as np
import torch.multiprocessing as mp
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from tests.test_gpu_dist import _rank, _port


def one(precision, merge, n_mb):
    from oracle import adaptive
    from synth import config, generate, init_params, sample_stream
    with tempfile.TemporaryDirectory() as tmp:
        shm = "/asgd_x_" + uuid.uuid4().hex[:8]
        mp.spawn(_rank, args=(2, _port(), shm, tmp, precision, n_mb, merge), nprocs=2, join=True)
        w0, w1 = (np.load(os.path.join(tmp, f"w{r}.npy")) for r in range(2))
        logs, stats = np.load(os.path.join(tmp, "s0.npy"), allow_pickle=True)
    cfg = config("tiny"); data = generate(cfg); M = cfg.mega_batch
    recs = adaptive.run(cfg.F, cfg.H, cfg.L, data, init_params(cfg), lambda mb: sample_stream(cfg, mb * M, M),
                        n_rep=2, n_mb=n_mb, M=M, b_max=cfg.b_max, b_min=cfg.b_min, beta=cfg.beta,
                        lr_max=cfg.lr_max, route_logs=list(logs))
    ref = recs[-1].w
    e = np.linalg.norm(w0 - ref) / np.linalg.norm(ref)
    print(precision, merge, n_mb, "eq", bool((w0 == w1).all()), "err %.3e" % e, "logs", [len(l) for l in logs],
          [list(l) for l in logs][:2], flush=True)


if __name__ == "__main__":
    for rep in range(int(sys.argv[1]) if len(sys.argv) > 1 else 4):
        for merge in ("fused", "nccl"):
            one("fp32", merge, 4)
