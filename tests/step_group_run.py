"""Helper of test_gpu_step_groups.py (run in a subprocess so ASGD_STEP_GROUP is read
fresh): one mega-batch of EURLex-shaped steps through asgd_run_tickets at N = 1 with a
ragged last ticket, then the parameters and per-step losses to an .npz."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_marws22_b200 import api  # noqa: E402
from synth import config, generate, init_params, sample_stream  # noqa: E402

out, name, prec = sys.argv[1], sys.argv[2], sys.argv[3]
cfg = config(name)
data = generate(cfg)
nz, nl = api.max_step_sizes([data], cfg.b_max)
rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, prec, w0=init_params(cfg))
dd = api.DeviceCsr(data)
rep.register(dd)
M = 23 * cfg.b_max + cfg.b_max // 3          # 23 full tickets and a ragged one
stream = torch.as_tensor(sample_stream(cfg, 0, M), dtype=torch.int32, device="cuda")
losses = torch.zeros(64, dtype=torch.float32, device="cuda")
sched = api.Scheduler(f"/asgd_sg_{os.getpid()}", 1, M, create=True)
n = 0
for mb in range(2):                          # two mega-batches: graphs captured, then replayed
    sched.reset(mb + 1)
    n = rep.run_tickets(sched, 0, cfg.b_max, stream, cfg.lr_max, losses, 2)
rep.sync()
np.savez(out, params=rep.params.cpu().numpy(), losses=losses[:n].cpu().numpy(), n=n, u=rep.updates())
sched.close()
rep.close()
