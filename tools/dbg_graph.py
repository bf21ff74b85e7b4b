import torch, numpy as np, traceback
from synth import config, generate, init_params, sample_stream
from paper_conf_ipps_marws22_b200 import api
cfg = config("tiny")
data = generate(cfg, "train")
for prec in ("fp32", "bf16"):
    nz, nl = api.max_step_sizes([data], cfg.b_max)
    rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, prec, device=0, w0=init_params(cfg))
    dd = api.DeviceCsr(data, device="cuda:0"); rep.register(dd)
    rows = torch.as_tensor(sample_stream(cfg, 0, 320), device="cuda:0")
    loss = torch.zeros(16, device="cuda:0")
    try:
        for k in range(6):
            rep.step(rows[32 * k:32 * k + 32], 0.5, loss[k:k + 1])
        torch.cuda.synchronize()
        print(prec, "ok", loss[:6].tolist(), "launches", rep.launches())
    except Exception as e:
        traceback.print_exc()
