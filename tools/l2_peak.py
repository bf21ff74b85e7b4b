"""L2-resident copy bandwidth of this B200 (a denominator for the L2-resident
EURLex kernels; MEASURED_PEAKS.json has only HBM and bf16 figures).

    python tools/l2_peak.py > profiles/l2_peak.json

b.copy_(a) over buffers that fit in L2 together (a + b up to 2 x 48 MB of the 126 MB
L2), 200 back-to-back copies after warm-up, CUDA events; read + write bytes.
"""
import json

import torch


def main():
    out = {}
    for mb in (16, 32, 40, 48):
        n = mb << 20
        a = torch.empty(n, dtype=torch.uint8, device="cuda")
        b = torch.empty(n, dtype=torch.uint8, device="cuda")
        a.fill_(1)
        for _ in range(20):
            b.copy_(a)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 200
        e0.record()
        for _ in range(reps):
            b.copy_(a)
        e1.record()
        torch.cuda.synchronize()
        s = e0.elapsed_time(e1) / 1e3
        out[f"copy_{mb}MB_GBs"] = round(2 * n * reps / s / 1e9, 1)
    out["l2_gbs"] = max(v for k, v in out.items() if k.startswith("copy_"))
    out["how"] = "torch b.copy_(a), a and b together <= 96 MB (L2-resident), 200 copies, CUDA events, read+write bytes"
    out["gpu"] = torch.cuda.get_device_name()
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
