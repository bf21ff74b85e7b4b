#!/usr/bin/env python
"""Benchmark of the Adaptive SGD hot path on B200: whole-box samples/s of the
local SGD steps + normalized merge (BASELINE.json metric).

A bench "step" is one mega-batch: M = 100 b_max samples routed batch by
batch to the ranks by the dynamic scheduler, one local SGD step per batch,
then the merge (Alg. 2) and batch size scaling (Alg. 1) -- every row of
DESIGN.md's hot-path table.  Default workload: EURLex-4K-shaped
(BASELINE.json configs[1], 1 B200).  Inputs are resident in HBM when the
timed region starts; L2 is flushed (256 MiB write) between timed steps,
outside the timed events.  `e2e` repeats the measurement through the C ABI
with host (pinned) buffers: every step copies its mega-batch CSR host->device
and reads its losses back.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config NAME]
                    [--precision auto|fp32|bf16] [--impl ours|reference]
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "samples/s (whole box) of local SGD step+merge"
UNIT = "samples/s"


def _args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--config", default="eurlex4k")
    p.add_argument("--precision", default="auto", choices=["auto", "fp32", "bf16"])
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--inflight", type=int, default=2)
    p.add_argument("--method", default="adaptive", choices=["adaptive", "elastic"],
                   help="adaptive: dynamic tickets + Alg. 1/2; elastic: Elastic SGD A/B (static batches, alpha = 1/N)")
    p.add_argument("--merge", default="fused", choices=["fused", "nccl"],
                   help="fused: peer-memory merge kernel over CUDA IPC (NEXT-1); nccl: prescale + all_reduce + epilogue")
    p.add_argument("--loss", default="softmax", choices=["softmax", "sigmoid"],
                   help="output head: softmax-CE (the paper's) or per-label sigmoid BCE (R11)")
    p.add_argument("--norm", default="u", choices=["u", "ub"],
                   help="Alg. 2 line 3: u_i-normalised (the paper's default) or u_i b_i (R12, P:1088-1090)")
    p.add_argument("--scale-every", type=int, default=1,
                   help="run Alg. 1 after every k-th mega-batch (R13, P:922-925; 1 = the paper's default; "
                        "0 = the adaptive frequency of R17)")
    p.add_argument("--e2e-steps", type=int, default=None)
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--cpu-seconds", type=float, default=12.0)
    p.add_argument("--ttp-megabatches", type=int, default=40, help="time-to-P@1 budget (0 = skip)")
    p.add_argument("--lr-max", type=float, default=None)
    p.add_argument("--train-rows", type=int, default=None, help="generate only the first N train rows")
    return p.parse_args()


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
                "sm_max_mhz": 1965.0}, "fallback"


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """NVML sampling of SM clock and throttle reasons during the timed region."""

    REASONS = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown",
               0x4: "sw_power_cap", 0x80: "hw_power_brake_slowdown"}

    def __init__(self, index: int, period: float = 0.01):
        self.index, self.period = index, period
        self.samples, self.reasons = [], set()
        self._stop = threading.Event()
        self.ok = False
        self.max_mhz = None
        if index < 0:   # disabled
            return
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.max_mhz = None

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.ok:
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                    "samples": 0}
        return {"sm_mhz": float(statistics.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------ CPU oracle
def cpu_baseline(cfg, data, budget_s: float, loss: str = "softmax"):
    """The oracle as it stands (fp64 numpy/scipy) on the host cores: consecutive
    b_max-row local steps of the same workload plus the per-mega-batch merge,
    amortised over the mega-batch's 100 steps."""
    from oracle import merge as omerge, model as omodel
    from synth import init_params, sample_stream
    cores, cpu_model, blas_threads = host_cores()
    w = init_params(cfg).astype(np.float64)
    b = cfg.b_max
    steps, samples = 0, 0
    t0 = time.perf_counter()
    while True:
        rows = sample_stream(cfg, steps * b, b)
        w, _, _ = omodel.sgd_step(w, data.row_slice(rows), cfg.lr_max, cfg.F, cfg.H, cfg.L, loss)
        steps += 1
        samples += b
        if time.perf_counter() - t0 > budget_s:
            break
    t_steps = time.perf_counter() - t0
    t1 = time.perf_counter()
    omerge.merge_models([w], [1.0], w, np.zeros_like(w), 0.9)
    t_merge = time.perf_counter() - t1
    steps_per_mb = cfg.mega_batch // b
    t_total = t_steps + t_merge * steps / steps_per_mb
    return {"value": samples / t_total, "unit": UNIT, "cores": int(cores), "kind": "oracle",
            "cpu_model": cpu_model, "blas_threads": blas_threads,
            "sample": f"{steps} local steps x {b} rows of {cfg.name} (fp64 numpy/scipy oracle) + "
                      f"merge amortised over {steps_per_mb} steps/mega-batch"}, t_total


def host_cores():
    """the cores the oracle may use = len(os.sched_getaffinity(0)), the
    CPU model from lscpu, and the BLAS thread pool size actually in use."""
    cores = len(os.sched_getaffinity(0))
    model = None
    try:
        import subprocess
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        model = next((ln.split(":", 1)[1].strip() for ln in out.splitlines() if ln.startswith("Model name")), None)
    except Exception:
        pass
    try:
        from threadpoolctl import threadpool_info
        blas = max([i.get("num_threads", 1) for i in threadpool_info()] + [1])
    except Exception:
        blas = None
    return cores, model, blas


# ------------------------------------------------------------------ roofline
def kernel_work(cls: str, cfg, bf16: bool, st, loss: str = "softmax"):
    """Algorithmic (bytes, flops) of one launch of a kernel class (DESIGN.md §5,
    SURVEY.md §8(d)): operands read once, outputs written once, no credit for
    cache reuse across kernels.  Logits traffic (Z, dZ), the W2 operand shadow's
    refresh and the fused softmax's Z recompute are IMPLEMENTATION bytes / flops
    (§8(d)) and are not counted: they show up as ncu traffic above the
    algorithmic bytes.  GEMM operands count in the precision the path feeds the
    tensor cores (bf16: 2 B; fp32 path: bf16x3 hi + lo, 4 B).  The kernel's bound
    is whichever of bytes / HBM peak and flops / compute peak is larger
    (`roofline_of`)."""
    B, H, L, F, P = st["B"], cfg.H, cfg.L, cfg.F, cfg.n_params
    nnz, U = st["nnz"], st["U"]
    e = 2.0 if bf16 else 4.0                      # bytes per GEMM operand element
    gemm = 2.0 * B * H * L
    if cls == "g1":     # Z = H1 . W2^T + b2: W2 and H1 operands, b2
        return (e * H * L + e * B * H + 4.0 * L, gemm)
    if cls == "g2":     # dH1 = dZ . W2: the W2 operand in, dH1 out (dZ is logits traffic)
        return (e * H * L + 4.0 * B * H, gemm)
    if cls == "g3":     # W2 -= lr dZ^T H1, b2 -= lr 1^T dZ: W2 and b2 read + written (fp32), the H1 operand
        return (8.0 * H * L + 8.0 * L + e * B * H, gemm)
    if cls == "spmm":
        return (8.0 * nnz + 12.0 * B + 4.0 * U * H + 4.0 * B * H, 2.0 * nnz * H)
    if cls == "scatter":
        return (8.0 * nnz + 4.0 * B * H + 8.0 * U * H, 2.0 * nnz * H)
    if cls == "softmax":   # the row loss from the labels; Z in / dZ out are logits traffic
        return (8.0 * st["nlab"] + 4.0 * B, 0.0)
    if cls == "touched":
        return (4.0 * nnz + 12.0 * nnz + 8.0 * F + 12.0 * B, 0.0)
    if cls == "dh_b1":
        return (4.0 * st.get("splitk", 1) * B * H + 8.0 * B * H, 0.0)
    if cls == "merge":
        return (12.0 * P, 0.0)   # 36 P per mega-batch over its 3 launches
    return (0.0, 0.0)


def roofline_of(cls, cfg, bf16, st, loss, avg_s, peaks):
    """Bound, achieved, peak and unit of one kernel class from its algorithmic
    (bytes, flops) per launch and its measured average launch time.  Tensor peak:
    the measured bf16 one (sustained: the kernels run inside a long step); the
    fp32 path issues three bf16 MMAs per product (bf16x3, R14), so its
    contraction ceiling is a third of it."""
    by, fl = kernel_work(cls, cfg, bf16, st, loss)
    hbm = peaks["hbm_gbs"]
    cpk, cb = peaks.get("bf16_tflops_sustained", peaks["bf16_tflops"]), "tensor"
    if not bf16:
        cpk = cpk / 3.0
    if cls in ("spmm", "scatter"):   # CUDA-core FMAs
        cpk, cb = 148 * 128 * 2 * peaks.get("sm_max_mhz", 1965.0) * 1e6 / 1e12, "alu"
    if fl / (cpk * 1e12) > by / (hbm * 1e9):
        return {"bound": cb, "achieved": fl / avg_s / 1e12, "peak": cpk, "unit": "TFLOP/s",
                "work_per_launch": fl}
    return {"bound": "hbm", "achieved": by / avg_s / 1e9, "peak": hbm, "unit": "GB/s", "work_per_launch": by}


def l2_view(cls, cfg, bf16, st, avg_s):
    """Secondary roofline for the sparse kernels, whose operands are L2-resident at
    EURLex size: the bytes they actually move through L2 per launch (K-1: fp32 W1 row
    gathers 4 nnz H + entries 8 nnz + H1 fp32/bf16 6 B H; K-5: W1 rows read and
    written 8 U H + entries 16 nnz + each CTA's staged dA1 slice) over the launch time,
    against the L2-resident copy bandwidth measured by tools/l2_peak.py."""
    try:
        with open(os.path.join(ROOT, "profiles", "l2_peak.json")) as f:
            peak = float(json.load(f)["l2_gbs"])
    except Exception:
        return None
    B, H, nnz, U = st["B"], cfg.H, st["nnz"], st["U"]
    if cls == "spmm":
        by = 4.0 * nnz * H + 8.0 * nnz + 6.0 * B * H
    elif cls == "scatter":
        elem = 2 if bf16 else 4
        cs = next((c for c in (256, 128, 64) if c <= H and H % c == 0 and cfg.b_max * c * elem <= 160 * 1024), H)
        by = 8.0 * U * H + 16.0 * nnz + 148.0 * B * cs * elem   # 148 CTAs each stage a B x cs slice
    else:
        return None
    ach = by / avg_s / 1e9
    return {"bytes_per_launch": by, "achieved": round(ach, 1), "peak": peak, "unit": "GB/s",
            "frac": round(ach / peak, 4), "peak_source": "profiles/l2_peak.json (torch copy, L2-resident)"}


def step_ideal_s(cfg, B, nnz, U, nlab, hbm_gbs, tc_tflops):
    """SURVEY.md §8(d) ideal time of one local step: max(algorithmic HBM bytes /
    HBM peak, algorithmic flops / tensor peak).  Bytes: 8 nnz + 12 B + 4 labels
    + 8 U H (touched W1 rows read+written) + 8 (H L + L) (W2/b2 read+written)
    + 8 H (b1); flops: 6 B H L (G1-G3) + 4 nnz H (K-1, K-5)."""
    H, L = cfg.H, cfg.L
    by = 8.0 * nnz + 12.0 * B + 4.0 * nlab + 8.0 * U * H + 8.0 * (H * L + L) + 8.0 * H
    fl = 6.0 * B * H * L + 4.0 * nnz * H
    return max(by / (hbm_gbs * 1e9), fl / (tc_tflops * 1e12))


def main():
    a = _args()
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    if a.impl == "reference":
        return reference_arm(a, rank, world)

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_marws22_b200 import api, train, _lib
    from synth import config, generate, init_params, sample_stream

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    cfg = config(a.config)
    prec = a.precision
    if prec == "auto":
        prec = "bf16" if _bf16_available() else "fp32"
    bf16 = prec == "bf16"
    data = generate(cfg, "train", a.train_rows)
    if a.train_rows:
        cfg = config(a.config, n_train=data.n_rows)
    w0 = init_params(cfg)
    nz, nl = api.max_step_sizes([data], cfg.b_max)
    rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, prec, device=local, w0=w0, loss=a.loss)
    dd = api.DeviceCsr(data, device=dev)
    rep.register(dd)
    h = train.Hyper.from_config(cfg, norm=a.norm, scale_every=a.scale_every)
    M = h.M
    shm = f"/asgd_bench_{os.environ.get('MASTER_PORT', os.getpid())}"
    if rank == 0:
        sched = api.Scheduler(shm, world, M, create=True)
    if world > 1:
        dist.barrier()
    if rank != 0:
        sched = api.Scheduler(shm, world, M, create=False)
    # the fused merge falls back to NCCL on EVERY rank when any rank cannot map its peers
    drv = train.DistributedAdaptiveSGD(rep, h, rank, world, sched, inflight=a.inflight, merge=a.merge,
                                       method=a.method)
    merge_used = drv.merge if not drv.merge_note else f"{drv.merge} (fused unavailable: {drv.merge_note})"
    K, W = a.steps, a.warmup
    Ke = a.e2e_steps if a.e2e_steps is not None else min(K, 10)
    ids = [sample_stream(cfg, mb * M, M) for mb in range(W + K + Ke)]
    rows_d = [torch.as_tensor(x, device=dev) for x in ids[:W + K]]
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    # warm-up with every kernel class timed: picks the dominant kernel, whose
    # launches alone are then timed live in the timed region (2 events/step).
    call = _lib.call
    NCLS = len(_lib.PROF_NAMES)
    call("asgd_profile", rep.ctx, (1 << NCLS) - 1)
    for mb in range(W):
        drv.megabatch(rows_d[mb])
    torch.cuda.synchronize()
    wms = np.zeros(NCLS, dtype=np.float64)
    wcnt = np.zeros(NCLS, dtype=np.int64)
    call("asgd_profile_read", rep.ctx, wms.ctypes.data, wcnt.ctypes.data)
    # dominant kernel: the largest per-step time among the kernels on the step's critical
    # path.  K-0 (`touched`) runs on side stream s2 after K-1 (its phase A folded into K-1), beside G1..G2, joined only
    # before K-5, so its duration does not bound the step; it is reported under
    # `side_stream` with its own roofline.
    crit = [i for i in range(NCLS) if _lib.PROF_NAMES[i] != "touched" and wcnt[i]]
    dom = max(crit, key=lambda i: wms[i]) if crit else int(np.argmax(wms))

    # ---------------------------------------------------------------- timed
    # pass 1 (the headline): K mega-batches with no profiling nodes in the step graph.
    # pass 2: the same K mega-batches again with CUDA events around every launch of the
    # dominant kernel class (live, on the stream it runs on) -> its average duration
    # for the roofline.  Event nodes on the critical path add latency, so they stay
    # out of the headline pass.
    def timed_pass(mask, sample_clocks, time_merge=False):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        drv.time_merge = time_merge
        call("asgd_profile", rep.ctx, mask)
        l0 = rep.launches()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
        st_l = []
        with ClockSampler(local if sample_clocks else -1) as clk:
            for k in range(K):
                flush.zero_()
                ev[k][0].record()
                st_l.append(drv.megabatch(rows_d[W + k], keep_log=True))
                ev[k][1].record()
            torch.cuda.synchronize()
        nl = rep.launches() - l0
        ms_ = np.zeros(NCLS, dtype=np.float64)
        cnt_ = np.zeros(NCLS, dtype=np.int64)
        call("asgd_profile_read", rep.ctx, ms_.ctypes.data, cnt_.ctypes.data)
        call("asgd_profile", rep.ctx, 0)
        drv.time_merge = False
        return sum(e0.elapsed_time(e1) for e0, e1 in ev), st_l, nl, ms_, cnt_, clk

    t_ms, stats, launches, _, _, clk = timed_pass(0, True)
    # pass 2 also times the merge phase (end of the rank's local steps -> merged model, which
    # includes waiting for the slowest rank at the statistics all-gather) and the merge kernels
    i_merge = _lib.PROF_NAMES.index("merge")
    t_prof_ms, stats2, _, ms, cnt, _ = timed_pass((1 << dom) | (1 << i_merge), False, time_merge=True)
    merge_ms = float(np.mean([s_.merge_events[0].elapsed_time(s_.merge_events[1]) for s_ in stats2]))
    mk_ms = float(ms[i_merge]) / K   # the merge kernels' time per mega-batch
    mt = torch.tensor([merge_ms, mk_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(mt, op=dist.ReduceOp.MAX)
    merge_ms, mk_ms = float(mt[0].item()), float(mt[1].item())
    t = torch.tensor([t_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    t_max = float(t.item())
    value = K * M / (t_max / 1e3)

    # ---------------------------------------------------------------- e2e
    e2e = None
    if Ke > 0:
        e2e = run_e2e(rep, drv, data, ids[W + K:W + K + Ke], dev, flush, world, M)

    if rank == 0:
        peaks, src = _peaks()
        # per-step workload statistics from the routing logs of the timed region
        B_list, nnz_l, U_l, lab_l = [], [], [], []
        lens = np.diff(data.row_ptr)
        llens = np.diff(data.lab_ptr)
        for k, s in enumerate(stats):
            for _, r, st, n in s.routes:
                rr = ids[W + k][st:st + n]
                B_list.append(n)
                nnz_l.append(int(lens[rr].sum()))
                lab_l.append(int(llens[rr].sum()))
                U_l.append(len(np.unique(np.concatenate([data.col[data.row_ptr[i]:data.row_ptr[i + 1]] for i in rr]))))
        wl = {"B": float(np.mean(B_list)), "nnz": float(np.mean(nnz_l)), "U": float(np.mean(U_l)),
              "nlab": float(np.mean(lab_l)), "splitk": 0}
        from paper_conf_ipps_marws22_b200.api import _lib as L_
        names = L_.PROF_NAMES
        per = {names[i]: {"us_per_launch": round(float(wms[i] / wcnt[i] * 1e3), 3) if wcnt[i] else None,
                          "launches": int(wcnt[i])}
               for i in range(len(names))}
        dname = names[dom]
        avg_s = ms[dom] / max(cnt[dom], 1) / 1e3
        r = roofline_of(dname, cfg, bf16, wl, a.loss, avg_s, peaks)
        traffic = _traffic(cfg.name, prec, dname)
        roof = {"bound": r["bound"], "achieved": round(r["achieved"], 3), "peak": round(r["peak"], 3),
                "unit": r["unit"], "frac": round(r["achieved"] / r["peak"], 4), "traffic": traffic,
                "kernel": dname, "peak_source": src, "work_per_launch": r["work_per_launch"],
                "step_share": round(float(ms[dom] / max(t_prof_ms, 1e-9)), 4),
                "timed_in": f"second pass of {K} mega-batches with CUDA events around each launch "
                            f"({t_prof_ms / K:.4f} ms per mega-batch there vs {t_ms / K:.4f} ms unprofiled)"}
        lv = l2_view(dname, cfg, bf16, wl, avg_s)
        if lv:
            roof["l2_view"] = lv
        side = {}
        for i in range(len(names)):
            if names[i] == "touched" and wcnt[i]:
                s_avg = wms[i] / wcnt[i] / 1e3
                rs = roofline_of("touched", cfg, bf16, wl, a.loss, s_avg, peaks)
                side["touched"] = {"us_per_launch": round(s_avg * 1e6, 3), "bound": rs["bound"],
                                   "frac": round(rs["achieved"] / rs["peak"], 4),
                                   "note": "side stream s2 after K-1 (phase A folded into K-1), overlapped with G1..G2 (warm-up profile)"}
        # whole-job roofline: sum of per-step ideal times with
        # each step's measured B, nnz, U, + merge 36 P bytes / HBM peak, over the timed time
        tc_peak = peaks.get("bf16_tflops_sustained", peaks["bf16_tflops"]) / (1.0 if bf16 else 3.0)
        t_ideal = sum(step_ideal_s(cfg, b_, z_, u_, l_, peaks["hbm_gbs"], tc_peak)
                      for b_, z_, u_, l_ in zip(B_list, nnz_l, U_l, lab_l))
        t_ideal += K * 36.0 * cfg.n_params / (peaks["hbm_gbs"] * 1e9)
        roof["whole_step_frac"] = round(t_ideal / world / (t_max / 1e3), 4)
        # merge share of a mega-batch; fused merge: NVLink bytes per rank =
        # every remote shard read (4 P (N-1)/N) and w' written back to every peer (same)
        merge_info = {"ms_per_megabatch": round(merge_ms, 4), "kernel_ms_per_megabatch": round(mk_ms, 4),
                      "fraction": round(merge_ms / max(t_prof_ms / K, 1e-9), 4), "kind": merge_used,
                      "hbm_bytes_alg": 36 * cfg.n_params,
                      "measured_in": "pass 2 (CUDA events from the end of the rank's local steps to the merged "
                                     "model; max over ranks)"}
        if world > 1 and str(merge_used).startswith("fused") and mk_ms > 0:
            nvb = 8.0 * cfg.n_params * (world - 1) / world
            merge_info["nvlink"] = {"bytes_per_rank": int(nvb), "GB/s": round(nvb / (mk_ms / 1e3) / 1e9, 1),
                                    "peak": 900.0, "note": "bytes / merge-kernel time (per direction peak 900 GB/s)"}
        out = {
            "metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": world, "steps": K,
            "warmup": W, "ms_per_step": round(t_max / K, 4), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "bf16" if bf16 else "f32",
            "data": "synthetic",
            "config": {"workload": cfg.name, "train_rows": int(data.n_rows), "F": cfg.F, "L": cfg.L, "H": cfg.H, "b_max": cfg.b_max,
                       "mega_batch_samples": M, "step": "1 mega-batch = local steps + merge",
                       "precision": prec, "l2": "flushed (256 MiB write) between timed steps",
                       "inflight": a.inflight, "parallelism": f"dp{world} (model averaging)",
                       "merge": merge_used, "method": a.method, "loss": a.loss,
                       "norm": a.norm, "scale_every": a.scale_every,
                       "mean_batch_nnz": round(wl["nnz"], 1), "mean_touched_rows": round(wl["U"], 1)},
            "roofline": roof,
            "merge": merge_info,
            "side_stream": side,
            "kernels_warmup_profile": per,
            "gpu_launches": int(launches),
            "clocks": clk.summary(),
            "e2e": e2e,
            "cpu_baseline": None,
        }
    if a.ttp_megabatches > 0:   # every rank trains; rank 0 evaluates after each merge (untimed)
        ttp = time_to_p1(cfg, prec, a.ttp_megabatches, dev, rank, world, lr_max=a.lr_max, loss=a.loss,
                         norm=a.norm, scale_every=a.scale_every, merge=a.merge, method=a.method)
        if rank == 0:
            out["time_to_p1"] = ttp
    if rank == 0:
        if world == 1 and not a.no_cpu_baseline:
            out["cpu_baseline"], _ = cpu_baseline(cfg, data, a.cpu_seconds, a.loss)
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.barrier()
    sched.close()
    if world > 1:
        dist.destroy_process_group()


def _bf16_available() -> bool:
    try:
        from paper_conf_ipps_marws22_b200 import _lib
        return "bf16-ready" in _lib.lib().asgd_version().decode()
    except Exception:
        return False


def _traffic(workload: str, prec: str, cls: str):
    """dram read+write bytes per launch of the kernel class, from the committed
    `ncu --set full` capture (profiles/traffic.json, tools/ncu_traffic.py)."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            return json.load(f)[f"{workload}/{prec}"]["per_launch_bytes"].get(cls)
    except Exception:
        return None


def run_e2e(rep, drv, data, ids_list, dev, flush, world, M):
    """Same metric through the C ABI from HOST buffers: per mega-batch, the H2D copy of its
    CSR from pinned memory (asgd_data_stage on a copy stream, into one of two device staging
    buffers, issued one mega-batch ahead so that it overlaps the previous mega-batch's
    steps), asgd_data_use, the mega-batch, and a D2H read of its losses.  Timed from the
    first copy to the last loss read (L2 flushes between mega-batches inside)."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_marws22_b200 import api
    hosts = [api.DeviceCsr(data.row_slice(x), device="cpu", pin=True) for x in ids_list]
    big = max(hosts, key=lambda hh: hh.nnz)
    stages = []
    for _ in range(2):
        stg = api.DeviceCsr.empty_like(big, device=dev)
        stg.col = torch.empty(max(hh.nnz for hh in hosts), dtype=torch.int32, device=dev)
        stg.val = torch.empty(max(hh.nnz for hh in hosts), dtype=torch.float32, device=dev)
        stg.lab = torch.empty(max(hh.n_lab for hh in hosts), dtype=torch.int32, device=dev)
        stg.nnz, stg.n_lab = stg.col.numel(), stg.lab.numel()
        stages.append(stg)
    ident = torch.arange(M, dtype=torch.int32, device=dev)
    Ke = len(hosts)
    loss_host = torch.zeros(Ke, drv.losses.numel(), dtype=torch.float32).pin_memory()
    copy = torch.cuda.Stream(device=dev)
    main = torch.cuda.current_stream(dev)
    done = [torch.cuda.Event(), torch.cuda.Event()]   # mega-batch using staging buffer b finished
    h2d = d2h = 0

    def stage(i):
        b = i % 2
        if i >= 2:
            copy.wait_event(done[b])   # the mega-batch that read this buffer is done
        rep.stage(hosts[i], stages[b], copy)

    # untimed: two mega-batches from each staging buffer (the step graphs are cached per
    # dataset: the first use of a buffer runs eagerly, the second captures)
    for i in range(4):
        rep.stage(hosts[i % Ke], stages[i % 2], None)
        rep.use(stages[i % 2], hosts[i % Ke].nnz, hosts[i % Ke].n_lab)
        drv.megabatch(ident)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    copy.wait_stream(main)
    stage(0)
    for i, hh in enumerate(hosts):
        if i + 1 < Ke:
            stage(i + 1)               # overlaps mega-batch i
        flush.zero_()
        rep.use(stages[i % 2], hh.nnz, hh.n_lab)
        st = drv.megabatch(ident)
        n = st.n_steps
        rep.copy_to_host(loss_host[i, :n], drv.losses[:n])
        done[i % 2].record(main)
        h2d += 8 * (hh.n_rows + 1) * 2 + 8 * hh.nnz + 4 * hh.n_lab
        d2h += 4 * n
    e1.record()
    torch.cuda.synchronize()
    t = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return {"value": round(Ke * M / (float(t.item()) / 1e3), 1), "unit": UNIT,
            "h2d_bytes_per_step": int(h2d * world / Ke), "d2h_bytes_per_step": int(d2h * world / Ke),
            "overlap": "mega-batch k+1's H2D copies (copy stream, second staging buffer) overlap mega-batch k's steps"}


def frozen_p1_target(name: str):
    """The per-config P@1 target frozen in configs/p1_targets.json (SURVEY §8(d):
    floor + 0.9 (p_best - floor), p_best = the best P@1 of the 1-GPU fp32 run
    within its budget), or None."""
    try:
        with open(os.path.join(ROOT, "configs", "p1_targets.json")) as f:
            return json.load(f).get(name)
    except Exception:
        return None


def time_to_p1(cfg, prec, n_mb, dev, rank=0, world=1, pert_renorm=False, lr_max=None, eval_rows=10000,
               loss="softmax", norm="u", scale_every=1, merge="fused", method="adaptive"):
    """Time-to-P@1 at N = world GPUs (Fig. 5a): cumulative
    device time of the mega-batches (local steps + merge, max over ranks) until test
    P@1 first reaches the target.  The target is the frozen per-config one
    (configs/p1_targets.json) when present, else floor + 0.9 (best - floor) of this
    run (self-referential, labelled so).  floor = the majority-label P@1 of the test
    subset.  Every rank trains a fresh replica from w0 with the same dynamic
    scheduler; rank 0 evaluates P@1 on the global model after every merge, outside
    the timed region.  Returns the record on rank 0, None elsewhere."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_marws22_b200 import api, train
    from synth import generate, init_params, sample_stream
    data = generate(cfg, "train")
    test = generate(cfg, "test", eval_rows)
    nz, nl = api.max_step_sizes([data, test], cfg.b_max)
    rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, prec, device=dev.index or 0, w0=init_params(cfg),
                      loss=loss)
    rep.register(api.DeviceCsr(data, device=dev))
    td = api.DeviceCsr(test, device=dev) if rank == 0 else None
    h = train.Hyper.from_config(cfg, pert_renorm=pert_renorm, norm=norm, scale_every=scale_every,
                                **({"lr_max": lr_max} if lr_max else {}))
    shm = f"/asgd_ttp_{os.environ.get('MASTER_PORT', os.getpid())}"
    if rank == 0:
        sched = api.Scheduler(shm, world, h.M, create=True)
    if world > 1:
        dist.barrier()
    if rank != 0:
        sched = api.Scheduler(shm, world, h.M, create=False)
    drv = train.DistributedAdaptiveSGD(rep, h, rank, world, sched, merge=merge, method=method)
    rows = np.arange(test.n_rows, dtype=np.int32)
    counts = np.bincount(test.lab, minlength=cfg.L)
    floor = float(np.mean([counts.argmax() in set(test.lab[test.lab_ptr[i]:test.lab_ptr[i + 1]].tolist())
                           for i in range(test.n_rows)]))
    curve, t_ms, work, steps = [], 0.0, [], 0
    for mb in range(n_mb):
        ids = torch.as_tensor(sample_stream(cfg, mb * h.M, h.M), device=dev)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        st = drv.megabatch(ids)
        e1.record()
        torch.cuda.synchronize()
        tt = torch.tensor([e0.elapsed_time(e1), float(st.n_steps)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(tt[:1], op=dist.ReduceOp.MAX)
            dist.all_reduce(tt[1:], op=dist.ReduceOp.SUM)
        t_ms += float(tt[0].item())
        steps += int(tt[1].item())
        work.append((steps, (mb + 1) * h.M / data.n_rows))
        if rank == 0:
            p1 = train.precision_at_k(rep, td, test, rows, 1)
            curve.append((round(t_ms / 1e3, 5), round(p1, 5)))
        if world > 1:
            dist.barrier()
    if world > 1:
        dist.barrier()
    sched.close()
    rep.close()
    if rank != 0:
        return None
    best = max(p for _, p in curve)
    frozen = frozen_p1_target(cfg.name)
    if frozen:
        target, floor_used, src = float(frozen["target_p1"]), float(frozen["p1_floor"]), "frozen"
    else:
        target, floor_used, src = floor + 0.9 * (best - floor), floor, "this run's best (self-referential)"
    k_hit = next((k for k, (t, p) in enumerate(curve) if p >= target), None)
    hit = curve[k_hit][0] if k_hit is not None else None
    # statistical efficiency (Fig. 5b): local steps (all ranks) and passes to the target
    return {"value": hit, "unit": "s", "n_gpus": world, "target_p1": round(target, 5), "target_source": src,
            "frozen": frozen, "p1_floor": round(floor_used, 5),
            "steps_to_target": work[k_hit][0] if k_hit is not None else None,
            "passes_to_target": round(work[k_hit][1], 4) if k_hit is not None else None,
            "p1_best": round(best, 5), "mega_batches": n_mb, "pert_renorm": pert_renorm,
            "lr_max": h.lr_max, "test_rows": int(test.n_rows), "precision": prec, "merge": drv.merge,
            "method": method, "curve_every_4": curve[::4],
            "note": "parity unpinned (the paper prints no time-to-accuracy values)"}


def reference_arm(a, rank, world):
    """--impl reference: the CPU oracle, as it stands, on the host cores."""
    if rank != 0:
        return
    from synth import config, generate
    cfg = config(a.config)
    data = generate(cfg, "train")
    per_step = max(1.0, min(a.cpu_seconds, 20.0) / max(1, a.steps))
    vals, secs = [], []
    base = None
    for k in range(a.warmup + a.steps):
        cb, t_s = cpu_baseline(cfg, data, per_step, a.loss)
        if k >= a.warmup:
            vals.append(cb["value"])
            secs.append(t_s)
            base = cb
    v = float(np.mean(vals))
    base["value"] = round(v, 2)
    # a timed step is one bounded sample of the workload (cpu_baseline's budget), its wall time
    out = {"metric": METRIC, "value": round(v, 2), "unit": UNIT, "n_gpus": world, "steps": a.steps,
           "warmup": a.warmup, "ms_per_step": round(1e3 * float(np.mean(secs)), 3), "higher_is_better": True,
           "scaling": "strong",
           "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
           "config": {"workload": cfg.name, "F": cfg.F, "L": cfg.L, "H": cfg.H, "b_max": cfg.b_max,
                      "mega_batch_samples": cfg.mega_batch, "loss": a.loss},
           "cpu_baseline": base,
           "e2e": {"value": round(v, 2), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
