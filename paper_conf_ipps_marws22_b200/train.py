"""Adaptive SGD driver: mega-batches of dynamically routed local steps, then
the normalized merge and batch size scaling (§III, P:619-1160;
§IV).

Two drivers over the same libasgd calls:
  * DistributedAdaptiveSGD -- one process per GPU (torch.distributed); batches
    come from the cross-process shm ticket scheduler; the merge is prescale
    (K-6) -> one all-reduce SUM (NCCL over NVLink) -> momentum epilogue (K-7).
  * SimulatedAdaptiveSGD -- N replicas on one GPU, routed by the simulated
    clock (or replayed); the all-reduce is replaced by the in-device weighted
    sum (the parity configuration of BASELINE.json configs[0]).
The host logic that sits between the kernels (ticket loop, statistics
exchange + Alg. 2 weights, Alg. 1) is written device-agnostic so the gloo CPU
tests exercise it unchanged.
"""
from __future__ import annotations

import dataclasses
import math
from typing import Callable, List, Optional, Sequence

import numpy as np
import torch
import torch.distributed as dist

from . import api


@dataclasses.dataclass
class Hyper:
    b_max: int
    b_min: int
    beta: int
    lr_max: float
    M: int                      # mega-batch samples (Q8)
    gamma: float = 0.9
    delta: float = 0.1
    pert_thr: float = 0.1
    pert_renorm: bool = False   # Q34 option (literal Alg. 2 by default)
    norm: str = "u"             # Alg. 2 line 3: "u", or "ub" = u_i b_i (R12)
    scale_every: int = 1        # Alg. 1 after every scale_every-th mega-batch (R13);
                                # 0: the adaptive frequency of R17 (asgd_scale_frequency)
    max_interval: int = 8       # R17's longest interval

    def __post_init__(self):
        if self.norm not in ("u", "ub"):
            raise ValueError(f"norm must be 'u' or 'ub', got {self.norm!r}")
        if self.scale_every < 0:
            raise ValueError(f"scale_every must be >= 0, got {self.scale_every}")

    @classmethod
    def from_config(cls, cfg, **kw):
        h = dict(b_max=cfg.b_max, b_min=cfg.b_min, beta=cfg.beta, lr_max=cfg.lr_max, M=cfg.mega_batch)
        h.update(kw)
        return cls(**h)


class ScaleClock:
    """When Alg. 1 runs (R13: every k-th mega-batch; R17: the adaptive frequency)."""

    def __init__(self, hyper: "Hyper", n: int):
        self.h = hyper
        self.interval, self.countdown, self.signs = 1, 1, [0] * n

    def step(self, mb: int, u, b):
        """Alg. 1 after mega-batch mb if due; returns (b, lr) or None."""
        h = self.h
        if h.scale_every > 0:
            if (mb + 1) % h.scale_every:
                return None
            return api.scale_batches(u, b, h.b_min, h.b_max, h.beta, h.lr_max)
        self.countdown -= 1
        if self.countdown:
            return None
        b_new, lr = api.scale_batches(u, b, h.b_min, h.b_max, h.beta, h.lr_max)
        self.interval, self.signs = api.scale_frequency(b, b_new, self.signs, self.interval, h.max_interval)
        self.countdown = self.interval
        return b_new, lr


@dataclasses.dataclass
class MegaBatchStats:
    mb: int
    u: List[int]
    b: List[int]
    lr: List[float]
    nu: List[float]
    alpha: List[float]
    r: int
    s: int
    perturbed: bool
    routes: list
    n_steps: int
    merge_events: Optional[tuple] = None   # (start, end) CUDA events of the merge phase (time_merge)


# --------------------------------------------------------------- host logic
def run_tickets(sched: api.Scheduler, rank: int, b_i: int,
                step: Callable[[int, int, int], None], inflight: int = 2,
                wait: Optional[Callable[[int], None]] = None) -> int:
    """Take tickets until the mega-batch is exhausted.

    step(k, start, len) enqueues local step k; wait(k) blocks until step k
    finished.  With inflight = 1 a rank asks for its next batch only after
    its previous step completed (paper-faithful); inflight = 2 lets the host
    take the next ticket while one step is still running (reading Q32)."""
    k = 0
    while True:
        if wait is not None and k >= inflight:
            wait(k - inflight)
        t = sched.next(rank, b_i)
        if t is None:
            return k
        step(k, t[0], t[1])
        k += 1


def exchange_stats(u: int, b: int, sqnorm: torch.Tensor, P: int, world: int,
                   group=None):
    """All-gather (u_i, b_i, ||w_i||^2) and return host lists + nu = ||w||_2 / P.

    sqnorm: fp64 scalar tensor on the collective's device."""
    dev = sqnorm.device
    mine = torch.stack([torch.tensor(float(u), dtype=torch.float64, device=dev),
                        torch.tensor(float(b), dtype=torch.float64, device=dev),
                        sqnorm.reshape(())])
    if world > 1:
        if dist.get_backend(group) == "gloo":
            mine = mine.cpu()
        allv = [torch.empty_like(mine) for _ in range(world)]
        dist.all_gather(allv, mine, group=group)
        allv = torch.stack(allv).cpu().numpy()
    else:
        allv = mine.reshape(1, 3).cpu().numpy()
    us = [int(round(x)) for x in allv[:, 0]]
    bs = [int(round(x)) for x in allv[:, 1]]
    nu = api.norm_per_param(allv[:, 2], P)
    return us, bs, nu


# --------------------------------------------------------------- drivers
class DistributedAdaptiveSGD:
    """Rank `rank` of `world` (one GPU each)."""

    def __init__(self, replica: api.Replica, hyper: Hyper, rank: int, world: int,
                 sched: api.Scheduler, group=None, inflight: int = 2, native: bool = True,
                 merge: str = "nccl", method: str = "adaptive"):
        """native: run the ticket loop in libasgd (asgd_run_tickets); False keeps
        the Python loop of run_tickets (same routing semantics).
        merge: "nccl" = prescale + all_reduce(SUM) + epilogue (K-6, NCCL, K-7);
        "fused" = asgd_merge_fused over CUDA-IPC peer memory (NEXT-1).
        method: "adaptive" (dynamic tickets, Alg. 1 + Alg. 2) or "elastic"
        (Elastic SGD: static equal batches, alpha = 1/N, same update rule)."""
        self.rep, self.h, self.rank, self.world = replica, hyper, rank, world
        self.native = native
        if method not in ("adaptive", "elastic"):
            raise ValueError(f"method={method!r}")
        self.method = method
        if merge not in ("nccl", "fused"):
            raise ValueError(f"merge={merge!r}")
        self.merge = merge
        self.merge_note = ""
        if merge == "fused":
            self.merge, self.merge_note = self._open_peers(replica, rank, world, group)
        self.sched, self.group, self.inflight = sched, group, inflight
        self.b = [hyper.b_max] * world            # initial b = b_max
        self.lr = [hyper.lr_max] * world
        dev = replica.device
        cap = hyper.M // max(1, hyper.b_min) + 2
        self.losses = torch.zeros(cap, dtype=torch.float32, device=dev)
        self.sq = torch.zeros(1, dtype=torch.float64, device=dev)
        self.events = [torch.cuda.Event() for _ in range(cap)]
        self.mb = 0
        self.clock = ScaleClock(hyper, world)
        self.time_merge = False   # record CUDA events around the merge phase of each mega-batch

    def megabatch(self, stream_rows: torch.Tensor, keep_log: bool = False) -> MegaBatchStats:
        """One mega-batch over the M sample ids stream_rows (device int32)."""
        rep, h, r = self.rep, self.h, self.rank
        if self.method == "elastic":
            return self._megabatch_elastic(stream_rows, keep_log)
        self.sched.wait(self.mb)
        b_i, lr_i = self.b[r], self.lr[r]

        if self.native:
            n_steps = rep.run_tickets(self.sched, r, b_i, stream_rows, lr_i, self.losses, self.inflight)
        else:
            def step(k, start, n):
                rep.step(stream_rows[start:start + n], lr_i, self.losses[k:k + 1])
                self.events[k].record(rep.stream)

            n_steps = run_tickets(self.sched, r, b_i, step, self.inflight,
                                  wait=lambda k: self.events[k].synchronize())
        # ---- merge (Alg. 2) -------------------------------------------------
        ev = None
        if self.time_merge:   # from the end of this rank's local steps to the merged model
            ev = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
            ev[0].record(rep.stream)
        if self.world == 1:
            # N = 1: Alg. 2 line 2 gives alpha = b / sum(b) = 1 and lines 4-6 skip the
            # perturbation (the only replica ties with itself, Q17) whatever nu is, so the
            # norm and its host round trip are not needed: the merge is enqueued behind the
            # steps without a device sync (nu is reported as NaN)
            us, bs, nu = [n_steps], [b_i], [float("nan")]
        else:
            rep.sqnorm(self.sq)
            us, bs, nu = exchange_stats(n_steps, b_i, self.sq, rep.P, self.world, self.group)
        routes = self.sched.log() if keep_log and r == 0 else []
        if r == 0:
            self.sched.reset(self.mb + 1)        # every rank is past its tickets
        alpha, rr, ss, pert = api.merge_weights(us, bs, nu, h.pert_thr, h.delta, h.pert_renorm, h.norm)
        self._merge(alpha)
        if ev is not None:
            ev[1].record(rep.stream)
        # ---- Alg. 1 ----------------------------------------------------------
        lr_used = list(self.lr)
        nb = self.clock.step(self.mb, us, bs)     # R13 / R17
        if nb is not None:
            self.b, self.lr = nb
        st = MegaBatchStats(self.mb, us, bs, lr_used, nu, alpha, rr, ss, pert, routes, n_steps, ev)
        self.mb += 1
        return st

    @staticmethod
    def _open_peers(replica: api.Replica, rank: int, world: int, group):
        """Map every rank's replica for the fused merge, or agree on the NCCL merge.

        Each rank tries export / all-gather / open locally, then the ranks take the
        MIN of a success flag, so either every rank runs asgd_merge_fused or every
        rank runs prescale + all_reduce + finish: a rank on the other path would
        spin in k_merge_wait or block in the all-reduce forever.  A rank whose
        peers opened but that falls back closes its mappings."""
        ok, why = 1, ""
        mine = b""
        try:
            mine = replica.peer_export()
        except Exception as e:          # e.g. IPC unsupported on this device
            ok, why = 0, f"peer_export: {type(e).__name__}: {str(e)[:100]}"
        if world > 1:
            handles = [None] * world
            dist.all_gather_object(handles, mine, group=group)
        else:
            handles = [mine]
        if ok and all(handles):
            try:
                replica.peer_open(rank, handles)
            except Exception as e:      # e.g. no P2P/IPC between these GPUs
                ok, why = 0, f"peer_open: {type(e).__name__}: {str(e)[:100]}"
        elif ok:
            ok, why = 0, "another rank could not export its replica"
        if world > 1:
            flag = torch.tensor([ok], dtype=torch.int32)
            if dist.get_backend(group) != "gloo":
                flag = flag.to(replica.device)
            dist.all_reduce(flag, op=dist.ReduceOp.MIN, group=group)
            ok_all = int(flag.item())
        else:
            ok_all = ok
        if ok_all:
            return "fused", ""
        if ok:
            replica.peer_close()
        return "nccl", why or "another rank could not open its peers"

    def _merge(self, alpha):
        rep, h = self.rep, self.h
        if self.merge == "fused":
            rep.merge_fused(alpha, h.gamma)
        else:
            rep.prescale(alpha[self.rank])
            if self.world > 1:
                dist.all_reduce(rep.params, op=dist.ReduceOp.SUM, group=self.group)
            rep.finish(h.gamma)

    def _megabatch_elastic(self, stream_rows: torch.Tensor, keep_log: bool) -> MegaBatchStats:
        """Elastic SGD: static equal batches of
        b_max, alpha_i = 1/N, the same momentum update; no Alg. 1."""
        rep, h, r, N = self.rep, self.h, self.rank, self.world
        M = int(stream_rows.numel())
        n_steps = rep.run_static(r, N, h.b_max, stream_rows, h.lr_max, self.losses, self.inflight)
        ev = None
        if self.time_merge:
            ev = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
            ev[0].record(rep.stream)
        if N == 1:   # alpha = 1/N = 1: no statistics to exchange (see megabatch)
            us, bs, nu = [n_steps], [h.b_max], [float("nan")]
        else:
            rep.sqnorm(self.sq)
            us, bs, nu = exchange_stats(n_steps, h.b_max, self.sq, rep.P, N, self.group)   # also the barrier
        alpha = api.elastic_weights(N)
        self._merge(alpha)
        if ev is not None:
            ev[1].record(rep.stream)
        routes = []
        if keep_log and r == 0:
            routes = [(k, k % N, c, min(h.b_max, M - c)) for k, c in enumerate(range(0, M, h.b_max))]
        st = MegaBatchStats(self.mb, us, bs, [h.lr_max] * N, nu, alpha, -1, -1, False, routes, n_steps, ev)
        self.mb += 1
        return st


class SimulatedAdaptiveSGD:
    """N replicas on one GPU; routing by the simulated clock (Q10) or replay."""

    def __init__(self, replicas: Sequence[api.Replica], hyper: Hyper, row_nnz: np.ndarray,
                 cost_factors: Sequence[float], per_row: float = 5.0, method: str = "adaptive"):
        """method "elastic": Elastic SGD's static routes of b_max (R10), alpha_i = 1/N,
        no Alg. 1 -- the NEXT-2 A/B arm under the same simulated clock."""
        if method not in ("adaptive", "elastic"):
            raise ValueError(f"method={method!r}")
        self.method = method
        self.reps, self.h = list(replicas), hyper
        self.n = len(self.reps)
        self.row_nnz = np.asarray(row_nnz, dtype=np.int64)
        self.cf = list(cost_factors)
        self.per_row = per_row
        self.b = [hyper.b_max] * self.n
        self.lr = [hyper.lr_max] * self.n
        dev = self.reps[0].device
        self.sq = torch.zeros(self.n, dtype=torch.float64, device=dev)
        cap = hyper.M // max(1, hyper.b_min) + 2
        self.losses = torch.zeros(cap, dtype=torch.float32, device=dev)
        self.mb = 0
        self.clock = ScaleClock(hyper, self.n)

    def megabatch(self, stream_rows: torch.Tensor, stream_ids: np.ndarray,
                  route_order: Optional[Sequence[int]] = None) -> MegaBatchStats:
        h = self.h
        if self.method == "elastic":
            routes = api.route_static(self.n, h.b_max, h.M)
        elif route_order is not None:
            routes = api.route_replay(route_order, self.b, h.M)
        else:
            routes = api.route_simulate(self.b, h.M, self.cf, self.per_row, self.row_nnz[stream_ids])
        for k, (r, start, n) in enumerate(routes):
            self.reps[r].step(stream_rows[start:start + n], self.lr[r], self.losses[k:k + 1])
        u = [0] * self.n
        for r, _, _ in routes:
            u[r] += 1
        for i, rep in enumerate(self.reps):
            rep.sqnorm(self.sq[i:i + 1])
        P = self.reps[0].P
        nu = api.norm_per_param(self.sq.cpu().numpy(), P)
        if self.method == "elastic":
            alpha, rr, ss, pert = api.elastic_weights(self.n), -1, -1, False
        else:
            alpha, rr, ss, pert = api.merge_weights(u, self.b, nu, h.pert_thr, h.delta, h.pert_renorm, h.norm)
        r0 = self.reps[0]
        r0.weighted_sum(self.reps, alpha, r0.params)
        r0.finish(h.gamma)
        for rep in self.reps[1:]:
            rep.params.copy_(r0.params)
            rep.params_changed()
        lr_used, b_used = list(self.lr), list(self.b)
        if self.method == "adaptive":
            nb = self.clock.step(self.mb, u, self.b)   # R13 / R17
            if nb is not None:
                self.b, self.lr = nb
        st = MegaBatchStats(self.mb, u, b_used, lr_used, nu, alpha, rr, ss, pert, routes, len(routes))
        self.mb += 1
        return st


def precision_at_k(replica: api.Replica, test: api.DeviceCsr, test_host, rows: np.ndarray, k: int = 1) -> float:
    """P@k of the replica's model on test rows (a13; untimed)."""
    rows_d = torch.as_tensor(np.asarray(rows, dtype=np.int32), device=replica.device)
    top = replica.eval_topk(test, rows_d, k).cpu().numpy()
    sub = test_host.row_slice(rows)
    hits = api.precision_at_k_hits(top, sub.lab_ptr, sub.lab, k)
    return hits / (k * len(rows))
