"""Oracle: the whole Adaptive SGD method over N simulated replicas, fp64.

PAPER.md §III and §IV:
  for every mega-batch:
    every replica starts from the global model (Q21);
    batches are routed one at a time (routing.py);
    each batch is one local SGD step on its replica (model.py);
    u_i = number of updates of replica i;
    Alg. 2 merges the replicas into the global model (merge.py);
    Alg. 1 rescales batch sizes and learning rates (scaling.py).
Within a mega-batch the replicas never interact, so they are stepped one
after another in routing order; the result is independent of the order.
Readings Q15 (the b_i in effect during the mega-batch enter Alg. 2) and Q31
(the sample stream is the concatenation of per-pass permutations).

Test infrastructure only (see oracle/__init__.py).
"""
from __future__ import annotations

import dataclasses
from typing import Callable, List, Optional, Sequence

import numpy as np

from . import merge as _merge
from . import model as _model
from . import routing as _routing
from . import scaling as _scaling


@dataclasses.dataclass
class MegaBatchRecord:
    routes: list
    losses: list
    u: list
    b: list            # batch sizes in effect during this mega-batch
    lr: list
    nu: list
    alpha: list
    perturbed: bool
    r: int
    s: int
    w: np.ndarray      # global model after the merge
    d: np.ndarray


def nnz_cost(factors: Sequence[float], data, stream_rows: np.ndarray, per_row: float = 5.0):
    """Simulated-clock cost c_i * (nnz + 5 rows) of a batch (SURVEY §8(d) tiny)."""
    lens = np.diff(data.row_ptr)

    def cost(rank: int, start: int, n: int) -> float:
        rows = stream_rows[start:start + n]
        return float(factors[rank]) * (float(lens[rows].sum()) + per_row * n)
    return cost


def run(F: int, H: int, L: int, data, w0: np.ndarray, stream_rows_of: Callable[[int], np.ndarray],
        n_rep: int, n_mb: int, M: int, b_max: int, b_min: int, beta: int, lr_max: float,
        gamma: float = 0.9, delta: float = 0.1, pert_thr: float = 0.1,
        pert_renorm: bool = False, cost_factors: Optional[Sequence[float]] = None,
        route_logs: Optional[List[List[int]]] = None, norm: str = "u",
        scale_every: int = 1, max_interval: int = 8) -> List[MegaBatchRecord]:
    """Run n_mb mega-batches.  stream_rows_of(mb) gives the M sample ids of
    mega-batch mb.  Routing is simulated with cost_factors, or replayed from
    route_logs[mb] (ranks in ticket order).  norm: Alg. 2 line 3 ("u") or the
    u_i b_i variant ("ub", R12).  scale_every: Alg. 1 runs after mega-batches
    mb with (mb + 1) % scale_every == 0 (R13; 1 = every mega-batch,
    the paper's default); scale_every = 0: the adaptive frequency of reading R17
    (scaling.scale_frequency, intervals up to max_interval)."""
    if scale_every < 0:
        raise ValueError(scale_every)
    interval, countdown, signs = 1, 1, [0] * n_rep     # R17 state
    w = np.asarray(w0, dtype=np.float64).copy()
    d = np.zeros_like(w)                                   # Q19: w_p = w_0
    b = [int(b_max)] * n_rep
    lr = [float(lr_max)] * n_rep
    out: List[MegaBatchRecord] = []
    for mb in range(n_mb):
        rows = stream_rows_of(mb)
        if route_logs is not None:
            routes = _routing.replay(route_logs[mb], b, M)
        else:
            f = cost_factors if cost_factors is not None else [1.0] * n_rep
            routes = _routing.simulate(b, M, nnz_cost(f, data, rows))
        replicas = [w.copy() for _ in range(n_rep)]
        losses = []
        for (r, start, n) in routes:
            batch = data.row_slice(rows[start:start + n])
            replicas[r], loss, _ = _model.sgd_step(replicas[r], batch, lr[r], F, H, L)
            losses.append(loss)
        u = _routing.updates(routes, n_rep)
        nu = [_merge.norm_per_param(x) for x in replicas]
        alpha, r, s, pert = _merge.merge_weights(u, b, nu, pert_thr, delta, pert_renorm, norm)
        w, d = _merge.merge_models(replicas, alpha, w, d, gamma)
        rec = MegaBatchRecord(routes, losses, u, list(b), list(lr), nu, alpha, pert, r, s,
                              w.copy(), d.copy())
        if scale_every == 0:                               # R17: adaptive frequency
            countdown -= 1
            if countdown == 0:
                b_new, lr = _scaling.scale_batches(u, b, b_min, b_max, beta, lr_max)
                interval, signs = _scaling.scale_frequency(b, b_new, signs, interval, max_interval)
                b, countdown = b_new, interval
        elif (mb + 1) % scale_every == 0:                  # R13
            b, lr = _scaling.scale_batches(u, b, b_min, b_max, beta, lr_max)
        out.append(rec)
    return out


def run_elastic(F: int, H: int, L: int, data, w0: np.ndarray, stream_rows_of: Callable[[int], np.ndarray],
                n_rep: int, n_mb: int, M: int, b: int, lr: float,
                gamma: float = 0.9) -> List[MegaBatchRecord]:
    """Elastic SGD (model averaging): static equal
    batches (routing.static), every replica starts from the global model, the
    merge averages the replicas with alpha_i = 1/N and applies the same
    momentum update rule as Adaptive SGD (both run in the same
    framework with the same model update).  No batch-size scaling, no
    perturbation."""
    w = np.asarray(w0, dtype=np.float64).copy()
    d = np.zeros_like(w)
    out: List[MegaBatchRecord] = []
    alpha = [1.0 / n_rep] * n_rep
    for mb in range(n_mb):
        rows = stream_rows_of(mb)
        routes = _routing.static(n_rep, b, M)
        replicas = [w.copy() for _ in range(n_rep)]
        losses = []
        for (r, start, n) in routes:
            batch = data.row_slice(rows[start:start + n])
            replicas[r], loss, _ = _model.sgd_step(replicas[r], batch, lr, F, H, L)
            losses.append(loss)
        u = _routing.updates(routes, n_rep)
        nu = [_merge.norm_per_param(x) for x in replicas]
        w, d = _merge.merge_models(replicas, alpha, w, d, gamma)
        out.append(MegaBatchRecord(routes, losses, u, [b] * n_rep, [lr] * n_rep, nu, list(alpha), False, -1, -1,
                                   w.copy(), d.copy()))
    return out
