"""Oracle: top-k precision on the test set.

PAPER.md P:1549-1551 (§V-A): "We measure the top-1 accuracy on the testing
dataset after processing every mega-batch"; P:457-463 (§II) test accuracy.
Reading Q23: P@1 = [argmax_j Z_nj in Y_n], ties to the lower label id;
P@k = |top-k(Z_n) cap Y_n| / k averaged over rows.  Brute force: a full sort
of every row.

Test infrastructure only (see oracle/__init__.py).
"""
from __future__ import annotations

import numpy as np


def topk(Z: np.ndarray, k: int) -> np.ndarray:
    """Per row the k label ids of largest score, ties to the lower id (full sort)."""
    B, L = Z.shape
    ids = np.arange(L)
    out = np.empty((B, k), dtype=np.int32)
    for n in range(B):
        order = np.lexsort((ids, -Z[n]))       # primary -score, secondary id
        out[n] = order[:k]
    return out


def precision_at_k(top: np.ndarray, lab_ptr: np.ndarray, lab: np.ndarray, k: int) -> float:
    hits = 0
    for n in range(top.shape[0]):
        y = set(lab[lab_ptr[n]:lab_ptr[n + 1]].tolist())
        hits += sum(1 for j in top[n, :k] if int(j) in y)
    return hits / (k * top.shape[0])
