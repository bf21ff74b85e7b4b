"""Oracle: dynamic scheduling of batches within a mega-batch.

PAPER.md P:619-643 (§III): "batches are dispatched one-by-one based on GPU
availability. Whenever a GPU finishes an epoch, it is assigned the next
batch ... controlled by fixing the number of training samples processed
between model merging stages -- we call these samples a mega-batch."
Fig. 2: 5 batches on 2 GPUs give 3 updates to GPU 1
and 2 to GPU 2.

Readings: Q8 the mega-batch is M samples in total; a ticket for
rank r takes the range [c, min(c + b_r, M)) of the sample stream and advances
the cursor c (Q9: the last batch is truncated and still counts as an
update); Q10 in a real run the order of tickets is whatever the shared
counter saw (replayed from its log); in the simulated-clock mode the rank
that becomes free first takes the next ticket, ties to the lower rank id.

Test infrastructure only (see oracle/__init__.py).
"""
from __future__ import annotations

from typing import Callable, List, Sequence, Tuple

Route = Tuple[int, int, int]       # (rank, start, len) in mega-batch coordinates


def replay(order: Sequence[int], b: Sequence[int], M: int) -> List[Route]:
    """Ranks in ticket order -> (rank, start, len); stops once c >= M."""
    out: List[Route] = []
    c = 0
    for r in order:
        if c >= M:
            break
        n = min(int(b[r]), M - c)
        out.append((int(r), c, n))
        c += n
    return out


def simulate(b: Sequence[int], M: int,
             cost: Callable[[int, int, int], float]) -> List[Route]:
    """Discrete-event simulation of the dispatcher.

    cost(rank, start, len) is the time rank takes on that batch.  Every rank
    is free at t = 0; repeatedly the rank with the smallest free time (ties:
    lowest id) takes the next batch."""
    N = len(b)
    free = [0.0] * N
    out: List[Route] = []
    c = 0
    while c < M:
        r = min(range(N), key=lambda i: (free[i], i))
        n = min(int(b[r]), M - c)
        out.append((r, c, n))
        free[r] += cost(r, c, n)
        c += n
    return out


def static(N: int, b: int, M: int) -> List[Route]:
    """Elastic model averaging's static schedule (§II; P:597-599:
    "every GPU has to process the same number of batches"): the mega-batch is
    cut into batches of b samples; batch k goes to rank k mod N (reading R10:
    when N does not divide the batch count the first ranks get one more)."""
    out: List[Route] = []
    k = 0
    for c in range(0, M, b):
        out.append((k % N, c, min(b, M - c)))
        k += 1
    return out


def updates(routes: Sequence[Route], N: int) -> List[int]:
    """u_i = number of batches (model updates) rank i received."""
    u = [0] * N
    for r, _, _ in routes:
        u[r] += 1
    return u
