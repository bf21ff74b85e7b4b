"""Pins of the oracle's Elastic SGD mode (PAPER.md
P:547-593 elastic model averaging, P:597-599 equal batch counts, P:1623-1628
Elastic and Adaptive coincide on one GPU) -- not gpu."""
import random

import numpy as np
import pytest

from oracle import adaptive, merge, model, routing
from synth import config, generate, init_params, sample_stream


def test_static_routing_equal_counts():
    rng = random.Random(5)
    for _ in range(200):
        N, b = rng.randint(1, 8), rng.randint(1, 40)
        M = rng.randint(1, 600)
        routes = routing.static(N, b, M)
        cur = 0
        for k, (r, s, n) in enumerate(routes):
            assert r == k % N and s == cur and 1 <= n <= b
            cur += n
        assert cur == M
        u = routing.updates(routes, N)
        assert max(u) - min(u) <= 1                       # "the same number of batches"
        if (-(-M // b)) % N == 0:
            assert len(set(u)) == 1


def _tiny(n_rows=1024):
    cfg = config("tiny", n_train=n_rows)
    return cfg, generate(cfg, "train", n_rows)


def test_elastic_equals_adaptive_on_one_gpu():
    """with one GPU both methods are mini-batch SGD with the same
    update rule (Alg. 1 keeps b_max, Alg. 2 gives alpha = 1)."""
    cfg, data = _tiny()
    M = cfg.mega_batch
    stream = lambda mb: sample_stream(cfg, mb * M, M)
    a = adaptive.run(cfg.F, cfg.H, cfg.L, data, init_params(cfg), stream, n_rep=1, n_mb=3, M=M,
                     b_max=cfg.b_max, b_min=cfg.b_min, beta=cfg.beta, lr_max=cfg.lr_max)
    e = adaptive.run_elastic(cfg.F, cfg.H, cfg.L, data, init_params(cfg), stream, n_rep=1, n_mb=3, M=M,
                             b=cfg.b_max, lr=cfg.lr_max)
    for ra, re in zip(a, e):
        assert ra.routes == re.routes
        np.testing.assert_array_equal(ra.w, re.w)


def test_elastic_two_replicas_is_the_average_of_two_sgd_runs():
    """N = 2: replica i runs SGD on batches i, i + 2, ... from the global model;
    the merge is w' = (w_0 + w_1)/2 + gamma d (alpha = 1/N)."""
    cfg, data = _tiny()
    M, b, lr, gamma = 8 * cfg.b_max, cfg.b_max, 0.5, 0.9
    rows = sample_stream(cfg, 0, M)
    w0 = init_params(cfg).astype(np.float64)
    rec = adaptive.run_elastic(cfg.F, cfg.H, cfg.L, data, w0, lambda mb: rows, n_rep=2, n_mb=1, M=M, b=b, lr=lr,
                               gamma=gamma)[0]
    reps = []
    for i in range(2):
        x = w0.copy()
        for k in range(i, M // b, 2):
            x, _, _ = model.sgd_step(x, data.row_slice(rows[k * b:(k + 1) * b]), lr, cfg.F, cfg.H, cfg.L)
        reps.append(x)
    want = 0.5 * (reps[0] + reps[1])              # d = 0 at the first merge (Q19)
    np.testing.assert_allclose(rec.w, want, rtol=0, atol=1e-12)
    assert rec.u == [4, 4] and rec.alpha == [0.5, 0.5]


def test_adaptive_scale_every_and_ub_norm():
    """R13: with scale_every = k, Alg. 1 runs only after mega-batches
    k-1, 2k-1, ...; b is frozen at b_max in between, and those mega-batches
    route exactly like the first one under the same costs.  R12: with the
    b-normalised line 2 untouched, the first mega-batch (all b_i = b_max) gives
    identical alphas in both norms."""
    cfg, data = _tiny()
    M = cfg.mega_batch
    stream = lambda mb: sample_stream(cfg, mb * M, M)
    kw = dict(n_rep=2, n_mb=3, M=M, b_max=cfg.b_max, b_min=cfg.b_min, beta=cfg.beta,
              lr_max=cfg.lr_max, cost_factors=[1.0, 1.6])
    every = adaptive.run(cfg.F, cfg.H, cfg.L, data, init_params(cfg), stream, **kw)
    frozen = adaptive.run(cfg.F, cfg.H, cfg.L, data, init_params(cfg), stream, scale_every=4, **kw)
    assert every[1].b != [cfg.b_max] * 2          # the 1.6x slower rank was rescaled
    for rec in frozen:
        assert rec.b == [cfg.b_max] * 2 and rec.lr == [cfg.lr_max] * 2
    np.testing.assert_array_equal(every[0].w, frozen[0].w)
    ub = adaptive.run(cfg.F, cfg.H, cfg.L, data, init_params(cfg), stream, norm="ub", **kw)
    assert ub[0].alpha == every[0].alpha
    assert ub[1].b == every[1].b                  # Alg. 1 does not read alpha
    u, b = ub[1].u, ub[1].b
    assert u[0] != u[1]
    tot = u[0] * b[0] + u[1] * b[1]
    want = [u[0] * b[0] / tot, u[1] * b[1] / tot]
    if ub[1].perturbed:                           # Alg. 2 lines 5-6, delta = 0.1
        want[ub[1].r] *= 1.1
        want[ub[1].s] *= 0.9
    assert ub[1].alpha == want
    with pytest.raises(ValueError):
        adaptive.run(cfg.F, cfg.H, cfg.L, data, init_params(cfg), stream, scale_every=-1, **kw)
