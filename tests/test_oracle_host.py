"""Pins of the oracle's host algorithms (Alg. 1, Alg. 2, routing, P@k) -- not gpu."""
import json
import os
import random
from fractions import Fraction

import numpy as np
import pytest

from oracle import merge, metrics, routing, scaling
from paper_conf_ipps_marws22_b200 import api
from tests.conftest import GOLDEN


def _load(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


# ----------------------------------------------------------------- Alg. 1
@pytest.mark.parametrize("case", _load("alg1_vectors.json")["cases"])
def test_alg1_golden(case):
    b, lr = scaling.scale_batches(case["u"], case["b"], case["b_min"], case["b_max"],
                                  case["beta"], lr_max=1.0)
    assert b == case["b_out"]
    assert lr == [float(Fraction(x)) for x in case["lr_ratio"]]


def test_alg1_invariants():
    rng = random.Random(1)
    for _ in range(3000):
        N = rng.choice([1, 2, 4, 8])
        beta, b_min, b_max = 64, 128, 1024
        u = [rng.randint(5, 20) for _ in range(N)]
        b = [rng.randint(b_min, b_max) for _ in range(N)]
        b2, lr2 = scaling.scale_batches(u, b, b_min, b_max, beta, lr_max=0.3)
        assert all(b_min <= x <= b_max for x in b2)
        for x, l in zip(b2, lr2):
            assert l == 0.3 * x / b_max                         # linear scaling rule
        if len(set(u)) == 1:
            assert b2 == b                                       # balanced: no change
        # unblocked -> sum of batch sizes conserved (N divides beta: exact)
        mu = Fraction(sum(u), N)
        unblocked = all(b_min <= b[i] + beta * (u[i] - mu) <= b_max for i in range(N))
        if unblocked:
            assert sum(b2) == sum(b)
        # faster GPUs (more updates) never get a smaller batch
        for i in range(N):
            if u[i] > mu:
                assert b2[i] >= b[i]
            if u[i] < mu:
                assert b2[i] <= b[i]


# ----------------------------------------------------------------- Alg. 2
@pytest.mark.parametrize("case", _load("alg2_vectors.json")["cases"])
def test_alg2_golden(case):
    g = _load("alg2_vectors.json")
    alpha, r, s, pert = merge.merge_weights(case["u"], case["b"], case["nu"],
                                            g["pert_thr"], g["delta"])
    want = [Fraction(x) for x in case["alpha"]]
    assert pert == case["perturbed"]
    for a, x in zip(alpha, want):
        assert abs(a - float(x)) <= 4e-16 * float(x)
    assert abs(sum(alpha) - float(Fraction(case["sum"]))) < 1e-15
    if pert:
        assert (r, s) == (case["r"], case["s"])


def test_alg2_weights_sum_to_one_before_perturbation():
    rng = random.Random(2)
    for _ in range(2000):
        N = rng.randint(1, 8)
        u = [rng.randint(1, 30) for _ in range(N)]
        b = [rng.randint(1, 1024) for _ in range(N)]
        a, r, s, p = merge.merge_weights(u, b, [1.0] * N)        # gate closed
        assert not p
        assert abs(sum(a) - 1.0) < 1e-14
        a2, r, s, p = merge.merge_weights(u, b, [0.0] * N, delta=0.1)
        if p:   # sum = 1 + delta (alpha_r - alpha_s) (no renormalisation, Q18)
            assert abs(sum(a2) - (1 + 0.1 * (a[r] - a[s]))) < 1e-14
            assert a[r] >= a[s]
        a3, *_ = merge.merge_weights(u, b, [0.0] * N, delta=0.1, pert_renorm=True)
        assert abs(sum(a3) - 1.0) < 1e-14


def test_merge_identity_and_linearity():
    rng = np.random.default_rng(0)
    w = rng.normal(size=1000)
    d = np.zeros_like(w)
    # identical replicas, equal alpha, gamma = 0 -> identity
    wn, dn = merge.merge_models([w, w, w, w], [0.25] * 4, w, d, gamma=0.0)
    np.testing.assert_allclose(wn, w, rtol=1e-15)
    np.testing.assert_allclose(dn, 0, atol=1e-15)
    # N = 1, gamma = 0 returns the replica
    x = rng.normal(size=1000)
    wn, _ = merge.merge_models([x], [1.0], w, d, gamma=0.0)
    np.testing.assert_array_equal(wn, x)
    # linear in the replicas
    a, bb = rng.normal(size=1000), rng.normal(size=1000)
    d1 = rng.normal(size=1000)
    s1, _ = merge.merge_models([a, bb], [0.3, 0.8], w, d1, gamma=0.9)
    s2, _ = merge.merge_models([2 * a, 2 * bb], [0.3, 0.8], w, 2 * d1, gamma=0.9)
    np.testing.assert_allclose(s2, 2 * s1, rtol=1e-13)


def test_merge_recurrence_closed_form():
    """lr = 0: replicas equal w, so k merges follow the scalar recurrence
    w_{k+1} = sigma w_k + gamma (w_k - w_{k-1}), sigma = sum(alpha) (reading Q34)."""
    w0 = np.linspace(-1, 1, 17)
    u, b, delta, gamma = [3, 2], [32, 32], 0.1, 0.9
    alpha, *_ = merge.merge_weights(u, b, [0.0, 0.0], 0.1, delta)
    sigma = sum(alpha)
    assert abs(sigma - 1.02) < 1e-15
    w, d = w0.copy(), np.zeros_like(w0)
    c_prev, c = 1.0, 1.0          # w_k = c_k w0
    for _ in range(40):
        w, d = merge.merge_models([w, w], alpha, w, d, gamma)
        c_prev, c = c, sigma * c + gamma * (c - c_prev)
        np.testing.assert_allclose(w, c * w0, rtol=1e-12)
    lam = ((sigma + gamma) + np.sqrt((sigma + gamma) ** 2 - 4 * gamma)) / 2
    assert lam > 1.0
    assert abs(np.log(c / c_prev) - np.log(lam)) < 1e-3      # geometric growth lambda


def test_norm_per_param():
    w = np.full(400, 0.5)
    assert merge.norm_per_param(w) == pytest.approx(np.sqrt(400 * 0.25) / 400)


# ----------------------------------------------------------------- routing
def test_fig2_routing():
    g = _load("fig2_routing.json")
    b = [10, 10]
    M = 10 * g["batches_in_megabatch"]
    cost = lambda r, s, n: g["cost_per_batch"][r]
    routes = routing.simulate(b, M, cost)
    assert [r for r, _, _ in routes] == g["expected_order"]
    assert routing.updates(routes, 2) == g["expected_updates"]
    # replay of the recorded order is the identity
    assert routing.replay([r for r, _, _ in routes], b, M) == routes


def test_routing_covers_megabatch_exactly():
    rng = random.Random(3)
    for _ in range(300):
        N = rng.randint(1, 8)
        b = [rng.randint(1, 50) for _ in range(N)]
        M = rng.randint(1, 500)
        c = [rng.uniform(0.5, 2.0) for _ in range(N)]
        routes = routing.simulate(b, M, lambda r, s, n: c[r] * n)
        cur = 0
        for r, s, n in routes:
            assert s == cur and 1 <= n <= b[r]
            cur += n
        assert cur == M
        assert all(n == b[r] for r, _, n in routes[:-1])      # only the last is truncated


def test_scaling_equalises_updates():
    """batch size scaling drives the GPUs to the same number of updates."""
    from oracle import scaling
    b, c = [32, 32], [1.0, 1.5]
    M = 320
    for _ in range(15):
        routes = routing.simulate(b, M, lambda r, s, n: c[r] * n)
        u = routing.updates(routes, 2)
        b, _ = scaling.scale_batches(u, b, 4, 32, 2, 1.0)
    assert abs(u[0] - u[1]) <= 1 and b[0] > b[1]


# ----------------------------------------------------------------- P@k
def test_precision_at_k_bruteforce():
    rng = np.random.default_rng(4)
    Z = rng.integers(0, 5, size=(30, 12)).astype(np.float64)   # many ties
    top = metrics.topk(Z, 3)
    for n in range(30):
        # pure-python brute force: best score, then lowest id
        cand = sorted(range(12), key=lambda j: (-Z[n, j], j))[:3]
        assert top[n].tolist() == cand
    lab_ptr = np.arange(0, 61, 2)
    lab = rng.integers(0, 12, size=60).astype(np.int32)
    p = metrics.precision_at_k(top, lab_ptr, lab, 3)
    hits = sum(len(set(top[n].tolist()) & set(lab[2 * n:2 * n + 2].tolist())) for n in range(30))
    assert p == hits / 90
    # hand example: ties resolve to the lower id
    Zh = np.array([[1.0, 3.0, 3.0, 0.0]])
    assert metrics.topk(Zh, 2).tolist() == [[1, 2]]
    assert metrics.precision_at_k(metrics.topk(Zh, 1), np.array([0, 1]), np.array([2]), 1) == 0.0


def test_alg2_ub_variant_pins():
    """R12: alpha_i = u_i b_i / sum_j u_j b_j in place of line 3."""
    # hand-worked: u = (3, 1), b = (100, 300): u b = (300, 300) -> (1/2, 1/2),
    # where line 3 alone gives (3/4, 1/4)
    a, *_ = merge.merge_weights([3, 1], [100, 300], [1.0, 1.0], norm="ub")
    assert a == [0.5, 0.5]
    a, *_ = merge.merge_weights([3, 1], [100, 300], [1.0, 1.0])
    assert a == [0.75, 0.25]
    # u = (2, 1, 1), b = (64, 64, 128): u b = (128, 64, 128) -> (0.4, 0.2, 0.4)
    a, *_ = merge.merge_weights([2, 1, 1], [64, 64, 128], [1.0] * 3, norm="ub")
    assert a == [0.4, 0.2, 0.4]
    rng = random.Random(7)
    for _ in range(1000):
        N = rng.randint(1, 8)
        u = [rng.randint(1, 30) for _ in range(N)]
        b = [rng.randint(1, 1024) for _ in range(N)]
        a, *_ = merge.merge_weights(u, b, [1.0] * N, norm="ub")
        assert abs(sum(a) - 1.0) < 1e-14
        # equal batch sizes: the product is proportional to u -> line 3's weights
        a_eq, *_ = merge.merge_weights(u, [64] * N, [1.0] * N, norm="ub")
        a_u, *_ = merge.merge_weights(u, [64] * N, [1.0] * N)
        assert all(abs(x - y) < 1e-15 for x, y in zip(a_eq, a_u))
        # all u equal: line 2 still applies (b-normalised)
        a_b, *_ = merge.merge_weights([5] * N, b, [1.0] * N, norm="ub")
        assert all(abs(x - bi / sum(b)) < 1e-15 for x, bi in zip(a_b, b))
    with pytest.raises(ValueError):
        merge.merge_weights([1], [1], [1.0], norm="bu")


def test_scale_frequency_r17():
    """Reading R17: stable or oscillating b doubles the Alg. 1 interval (up to
    the cap), a consistent move resets it to 1; the C function equals the oracle."""
    from oracle.scaling import scale_frequency
    # stable: 1 -> 2 -> 4 -> 8 -> 8
    k, s = 1, [0, 0]
    seq = []
    for _ in range(4):
        k, s = scale_frequency([32, 32], [32, 32], s, k, 8)
        seq.append(k)
    assert seq == [2, 4, 8, 8] and s == [0, 0]
    # consistent moves reset to 1, an opposite move (oscillation) doubles
    k, s = scale_frequency([32, 32], [32, 28], [0, 0], 4, 8)
    assert (k, s) == (1, [0, -1])
    k, s = scale_frequency([32, 28], [32, 26], s, k, 8)
    assert (k, s) == (1, [0, -1])
    k, s = scale_frequency([32, 26], [32, 29], s, k, 8)
    assert (k, s) == (2, [0, 1])
    rng = random.Random(17)
    for _ in range(2000):
        n = rng.randint(1, 8)
        bb = [rng.choice([28, 30, 32]) for _ in range(n)]
        ba = [x + rng.choice([-2, 0, 0, 2]) for x in bb]
        sg = [rng.choice([-1, 0, 1]) for _ in range(n)]
        k0, cap = rng.choice([1, 2, 4, 8]), rng.choice([4, 8, 16])
        assert api.scale_frequency(bb, ba, sg, k0, cap) == scale_frequency(bb, ba, sg, k0, cap)


def test_adaptive_frequency_in_the_run():
    """adaptive.run with scale_every = 0 runs Alg. 1 after mega-batch 0, then after the
    R17 intervals; b changes only at those mega-batches."""
    from oracle import adaptive
    from synth import config, generate, init_params, sample_stream
    cfg = config("tiny", n_train=1024)
    data = generate(cfg, "train", 1024)
    M = cfg.mega_batch
    recs = adaptive.run(cfg.F, cfg.H, cfg.L, data, init_params(cfg), lambda mb: sample_stream(cfg, mb * M, M),
                        n_rep=2, n_mb=8, M=M, b_max=cfg.b_max, b_min=cfg.b_min, beta=cfg.beta, lr_max=cfg.lr_max,
                        cost_factors=[1.0, 1.6], scale_every=0)
    from oracle.scaling import scale_batches, scale_frequency
    k, cd, sg = 1, 1, [0, 0]
    b = [cfg.b_max] * 2
    for mb, rec in enumerate(recs):
        assert rec.b == b
        cd -= 1
        if cd == 0:
            bn, _ = scale_batches(rec.u, b, cfg.b_min, cfg.b_max, cfg.beta, cfg.lr_max)
            k, sg = scale_frequency(b, bn, sg, k, 8)
            b, cd = bn, k
    assert recs[1].b != recs[0].b           # the slower replica was rescaled after mega-batch 0
