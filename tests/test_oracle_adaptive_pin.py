"""Independent pins of oracle/adaptive.py:run at N > 1 (not gpu).

adaptive.run drives every multi-replica GPU parity test, so a misreading shared
with train.py would pass them.  These pins re-derive its output without calling
any of its pieces except the replayed routing:

* Equal batch sizes and alternating tickets [0, 1, 0, 1, ...]: u_0 = u_1 and
  b_0 = b_1, so Alg. 2 line 2 gives alpha = (1/2, 1/2), the key tie (u, b) skips
  the perturbation (Q17) and Alg. 1 changes nothing (u_i = mu~).  The result must
  be bit-for-bit run_elastic(N = 2), which is itself pinned against two plain
  SGD runs (test_oracle_elastic.py).
* A hand-written 2-replica loop with UNEQUAL tickets: each replica restarts from
  the global w at every mega-batch start (Q21), steps with its own
  lr_i, the truncated last batch still counts (Q9); the step's
  gradient is PyTorch fp64 autograd (not oracle/model.py), Alg. 1 and Alg. 2's
  weights are exact Fractions written from PAPER.md P:891-916 / P:1005-1044, and
  the momentum update is w' = sum alpha_i w_i + gamma (w - w_p).
"""
from fractions import Fraction

import numpy as np

from oracle import adaptive, routing
from synth import config, generate, init_params, sample_stream
from tests.test_oracle_model import _torch_loss


def _cfg():
    # small and fast: the tiny shape cut to F = 300, H = 8, L = 12; b_max = 16 gives
    # b_min = 2 and beta = 1
    return config("tiny", index=17, F=300, L=12, H=8, n_train=512, n_test=64, s_bar=8.0, b_max=16)


def test_alternating_tickets_equal_b_is_elastic():
    cfg = _cfg()
    data = generate(cfg)
    w0 = init_params(cfg).astype(np.float64)
    M, n_mb = 10 * cfg.b_max, 3
    stream = lambda mb: sample_stream(cfg, mb * M, M)
    order = [0, 1] * 5                                 # 10 tickets of b_max: u = (5, 5)
    a = adaptive.run(cfg.F, cfg.H, cfg.L, data, w0, stream, n_rep=2, n_mb=n_mb, M=M, b_max=cfg.b_max,
                     b_min=cfg.b_min, beta=cfg.beta, lr_max=0.7, route_logs=[order] * n_mb)
    e = adaptive.run_elastic(cfg.F, cfg.H, cfg.L, data, w0, stream, n_rep=2, n_mb=n_mb, M=M,
                             b=cfg.b_max, lr=0.7)
    for ra, re in zip(a, e):
        assert ra.routes == re.routes
        assert ra.u == [5, 5] and ra.b == [cfg.b_max] * 2 and ra.lr == [0.7, 0.7]
        assert ra.alpha == [0.5, 0.5] and not ra.perturbed
        np.testing.assert_array_equal(ra.w, re.w)
        np.testing.assert_array_equal(ra.d, re.d)


def _alg1(u, b, b_min, b_max, beta):
    """PAPER.md P:891-916 in exact rationals; Q12: a fractional increment is
    truncated toward zero; Q13: a violated bound leaves b_i unchanged."""
    N = len(u)
    mu = Fraction(sum(u), N)                                        # line 1
    out = list(b)
    for i in range(N):
        inc = int(beta * (u[i] - mu))                               # int() truncates toward zero
        if u[i] > mu and b[i] + inc <= b_max:                       # lines 3-5
            out[i] = b[i] + inc
        elif u[i] < mu and b[i] + inc >= b_min:                     # lines 6-8
            out[i] = b[i] + inc
    return out


def _alg2_alpha(u, b, nu, thr=Fraction(1, 10), delta=Fraction(1, 10)):
    """PAPER.md P:1005-1036 lines 1-7 in exact rationals (Q16-Q18)."""
    N = len(u)
    if len(set(u)) == 1:
        alpha = [Fraction(b[i], sum(b)) for i in range(N)]          # line 2
    else:
        alpha = [Fraction(u[i], sum(u)) for i in range(N)]          # line 3
    if all(x < thr for x in nu):                                    # line 4
        keys = [(u[i], b[i]) for i in range(N)]
        r = max(range(N), key=lambda i: (keys[i], -i))              # line 5, Q17
        s = min(range(N), key=lambda i: (keys[i], i))
        if keys[r] != keys[s]:
            alpha[r] *= 1 + delta                                    # line 6
            alpha[s] *= 1 - delta
    return alpha


def test_hand_written_two_replica_loop():
    cfg = _cfg()
    data = generate(cfg)
    F, H, L = cfg.F, cfg.H, cfg.L
    w0 = init_params(cfg).astype(np.float64)
    b_max, b_min, beta, lr_max, gamma = cfg.b_max, cfg.b_min, cfg.beta, 0.9, 0.9
    M = 10 * b_max
    # mega-batch 0: rank 0 takes 7 of the 10 tickets -> u = (7, 3) -> Alg. 1 shrinks b_1;
    # mega-batch 1: b = (16, 14): 11 tickets, the last one truncated (Q9);
    # mega-batch 2: another uneven split under the new b.
    orders = [[0, 1, 0, 0, 1, 0, 0, 1, 0, 0],
              [1, 0, 1, 1, 0, 1, 0, 1, 1, 0, 1, 0, 1],
              [0, 0, 1, 0, 1, 0, 0, 1, 0, 1, 0, 0, 1]]
    stream = lambda mb: sample_stream(cfg, mb * M, M)
    recs = adaptive.run(F, H, L, data, w0, stream, n_rep=2, n_mb=3, M=M, b_max=b_max, b_min=b_min,
                        beta=beta, lr_max=lr_max, gamma=gamma, route_logs=orders)

    w, wp = w0.copy(), w0.copy()
    b = [b_max, b_max]
    for mb, order in enumerate(orders):
        lr = [lr_max * Fraction(bi, b_max) for bi in b]            # P:910, P:914 (Q14)
        rows = stream(mb)
        reps = [w.copy(), w.copy()]                                 # start from w
        u = [0, 0]
        c = 0
        routes = []
        for r in order:
            if c >= M:
                break
            n = min(b[r], M - c)                                    # Q9: truncated last batch
            batch = data.row_slice(rows[c:c + n])
            _, g = _torch_loss(reps[r], batch, F, H, L)
            reps[r] = reps[r] - float(lr[r]) * g
            u[r] += 1
            routes.append((r, c, n))
            c += n
        rec = recs[mb]
        assert rec.routes == routes
        assert rec.u == u and rec.b == b and rec.lr == [float(x) for x in lr]
        nu = [Fraction(float(np.linalg.norm(x))) / len(x) for x in reps]
        alpha = _alg2_alpha(u, b, nu)
        # the oracle rounds at each fp64 operation, the rationals once: a few ulps
        np.testing.assert_allclose(rec.alpha, [float(a) for a in alpha], rtol=1e-15, atol=0)
        assert rec.perturbed == (u[0] != u[1])
        w_new = float(alpha[0]) * reps[0] + float(alpha[1]) * reps[1] + gamma * (w - wp)
        np.testing.assert_allclose(rec.w, w_new, rtol=1e-10, atol=1e-13)
        wp, w = w, w_new
        b = _alg1(u, b, b_min, b_max, beta)
    # the trajectory did exercise unequal b and per-rank lr
    assert recs[1].b == [b_max, 14] and recs[1].lr == [lr_max, lr_max * 14 / 16]
    assert routing.updates(recs[1].routes, 2) == recs[1].u
    assert recs[1].routes[-1][2] < max(recs[1].b)                  # truncated last batch
