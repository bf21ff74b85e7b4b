"""Pins of the bf16-rounding reference tests/bf16_emul.py (not gpu): with the
rounding switched off it is the oracle's gradient (softmax and the centred
sigmoid, whose constants must cancel exactly); chunks with B_full sum to the
whole batch; rounding is round-to-nearest-even."""
import numpy as np
import pytest

from oracle import model
from synth import config, generate, init_params, planted_params
from tests import bf16_emul


def test_bf16_rounding_is_rne():
    x = np.array([1.0, 1.0 + 2.0 ** -8, 1.0 + 3 * 2.0 ** -8, 1.0 + 2.0 ** -9, -2.5, 0.0])
    got = bf16_emul.bf16(x)
    # 1 + 2^-8 is a tie between 1 and 1 + 2^-7 -> even (1); 1 + 3 * 2^-8 -> 1 + 2^-6 (even)
    assert got.tolist() == [1.0, 1.0, 1.0 + 2.0 ** -6, 1.0, -2.5, 0.0]


@pytest.mark.parametrize("loss", ["softmax", "sigmoid"])
@pytest.mark.parametrize("planted", [False, True])
def test_without_rounding_equals_oracle(monkeypatch, loss, planted):
    cfg = config("tiny")
    data = generate(cfg, "train", 256)
    batch = data.row_slice(np.arange(40))
    w = (planted_params(cfg) if planted else init_params(cfg)).astype(np.float64)
    _, go = model.loss_and_grad(w, batch, cfg.F, cfg.H, cfg.L, loss)
    monkeypatch.setattr(bf16_emul, "bf16", lambda x: np.asarray(x, dtype=np.float64))
    ge = bf16_emul.grads_bf16(w, batch, cfg.F, cfg.H, cfg.L, loss)
    assert np.linalg.norm(ge - go) <= 1e-12 * np.linalg.norm(go)


def test_chunks_sum_to_batch():
    cfg = config("tiny")
    data = generate(cfg, "train", 256)
    batch = data.row_slice(np.arange(48))
    w = planted_params(cfg).astype(np.float64)
    full = bf16_emul.grads_bf16(w, batch, cfg.F, cfg.H, cfg.L)
    parts = sum(bf16_emul.grads_bf16(w, batch.row_slice(np.arange(r, r + 16)), cfg.F, cfg.H, cfg.L, B_full=48)
                for r in (0, 16, 32))
    assert np.linalg.norm(parts - full) <= 1e-13 * np.linalg.norm(full)
    _, go = model.loss_and_grad(w, batch, cfg.F, cfg.H, cfg.L)
    e = np.linalg.norm(full - go) / np.linalg.norm(go)
    assert 1e-4 < e < 2e-2          # bf16 rounding is visible and inside the bf16 bar


@pytest.mark.parametrize("mode", ["bf16", "x3"])
def test_slack_is_small_except_at_the_kink(mode):
    """The componentwise slack is a small fraction of the gradient (the elementwise check
    keeps its bite), except where a pre-activation sits on the ReLU kink."""
    cfg = config("tiny")
    data = generate(cfg, "train", 256)
    batch = data.row_slice(np.arange(40))
    w = init_params(cfg).astype(np.float64)
    g, sl = bf16_emul.grads_bf16(w, batch, cfg.F, cfg.H, cfg.L, with_slack=True, rounding=mode)
    assert np.array_equal(g, bf16_emul.grads_bf16(w, batch, cfg.F, cfg.H, cfg.L, rounding=mode))
    assert np.all(sl >= 0)
    o1, o2 = cfg.F * cfg.H, cfg.F * cfg.H + cfg.H
    for a_, b_ in ((0, o1), (o2, o2 + cfg.L * cfg.H)):      # W1, W2: slack well below the values
        assert np.linalg.norm(sl[a_:b_]) < 0.05 * np.linalg.norm(g[a_:b_])
    # put one pre-activation exactly on the kink: its row's features get slack in that column
    X = batch.row_slice(np.arange(1))
    A1 = np.zeros(cfg.H)
    for k in range(X.row_ptr[1]):
        A1 += X.val[k] * w[X.col[k] * cfg.H:(X.col[k] + 1) * cfg.H]
    w2 = w.copy()
    w2[o1 + 3] = -A1[3]                       # b1[3] cancels row 0's A1[:, 3]
    g2, sl2 = bf16_emul.grads_bf16(w2, batch, cfg.F, cfg.H, cfg.L, with_slack=True, rounding=mode)
    f = X.col[0] * cfg.H + 3
    assert sl2[f] > 10 * sl[f] and sl2[o1 + 3] > 10 * sl[o1 + 3]


def test_x3_mode_is_close_to_exact():
    """bf16x3 products lose ~2^-16 relative: the x3 reference sits within 1e-4 of the
    exact gradient (the fp32 path's bar) but is not the exact gradient."""
    cfg = config("tiny")
    data = generate(cfg, "train", 256)
    batch = data.row_slice(np.arange(32))
    w = planted_params(cfg).astype(np.float64)
    _, go = model.loss_and_grad(w, batch, cfg.F, cfg.H, cfg.L)
    for loss in ("softmax", "sigmoid"):
        _, go = model.loss_and_grad(w, batch, cfg.F, cfg.H, cfg.L, loss)
        g3 = bf16_emul.grads_bf16(w, batch, cfg.F, cfg.H, cfg.L, loss, rounding="x3")
        e = np.linalg.norm(g3 - go) / np.linalg.norm(go)
        assert 1e-9 < e < 2e-5, (loss, e)
