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
