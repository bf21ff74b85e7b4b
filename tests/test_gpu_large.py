"""Parity at the big BASELINE.json shapes, in the launch configuration bench.py
times (full F, L, H and b_max; the dataset is a generated prefix of the
split).  The oracle's batch-mean gradient is evaluated in row chunks:
grad(B rows) = sum_chunks (|chunk| / B) grad(chunk), which is the definition
of the mean and keeps the fp64 working set bounded."""
import numpy as np
import pytest
import torch

from oracle import model as omodel
from synth import config, init_params, planted_params, sample_stream
from tests.bf16_emul import grads_bf16
from tests.gpu_helpers import check_grads, dataset, make_replica, split_grad

pytestmark = pytest.mark.gpu

TOL = {"fp32": 1e-4, "bf16": 2e-2}


def _chunked_oracle(w, batch, F, H, L, chunk, loss_kind="softmax", emulate=False):
    """Oracle loss and gradient of the batch in row chunks; with emulate, also the
    bf16-rounding reference (tests/bf16_emul.py), whose chunks sum directly (the
    1/B of the full batch is applied before its dZ rounding)."""
    B = batch.n_rows
    loss, g, e = 0.0, None, None
    for r0 in range(0, B, chunk):
        sub = batch.row_slice(np.arange(r0, min(B, r0 + chunk)))
        lo, go = omodel.loss_and_grad(w, sub, F, H, L, loss_kind)
        f = sub.n_rows / B
        loss += f * lo
        g = f * go if g is None else g + f * go
        ge = grads_bf16(w, sub, F, H, L, loss_kind, B_full=B, with_slack=True, rounding=emulate)
        e = ge if e is None else (e[0] + ge[0], e[1] + ge[1])
    return loss, g, e


def _check_big(name, n_rows, precision, chunk, seed_pos=0, loss_kind="softmax", planted=False, batch=None):
    cfg = config(name)
    data = dataset(name, n_rows)
    cfg_sub = config(name, n_train=data.n_rows)
    rows = sample_stream(cfg_sub, seed_pos, batch or cfg.b_max)
    w0 = planted_params(cfg) if planted else init_params(cfg)
    rep = make_replica(cfg, data, precision, w0=w0, loss=loss_kind)
    g = torch.zeros(rep.P, dtype=torch.float32, device="cuda")
    loss = torch.zeros(1, dtype=torch.float32, device="cuda")
    rep.set_debug_grads(g)
    rep.step(torch.as_tensor(rows, device="cuda"), 0.5, loss)
    rep.sync()
    touched = rep.last_touched().cpu().numpy()
    batch = data.row_slice(rows)
    lo, go, em = _chunked_oracle(w0.astype(np.float64), batch, cfg.F, cfg.H, cfg.L, chunk, loss_kind,
                                 emulate="bf16" if precision == "bf16" else "x3")
    tol = TOL[precision]
    assert abs(loss.item() - lo) <= tol * abs(lo)
    np.testing.assert_array_equal(touched, omodel.touched_features(batch))
    gg, og = split_grad(g.cpu().numpy(), cfg.F, cfg.H, cfg.L), split_grad(go, cfg.F, cfg.H, cfg.L)
    eg = split_grad(em[0], cfg.F, cfg.H, cfg.L)
    es = split_grad(em[1], cfg.F, cfg.H, cfg.L)
    check_grads(gg, og, tol, cfg.F, cfg.H, touched,
                tag=f"{name}/{precision}/{loss_kind}/{'planted' if planted else 'init'}", emul=eg, slack=es)


@pytest.mark.parametrize("precision", ["bf16", "fp32"])
def test_amazoncat_bench_launch(precision):
    _check_big("amazoncat13k", 32768, precision, chunk=1024)


def test_amazon670k_fp32_bench_launch():
    """The fp32 path (bf16x3 on tcgen05, R14) at L = 670,091: Z stored (2.7 GB), dZ as
    bf16 hi + lo halves; 1e-4 against the fp64 oracle."""
    _check_big("amazon670k", 16384, "fp32", chunk=128)


def test_amazon670k_bench_launch():
    """L = 670,091: the fused softmax-CE path (Z never stored), G2 splits K."""
    _check_big("amazon670k", 16384, "bf16", chunk=128)


def test_wiki10_full_split_bench_launch():
    _check_big("wiki10_31k", None, "bf16", chunk=256)


def test_delicious200k_bench_launch():
    """NEXT-3: F = 782,585 (800 MB of W1), L = 205,443, 75 labels per row."""
    _check_big("delicious200k", 8192, "bf16", chunk=128)


def test_amazon670k_sigmoid_bench_launch():
    """Sigmoid-BCE head (R11) at L = 670,091: one G1 pass writes dZ, no lse pass."""
    _check_big("amazon670k", 16384, "bf16", chunk=128, loss_kind="sigmoid")


# ------------------------------------------------ trained-like (peaked softmax) states
# synth.planted_params: W2 rows aligned with the labels' feature signatures, |W2 row| = 100,
# so the softmax is peaked (logit range ~30-40) and dZ = p - T cancels on the true labels.
# Batches come from a later pass of the sample stream (pass 20).

@pytest.mark.parametrize("precision", ["bf16", "fp32"])
def test_amazoncat_planted_state(precision):
    _check_big("amazoncat13k", 32768, precision, chunk=1024, seed_pos=20 * 32768 + 5, planted=True)


def test_amazon670k_planted_state():
    """Peaked softmax over 670,091 labels through k_lse + the G1b label walk."""
    _check_big("amazon670k", 16384, "bf16", chunk=128, seed_pos=20 * 16384 + 5, planted=True)


def test_delicious200k_planted_state():
    _check_big("delicious200k", 8192, "bf16", chunk=128, seed_pos=20 * 8192 + 5, planted=True)


def test_wiki10_planted_state():
    _check_big("wiki10_31k", None, "bf16", chunk=256, seed_pos=20 * 14146 + 5, planted=True)


def test_amazoncat_ragged_batch_k3():
    """A 300-row batch at the AmazonCat shape (fused softmax-CE regime, K-3's k_bwd_dh):
    the last 128-row block is partial (44 rows) and L = 13,330 ends in a partial 64-label
    tile; planted (peaked) state."""
    _check_big("amazoncat13k", 32768, "bf16", chunk=300, seed_pos=7 * 32768 + 11, planted=True, batch=300)
