"""Pins of oracle/model.py against things other than itself (not gpu).

* central finite differences of the loss (fp64) -- catches any dropped term,
  sign or transposed operand in the backward pass;
* PyTorch CPU fp64 autograd of the same network and loss (library routine);
* the sparse forward against a dense numpy product;
* N = 1, gamma = 0 Adaptive SGD == textbook torch.optim.SGD.
"""
import numpy as np
import pytest
import torch

from synth import config, generate, init_params, sample_stream
from oracle import model, adaptive

SMALL = dict(F=50, L=10, H=8, n_train=64, n_test=16, s_bar=6.0, s_sigma=0.3, y_bar=2.0, b_max=4)


def _small(seed_index=7, **kw):
    args = dict(SMALL)
    args.update(kw)
    return config("tiny", index=seed_index, **args)


def _batch_and_params(cfg, B=4, rng_seed=0):
    data = generate(cfg)
    rows = np.arange(B)
    batch = data.row_slice(rows)
    rng = np.random.default_rng(rng_seed)
    w = init_params(cfg).astype(np.float64)
    # non-zero biases so every term of the gradient is exercised
    from synth import param_layout
    lay = param_layout(cfg.F, cfg.H, cfg.L)
    o, _ = lay["b1"]
    w[o:o + cfg.H] = rng.normal(0, 0.3, cfg.H)
    o, _ = lay["b2"]
    w[o:o + cfg.L] = rng.normal(0, 0.3, cfg.L)
    o, _ = lay["W2"]
    w[o:o + cfg.L * cfg.H] *= 3.0
    return data, batch, w


@pytest.mark.parametrize("loss_kind", ["softmax", "sigmoid"])
def test_finite_differences(loss_kind):
    cfg = _small()
    F, H, L = cfg.F, cfg.H, cfg.L
    _, batch, w = _batch_and_params(cfg)
    A1, _, _ = model.forward(w, batch, F, H, L)
    h = 1e-6
    assert np.abs(A1).min() > 100 * h, "a ReLU kink is within FD reach; pick another seed"
    loss, g = model.loss_and_grad(w, batch, F, H, L, loss_kind)
    fd = np.zeros_like(w)
    for i in range(len(w)):
        wp = w.copy(); wp[i] += h
        wm = w.copy(); wm[i] -= h
        fd[i] = (model.loss_only(wp, batch, F, H, L, loss_kind) - model.loss_only(wm, batch, F, H, L, loss_kind)) / (2 * h)
    from synth import param_layout
    lay = param_layout(F, H, L)
    for name in ("W1", "b1", "W2", "b2"):
        o, shp = lay[name]
        n = int(np.prod(shp))
        a, b = g[o:o + n], fd[o:o + n]
        err = np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-30)
        assert err < 1e-6, (name, err)
        assert np.linalg.norm(b) > 0, name
    assert np.isfinite(loss) and loss > 0


def _torch_loss(w, batch, F, H, L, loss_kind="softmax"):
    from synth import param_layout
    lay = param_layout(F, H, L)
    wt = torch.tensor(w, dtype=torch.float64, requires_grad=True)
    def view(name):
        o, shp = lay[name]
        return wt[o:o + int(np.prod(shp))].view(*shp)
    W1, b1, W2, b2 = view("W1"), view("b1"), view("W2"), view("b2")
    B = batch.n_rows
    X = torch.zeros(B, F, dtype=torch.float64)
    T = torch.zeros(B, L, dtype=torch.float64)
    for n in range(B):
        cols = batch.col[batch.row_ptr[n]:batch.row_ptr[n + 1]]
        X[n, torch.as_tensor(cols, dtype=torch.long)] = torch.as_tensor(
            batch.val[batch.row_ptr[n]:batch.row_ptr[n + 1]], dtype=torch.float64)
        labs = batch.lab[batch.lab_ptr[n]:batch.lab_ptr[n + 1]]
        T[n, torch.as_tensor(labs, dtype=torch.long)] = 1.0 / len(labs) if loss_kind == "softmax" else 1.0
    Z = torch.relu(X @ W1 + b1) @ W2.T + b2
    if loss_kind == "softmax":
        loss = torch.nn.functional.cross_entropy(Z, T)   # soft targets, batch mean
    else:   # per-label BCE summed over labels, batch mean (R11)
        loss = torch.nn.functional.binary_cross_entropy_with_logits(Z, T, reduction="sum") / B
    loss.backward()
    return float(loss), wt.grad.numpy()


@pytest.mark.parametrize("loss_kind", ["softmax", "sigmoid"])
@pytest.mark.parametrize("seed_index,B", [(7, 4), (11, 16)])
def test_against_torch_autograd(seed_index, B, loss_kind):
    cfg = _small(seed_index, n_train=64)
    F, H, L = cfg.F, cfg.H, cfg.L
    _, batch, w = _batch_and_params(cfg, B=B)
    loss, g = model.loss_and_grad(w, batch, F, H, L, loss_kind)
    tl, tg = _torch_loss(w, batch, F, H, L, loss_kind)
    assert abs(loss - tl) <= 1e-12 * abs(tl)
    assert np.linalg.norm(g - tg) <= 1e-12 * np.linalg.norm(tg)


def test_sparse_forward_matches_dense():
    cfg = _small(5, F=300, L=40, H=16, s_bar=20.0)
    F, H, L = cfg.F, cfg.H, cfg.L
    _, batch, w = _batch_and_params(cfg, B=8)
    A1, H1, Z = model.forward(w, batch, F, H, L)
    W1, b1, W2, b2 = model.split_params(w, F, H, L)
    Xd = np.zeros((batch.n_rows, F))
    for n in range(batch.n_rows):
        for k in range(batch.row_ptr[n], batch.row_ptr[n + 1]):
            Xd[n, batch.col[k]] += batch.val[k]
    ref = Xd @ W1 + b1
    np.testing.assert_allclose(A1, ref, rtol=1e-13, atol=1e-15)
    np.testing.assert_allclose(Z, np.maximum(ref, 0) @ W2.T + b2, rtol=1e-12, atol=1e-14)


def test_touched_features_is_unique_of_cols():
    cfg = _small(5, F=300, L=40, H=16, s_bar=20.0)
    _, batch, _ = _batch_and_params(cfg, B=8)
    t = model.touched_features(batch)
    brute = sorted({int(c) for c in batch.col})
    assert t.tolist() == brute


def test_single_replica_no_momentum_is_minibatch_sgd():
    """with one GPU every method becomes mini-batch SGD
    (exactly so when gamma = 0, reading on N = 1)."""
    cfg = _small(3, F=120, L=12, H=8, n_train=96, b_max=8)
    F, H, L = cfg.F, cfg.H, cfg.L
    data = generate(cfg)
    w0 = init_params(cfg).astype(np.float64)
    M, lr, n_mb = 24, 0.5, 3
    recs = adaptive.run(F, H, L, data, w0, lambda mb: sample_stream(cfg, mb * M, M),
                        n_rep=1, n_mb=n_mb, M=M, b_max=8, b_min=1, beta=1, lr_max=lr, gamma=0.0)
    # textbook loop
    from synth import param_layout
    lay = param_layout(F, H, L)
    wt = torch.tensor(w0, dtype=torch.float64, requires_grad=True)
    opt = torch.optim.SGD([wt], lr=lr)
    for mb in range(n_mb):
        rows = sample_stream(cfg, mb * M, M)
        for s in range(0, M, 8):
            batch = data.row_slice(rows[s:s + 8])
            opt.zero_grad()
            _, g = _torch_loss(wt.detach().numpy().copy(), batch, F, H, L)
            wt.grad = torch.tensor(g)
            opt.step()
    np.testing.assert_allclose(recs[-1].w, wt.detach().numpy(), rtol=1e-12, atol=1e-14)
    assert [len(r.routes) for r in recs] == [3, 3, 3]
