"""Oracle: one local minibatch SGD step of the paper's XML network, fp64.

Model (§V-A "3-layer MLP ... ReLU layer activation, softmax
multi-class probability, and cross-entropy loss"), readings from DESIGN.md:
  A1 = X W1 + b1,  H1 = max(A1, 0),  Z = H1 W2^T + b2         (Q1, Q2)
  loss = (1/B) sum_n [ lse(Z_n) - sum_j T_nj Z_nj ],  T_nj = 1/|Y_n| on Y_n (Q3, Q4)
Variant (north star "softmax/sigmoid cross-entropy"; reading
R11): loss="sigmoid" is the per-label binary cross-entropy with 0/1 targets,
  loss = (1/B) sum_n sum_j [ softplus(Z_nj) - Y_nj Z_nj ],  dZ = (sigmoid(Z) - Y) / B.
SGD (§II): forward pass, backward pass by the chain rule, update
theta <- theta - lr * grad with pre-step values (Q26, plain SGD).
ReLU'(0) = 0 (Q6).  Parameters are one flat vector W1 (F x H), b1 (H),
W2 (L x H), b2 (L).

Test infrastructure only (see oracle/__init__.py).
"""
from __future__ import annotations

import numpy as np
import scipy.sparse as sp


def split_params(w: np.ndarray, F: int, H: int, L: int):
    """Views W1, b1, W2, b2 of the flat vector (layout SURVEY D3)."""
    o = 0
    W1 = w[o:o + F * H].reshape(F, H); o += F * H
    b1 = w[o:o + H]; o += H
    W2 = w[o:o + L * H].reshape(L, H); o += L * H
    b2 = w[o:o + L]; o += L
    assert o == len(w)
    return W1, b1, W2, b2


def batch_matrices(batch, F: int, L: int, loss: str = "softmax"):
    """X (B x F) and the target T (B x L) of a CSR batch, both fp64 sparse.

    softmax: T_nj = 1/|Y_n| for j in Y_n (reading Q3: uniform target over true
    labels); sigmoid: T_nj = 1 for j in Y_n (binary targets, R11)."""
    B = batch.n_rows
    X = sp.csr_matrix((batch.val.astype(np.float64), batch.col, batch.row_ptr), shape=(B, F))
    cnt = np.diff(batch.lab_ptr)
    tv = np.repeat(1.0 / np.maximum(cnt, 1), cnt) if loss == "softmax" else np.ones(int(cnt.sum()))
    T = sp.csr_matrix((tv, batch.lab, batch.lab_ptr), shape=(B, L))
    return X, T


def logsumexp_rows(Z: np.ndarray) -> np.ndarray:
    m = Z.max(axis=1, keepdims=True)
    return (m + np.log(np.exp(Z - m).sum(axis=1, keepdims=True)))[:, 0]


def forward(w, batch, F, H, L):
    """Forward pass: returns A1, H1, Z."""
    W1, b1, W2, b2 = split_params(w, F, H, L)
    X, _ = batch_matrices(batch, F, L)
    A1 = np.asarray(X @ W1) + b1
    H1 = np.maximum(A1, 0.0)
    Z = H1 @ W2.T + b2
    return A1, H1, Z


def softplus(Z: np.ndarray) -> np.ndarray:
    """log(1 + e^Z) without overflow: max(Z, 0) + log1p(e^-|Z|)."""
    return np.maximum(Z, 0.0) + np.log1p(np.exp(-np.abs(Z)))


def _head(Z, T, loss):
    """Mean loss and dZ * B of the output layer for the chosen loss."""
    B = Z.shape[0]
    TZ = np.asarray(T.multiply(Z).sum(axis=1))[:, 0]
    if loss == "softmax":
        lse = logsumexp_rows(Z)
        return float(np.mean(lse - TZ)), np.exp(Z - lse[:, None]) - T.toarray()
    if loss == "sigmoid":
        return float(np.mean(softplus(Z).sum(axis=1) - TZ)), 1.0 / (1.0 + np.exp(-Z)) - T.toarray()
    raise ValueError(loss)


def loss_and_grad(w, batch, F, H, L, loss: str = "softmax"):
    """Loss and full gradient (flat, same layout as w) of one batch, fp64.

    Backward pass = chain rule:
      dZ  = (softmax(Z) - T) / B        [sigmoid: (sigmoid(Z) - Y) / B]
      dW2 = dZ^T H1,   db2 = 1^T dZ,   dH1 = dZ W2
      dA1 = dH1 * [A1 > 0]
      dW1 = X^T dA1,   db1 = 1^T dA1
    """
    W1, b1, W2, b2 = split_params(w, F, H, L)
    X, T = batch_matrices(batch, F, L, loss)
    B = batch.n_rows
    A1 = np.asarray(X @ W1) + b1
    H1 = np.maximum(A1, 0.0)
    Z = H1 @ W2.T + b2
    lval, dZB = _head(Z, T, loss)
    dZ = dZB / B
    dW2 = dZ.T @ H1
    db2 = dZ.sum(axis=0)
    dH1 = dZ @ W2
    dA1 = dH1 * (A1 > 0.0)
    dW1 = np.asarray(X.T @ dA1)
    db1 = dA1.sum(axis=0)
    g = np.concatenate([dW1.ravel(), db1, dW2.ravel(), db2])
    return lval, g


def loss_only(w, batch, F, H, L, loss: str = "softmax") -> float:
    _, _, Z = forward(w, batch, F, H, L)
    _, T = batch_matrices(batch, F, L, loss)
    return _head(Z, T, loss)[0]


def touched_features(batch) -> np.ndarray:
    """Sorted unique feature ids the batch touches (rows of W1 with a
    possibly non-zero gradient); np.unique is the library routine."""
    return np.unique(batch.col).astype(np.int32)


def sgd_step(w, batch, lr, F, H, L, loss: str = "softmax"):
    """One SGD step: theta <- theta - lr * grad (pre-step values).

    Returns (new w, loss, grad)."""
    lval, g = loss_and_grad(w, batch, F, H, L, loss)
    return w - lr * g, lval, g
