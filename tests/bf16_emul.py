"""fp64 reference of the bf16 path's rounding points (R3, R4, R11) --
test helper, not the oracle.

The north-star check of the bf16 path is normwise against the fp64 oracle
(2e-2).  That bar cannot see a localized bug (one wrong row moves a normwise
error by ~1/sqrt(rows)), and a per-row or per-element comparison against the
exact gradient fails on bf16's own rounding: a W2 gradient row is a sum of
p - T terms that cancel, and rounding its operands to 8 bits moves it by a few
percent of its norm (measured by this module: up to 2.2 % at the planted
state).  So per-row and elementwise parity of the bf16 path is checked against
this reference instead, which is the same mathematics with the operands
rounded where the kernels round them (round-to-nearest-even to bf16) and every
product and sum in fp64:

  softmax (R3, R4):  Hq = bf(H1), Wq = bf(W2)   (the bf16 W2 shadow)
                     Z = Hq Wq^T + b2;  dZq = bf((softmax(Z) - T) / B)
                     dW2 = dZq^T Hq;  db2 = 1^T dZq;  dH1 = dZq Wq
                     dA1 = dH1 * [A1 > 0];  db1 = 1^T dA1;  dW1 = X^T bf(dA1)
  sigmoid (R11):     dZc = bf((sigmoid(Z) - 1/2 - Y) / B)   (centred)
                     dW2 = dZc^T Hq + (1/(2B)) 1 (sum_n H1_n)^T;  db2 = 1^T dZc + 1/2
                     dH1 = dZc Wq + (1/(2B)) sum_j Wq_j
What is left between it and the kernels is fp32 accumulation order, ex2.approx,
the rare element whose fp32 value sits at a bf16 rounding midpoint, and the
ReLU mask where the GPU's fp32 A1 and the fp64 one straddle zero.  For the last
one `slack` bounds what a flipped mask element can move: every (n, h) with
|A1_nh| within the fp32 SpMM error bound (s_n 2^-24 sum_f |x_nf| |W1_fh| +
2^-24 |b1_h|, s_n = the row's nnz) may go either way, moving dW1[f, h] by at
most |x_nf| |dH1_nh| (1 + 2^-7) and db1[h] by |dH1_nh|."""
import numpy as np
import scipy.sparse as sp


def bf16(x):
    """Round-to-nearest-even to bf16 of fp32(x), returned as fp64."""
    f = np.asarray(x, dtype=np.float32).copy()
    u = f.view(np.uint32)
    u += 0x7FFF + ((u >> 16) & 1)
    u &= 0xFFFF0000
    return f.astype(np.float64)


def grads_bf16(w, batch, F, H, L, loss="softmax", B_full=None, with_slack=False, rounding=True):
    """Flat gradient (layout W1, b1, W2, b2) of the rows of `batch` as the bf16
    path computes it; B_full = the step's row count when `batch` is a chunk of
    it (the 1/B scale is applied before the dZ rounding, as in the kernels).
    with_slack: also the flat per-element slack of ReLU-kink elements (above).
    rounding=False: the same code with every rounding point the identity (the exact
    gradient; its slack serves the fp32 path's elementwise check)."""
    bf = bf16 if rounding else (lambda x: np.asarray(x, dtype=np.float64))
    w = np.asarray(w, dtype=np.float64)
    o = 0
    W1 = w[o:o + F * H].reshape(F, H); o += F * H
    b1 = w[o:o + H]; o += H
    W2 = w[o:o + L * H].reshape(L, H); o += L * H
    b2 = w[o:o + L]
    n = batch.n_rows
    B = n if B_full is None else B_full
    X = sp.csr_matrix((batch.val.astype(np.float64), batch.col, batch.row_ptr), shape=(n, F))
    cnt = np.diff(batch.lab_ptr)
    A1 = np.asarray(X @ W1) + b1
    H1 = np.maximum(A1, 0.0)
    Hq, Wq = bf(H1), bf(W2)
    Z = Hq @ Wq.T + b2
    if loss == "softmax":
        tv = np.repeat(1.0 / np.maximum(cnt, 1), cnt)
        T = sp.csr_matrix((tv, batch.lab, batch.lab_ptr), shape=(n, L)).toarray()
        m = Z.max(axis=1, keepdims=True)
        P = np.exp(Z - m)
        P /= P.sum(axis=1, keepdims=True)
        dZ = bf((P - T) / B)
        dW2 = dZ.T @ Hq
        db2 = dZ.sum(axis=0)
        dH1 = dZ @ Wq
    elif loss == "sigmoid":
        Y = sp.csr_matrix((np.ones(int(cnt.sum())), batch.lab, batch.lab_ptr), shape=(n, L)).toarray()
        S = 1.0 / (1.0 + np.exp(-Z))
        dZ = bf((S - 0.5 - Y) / B)
        dW2 = dZ.T @ Hq + (1.0 / (2 * B)) * H1.sum(axis=0)[None, :]
        db2 = dZ.sum(axis=0) + 0.5 * n / B
        dH1 = dZ @ Wq + (1.0 / (2 * B)) * Wq.sum(axis=0)[None, :]
    else:
        raise ValueError(loss)
    dA1 = dH1 * (A1 > 0.0)
    db1 = dA1.sum(axis=0)
    dW1 = np.asarray(X.T @ bf(dA1))
    g = np.concatenate([dW1.ravel(), db1, dW2.ravel(), db2])
    if not with_slack:
        return g
    Xa = abs(X)
    nnz_row = np.diff(batch.row_ptr).astype(np.float64)[:, None]
    bound = nnz_row * 2.0 ** -24 * np.asarray(Xa @ np.abs(W1)) + 2.0 ** -24 * np.abs(b1)[None, :]
    kink = (np.abs(A1) <= bound) * np.abs(dH1) * (1 + 2.0 ** -7)
    sl = np.zeros_like(g)
    sl[:F * H] = np.asarray(Xa.T @ kink).ravel()
    sl[F * H:F * H + H] = kink.sum(axis=0)
    return g, sl
