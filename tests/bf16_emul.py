"""fp64 reference of the tensor-core paths' rounding points (R3, R4,
R11, R14) -- test helper, not the oracle.

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
  fp32 path as bf16x3 (R14): every product of the three GEMMs is
                     hi_a hi_b + hi_a lo_b + lo_a hi_b of the fp32 operands split into
                     bf16 hi = bf(x), lo = bf(x - hi); dZ (softmax: fp32; sigmoid: the
                     centred fp32 value) is split the same way; db2 = 1^T (hi + lo)
                     of dZ; dW1 = X^T dA1 with fp32 dA1; the centred-sigmoid offsets
                     use the fp32 W2 and H1.
What is left between the reference and the kernels are decisions the two sides
may take differently: the GPU's fp32 A1 (K-1) straddling the ReLU kink or a bf16
rounding midpoint where the fp64 one does not, its fp32 Z / lse / exp moving p
by a few ulps (and through that a dZ rounding), and fp32 accumulation orders.
With `with_slack` the function also returns a first-order componentwise bound of
what those can move, per element of dW1, db1, dW2 and db2 (slack below), so the
elementwise check can stay at the tolerance everywhere else.  R(.) is the
rounding the path applies to a GEMM operand (bf16; the bf16x3 hi + lo; or none),
flip(q, d) = max over q' in [q - d, q + d] of |R(q') - R(q)| (exact, elementwise),
u = 2^-24:
fp32 sums are bounded by the 4-sigma rounding walk g(k) = 4 sqrt(k) u over k terms
(worst-case k u bounds would cover every element and leave the check no bite):
  dH  = flip(H1, eA1),  eA1 = g(s_n) sum_f |x_nf||W1_fh| + u |b1_h|   (K-1's fp32 sum)
  dZl = dH |Wq|^T + g(H) |Hq||Wq|^T                      (logits)
  dp  = p (dZl + sum_j p_j dZl_j + 4e-6)                 (softmax: the lse error is at most
                                                          the p-weighted logit error; 4e-6:
                                                          fp32 exp / log); sigmoid: dZl / 4
  ddZ = flip(dZ, dp / B + u |dZ|)
  dW2 : ddZ^T |Hq| + |dZq|^T dH + g(B) |dZq|^T |Hq|
  db2 : sum_n ddZ + g(B) sum_n |dZq|
  dH1 : ddZ |Wq| + g(L) |dZq| |Wq|
  dA1 : [A1 > 0] dH1-error + [|A1| <= eA1] (|dH1| + its error)   (the kink)
  dW1 : |X|^T flip(dA1, dA1-error) + g(B) |X|^T |dA1|;   db1: sum_n dA1-error + g(B) sum_n |dA1|
"""
import numpy as np
import scipy.sparse as sp


def bf16(x):
    """Round-to-nearest-even to bf16 of fp32(x), returned as fp64."""
    f = np.asarray(x, dtype=np.float32).copy()
    u = f.view(np.uint32)
    u += 0x7FFF + ((u >> 16) & 1)
    u &= 0xFFFF0000
    return f.astype(np.float64)


def f32(x):
    return np.asarray(x, dtype=np.float32).astype(np.float64)


def split3(x):
    """bf16x3 halves (R14) of fp32(x): hi = bf(x), lo = bf(x - hi)."""
    xf = f32(x)
    hi = bf16(xf)
    return hi, bf16(xf - hi)


def mm3(A, B):
    """A @ B as the bf16x3 GEMMs form it: hi.hi + hi.lo + lo.hi (fp64 sums)."""
    Ah, Al = split3(A)
    Bh, Bl = split3(B)
    return Ah @ Bh + (Ah @ Bl + Al @ Bh)


def grads_bf16(w, batch, F, H, L, loss="softmax", B_full=None, with_slack=False, rounding=True):
    """Flat gradient (layout W1, b1, W2, b2) of the rows of `batch` as the bf16
    path computes it; B_full = the step's row count when `batch` is a chunk of
    it (the 1/B scale is applied before the dZ rounding, as in the kernels).
    with_slack: also the flat per-element slack of ReLU-kink elements (above).
    rounding: True / "bf16" = the bf16 path; "x3" = the fp32 path's bf16x3 products;
    False = every rounding point the identity (the exact gradient)."""
    mode = {True: "bf16", False: "exact"}.get(rounding, rounding)
    ident = lambda x: np.asarray(x, dtype=np.float64)   # noqa: E731
    bf = bf16 if mode == "bf16" else ident
    if mode == "x3":
        mm = mm3
    else:
        mm = lambda A, Bm: A @ Bm                          # noqa: E731
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
    Z = mm(Hq, Wq.T) + b2
    if loss == "softmax":
        tv = np.repeat(1.0 / np.maximum(cnt, 1), cnt)
        T = sp.csr_matrix((tv, batch.lab, batch.lab_ptr), shape=(n, L)).toarray()
        m = Z.max(axis=1, keepdims=True)
        P = np.exp(Z - m)
        P /= P.sum(axis=1, keepdims=True)
        dZ = bf((P - T) / B)
        if mode == "x3":
            dZ = f32(dZ)
        dW2 = mm(dZ.T, Hq)
        db2 = (sum(split3(dZ)) if mode == "x3" else dZ).sum(axis=0)
        dH1 = mm(dZ, Wq)
    elif loss == "sigmoid":
        Y = sp.csr_matrix((np.ones(int(cnt.sum())), batch.lab, batch.lab_ptr), shape=(n, L)).toarray()
        S = 1.0 / (1.0 + np.exp(-Z))
        dZ = bf((S - 0.5 - Y) / B)
        if mode == "x3":
            dZ = f32(dZ)
        dW2 = mm(dZ.T, Hq) + (1.0 / (2 * B)) * H1.sum(axis=0)[None, :]
        db2 = (sum(split3(dZ)) if mode == "x3" else dZ).sum(axis=0) + 0.5 * n / B
        dH1 = mm(dZ, Wq) + (1.0 / (2 * B)) * (W2 if mode == "x3" else Wq).sum(axis=0)[None, :]
    else:
        raise ValueError(loss)
    dA1 = dH1 * (A1 > 0.0)
    db1 = dA1.sum(axis=0)
    dW1 = np.asarray(X.T @ (f32(dA1) if mode == "x3" else bf(dA1)))
    g = np.concatenate([dW1.ravel(), db1, dW2.ravel(), db2])
    if not with_slack:
        return g
    return g, _slack(mode, X, W1, b1, A1, H1, Hq, Wq, W2, Z, dZ, dH1, dA1, B, L, F, H, loss,
                     P if loss == "softmax" else S)


def _rnd(mode):
    if mode == "bf16":
        return bf16
    if mode == "x3":
        return lambda x: sum(split3(x))
    return lambda x: np.asarray(x, dtype=np.float64)


def _flip(mode, q, d):
    """max |R(q') - R(q)| over q' in [q - d, q + d] (R monotone: the two ends)."""
    if mode == "exact":
        return np.asarray(d, dtype=np.float64)
    R = _rnd(mode)
    r0 = R(q)
    return np.maximum(np.abs(R(q + d) - r0), np.abs(R(q - d) - r0))


def _slack(mode, X, W1, b1, A1, H1, Hq, Wq, W2, Z, dZ, dH1, dA1, B, L, F, H, loss, P):
    u = 2.0 ** -24
    Xa = abs(X)
    n = X.shape[0]
    nnz_row = np.diff(X.indptr).astype(np.float64)[:, None]
    g4 = lambda k: 4.0 * np.sqrt(k) * u   # noqa: E731  4-sigma fp32 rounding walk over k terms
    eA1 = g4(nnz_row) * np.asarray(Xa @ np.abs(W1)) + u * np.abs(b1)[None, :]
    dH = _flip(mode, H1, eA1) * (A1 > -eA1)
    aH, aW = np.abs(Hq), np.abs(Wq)
    dZl = dH @ aW.T + g4(H) * (aH @ aW.T)
    if loss == "softmax":   # lse error <= the p-weighted logit error; 4e-6: fp32 exp / log
        dp = P * (dZl + (P * dZl).sum(axis=1, keepdims=True) + 4e-6)
    else:
        dp = dZl / 4.0
    ddZ = _flip(mode, dZ, dp / B + u * np.abs(dZ))
    aZ = np.abs(dZ)
    s_W2 = ddZ.T @ aH + aZ.T @ dH + g4(B) * (aZ.T @ aH)
    s_b2 = ddZ.sum(axis=0) + g4(B) * aZ.sum(axis=0)
    e_dH1 = ddZ @ aW + g4(L) * (aZ @ aW)
    kink = np.abs(A1) <= eA1
    e_dA1 = (A1 > 0.0) * e_dH1 + kink * (np.abs(dH1) + e_dH1)
    k5 = _flip("bf16", dA1, e_dA1) if mode == "bf16" else e_dA1 + u * np.abs(dA1)
    s_W1 = np.asarray(Xa.T @ k5) + g4(B) * np.asarray(Xa.T @ np.abs(dA1))
    s_b1 = e_dA1.sum(axis=0) + g4(B) * np.abs(dA1).sum(axis=0)
    return np.concatenate([s_W1.ravel(), s_b1, s_W2.ravel(), s_b2])
