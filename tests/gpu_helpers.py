"""Shared helpers of the GPU parity tests (CUDA path vs the CPU oracle)."""
import functools
import json
import os

import numpy as np
import torch

from synth import config, generate, init_params, param_layout, sample_stream
from synth.xmlgen import Dataset


@functools.lru_cache(maxsize=None)
def dataset(name: str, n_rows=None, split="train"):
    return generate(config(name), split, n_rows)


def normwise(a, b):
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    nb = np.linalg.norm(b)
    return np.linalg.norm(a - b) / (nb if nb > 0 else 1.0)


def _row_errors(a, b, slack=None):
    """Per-row error ||a_r - b_r|| / max(||b_r||, rms row norm of b): relative to
    the row's own norm, with rows far below the typical norm measured against
    the typical norm (a row wrong by 100 % of a typical row fails).  With slack,
    each element's difference is first reduced by its allowance, max(|a - b| -
    slack, 0), as in the elementwise check (R16)."""
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    if a.shape[0] == 0:
        return np.zeros(0)
    nb = np.linalg.norm(b, axis=1)
    floor = np.sqrt(np.mean(nb * nb))
    d = np.abs(a - b)
    if slack is not None:
        d = np.maximum(d - np.asarray(slack, dtype=np.float64).reshape(d.shape), 0.0)
    return np.linalg.norm(d, axis=1) / np.maximum(nb, floor if floor > 0 else 1.0)


def _elem_err(a, b, tol, per_row, slack=None):
    """max (|a - b| - slack) / (tol |b| + tol s): s = the RMS of b's row (per_row)
    or of the whole tensor; <= 1 passes."""
    a = np.asarray(a, dtype=np.float64)
    b = np.asarray(b, dtype=np.float64)
    if b.size == 0:
        return 0.0
    if per_row and b.ndim == 2:
        s = np.sqrt(np.mean(b * b, axis=1, keepdims=True))
    else:
        s = np.sqrt(np.mean(b * b))
    d = np.abs(a - b)
    if slack is not None:
        d = np.maximum(d - np.asarray(slack, dtype=np.float64).reshape(d.shape), 0.0)
    return float((d / (tol * np.abs(b) + tol * s + 1e-300)).max(initial=0.0))


def check_grads(gg, og, tol, F, H, touched, tag="", emul=None, slack=None):
    """Normwise, per-row and elementwise parity of the four gradient tensors.

    * normwise ||g - o|| / ||o|| <= tol per tensor against the fp64 oracle
      (north_star tolerance);
    * per row (W1 touched rows, W2 rows): _row_errors <= tol;
    * elementwise: |g - r| - slack <= tol |r| + tol rms_row(r) (numpy assert_allclose
      with rtol = tol and atol = tol times the RMS of the element's row), W1
      restricted to the touched rows; slack = the componentwise allowance of
      tests/bf16_emul.py for the rounding decisions and fp32 accumulation orders the
      GPU and the reference may take differently (ReLU kink, bf16 midpoints, ...).
      The row RMS, not the tensor's: the tensor-core paths round operands, so an
      element's error scales with its row's summands (a head feature's W1 row is
      ~100x the typical one), not with the tensor's typical element.
    With emul (the gradient of tests/bf16_emul.py: the same mathematics with the
    kernels' rounding points -- bf16 operands, or the fp32 path's bf16x3 products),
    r is that reference; without, the fp64 oracle.  bf16 operand
    rounding alone moves single W2 rows of the exact gradient by a few percent
    (see bf16_emul.py), so a localized bug is looked for against the rounded
    arithmetic, while the exact-gradient bar stays the normwise one.
    The achieved errors are returned and appended to $ASGD_PARITY_LOG (JSON
    lines) when that is set, so the margin under each bar is on record."""
    L = len(og["b2"])
    rec = {"tag": tag, "tol": tol, "ref": "rounding-emulation" if emul is not None else "oracle"}
    for k in ("W1", "b1", "W2", "b2"):
        rec[f"norm_{k}"] = float(normwise(gg[k], og[k]))
    ref = emul if emul is not None else og
    W1g = np.asarray(gg["W1"]).reshape(F, H)[touched]
    W1r = np.asarray(ref["W1"]).reshape(F, H)[touched]
    W2g = np.asarray(gg["W2"]).reshape(L, H)
    W2r = np.asarray(ref["W2"]).reshape(L, H)
    pairs = {"W1": (W1g, W1r), "b1": (gg["b1"], ref["b1"]), "W2": (W2g, W2r), "b2": (gg["b2"], ref["b2"])}
    sl = {}
    if slack is not None:
        sl = {"W1": np.asarray(slack["W1"]).reshape(F, H)[touched], "b1": slack["b1"],
              "W2": np.asarray(slack["W2"]).reshape(L, H), "b2": slack["b2"]}
        rec["slack_rel"] = {k: float(np.linalg.norm(v) / (np.linalg.norm(np.asarray(pairs[k][1])) + 1e-300))
                            for k, v in sl.items()}
    # per row, with the same componentwise allowance as the elementwise check (R16); the
    # unreduced row error is logged beside it
    rec["row_W1_max"] = float(_row_errors(W1g, W1r, sl.get("W1")).max(initial=0.0))
    rec["row_W2_max"] = float(_row_errors(W2g, W2r, sl.get("W2")).max(initial=0.0))
    if sl:
        rec["row_W1_max_raw"] = float(_row_errors(W1g, W1r).max(initial=0.0))
        rec["row_W2_max_raw"] = float(_row_errors(W2g, W2r).max(initial=0.0))
    if emul is not None:   # for the record: per-row distance of the bf16 path to the exact gradient
        rec["row_W2_max_vs_oracle"] = float(_row_errors(W2g, np.asarray(og["W2"]).reshape(L, H)).max(initial=0.0))
    for k, (a, b) in pairs.items():
        rec[f"elem_{k}"] = _elem_err(a, b, tol, per_row=True, slack=sl.get(k))
    # where the worst W1 / W2 elements sit (diagnostics for the log)
    if W2r.size:
        d = np.abs(W2g - W2r)
        if "W2" in sl:
            d = np.maximum(d - sl["W2"], 0.0)
        rr = np.sqrt(np.mean(W2r * W2r, axis=1, keepdims=True))
        q = d / (tol * np.abs(W2r) + tol * rr + 1e-300)
        i, j = np.unravel_index(int(np.argmax(q)), q.shape)
        rec["worst_W2"] = {"label": int(i), "col": int(j), "got": float(W2g[i, j]), "ref": float(W2r[i, j]),
                           "row_rms": float(rr[i, 0]), "row_norm_got": float(np.linalg.norm(W2g[i])),
                           "oracle": float(np.asarray(og["W2"]).reshape(L, H)[i, j])}
    if W1r.size:
        d = np.abs(W1g - W1r)
        if "W1" in sl:
            d = np.maximum(d - sl["W1"], 0.0)
        rr = np.sqrt(np.mean(W1r * W1r, axis=1, keepdims=True))
        q = d / (tol * np.abs(W1r) + tol * rr + 1e-300)
        i, j = np.unravel_index(int(np.argmax(q)), q.shape)
        rec["worst_W1"] = {"feature": int(np.asarray(touched)[i]), "col": int(j), "got": float(W1g[i, j]),
                           "ref": float(W1r[i, j]), "row_rms": float(rr[i, 0]),
                           "slack": float(sl["W1"][i, j]) if "W1" in sl else 0.0}
    log = os.environ.get("ASGD_PARITY_LOG")
    if log:
        with open(log, "a") as f:
            f.write(json.dumps(rec) + "\n")
    for k in ("W1", "b1", "W2", "b2"):
        assert rec[f"norm_{k}"] <= tol, (tag, k, rec)
        assert rec[f"elem_{k}"] <= 1.0, (tag, "elementwise", k, rec)
    assert rec["row_W1_max"] <= tol, (tag, "W1 row", rec)
    assert rec["row_W2_max"] <= tol, (tag, "W2 row", rec)
    return rec


def split_grad(g, F, H, L):
    lay = param_layout(F, H, L)
    out = {}
    for k in ("W1", "b1", "W2", "b2"):
        o, shp = lay[k]
        out[k] = g[o:o + int(np.prod(shp))]
    return out


def make_replica(cfg, data, precision="fp32", w0=None, b_max=None, extra=(), loss="softmax"):
    from paper_conf_ipps_marws22_b200 import api
    b_max = b_max or cfg.b_max
    nz, nl = api.max_step_sizes([data, *extra], b_max)
    if w0 is None:
        w0 = init_params(cfg)
    rep = api.Replica(cfg.F, cfg.L, cfg.H, b_max, nz, nl, precision, w0=w0, loss=loss)
    dd = api.DeviceCsr(data)
    rep.register(dd)
    rep._keep_data = dd
    return rep


def with_empty_row(ds: Dataset, at: int) -> Dataset:
    """Copy of ds where row `at` has no features (labels kept)."""
    rp = ds.row_ptr.copy()
    n0 = rp[at + 1] - rp[at]
    keep = np.ones(len(ds.col), dtype=bool)
    keep[rp[at]:rp[at + 1]] = False
    rp[at + 1:] -= n0
    return Dataset(rp, ds.col[keep], ds.val[keep], ds.lab_ptr, ds.lab, ds.n_features, ds.n_labels)
