"""Shared helpers of the GPU parity tests (CUDA path vs the CPU oracle)."""
import functools

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
