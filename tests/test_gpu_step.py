"""Parity of the CUDA local step (libasgd, sm_100a) with the fp64 oracle.

Bit-exact: touched-feature sets.  Normwise relative error per tensor:
<= 1e-4 on the fp32 path, <= 2e-2 on the bf16 tensor-core path, for the
per-step loss and the debug-dumped gradients (north_star tolerances)."""
import numpy as np
import pytest
import torch

from oracle import model as omodel
from synth import config, init_params, planted_params, sample_stream
from tests.bf16_emul import grads_bf16
from tests.gpu_helpers import check_grads, dataset, make_replica, normwise, split_grad, with_empty_row

pytestmark = pytest.mark.gpu

TOL = {"fp32": 1e-4, "bf16": 2e-2}


def _one_step(cfg, data, rows, precision, lr=0.5, w0=None, b_max=None, loss_kind="softmax"):
    rep = make_replica(cfg, data, precision, w0=w0, b_max=b_max, loss=loss_kind)
    w0 = init_params(cfg) if w0 is None else w0
    g = torch.zeros(rep.P, dtype=torch.float32, device="cuda")
    loss = torch.zeros(1, dtype=torch.float32, device="cuda")
    rep.set_debug_grads(g)
    rows_d = torch.as_tensor(rows, dtype=torch.int32, device="cuda")
    rep.step(rows_d, lr, loss)
    rep.sync()
    touched = rep.last_touched().cpu().numpy()
    batch = data.row_slice(rows)
    lo, go = omodel.loss_and_grad(np.asarray(w0, dtype=np.float64), batch, cfg.F, cfg.H, cfg.L, loss_kind)
    em = grads_bf16(w0, batch, cfg.F, cfg.H, cfg.L, loss_kind, with_slack=True, rounding="bf16" if precision == "bf16" else "x3")
    return rep, g.cpu().numpy(), float(loss.item()), touched, lo, (go, em), batch


def _check(cfg, rep, g, loss, touched, lo, go_em, batch, precision, tag=""):
    go, em = go_em
    tol = TOL[precision]
    assert abs(loss - lo) <= tol * abs(lo), (loss, lo)
    np.testing.assert_array_equal(touched, omodel.touched_features(batch))
    gg, og = split_grad(g, cfg.F, cfg.H, cfg.L), split_grad(go, cfg.F, cfg.H, cfg.L)
    eg = split_grad(em[0], cfg.F, cfg.H, cfg.L)
    es = split_grad(em[1], cfg.F, cfg.H, cfg.L)
    check_grads(gg, og, tol, cfg.F, cfg.H, touched, tag=f"{cfg.name}/{precision}/{tag}", emul=eg, slack=es)
    # W1 gradient is exactly zero off the touched rows
    W1g = gg["W1"].reshape(cfg.F, cfg.H)
    off = np.ones(cfg.F, dtype=bool)
    off[touched] = False
    assert not W1g[off].any()


@pytest.mark.parametrize("precision", ["fp32", "bf16"])
def test_step_tiny(precision):
    cfg = config("tiny")
    data = dataset("tiny")
    rows = sample_stream(cfg, 0, cfg.b_max)
    _check(cfg, *_one_step(cfg, data, rows, precision), precision, "init")


@pytest.mark.parametrize("precision", ["fp32", "bf16"])
def test_step_eurlex_full_batch(precision):
    cfg = config("eurlex4k")
    data = dataset("eurlex4k")
    rows = sample_stream(cfg, 0, cfg.b_max)
    _check(cfg, *_one_step(cfg, data, rows, precision), precision, "init")


@pytest.mark.parametrize("precision", ["fp32", "bf16"])
@pytest.mark.parametrize("name", ["tiny", "eurlex4k"])
def test_step_planted_peaked_softmax(name, precision):
    """Teacher-forced step from the trained-like planted state (synth.planted_params:
    peaked softmax, logit range ~30, large W2), full batch, rows from pass 3."""
    cfg = config(name)
    data = dataset(name)
    rows = sample_stream(cfg, 3 * cfg.n_train + 7, cfg.b_max)
    w0 = planted_params(cfg)
    _check(cfg, *_one_step(cfg, data, rows, precision, w0=w0), precision, "planted")


@pytest.mark.parametrize("precision", ["fp32", "bf16"])
def test_step_ragged_and_empty_rows(precision):
    """Truncated batch (37 rows, Q9) with a feature-less row and a repeated row."""
    cfg = config("eurlex4k")
    data = with_empty_row(dataset("eurlex4k"), 5)
    rows = np.array([5, 0, 17, 5, 1000] + list(range(2000, 2032)), dtype=np.int32)
    _check(cfg, *_one_step(cfg, data, rows, precision), precision)


@pytest.mark.parametrize("precision", ["fp32", "bf16"])
def test_step_wiki10_skewed(precision):
    """Heavy nnz skew: rows of 10^3-10^4 entries span many K-1 pieces."""
    cfg = config("wiki10_31k")
    data = dataset("wiki10_31k", 2048)
    lens = np.diff(data.row_ptr)
    longest = np.argsort(lens)[-8:]
    rows = np.concatenate([longest, np.arange(0, cfg.b_max - 8)]).astype(np.int32)
    assert lens[rows].max() > 2000
    _check(cfg, *_one_step(cfg, data, rows, precision), precision)


@pytest.mark.parametrize("precision", ["fp32", "bf16"])
def test_step_is_deterministic(precision):
    cfg = config("eurlex4k")
    data = dataset("eurlex4k")
    rows = torch.as_tensor(sample_stream(cfg, 0, cfg.b_max), device="cuda")
    outs = []
    for _ in range(2):
        rep = make_replica(cfg, data, precision)
        for _ in range(3):
            rep.step(rows, 0.5)
        rep.sync()
        outs.append(rep.params.cpu().numpy())
    np.testing.assert_array_equal(outs[0], outs[1])


@pytest.mark.parametrize("precision", ["fp32", "bf16"])
def test_teacher_forced_steps_tiny(precision):
    """Every step starts both sides from the same state: the ORACLE's free-running
    trajectory (fp64 SGD from w0) is rounded to fp32 and loaded into the replica
    before each GPU step (no oracle input ever comes from the GPU)."""
    cfg = config("tiny")
    data = dataset("tiny")
    rep = make_replica(cfg, data, precision)
    g = torch.zeros(rep.P, dtype=torch.float32, device="cuda")
    rep.set_debug_grads(g)
    w = init_params(cfg).astype(np.float64)
    tol = TOL[precision]
    for k in range(10):
        rows = sample_stream(cfg, k * 32, 32)
        w32 = w.astype(np.float32)
        rep.params.copy_(torch.from_numpy(w32))
        rep.params_changed()
        rep.step(torch.as_tensor(rows, device="cuda"), 0.7)
        rep.sync()
        batch = data.row_slice(rows)
        _, go = omodel.loss_and_grad(w32.astype(np.float64), batch, cfg.F, cfg.H, cfg.L)
        gg, og = split_grad(g.cpu().numpy(), cfg.F, cfg.H, cfg.L), split_grad(go, cfg.F, cfg.H, cfg.L)
        e_, s_ = grads_bf16(w32, batch, cfg.F, cfg.H, cfg.L, with_slack=True, rounding="bf16" if precision == "bf16" else "x3")
        eg = split_grad(e_, cfg.F, cfg.H, cfg.L)
        es = split_grad(s_, cfg.F, cfg.H, cfg.L)
        check_grads(gg, og, tol, cfg.F, cfg.H, omodel.touched_features(batch), tag=f"tiny/{precision}/tf{k}",
                    emul=eg, slack=es)
        if precision == "fp32":
            w_after = rep.params.cpu().numpy().astype(np.float64)
            assert normwise(w_after, w32 - 0.7 * go) <= 1e-6
        w, _, _ = omodel.sgd_step(w, batch, 0.7, cfg.F, cfg.H, cfg.L)


# ---------------------------------------------------------------- sigmoid-BCE head (R11)
@pytest.mark.parametrize("precision", ["fp32", "bf16"])
@pytest.mark.parametrize("name", ["tiny", "eurlex4k"])
def test_step_sigmoid_bce(name, precision):
    """loss = ASGD_LOSS_SIGMOID: per-label BCE (R11); bf16 fuses it into G1's epilogue."""
    cfg = config(name)
    data = dataset(name)
    rows = sample_stream(cfg, 0, cfg.b_max)
    _check(cfg, *_one_step(cfg, data, rows, precision, loss_kind="sigmoid"), precision)


@pytest.mark.parametrize("precision", ["fp32", "bf16"])
def test_step_sigmoid_ragged_trained(precision):
    """Ragged batch (37 rows, an empty and a repeated row) from a model whose logits are
    far from 0 (W2 and b2 scaled up), so both sigmoid branches and the saturated softplus
    tail are exercised."""
    cfg = config("eurlex4k")
    data = with_empty_row(dataset("eurlex4k"), 5)
    rows = np.array([5, 0, 17, 5, 1000] + list(range(2000, 2032)), dtype=np.int32)
    w0 = init_params(cfg).astype(np.float64)
    F, H, L = cfg.F, cfg.H, cfg.L
    o2 = F * H + H
    w0[o2:o2 + L * H] *= 40.0
    w0[o2 + L * H:] = np.linspace(-12.0, 6.0, L)
    w0 = w0.astype(np.float32)
    _check(cfg, *_one_step(cfg, data, rows, precision, w0=w0, loss_kind="sigmoid"), precision)


def test_step_trace():
    """asgd_trace_enable / asgd_trace_read: one (start, rows, t0, t1) per local step, in
    order, times increasing; starts are the tickets' stream positions."""
    from paper_conf_ipps_marws22_b200 import api, train
    cfg = config("tiny")
    data = dataset("tiny")
    rep = make_replica(cfg, data, "bf16")
    h = train.Hyper.from_config(cfg)
    sched = api.Scheduler("/asgd_tr_" + str(np.random.randint(1 << 30)), 1, h.M, create=True)
    drv = train.DistributedAdaptiveSGD(rep, h, 0, 1, sched)
    ids = sample_stream(cfg, 0, h.M)
    rep.trace_enable(True)
    st = drv.megabatch(torch.as_tensor(ids, device="cuda"), keep_log=True)
    tr = rep.trace_read()
    sched.close()
    assert len(tr) == st.n_steps == len(st.routes)
    assert [(s, n) for s, n, _, _ in tr] == [(s, n) for _, _, s, n in st.routes]
    assert all(t1 >= t0 for _, _, t0, t1 in tr)
    assert all(tr[i + 1][2] >= tr[i][2] for i in range(len(tr) - 1))
