"""Parity of the merge kernels and of the whole method on simulated replicas
(CUDA path vs oracle), plus top-k evaluation."""
import numpy as np
import pytest
import torch

from oracle import adaptive, merge as omerge, metrics, model as omodel
from synth import config, init_params, sample_stream
from tests.gpu_helpers import dataset, make_replica, normwise

pytestmark = pytest.mark.gpu


def test_sqnorm_prescale_finish():
    cfg = config("tiny")
    data = dataset("tiny")
    rng = np.random.default_rng(0)
    w0 = init_params(cfg)
    rep = make_replica(cfg, data, "fp32", w0=w0)
    x = (w0 + rng.normal(0, 0.01, w0.shape)).astype(np.float32)
    d0 = rng.normal(0, 0.01, w0.shape).astype(np.float32)
    rep.params.copy_(torch.from_numpy(x))
    rep.d.copy_(torch.from_numpy(d0))
    sq = torch.zeros(1, dtype=torch.float64, device="cuda")
    rep.sqnorm(sq)
    rep.sync()
    ref = float(np.dot(x.astype(np.float64), x.astype(np.float64)))
    assert abs(sq.item() - ref) <= 1e-12 * ref
    rep.prescale(0.37)
    rep.finish(0.9)
    rep.sync()
    wn, dn = omerge.merge_models([x], [0.37], w0, d0, 0.9)
    assert normwise(rep.params.cpu().numpy(), wn) <= 1e-6
    assert normwise(rep.w.cpu().numpy(), wn) <= 1e-6
    assert normwise(rep.d.cpu().numpy(), dn) <= 1e-5
    assert rep.updates() == 0


@pytest.mark.parametrize("precision,tol,norm,scale_every", [
    ("fp32", 1e-4, "u", 1), ("bf16", 2e-2, "u", 1),
    ("fp32", 1e-4, "ub", 2),         # R12 u_i b_i weights, R13 Alg. 1 every 2nd mega-batch
    ("bf16", 2e-2, "u", 0)])         # R17 adaptive Alg. 1 frequency
def test_simulated_two_replicas_tiny_trajectory(precision, tol, norm, scale_every):
    """BASELINE.json configs[0]: 2 simulated replicas, ~50 steps, free-running."""
    from paper_conf_ipps_marws22_b200 import api, train
    cfg = config("tiny")
    data = dataset("tiny")
    w0 = init_params(cfg)
    h = train.Hyper.from_config(cfg, norm=norm, scale_every=scale_every)
    r0 = make_replica(cfg, data, precision, w0=w0)
    r1 = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, r0.desc.max_step_nnz, r0.desc.max_step_labels,
                     precision, w0=w0, share_global=r0)
    r1.register(r0._keep_data)
    lens = np.diff(data.row_ptr)
    cf = [1.0, 1.32]
    sim = train.SimulatedAdaptiveSGD([r0, r1], h, lens, cf)
    n_mb = 5
    stats = []
    for mb in range(n_mb):
        ids = sample_stream(cfg, mb * h.M, h.M)
        stats.append(sim.megabatch(torch.as_tensor(ids, device="cuda"), ids))
    recs = adaptive.run(cfg.F, cfg.H, cfg.L, data, w0, lambda mb: sample_stream(cfg, mb * h.M, h.M),
                        n_rep=2, n_mb=n_mb, M=h.M, b_max=h.b_max, b_min=h.b_min, beta=h.beta,
                        lr_max=h.lr_max, cost_factors=cf, norm=norm, scale_every=scale_every)
    for st, rec in zip(stats, recs):
        assert [tuple(x) for x in st.routes] == [tuple(x) for x in rec.routes]   # bit-exact
        assert st.u == rec.u and st.b == rec.b and st.lr == rec.lr
        assert st.perturbed == rec.perturbed
        np.testing.assert_allclose(st.alpha, rec.alpha, rtol=1e-12)
    assert normwise(r0.w.cpu().numpy(), recs[-1].w) <= tol
    assert sum(s.n_steps for s in stats) >= 45


def test_eval_topk_matches_oracle():
    cfg = config("tiny")
    data = dataset("tiny")
    test = dataset("tiny", None, "test")
    from paper_conf_ipps_marws22_b200 import api
    rep = make_replica(cfg, data, "fp32", extra=(test,))
    td = api.DeviceCsr(test)
    rows = np.arange(300, dtype=np.int32)
    top = rep.eval_topk(td, torch.as_tensor(rows, device="cuda"), 5).cpu().numpy()
    _, _, Z = omodel.forward(init_params(cfg).astype(np.float64), test.row_slice(rows), cfg.F, cfg.H, cfg.L)
    ref = metrics.topk(Z, 5)
    # exact where the ranking is not within fp32 rounding of a tie
    srt = -np.sort(-Z, axis=1)
    clear = (srt[:, :5] - srt[:, 1:6]).min(axis=1) > 1e-5
    assert clear.sum() > 250
    np.testing.assert_array_equal(top[clear], ref[clear])
    sub = test.row_slice(rows)
    assert api.precision_at_k_hits(top[clear], *_lab(sub, clear), 5) == \
        round(metrics.precision_at_k(ref[clear], *_lab(sub, clear), 5) * 5 * clear.sum())


def _lab(sub, mask):
    idx = np.nonzero(mask)[0]
    s2 = sub.row_slice(idx)
    return s2.lab_ptr, s2.lab


def _bf16(x):
    """Round-to-nearest-even to bf16 of fp32(x) (the kernels' __float2bfloat16_rn),
    returned as fp64, and per element the bf16 ulp where fp32(x) lies within 64
    fp32 ulps of a rounding midpoint (0 elsewhere): there the GPU's fp32 H1
    (~1e-6 relative, i.e. ~8 fp32 ulps, off the fp64 one) may round the other
    way, by one bf16 ulp."""
    f = np.asarray(x, dtype=np.float32).copy()
    u = f.view(np.uint32)
    low = (u & 0xFFFF).astype(np.int64)
    near = np.abs(low - 0x8000) < 64
    u += 0x7FFF + ((u >> 16) & 1)
    u &= 0xFFFF0000
    q = f.astype(np.float64)
    ulp = np.abs(q) * 2.0 ** -7
    return q, np.where(near, ulp, 0.0)


@pytest.mark.parametrize("precision", ["bf16", "fp32"])
@pytest.mark.parametrize("name", ["eurlex4k", "amazoncat13k"])
def test_eval_topk_planted_state(name, precision):
    """asgd_eval_topk on the bf16 path (H1 and the W2 shadow rounded to bf16, fp32
    accumulation) -- the path bench.py's time_to_p1 evaluates with -- and on the
    fp32 path, from the trained-like planted state (peaked, structured logits).

    The top-k is an integer decided by floating point, so both sides decide it in
    the kernel's precision: for bf16 the reference logits are formed from the same
    bf16-rounded operands (exact products, fp64 sums), which leaves the fp32
    accumulation order: |Z^ - Zq| <= 300 * 2^-24 * sum_h |Hq_nh| |Wq_jh| + 2^-23 |b2_j|
    (fp32 path: 600 * 2^-24 to cover the fp32 SpMM's H1 as well).  Rows whose
    consecutive top-(k+1) gaps all exceed twice the row's largest bound (bf16:
    plus one bf16 ulp of every H1 element near a rounding midpoint, times |Wq_j|)
    must match the oracle's top-k exactly (ids and order); every row must return
    a valid top-k: each returned id's reference logit is within that bound of the
    reference logit of the same rank."""
    from paper_conf_ipps_marws22_b200 import api
    from synth import planted_params
    cfg = config(name)
    data = dataset(name, 4096)
    test = dataset(name, 2048, "test")
    w0 = planted_params(cfg)
    rep = make_replica(cfg, data, precision, w0=w0, extra=(test,))
    td = api.DeviceCsr(test)
    k = 5
    rows = np.arange(min(1024, test.n_rows), dtype=np.int32)
    top = rep.eval_topk(td, torch.as_tensor(rows, device="cuda"), k).cpu().numpy()
    sub = test.row_slice(rows)
    w = w0.astype(np.float64)
    A1, H1, _ = omodel.forward(w, sub, cfg.F, cfg.H, cfg.L)
    W1, b1, W2, b2 = omodel.split_params(w, cfg.F, cfg.H, cfg.L)
    if precision == "bf16":
        Hq, flip = _bf16(H1)
        Wq, _ = _bf16(W2)
        e = 300 * 2.0 ** -24
    else:
        Hq, Wq, e = H1, W2, 600 * 2.0 ** -24
        flip = np.zeros_like(H1)
    Z = Hq @ Wq.T + b2[None, :]
    E = e * (np.abs(Hq) @ np.abs(Wq).T) + 2.0 ** -23 * np.abs(b2)[None, :] + flip @ np.abs(Wq).T
    bound = 2.0 * E.max(axis=1)
    ref = metrics.topk(Z, k)
    srt = -np.sort(-Z, axis=1)[:, :k + 1]
    clear = (srt[:, :k] - srt[:, 1:k + 1]).min(axis=1) > bound
    assert clear.mean() >= 0.8, clear.mean()
    np.testing.assert_array_equal(top[clear], ref[clear])
    got = np.take_along_axis(Z, top.astype(np.int64), axis=1)
    assert np.all(np.abs(got - srt[:, :k]) <= bound[:, None])
    assert len(set(map(tuple, top.tolist()))) > 1
    # P@k over all rows: the library's count equals the brute-force count of the same ids
    assert api.precision_at_k_hits(top, sub.lab_ptr, sub.lab, k) == \
        round(metrics.precision_at_k(top, sub.lab_ptr, sub.lab, k) * k * len(rows))
