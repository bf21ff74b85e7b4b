"""C-ABI checks that need no GPU: the library loads, exports every symbol the
header declares, its host-pure functions agree bit-exactly with the oracle,
and device entry points fail cleanly (no crash) without a usable GPU."""
import ctypes as C
import json
import os
import random
import uuid

import numpy as np
import pytest

from paper_conf_ipps_marws22_b200 import _lib, api
from paper_conf_ipps_marws22_b200.build import build
from oracle import merge, metrics, routing, scaling
from tests.conftest import GOLDEN


@pytest.fixture(scope="module", autouse=True)
def _built():
    build()


def test_exports_every_header_symbol():
    syms = _lib.header_symbols()
    assert len(syms) >= 30
    L = _lib.lib()
    missing = [s for s in syms if not hasattr(L, s)]
    assert not missing, missing
    assert set(syms) == set(_lib._SIGS), set(syms) ^ set(_lib._SIGS)
    assert "sm_100a" in api.version()


def test_device_entry_points_fail_cleanly_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    desc = _lib.ModelDesc(100, 10, 64, 0, 8, 100, 10)
    assert _lib.lib().asgd_workspace_bytes(C.byref(desc)) > 0
    h = C.c_void_p()
    buf = (C.c_float * 64)()
    p = C.addressof(buf) + (-C.addressof(buf)) % 16
    rc = _lib.lib().asgd_replica_init(C.byref(h), C.byref(desc), 0, None, p, p, p, p, 1 << 40)
    assert rc in (_lib.E_CUDA, _lib.E_UNSUPPORTED)
    assert _lib.lib().asgd_last_error()
    # argument validation before any device work
    rc = _lib.lib().asgd_replica_init(C.byref(h), C.byref(desc), 0, None, p + 4, p, p, p, 1 << 40)
    assert rc == _lib.E_ARG
    bad = _lib.ModelDesc(100, 10, 96, 0, 8, 100, 10)
    rc = _lib.lib().asgd_replica_init(C.byref(h), C.byref(bad), 0, None, p, p, p, p, 1 << 40)
    assert rc == _lib.E_UNSUPPORTED


def test_timeline_probes_compiled_out_by_default():
    """asgd_timeline_set: the kernel-timeline probes exist only in a -DASGD_TIMELINE build
    (tools/timeline.py); the default library reports ASGD_E_UNSUPPORTED without touching
    the device, for a buffer and for NULL alike."""
    lib = _lib.lib()
    buf = (C.c_uint64 * 60)()
    assert lib.asgd_timeline_set(C.addressof(buf)) == _lib.E_UNSUPPORTED
    assert lib.asgd_timeline_set(None) == _lib.E_UNSUPPORTED
    assert b"ASGD_TIMELINE" in lib.asgd_last_error()


def test_workspace_holds_one_dh_partial_per_label_tile_in_the_stored_z_regime():
    """The K-3 one-pass / softmax-only modes keep up to one dH1 partial per label tile
    (<= 64) in the stored-Z regime (bf16 softmax, H = 256): the workspace of that regime
    grows by those slices, the fp32 path and the fused-CE regime do not."""
    lib = _lib.lib()
    bf = _lib.ModelDesc(5000, 3993, 256, _lib.PREC_BF16, 256, 80000, 3000, _lib.LOSS_SOFTMAX, 0)
    f32 = _lib.ModelDesc(5000, 3993, 256, _lib.PREC_FP32, 256, 80000, 3000, _lib.LOSS_SOFTMAX, 0)
    wb, wf = lib.asgd_workspace_bytes(C.byref(bf)), lib.asgd_workspace_bytes(C.byref(f32))
    assert wb > 0 and wf > 0
    # 63 label tiles x 256 rows x 256 x 4 B of partials at least (G2's split-K is 15 slices)
    assert wb >= 63 * 256 * 256 * 4


def _load(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


@pytest.mark.parametrize("case", _load("alg2_vectors.json")["cases"])
def test_merge_weights_golden_bitexact(case):
    a, r, s, p = api.merge_weights(case["u"], case["b"], case["nu"], 0.1, 0.1)
    ao, ro, so, po = merge.merge_weights(case["u"], case["b"], case["nu"], 0.1, 0.1)
    assert a == ao and p == po == case["perturbed"]
    if p:
        assert (r, s) == (ro, so)


def test_merge_weights_random_bitexact():
    rng = random.Random(5)
    for _ in range(3000):
        n = rng.randint(1, 8)
        u = [rng.randint(0, 6) for _ in range(n)]
        if sum(u) == 0:
            u[0] = 1
        b = [rng.choice([32, 64, 100, 128]) for _ in range(n)]
        nu = [rng.choice([0.01, 0.05, 0.2]) for _ in range(n)]
        renorm = rng.random() < 0.3
        norm = rng.choice(["u", "ub"])
        got = api.merge_weights(u, b, nu, 0.1, 0.1, renorm, norm)
        want = merge.merge_weights(u, b, nu, 0.1, 0.1, renorm, norm)
        assert got[0] == want[0] and got[3] == want[3], (u, b, nu)
        if want[3]:
            assert got[1:3] == want[1:3]


@pytest.mark.parametrize("case", _load("alg1_vectors.json")["cases"])
def test_scale_batches_golden(case):
    b, lr = api.scale_batches(case["u"], case["b"], case["b_min"], case["b_max"], case["beta"], 1.0)
    assert b == case["b_out"]
    bo, lro = scaling.scale_batches(case["u"], case["b"], case["b_min"], case["b_max"], case["beta"], 1.0)
    assert lr == lro


def test_scale_batches_random_bitexact():
    rng = random.Random(6)
    for _ in range(3000):
        n = rng.randint(1, 8)
        u = [rng.randint(0, 30) for _ in range(n)]
        b_max = rng.choice([32, 256, 1024])
        b_min = b_max // 8
        beta = rng.choice([b_min // 2, 3, 7])
        b = [rng.randint(b_min, b_max) for _ in range(n)]
        lr_max = rng.choice([1.0, 0.1, 0.3])
        assert api.scale_batches(u, b, b_min, b_max, beta, lr_max) == \
            tuple(scaling.scale_batches(u, b, b_min, b_max, beta, lr_max))


def test_routing_bitexact():
    g = _load("fig2_routing.json")
    rng = random.Random(7)
    for _ in range(300):
        n = rng.randint(1, 6)
        b = [rng.randint(1, 40) for _ in range(n)]
        M = rng.randint(1, 400)
        row_nnz = np.array([rng.randint(0, 50) for _ in range(M)], dtype=np.int64)
        cf = [rng.choice([1.0, 1.1, 1.2, 1.32]) for _ in range(n)]
        got = api.route_simulate(b, M, cf, 5.0, row_nnz)
        want = routing.simulate(b, M, lambda r, s, l: cf[r] * (float(row_nnz[s:s + l].sum()) + 5.0 * l))
        assert got == want
        order = [rr for rr, _, _ in want]
        assert api.route_replay(order, b, M) == routing.replay(order, b, M)
    # Fig. 2: per-batch costs via one nnz-free row per batch
    b = [1, 1]
    got = api.route_simulate(b, 5, [1.0, 1.5], 1.0, np.zeros(5, dtype=np.int64))
    assert [r for r, _, _ in got] == g["expected_order"]


def test_precision_at_k_matches_oracle():
    rng = np.random.default_rng(8)
    Z = rng.integers(0, 4, size=(40, 9)).astype(np.float64)
    for k in (1, 3, 5):
        top = metrics.topk(Z, k)
        lab_ptr = np.arange(0, 81, 2, dtype=np.int64)
        lab = np.concatenate([np.sort(rng.choice(9, 2, replace=False)) for _ in range(40)]).astype(np.int32)
        hits = api.precision_at_k_hits(top, lab_ptr, lab, k)
        assert hits / (k * 40) == metrics.precision_at_k(top, lab_ptr, lab, k)


def test_scheduler_single_process():
    name = "/asgd_t_" + uuid.uuid4().hex[:8]
    s = api.Scheduler(name, 1, 100, create=True)
    try:
        got = []
        while True:
            t = s.next(0, 32)
            if t is None:
                break
            got.append(t)
        assert got == [(0, 32), (32, 32), (64, 32), (96, 4)]
        assert [(r, st, n) for _, r, st, n in s.log()] == [(0, 0, 32), (0, 32, 32), (0, 64, 32), (0, 96, 4)]
        s.reset(1)
        s.wait(1, 10)
        assert s.next(0, 100) == (0, 100)
        assert s.next(0, 1) is None
    finally:
        s.close()


def test_merge_weights_unknown_flag_rejected():
    import ctypes as C
    import numpy as np
    from paper_conf_ipps_marws22_b200 import _lib
    u = np.array([1, 2], dtype=np.int64)
    b = np.array([32, 32], dtype=np.int64)
    nu = np.array([1.0, 1.0])
    a = np.zeros(2)
    rc = _lib.lib().asgd_merge_weights(2, u.ctypes.data, b.ctypes.data, nu.ctypes.data, 0.1, 0.1, 4,
                                       a.ctypes.data, None, None, None)
    assert rc == 1      # ASGD_E_ARG


def test_hyper_rejects_unknown_method_switches():
    from paper_conf_ipps_marws22_b200 import train
    base = dict(b_max=256, b_min=32, beta=4, lr_max=1.0, M=25600)
    assert train.Hyper(**base, norm="ub", scale_every=3).scale_every == 3
    with pytest.raises(ValueError):
        train.Hyper(**base, norm="b")
    assert train.Hyper(**base, scale_every=0).scale_every == 0      # R17 adaptive frequency
    with pytest.raises(ValueError):
        train.Hyper(**base, scale_every=-1)
    with pytest.raises(ValueError):
        api.merge_weights([1, 2], [32, 32], [1.0, 1.0], norm="uu")


def test_route_replay_rejects_out_of_range_ranks():
    from paper_conf_ipps_marws22_b200 import _lib
    for bad in ([0, 2, 1], [0, -1]):
        with pytest.raises(_lib.AsgdError):
            api.route_replay(bad, [8, 8], 40)


def test_norm_per_param_and_elastic_weights():
    """Alg. 2 line 4's nu (Q16) from squared norms equals the oracle's
    ||w||_2 / |w|; Elastic's alpha_i = 1/N (R10)."""
    from oracle import merge as omerge
    rng = np.random.default_rng(3)
    for _ in range(50):
        n = int(rng.integers(1, 9))
        reps = [rng.normal(0, rng.uniform(0.01, 3.0), int(rng.integers(1, 5000))) for _ in range(n)]
        P = len(reps[0])
        reps = [r[:P] if len(r) >= P else np.resize(r, P) for r in reps]
        sq = [float(np.dot(r, r)) for r in reps]
        assert api.norm_per_param(sq, P) == [omerge.norm_per_param(r) for r in reps]
    from paper_conf_ipps_marws22_b200 import _lib
    with pytest.raises(_lib.AsgdError):
        api.norm_per_param([-1.0], 10)
    for n in range(1, 9):
        assert api.elastic_weights(n) == [1.0 / n] * n


def test_route_static_matches_oracle():
    rng = random.Random(11)
    for _ in range(300):
        n, b, M = rng.randint(1, 8), rng.randint(1, 40), rng.randint(0, 500)
        assert api.route_static(n, b, M) == [tuple(r) for r in routing.static(n, b, M)]


def test_single_replica_weights_ignore_nu():
    """N = 1: Alg. 2 gives alpha = [1] whatever the norm (line 2: b / sum b; lines 4-6: the
    only replica ties with itself, Q17) -- why the N = 1 driver skips the norm and its host
    round trip (train.DistributedAdaptiveSGD)."""
    for u in (1, 7, 100):
        for b in (1, 32, 1024):
            for nu in (float("nan"), 0.0, 1e-6, 0.5, 1e9):
                for renorm in (False, True):
                    for norm in ("u", "ub"):
                        assert api.merge_weights([u], [b], [nu], 0.1, 0.1, renorm, norm) == ([1.0], 0, 0, False)
                        assert merge.merge_weights([u], [b], [nu], 0.1, 0.1, renorm, norm)[0] == [1.0]
