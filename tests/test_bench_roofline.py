"""bench.py's roofline bookkeeping (no GPU): the algorithmic bytes and flops per
kernel class, the choice of the binding resource, and the L2 view."""
import importlib.util
import os

import pytest

from synth import config

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench():
    spec = importlib.util.spec_from_file_location("bench", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


PEAKS = {"hbm_gbs": 6453.4, "bf16_tflops": 1677.6, "bf16_tflops_sustained": 1419.3, "sm_max_mhz": 1965.0}


def _st(cfg, B, nnz, U, nlab):
    return {"B": float(B), "nnz": float(nnz), "U": float(U), "nlab": float(nlab), "splitk": 0}


def test_gemm_classes_count_2BHL_flops():
    b = _bench()
    cfg = config("amazon670k")
    st = _st(cfg, 1024, 77800, 22300, 5120)
    for cls in ("g1", "g2", "g3"):
        by, fl = b.kernel_work(cls, cfg, True, st)
        assert fl == 2.0 * 1024 * cfg.H * cfg.L
        assert by > 0


def test_g3_bytes_follow_survey_8d():
    # W2 / b2 read + written (fp32) and the H1 operand are algorithmic;
    # dZ (logits traffic) and the bf16 shadow refresh are implementation bytes
    b = _bench()
    cfg = config("amazon670k")
    B, H, L = 1024, cfg.H, cfg.L
    by, fl = b.kernel_work("g3", cfg, True, _st(cfg, B, 0, 0, 0))
    assert by == 8 * H * L + 8 * L + 2 * B * H
    # round 1's ncu capture measured 3.095e9 dram bytes per launch: the dZ^T read (1.37 GB)
    # and the shadow write (0.34 GB) on top of the 1.37 GB W2 read-modify-write
    assert 3.095e9 - by > 1.5e9
    # at the sustained tensor peak the GEMM (351 GFLOP) takes longer than its bytes: tensor-bound
    assert fl / (PEAKS["bf16_tflops_sustained"] * 1e12) > by / (PEAKS["hbm_gbs"] * 1e9)


def test_binding_resource():
    b = _bench()
    a670 = config("amazon670k")
    st = _st(a670, 1024, 77800, 22300, 5120)
    # G3's algorithmic 1.37 GB vs 351 GFLOP: tensor-bound on B200 (0.25 ms vs 0.21 ms)
    assert b.roofline_of("g3", a670, True, st, "softmax", 1e-3, PEAKS)["bound"] == "tensor"
    # whichever of bytes / HBM peak and flops / tensor peak is larger binds: the fused
    # softmax GEMM (G1b: W2 shadow read, dZ written) sits right at the ridge
    for cls in ("softmax", "g1", "g2"):
        by, fl = b.kernel_work(cls, a670, True, st)
        want = "hbm" if by / (PEAKS["hbm_gbs"] * 1e9) >= fl / (PEAKS["bf16_tflops_sustained"] * 1e12) else "tensor"
        assert b.roofline_of(cls, a670, True, st, "softmax", 1e-3, PEAKS)["bound"] == want
    # G1 (stats only: W2 shadow read, 351 GFLOP) is tensor-bound
    assert b.roofline_of("g1", a670, True, st, "softmax", 1e-3, PEAKS)["bound"] == "tensor"
    # the fp32 path's GEMMs (bf16x3: three bf16 MMAs per product) report against a third
    # of the bf16 tensor peak
    r = b.roofline_of("g1", a670, False, st, "softmax", 1e-3, PEAKS)
    assert r["bound"] == "tensor" and r["peak"] == pytest.approx(PEAKS["bf16_tflops_sustained"] / 3)
    eur = config("eurlex4k")
    # sparse kernels are byte-bound
    assert b.roofline_of("spmm", eur, True, _st(eur, 256, 60000, 4900, 1360), "softmax", 1e-5, PEAKS)["bound"] == "hbm"


def test_achieved_is_work_over_time():
    b = _bench()
    eur = config("eurlex4k")
    st = _st(eur, 256, 60000, 4900, 1360)
    by, _ = b.kernel_work("spmm", eur, True, st)
    r = b.roofline_of("spmm", eur, True, st, "softmax", 20e-6, PEAKS)
    assert r["achieved"] == pytest.approx(by / 20e-6 / 1e9)
    assert r["work_per_launch"] == by


def test_l2_view_counts_the_w1_gathers():
    b = _bench()
    eur = config("eurlex4k")
    st = _st(eur, 256, 60000, 4900, 1360)
    v = b.l2_view("spmm", eur, True, st, 20e-6)
    assert v is not None and v["bytes_per_launch"] == 4.0 * 60000 * eur.H + 8.0 * 60000 + 6.0 * 256 * eur.H
    assert b.l2_view("g1", eur, True, st, 20e-6) is None


def test_step_ideal_is_max_of_bytes_and_flops():
    b = _bench()
    a670 = config("amazon670k")
    t = b.step_ideal_s(a670, 1024, 77800, 22300, 5120, PEAKS["hbm_gbs"], PEAKS["bf16_tflops_sustained"])
    fl = 6.0 * 1024 * a670.H * a670.L + 4.0 * 77800 * a670.H
    assert t >= fl / (PEAKS["bf16_tflops_sustained"] * 1e12) * 0.999
