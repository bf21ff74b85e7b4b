"""Thin Python binding over libasgd's C ABI (argument marshalling only).

Torch provides the device memory and the stream; every step of the method
runs inside libasgd (CUDA kernels for sm_100a, or its host C++ for the
scheduler / Alg. 1 / Alg. 2).  Names follow include/asgd.h.
"""
from __future__ import annotations

import ctypes as C
from typing import List, Optional, Sequence, Tuple

import numpy as np
import torch

from . import _lib
from ._lib import Csr, ModelDesc, call, lib

PRECISIONS = {"fp32": _lib.PREC_FP32, "bf16": _lib.PREC_BF16}
LOSSES = {"softmax": _lib.LOSS_SOFTMAX, "sigmoid": _lib.LOSS_SIGMOID}


def _ptr(t) -> int:
    if t is None:
        return None
    if isinstance(t, torch.Tensor):
        return t.data_ptr()
    if isinstance(t, np.ndarray):
        return t.ctypes.data
    raise TypeError(type(t))


def _np(a, dtype):
    return np.ascontiguousarray(np.asarray(a, dtype=dtype))


# ----------------------------------------------------------------- data
class DeviceCsr:
    """A CSR split (features + labels) resident in device memory."""

    def __init__(self, ds, device="cuda", pin: bool = False):
        dev = torch.device(device)
        mk = (lambda a, dt: torch.from_numpy(_np(a, dt)).pin_memory()) if dev.type == "cpu" and pin \
            else (lambda a, dt: torch.from_numpy(_np(a, dt)).to(dev))
        self.row_ptr = mk(ds.row_ptr, np.int64)
        self.col = mk(ds.col, np.int32)
        self.val = mk(ds.val, np.float32)
        self.lab_ptr = mk(ds.lab_ptr, np.int64)
        self.lab = mk(ds.lab, np.int32)
        self.n_rows = int(len(ds.row_ptr) - 1)
        self.nnz = int(ds.row_ptr[-1])
        self.n_lab = int(ds.lab_ptr[-1])

    @classmethod
    def empty_like(cls, other: "DeviceCsr", device="cuda"):
        obj = cls.__new__(cls)
        for k in ("row_ptr", "col", "val", "lab_ptr", "lab"):
            setattr(obj, k, torch.empty_like(getattr(other, k), device=device))
        obj.n_rows, obj.nnz, obj.n_lab = other.n_rows, other.nnz, other.n_lab
        return obj

    def csr(self) -> Csr:
        return Csr(self.row_ptr.data_ptr(), self.col.data_ptr(), self.val.data_ptr(),
                   self.lab_ptr.data_ptr(), self.lab.data_ptr(), self.n_rows, self.nnz, self.n_lab)


def max_step_sizes(datasets: Sequence, b_max: int) -> Tuple[int, int]:
    """Upper bounds of one step's feature / label nnz: the b_max largest rows."""
    nz = nl = 1
    for ds in datasets:
        rl = np.diff(ds.row_ptr)
        ll = np.diff(ds.lab_ptr)
        k = min(b_max, len(rl))
        nz = max(nz, int(np.sort(rl)[-k:].sum()))
        nl = max(nl, int(np.sort(ll)[-k:].sum()))
    return nz, nl


# ----------------------------------------------------------------- replica
class Replica:
    """One model replica on one GPU (the paper's GPU manager)."""

    def __init__(self, F: int, L: int, H: int, b_max: int, max_step_nnz: int, max_step_labels: int,
                 precision: str = "fp32", device: int = 0, w0=None, stream=None,
                 share_global: Optional["Replica"] = None, loss: str = "softmax"):
        self.F, self.L, self.H, self.b_max = F, L, H, b_max
        self.P = F * H + H + L * H + L
        self.device = torch.device("cuda", device)
        self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
        self.desc = ModelDesc(F, L, H, PRECISIONS[precision], b_max, max_step_nnz, max_step_labels,
                              LOSSES[loss], 0)
        self.precision, self.loss = precision, loss
        ws_bytes = lib().asgd_workspace_bytes(C.byref(self.desc))
        if ws_bytes == 0:
            raise _lib.AsgdError("asgd_workspace_bytes", _lib.E_SHAPE, "bad model desc")
        self.params = torch.empty(self.P, dtype=torch.float32, device=self.device)
        if share_global is None:
            self.w = torch.empty(self.P, dtype=torch.float32, device=self.device)
            self.d = torch.zeros(self.P, dtype=torch.float32, device=self.device)
        else:
            self.w, self.d = share_global.w, share_global.d
        if w0 is not None:
            t = torch.as_tensor(w0, dtype=torch.float32).reshape(-1)
            self.params.copy_(t)
            if share_global is None:
                self.w.copy_(t)
        self.ws = torch.empty(ws_bytes, dtype=torch.uint8, device=self.device)
        torch.cuda.synchronize(self.device)
        h = C.c_void_p()
        call("asgd_replica_init", C.byref(h), C.byref(self.desc), device, self.stream.cuda_stream,
             _ptr(self.params), _ptr(self.w), _ptr(self.d), _ptr(self.ws), ws_bytes)
        self.ctx = h
        self._data = None

    # -- data
    def register(self, data: DeviceCsr):
        self._data = data
        self._csr = data.csr()
        call("asgd_data_register", self.ctx, C.byref(self._csr))

    def upload(self, host: DeviceCsr, dev: DeviceCsr):
        self._data = dev
        self._hcsr, self._csr = host.csr(), dev.csr()
        call("asgd_data_upload", self.ctx, C.byref(self._hcsr), C.byref(self._csr))

    def stage(self, host: DeviceCsr, dev: DeviceCsr, stream: Optional[torch.cuda.Stream] = None):
        """asgd_data_stage: host -> dev copies on `stream` (None: the ctx stream), not registered."""
        h, d = host.csr(), dev.csr()
        call("asgd_data_stage", self.ctx, C.byref(h), C.byref(d), stream.cuda_stream if stream is not None else None)

    def use(self, dev: DeviceCsr, nnz: int, n_lab: int):
        """asgd_data_use: register a staged buffer (the staged split's nnz / n_lab) for the next steps."""
        self._data = dev
        self._csr = dev.csr()
        self._csr.nnz, self._csr.n_lab = int(nnz), int(n_lab)
        call("asgd_data_use", self.ctx, C.byref(self._csr))

    # -- local step
    def step(self, rows: torch.Tensor, lr: float, loss_out: Optional[torch.Tensor] = None):
        assert rows.dtype == torch.int32 and rows.is_cuda
        call("asgd_local_step", self.ctx, _ptr(rows), int(rows.numel()), float(lr),
             _ptr(loss_out) if loss_out is not None else None)

    def run_tickets(self, sched: "Scheduler", rank: int, b: int, stream_rows: torch.Tensor, lr: float,
                    losses: Optional[torch.Tensor] = None, inflight: int = 2) -> int:
        """This rank's share of the mega-batch (asgd_run_tickets): the ticket loop
        in native code; returns the number of local steps enqueued."""
        assert stream_rows.dtype == torch.int32 and stream_rows.is_cuda and stream_rows.is_contiguous()
        n = C.c_int64()
        call("asgd_run_tickets", self.ctx, sched.h, int(rank), int(b), _ptr(stream_rows), float(lr),
             _ptr(losses) if losses is not None else None, int(losses.numel()) if losses is not None else 0,
             int(inflight), C.byref(n))
        return n.value

    def run_static(self, rank: int, world: int, b: int, stream_rows: torch.Tensor, lr: float,
                   losses: Optional[torch.Tensor] = None, inflight: int = 2) -> int:
        """Elastic SGD's static share of the mega-batch (asgd_run_static)."""
        assert stream_rows.dtype == torch.int32 and stream_rows.is_cuda and stream_rows.is_contiguous()
        n = C.c_int64()
        call("asgd_run_static", self.ctx, int(rank), int(world), int(b), _ptr(stream_rows), int(stream_rows.numel()),
             float(lr), _ptr(losses) if losses is not None else None,
             int(losses.numel()) if losses is not None else 0, int(inflight), C.byref(n))
        return n.value

    def trace_enable(self, on: bool = True):
        call("asgd_trace_enable", self.ctx, int(bool(on)))

    def trace_read(self, cap: int = 1 << 16) -> List[Tuple[int, int, int, int]]:
        """(stream start, rows, t0_ns, t1_ns) of each traced step since trace_enable."""
        out = np.zeros(4 * cap, dtype=np.int64)
        n = C.c_int64()
        call("asgd_trace_read", self.ctx, _ptr(out), int(cap), C.byref(n))
        return [tuple(int(x) for x in out[4 * i:4 * i + 4]) for i in range(n.value)]

    def updates(self) -> int:
        u = C.c_int64()
        call("asgd_updates", self.ctx, C.byref(u))
        return u.value

    def set_debug_grads(self, grad: Optional[torch.Tensor]):
        call("asgd_set_debug_grads", self.ctx, _ptr(grad) if grad is not None else None)

    def last_touched(self) -> torch.Tensor:
        out = torch.empty(min(self.F, self.desc.max_step_nnz), dtype=torch.int32, device=self.device)
        n = C.c_int64()
        call("asgd_last_touched", self.ctx, _ptr(out), out.numel(), C.byref(n))
        return out[:n.value]

    # -- merge
    def sqnorm(self, out: torch.Tensor):
        assert out.dtype == torch.float64 and out.is_cuda
        call("asgd_replica_sqnorm", self.ctx, _ptr(out))

    def prescale(self, alpha: float):
        call("asgd_merge_prescale", self.ctx, float(alpha))

    def finish(self, gamma: float):
        call("asgd_merge_finish", self.ctx, float(gamma))

    # -- fused peer-memory merge (asgd_peer_* / asgd_merge_fused)
    def peer_export(self) -> bytes:
        buf = (C.c_char * _lib.PEER_HANDLE_BYTES)()
        call("asgd_peer_export", self.ctx, buf)
        return bytes(buf)

    def peer_open(self, rank: int, handles: Sequence[bytes]):
        blob = b"".join(bytes(h).ljust(_lib.PEER_HANDLE_BYTES, b"\0") for h in handles)
        buf = (C.c_char * len(blob)).from_buffer_copy(blob)
        call("asgd_peer_open", self.ctx, int(rank), len(handles), buf)

    def peer_close(self):
        call("asgd_peer_close", self.ctx)

    def merge_fused(self, alpha: Sequence[float], gamma: float):
        al = (C.c_double * len(alpha))(*[float(a) for a in alpha])
        call("asgd_merge_fused", self.ctx, al, float(gamma))

    def params_changed(self):
        call("asgd_params_changed", self.ctx)

    def weighted_sum(self, replicas: Sequence["Replica"], alpha: Sequence[float], out: torch.Tensor):
        ptrs = torch.tensor([r.params.data_ptr() for r in replicas], dtype=torch.int64, device=self.device)
        al = torch.tensor(list(alpha), dtype=torch.float64, device=self.device)
        call("asgd_replicas_weighted_sum", self.ctx, _ptr(ptrs), _ptr(al), len(replicas), _ptr(out))
        self._keep = (ptrs, al)

    # -- evaluate
    def eval_topk(self, test: DeviceCsr, rows: torch.Tensor, k: int) -> torch.Tensor:
        out = torch.empty(rows.numel() * k, dtype=torch.int32, device=self.device)
        self._tcsr = test.csr()
        call("asgd_eval_topk", self.ctx, C.byref(self._tcsr), _ptr(rows), int(rows.numel()), int(k), _ptr(out))
        return out.view(-1, k)

    def sync(self):
        call("asgd_sync", self.ctx)

    def launches(self) -> int:
        n = C.c_int64()
        call("asgd_kernel_launches", self.ctx, C.byref(n))
        return n.value

    def copy_to_host(self, dst: torch.Tensor, src: torch.Tensor):
        call("asgd_copy_to_host", self.ctx, _ptr(dst), _ptr(src), src.numel() * src.element_size())

    def close(self):
        if getattr(self, "ctx", None):
            lib().asgd_replica_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ----------------------------------------------------------------- host-pure
MERGE_RENORM, MERGE_NORM_UB = 1, 2       # asgd.h flags of asgd_merge_weights


def merge_weights(u, b, nu, pert_thr=0.1, delta=0.1, pert_renorm=False, norm="u"):
    if norm not in ("u", "ub"):
        raise ValueError(f"norm must be 'u' or 'ub', got {norm!r}")
    flags = (MERGE_RENORM if pert_renorm else 0) | (MERGE_NORM_UB if norm == "ub" else 0)
    n = len(u)
    u_, b_, nu_ = _np(u, np.int64), _np(b, np.int64), _np(nu, np.float64)
    alpha = np.zeros(n, dtype=np.float64)
    r, s, p = C.c_int32(), C.c_int32(), C.c_int32()
    call("asgd_merge_weights", n, _ptr(u_), _ptr(b_), _ptr(nu_), float(pert_thr), float(delta),
         flags, _ptr(alpha), C.byref(r), C.byref(s), C.byref(p))
    return alpha.tolist(), r.value, s.value, bool(p.value)


def scale_batches(u, b, b_min, b_max, beta, lr_max):
    n = len(u)
    u_, b_ = _np(u, np.int64), _np(b, np.int64).copy()
    lr = np.zeros(n, dtype=np.float64)
    call("asgd_scale_batches", n, _ptr(u_), _ptr(b_), _ptr(lr), int(b_min), int(b_max), int(beta), float(lr_max))
    return b_.tolist(), lr.tolist()


def norm_per_param(sqnorm, P: int) -> List[float]:
    """Alg. 2 line 4's ||w_i||_2 / |w| from the all-gathered squared norms (Q16)."""
    sq = _np(sqnorm, np.float64)
    nu = np.zeros(len(sq), dtype=np.float64)
    call("asgd_norm_per_param", len(sq), _ptr(sq), int(P), _ptr(nu))
    return nu.tolist()


def elastic_weights(n: int) -> List[float]:
    """Elastic SGD's alpha_i = 1/N (R10)."""
    al = np.zeros(int(n), dtype=np.float64)
    call("asgd_elastic_weights", int(n), _ptr(al))
    return al.tolist()


def route_replay(order, b, M) -> List[Tuple[int, int, int]]:
    o = _np(order, np.int32)
    b_ = _np(b, np.int64)
    out = np.zeros(3 * (len(o) + 1), dtype=np.int64)
    n = C.c_int64()
    call("asgd_route_replay", len(b_), len(o), _ptr(o) if len(o) else None, _ptr(b_), int(M), _ptr(out),
         len(o) + 1, C.byref(n))
    return [tuple(int(x) for x in out[3 * i:3 * i + 3]) for i in range(n.value)]


def scale_frequency(b_before, b_after, last_sign, interval: int, max_interval: int = 8):
    """R17: the next Alg. 1 interval and the updated last move signs."""
    bb, ba = _np(b_before, np.int64), _np(b_after, np.int64)
    sg = _np(last_sign, np.int32).copy()
    out = C.c_int32()
    call("asgd_scale_frequency", len(bb), _ptr(bb), _ptr(ba), _ptr(sg), int(interval), int(max_interval),
         C.byref(out))
    return out.value, sg.tolist()


def route_static(n, b, M) -> List[Tuple[int, int, int]]:
    """Elastic SGD's static routes (R10): batch k of b samples -> rank k mod n."""
    cap = int(M) // max(1, int(b)) + 2
    out = np.zeros(3 * cap, dtype=np.int64)
    k = C.c_int64()
    call("asgd_route_static", int(n), int(b), int(M), _ptr(out), cap, C.byref(k))
    return [tuple(int(x) for x in out[3 * i:3 * i + 3]) for i in range(k.value)]


def route_simulate(b, M, cost_factor, per_row, row_nnz) -> List[Tuple[int, int, int]]:
    b_ = _np(b, np.int64)
    cf = _np(cost_factor, np.float64)
    rn = _np(row_nnz, np.int64)
    cap = int(M) + 1
    out = np.zeros(3 * cap, dtype=np.int64)
    n = C.c_int64()
    call("asgd_route_simulate", len(b_), _ptr(b_), int(M), _ptr(cf), float(per_row), _ptr(rn), _ptr(out), cap, C.byref(n))
    return [tuple(int(x) for x in out[3 * i:3 * i + 3]) for i in range(n.value)]


def precision_at_k_hits(topk: np.ndarray, lab_ptr: np.ndarray, lab: np.ndarray, k: int) -> int:
    t = _np(topk, np.int32)
    lp, lb = _np(lab_ptr, np.int64), _np(lab, np.int32)
    hits = C.c_int64()
    call("asgd_precision_at_k", _ptr(t), _ptr(lp), _ptr(lb), int(t.shape[0]), int(k), C.byref(hits))
    return hits.value


class Scheduler:
    """Cross-process dynamic batch scheduler in POSIX shm."""

    def __init__(self, name: str, n_ranks: int, M: int, create: bool):
        h = C.c_void_p()
        call("asgd_sched_open", name.encode(), int(n_ranks), int(M), int(create), C.byref(h))
        self.h, self.name, self.M, self.creator = h, name, M, create

    def next(self, rank: int, b: int) -> Optional[Tuple[int, int]]:
        s, n = C.c_int64(), C.c_int64()
        rc = lib().asgd_sched_next(self.h, int(rank), int(b), C.byref(s), C.byref(n))
        if rc < 0:
            _lib.check("asgd_sched_next", -rc)
        return (s.value, n.value) if rc == 1 else None

    def log(self) -> List[Tuple[int, int, int, int]]:
        cap = self.M + 1
        out = np.zeros(4 * cap, dtype=np.int64)
        n = C.c_int64()
        call("asgd_sched_log", self.h, _ptr(out), cap, C.byref(n))
        return [tuple(int(x) for x in out[4 * i:4 * i + 4]) for i in range(n.value)]

    def reset(self, mb: int):
        call("asgd_sched_reset", self.h, int(mb))

    def wait(self, mb: int, timeout_ms: int = 60000):
        call("asgd_sched_wait", self.h, int(mb), int(timeout_ms))

    def close(self, unlink: Optional[bool] = None):
        if self.h:
            call("asgd_sched_close", self.h, int(self.creator if unlink is None else unlink))
            self.h = None


def version() -> str:
    return lib().asgd_version().decode()


TIMELINE_KERNELS = ["touched", "spmm", "g1", "softmax", "g2", "dh", "b1", "g3", "scatter", "g1b", "merge", "other",
                    "ph0", "ph1", "ph2", "ph3", "ph4", "ph5", "ph6", "ph7"]


def timeline_set(buf: Optional[torch.Tensor]):
    """asgd_timeline_set: uint64[3 * len(TIMELINE_KERNELS)] device buffer (int64 tensor) or None."""
    call("asgd_timeline_set", _ptr(buf) if buf is not None else None)
