"""The real multi-process driver (DistributedAdaptiveSGD) on one GPU: two ranks
share cuda:0, take tickets from the shm scheduler, merge through
torch.distributed (gloo all-reduce here; NCCL on multi-GPU boxes) or through
the fused peer-memory merge kernel (CUDA IPC between the two processes), and
must end with bitwise-identical global models equal to the oracle replaying
their ticket log."""
import os
import socket
import uuid

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank(rank, world, port, shm, out, precision, n_mb, merge, method="adaptive"):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_marws22_b200 import api, train
    from synth import config, generate, init_params, sample_stream
    cfg = config("tiny")
    data = generate(cfg)
    w0 = init_params(cfg)
    nz, nl = api.max_step_sizes([data], cfg.b_max)
    rep = api.Replica(cfg.F, cfg.L, cfg.H, cfg.b_max, nz, nl, precision, device=0, w0=w0)
    dd = api.DeviceCsr(data, device="cuda:0")
    rep.register(dd)
    h = train.Hyper.from_config(cfg)
    if rank == 0:
        sched = api.Scheduler(shm, world, h.M, create=True)
    dist.barrier()
    if rank != 0:
        sched = api.Scheduler(shm, world, h.M, create=False)
    drv = train.DistributedAdaptiveSGD(rep, h, rank, world, sched, inflight=1, merge=merge, method=method)
    logs, stats = [], []
    for mb in range(n_mb):
        ids = sample_stream(cfg, mb * h.M, h.M)
        st = drv.megabatch(torch.as_tensor(ids, device="cuda:0"), keep_log=True)
        logs.append([r for _, r, _, _ in st.routes])
        stats.append((st.u, st.b, st.lr, st.alpha, st.perturbed))
    torch.cuda.synchronize()
    np.save(os.path.join(out, f"w{rank}.npy"), rep.params.cpu().numpy())   # = w' after every merge
    np.save(os.path.join(out, f"s{rank}.npy"), np.array([logs, stats, drv.merge], dtype=object), allow_pickle=True)
    dist.barrier()
    sched.close()
    dist.destroy_process_group()


def _check_world(tmp_path, world, n_mb, precision, tol, merge):
    ws = [np.load(tmp_path / f"w{r}.npy") for r in range(world)]
    for w in ws[1:]:
        np.testing.assert_array_equal(ws[0], w)    # replicas end bitwise identical (Q20)
    logs, stats, used = np.load(tmp_path / "s0.npy", allow_pickle=True)
    assert used == merge                          # no silent fallback from the fused merge
    for r in range(1, world):
        _, stats_r, _ = np.load(tmp_path / f"s{r}.npy", allow_pickle=True)
        assert [s[:4] for s in stats] == [s[:4] for s in stats_r]
    from oracle import adaptive
    from synth import config, generate, init_params, sample_stream
    cfg = config("tiny")
    data = generate(cfg)
    M = cfg.mega_batch
    recs = adaptive.run(cfg.F, cfg.H, cfg.L, data, init_params(cfg), lambda mb: sample_stream(cfg, mb * M, M),
                        n_rep=world, n_mb=n_mb, M=M, b_max=cfg.b_max, b_min=cfg.b_min, beta=cfg.beta,
                        lr_max=cfg.lr_max, route_logs=list(logs))
    for (u, b, lr, alpha, pert), rec in zip(stats, recs):
        assert list(u) == rec.u and list(b) == rec.b and list(lr) == rec.lr and pert == rec.perturbed
        np.testing.assert_allclose(alpha, rec.alpha, rtol=1e-12)
    ref = recs[-1].w
    assert np.linalg.norm(ws[0] - ref) / np.linalg.norm(ref) <= tol


@pytest.mark.parametrize("merge", ["nccl", "fused"])
@pytest.mark.parametrize("precision,tol", [("fp32", 1e-4), ("bf16", 2e-2)])
def test_two_ranks_one_gpu(tmp_path, precision, tol, merge):
    world, n_mb = 2, 4
    shm = "/asgd_d_" + uuid.uuid4().hex[:8]
    mp.spawn(_rank, args=(world, _port(), shm, str(tmp_path), precision, n_mb, merge), nprocs=world, join=True)
    _check_world(tmp_path, world, n_mb, precision, tol, merge)


@pytest.mark.parametrize("world", [3, 4])
def test_fused_merge_three_and_four_ranks(tmp_path, world):
    """N > 2 ranks on one GPU through the fused peer-memory merge: the parameter
    vector (P = 134,564) splits into uneven shards; every rank reduces its shard
    over CUDA IPC and stores w' into every replica."""
    n_mb = 3
    shm = "/asgd_w_" + uuid.uuid4().hex[:8]
    mp.spawn(_rank, args=(world, _port(), shm, str(tmp_path), "fp32", n_mb, "fused"), nprocs=world, join=True)
    _check_world(tmp_path, world, n_mb, "fp32", 1e-4, "fused")


@pytest.mark.parametrize("precision,tol", [("fp32", 1e-4), ("bf16", 2e-2)])
def test_two_ranks_elastic(tmp_path, precision, tol):
    """Elastic SGD mode (NEXT-2): static equal batches, alpha = 1/N, fused merge."""
    world, n_mb = 2, 3
    shm = "/asgd_e_" + uuid.uuid4().hex[:8]
    mp.spawn(_rank, args=(world, _port(), shm, str(tmp_path), precision, n_mb, "fused", "elastic"), nprocs=world,
             join=True)
    w0, w1 = (np.load(tmp_path / f"w{r}.npy") for r in range(world))
    np.testing.assert_array_equal(w0, w1)
    logs, stats, _ = np.load(tmp_path / "s0.npy", allow_pickle=True)
    from oracle import adaptive
    from synth import config, generate, init_params, sample_stream
    cfg = config("tiny")
    data = generate(cfg)
    M = cfg.mega_batch
    recs = adaptive.run_elastic(cfg.F, cfg.H, cfg.L, data, init_params(cfg), lambda mb: sample_stream(cfg, mb * M, M),
                                n_rep=world, n_mb=n_mb, M=M, b=cfg.b_max, lr=cfg.lr_max)
    for log, (u, b, lr, alpha, pert), rec in zip(logs, stats, recs):
        assert log == [r for r, _, _ in rec.routes]
        assert list(u) == rec.u and list(alpha) == rec.alpha and not pert
    ref = recs[-1].w
    assert np.linalg.norm(w0 - ref) / np.linalg.norm(ref) <= tol
