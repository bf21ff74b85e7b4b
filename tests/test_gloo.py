"""The N > 1 host path with world_size 2 on CPU (gloo): cross-process ticket
routing through the shm scheduler, the statistics exchange, Alg. 2 weights
and Alg. 1 computed identically on every rank, and the prescale + all-reduce
SUM merge reproducing the oracle's sum_i alpha_i w_i (not gpu)."""
import os
import socket
import uuid

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, shm, M, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_marws22_b200 import api, train
    from oracle import merge as omerge
    if rank == 0:
        sched = api.Scheduler(shm, world, M, create=True)
    dist.barrier()
    if rank != 0:
        sched = api.Scheduler(shm, world, M, create=False)
    results = {}
    b = [24, 16][rank]
    rng = np.random.default_rng(rank)
    w_global = np.linspace(-1, 1, 1003).astype(np.float32)
    for mb in range(3):
        sched.wait(mb)
        got = []

        def step(k, start, n):
            got.append((start, n))
            # ranks progress at different speeds
            import time
            time.sleep(0.001 * (1 + rank))

        n_steps = train.run_tickets(sched, rank, b, step, inflight=1)
        replica = (w_global + rng.normal(0, 0.01, w_global.shape).astype(np.float32)).astype(np.float32)
        sq = torch.tensor([float(np.dot(replica.astype(np.float64), replica))], dtype=torch.float64)
        us, bs, nu = train.exchange_stats(n_steps, b, sq, replica.size, world)
        log = sched.log() if rank == 0 else None
        if rank == 0:
            sched.reset(mb + 1)
        norm = "ub" if mb == 2 else "u"          # R12 on the last mega-batch
        alpha, r, s, p = api.merge_weights(us, bs, nu, 0.1, 0.1, False, norm)
        # prescale + all-reduce SUM == sum_i alpha_i w_i
        t = torch.from_numpy(replica.astype(np.float64) * alpha[rank])
        dist.all_reduce(t)
        allrep = [torch.zeros(replica.size, dtype=torch.float32) for _ in range(world)]
        dist.all_gather(allrep, torch.from_numpy(replica))
        S_ref, _ = omerge.merge_models([x.numpy() for x in allrep], alpha, w_global, np.zeros_like(w_global), 0.0)
        allsteps = [None] * world
        dist.all_gather_object(allsteps, got)
        results[mb] = dict(us=us, bs=bs, nu=nu, alpha=alpha, pert=p, norm=norm, log=log, steps=allsteps,
                           merge_err=float(np.abs(t.numpy() - S_ref).max()))
    np.save(os.path.join(out_dir, f"r{rank}.npy"), np.array([results], dtype=object), allow_pickle=True)
    dist.barrier()
    sched.close()
    dist.destroy_process_group()


def test_two_ranks_gloo(tmp_path):
    world, M = 2, 200
    shm = "/asgd_g_" + uuid.uuid4().hex[:8]
    mp.spawn(_worker, args=(world, _free_port(), shm, M, str(tmp_path)), nprocs=world, join=True)
    res = [np.load(tmp_path / f"r{r}.npy", allow_pickle=True)[0] for r in range(world)]
    from oracle import merge as omerge, routing as orouting
    for mb in range(3):
        a, b = res[0][mb], res[1][mb]
        # every rank computed the same weights
        assert a["alpha"] == b["alpha"] and a["us"] == b["us"] and a["bs"] == b["bs"]
        steps = a["steps"]
        # the tickets cover the mega-batch exactly once
        ranges = sorted(x for rs in steps for x in rs)
        cur = 0
        for st, n in ranges:
            assert st == cur
            cur += n
        assert cur == M
        assert a["us"] == [len(steps[0]), len(steps[1])]
        # the shm log equals the oracle's replay of its own ticket order
        log = a["log"]
        order = [r for _, r, _, _ in log]
        assert [(r, s, n) for _, r, s, n in log] == orouting.replay(order, a["bs"], M)
        # Alg. 2 on the exchanged statistics equals the oracle
        assert a["nu"] == b["nu"]
        ow = omerge.merge_weights(a["us"], a["bs"], a["nu"], 0.1, 0.1, False, a["norm"])
        assert a["alpha"] == ow[0] and a["pert"] == ow[3]
        assert a["merge_err"] < 1e-12


class _FakeReplica:
    """Stands in for api.Replica in the fused-merge consensus: rank `bad` cannot
    export (or open) its peers."""
    def __init__(self, rank, fail_export, fail_open):
        self.rank, self.fail_export, self.fail_open = rank, fail_export, fail_open
        self.device = torch.device("cpu")
        self.opened = self.closed = False

    def peer_export(self):
        if self.fail_export:
            raise RuntimeError("no IPC")
        return b"h%d" % self.rank

    def peer_open(self, rank, handles):
        if self.fail_open:
            raise RuntimeError("no P2P")
        self.opened = True

    def peer_close(self):
        self.closed = True


def _consensus_worker(rank, world, port, case, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_marws22_b200 import train
    fe = case == "export" and rank == 1
    fo = case == "open" and rank == 1
    rep = _FakeReplica(rank, fe, fo)
    merge, note = train.DistributedAdaptiveSGD._open_peers(rep, rank, world, None)
    np.save(os.path.join(out_dir, f"c{rank}.npy"),
            np.array([dict(merge=merge, note=note, opened=rep.opened, closed=rep.closed)], dtype=object),
            allow_pickle=True)
    dist.destroy_process_group()


@pytest.mark.parametrize("case", ["ok", "export", "open"])
def test_fused_merge_consensus(tmp_path, case):
    """every rank takes the same merge path.  If one rank cannot map
    its peers all ranks fall back to NCCL, and a rank that had opened its
    mappings closes them."""
    world = 2
    mp.spawn(_consensus_worker, args=(world, _free_port(), case, str(tmp_path)), nprocs=world, join=True)
    res = [np.load(tmp_path / f"c{r}.npy", allow_pickle=True)[0] for r in range(world)]
    merges = {r["merge"] for r in res}
    assert len(merges) == 1
    if case == "ok":
        assert merges == {"fused"} and all(r["opened"] and not r["closed"] for r in res)
    else:
        assert merges == {"nccl"} and all(r["note"] for r in res)
        # rank 0 opened (case "open": rank 1 failed after the all-gather) and must close
        assert res[0]["closed"] == res[0]["opened"]
        assert not res[1]["opened"]
