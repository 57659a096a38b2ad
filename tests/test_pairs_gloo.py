"""Multi-process (world_size 2, gloo, CPU) tests of the process-per-GPU peer control plane.

The data path (IPC-mapped peer store) needs GPUs; here the host logic is checked with a
fake runtime adapter: IPC-handle exchange, ordered handoff records, lockstep alternation of
the job between the two ranks, and preempt-to-resume accounting.
"""
import os
import socket
import time

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class FakeOps:
    """Stands in for the runtime: a job at (iter, k) with n subgraphs per iteration."""

    def __init__(self, rank, n=5):
        self.rank, self.n = rank, n
        self.it, self.k = (0, 0) if rank == 0 else (None, None)
        self.log = []

    def request(self):
        self.k += 1  # the job ran one subgraph before the request cut it
        if self.k == self.n:
            self.it, self.k = self.it + 1, 0
        return {"lat_ms": 0.1 + 0.01 * self.rank, "pre_ms": 0.05}

    def wait_out(self):
        cut = {"iter": self.it, "k": self.k, "t_stop_ns": time.monotonic_ns()}
        self.log.append(("out", self.it, self.k))
        self.it = self.k = None
        return cut

    def adopt(self, it, k):
        assert self.it is None
        self.it, self.k = it, k
        self.log.append(("adopt", it, k))

    def resume_ns(self):
        return time.monotonic_ns()  # one host-wide clock, like CLOCK_MONOTONIC in sf_now_ns


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_middleware_wur0hdh21_b200.pairs import PairLink, run_pair_steps
    link = PairLink()
    other = link.exchange_bytes(f"handle-of-{rank}".encode())
    ops = FakeOps(rank)
    S = run_pair_steps(link, ops, steps=6, warmup=2)
    q.put((rank, other, S, ops.log))
    dist.barrier()
    dist.destroy_process_group()


def test_pair_protocol_two_ranks():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(2):
        r, other, S, log = q.get(timeout=120)
        res[r] = (other, S, log)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res[0][0] == b"handle-of-1" and res[1][0] == b"handle-of-0"
    # 8 steps alternate: rank 0 holds at steps 0,2,4,6; rank 1 at 1,3,5,7
    log0, log1 = res[0][2], res[1][2]
    assert [e[0] for e in log0] == ["out", "adopt"] * 4
    assert [e[0] for e in log1] == ["adopt", "out"] * 4
    # every adopt sees exactly the cut the partner sent out
    outs = [e for e in log0 if e[0] == "out"] + [e for e in log1 if e[0] == "out"]
    adopts = [e for e in log0 if e[0] == "adopt"] + [e for e in log1 if e[0] == "adopt"]
    assert sorted((i, k) for _, i, k in outs) == sorted((i, k) for _, i, k in adopts)
    # the job advanced one subgraph per step, never duplicated or lost
    cuts = sorted((i, k) for _, i, k in outs)
    assert cuts == [(0, j) for j in range(1, 5)] + [(1, j) for j in range(0, 4)]
    S0, S1 = res[0][1], res[1][1]
    assert len(S0["lat"]) == 3 and len(S1["lat"]) == 3  # timed holder steps
    assert len(S0["p2r"]) == 3 and len(S1["p2r"]) == 3
    assert all(x > 0 for x in S0["p2r"] + S1["p2r"])


def test_partner_of():
    from paper_conf_middleware_wur0hdh21_b200.pairs import partner_of
    assert [partner_of(r, 8) for r in range(8)] == [1, 0, 3, 2, 5, 4, 7, 6]
    assert partner_of(2, 3) is None


class FakePoissonOps:
    """The open-loop chase protocol against a fake runtime: a job advances one subgraph per
    1 ms while it runs here; a request submitted while it runs preempts it (it migrates out
    after a 0.5 ms copy); requests complete after 0.2 ms."""

    def __init__(self, rank, log):
        self.rank, self.log = rank, log
        self.job = None  # [iter, k, t_state_change, state]
        self.reqs = {}
        self.nreq = 0
        self.adopts = 0

    def _advance(self):
        if self.job and self.job[3] == "running":
            t = time.monotonic()
            steps = int((t - self.job[2]) / 1e-3)
            for _ in range(steps):
                self.job[1] += 1
                if self.job[1] == 5:
                    self.job[0], self.job[1] = self.job[0] + 1, 0
            self.job[2] += steps * 1e-3

    def start(self):
        self.job = [0, 0, time.monotonic(), "running"]

    def has_job(self):
        self._advance()
        return self.job is not None and self.job[3] == "running"

    def in_transit(self):
        return self.job is not None and self.job[3] == "migrating"

    def job_gone(self):
        return self.job is None

    def migrated_out(self):
        if self.job and self.job[3] == "migrating" and time.monotonic() >= self.job[2]:
            it, k = self.job[0], self.job[1]
            self.job = None
            self.log.append(("out", it, k))
            return {"iter": it, "k": k, "t_stop_ns": time.monotonic_ns()}
        return None

    def adopt(self, it, k):
        assert self.job is None
        self.job = [it, k, time.monotonic(), "running"]
        self.log.append(("adopt", it, k))

    def resume_ns(self):
        return time.monotonic_ns() if self.job else 0

    def submit(self, arrival_ns):
        self.nreq += 1
        preempted = self.has_job()
        if preempted:
            self.job[3] = "migrating"
            self.job[2] = time.monotonic() + 0.5e-3
        self.reqs[self.nreq] = (arrival_ns, time.monotonic() + 0.2e-3, preempted)
        self.log.append(("req", arrival_ns, preempted))
        return self.nreq

    def poll(self, r):
        a, done, pre = self.reqs[r]
        if time.monotonic() < done:
            return None
        return {"arrival_ns": a, "start_ns": a + 1000, "end_ns": time.monotonic_ns(),
                "preempted_job": 0 if pre else -1}

    def stop(self):
        if self.job:
            self.log.append(("stop", self.job[0], self.job[1]))


def _poisson_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import numpy as np
    from paper_conf_middleware_wur0hdh21_b200.pairs import ShmLink, finish_pair, run_pair_poisson, shm_path
    path = shm_path(rank // 2)
    if rank % 2 == 0:
        shm = ShmLink(path, create=True)
    dist.barrier()
    if rank % 2:
        shm = ShmLink(path, create=False)
    log = []
    ops = FakePoissonOps(rank, log)
    if rank % 2 == 0:
        shm.set(ShmLink.HOLDER, rank)
        ops.start()
    t0 = [time.monotonic_ns() + 20_000_000]
    dist.broadcast_object_list(t0, src=0)
    rng = np.random.default_rng(7)
    arr = (t0[0] + np.cumsum(rng.exponential(1 / 400, 60) * 1e9).astype(np.int64)).tolist()
    S = run_pair_poisson(shm, ops, rank, rank ^ 1, arr, time.monotonic_ns, warmup=5)
    finish_pair(shm, ops, rank, S["seen"])
    dist.barrier()
    shm.close(unlink=rank % 2 == 0)
    q.put((rank, S, log))
    dist.destroy_process_group()


def test_pair_poisson_chase_protocol_two_ranks():
    """Open-loop chase (C4 at N > 1): each of the 60 arrivals is served by exactly one rank;
    a request preempts only a job that runs on its rank; every migration out is adopted by the
    partner at the same cut; the job ends on exactly one rank."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_poisson_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(2):
        r, S, log = q.get(timeout=120)
        res[r] = (S, log)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    reqs = [e for r in (0, 1) for e in res[r][1] if e[0] == "req"]
    assert len(reqs) == 60 and len({e[1] for e in reqs}) == 60  # every arrival served once
    outs = sorted(e[1:] for r in (0, 1) for e in res[r][1] if e[0] == "out")
    adopts = sorted(e[1:] for r in (0, 1) for e in res[r][1] if e[0] == "adopt")
    assert outs == adopts and len(outs) >= 3  # every cut adopted by the partner
    assert sum(e[2] for e in reqs) == len(outs)  # a preempting request = one migration
    assert sum(e[2] for e in reqs) >= 10  # the stream keeps finding the job (chase)
    stops = [e for r in (0, 1) for e in res[r][1] if e[0] == "stop"]
    assert len(stops) == 1  # the job ends on exactly one rank
    assert len(res[0][0]["lat"]) + len(res[1][0]["lat"]) == 55  # after the 5 warm-up requests
