"""Control plane of process-per-GPU peer migration (torch.distributed plumbing only).

Ranks are paired (2i, 2i+1) (SURVEY.md reading Q6: fixed pairs).  Each pair:
  1. exchanges its arenas' CUDA IPC handles once (``exchange_bytes``), so each process maps
     the partner's arena into a REMOTE slot (sf_import_arena);
  2. passes a handoff record {iter, k, t_stop_ns, seq} when a job migrated across: the
     source process's runtime has already peer-stored the live set into the partner's arena
     over NVLink and waited for the copy (sf_* data path); the partner then calls
     sf_adopt_job(iter, k).
Messages go over a gloo group (CPU tensors), independent of any NCCL data-path group — the
path itself has no collective.
"""
from __future__ import annotations

import mmap
import os
import struct
import time
from typing import List, Optional

import torch
import torch.distributed as dist

HANDOFF_FIELDS = ("iter", "k", "t_stop_ns", "seq")


def partner_of(rank: int, world: int) -> Optional[int]:
    p = rank ^ 1
    return p if p < world else None


class PairLink:
    def __init__(self, group=None):
        self.rank = dist.get_rank()
        self.world = dist.get_world_size()
        self.group = group
        self.partner = partner_of(self.rank, self.world)
        self.sent = 0
        self.received = 0

    @property
    def starts_holding(self) -> bool:
        """The even rank of a pair starts with the training job."""
        return self.rank % 2 == 0

    def exchange_bytes(self, blob: bytes) -> Optional[bytes]:
        objs = [None] * self.world
        dist.all_gather_object(objs, blob, group=self.group)
        return objs[self.partner] if self.partner is not None else None

    def send_handoff(self, it: int, k: int, t_stop_ns: int) -> None:
        self.sent += 1
        t = torch.tensor([it, k, t_stop_ns, self.sent], dtype=torch.int64)
        dist.send(t, self.partner, group=self.group)

    def recv_handoff(self) -> dict:
        t = torch.empty(len(HANDOFF_FIELDS), dtype=torch.int64)
        dist.recv(t, self.partner, group=self.group)
        self.received += 1
        rec = dict(zip(HANDOFF_FIELDS, (int(v) for v in t.tolist())))
        if rec["seq"] != self.received:
            raise RuntimeError(f"handoff out of order: got seq {rec['seq']}, expected {self.received}")
        return rec


def run_pair_steps(link: PairLink, ops, steps: int, warmup: int,
                   holding: Optional[bool] = None) -> dict:
    """Lockstep ping-pong of one training job inside a pair, one preemption per step.

    The holder serves one batch-1 request (which preempts its job to the partner: the
    request 'chases' the job) and sends the handoff; the other rank
    adopts the job and records preempt-to-resume against the source's stop time (both
    CLOCK_MONOTONIC on one host).  ``ops`` adapts the runtime:
      request() -> {"lat_ms", "pre_ms"}; wait_out() -> {"iter", "k", "t_stop_ns", ...};
      adopt(iter, k) -> None; resume_ns() -> int.
    """
    holding = link.starts_holding if holding is None else holding
    S = {"lat": [], "pre": [], "p2r": [], "cuts": [], "out": []}
    for s in range(warmup + steps):
        timed = s >= warmup
        if holding:
            r = ops.request()
            cut = ops.wait_out()
            link.send_handoff(cut["iter"], cut["k"], cut["t_stop_ns"])
            if timed:
                S["lat"].append(r["lat_ms"])
                S["pre"].append(r["pre_ms"])
                S["out"].append(cut)
        else:
            rec = link.recv_handoff()
            ops.adopt(rec["iter"], rec["k"])
            t = ops.resume_ns()
            if timed:
                S["p2r"].append((t - rec["t_stop_ns"]) * 1e-6)
                S["cuts"].append((rec["iter"], rec["k"]))
        holding = not holding
    S["holding_at_end"] = holding
    return S


class RuntimeOps:
    """Adapter of run_pair_steps onto a Runtime whose slot ``local`` is this process's GPU and
    slot ``remote`` maps the partner's arena (auto-preemption target)."""

    def __init__(self, rt, gh, ghi, local: int, remote: int, x_ptrs, out_ptrs, sub_ms: float,
                 rng, iters: int = 1 << 40, timeout_s: float = 60.0):
        self.rt, self.gh, self.ghi = rt, gh, ghi
        self.local, self.remote = local, remote
        self.x_ptrs, self.out_ptrs = x_ptrs, out_ptrs
        self.sub_ms, self.rng, self.iters, self.timeout = sub_ms, rng, iters, timeout_s
        self.job = None
        self.n = 0

    def start(self) -> None:
        self.job = self.rt.start_training(self.gh, self.local, self.iters, self.remote)

    def _poll(self, pred, what):
        import time
        t0 = time.perf_counter()
        while True:
            info = self.rt.job_info(self.job)
            if pred(info):
                return info
            if info["state_name"] == "failed" or time.perf_counter() - t0 > self.timeout:
                raise RuntimeError(f"{what}: {info}")

    def request(self) -> dict:
        import time
        i0 = self._poll(lambda i: i["state_name"] == "running", "job not running")
        # the job holds the device once its launch cursor moved (a request arriving before
        # that finds the device free and preempts nothing)
        key0 = (i0["iter"], i0["k"])
        self._poll(lambda i: i["state_name"] == "running" and (i["iter"], i["k"]) != key0,
                   "job not advancing")
        t_arr = time.perf_counter() + self.rng.uniform(0.2, 1.0) * self.sub_ms * 2e-3
        while time.perf_counter() < t_arr:
            pass
        i = self.n % len(self.x_ptrs)
        self.n += 1
        req = self.rt.submit(self.ghi, self.local, self.x_ptrs[i], self.out_ptrs[i])
        tm = self.rt.wait(req, self.timeout)
        return {"lat_ms": (tm["end_ns"] - tm["arrival_ns"]) * 1e-6,
                "pre_ms": (tm["start_ns"] - tm["arrival_ns"]) * 1e-6}

    def wait_out(self) -> dict:
        info = self._poll(lambda i: i["state_name"] == "migrated_out", "no migration")
        return {"iter": info["iter"], "k": info["k"], "t_stop_ns": info["last_stop_ns"],
                "xfer_us": info["last_xfer_us"], "bytes": info["migrated_bytes"]}

    def adopt(self, it: int, k: int) -> None:
        self.job = self.rt.adopt_job(self.gh, self.local, self.iters, it, k, self.remote)

    def resume_ns(self) -> int:
        return self._poll(lambda i: i["last_resume_ns"] > 0, "no resume")["last_resume_ns"]


# ---- open-loop Poisson chase inside a pair (C4 at N > 1) -------------------
class ShmLink:
    """Same-host coordination of one pair through a 4 KB shared mapping (/dev/shm): the holder
    word (the rank that runs the job or is receiving it) and the handoff record {seq, iter, k,
    t_stop_ns}.  Microsecond latency where a gloo message costs ~ms; the record's fields are
    written before its sequence number (x86 TSO keeps the order for the reader)."""
    HOLDER, SEQ, ITER, K, TSTOP = range(5)
    OWNERS, RING = 64, 256  # routing decisions of arrivals i: word OWNERS + i % RING

    def __init__(self, path: str, create: bool):
        self.path = path
        if create:
            with open(path, "wb") as f:
                f.write(b"\0" * 4096)
        self.f = open(path, "r+b")
        self.m = mmap.mmap(self.f.fileno(), 4096)

    def get(self, i: int) -> int:
        return struct.unpack_from("<q", self.m, 8 * i)[0]

    def set(self, i: int, v: int) -> None:
        struct.pack_into("<q", self.m, 8 * i, int(v))

    def send_handoff(self, it: int, k: int, t_stop_ns: int) -> int:
        seq = self.get(self.SEQ) + 1
        self.set(self.ITER, it)
        self.set(self.K, k)
        self.set(self.TSTOP, t_stop_ns)
        self.set(self.SEQ, seq)
        return seq

    def decide(self, i: int, owner: int) -> None:
        """The even rank routes arrival i (single writer: an arrival is never served twice)."""
        self.set(self.OWNERS + i % self.RING, ((i + 1) << 1) | (owner & 1))

    def owner_of(self, i: int) -> Optional[int]:
        v = self.get(self.OWNERS + i % self.RING)
        return v & 1 if (v >> 1) == i + 1 else None

    def close(self, unlink: bool = False) -> None:
        self.m.close()
        self.f.close()
        if unlink:
            try:
                os.unlink(self.path)
            except OSError:
                pass


def shm_path(pair: int) -> str:
    return f"/dev/shm/sf_pair_{os.environ.get('MASTER_PORT', '0')}_{pair}"


def run_pair_poisson(shm: ShmLink, ops, me: int, partner: int, arrivals_ns: List[int],
                     now_ns, warmup: int = 0) -> dict:
    """Open-loop Poisson stream of one pair, chasing the job (SURVEY.md 8(d) C4 at N > 1).

    Both ranks walk the same seeded arrival list; the even rank routes each arrival to the
    holder (single writer).  The holder submits the request at its scheduled arrival; if the
    job runs there, the request preempts it and the job migrates to the partner; the holder
    flips when the migrated-out record is published.  A request that arrives while the job is
    in transit runs where it was routed, without a cut.  The rank whose job migrated
    out publishes the handoff; the partner adopts it.  ``ops``: submit(arrival_ns) -> req,
    poll(req) -> timing | None, has_job(), migrated_out() -> cut | None, adopt(iter, k),
    resume_ns().  Returns latency samples of the requests this rank served (after warmup)."""
    S = {"lat": [], "pre": [], "p2r": [], "cuts": [], "out": [], "n_submitted": 0}
    seen = 0  # a fresh link: every record (even one written before this rank got here) is new
    pending = []  # (index, req)
    i, n = 0, len(arrivals_ns)
    pending_resume = None
    while i < n or pending:
        t = now_ns()
        cut = ops.migrated_out()
        if cut is not None:
            # the job left (a request here preempted it, possibly one queued before the job
            # arrived): requests now go to the partner; our own record is not ours to adopt
            shm.set(ShmLink.HOLDER, partner)
            seen = shm.send_handoff(cut["iter"], cut["k"], cut["t_stop_ns"])
            S["out"].append(cut)
        seq = shm.get(ShmLink.SEQ)
        if seq > seen and ops.job_gone():  # the partner's record: the job is ours now
            seen = seq
            rec = (shm.get(ShmLink.ITER), shm.get(ShmLink.K), shm.get(ShmLink.TSTOP))
            ops.adopt(rec[0], rec[1])
            pending_resume = rec
        if pending_resume is not None:
            r = ops.resume_ns()
            if r:
                S["p2r"].append((r - pending_resume[2]) * 1e-6)
                S["cuts"].append(pending_resume[:2])
                pending_resume = None
        if i < n and t >= arrivals_ns[i]:
            # the even rank routes each arrival to the rank holding (or receiving) the job; the
            # odd rank follows its decision
            if me % 2 == 0:
                shm.decide(i, shm.get(ShmLink.HOLDER))
            owner = shm.owner_of(i)
            if owner is not None:
                if owner == me % 2:
                    # the holder flips only when the job has actually left (its record is
                    # published): a request that ran in a gap between two of the job's
                    # subgraphs preempts nothing, and the job stays here
                    pending.append((i, ops.submit(arrivals_ns[i])))
                    S["n_submitted"] += 1
                i += 1
        still = []
        for (k, req) in pending:
            tm = ops.poll(req)
            if tm is None:
                if now_ns() - arrivals_ns[k] > 20_000_000_000:
                    raise RuntimeError(f"rank {me}: request {k} pending for 20 s; job "
                                       f"{ops.rt.job_info(ops.job) if ops.job is not None else None}; "
                                       f"slot {ops.rt.slot_info(0)}; holder {shm.get(ShmLink.HOLDER)} "
                                       f"seq {shm.get(ShmLink.SEQ)} seen {seen}")
                still.append((k, req))
            elif k >= warmup:
                S["lat"].append((tm["end_ns"] - tm["arrival_ns"]) * 1e-6)
                if tm["preempted_job"] >= 0:
                    S["pre"].append((tm["start_ns"] - tm["arrival_ns"]) * 1e-6)
        pending = still
    S["seen"] = seen
    return S


def finish_pair(shm: ShmLink, ops, me: int, seen: int, group=None, timeout_s: float = 60.0) -> int:
    """Stop the pair's job wherever it is: a migration still in flight lands and is adopted
    first.  Returns the handoff sequence number this rank has consumed."""
    t0 = time.monotonic()
    while True:
        cut = ops.migrated_out()
        if cut is not None:
            shm.set(ShmLink.HOLDER, me ^ 1)
            seen = shm.send_handoff(cut["iter"], cut["k"], cut["t_stop_ns"])
        dist.barrier(group=group)
        seq = shm.get(ShmLink.SEQ)
        if seq > seen and ops.job_gone():
            seen = seq
            ops.adopt(shm.get(ShmLink.ITER), shm.get(ShmLink.K))
        dist.barrier(group=group)
        states = [None, None]
        dist.all_gather_object(states, (me, ops.has_job(), ops.in_transit()), group=group)
        if sum(1 for _, h, _ in states if h) == 1 and not any(t for _, _, t in states):
            break
        if time.monotonic() - t0 > timeout_s:
            info = ops.rt.job_info(ops.job) if getattr(ops, "job", None) is not None else None
            raise RuntimeError(f"pair finish: job not settled {states}; rank {me}: job {info}, "
                               f"holder {shm.get(ShmLink.HOLDER)}, seq {shm.get(ShmLink.SEQ)}, seen {seen}")
        time.sleep(0.001)
    ops.stop()
    dist.barrier(group=group)
    return seen


class PoissonOps:
    """run_pair_poisson adapter onto a Runtime whose slot ``local`` is this process's GPU and
    slot ``remote`` maps the partner's arena (auto-preemption target)."""

    def __init__(self, rt, gh, ghi, local: int, remote: int, x_ptrs, out_ptrs,
                 iters: int = 1 << 40):
        self.rt, self.gh, self.ghi = rt, gh, ghi
        self.local, self.remote = local, remote
        self.x_ptrs, self.out_ptrs, self.iters = x_ptrs, out_ptrs, iters
        self.job = None
        self.n = 0
        self.iters_run = 0  # iterations this rank's tenures advanced the job

    def start(self) -> None:
        self.job = self.rt.start_training(self.gh, self.local, self.iters, self.remote)
        self._it0 = 0

    def _info(self):
        return self.rt.job_info(self.job) if self.job is not None else None

    def has_job(self) -> bool:
        i = self._info()
        return i is not None and i["state_name"] == "running"

    def job_gone(self) -> bool:
        """No job object on this rank (never had one, or it migrated out)."""
        return self.job is None

    def in_transit(self) -> bool:
        i = self._info()
        return i is not None and i["state_name"] in ("migrating", "stopping")

    def migrated_out(self):
        i = self._info()
        if i is None or i["state_name"] != "migrated_out":
            if i is not None and i["state_name"] == "failed":
                raise RuntimeError(f"job failed: {i}")
            return None
        self.iters_run += i["iter"] - self._it0
        self.job = None
        return {"iter": i["iter"], "k": i["k"], "t_stop_ns": i["last_stop_ns"], "xfer_us": i["last_xfer_us"],
                "bytes": i["migrated_bytes"]}

    def adopt(self, it: int, k: int) -> None:
        self.job = self.rt.adopt_job(self.gh, self.local, self.iters, it, k, self.remote)
        self._it0 = it

    def resume_ns(self) -> int:
        i = self._info()
        return i["last_resume_ns"] if i is not None else 0

    def submit(self, arrival_ns: int) -> int:
        j = self.n % len(self.x_ptrs)
        self.n += 1
        return self.rt.submit(self.ghi, self.local, self.x_ptrs[j], self.out_ptrs[j], arrival_ns=int(arrival_ns))

    def poll(self, req: int):
        return self.rt.poll(req)

    def stop(self) -> None:
        if self.job is not None:
            i = self._info()
            self.rt.stop_job(self.job)
            self.rt.wait_job(self.job, 120)
            self.iters_run += self._info()["iter"] - self._it0
