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

from typing import Optional

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
