"""Oracle for the preemption scheduler: invariant checker + discrete-event model.

Invariants (each from the paper, checked on any trace — the oracle's own simulated
trace or the GPU runtime's recorded one):

  I1  "no two GPU executors are scheduled on a single GPU simultaneously"
      (section 3.4): on a device, compute intervals of different
      models are disjoint.
  I2  per-job order: "executors from consecutive runs of the same session follow
      sequential order" (section 3.2); with "no work is lost"
       every (iter, k) of a job runs exactly once, in order, and a
      job's subgraphs never overlap each other.
  I3  preemption latency is bounded by the outstanding work of the preemptee: "Only
      waiting for the outstanding nodes of a preempted job to complete is on the
      critical path" (section 5.2.3).  Checked as
      start(infer) - max(arrival, end of the previous inference on that device)
      <= window x max train-subgraph duration on that device + slack, where ``window`` is
      the number of subgraphs the runtime may have dispatched ahead of its boundary gate.
  I4  cut rule (reading Q13): a request arriving while S_k runs is served at the
      boundary after S_k — more precisely, no training subgraph is DISPATCHED after the
      arrival and before the inference starts (subgraphs already dispatched to the GPU are
      allowed to finish); events may carry "launch" (dispatch time),
      else t0 is the dispatch time.
  I5  training priority ("a high priority job is allowed to start
      immediately after submission"; "upon the arrival of a high
      priority model, the low priority one is preempted and migrated"): on a device, from a
      job's submission there until its last subgraph there ends, no training subgraph of a
      lower-priority job is DISPATCHED there; at most ``window`` lower-priority subgraphs
      execute on the device after the submission and before the high-priority job's first
      subgraph (the outstanding subgraphs drain, nothing more); and that first subgraph
      starts within ``window`` x (longest lower-priority subgraph on the device) + slack of
      the submission.

Event dicts: {"dev", "job", "kind": "train"|"infer", "iter", "k", "t0", "t1",
"arrival" (infer only), "after" (infer only, optional: the training job it was ordered
after on the device), "launch" (train only, optional: dispatch time), "d0"/"d1"
(optional: the DEVICE execution interval on the same clock, 0 if unknown)}; times in any
consistent unit.  ``device_view`` turns a recorded trace into device intervals: every
invariant is then checked on when the GPU executed the work, not on when the host saw it.

Pins (tests/test_oracle_schedule.py): hand-built violating traces for I1..I4 are
rejected; the discrete-event model's traces satisfy them; closed-form latencies of
the model for single arrivals.
"""
from __future__ import annotations

import heapq
from typing import Dict, List, Sequence


class InvariantError(AssertionError):
    pass


def _device_ordered(a: dict, b: dict) -> bool:
    """True when one of two overlapping HOST intervals is an inference event that the GPU
    ran after the other, a training subgraph: the request carries ``after`` = that job
    (its chain waited, on the device, for the job's newest subgraph dispatched before the
    request's own dispatch t0 — stream order covers every earlier one) and the subgraph
    was dispatched ("launch", else t0) no later than the request.  Host intervals are
    supersets of device execution, so only such a dependency makes an overlap legal."""
    for r, t in ((a, b), (b, a)):
        if (r["kind"] == "infer" and t["kind"] == "train" and r.get("after") == t["job"]
                and t.get("launch", t["t0"]) <= r["t0"]):
            return True
    return False


def device_view(events: Sequence[dict]) -> List[dict]:
    """Train / infer events on the DEVICE timeline: t0, t1 := d0, d1 (the GPU execution
    interval); the host interval is kept as h0, h1 and the host-side "after" dependency is
    dropped (device intervals of dependent work are disjoint by themselves).  Events that
    carry no device interval (host stages, or d0 == 0) are returned unchanged."""
    out = []
    for e in events:
        e = dict(e)
        if e.get("kind") in ("train", "infer") and e.get("d0") and e.get("d1"):
            e["h0"], e["h1"] = e["t0"], e["t1"]
            e["t0"], e["t1"] = e["d0"], e["d1"]
            e.pop("after", None)
        out.append(e)
    return out


def check_no_corun(events: Sequence[dict]) -> None:
    """I1: per device, intervals of different jobs never overlap (unless device-ordered,
    see _device_ordered)."""
    by_dev: Dict[int, List[dict]] = {}
    for e in events:
        by_dev.setdefault(e["dev"], []).append(e)
    for d, evs in by_dev.items():
        evs = sorted(evs, key=lambda e: (e["t0"], e["t1"]))
        active: List[dict] = []
        for b in evs:
            active = [a for a in active if a["t1"] > b["t0"]]
            for a in active:
                if a["job"] != b["job"] and not _device_ordered(a, b):
                    raise InvariantError(f"dev {d}: job {a['job']} [{a['t0']},{a['t1']}) overlaps "
                                         f"job {b['job']} [{b['t0']},{b['t1']})")
            active.append(b)


def check_job_order(events: Sequence[dict], n_sub: Dict[int, int],
                    start: Dict[int, tuple] | None = None) -> None:
    """I2: each training job's (iter, k) sequence is the contiguous enumeration."""
    by_job: Dict[int, List[dict]] = {}
    for e in events:
        if e["kind"] == "train":
            by_job.setdefault(e["job"], []).append(e)
    for j, evs in by_job.items():
        evs = sorted(evs, key=lambda e: e["t0"])
        n = n_sub[j]
        it, k = (start or {}).get(j, (evs[0]["iter"], evs[0]["k"]))
        prev_t1 = None
        for e in evs:
            if (e["iter"], e["k"]) != (it, k):
                raise InvariantError(f"job {j}: expected ({it},{k}) got ({e['iter']},{e['k']})")
            if prev_t1 is not None and e["t0"] < prev_t1:
                raise InvariantError(f"job {j}: subgraph ({it},{k}) overlaps its predecessor")
            prev_t1 = e["t1"]
            k += 1
            if k == n:
                it, k = it + 1, 0


def preempt_latency_report(events: Sequence[dict], slack: float, window: int = 1) -> dict:
    """I3 per request: wait = start - ready, ready = max(arrival, end of the previous
    inference on the device); bound = window x (longest training subgraph on the device) +
    slack (``window`` subgraphs may be dispatched ahead of the boundary gate).  A request over
    the bound is a HOST outlier when its host dispatch decision ("h0", device_view) itself came
    later than ready + bound — the dispatcher thread was late, which no device-side drain
    explains — or when it recorded no device dependency (``iter == -1``: nothing drained
    before it), else a violation.  Returns {"n", "bound", "violations", "host_outliers",
    "waits"}."""
    by_dev: Dict[int, List[dict]] = {}
    for e in events:
        by_dev.setdefault(e["dev"], []).append(e)
    rep = {"n": 0, "bound": {}, "violations": [], "host_outliers": [], "waits": []}
    for d, evs in by_dev.items():
        longest = max([e["t1"] - e["t0"] for e in evs if e["kind"] == "train"], default=0.0)
        bound = window * longest + slack
        rep["bound"][d] = bound
        prev_end = float("-inf")
        for e in sorted([e for e in evs if e["kind"] == "infer"], key=lambda e: e["t0"]):
            ready = max(e["arrival"], prev_end)
            wait = e["t0"] - ready
            rep["n"] += 1
            rep["waits"].append(wait)
            if wait > bound:
                # no device dependency recorded (iter == -1: the device was free, nothing of a
                # training job drained before it): the wait is dispatch / launch time, not a drain
                no_dep = e.get("iter") == -1
                host_late = no_dep or (e.get("h0") is not None and e["h0"] - ready > bound)
                (rep["host_outliers"] if host_late else rep["violations"]).append((e, wait))
            prev_end = e["t1"]
    return rep


def check_preempt_latency(events: Sequence[dict], slack: float, window: int = 1) -> None:
    """I3: inference start - ready time <= window x longest training subgraph on that
    device + slack, for every request."""
    r = preempt_latency_report(events, slack, window)
    bad = r["violations"] + r["host_outliers"]
    if bad:
        e, w = bad[0]
        raise InvariantError(f"dev {e['dev']}: inference waited {w} > {r['bound'][e['dev']]} "
                             f"({len(bad)} of {r['n']} requests)")


def check_cut_rule(events: Sequence[dict]) -> None:
    """I4: the first training subgraph that starts on a device after an arrival but
    before the inference ran must not exist (the job stops at the next boundary)."""
    by_dev: Dict[int, List[dict]] = {}
    for e in events:
        by_dev.setdefault(e["dev"], []).append(e)
    for d, evs in by_dev.items():
        trains = [e for e in evs if e["kind"] == "train"]
        for r in (e for e in evs if e["kind"] == "infer"):
            for t in trains:
                if r["arrival"] <= t.get("launch", t["t0"]) < r["t0"]:
                    raise InvariantError(f"dev {d}: subgraph ({t['iter']},{t['k']}) started at "
                                         f"{t['t0']} after arrival {r['arrival']} before the "
                                         f"inference at {r['t0']}")


def check_priority(events: Sequence[dict], prio: Dict[int, int],
                   submit: Dict[int, tuple], slack: float = 0.0, window: int = 1) -> None:
    """I5: ``prio[job]`` = priority, ``submit[job]`` = (device, submission time)."""
    trains = [e for e in events if e["kind"] == "train"]
    for hj, (dev, ts) in submit.items():
        mine = sorted((e for e in trains if e["job"] == hj and e["dev"] == dev),
                      key=lambda e: e["t0"])
        if not mine:
            continue
        end = mine[-1]["t1"]
        lower = [e for e in trains if e["dev"] == dev and prio[e["job"]] < prio[hj]]
        for e in lower:
            if ts <= e.get("launch", e["t0"]) < end:
                raise InvariantError(
                    f"dev {dev}: job {e['job']} (prio {prio[e['job']]}) dispatched "
                    f"({e['iter']},{e['k']}) at {e.get('launch', e['t0'])} while job {hj} "
                    f"(prio {prio[hj]}) was present [{ts},{end})")
        drained = [e for e in lower if e["t1"] > ts and e["t0"] < mine[0]["t0"]]
        if len(drained) > window:
            raise InvariantError(f"dev {dev}: {len(drained)} lower-priority subgraphs ran after "
                                 f"job {hj}'s submission at {ts} (window {window})")
        longest = max([e["t1"] - e["t0"] for e in lower], default=0.0)
        if mine[0]["t0"] - ts > window * longest + slack:
            raise InvariantError(f"dev {dev}: job {hj} started {mine[0]['t0'] - ts} after "
                                 f"submission > {window} x {longest} + {slack}")


def check_lockstep(events: Sequence[dict], members: Sequence[int]) -> None:
    """I6, input reuse ("all models should finish processing an input
    tensor before moving onto the next input batch ... each model's GPU executor in a
    round-robin manner"): ordered by start time, the training subgraphs of the member jobs
    form contiguous blocks (iteration i of member m) in the order (i, m) = (0, 0), (0, 1),
    ..., (1, 0), ... — a member absent from the tail (it finished) is skipped."""
    order = {j: m for m, j in enumerate(members)}
    ev = sorted((e for e in events if e["kind"] == "train" and e["job"] in order),
                key=lambda e: e["t0"])
    blocks = []
    for e in ev:
        key = (e["iter"], order[e["job"]])
        if not blocks or blocks[-1] != key:
            blocks.append(key)
    if len(set(blocks)) != len(blocks):
        raise InvariantError(f"lockstep: a (iteration, member) block is split: {blocks}")
    if blocks != sorted(blocks):
        raise InvariantError(f"lockstep: blocks out of round-robin order: {blocks}")


def check_all(events: Sequence[dict], n_sub: Dict[int, int], slack: float = 0.0) -> None:
    check_no_corun(events)
    check_job_order(events, n_sub)
    check_preempt_latency(events, slack)
    check_cut_rule(events)


def simulate(durations: Sequence[float], iters: int, arrivals: Sequence[float],
             infer_dur: float, tier: str = "host", swap_out: float = 0.0,
             swap_in: float = 0.0, gate: float = 0.0) -> List[dict]:
    """Discrete-event model of one training job (job 0) + an inference stream (job 1).

    Policy (readings Q4-Q7, Q13):
      * training runs S_0..S_{n-1} per iteration back to back on device 0, ``gate``
        between subgraphs;
      * a request arriving while S_k runs is served once S_k finishes; requests are
        FIFO by arrival and all queued ones run before the job resumes;
      * host tier: state goes out (``swap_out``, concurrent with inference) and comes
        back (``swap_in``) after the queue drained; the job resumes on device 0;
      * peer tier: the job migrates (``swap_out``) and resumes on device 1, where it
        stays (Q7); later requests on device 0 find no training job to preempt.
    """
    n = len(durations)
    ev: List[dict] = []
    t = 0.0
    dev = 0
    q = list(arrivals)
    heapq.heapify(q)
    it, k = 0, 0
    free0 = 0.0  # device-0 time after the last inference

    def serve_pending(now):
        nonlocal free0
        end = max(now, free0)
        while q and q[0] <= end:
            a = heapq.heappop(q)
            s = max(end, a)
            ev.append({"dev": 0, "job": 1, "kind": "infer", "iter": 0, "k": 0, "t0": s,
                       "t1": s + infer_dur, "arrival": a})
            end = s + infer_dur
        free0 = end
        return end

    while it < iters:
        if dev == 0 and q and q[0] <= t:
            # preempt at this boundary
            cut_t = t
            drained = serve_pending(cut_t)
            if tier == "host":
                t = max(drained, cut_t + swap_out) + swap_in
            else:
                dev = 1
                t = cut_t + swap_out
            continue
        s = t
        e = s + durations[k]
        ev.append({"dev": dev, "job": 0, "kind": "train", "iter": it, "k": k, "t0": s, "t1": e})
        t = e + gate
        k += 1
        if k == n:
            it, k = it + 1, 0
    # serve requests that arrive after training finished (or on a now-free device 0)
    while q:
        a = heapq.heappop(q)
        s = max(a, free0)
        ev.append({"dev": 0, "job": 1, "kind": "infer", "iter": 0, "k": 0, "t0": s,
                   "t1": s + infer_dur, "arrival": a})
        free0 = s + infer_dur
    return ev


def simulate_priority(dur_lo: Sequence[float], iters_lo: int, dur_hi: Sequence[float],
                      iters_hi: int, t_hi: float, tier: str = "host", swap_out: float = 0.0,
                      swap_in: float = 0.0, home: bool = False) -> List[dict]:
    """Discrete-event model of the Fig. 7 scenario: job 0 (low
    priority) trains on device 0; job 1 (high priority) is submitted on device 0 at
    ``t_hi``.  Job 0 stops at its first boundary >= t_hi (the subgraph running at t_hi
    finishes); job 1 starts right then and runs to completion on
    device 0.  Host tier: job 0's state goes out (``swap_out``, concurrent with job 1) and
    comes back (``swap_in``) once job 1 finished, then job 0 continues on device 0.  Peer
    tier: job 0 resumes on device 1 at cut + swap_out (reading Q7: it stays there), or
    with ``home`` migrates back to device 0 at its first boundary after job 1 finished
    (another ``swap_out``)."""
    ev: List[dict] = []
    n_lo = len(dur_lo)
    t, dev, it, k = 0.0, 0, 0, 0
    hi_end = None
    moved_home = False
    while it < iters_lo:
        if hi_end is None and t >= t_hi:
            # cut: job 1 runs its whole job on device 0 from here
            cut = t
            s = cut
            for i in range(iters_hi):
                for j, d in enumerate(dur_hi):
                    ev.append({"dev": 0, "job": 1, "kind": "train", "iter": i, "k": j,
                               "t0": s, "t1": s + d})
                    s += d
            hi_end = s
            if tier == "host":
                t = max(hi_end, cut + swap_out) + swap_in
            else:
                dev, t = 1, cut + swap_out
            continue
        if home and dev == 1 and hi_end is not None and t >= hi_end and not moved_home:
            dev, t, moved_home = 0, t + swap_out, True
            continue
        ev.append({"dev": dev, "job": 0, "kind": "train", "iter": it, "k": k, "t0": t,
                   "t1": t + dur_lo[k]})
        t += dur_lo[k]
        k += 1
        if k == n_lo:
            it, k = it + 1, 0
    if hi_end is None:  # job 0 finished before job 1 arrived
        s = max(t, t_hi)
        for i in range(iters_hi):
            for j, d in enumerate(dur_hi):
                ev.append({"dev": 0, "job": 1, "kind": "train", "iter": i, "k": j,
                           "t0": s, "t1": s + d})
                s += d
    return ev
