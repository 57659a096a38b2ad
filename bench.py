#!/usr/bin/env python
"""SwitchFlow subgraph-preemption benchmark on B200 (driver contract: one JSON line).

Metric (BASELINE.json): p99 inference latency + preempt-to-resume ms; migration GB/s vs
NVLink / HBM peak.  `value` = p99 latency (ms, lower is better) of batch-1 inference
requests that each preempt a running training job.

Workload at N=1 ("C4@1GPU", the largest single-GPU config): a training
job with the ResNet-50-shaped state (Keras variable list, 534 tensors, 204.9 MB params +
momentum; per-layer softmax-regression compute at batch 8, reading Q16) runs
on the GPU while an OPEN-LOOP Poisson stream of batch-1 requests of a 2048-4096-4096-1000
MLP (29.3M params; rate --rate, default 100 req/s, arrival seed 7) arrives.  A request that
finds the job on the GPU stops it at the next subgraph boundary; the job's live set is
packed and parked in pinned host memory (host tier), the request runs, the state is
swapped back and the job resumes.  `value` = p99 latency from the scheduled arrival to the
completion observed on the host, inputs resident in HBM; `e2e` repeats it with the
request's input / output in pinned host memory (H2D + D2H inside each request, through
sf_submit_inference).  The closed-loop "chase" arm (every request preempts; the next one
is issued after the resume) supplies the per-cycle migration numbers (pack GB/s,
preempt-to-resume split).

Under torchrun (N>1) every rank runs the same job + request stream on its own GPU
(independent replicas, weak scaling) and rank 0 pools the samples.

--impl reference times the CPU oracle (oracle/, plain numpy fp64) on the host cores on a
bounded sample of the same workload (each distinct subgraph timed once).
"""
from __future__ import annotations

import argparse
import json
import os

import subprocess
import sys
import threading
import time

import numpy as np


def _gate_requested(argv) -> bool:
    """--gate 1 / --gate=1 on the command line (read before any CUDA context exists)."""
    for i, a in enumerate(argv):
        if a == "--gate" and i + 1 < len(argv):
            return argv[i + 1] == "1"
        if a.startswith("--gate="):
            return a.split("=", 1)[1] == "1"
    return False


if _gate_requested(sys.argv):  # the drain gate parks a stream: 32 hardware queues (see the package)
    os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

HOST = -1
METRIC = "p99 inference latency + preempt-to-resume ms; migration GB/s vs NVLink/HBM peak"
UNIT = "ms"
WORKLOAD = "C4@1GPU: ResNet-50-shaped training job (534 tensors, 204.9 MB) + open-loop Poisson " \
           "batch-1 inference stream, repeated preemptions, host-tier migration"


def pct(x, q):
    return float(np.percentile(np.asarray(x, np.float64), q)) if len(x) else None


def block_size(args) -> int:
    """Requests per timed step: --requests-per-step, raised so that the headline percentiles rest
    on at least 1,000 requests whatever --steps is (round-1 verdict: a p99 of 20 samples)."""
    return max(args.requests_per_step, -(-getattr(args, "min_requests", 1000) // max(1, args.steps)))


def load_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,"
                 "clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
                 "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
                 "clocks_event_reasons.sw_power_cap", "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 7:
                self.rows.append(parts)

    def __exit__(self, *exc):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[3 + i] == "Active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


# ------------------------------------------------------------------------------------------
def build_workload(batch: int, spatial_div: int):
    from sf_inputs import graphs as G
    g = G.resnet50_forest(batch=batch, spatial_div=spatial_div)
    # SF_BENCH_WT=1: output-major weights ([N][K], GEMM TB, row-streaming GEMV); measured
    # slower than the [K][N] TMA cluster GEMV on this workload (reading Q30)
    gi = G.mlp_infer((2048, 4096, 4096, 1000), name="infer_mlp_29M",
                     wt=os.environ.get("SF_BENCH_WT", "0") == "1")
    return g, gi


_CACHE = {}


def workload_arrays(g, gi, key):
    from sf_inputs import data as D
    if key not in _CACHE:
        _CACHE[key] = ({**D.init_state(g), **D.datasets(g)}, D.init_state(gi, seed=D.SEED_INFER))
    return _CACHE[key]


def run_arm(args, local_dev: int, steps: int, warmup: int, host_io: bool, exclusive=True,
            iteration_granularity=False, measure=True, defer=None, duplex=None,
            early=None, target=HOST, gate=None):
    """One runtime instance: training job + one request per step.  Returns samples."""
    import torch
    from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime, kernel_launches, now_ns
    from sf_inputs import data as D

    g, gi = build_workload(args.batch, args.spatial_div)
    rt = Runtime([local_dev], exclusive=exclusive, auto_preempt=True,
                 iteration_granularity=iteration_granularity, max_inflight=args.max_inflight,
                 defer_migration=args.defer if defer is None else defer,
                 dispatch_spin_us=args.dispatch_spin_us,
                 inflight_budget_us=args.inflight_budget_us,
                 host_duplex=bool(args.duplex if duplex is None else duplex),
                 early_launch=bool(args.early if early is None else early),
                 drain_gate=bool(args.gate if gate is None else gate),
                 infer_l2_persist_bytes=int(args.l2_persist_mb * (1 << 20)))
    gh = rt.register(g)
    info = gh.partition("max_ops" if args.max_ops else "phase", args.max_ops,
                        update_chunks=args.update_chunks)
    gh.bind(0, staging=True, host_staging=True)
    arrays, arrays_i = workload_arrays(g, gi, (args.batch, args.spatial_div))
    gh.load(0, arrays)
    ghi = rt.register(gi, priority=1)
    ghi.partition()
    ghi.bind(0, staging=False)
    ghi.load(0, arrays_i)
    n_in = steps + warmup
    xs = D.infer_inputs(gi, min(n_in, 64))
    dev = torch.device("cuda", local_dev)
    if host_io:
        x_t = torch.from_numpy(xs).pin_memory()
        out_t = torch.zeros(len(xs), 1, 1000).pin_memory()
    else:
        x_t = torch.from_numpy(xs).to(dev)
        out_t = torch.zeros(len(xs), 1, 1000, device=dev)
    rng = np.random.default_rng(1234 + local_dev)
    job = rt.start_training(gh, 0, 1 << 40, target)
    # estimate the mean training-subgraph duration from the trace (for arrival jitter)
    time.sleep(0.3)
    tr = [e for e in rt.trace() if e["kind"] == "train"]
    sub_ms = float(np.mean([(e["t1"] - e["t0"]) * 1e-6 for e in tr])) if tr else 0.5
    iters_ms = sub_ms * gh.n_subgraphs
    S = {"lat": [], "pre": [], "p2r": [], "pack_us": [], "xfer_us": [], "unpack_us": [],
         "bytes": [], "staging": [], "cut_k": []}
    t_region = None
    launches0 = None
    sampler = None
    torch.cuda.synchronize(dev)
    for s in range(n_in):
        timed = s >= warmup
        if timed and t_region is None:
            if args.world > 1:
                import torch.distributed as dist
                dist.barrier()
            torch.cuda.synchronize(dev)
            sampler = ClockSampler(local_dev).__enter__() if measure else None
            ev0 = torch.cuda.Event(enable_timing=True)
            ev0.record()
            t_region = time.perf_counter()
            launches0 = kernel_launches()
        # wait until the job runs again (the previous preemption resumed)
        t_wait = time.perf_counter()
        while True:
            ji = rt.job_info(job)
            if ji["state_name"] == "running":
                break
            if time.perf_counter() - t_wait > 30:
                raise RuntimeError(f"job stuck: {ji}")
            time.sleep(2e-4)
        # seeded arrival inside a training subgraph
        delay = rng.uniform(0.2, 1.0) * sub_ms * 1e-3 * 2
        t_arr = time.perf_counter() + delay
        while time.perf_counter() < t_arr:
            pass
        before = rt.job_info(job)
        i = s % len(xs)
        req = rt.submit(ghi, 0, x_t[i].data_ptr(), out_t[i].data_ptr())
        tm = rt.wait(req, 60)
        # wait for the resume of this preemption
        t_wait = time.perf_counter()
        while True:
            ji = rt.job_info(job)
            if ji["n_preemptions"] > before["n_preemptions"] and ji["last_resume_ns"] > ji["last_stop_ns"]:
                break
            if not exclusive or time.perf_counter() - t_wait > 30:
                break
            time.sleep(2e-4)
        if timed:
            S["lat"].append((tm["end_ns"] - tm["arrival_ns"]) * 1e-6)
            S["pre"].append((tm["start_ns"] - tm["arrival_ns"]) * 1e-6)
            S["cut_k"].append(tm["cut_k"])
            if exclusive and ji["n_preemptions"] > before["n_preemptions"]:
                S["p2r"].append((ji["last_resume_ns"] - ji["last_stop_ns"]) * 1e-6)
                S["pack_us"].append(ji["last_pack_us"])
                S["xfer_us"].append(ji["last_xfer_us"])
                S["unpack_us"].append(ji["last_unpack_us"])
                S["bytes"].append(ji["migrated_bytes"] - before["migrated_bytes"])
    ev1 = torch.cuda.Event(enable_timing=True)
    ev1.record()
    torch.cuda.synchronize(dev)
    if args.world > 1:
        import torch.distributed as dist
        dist.barrier()
    wall = time.perf_counter() - t_region
    launches = kernel_launches() - launches0
    if sampler:
        sampler.__exit__()
    S["region_ms"] = ev0.elapsed_time(ev1)
    S["wall_s"] = wall
    S["launches"] = launches
    S["clocks"] = sampler.summary() if sampler else None
    S["sub_ms"] = sub_ms
    tr = [e for e in rt.trace() if e["kind"] == "train"]
    per_it = {}
    for e in tr:
        a, b_ = per_it.get(e["iter"], (e["t0"], e["t1"]))
        per_it[e["iter"]] = (min(a, e["t0"]), max(b_, e["t1"]))
    spans = sorted((b_ - a) * 1e-6 for a, b_ in per_it.values())
    S["iter_ms"] = spans[len(spans) // 2] if spans else iters_ms
    S["n_subgraphs"] = gh.n_subgraphs
    S["info"] = {"arena_bytes": info.arena_bytes, "persistent_bytes": info.persistent_bytes,
                 "max_live_bytes": info.max_live_bytes, "staging_bytes": info.staging_bytes}
    rt.stop_job(job)
    rt.wait_job(job, 120)
    rt.close()
    return S


def wait_or_dump(rt, req, job, timeout_s):
    """rt.wait with a diagnostic dump (slot / job state, trace tail) to stderr when a request
    does not complete in time; then the process ends without running destructors."""
    try:
        return rt.wait(req, timeout_s)
    except Exception as ex:  # noqa: BLE001 (diagnostics, then exit)
        import traceback
        print(f"request {req} did not complete: {ex}", file=sys.stderr)
        try:
            print("slot 0", rt.slot_info(0), file=sys.stderr)
            print("job", rt.job_info(job), file=sys.stderr)
            for e in rt.trace()[-12:]:
                print("trace", e, file=sys.stderr)
        except Exception:  # noqa: BLE001
            traceback.print_exc()
        sys.stderr.flush()
        os._exit(3)


def run_poisson_arm(args, local_dev: int, n_req: int, warmup: int, host_io: bool, exclusive=True,
                    iteration_granularity=False, measure=True, defer=None, duplex=None,
            early=None, target=HOST, gate=None):
    """C4 as specified: an OPEN-LOOP Poisson request stream (rate args.rate
    req/s, arrival seed 7 + pair) against the running training job.  Each request is submitted
    at its scheduled arrival time (passed to sf_submit_inference, so any host delay counts
    against the latency); a request that finds the job on the GPU preempts it, one that
    arrives while the job is parked / migrating runs at once.  Returns samples."""
    import torch
    from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime, kernel_launches, now_ns
    from sf_inputs import data as D

    g, gi = build_workload(args.batch, args.spatial_div)
    rt = Runtime([local_dev], exclusive=exclusive, auto_preempt=True,
                 iteration_granularity=iteration_granularity, max_inflight=args.max_inflight,
                 defer_migration=args.defer if defer is None else defer,
                 dispatch_spin_us=args.dispatch_spin_us,
                 inflight_budget_us=args.inflight_budget_us,
                 host_duplex=bool(args.duplex if duplex is None else duplex),
                 early_launch=bool(args.early if early is None else early),
                 drain_gate=bool(args.gate if gate is None else gate),
                 infer_l2_persist_bytes=int(args.l2_persist_mb * (1 << 20)))
    gh = rt.register(g)
    gh.partition("max_ops" if args.max_ops else "phase", args.max_ops, update_chunks=args.update_chunks)
    gh.bind(0, staging=True, host_staging=True)
    arrays, arrays_i = workload_arrays(g, gi, (args.batch, args.spatial_div))
    gh.load(0, arrays)
    ghi = rt.register(gi, priority=1)
    ghi.partition()
    ghi.bind(0, staging=False)
    ghi.load(0, arrays_i)
    n_in = n_req + warmup
    xs = D.infer_inputs(gi, min(n_in, 64))
    dev = torch.device("cuda", local_dev)
    if host_io:
        x_t = torch.from_numpy(xs).pin_memory()
        out_t = torch.zeros(len(xs), 1, 1000).pin_memory()
    else:
        x_t = torch.from_numpy(xs).to(dev)
        out_t = torch.zeros(len(xs), 1, 1000, device=dev)
    job = rt.start_training(gh, 0, 1 << 40, target)
    time.sleep(0.3)
    # solo training throughput of this very job before the request stream starts (the
    # reference point of the collocated throughput loss)
    solo_it0, solo_t0 = rt.job_info(job)["iter"], time.perf_counter()
    time.sleep(args.solo_s)
    solo_it_s = (rt.job_info(job)["iter"] - solo_it0) / (time.perf_counter() - solo_t0)
    rng = np.random.default_rng(7 + args.rank // 2)
    gaps_ns = (rng.exponential(1.0 / args.rate, n_in) * 1e9).astype(np.int64)
    torch.cuda.synchronize(dev)
    t0 = now_ns() + 2_000_000
    arr = t0 + np.cumsum(gaps_ns)
    reqs, p2r, last = [], [], None
    sampler, ev0, launches0, t_region = None, None, None, None
    for i in range(n_in):
        if i == warmup:
            sampler = ClockSampler(local_dev).__enter__() if measure else None
            ev0 = torch.cuda.Event(enable_timing=True)
            ev0.record()
            t_region = time.perf_counter()
            launches0 = kernel_launches()
            ji0 = rt.job_info(job)
        next_poll = 0
        while True:
            t = now_ns()
            if t >= arr[i]:
                break
            if t >= next_poll and arr[i] - t > 300_000:
                # preempt-to-resume of every completed cycle (a cycle lasts ~8 ms); polled
                # sparsely so the bench never contends for the runtime lock near an arrival
                next_poll = t + 500_000
                ji = rt.job_info(job)
                key = (ji["last_stop_ns"], ji["last_resume_ns"])
                if key != last and ji["last_resume_ns"] > ji["last_stop_ns"] > 0:
                    if i >= warmup:
                        p2r.append((ji["last_resume_ns"] - ji["last_stop_ns"]) * 1e-6)
                    last = key
        j = i % len(xs)
        reqs.append(rt.submit(ghi, 0, x_t[j].data_ptr(), out_t[j].data_ptr(), arrival_ns=int(arr[i])))
    tms = [wait_or_dump(rt, r, job, 120) for r in reqs]
    ji1 = rt.job_info(job)
    ev1 = torch.cuda.Event(enable_timing=True)
    ev1.record()
    torch.cuda.synchronize(dev)
    wall = time.perf_counter() - t_region
    coloc_it_s = (ji1["iter"] - ji0["iter"]) / max(wall, 1e-9)
    launches = kernel_launches() - launches0
    if sampler:
        sampler.__exit__()
    info_j = rt.job_info(job)
    tr = [e for e in rt.trace() if e["kind"] == "train"]
    rt.stop_job(job)
    rt.wait_job(job, 120)
    rt.close()
    T = tms[warmup:]
    lat = [(t["end_ns"] - t["arrival_ns"]) * 1e-6 for t in T]
    pre = [(t["start_ns"] - t["arrival_ns"]) * 1e-6 for t in T if t["preempted_job"] == job]
    dev_us = [t["device_us"] for t in T if t["device_us"] > 0]
    per_it = {}
    for e in tr:
        a, b_ = per_it.get(e["iter"], (e["t0"], e["t1"]))
        per_it[e["iter"]] = (min(a, e["t0"]), max(b_, e["t1"]))
    if os.environ.get("SF_BENCH_DIAG"):
        for name, sel in (("preempting", [t for t in T if t["preempted_job"] == job]),
                          ("not preempting", [t for t in T if t["preempted_job"] != job])):
            if not sel:
                continue
            w = np.array([(t["start_ns"] - t["arrival_ns"]) * 1e-3 for t in sel])
            dv = np.array([t["device_us"] for t in sel])
            tot = np.array([(t["end_ns"] - t["arrival_ns"]) * 1e-3 for t in sel])
            print(f"[diag] {name:15s} n={len(sel):4d} wait us p50/p99 {np.median(w):7.1f}/{np.percentile(w, 99):7.1f}"
                  f"  device us p50/p99 {np.median(dv):6.1f}/{np.percentile(dv, 99):6.1f}"
                  f"  total p50/p99 {np.median(tot):6.1f}/{np.percentile(tot, 99):6.1f}", file=sys.stderr)
    # where a request's latency goes: wait for the device (drain of the preempted job's
    # in-flight subgraphs, or an earlier request), device time of the chain, host overhead
    # (dispatch decision .. first event on the device, last kernel .. completion observed)
    bd = {}
    for name, sel in (("preempting", [t for t in T if t["preempted_job"] == job]),
                      ("not_preempting", [t for t in T if t["preempted_job"] != job])):
        sel = [t for t in sel if t["device_us"] > 0]
        if not sel:
            continue
        w = np.array([(t["start_ns"] - t["arrival_ns"]) * 1e-3 for t in sel])
        dv = np.array([t["device_us"] for t in sel])
        ho = np.array([(t["end_ns"] - t["start_ns"]) * 1e-3 - t["device_us"] for t in sel])
        lu = np.array([t["launch_us"] for t in sel])
        du = np.array([t["dispatch_us"] for t in sel])
        bd[name] = {"n": len(sel), **{f"{k}_p{q}": round(float(np.percentile(v, q)), 2)
                                       for k, v in (("wait", w), ("device", dv), ("host_overhead", ho),
                                                    ("launch", lu), ("dispatch", du))
                                       for q in (50, 99)}}
    return {"lat": lat, "pre": pre, "p2r": p2r, "frac_preempting": len(pre) / max(1, len(T)),
            "breakdown": bd,
            "device_us": dev_us, "region_ms": ev0.elapsed_time(ev1), "wall_s": wall,
            "launches": launches, "clocks": sampler.summary() if sampler else None,
            "reparks": info_j["n_reparks"], "iters_done": len(per_it),
            "training": {"solo_it_per_s": solo_it_s, "collocated_it_per_s": coloc_it_s,
                         "loss_frac": 1.0 - coloc_it_s / solo_it_s if solo_it_s > 0 else None,
                         "preemptions_in_region": ji1["n_preemptions"] - ji0["n_preemptions"],
                         "solo_window_s": args.solo_s}}


def run_pair_arm(args, local_dev: int, steps: int, warmup: int, host_io: bool, gloo):
    """N>1: ranks (2i, 2i+1) ping-pong one training job; each request preempts it into the
    partner's arena (peer-store kernel over NVLink, CUDA IPC mapping); pairs are independent."""
    import torch
    import torch.distributed as dist
    from paper_conf_middleware_wur0hdh21_b200.pairs import PairLink, RuntimeOps, run_pair_steps
    from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime, kernel_launches
    from sf_inputs import data as D

    g, gi = build_workload(args.batch, args.spatial_div)
    rt = Runtime([local_dev, -1], exclusive=True, auto_preempt=True, defer_migration=bool(args.defer),
                 dispatch_spin_us=args.dispatch_spin_us, inflight_budget_us=args.inflight_budget_us,
                 max_inflight=args.max_inflight)
    gh = rt.register(g)
    info = gh.partition("max_ops" if args.max_ops else "phase", args.max_ops,
                        update_chunks=args.update_chunks)
    gh.bind(0, staging=False, host_staging=False)
    arrays, arrays_i = workload_arrays(g, gi, (args.batch, args.spatial_div))
    link = PairLink(gloo)
    gh.load(0, arrays if link.starts_holding else {i: a for i, a in arrays.items()
                                                   if g.tensors[i].kind == 3})
    ghi = rt.register(gi, priority=1)
    ghi.partition()
    ghi.bind(0, staging=False)
    ghi.load(0, arrays_i)
    rt.import_arena(gh, 1, link.exchange_bytes(rt.export_arena(gh, 0)))
    xs = D.infer_inputs(gi, 64)
    dev = torch.device("cuda", local_dev)
    if host_io:
        x_t, out_t = torch.from_numpy(xs).pin_memory(), torch.zeros(64, 1, 1000).pin_memory()
    else:
        x_t, out_t = torch.from_numpy(xs).to(dev), torch.zeros(64, 1, 1000, device=dev)
    ops = RuntimeOps(rt, gh, ghi, 0, 1, [x.data_ptr() for x in x_t], [o.data_ptr() for o in out_t],
                     sub_ms=0.06, rng=np.random.default_rng(4321 + args.rank))
    if link.starts_holding:
        ops.start()
    Sw = run_pair_steps(link, ops, 0, warmup)
    dist.barrier(group=gloo)
    torch.cuda.synchronize(dev)
    sampler = ClockSampler(local_dev).__enter__() if not host_io else None
    ev0 = torch.cuda.Event(enable_timing=True)
    ev0.record()
    launches0 = kernel_launches()
    S = run_pair_steps(link, ops, steps, 0, holding=Sw["holding_at_end"])
    ev1 = torch.cuda.Event(enable_timing=True)
    ev1.record()
    torch.cuda.synchronize(dev)
    dist.barrier(group=gloo)
    if sampler:
        sampler.__exit__()
    S["region_ms"] = ev0.elapsed_time(ev1)
    S["launches"] = kernel_launches() - launches0
    S["clocks"] = sampler.summary() if sampler else None
    S["n_subgraphs"] = gh.n_subgraphs
    S["sub_ms"] = 0.06
    S["xfer_us"] = [c["xfer_us"] for c in S["out"]]
    S["bytes"] = [c["bytes"] for c in S["out"]]
    if S["holding_at_end"] and ops.job is not None:
        rt.stop_job(ops.job)
        rt.wait_job(ops.job, 120)
    dist.barrier(group=gloo)
    rt.close()
    return S


# ------------------------------------------------------------------------------------------
def _oracle_setup(args):
    from oracle import graph as OG
    from sf_inputs import data as D
    g, gi = build_workload(args.batch, args.spatial_div)
    parts = OG.partition(g, "max_ops" if args.max_ops else "phase", args.max_ops,
                         update_chunks=args.update_chunks)
    st, ds = D.init_state(g), D.datasets(g)
    return g, gi, parts, st, ds


def oracle_timeline(args, threads=None):
    """CPU oracle (oracle/, fp64 numpy) timed on this host: ONE full training iteration of
    the bench's job (every subgraph of the same partition, timed one by one), three batch-1
    forwards of the inference MLP, and the host pack / unpack of the cut-0 live set (the
    oracle's migration).  threads: BLAS threads (threadpoolctl; None = all cores)."""
    import threadpoolctl
    from oracle import graph as OG, ops as O, runner as R, staging as ST
    from sf_inputs import data as D
    g, gi, parts, st, ds = _oracle_setup(args)
    shapes = {i: (t.rows, t.cols) for i, t in enumerate(g.tensors)}
    T = {**{i: a.copy() for i, a in st.items()}, **ds}
    with threadpoolctl.threadpool_limits(threads):
        t_start = time.perf_counter()
        sub_s = []
        for (a, b) in parts:
            t0 = time.perf_counter()
            for j in range(a, b):
                O.apply_op(g.ops[j], T, shapes)
            sub_s.append(time.perf_counter() - t0)
        sti = D.init_state(gi, seed=D.SEED_INFER)
        x = D.infer_inputs(gi, 1)[0]
        tinf = []
        for _ in range(3):
            t0 = time.perf_counter()
            R.run_inference(gi, sti, x)
            tinf.append(time.perf_counter() - t0)
        L = OG.live_set(g, parts, 0)
        t0 = time.perf_counter()
        buf = ST.pack(g, L, T, 0, 0)
        t_pack = time.perf_counter() - t0
        t0 = time.perf_counter()
        ST.unpack(g, buf, {})
        t_unpack = time.perf_counter() - t0
        elapsed = time.perf_counter() - t_start
    live = OG.live_bytes(g, L)
    return {"sub_s": sub_s, "t_inf_s": float(np.median(tinf)), "t_pack_s": t_pack,
            "t_unpack_s": t_unpack, "live_bytes": live, "iter_s": float(sum(sub_s)),
            "elapsed_s": elapsed, "threads": threads or cores()}


def oracle_latencies(tl, n, seed=99):
    """Open-loop arrivals on the oracle's measured timeline: a request arriving at a uniform
    point of the iteration waits for the rest of the subgraph running then (the cut rule),
    then runs the inference forward; preempt-to-resume = pack + inference + unpack."""
    rng = np.random.default_rng(seed)
    ends = np.cumsum(tl["sub_s"])
    arr = rng.uniform(0.0, ends[-1], n)
    k = np.searchsorted(ends, arr, side="right")
    lat = (ends[np.minimum(k, len(ends) - 1)] - arr + tl["t_inf_s"]) * 1e3
    p2r = (tl["t_pack_s"] + tl["t_inf_s"] + tl["t_unpack_s"]) * 1e3
    return lat.tolist(), p2r


def cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count()


def reference_main(args):
    """--impl reference: the CPU oracle as it stands, on this host's cores, on the same
    workload, metric and unit.  Each step is one live, timed, bounded sample of the workload:
    a seeded training subgraph of the bench's partition is executed (the subgraph a request
    arriving at a uniform point u of it waits for: (1 - u) of its time) followed by the
    inference forward; per-step latency = (1 - u) t_subgraph + t_inference."""
    if args.rank != 0:
        return
    from oracle import ops as O, runner as R
    from sf_inputs import data as D
    g, gi, parts, st, ds = _oracle_setup(args)
    shapes = {i: (t.rows, t.cols) for i, t in enumerate(g.tensors)}
    T = {**{i: a.copy() for i, a in st.items()}, **ds}
    sti = D.init_state(gi, seed=D.SEED_INFER)
    x = D.infer_inputs(gi, 1)[0]
    rng = np.random.default_rng(99)
    lat, t_all = [], time.perf_counter()
    for op in g.ops:  # one untimed iteration: every subgraph's inputs then exist
        O.apply_op(op, T, shapes)
    for s in range(args.warmup + args.steps):
        k = int(rng.integers(0, len(parts)))
        a, b = parts[k]
        t0 = time.perf_counter()
        for j in range(a, b):
            O.apply_op(g.ops[j], T, shapes)
        t_sub = time.perf_counter() - t0
        t0 = time.perf_counter()
        R.run_inference(gi, sti, x)
        t_inf = time.perf_counter() - t0
        if s >= args.warmup:
            lat.append(((1.0 - rng.uniform()) * t_sub + t_inf) * 1e3)
    p99 = pct(lat, 99)
    line = {"impl": "reference", "metric": METRIC, "value": p99, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": float(np.mean(lat)),
            "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (seeded, sf_inputs)",
            "config": {"workload": WORKLOAD + " [CPU oracle]", "batch": args.batch},
            "p50_ms": pct(lat, 50), "n_requests": len(lat),
            "cpu_baseline": {"value": p99, "unit": UNIT, "cores": cores(), "kind": "oracle",
                             "sample": f"{args.steps} timed steps, each one seeded training subgraph "
                                       f"of the {len(parts)}-subgraph partition (batch {args.batch}) "
                                       "executed live + one batch-1 inference forward; latency = "
                                       "(1-u) t_subgraph + t_inference, u ~ U(0,1) seeded",
                             "elapsed_s": time.perf_counter() - t_all},
            "e2e": {"value": p99, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_pair_poisson_arm(args, local_dev: int, n_req: int, warmup: int, host_io: bool, gloo,
                         measure=True):
    """C4 at N > 1 as specified: per pair (2i, 2i+1) one training job and one
    OPEN-LOOP Poisson request stream (rate args.rate, arrival seed 7 + pair) that chases the
    job: every request goes to the GPU the job is on (or heading to) and preempts it there, so
    the job ping-pongs between the two GPUs through the peer-store kernel over NVLink (CUDA IPC
    mapping).  Pairs are independent; coordination inside a pair goes through a shared mapping
    (pairs.ShmLink)."""
    import torch
    import torch.distributed as dist
    from paper_conf_middleware_wur0hdh21_b200.pairs import PoissonOps, ShmLink, finish_pair, run_pair_poisson, shm_path
    from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime, kernel_launches, now_ns
    from sf_inputs import data as D

    g, gi = build_workload(args.batch, args.spatial_div)
    # drain gate: validated at N = 1; two processes sharing one GPU (SF_BENCH_SAME_GPU) deadlock on
    # it (a held stream wait in one context), so pairs run without it unless --pair-gate 1
    rt = Runtime([local_dev, -1], exclusive=True, auto_preempt=True, defer_migration=bool(args.defer),
                 dispatch_spin_us=args.dispatch_spin_us, inflight_budget_us=args.inflight_budget_us,
                 max_inflight=args.max_inflight, early_launch=bool(args.early),
                 drain_gate=bool(args.gate and args.pair_gate))
    gh = rt.register(g)
    gh.partition("max_ops" if args.max_ops else "phase", args.max_ops, update_chunks=args.update_chunks)
    gh.bind(0, staging=False, host_staging=False)
    arrays, arrays_i = workload_arrays(g, gi, (args.batch, args.spatial_div))
    even = args.rank % 2 == 0
    gh.load(0, arrays if even else {i: a for i, a in arrays.items() if g.tensors[i].kind == 3})
    ghi = rt.register(gi, priority=1)
    ghi.partition()
    ghi.bind(0, staging=False)
    ghi.load(0, arrays_i)
    objs = [None] * args.world
    dist.all_gather_object(objs, rt.export_arena(gh, 0), group=gloo)
    rt.import_arena(gh, 1, objs[args.rank ^ 1])
    xs = D.infer_inputs(gi, 64)
    dev = torch.device("cuda", local_dev)
    if host_io:
        x_t, out_t = torch.from_numpy(xs).pin_memory(), torch.zeros(64, 1, 1000).pin_memory()
    else:
        x_t, out_t = torch.from_numpy(xs).to(dev), torch.zeros(64, 1, 1000, device=dev)
    path = shm_path(args.rank // 2) + ("_e2e" if host_io else "")
    if even:
        shm = ShmLink(path, create=True)
    dist.barrier(group=gloo)
    if not even:
        shm = ShmLink(path, create=False)
    ops = PoissonOps(rt, gh, ghi, 0, 1, [x.data_ptr() for x in x_t], [o.data_ptr() for o in out_t])
    solo = None
    if even:
        shm.set(ShmLink.HOLDER, args.rank)
        ops.start()
        time.sleep(0.3)
        i0, t0s = rt.job_info(ops.job)["iter"], time.perf_counter()
        time.sleep(args.solo_s)
        solo = (rt.job_info(ops.job)["iter"] - i0) / (time.perf_counter() - t0s)
    dist.barrier(group=gloo)
    rng = np.random.default_rng(7 + args.rank // 2)
    gaps = (rng.exponential(1.0 / args.rate, n_req + warmup) * 1e9).astype(np.int64)
    t_start = [now_ns() + 20_000_000]
    dist.broadcast_object_list(t_start, src=0, group=gloo)  # one clock (CLOCK_MONOTONIC) per host
    arr = (t_start[0] + np.cumsum(gaps)).tolist()
    it_start = None
    if even:  # the job's iteration at the first arrival
        while now_ns() < arr[0]:
            pass
        it_start = rt.job_info(ops.job)["iter"]
    torch.cuda.synchronize(dev)
    sampler = ClockSampler(local_dev).__enter__() if measure else None
    ev0 = torch.cuda.Event(enable_timing=True)
    ev0.record()
    launches0 = kernel_launches()
    S = run_pair_poisson(shm, ops, args.rank, args.rank ^ 1, arr, now_ns, warmup=warmup)
    # the job's progress is counted from the stream's first arrival (it_start) to its end
    t_stream = (now_ns() - arr[0]) * 1e-9
    ev1 = torch.cuda.Event(enable_timing=True)
    ev1.record()
    torch.cuda.synchronize(dev)
    if sampler:
        sampler.__exit__()
    finish_pair(shm, ops, args.rank, S["seen"], group=gloo)
    fin = rt.job_info(ops.job)["iter"] if ops.job is not None else None
    S["region_ms"] = ev0.elapsed_time(ev1)
    S["launches"] = kernel_launches() - launches0
    S["clocks"] = sampler.summary() if sampler else None
    S["solo_it_per_s"] = solo
    S["it_start"], S["it_final"], S["t_stream_s"] = it_start, fin, t_stream
    S["xfer_us"] = [c["xfer_us"] for c in S["out"]]
    S["bytes"] = [c["bytes"] for c in S["out"]]
    dist.barrier(group=gloo)
    shm.close(unlink=even)
    rt.close()
    return S


def pair_main(args, local):
    """N>1 bench: independent GPU pairs, peer tier over NVLink.  Default:
    open-loop Poisson streams that chase each pair's job (C4 as specified); --arrivals chase:
    the closed-loop lockstep ping-pong (one request per handoff)."""
    import torch.distributed as dist
    gloo = dist.new_group(backend="gloo")
    rps = block_size(args)
    if args.arrivals == "poisson":
        main_s = run_pair_poisson_arm(args, local, args.steps * rps, args.warmup * rps, False, gloo)
        e2e_s = run_pair_poisson_arm(args, local, max(200, args.steps * rps // 2), 20, True, gloo, measure=False)
    else:
        main_s = run_pair_arm(args, local, args.steps, args.warmup, host_io=False, gloo=gloo)
        e2e_s = run_pair_arm(args, local, max(20, args.steps // 2), 4, host_io=True, gloo=gloo)
    allv = [None] * args.world
    dist.all_gather_object(allv, {"main": main_s, "e2e": e2e_s}, group=gloo)
    dist.barrier(group=gloo)
    if args.rank != 0:
        dist.destroy_process_group()
        return
    lat = sum((a["main"]["lat"] for a in allv), [])
    pre = sum((a["main"]["pre"] for a in allv), [])
    p2r = sum((a["main"]["p2r"] for a in allv), [])
    xfer = np.asarray(sum((a["main"]["xfer_us"] for a in allv), []), np.float64)
    byts = np.asarray(sum((a["main"]["bytes"] for a in allv), []), np.float64)
    # every adopted job migrates out once: its counter is that migration's live bytes
    live = float(np.median(byts)) if len(byts) else float("nan")
    ok = xfer > 0
    link_gbs = float(live / (np.median(xfer[ok]) * 1e-6) / 1e9) if ok.any() else None
    E = sum((a["e2e"]["lat"] for a in allv), [])
    region_ms = max(a["main"]["region_ms"] for a in allv)
    same_gpu = os.environ.get("SF_BENCH_SAME_GPU") == "1"
    peaks = load_peaks()
    nvl_meas = peaks.get("nvlink_peer_gbs") or 770.0  # B200_PROFILING.md measured peer copy
    nvl_nominal = 900.0
    train = None
    if args.arrivals == "poisson":
        pairs = []
        for r in range(0, args.world, 2):
            a, b = allv[r]["main"], allv[r + 1]["main"]
            fin = a["it_final"] if a["it_final"] is not None else b["it_final"]
            t = max(a["t_stream_s"], b["t_stream_s"])
            if fin is not None and a["it_start"] is not None and t > 0 and a["solo_it_per_s"]:
                co = (fin - a["it_start"]) / t
                pairs.append({"solo_it_per_s": a["solo_it_per_s"], "collocated_it_per_s": co,
                              "loss_frac": 1.0 - co / a["solo_it_per_s"]})
        if pairs:
            train = {"per_pair": pairs, "loss_frac_mean": float(np.mean([p["loss_frac"] for p in pairs])),
                     "desc": "job iterations/s while its pair's request stream chases it vs the same "
                             "job alone just before"}
    line = {
        "metric": METRIC, "value": pct(lat, 99), "unit": UNIT, "n_gpus": args.world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": region_ms / args.steps,
        "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic (seeded: glorot weights, U[0,1) features, uniform labels)",
        "config": {"workload": f"C4@{args.world}GPU: {args.world // 2} independent GPU pairs, each one "
                               "ResNet-50-shaped training job chased by an open-loop Poisson stream of "
                               "batch-1 requests (peer-tier migration, CUDA IPC + NVLink peer store)"
                   if args.arrivals == "poisson" else
                   f"C4@{args.world}GPU: {args.world // 2} pairs, closed-loop ping-pong",
                   "step": f"one block of {rps} Poisson arrivals per pair" if args.arrivals == "poisson"
                   else "one handoff", "rate_per_s_per_pair": args.rate,
                   "batch": args.batch, "update_chunks": args.update_chunks,
                   "parallelism": f"{args.world // 2} pairs", "tier": "peer (NVLink)",
                   "drain_gate": bool(args.gate and args.pair_gate), "early_launch": bool(args.early),
                   "same_gpu_functional_check": same_gpu},
        "n_requests": len(lat),
        "p50_ms": pct(lat, 50), "p95_ms": pct(lat, 95), "p99_ms": pct(lat, 99),
        "n_preempting": len(pre),
        "preempt_latency_p50_ms": pct(pre, 50), "preempt_latency_p99_ms": pct(pre, 99),
        "n_migrations": len(p2r),
        "preempt_to_resume_p50_ms": pct(p2r, 50), "preempt_to_resume_p99_ms": pct(p2r, 99),
        "training_throughput": train,
        "migration": {"live_bytes_median": live, "peer_store_us_median": float(np.median(xfer[ok])) if ok.any() else None,
                      "peer_gbs": link_gbs},
        "roofline": {"kernel": "mtcopy_kernel (peer store: local arena -> partner arena over NVLink)",
                     "bound": "nvlink", "achieved": link_gbs, "peak": nvl_meas, "unit": "GB/s",
                     "frac": (link_gbs / nvl_meas) if link_gbs and not same_gpu else None,
                     "frac_of_nominal_900": (link_gbs / nvl_nominal) if link_gbs and not same_gpu else None,
                     "traffic": None,
                     "peak_source": "measured peer copy per direction (B200_PROFILING.md; 900 nominal)",
                     "note": "same-GPU functional run: the 'peer' is local HBM, no NVLink frac"
                     if same_gpu else None,
                     "algorithmic_bytes": "live bytes per migration (one direction)"},
        "e2e": {"value": pct(E, 99), "unit": UNIT, "n": len(E), "h2d_bytes_per_step": 2048 * 4 * rps,
                "d2h_bytes_per_step": 1000 * 4 * rps, "p50_ms": pct(E, 50)},
        "gpu_launches": int(sum(a["main"]["launches"] for a in allv)),
        "clocks": allv[0]["main"]["clocks"],
    }
    print(json.dumps(line), flush=True)
    dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20,
                    help="timed steps; a step is one block of --requests-per-step Poisson arrivals")
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--requests-per-step", type=int, default=50)
    ap.add_argument("--min-requests", type=int, default=1000,
                    help="timed requests at least (the block per step grows); 0 for short profiling runs")
    ap.add_argument("--baseline-requests", type=int, default=500,
                    help="requests per same-run baseline arm")
    ap.add_argument("--chase-cycles", type=int, default=300,
                    help="closed-loop preemption cycles of the chase arm")
    ap.add_argument("--solo-s", type=float, default=1.0,
                    help="solo training window before each Poisson arm (throughput reference)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--batch", type=int, default=8)
    ap.add_argument("--spatial-div", type=int, default=1)
    ap.add_argument("--no-baselines", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--max-ops", type=int, default=1,
                    help="MAX_OPS partition: at most this many ops per subgraph (0 = per layer)")
    ap.add_argument("--max-inflight", type=int, default=2,
                    help="subgraphs queued on the GPU ahead of the host (1 = strict boundaries)")
    ap.add_argument("--update-chunks", type=int, default=8,
                    help="split the SGD update subgraph into byte-balanced chunks (Q2)")
    ap.add_argument("--dispatch-spin-us", type=int, default=-1,
                    help="idle dispatcher busy-polls its queue (-1: always; one core per GPU)")
    ap.add_argument("--inflight-budget-us", type=int, default=50,
                    help="queue a subgraph behind in-flight ones only within this est. device time")
    ap.add_argument("--arrivals", default="poisson", choices=["poisson", "chase"],
                    help="poisson: open-loop stream (C4); chase: one request per step, each preempts")
    ap.add_argument("--rate", type=float, default=100.0, help="Poisson arrival rate, req/s")
    ap.add_argument("--defer", type=int, default=1,
                    help="1: migrate after the preempter drained (default); 0: concurrently")
    ap.add_argument("--duplex", type=int, default=1,
                    help="1: full-duplex host round trip when nothing waits for the device "
                         "(default); 0: D2H, then H2D")
    ap.add_argument("--l2-persist-mb", type=float, default=0.0,
                    help="persisting L2 set-aside for the inference weights, MB (0: none)")
    ap.add_argument("--gate", type=int, default=0,
                    help="1: drain gate (a preempting request runs before the job's queued "
                         "subgraph); 0 (default, measured faster: DESIGN.md Q38): it waits for "
                         "every dispatched subgraph")
    ap.add_argument("--pair-gate", type=int, default=0,
                    help="N > 1: use the drain gate in the pair processes too (default 0)")
    ap.add_argument("--early", type=int, default=1,
                    help="1: a preempting request is enqueued behind a device-side wait on the "
                         "job's in-flight subgraphs (default); 0: launched after the drain")
    args = ap.parse_args()
    # watchdog: dump every thread's stack, then exit (default on for N > 1: a rank stuck on a
    # never-completing peer handoff ends the run instead of holding every GPU of the node)
    wd = os.environ.get("SF_BENCH_WATCHDOG_S") or ("1500" if int(os.environ.get("WORLD_SIZE", "1")) > 1 else "")
    if wd:
        import faulthandler
        faulthandler.enable()  # a fatal signal also dumps every thread's Python stack
        faulthandler.dump_traceback_later(float(wd), exit=True)
    args.world = int(os.environ.get("WORLD_SIZE", "1"))
    args.rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("SF_BENCH_SAME_GPU") == "1":
        local = 0  # functional check of the N>1 path on a 1-GPU box (not a scaling number)
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        return reference_main(args)

    import torch
    import __graft_entry__
    if args.rank == 0 or args.world == 1:
        __graft_entry__.build()
    if args.world > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        if os.environ.get("SF_BENCH_SAME_GPU") == "1":
            dist.init_process_group("gloo")  # NCCL refuses two ranks on one device
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        dist.barrier()
        __graft_entry__.build()
    torch.cuda.set_device(local)

    if args.world > 1:
        return pair_main(args, local)
    # headline: open-loop Poisson stream (C4 as specified).  A timed step is a fixed block of
    # --requests-per-step arrivals, so the percentiles rest on steps x block requests
    # (>= 1,000 at the driver's --steps 20).  The closed-loop "chase" arm (every request
    # preempts, the next one waits for the resume) gives the per-cycle migration numbers.
    rps = block_size(args)
    if args.arrivals == "poisson":
        main_s = run_poisson_arm(args, local, args.steps * rps, args.warmup * rps, host_io=False)
        chase_s = run_arm(args, local, args.chase_cycles, 5, host_io=False, measure=False)
        e2e_s = run_poisson_arm(args, local, args.steps * rps, args.warmup * rps, host_io=True,
                                measure=False)
    else:
        main_s = run_arm(args, local, args.steps, args.warmup, host_io=False)
        chase_s = main_s
        e2e_s = run_arm(args, local, args.steps, args.warmup, host_io=True, measure=False)
    hi_rate = None
    nb = args.baseline_requests
    if args.arrivals == "poisson" and not args.no_baselines:
        r0 = args.rate
        args.rate = 1000.0  # lambda in {100, 1000} req/s
        hr = run_poisson_arm(args, local, max(1000, args.steps * rps), 100, host_io=False, measure=False)
        args.rate = r0
        hi_rate = {"rate_per_s": 1000.0, "n": len(hr["lat"]), "p50_ms": pct(hr["lat"], 50),
                   "p95_ms": pct(hr["lat"], 95), "p99_ms": pct(hr["lat"], 99),
                   "preempt_latency_p99_ms": pct(hr["pre"], 99), "frac_preempting": hr["frac_preempting"],
                   "reparks": hr["reparks"], "training_iterations_done": hr["iters_done"],
                   "training": hr["training"]}
    base = {}
    if not args.no_baselines:
        arm = run_poisson_arm if args.arrivals == "poisson" else run_arm
        co = arm(args, local, nb, 50, host_io=False, exclusive=False, measure=False)
        itg = arm(args, local, nb, 50, host_io=False, iteration_granularity=True, measure=False)
        alt = arm(args, local, nb, 50, host_io=False, measure=False, defer=not args.defer)
        # the other host round-trip order, per preemption cycle (closed loop, every request preempts)
        seq = run_arm(args, local, min(nb, args.chase_cycles), 5, host_io=False, measure=False,
                      duplex=not args.duplex)
        # the other preempter launch policy (same arrivals)
        lat_other = arm(args, local, nb, 50, host_io=False, measure=False, early=not args.early)
        # no migration at all: the job stops at the boundary and waits in place (what the host
        # tier costs the requests that arrive during its round trip)
        inplace = arm(args, local, nb, 50, host_io=False, measure=False, target=0)
        # the other drain-gate setting (same arrivals)
        gate_other = arm(args, local, nb, 50, host_io=False, measure=False, gate=not args.gate)

        def q(x):
            return {"n": len(x["lat"]), "p50_ms": pct(x["lat"], 50), "p99_ms": pct(x["lat"], 99)}
        base = {"arrivals": args.arrivals,
                "free_corun": q(co),
                ("concurrent" if args.defer else "deferred") + "_migration": q(alt),
                ("sequential" if args.duplex else "duplex") + "_host_round_trip": {
                    "n": len(seq["p2r"]),
                    "preempt_to_resume_p50_ms": pct(seq["p2r"], 50),
                    "preempt_to_resume_p99_ms": pct(seq["p2r"], 99),
                    "d2h_plus_h2d_us_mean": float(np.mean([x for x in seq["xfer_us"] if x > 0]))
                    if any(x > 0 for x in seq["xfer_us"]) else None},
                ("launch_after_drain" if args.early else "early_launch"): {
                    **q(lat_other), "preempt_latency_p99_ms": pct(lat_other["pre"], 99)},
                "no_migration_wait_in_place": q(inplace),
                ("no_drain_gate" if args.gate else "drain_gate"): {
                    **q(gate_other), "preempt_latency_p50_ms": pct(gate_other["pre"], 50),
                    "preempt_latency_p99_ms": pct(gate_other["pre"], 99)},
                "iteration_slicing": q(itg)}

    samples = {"main": main_s, "e2e": e2e_s, "chase": chase_s}
    allv = [samples]
    M = {k: sum((a["main"][k] for a in allv), []) for k in ("lat", "pre", "p2r")}
    Cc = {k: sum((a["chase"][k] for a in allv), []) for k in ("lat", "pre", "p2r", "pack_us", "xfer_us",
                                                            "unpack_us", "bytes")}
    E = sum((a["e2e"]["lat"] for a in allv), [])
    region_ms = max(a["main"]["region_ms"] for a in allv)
    peaks = load_peaks()
    hbm = peaks.get("hbm_gbs")
    peak_src = "measured (MEASURED_PEAKS.json)" if hbm else "fallback (B200_PROFILING.md)"
    hbm = hbm or 6650.0
    pack_us = np.asarray(Cc["pack_us"], np.float64)
    byts = np.asarray(Cc["bytes"], np.float64)
    ok = pack_us > 0
    pack_achieved = float((2 * byts[ok]).mean() / (pack_us[ok].mean() * 1e-6) / 1e9) if ok.any() else None
    xfer = np.asarray(Cc["xfer_us"], np.float64)
    unpack = np.asarray(Cc["unpack_us"], np.float64)
    migr_gbs = float((2 * byts[ok]).mean() / (xfer[ok].mean() * 1e-6) / 1e9) if ok.any() else None
    prof = {}
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "pack_traffic.json")))
    except Exception:
        pass
    probe = probe_pack(args, local, hbm)
    m0 = chase_s
    link = host_link_peaks()
    dev_us = pct(main_s.get("device_us", []), 50)
    bd = main_s.get("breakdown") or {}
    w_bytes = (2048 * 4096 + 4096 * 4096 + 4096 * 1000 + 4096 + 4096 + 1000) * 4
    tr = main_s.get("training", {})
    line = {
        "metric": METRIC, "value": pct(M["lat"], 99), "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": region_ms / args.steps,
        "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic (seeded: glorot weights, U[0,1) features, uniform labels)",
        "config": {"workload": WORKLOAD, "batch": args.batch, "spatial_div": args.spatial_div,
                   "step": f"one block of {rps} open-loop Poisson arrivals" if args.arrivals == "poisson"
                   else "one preemption cycle",
                   "tensors_live_cut0": 535, "inference_model": "MLP 2048-4096-4096-1000 (29.3M params)",
                   "tier": "host (pinned, copy engine)", "parallelism": f"replicas x{args.world}",
                   "update_chunks": args.update_chunks,
                   "partition": f"MAX_OPS={args.max_ops}" if args.max_ops else "PER_LAYER_PHASE",
                   "max_inflight": args.max_inflight,
                   "dispatch_spin_us": args.dispatch_spin_us,
                   "inflight_budget_us": args.inflight_budget_us,
                   "early_launch": bool(args.early), "host_duplex": bool(args.duplex),
                   "drain_gate": bool(args.gate), "l2_persist_mb": args.l2_persist_mb,
                   "migration_policy": "deferred until the preempter drained" if args.defer
                   else "concurrent with the preempter",
                   "l2": "state 205 MB + datasets 666 MB > 126 MB L2 (no flush needed); the pack "
                         "probe reports warm and flushed-L2 runs"},
        "n_requests": len(M["lat"]),
        "p50_ms": pct(M["lat"], 50), "p95_ms": pct(M["lat"], 95), "p99_ms": pct(M["lat"], 99),
        "n_preempting": len(M["pre"]),
        "preempt_latency_p50_ms": pct(M["pre"], 50), "preempt_latency_p99_ms": pct(M["pre"], 99),
        "n_cycles": len(M["p2r"]),
        "preempt_to_resume_p50_ms": pct(M["p2r"], 50), "preempt_to_resume_p99_ms": pct(M["p2r"], 99),
        "arrivals": {"process": args.arrivals, "rate_per_s": args.rate if args.arrivals == "poisson" else None,
                     "seed": "7 + pair" if args.arrivals == "poisson" else "1234 + device",
                     "frac_preempting": main_s.get("frac_preempting"), "reparks": main_s.get("reparks"),
                     "inference_device_us_p50": pct(main_s.get("device_us", []), 50),
                     "latency_breakdown_us": main_s.get("breakdown")},
        "training_throughput": {**tr, "desc": "iterations/s of the collocated job during the timed "
                                              "region vs the same job alone just before it"},
        "poisson_1000": hi_rate,
        "chase": {"desc": "closed loop: every request preempts the running job; next request after its resume",
                  "n": len(Cc["lat"]),
                  "p50_ms": pct(Cc["lat"], 50), "p99_ms": pct(Cc["lat"], 99),
                  "preempt_latency_p50_ms": pct(Cc["pre"], 50), "preempt_latency_p99_ms": pct(Cc["pre"], 99),
                  "preempt_to_resume_p50_ms": pct(Cc["p2r"], 50),
                  "preempt_to_resume_p99_ms": pct(Cc["p2r"], 99)},
        "migration": {"live_bytes_mean": float(byts.mean()) if len(byts) else None,
                      "pack_us_mean": float(pack_us[ok].mean()) if ok.any() else None,
                      "pack_gbs": pack_achieved,
                      "pack_probe_cut0": probe,
                      "d2h_plus_h2d_us_mean": float(xfer[ok].mean()) if ok.any() else None,
                      "host_link_gbs": migr_gbs,
                      "host_link_peak_gbs": link or None,
                      # roofline time of the round trip over the measured per-direction
                      # peaks (duplex: the slower direction; sequential: both) / measured
                      "host_link_frac": ((max(1.0 / link["d2h"], 1.0 / link["h2d"],
                                              2.0 / link["duplex_total"]) if args.duplex
                                          else 1.0 / link["d2h"] + 1.0 / link["h2d"])
                                         * byts[ok].mean() / 1e9 / (xfer[ok].mean() * 1e-6))
                      if link and migr_gbs else None,
                      "host_round_trip": "full duplex (chunk c returns H2D as soon as its D2H "
                      "landed)" if args.duplex else "sequential (D2H, then H2D)",
                      "unpack_us_mean": float(unpack[ok].mean()) if ok.any() else None},
        "training_subgraph_ms_mean": m0["sub_ms"], "n_subgraphs": m0["n_subgraphs"],
        "training_iteration_ms_median": m0["iter_ms"],
        "baselines": base,
        "roofline": {"kernel": "mtcopy_kernel (pack: arena -> staging)", "bound": "hbm",
                     "achieved": pack_achieved, "peak": hbm, "unit": "GB/s",
                     "frac": (pack_achieved / hbm) if pack_achieved else None,
                     "traffic": prof.get("bytes_per_launch"), "peak_source": peak_src,
                     "traffic_algorithmic_bytes": prof.get("algorithmic_bytes_per_launch"),
                     "traffic_source": prof.get("source"),
                     "dram_frac": prof.get("dram_frac"),
                     "algorithmic_bytes": "2 x live bytes per launch (read + write)"},
        "inference_roofline": {"kernel": ("request chain (mlp_fold_kernel: the whole MLP + softmax in one "
                                          "cooperative kernel, column-split layer 0 over W0^T, row-split "
                                          "layers after, one grid barrier; device time p50)")
                               if os.environ.get("SF_CHAIN", "0") == "1" else
                               "request chain (3 LDG-streamed cluster GEMVs over blocked weights "
                               "under PDL, fused bias/ReLU, fused softmax; direct launches behind a "
                               "drain, one captured graph launch when the device is free; device time p50)",
                               "bound": "hbm", "algorithmic_bytes": w_bytes,
                               "achieved": (w_bytes / (dev_us * 1e-6) / 1e9) if dev_us else None,
                               "peak": hbm, "unit": "GB/s",
                               "frac": (w_bytes / (dev_us * 1e-6) / 1e9 / hbm) if dev_us else None,
                               # the same p50 per request group: preempting requests run on an idle
                               # device; the others land during a host round trip and share PCIe
                               "by_group": {g: {"device_us_p50": bd[g]["device_p50"],
                                                "frac": w_bytes / (bd[g]["device_p50"] * 1e-6) / 1e9 / hbm}
                                            for g in ("preempting", "not_preempting")
                                            if bd.get(g) and bd[g].get("device_p50")}},
        "e2e": {"value": pct(E, 99), "unit": UNIT, "n": len(E), "h2d_bytes_per_step": 2048 * 4 * rps,
                "d2h_bytes_per_step": 1000 * 4 * rps, "p50_ms": pct(E, 50)},
        "gpu_launches": int(sum(a["main"]["launches"] for a in allv)),
        "clocks": main_s["clocks"],
    }
    if not args.no_cpu_baseline:
        tl = oracle_timeline(args)
        tl1 = oracle_timeline(args, threads=1)
        lat, p2r = oracle_latencies(tl, 2000)
        line["cpu_baseline"] = {
            "value": pct(lat, 99), "unit": UNIT, "cores": tl["threads"], "kind": "oracle",
            "sample": f"one full training iteration of the bench job ({len(tl['sub_s'])} subgraphs, each "
                      "timed), 3 batch-1 inference forwards and the host pack / unpack of L_0, run "
                      "live on this host; p99 over 2000 seeded uniform arrivals on that measured "
                      "timeline (wait for the running subgraph, then the forward)",
            "iteration_ms": {"all_cores": tl["iter_s"] * 1e3, "single_thread": tl1["iter_s"] * 1e3,
                             "all_cores_n": tl["threads"]},
            "inference_ms": {"all_cores": tl["t_inf_s"] * 1e3, "single_thread": tl1["t_inf_s"] * 1e3},
            "host_pack_gbs": tl["live_bytes"] / tl["t_pack_s"] / 1e9,
            "host_unpack_gbs": tl["live_bytes"] / tl["t_unpack_s"] / 1e9,
            "preempt_to_resume_ms": p2r,
            "elapsed_s": tl["elapsed_s"] + tl1["elapsed_s"]}
    print(json.dumps(line), flush=True)


def host_link_peaks():
    """The box's pinned-memory copy peak per direction and full duplex."""
    import torch
    link = {}
    try:
        hb = torch.empty(256 << 20, dtype=torch.uint8).pin_memory()
        db = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
        for name, (dst, src) in (("h2d", (db, hb)), ("d2h", (hb, db))):
            best = 0.0
            for _ in range(4):
                e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
                e0.record(); dst.copy_(src, non_blocking=True); e1.record(); e1.synchronize()
                best = max(best, hb.numel() / (e0.elapsed_time(e1) * 1e-3) / 1e9)
            link[name] = best
        hb2 = torch.empty_like(hb).pin_memory()
        db2 = torch.empty_like(db)
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        best = 0.0
        for _ in range(4):
            torch.cuda.synchronize()
            e0, e1, e2 = torch.cuda.Event(True), torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record()
            s1.wait_event(e0)
            s2.wait_event(e0)
            with torch.cuda.stream(s1):
                db.copy_(hb, non_blocking=True)
                e1.record(s1)
            with torch.cuda.stream(s2):
                hb2.copy_(db2, non_blocking=True)
                e2.record(s2)
            e1.synchronize(); e2.synchronize()
            t = max(e0.elapsed_time(e1), e0.elapsed_time(e2)) * 1e-3
            best = max(best, 2 * hb.numel() / t / 1e9)
        link["duplex_total"] = best
        del hb, db, hb2, db2
    except Exception:
        link = {}
    return link


def probe_pack(args, local, hbm):
    """Pack / unpack of the cut-0 live set (535 tensors, 204.9 MB) through the bound descriptor
    lists, kernel-only durations, with L2 warm (back to back), clean-cold (a 2 x L2 read first)
    and dirty-cold (a 2 x L2 write first: the write-back shares HBM with the walk, as after a
    training subgraph)."""
    from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
    g, _ = build_workload(args.batch, args.spatial_div)
    out = {}
    with Runtime([local]) as rt:
        gh = rt.register(g)
        gh.partition("max_ops" if args.max_ops else "phase", args.max_ops, update_chunks=args.update_chunks)
        gh.bind(0, staging=True)
        for name, mode in (("warm", 0), ("cold_clean", 1), ("cold_dirty", 2)):
            rs = [rt.probe_migration(gh, 0, 0, mode) for _ in range(5)]
            pk = float(np.median([r["pack_us"] for r in rs]))
            up = float(np.median([r["unpack_us"] for r in rs]))
            b = rs[0]["live_bytes"]
            out[name] = {"pack_us": pk, "unpack_us": up,
                         "pack_gbs": 2 * b / (pk * 1e-6) / 1e9, "unpack_gbs": 2 * b / (up * 1e-6) / 1e9,
                         "pack_frac": 2 * b / (pk * 1e-6) / 1e9 / hbm}
        out["live_bytes"] = b
    return out


if __name__ == "__main__":
    main()
