#!/usr/bin/env python
"""Training-preempts-training measurement (Fig. 7).

Two C2-shaped training jobs (ResNet-50 state forest, batch 8, seeds 3 and 13) on one B200:
  solo        each job alone: iterations/s;
  free_corun  both on one slot with exclusive_gpu = 0 (the multi-threaded-TF baseline the
              paper compares against): each job's iterations/s while both
              run;
  switchflow  the low-priority job trains; the high-priority job is submitted on the same
              slot; the low one stops at its next subgraph boundary and parks on the host
              tier (pinned memory; the paper's "CPU" target, reading Q4), the high one runs
              with the whole GPU, and the low one swaps back in once it finished.  Reported:
              the high-priority job's iterations/s (vs solo), its start latency after
              submission (the drain of the low job's in-flight subgraphs), the low job's
              preempt-to-resume (includes the whole high-priority run) and migration split.
Only one GPU is available here, so the peer-GPU variant of Fig. 7 (migration to "another
slower GPU") is covered functionally by tests/test_gpu_priority.py with two slots on one
B200, not measured.
"""
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime  # noqa: E402
from sf_inputs import data as D, graphs as G  # noqa: E402

HOST = -1
LO_SEED, HI_SEED = 3, 13


def setup(rt, g, prio, seed, host=True):
    gh = rt.register(g, priority=prio)
    gh.partition(policy="max_ops", max_ops=1, update_chunks=8)
    gh.bind(0, staging=True, host_staging=host)
    gh.load(0, {**D.init_state(g, seed=seed), **D.datasets(g)})
    return gh


def iter_times(trace, job, n_sub):
    """Per-iteration (t_first_start, t_last_end) of a job from the runtime trace (ns)."""
    ev = sorted((e for e in trace if e["kind"] == "train" and e["job"] == job), key=lambda e: e["t0"])
    its = {}
    for e in ev:
        a, b = its.get(e["iter"], (e["t0"], e["t1"]))
        its[e["iter"]] = (min(a, e["t0"]), max(b, e["t1"]))
    return [its[i] for i in sorted(its) if i in its]


def rate(spans, t_lo=None, t_hi=None):
    """Iterations per second over complete iterations inside [t_lo, t_hi]."""
    sel = [s for s in spans if (t_lo is None or s[0] >= t_lo) and (t_hi is None or s[1] <= t_hi)]
    if len(sel) < 2:
        return None, len(sel)
    return (len(sel) - 1) / ((sel[-1][0] - sel[0][0]) * 1e-9), len(sel)


def rt_kw():
    return dict(max_inflight=2, inflight_budget_us=50, dispatch_spin_us=-1)


def solo(g, seed, iters):
    with Runtime([0], **rt_kw()) as rt:
        gh = setup(rt, g, 0, seed, host=False)
        j = rt.start_training(gh, 0, iters, 0)
        rt.wait_job(j, 600)
        sp = iter_times(rt.trace(), j, gh.n_subgraphs)
    r, n = rate(sp[2:])
    return {"iters_per_s": r, "iter_ms_median": float(np.median([(b - a) * 1e-6 for a, b in sp[2:]]))}


def free_corun(g_lo, g_hi, iters):
    kw = rt_kw()
    with Runtime([0], exclusive=False, **kw) as rt:
        gl = setup(rt, g_lo, 0, LO_SEED, host=False)
        gh = setup(rt, g_hi, 1, HI_SEED, host=False)
        jl = rt.start_training(gl, 0, iters * 4, 0)
        time.sleep(0.05)
        jh = rt.start_training(gh, 0, iters, 0)
        rt.wait_job(jh, 600)
        rt.stop_job(jl)
        rt.wait_job(jl, 600)
        tr = rt.trace()
    sh = iter_times(tr, jh, 0)
    sl = iter_times(tr, jl, 0)
    t_a, t_b = sh[0][0], sh[-1][1]
    rh, _ = rate(sh[2:])
    rl, nl = rate(sl, t_a, t_b)
    return {"hi_iters_per_s": rh, "lo_iters_per_s_while_hi_runs": rl, "lo_iters_in_window": nl,
            "note": "exclusive_gpu=0: both jobs' kernels share the GPU (violates invariant 1)"}


def switchflow(g_lo, g_hi, iters):
    with Runtime([0], **rt_kw()) as rt:
        gl = setup(rt, g_lo, 0, LO_SEED)
        gh = setup(rt, g_hi, 1, HI_SEED, host=False)
        jl = rt.start_training(gl, 0, 100000, HOST)
        while rt.job_info(jl)["iter"] < 5:
            time.sleep(0.001)
        jh = rt.start_training(gh, 0, iters, 0)
        rt.wait_job(jh, 600)
        ih = rt.job_info(jh)
        # let the low-priority job swap back in and run a few iterations
        t_end = time.time() + 5
        it_back = rt.job_info(jl)["iter"]
        while rt.job_info(jl)["iter"] < it_back + 5 and time.time() < t_end:
            time.sleep(0.001)
        rt.stop_job(jl)
        rt.wait_job(jl, 600)
        il = rt.job_info(jl)
        tr = rt.trace()
    sh = iter_times(tr, jh, 0)
    rh, _ = rate(sh[2:])
    first_hi = min(e["t0"] for e in tr if e["kind"] == "train" and e["job"] == jh)
    lo_during = [e for e in tr if e["kind"] == "train" and e["job"] == jl and
                 first_hi <= e["t0"] < sh[-1][1]]
    return {
        "hi_iters_per_s": rh,
        "hi_start_latency_us": (first_hi - ih["submit_ns"]) * 1e-3,
        "lo_subgraphs_while_hi_present": len(lo_during),
        "lo_n_preemptions": il["n_preemptions"],
        "lo_preempt_to_resume_ms": (il["last_resume_ns"] - il["last_stop_ns"]) * 1e-6,
        "hi_run_ms": (sh[-1][1] - first_hi) * 1e-6,
        "lo_pack_us": il["last_pack_us"], "lo_d2h_plus_h2d_us": il["last_xfer_us"],
        "lo_unpack_us": il["last_unpack_us"], "lo_live_bytes": il["migrated_bytes"] // max(1, il["n_preemptions"]),
    }


def main():
    g_lo = G.resnet50_forest(batch=8)
    g_hi = G.resnet50_forest(batch=8)
    iters = int(os.environ.get("T2T_ITERS", "40"))
    out = {"workload": "two C2-shaped training jobs (ResNet-50 state forest, batch 8), one B200",
           "partition": "MAX_OPS=1, update_chunks=8, window 2, 50 us in-flight budget"}
    out["solo_hi"] = solo(g_hi, HI_SEED, iters)
    out["solo_lo"] = solo(g_lo, LO_SEED, iters)
    out["free_corun"] = free_corun(g_lo, g_hi, iters)
    out["switchflow_host"] = switchflow(g_lo, g_hi, iters)
    s = out["solo_hi"]["iters_per_s"]
    out["hi_vs_solo"] = {"switchflow": out["switchflow_host"]["hi_iters_per_s"] / s,
                         "free_corun": out["free_corun"]["hi_iters_per_s"] / s}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
