#!/usr/bin/env python
"""Per-config measurements beside bench.py (BASELINE.json configs C1, C3, C5) -> JSON.

C5: migration sweep (live-set size 1 MB - 8 GB x size mix) through the runtime's own
    preemption path: a graph whose cut-0 live set is the requested tensor list, preempted to
    a second slot on the same B200 (peer-store kernel arena -> arena; HBM-bound on one GPU),
    kernel-only time from the in-kernel globaltimer stamps.
C3: BERT-large-shaped state, cut after layer 12's forward, peer slot: live bytes,
    preempt-to-resume, peer-store time; one training iteration's time.
C1: MLP, host tier, one preemption at each cut k: preempt-to-resume split.
"""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime  # noqa: E402
from sf_inputs import data as D, graphs as G  # noqa: E402
from sf_inputs.ir import F32, I32, PARAM, SCALAR_STATE, STEP_INC, Graph  # noqa: E402

HOST = -1
PEAK = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6553.0


def sizes_for(total, mix):
    if mix == "single":
        return [total]
    if mix == "uniform_1MB":
        return [1 << 20] * max(1, total >> 20)
    if mix == "all_4KB":
        return [4096] * max(1, min(total // 4096, 1 << 17))  # cap 128k tensors
    # ResNet-50 Keras histogram rescaled to `total`
    r = G.resnet50_forest(batch=1)
    base = [t.nbytes for t in r.tensors if t.kind in (0, 1)]
    f = total / sum(base)
    return [max(4, int(b * f) // 4 * 4) for b in base]


def state_graph(sizes):
    g = Graph("c5")
    for i, b in enumerate(sizes):
        n = b // 4
        rows = 1
        while n // rows > (1 << 28) or n % rows:
            rows *= 2
        g.add(f"t{i}", rows, n // rows, F32, PARAM)
    st = g.add("step", 1, 1, I32, SCALAR_STATE)
    g.op(STEP_INC, [], [st])
    return g


def c5(reps=4, engine=0, totals=None, mixes=None):
    out = []
    totals = totals or [1 << 20, 4 << 20, 16 << 20, 64 << 20, 256 << 20, 1 << 30, 2 << 30, 4 << 30, 8 << 30]
    for mix in mixes or ("single", "resnet_hist", "uniform_1MB", "all_4KB"):
        for tot in totals:
            if mix == "all_4KB" and tot > (512 << 20):
                continue
            sizes = sizes_for(tot, mix)
            g = state_graph(sizes)
            with Runtime([0, 0], migration_engine=engine) as rt:
                gh = rt.register(g)
                gh.partition()
                gh.bind(0, staging=False)
                gh.bind(1, staging=False)
                sched = [(it, 0, 1 if it % 2 else 0) for it in range(1, reps + 1)]
                # ping-pong 0 -> 1 -> 0 ...: each scheduled cut moves the whole live set
                job = rt.start_training(gh, 0, reps + 2, 1, schedule=sched)
                times, byts = [], []
                last = 0
                while True:
                    ji = rt.job_info(job)
                    if ji["n_preemptions"] > last:
                        times.append(ji["last_xfer_us"])
                        last = ji["n_preemptions"]
                    if ji["state_name"] in ("done", "failed"):
                        break
                rt.wait_job(job, 600)
                ji = rt.job_info(job)
                live = gh.live_set(0)[1]
            t = float(np.median([x for x in times if x > 0])) if times else float("nan")
            out.append({"engine": ["sm", "ce"][engine], "mix": mix, "bytes": live, "tensors": len(sizes) + 1, "kernel_us": t,
                        "gbs_2x": 2 * live / (t * 1e-6) / 1e9, "frac_hbm": 2 * live / (t * 1e-6) / 1e9 / PEAK,
                        "preemptions": ji["n_preemptions"]})
            print(json.dumps(out[-1]), flush=True)
    return out


def c5ce():
    """Copy-engine-only peer migration (per-segment cudaMemcpyAsync in 2 MB groups, no SM work) vs the SM
    descriptor walk on the same live sets (same GPU: HBM -> HBM)."""
    totals = [1 << 20, 16 << 20, 256 << 20, 1 << 30]
    mixes = ("single", "resnet_hist", "all_4KB")
    return {"sm": c5(engine=0, totals=totals, mixes=mixes), "ce": c5(engine=1, totals=totals, mixes=mixes)}


def c2host():
    """C2-shaped job (ResNet-50 state, batch 8) parked on the host tier at several cuts:
    SM engine (pack kernel + one D2H of the staging; H2D + unpack kernel) vs CE engine
    (per-tensor batched D2H / H2D, no SM work)."""
    g = G.resnet50_forest(batch=8)
    st, ds = D.init_state(g), D.datasets(g)
    rows = []
    for engine in (0, 1):
        with Runtime([0], migration_engine=engine) as rt:
            gh = rt.register(g)
            gh.partition(policy="max_ops", max_ops=1, update_chunks=8)
            gh.bind(0, host_staging=True)
            gh.load(0, {**st, **ds})
            n = gh.n_subgraphs
            cuts = [0, n // 3, 2 * n // 3, n - 1]
            for c, k in enumerate(cuts):
                job = rt.start_training(gh, 0, 3, HOST, schedule=[(1, k, HOST)])
                rt.wait_job(job, 120)
                ji = rt.job_info(job)
                rows.append({"engine": ["sm", "ce"][engine], "k": k, "live_bytes": gh.live_set(k)[1],
                             "tensors": len(gh.live_set(k)[0]), "pack_us": ji["last_pack_us"],
                             "d2h_h2d_us": ji["last_xfer_us"], "unpack_us": ji["last_unpack_us"],
                             "preempt_to_resume_ms": (ji["last_resume_ns"] - ji["last_stop_ns"]) * 1e-6})
                print(json.dumps(rows[-1]), flush=True)
    return rows


def c3():
    g = G.bert_chain()
    st, ds = D.init_state(g), D.datasets(g)
    cut = G.bert_mid_cut_phase()
    res = {}
    with Runtime([0, 0]) as rt:
        gh = rt.register(g)
        gh.partition(update_chunks=8)
        for s in (0, 1):
            gh.bind(s, staging=False)
            gh.load(s, ds)
        gh.load(0, st)
        job = rt.start_training(gh, 0, 3, 1, schedule=[(2, cut, 1)])
        rt.wait_job(job, 600)
        ji = rt.job_info(job)
        tr = [e for e in rt.trace() if e["kind"] == "train"]
        it1 = [e for e in tr if e["iter"] == 1]
        res = {"live_bytes": gh.live_set(cut)[1], "peer_store_us": ji["last_xfer_us"],
               "preempt_to_resume_ms": (ji["last_resume_ns"] - ji["last_stop_ns"]) * 1e-6,
               "device_copy_gbs_2x": 2 * gh.live_set(cut)[1] / (ji["last_xfer_us"] * 1e-6) / 1e9,
               "iteration_ms": (max(e["t1"] for e in it1) - min(e["t0"] for e in it1)) * 1e-6,
               "n_subgraphs": gh.n_subgraphs,
               "iteration_gflop": 3 * 2 * 512 * (24 * (4 * 1024 * 1024 + 2 * 1024 * 4096) + 1024 * 1024 + 1024 * 30522) / 1e9}
        res["algorithmic_tflops"] = res["iteration_gflop"] / res["iteration_ms"]
    print(json.dumps({"c3": res}), flush=True)
    return res


def c1():
    g = G.mlp_train()
    st, ds = D.init_state(g), D.datasets(g)
    rows = []
    for k, dx in [(k, dx) for dx in (False, True) for k in range(5)]:
        with Runtime([0], host_duplex=dx) as rt:
            gh = rt.register(g)
            gh.partition()
            gh.bind(0, host_staging=True)
            gh.load(0, {**st, **ds})
            job = rt.start_training(gh, 0, 60, HOST, schedule=[(50, k, HOST)])
            rt.wait_job(job, 60)
            ji = rt.job_info(job)
            rows.append({"k": k, "host_duplex": dx, "live_bytes": gh.live_set(k)[1], "pack_us": ji["last_pack_us"],
                         "d2h_h2d_us": ji["last_xfer_us"], "unpack_us": ji["last_unpack_us"],
                         "preempt_to_resume_us": (ji["last_resume_ns"] - ji["last_stop_ns"]) * 1e-3})
    print(json.dumps({"c1": rows}), flush=True)
    return rows


if __name__ == "__main__":
    import __graft_entry__
    __graft_entry__.build()
    which = sys.argv[1:] or ["c1", "c3", "c5"]
    res = {}
    for w in which:
        res[w] = globals()[w]()
    os.makedirs("gpurun_out", exist_ok=True)
    json.dump(res, open("gpurun_out/configs.json", "w"), indent=1)
